# ncu: Amazon-670K output-layer GEMMs (softmax + sigmoid) and one EURLex step, full set + source
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_gemm_tc|k_lse|k_tile_loss" -s 12 -c 5 \
  -o gpurun_out/r3f_a670k_softmax python tools/prof_step.py amazon670k bf16 softmax 3 1 65536 > gpurun_out/r3f_1.log 2>&1; echo a $?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_gemm_tc|k_tile_loss" -s 9 -c 4 \
  -o gpurun_out/r3f_a670k_sigmoid python tools/prof_step.py amazon670k bf16 sigmoid 3 1 65536 > gpurun_out/r3f_2.log 2>&1; echo b $?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_" -s 40 -c 12 \
  -o gpurun_out/r3f_eurlex python tools/prof_step.py eurlex4k bf16 softmax 4 1 > gpurun_out/r3f_3.log 2>&1; echo c $?
ls -la gpurun_out/*.ncu-rep
