mkdir -p gpurun_out
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"k_gemm_tc" -s 40 -c 1 \
  -o gpurun_out/r4i_csm python tools/prof_step.py eurlex4k bf16 softmax 10 2 > gpurun_out/r4i_1.log 2>&1; echo ncu $?
