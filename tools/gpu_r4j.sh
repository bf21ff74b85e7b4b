mkdir -p gpurun_out
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"k_gemm_tc" -s 30 -c 1 \
  -o gpurun_out/r4j_csm python tools/prof_step.py eurlex4k bf16 softmax 10 2 > gpurun_out/r4j_1.log 2>&1; echo ncu $?; tail -2 gpurun_out/r4j_1.log
