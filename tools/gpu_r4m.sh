# AmazonCat-13K sparse kernels, source-level
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_spmm_fwd|k_scatter|k_touched" -s 30 -c 3 \
  -o gpurun_out/r4m_acat_sparse python tools/prof_step.py amazoncat13k bf16 softmax 10 2 262144 > gpurun_out/r4m_1.log 2>&1; echo ncu $?; tail -2 gpurun_out/r4m_1.log
