mkdir -p gpurun_out
timeout 900 ncu --set full --cache-control none --clock-control none --import-source on -k regex:"k_spmm_fwd|k_scatter_sgd|k_softmax_ce|k_gemm_tc|k_dh_reduce" -s 60 -c 7 -o gpurun_out/prof_warm python bench.py --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1; echo ncu $?
