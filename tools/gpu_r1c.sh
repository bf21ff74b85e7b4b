mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/launches_bf16.csv python bench.py --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline --precision bf16 > /dev/null 2>&1; echo ncu1 $?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tc -s 30 -c 3 -o gpurun_out/prof_gemm_tc python bench.py --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline --precision bf16 > /dev/null 2>&1; echo ncu2 $?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_spmm_fwd|k_scatter_sgd|k_softmax_ce" -s 30 -c 3 -o gpurun_out/prof_sparse python bench.py --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline --precision bf16 > /dev/null 2>&1; echo ncu3 $?
