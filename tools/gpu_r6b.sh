# R12/R13 on the GPU: merge/trajectory parity tests (incl. norm=ub, scale_every=2), heterogeneity + M sweep telemetry, bench with --norm ub
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_merge.py tests/test_abi.py -q > gpurun_out/r6b_pytest.log 2>&1; echo pytest $?; tail -3 gpurun_out/r6b_pytest.log
timeout 900 python tools/hetero_sweep.py --config eurlex4k --replicas 4 --hetero 0,0.5,1,2 --mega-batch-steps 100 --megabatches 20 --out gpurun_out/r6b_hetero_eurlex.json > gpurun_out/r6b_hetero.log 2>&1; echo hetero $?; tail -6 gpurun_out/r6b_hetero.log
timeout 900 python tools/hetero_sweep.py --config eurlex4k --replicas 4 --hetero 1 --mega-batch-steps 25,50,200 --megabatches 20 --out gpurun_out/r6b_msweep_eurlex.json > gpurun_out/r6b_msweep.log 2>&1; echo msweep $?; tail -4 gpurun_out/r6b_msweep.log
timeout 900 python tools/hetero_sweep.py --config eurlex4k --replicas 4 --hetero 1 --mega-batch-steps 100 --megabatches 20 --norm ub --scale-every 2 --out gpurun_out/r6b_hetero_ub.json > gpurun_out/r6b_ub.log 2>&1; echo ub $?; tail -2 gpurun_out/r6b_ub.log
timeout 600 python bench.py --norm ub --ttp-megabatches 0 --no-cpu-baseline > gpurun_out/r6b_bench_ub.json 2> gpurun_out/r6b_bench_ub.err; echo bench $?; tail -c 300 gpurun_out/r6b_bench_ub.json
