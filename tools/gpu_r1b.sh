mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_step.py -x -q -k "tiny and bf16" 2>&1 | tail -25
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -25
timeout 300 python bench.py --steps 20 --warmup 3 --precision bf16 --no-cpu-baseline > gpurun_out/bench_bf16.json 2> gpurun_out/bench_bf16.err; tail -5 gpurun_out/bench_bf16.err; cat gpurun_out/bench_bf16.json
timeout 300 python bench.py --steps 20 --warmup 3 --precision fp32 --no-cpu-baseline > gpurun_out/bench_fp32b.json 2> gpurun_out/bench_fp32b.err; tail -5 gpurun_out/bench_fp32b.err; cat gpurun_out/bench_fp32b.json
