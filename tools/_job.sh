python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1 || echo "build failed"
timeout 900 python bench.py > gpurun_out/r2e_bench_eurlex4k_bf16.json 2> gpurun_out/r2e_bench_eurlex4k_bf16.err; echo "bench $?"
timeout 900 python bench.py --precision fp32 --ttp-megabatches 0 > gpurun_out/r2e_bench_eurlex4k_fp32.json 2> gpurun_out/r2e_bench_eurlex4k_fp32.err; echo "bench fp32 $?"
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r2e_bench_reference.json 2> gpurun_out/r2e_bench_reference.err; echo "ref $?"; cat gpurun_out/r2e_bench_reference.json | cut -c1-300
bash tools/gpu.sh r2e smoke suite
