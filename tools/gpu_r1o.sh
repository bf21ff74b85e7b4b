mkdir -p gpurun_out
nproc; free -g | head -2
timeout 600 python bench.py --config amazoncat13k --train-rows 262144 --steps 5 --warmup 2 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 2 > gpurun_out/bench_ac.json 2> gpurun_out/bench_ac.err; tail -3 gpurun_out/bench_ac.err; cat gpurun_out/bench_ac.json
timeout 900 python bench.py --config amazon670k --train-rows 65536 --steps 3 --warmup 2 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 1 > gpurun_out/bench_a670.json 2> gpurun_out/bench_a670.err; tail -3 gpurun_out/bench_a670.err; cat gpurun_out/bench_a670.json
timeout 600 python bench.py --config wiki10_31k --steps 10 --warmup 2 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 2 > gpurun_out/bench_w10.json 2> gpurun_out/bench_w10.err; tail -3 gpurun_out/bench_w10.err; cat gpurun_out/bench_w10.json
