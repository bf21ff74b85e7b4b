python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1 || echo "build failed"
timeout 900 python bench.py > gpurun_out/r2f_bench_eurlex4k_bf16.json 2> gpurun_out/r2f_bench_eurlex4k_bf16.err; echo "bench $?"
python -c "import json; j=json.load(open('gpurun_out/r2f_bench_eurlex4k_bf16.json')); print(j['value'], j['ms_per_step'], j['e2e']['value'], j['roofline']['frac'], j['clocks'])"
bash tools/gpu.sh r2f smoke suite
