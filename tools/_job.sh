python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1 || echo "build failed"
grep -l "upload" tests/*.py
timeout 900 python -m pytest $(grep -l "upload" tests/test_gpu*.py) -m gpu -q -p no:cacheprovider -x > gpurun_out/h29_pytest.log 2>&1; echo "pytest $?"; tail -2 gpurun_out/h29_pytest.log
timeout 900 python bench.py --ttp-megabatches 0 --no-cpu-baseline > gpurun_out/h29_bench.json 2> gpurun_out/h29_bench.err; echo "bench $?"; python -c "import json; d=json.load(open('gpurun_out/h29_bench.json')); print(d['value'], d['e2e'])" || tail -5 gpurun_out/h29_bench.err
timeout 900 python bench.py --config amazoncat13k --ttp-megabatches 0 --no-cpu-baseline > gpurun_out/h29_bench_acat.json 2> gpurun_out/h29_bench_acat.err; python -c "import json; d=json.load(open('gpurun_out/h29_bench_acat.json')); print(d['value'], d['e2e'])" || tail -5 gpurun_out/h29_bench_acat.err
