python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1 || echo "build failed"
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_step_groups.py tests/test_gpu_large.py tests/test_gpu_dist.py -k "tiny or eurlex or groups or wiki10 or amazoncat" -m gpu -q -p no:cacheprovider -x > gpurun_out/h22_pytest.log 2>&1; echo "pytest $?"; tail -3 gpurun_out/h22_pytest.log
b() { tag=$1; shift; env "$@" timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/h22_$tag.json 2>gpurun_out/h22_$tag.err; python -c "import json; d=json.load(open('gpurun_out/h22_$tag.json')); print('$tag', d['value'], d['ms_per_step'])" || tail -3 gpurun_out/h22_$tag.err; }
b g4 X=1
b g4b X=1
b g8 ASGD_STEP_GROUP=8
b g1 ASGD_STEP_GROUP=1
