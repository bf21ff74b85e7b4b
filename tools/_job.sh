python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1 || echo "build failed"
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_large.py tests/test_gpu_step_groups.py -k "tiny or eurlex or groups or wiki10" -m gpu -q -p no:cacheprovider -x > gpurun_out/h31_pytest.log 2>&1; echo "pytest $?"; tail -2 gpurun_out/h31_pytest.log
b() { tag=$1; shift; env "$@" timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 "${EXTRA[@]}" > gpurun_out/h31_$tag.json 2>gpurun_out/h31_$tag.err; python -c "import json; d=json.load(open('gpurun_out/h31_$tag.json')); print('$tag', d['config']['workload'], d['dtype'], d['value'], d['ms_per_step'])" || tail -3 gpurun_out/h31_$tag.err; }
EXTRA=(); b bf16 X=1; b bf16b X=1
EXTRA=(--precision fp32); b fp32 X=1
EXTRA=(--config wiki10_31k); b wiki X=1
