bash tools/gpu.sh h16 build
ASGD_K0_FOLD=1 timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_large.py -k "tiny or eurlex or wiki10" -m gpu -q -p no:cacheprovider -x > gpurun_out/h16_pytest.log 2>&1; echo "pytest $?"; tail -2 gpurun_out/h16_pytest.log
ab() { tag=$1; shift; env "$@" timeout 300 python tools/ab_step.py --tag $tag "${EXTRA[@]}" 2>/dev/null | tee -a gpurun_out/h16_ab.jsonl | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['tag'], d['config'], round(d['us_per_step'],2), round(d['min'],2), round(d['max'],2))"; }
EXTRA=(); ab acqrel X=1
for c in amazoncat13k wiki10_31k; do EXTRA=(--config $c); ab acqrel X=1; done
ASGD_NVCC_EXTRA=-DASGD_FENCE_SC python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1
EXTRA=(); ab sc X=1
for c in amazoncat13k wiki10_31k; do EXTRA=(--config $c); ab sc X=1; done
python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1
