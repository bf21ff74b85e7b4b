bash tools/gpu.sh h19 build
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_large.py tests/test_gpu_dist.py -k "tiny or eurlex or wiki10 or amazoncat" -m gpu -q -p no:cacheprovider -x > gpurun_out/h19_pytest.log 2>&1; echo "pytest $?"; tail -2 gpurun_out/h19_pytest.log
ab() { tag=$1; shift; env "$@" timeout 300 python tools/ab_step.py --tag $tag "${EXTRA[@]}" 2>/dev/null | tee -a gpurun_out/h19_ab.jsonl | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['tag'], d['config'], round(d['us_per_step'],2), round(d['min'],2), round(d['max'],2))"; }
EXTRA=(); ab after1cta X=1; ab after1cta_t256 ASGD_K0_THREADS=256; ab early ASGD_K0_AFTER=0
for c in amazoncat13k wiki10_31k; do EXTRA=(--config $c); ab after X=1; ab early ASGD_K0_AFTER=0; done
