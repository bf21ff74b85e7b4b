python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1 || echo "build failed"
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_large.py -k "tiny or eurlex or wiki10 or amazoncat" -m gpu -q -p no:cacheprovider -x > gpurun_out/h28_pytest.log 2>&1; echo "pytest $?"; tail -2 gpurun_out/h28_pytest.log
ab() { tag=$1; shift; env "$@" timeout 300 python tools/ab_step.py --tag $tag "${EXTRA[@]}" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['tag'], d['config'], round(d['us_per_step'],2), round(d['min'],2), round(d['max'],2))"; }
for c in eurlex4k wiki10_31k amazoncat13k; do EXTRA=(--config $c); ab base X=1; ab after ASGD_K0_AFTER=1; done
bash tools/gpu.sh h28 timeline:eurlex4k | grep -E "spmm|touched|g1 |softmax|g2 |dh |scatter|ph|isolated|back"
