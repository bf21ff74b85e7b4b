# clustered G1 + softmax-CE (TC_EPI_CSM) for L <= 4096
mkdir -p gpurun_out
show() { python -c "
import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; }
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_large.py -m gpu -x -q > gpurun_out/r4h_pytest.log 2>&1; echo pytest $?; tail -30 gpurun_out/r4h_pytest.log | grep -E "Error|error|assert|passed|failed" | head -20
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4h_eurlex.json 2>&1; show gpurun_out/r4h_eurlex.json; tail -3 gpurun_out/r4h_eurlex.json
ASGD_CSM=0 timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4h_eurlex_nocsm.json 2>&1; show gpurun_out/r4h_eurlex_nocsm.json
