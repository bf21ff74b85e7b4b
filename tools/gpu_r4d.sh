# bias prefetch + poly exp2 split in G1/G1b; A/B against all-MUFU
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r4d_pytest.log 2>&1; echo pytest $?; tail -2 gpurun_out/r4d_pytest.log
show() { python -c "
import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; }
timeout 900 python bench.py --config amazon670k --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4d_a670k.json 2>&1; show gpurun_out/r4d_a670k.json
timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4d_eurlex.json 2>&1; show gpurun_out/r4d_eurlex.json
ASGD_NVCC_EXTRA=-DASGD_POLY_EXP=0 python -m paper_conf_ipps_marws22_b200.build --force > /dev/null
timeout 900 python bench.py --config amazon670k --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4d_a670k_nopoly.json 2>&1; show gpurun_out/r4d_a670k_nopoly.json
