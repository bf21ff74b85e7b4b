# PDL for every kernel: full GPU suite + bench lines on all configs
mkdir -p gpurun_out
show() { python -c "
import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; }
export ASGD_PDL=1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r4z2_pytest.log 2>&1; echo pytest $?; tail -30 gpurun_out/r4z2_pytest.log | grep -E "^E |Error|assert|passed|failed" | head -20
for c in amazoncat13k wiki10_31k amazon670k delicious200k; do
  for v in 0 1; do
    ASGD_PDL=$v timeout 900 python bench.py --config $c --steps 3 --train-rows 262144 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4z2_${c}_$v.json 2>&1; show gpurun_out/r4z2_${c}_$v.json
  done
done
ASGD_PDL=1 timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 --precision fp32 > gpurun_out/r4z2_eurlex_fp32_1.json 2>&1; show gpurun_out/r4z2_eurlex_fp32_1.json
ASGD_PDL=0 timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 --precision fp32 > gpurun_out/r4z2_eurlex_fp32_0.json 2>&1; show gpurun_out/r4z2_eurlex_fp32_0.json
