# EURLex: K-0 placement / CTA count against the 16-warp K-1
mkdir -p gpurun_out
show() { python -c "
import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; }
for v in "X=0" "ASGD_K0_CTAS=32" "ASGD_K0_CTAS=16" "ASGD_K0_LATE=1" "ASGD_K0_CTAS=128"; do
  env $v timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4u_$v.json 2>&1; show gpurun_out/r4u_$v.json
done
for v in "X=0" "ASGD_K0_CTAS=32"; do
  env $v timeout 900 python bench.py --config amazoncat13k --train-rows 262144 --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4u_acat_$v.json 2>&1; show gpurun_out/r4u_acat_$v.json
done
