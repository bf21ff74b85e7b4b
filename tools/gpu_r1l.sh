mkdir -p gpurun_out
for pdl in 1 0 1 0; do
ASGD_PDL=$pdl timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_pdl$pdl.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/b_pdl$pdl.json')); print('pdl=$pdl', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['step_share'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"
done
