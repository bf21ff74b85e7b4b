B="--steps 20 --warmup 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0"
for V in "ASGD_K0_LATE=0 ASGD_K0_CTAS=148" "ASGD_K0_LATE=1 ASGD_K0_CTAS=148" "ASGD_K0_LATE=0 ASGD_K0_CTAS=64" "ASGD_K0_LATE=1 ASGD_K0_CTAS=64" "ASGD_K0_LATE=0 ASGD_K0_CTAS=32" "ASGD_K0_LATE=1 ASGD_K0_CTAS=32"; do
env $V timeout 300 python bench.py $B 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('eurlex $V', d['value'], d['ms_per_step'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"
done
