timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | grep -E "^E |FAILED|passed|failed|Error" | head -20
B="--steps 20 --warmup 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0"
for G in 1 0; do
ASGD_GRAPH=$G timeout 300 python bench.py $B 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('eurlex graph=$G', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], d['roofline']['whole_step_frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"
done
timeout 300 python bench.py --config amazoncat13k --train-rows 262144 --steps 5 --warmup 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('acat', d['value'], d['ms_per_step'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"
timeout 300 python bench.py --steps 5 --warmup 3 --ttp-megabatches 0 --no-cpu-baseline 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('eurlex e2e', d['value'], d['e2e'])"
