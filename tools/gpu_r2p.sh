timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | grep -E "^E |FAILED|passed|failed|Error" | head -20
B="--steps 20 --warmup 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0"
for V in fused nccl; do
timeout 300 python bench.py $B --merge $V 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('eurlex $V', d['value'], d['ms_per_step'], d['config']['merge'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"
done
timeout 900 python bench.py --config amazon670k --train-rows 65536 --steps 3 --warmup 2 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('a670k', d['value'], d['ms_per_step'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"
