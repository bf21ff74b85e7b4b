B="--steps 20 --warmup 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0"
timeout 300 python bench.py $B 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('eurlex', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"
timeout 900 python bench.py --config amazon670k --train-rows 65536 --steps 3 --warmup 2 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('a670k', d['value'], d['ms_per_step'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"
timeout 600 python -m pytest tests/test_gpu_step.py -x -q 2>&1 | tail -1
