timeout 1500 python -m pytest tests/test_gpu_large.py -x -q -k delicious 2>&1 | grep -E "^E |FAILED|passed|failed|Error" | head -20
timeout 900 python bench.py --config delicious200k --train-rows 65536 --steps 3 --warmup 2 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('delicious', d['value'], d['ms_per_step'], d['roofline'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"
