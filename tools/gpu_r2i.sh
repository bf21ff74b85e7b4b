timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | grep -E "^E |FAILED|passed|failed|Error" | head -20
B="--steps 20 --warmup 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0"
timeout 300 python bench.py $B 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('eurlex', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], d['roofline']['whole_step_frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"
for C in amazoncat13k wiki10_31k; do
timeout 600 python bench.py --config $C --train-rows 262144 --steps 5 --warmup 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$C', d['value'], d['ms_per_step'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"
done
A="--steps 1 --warmup 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0"
timeout 900 ncu --metrics gpu__time_duration.sum --cache-control none --clock-control none -k regex:"k_" -s 600 -c 300 --csv \
  --log-file gpurun_out/launches_eurlex_warm3.csv python bench.py $A > /dev/null 2>&1; echo l1 $?
