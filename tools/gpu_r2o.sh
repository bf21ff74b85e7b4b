timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | grep -E "^E |FAILED|passed|failed|Error" | head -20
B="--steps 20 --warmup 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0"
for V in "ASGD_GRAPH=1" "ASGD_GRAPH=0"; do
env $V timeout 300 python bench.py $B 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('eurlex $V', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"
done
A="--steps 1 --warmup 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0"
timeout 900 ncu --metrics gpu__time_duration.sum --cache-control none --clock-control none -k regex:"k_" -s 600 -c 300 --csv \
  --log-file gpurun_out/launches_eurlex_warm5.csv python bench.py $A > /dev/null 2>&1; echo l1 $?
