# session-3 re-entry check: full GPU suite, default bench line (with CPU baseline), Amazon-670K line, launch list
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r4a_pytest.log 2>&1; echo pytest $?
tail -5 gpurun_out/r4a_pytest.log | grep -E "passed|failed|Error|error|assert" | head
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r4a_smoke.log 2>&1; echo smoke $?; tail -2 gpurun_out/r4a_smoke.log
timeout 900 python bench.py > gpurun_out/r4a_eurlex.json 2> gpurun_out/r4a_eurlex.err; echo bench1 $?
timeout 900 python bench.py --config amazon670k --steps 5 --no-cpu-baseline --ttp-megabatches 0 > gpurun_out/r4a_a670k.json 2>gpurun_out/r4a_a670k.err; echo bench2 $?
for f in gpurun_out/r4a_eurlex.json gpurun_out/r4a_a670k.json; do python -c "
import json,sys; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f', d['value'], d['ms_per_step'], d['roofline'], d.get('e2e'), d.get('cpu_baseline'), {k:v['us_per_launch'] for k,v in d.get('kernels_warmup_profile',{}).items()})"; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r4a_launches_eurlex.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > /dev/null 2>&1; echo ncu1 $?
