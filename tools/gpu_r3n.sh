mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r3n_pytest.log 2>&1; echo pytest $?
tail -5 gpurun_out/r3n_pytest.log | grep -E "passed|failed|Error|error|assert" | head
timeout 900 python bench.py --config amazon670k --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r3n_a670k.json 2>&1; echo bench2 $?
python -c "
import json,sys; d=json.loads(open('gpurun_out/r3n_a670k.json').read().strip().splitlines()[-1]); print(d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_gemm_tc" -s 12 -c 4 \
  -o gpurun_out/r3n_a670k python tools/prof_step.py amazon670k bf16 softmax 3 1 65536 > gpurun_out/r3n_1.log 2>&1; echo a $?
