mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_large.py -q -k "sigmoid" > gpurun_out/r3h_pytest.log 2>&1; echo pytest $?
grep -E "passed|failed|^E  .*Error" gpurun_out/r3h_pytest.log | head
timeout 900 python bench.py --config amazon670k --loss sigmoid --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r3h_a670k_sig.json 2>&1; echo bench2 $?
python -c "
import json,sys; d=json.loads(open('gpurun_out/r3h_a670k_sig.json').read().strip().splitlines()[-1]); print(d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"
