# K-5 dA1 staging by bulk async copy
mkdir -p gpurun_out
show() { python -c "
import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; }
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_large.py -m gpu -x -q > gpurun_out/r4g_pytest.log 2>&1; echo pytest $?; tail -2 gpurun_out/r4g_pytest.log
timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4g_eurlex.json 2>&1; show gpurun_out/r4g_eurlex.json
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"k_scatter" -s 10 -c 1 \
  -o gpurun_out/r4g_eurlex_k5 python tools/prof_step.py eurlex4k bf16 softmax 10 2 > gpurun_out/r4g_1.log 2>&1; echo ncu $?
