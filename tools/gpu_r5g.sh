# K-1: no trailing barrier after a CTA's last group
mkdir -p gpurun_out
show() { python -c "
import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; }
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_large.py -m gpu -x -q 2>&1 | tail -1
for i in 1 2 3; do timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r5g_eurlex_$i.json 2>&1; show gpurun_out/r5g_eurlex_$i.json; done
timeout 900 python bench.py --config wiki10_31k --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r5g_wiki.json 2>&1; show gpurun_out/r5g_wiki.json
