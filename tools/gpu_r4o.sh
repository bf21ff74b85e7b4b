# K-5 1024-thread CTAs for bf16 64-column slices; fused softmax-CE threshold A/B at AmazonCat
mkdir -p gpurun_out
show() { python -c "
import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; }
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_large.py -m gpu -x -q > gpurun_out/r4o_pytest.log 2>&1; echo pytest $?; tail -3 gpurun_out/r4o_pytest.log
timeout 900 python bench.py --config amazoncat13k --train-rows 262144 --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4o_acat.json 2>&1; show gpurun_out/r4o_acat.json
ASGD_FUSED_CE_MB=32 timeout 900 python bench.py --config amazoncat13k --train-rows 262144 --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4o_acat_f.json 2>&1; show gpurun_out/r4o_acat_f.json
timeout 900 python bench.py --config amazon670k --steps 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4o_a670k.json 2>&1; show gpurun_out/r4o_a670k.json
timeout 900 python bench.py --config wiki10_31k --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4o_wiki.json 2>&1; show gpurun_out/r4o_wiki.json
ASGD_FUSED_CE_MB=16 timeout 900 python bench.py --config wiki10_31k --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4o_wiki_f.json 2>&1; show gpurun_out/r4o_wiki_f.json
