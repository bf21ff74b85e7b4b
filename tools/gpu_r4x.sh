# restored K-1 group combine (16 warps), G2 2 waves, fused CE > 32 MB
mkdir -p gpurun_out
show() { python -c "
import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; }
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r4x_pytest.log 2>&1; echo pytest $?; tail -30 gpurun_out/r4x_pytest.log | grep -E "^E |Error|assert|passed|failed" | head -20
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4x_eurlex.json 2>&1; show gpurun_out/r4x_eurlex.json
timeout 900 python bench.py --config amazoncat13k --train-rows 262144 --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4x_acat.json 2>&1; show gpurun_out/r4x_acat.json
timeout 900 python bench.py --config amazon670k --steps 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4x_a670k.json 2>&1; show gpurun_out/r4x_a670k.json
timeout 900 python bench.py --config wiki10_31k --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4x_wiki.json 2>&1; show gpurun_out/r4x_wiki.json
