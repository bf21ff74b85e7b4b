# K-5 staging copies issued by every thread; A/B of W1 segment look-ahead (1 vs 8)
mkdir -p gpurun_out
show() { python -c "
import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; }
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_large.py -m gpu -x -q > gpurun_out/r4n_pytest.log 2>&1; echo pytest $?; tail -3 gpurun_out/r4n_pytest.log
for tag in a1 a8; do
  if [ $tag = a8 ]; then ASGD_NVCC_EXTRA=-DASGD_SEG_AHEAD=8 python -m paper_conf_ipps_marws22_b200.build --force > /dev/null; fi
  timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4n_eurlex_$tag.json 2>&1; show gpurun_out/r4n_eurlex_$tag.json
  timeout 900 python bench.py --config amazoncat13k --train-rows 262144 --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4n_acat_$tag.json 2>&1; show gpurun_out/r4n_acat_$tag.json
  timeout 900 python bench.py --config amazon670k --steps 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4n_a670k_$tag.json 2>&1; show gpurun_out/r4n_a670k_$tag.json
done
