# G2 split-K: one wave (new default) vs two waves
mkdir -p gpurun_out
show() { python -c "
import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; }
for v in "X=0" "ASGD_G2_WAVES=2"; do
  env $v timeout 900 python bench.py --config amazoncat13k --train-rows 262144 --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4w_acat_$v.json 2>&1; show gpurun_out/r4w_acat_$v.json
  env $v timeout 900 python bench.py --config wiki10_31k --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4w_wiki_$v.json 2>&1; show gpurun_out/r4w_wiki_$v.json
  env $v timeout 900 python bench.py --config amazon670k --steps 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4w_a670k_$v.json 2>&1; show gpurun_out/r4w_a670k_$v.json
  env $v timeout 900 python bench.py --config delicious200k --steps 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4w_del_$v.json 2>&1; show gpurun_out/r4w_del_$v.json
done
timeout 900 python -m pytest tests/test_gpu_large.py -m gpu -x -q 2>&1 | tail -1
