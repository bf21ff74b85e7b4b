# programmatic dependent launch A/B: off / all kernels / GEMMs only
mkdir -p gpurun_out
show() { python -c "
import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; }
for v in "ASGD_PDL=0" "ASGD_PDL=1" "ASGD_PDL=2" "ASGD_PDL=0"; do
  env $v timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4y_$v.json 2>&1; show gpurun_out/r4y_$v.json
done
for v in "ASGD_PDL=0" "ASGD_PDL=2"; do
  env $v timeout 900 python bench.py --config amazoncat13k --train-rows 262144 --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4y_acat_$v.json 2>&1; show gpurun_out/r4y_acat_$v.json
done
ASGD_PDL=2 timeout 900 python -m pytest tests/test_gpu_step.py -m gpu -x -q 2>&1 | tail -1
