# K-1 A/B: per-piece partials (HEAD) vs group combine with 8 or 16 warps per CTA
mkdir -p gpurun_out
show() { python -c "
import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; }
run() {
  timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4r_eurlex_$1.json 2>&1; show gpurun_out/r4r_eurlex_$1.json
  timeout 900 python bench.py --config wiki10_31k --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4r_wiki_$1.json 2>&1; show gpurun_out/r4r_wiki_$1.json
  timeout 900 python bench.py --config amazoncat13k --train-rows 262144 --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4r_acat_$1.json 2>&1; show gpurun_out/r4r_acat_$1.json
}
run g8
ASGD_NVCC_EXTRA=-DASGD_K1_GROUP=16 python -m paper_conf_ipps_marws22_b200.build --force > /dev/null
timeout 600 python -m pytest tests/test_gpu_step.py -m gpu -x -q 2>&1 | tail -1
run g16
cp gpurun_ab/kernels_sparse_head.cu paper_conf_ipps_marws22_b200/csrc/kernels_sparse.cu
python -m paper_conf_ipps_marws22_b200.build --force > /dev/null
run head
