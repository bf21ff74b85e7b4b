# G3 serial at Amazon-670K; EURLex sparse-kernel source-level ncu (K-1, K-5, K-0)
mkdir -p gpurun_out
timeout 900 python bench.py --config amazon670k --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4b_a670k.json 2>&1; echo bench2 $?
timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4b_eurlex.json 2>&1; echo bench1 $?
for f in gpurun_out/r4b_a670k.json gpurun_out/r4b_eurlex.json; do python -c "
import json,sys; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; done
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"k_spmm_fwd|k_scatter|k_touched" -s 30 -c 3 \
  -o gpurun_out/r4b_eurlex_sparse python tools/prof_step.py eurlex4k bf16 softmax 10 2 > gpurun_out/r4b_1.log 2>&1; echo ncu $?
