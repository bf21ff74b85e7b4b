# G1 stats tree reductions; source-level ncu of G1 / G1b at Amazon-670K; bench lines with the new roofline choice
mkdir -p gpurun_out
show() { python -c "
import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], d['roofline'], d.get('side_stream'), {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; }
timeout 900 python bench.py --config amazon670k --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4e_a670k.json 2>&1; show gpurun_out/r4e_a670k.json
timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4e_eurlex.json 2>&1; show gpurun_out/r4e_eurlex.json
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_gemm_tc" -s 12 -c 2 \
  -o gpurun_out/r4e_a670k python tools/prof_step.py amazon670k bf16 softmax 3 1 65536 > gpurun_out/r4e_1.log 2>&1; echo ncu $?
