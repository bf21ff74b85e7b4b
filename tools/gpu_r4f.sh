# two-pass bench (clean headline, profiled roofline pass); G1 sum chains restored; EURLex sparse ncu
mkdir -p gpurun_out
show() { python -c "
import json,sys; d=json.loads(open('$1').read().strip().splitlines()[-1]); print('$1', d['value'], d['ms_per_step'], d['roofline'], d.get('clocks'), {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; }
timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4f_eurlex.json 2>&1; show gpurun_out/r4f_eurlex.json
timeout 900 python bench.py --config amazon670k --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4f_a670k.json 2>&1; show gpurun_out/r4f_a670k.json
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"k_spmm_fwd|k_scatter|k_touched" -s 30 -c 3 \
  -o gpurun_out/r4f_eurlex_sparse python tools/prof_step.py eurlex4k bf16 softmax 10 2 > gpurun_out/r4f_1.log 2>&1; echo ncu $?
