# build_view spread over all threads (K-0, K-1); G1/G1b/G2/G3 full ncu at Amazon-670K
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_step.py -m gpu -x -q > gpurun_out/r4c_pytest.log 2>&1; echo pytest $?; tail -2 gpurun_out/r4c_pytest.log
timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r4c_eurlex.json 2>&1; echo bench1 $?
for f in gpurun_out/r4c_eurlex.json; do python -c "
import json,sys; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; done
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_gemm_tc" -s 12 -c 4 \
  -o gpurun_out/r4c_a670k python tools/prof_step.py amazon670k bf16 softmax 3 1 65536 > gpurun_out/r4c_1.log 2>&1; echo ncu $?
