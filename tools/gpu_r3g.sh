# chunked G1 tile order + cached row state + smem bias: parity + bench + ncu of the G1 variants
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r3g_pytest.log 2>&1; echo pytest $?
tail -15 gpurun_out/r3g_pytest.log | grep -E "passed|failed|Error|error|assert" | head
for L in softmax sigmoid; do
timeout 600 python bench.py --loss $L --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r3g_eurlex_$L.json 2>&1; echo bench $?
timeout 900 python bench.py --config amazon670k --loss $L --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r3g_a670k_$L.json 2>&1; echo bench2 $?
done
for f in gpurun_out/r3g_*_*.json; do python -c "
import json,sys; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; done
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_gemm_tc|k_lse" -s 12 -c 5 \
  -o gpurun_out/r3g_a670k_softmax python tools/prof_step.py amazon670k bf16 softmax 3 1 65536 > gpurun_out/r3g_1.log 2>&1; echo a $?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_gemm_tc|k_tile_loss" -s 9 -c 4 \
  -o gpurun_out/r3g_a670k_sigmoid python tools/prof_step.py amazon670k bf16 sigmoid 3 1 65536 > gpurun_out/r3g_2.log 2>&1; echo b $?
