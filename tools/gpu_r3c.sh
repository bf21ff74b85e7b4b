# 16-warp MUFU epilogues, vector bias, log1p polynomial: parity + bench
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r3c_pytest.log 2>&1; echo pytest $?
tail -15 gpurun_out/r3c_pytest.log | grep -E "passed|failed|Error|error|assert" | head
for L in softmax sigmoid; do
timeout 600 python bench.py --loss $L --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r3c_eurlex_$L.json 2>&1; echo bench $?
timeout 900 python bench.py --config amazon670k --loss $L --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r3c_a670k_$L.json 2>&1; echo bench2 $?
done
for f in gpurun_out/r3c_*_*.json; do python -c "
import json,sys; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"; done
