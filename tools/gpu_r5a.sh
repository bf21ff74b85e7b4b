# PDL default on (bf16): full GPU suite, smoke, default bench line (with CPU baseline, time-to-P@1, e2e), fp32 line
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r5a_pytest.log 2>&1; echo pytest $?; tail -30 gpurun_out/r5a_pytest.log | grep -E "^E |Error|assert|passed|failed" | head -20
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/r5a_bench.json 2> gpurun_out/r5a_bench.err; echo bench $?; tail -c 3000 gpurun_out/r5a_bench.json
timeout 600 python bench.py --precision fp32 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r5a_fp32.json 2>&1; python -c "
import json; d=json.loads(open('gpurun_out/r5a_fp32.json').read().strip().splitlines()[-1]); print('fp32', d['value'], d['roofline'])"
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/r5a_ref.json 2>&1; echo ref $?; tail -c 800 gpurun_out/r5a_ref.json
