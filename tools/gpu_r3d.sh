mkdir -p gpurun_out
timeout 600 python tools/dbg_dist.py 6 2>&1 | grep -E "fp32|Error|error" | head -20
echo "--- no graphs"
ASGD_GRAPH=0 timeout 600 python tools/dbg_dist.py 4 2>&1 | grep -E "fp32|Error|error" | head -20
