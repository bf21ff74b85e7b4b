timeout 600 python -m pytest tests/test_gpu_dist.py -x -q -k bf16 2>&1 | grep -E "Error|error|assert|Exception|raise|line [0-9]+" | head -30
timeout 600 python -m pytest tests/test_gpu_step.py tests/test_gpu_merge.py -x -q 2>&1 | tail -15
