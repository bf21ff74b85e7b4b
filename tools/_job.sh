ASGD_NVCC_EXTRA=-DASGD_TIMELINE python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1
timeout 300 python tools/timeline.py --config eurlex4k --out gpurun_out/r2g_timeline_eurlex4k.json > gpurun_out/r2g_timeline_eurlex4k.txt 2>&1
ASGD_K0_AFTER=0 timeout 300 python tools/timeline.py --config eurlex4k --out gpurun_out/r2g_timeline_eurlex4k_k0early.json > gpurun_out/r2g_timeline_eurlex4k_k0early.txt 2>&1
python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1
cat gpurun_out/r2g_timeline_eurlex4k.txt | grep -v Warn
