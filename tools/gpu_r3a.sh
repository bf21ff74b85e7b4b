# re-entry check: full GPU suite, smoke, default bench, Amazon-670K bench
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
ls -la MEASURED_PEAKS.json 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r3a_pytest.log 2>&1; echo pytest $?
tail -5 gpurun_out/r3a_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -2
timeout 600 python bench.py > gpurun_out/r3a_bench_eurlex.json 2> gpurun_out/r3a_bench_eurlex.err; echo bench $?
cat gpurun_out/r3a_bench_eurlex.json
timeout 900 python bench.py --config amazon670k --no-cpu-baseline --ttp-megabatches 0 > gpurun_out/r3a_bench_a670k.json 2> gpurun_out/r3a_bench_a670k.err; echo bench2 $?
cat gpurun_out/r3a_bench_a670k.json
