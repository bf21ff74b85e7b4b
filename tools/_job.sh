python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1 || echo "build failed"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_" -c 1200 --csv \
  --log-file gpurun_out/r2h_launches_amazon670k.csv python bench.py --config amazon670k --steps 1 --warmup 1 \
  --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > /dev/null 2>&1; echo "launches $?"
python tools/ncu_summary.py gpurun_out/r2h_launches_amazon670k.csv --skip 300 > gpurun_out/r2h_launches_amazon670k.md 2>&1
timeout 900 ncu --set full --cache-control none --clock-control none -k regex:"k_bwd_dh|k_gemm_tc" -s 6 -c 3 \
  -o gpurun_out/r2h_full_a670k python tools/prof_step.py amazon670k bf16 softmax 2 1 > gpurun_out/r2h_full.log 2>&1; echo "full $?"
python tools/ncu_details.py gpurun_out/r2h_full_a670k.ncu-rep > gpurun_out/r2h_full_a670k.details.md 2>&1
python tools/ncu_tensor.py gpurun_out/r2h_full_a670k.ncu-rep > gpurun_out/r2h_full_a670k.tensor.md 2>&1
rm -f gpurun_out/r2h_full_a670k.ncu-rep
head -20 gpurun_out/r2h_launches_amazon670k.md; cat gpurun_out/r2h_full_a670k.tensor.md
