python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1 || echo "build failed"
for c in amazoncat13k amazon670k delicious200k; do
  timeout 900 python bench.py --config $c --ttp-megabatches 0 > gpurun_out/r2d_bench_${c}_bf16.json 2> gpurun_out/r2d_bench_${c}_bf16.err; echo "bench $c $?"
  python -c "import json; j=json.load(open('gpurun_out/r2d_bench_${c}_bf16.json')); r=j['roofline']; print(j['config']['workload'], round(j['value']), j['ms_per_step'], r['kernel'], r['bound'], round(r['frac'],4), j['clocks'])"
done
ASGD_STEP_GROUP=4 timeout 300 python tools/ab_step.py --config wiki10_31k --tag fold 2>/dev/null | cut -c1-100
