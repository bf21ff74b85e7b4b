# Round-2 ncu evidence: one `--set full` capture per workload (a local step's kernels + the
# merge kernels, warm L2: --cache-control none), for profiles/r02_ncu_full_*.md and traffic.json
mkdir -p gpurun_out
R="k_(touched|spmm|gemm_tc|softmax|lse|bwd_dh|dh_reduce|b1_update|scatter|merge|sqnorm)"
for spec in "eurlex4k bf16 400" "eurlex4k fp32 400" "amazoncat13k bf16 260" "amazon670k bf16 260"; do
  set -- $spec
  timeout 1500 ncu --set full --cache-control none --clock-control none --import-source on -k regex:"$R" \
    -s $3 -c 14 -o gpurun_out/e1_full_$1_$2 python bench.py --config $1 --precision $2 --steps 1 --warmup 1 \
    --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/e1_full_$1_$2.log 2>&1
  echo "full $1 $2 $?"
done
# summaries on the box (the reports themselves exceed gpurun's 64 MiB pull limit)
for f in gpurun_out/e1_full_*.ncu-rep; do
  b=${f%.ncu-rep}
  python tools/ncu_details.py $f > $b.details.md 2>&1
  python tools/ncu_tensor.py $f > $b.tensor.md 2>&1
  ncu -i $f --page source --csv --print-source sass -k regex:"k_(spmm|scatter|bwd_dh|softmax)" > $b.src.csv 2>/dev/null
  k=$(basename $b | sed 's/e1_full_//; s/_\(bf16\|fp32\)$//'); p=$(basename $b | sed 's/.*_//')
  python tools/ncu_traffic.py $k/$p gpurun_out/e1_traffic_$k_$p.json $f > /dev/null 2>&1
  python tools/ncu_traffic.py $k/$p - $f > $b.traffic.json 2>&1
  rm -f $f
done
