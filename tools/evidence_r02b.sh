# Round-2 (second session) evidence of the committed state, through gpurun from the repo root:
# bench lines (EURLex bf16 / fp32, AmazonCat, Wiki10, Amazon-670K), the EURLex launch list, one
# `ncu --set full` capture of an EURLex step's kernels (summaries + dram traffic), the step A/B
# table (tools/ab_step.py) and the live kernel timeline (tools/timeline.py, probe build).
T=${1:-r2b}
mkdir -p gpurun_out
python -m paper_conf_ipps_marws22_b200.build --force > gpurun_out/${T}_build.log 2>&1 || exit 1
python -c "from paper_conf_ipps_marws22_b200 import api; print(api.version())"
timeout 900 python bench.py > gpurun_out/${T}_bench_eurlex4k_bf16.json 2> gpurun_out/${T}_bench_eurlex4k_bf16.err; echo "bench $?"
timeout 900 python bench.py --precision fp32 --ttp-megabatches 0 > gpurun_out/${T}_bench_eurlex4k_fp32.json 2> gpurun_out/${T}_bench_eurlex4k_fp32.err; echo "bench fp32 $?"
for c in amazoncat13k wiki10_31k amazon670k; do
  timeout 900 python bench.py --config $c --ttp-megabatches 0 > gpurun_out/${T}_bench_${c}_bf16.json 2> gpurun_out/${T}_bench_${c}_bf16.err; echo "bench $c $?"
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_" -c 2500 --csv \
  --log-file gpurun_out/${T}_launches_eurlex4k.csv python bench.py --steps 1 --warmup 1 \
  --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > /dev/null 2>&1; echo "launches $?"
python tools/ncu_summary.py gpurun_out/${T}_launches_eurlex4k.csv --skip 300 > gpurun_out/${T}_launches_eurlex4k.md 2>&1
R="k_(touched|spmm|gemm_tc|softmax|lse|bwd_dh|dh_reduce|b1_update|scatter)"
timeout 900 ncu --set full --cache-control none --clock-control none --import-source on -k regex:"$R" -s 90 -c 9 \
  -o gpurun_out/${T}_full_eurlex4k python tools/prof_step.py eurlex4k bf16 softmax 12 2 > gpurun_out/${T}_full.log 2>&1; echo "full $?"
f=gpurun_out/${T}_full_eurlex4k.ncu-rep
python tools/ncu_details.py $f > gpurun_out/${T}_full_eurlex4k.details.md 2>&1
python tools/ncu_tensor.py $f > gpurun_out/${T}_full_eurlex4k.tensor.md 2>&1
python tools/ncu_traffic.py eurlex4k/bf16 - $f > gpurun_out/${T}_full_eurlex4k.traffic.json 2>&1
ncu -i $f --page source --csv --print-source sass -k regex:"k_(spmm|scatter|touched)" > gpurun_out/${T}_full_eurlex4k.src.csv 2>/dev/null
rm -f $f
for tag in "fold X=1" "nofold ASGD_K0_FOLD=0" "k0after ASGD_K0_AFTER=1" "k3dz ASGD_K3DZ=1" "onepass ASGD_ONEPASS=1" "k1tma ASGD_K1_TMA=1" "nopdl ASGD_PDL=0"; do
  set -- $tag; n=$1; shift
  env "$@" timeout 300 python tools/ab_step.py --tag $n >> gpurun_out/${T}_ab_step.jsonl 2>/dev/null
done
for c in amazoncat13k wiki10_31k; do
  timeout 300 python tools/ab_step.py --tag fold --config $c >> gpurun_out/${T}_ab_step.jsonl 2>/dev/null
  ASGD_K0_FOLD=0 timeout 300 python tools/ab_step.py --tag nofold --config $c >> gpurun_out/${T}_ab_step.jsonl 2>/dev/null
done
cat gpurun_out/${T}_ab_step.jsonl | cut -c1-120
ASGD_NVCC_EXTRA=-DASGD_TIMELINE python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1
timeout 300 python tools/timeline.py --config eurlex4k --out gpurun_out/${T}_timeline_eurlex4k.json > gpurun_out/${T}_timeline_eurlex4k.txt 2>&1
ASGD_K0_FOLD=0 timeout 300 python tools/timeline.py --config eurlex4k --out gpurun_out/${T}_timeline_eurlex4k_nofold.json > gpurun_out/${T}_timeline_eurlex4k_nofold.txt 2>&1
python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1
for f in gpurun_out/${T}_bench_*.json; do python tools/bench_brief.py $f | head -1; done
