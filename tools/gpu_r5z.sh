# round-1 evidence refresh (final kernels, PDL on): headline bench (defaults), launch lists and full ncu captures (EURLex bf16, Amazon-670K bf16)
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/z2_bench_eurlex.json 2> gpurun_out/z2_bench_eurlex.err; echo bench $?
timeout 900 python bench.py --config amazon670k --steps 5 --no-cpu-baseline --ttp-megabatches 0 > gpurun_out/z2_bench_a670k.json 2> gpurun_out/z2_bench_a670k.err; echo bench2 $?
A="--steps 1 --warmup 3 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_" -c 1600 --csv \
  --log-file gpurun_out/z2_launches_eurlex.csv python bench.py $A > /dev/null 2>&1; echo l1 $?
timeout 900 ncu --set full --cache-control none --clock-control none --import-source on -k regex:"k_(touched|spmm|gemm|softmax|lse|dh|b1|scatter)" \
  -s 1300 -c 10 -o gpurun_out/z2_full_eurlex python bench.py $A > /dev/null 2>&1; echo f1 $?
timeout 600 ncu --set full --cache-control none --clock-control none -k regex:"k_(sqnorm|scale|finish|merge)" \
  -c 4 -o gpurun_out/z2_full_eurlex_merge python bench.py $A > /dev/null 2>&1; echo f1m $?
B="--config amazon670k --train-rows 65536 --steps 1 --warmup 1 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_" -c 1500 --csv \
  --log-file gpurun_out/z2_launches_a670k.csv python bench.py $B > /dev/null 2>&1; echo l2 $?
timeout 1500 ncu --set full --cache-control none --clock-control none --import-source on -k regex:"k_(touched|spmm|gemm|softmax|lse|dh|b1|scatter)" \
  -s 400 -c 11 -o gpurun_out/z2_full_a670k python bench.py $B > /dev/null 2>&1; echo f2 $?
timeout 600 ncu --set full --cache-control none --clock-control none -k regex:"k_(sqnorm|scale|finish|merge)" \
  -c 4 -o gpurun_out/z2_full_a670k_merge python bench.py $B > /dev/null 2>&1; echo f2m $?
ls -la gpurun_out | tail -20
