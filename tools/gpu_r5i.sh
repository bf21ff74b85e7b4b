# AmazonCat-13K evidence: launch list + full ncu capture of one step
mkdir -p gpurun_out
C="--config amazoncat13k --train-rows 262144 --steps 1 --warmup 1 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_" -c 1500 --csv \
  --log-file gpurun_out/z3_launches_acat.csv python bench.py $C > /dev/null 2>&1; echo l $?
timeout 1200 ncu --set full --cache-control none --clock-control none --import-source on -k regex:"k_(touched|spmm|gemm|softmax|lse|dh|b1|scatter)" \
  -s 400 -c 11 -o gpurun_out/z3_full_acat python bench.py $C > /dev/null 2>&1; echo f $?
