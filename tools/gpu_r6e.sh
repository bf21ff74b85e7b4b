# Wiki10-31K and Delicious-200K evidence: launch lists + full ncu capture of one step's kernels
mkdir -p gpurun_out
for W in wiki10_31k delicious200k; do
C="--config $W --steps 1 --warmup 1 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_" -c 1500 --csv \
  --log-file gpurun_out/z6_launches_$W.csv python bench.py $C > /dev/null 2>&1; echo l $W $?
timeout 1200 ncu --set full --cache-control none --clock-control none --import-source on -k regex:"k_(touched|spmm|gemm|softmax|lse|dh|b1|scatter)" \
  -s 400 -c 11 -o gpurun_out/z6_full_$W python bench.py $C > /dev/null 2>&1; echo f $W $?
done
timeout 900 python bench.py --config wiki10_31k --no-cpu-baseline --ttp-megabatches 0 > gpurun_out/z6_bench_wiki10.json 2>/dev/null; echo b1 $?
timeout 900 python bench.py --config delicious200k --no-cpu-baseline --ttp-megabatches 0 > gpurun_out/z6_bench_delicious.json 2>/dev/null; echo b2 $?
ls -la gpurun_out | tail -12
