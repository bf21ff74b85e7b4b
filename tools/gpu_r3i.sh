mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --cache-control none --clock-control none -k regex:"k_touched|k_spmm|k_scatter" -s 9 -c 3 \
  -o gpurun_out/r3i_eurlex_sparse python tools/prof_step.py eurlex4k bf16 softmax 4 1 > gpurun_out/r3i_1.log 2>&1; echo a $?
timeout 900 ncu --metrics gpu__time_duration.sum --cache-control none --clock-control none -k regex:"k_" -s 200 -c 300 --csv \
  --log-file gpurun_out/r3i_launches_eurlex.csv python tools/prof_step.py eurlex4k bf16 softmax 30 10 > gpurun_out/r3i_2.log 2>&1; echo b $?
