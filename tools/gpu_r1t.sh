mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_gemm_tc" -s 12 -c 3 -o gpurun_out/prof_a670b python bench.py --config amazon670k --train-rows 32768 --steps 1 --warmup 1 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > /dev/null 2>&1; echo ncu $?
