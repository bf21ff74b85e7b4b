# Fig. 1 analogue tool on one GPU (run-to-run spread), AmazonCat-13K bench line
mkdir -p gpurun_out
timeout 600 python tools/gpu_spread.py --steps 400 --repeats 5 > gpurun_out/r6d_spread.json 2> gpurun_out/r6d_spread.err; echo spread $?; cat gpurun_out/r6d_spread.json; tail -3 gpurun_out/r6d_spread.err
timeout 900 python bench.py --config amazoncat13k --no-cpu-baseline --ttp-megabatches 0 > gpurun_out/r6d_bench_acat.json 2> gpurun_out/r6d_bench_acat.err; echo bench $?; python -c "
import json; d=json.loads(open('gpurun_out/r6d_bench_acat.json').read().strip().splitlines()[-1]); print(d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], d['e2e']['value'], d['clocks'])"
