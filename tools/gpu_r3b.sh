# sigmoid-BCE head: parity + bench lines
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_step.py tests/test_gpu_large.py -x -q -k "sigmoid" > gpurun_out/r3b_pytest.log 2>&1; echo pytest $?
tail -15 gpurun_out/r3b_pytest.log
timeout 600 python bench.py --loss sigmoid --no-cpu-baseline --ttp-megabatches 20 --e2e-steps 0 > gpurun_out/r3b_bench_eurlex_sig.json 2> gpurun_out/r3b_bench_eurlex_sig.err; echo bench $?
python -c "
import json; d=json.load(open('gpurun_out/r3b_bench_eurlex_sig.json')); print('eurlex sig', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()}, d.get('time_to_p1',{}).get('p1_best'))"
timeout 900 python bench.py --config amazon670k --loss sigmoid --steps 5 --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/r3b_bench_a670k_sig.json 2> gpurun_out/r3b_bench_a670k_sig.err; echo bench2 $?
python -c "
import json; d=json.load(open('gpurun_out/r3b_bench_a670k_sig.json')); print('a670k sig', d['value'], d['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], {k:v['us_per_launch'] for k,v in d['kernels_warmup_profile'].items()})"
tail -3 gpurun_out/r3b_bench_a670k_sig.err
