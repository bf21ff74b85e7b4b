# final check of the round-1 HEAD: full GPU suite, smoke, default bench line
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r6f_pytest.log 2>&1; echo pytest $?; tail -3 gpurun_out/r6f_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/r6f_bench.json 2> gpurun_out/r6f_bench.err; echo bench $?; python -c "
import json; d=json.loads(open('gpurun_out/r6f_bench.json').read().strip().splitlines()[-1]); print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['e2e']['value'], d['cpu_baseline']['value'], {k: v for k, v in d['time_to_p1'].items() if k != 'curve_every_4'}, d['clocks'])"
