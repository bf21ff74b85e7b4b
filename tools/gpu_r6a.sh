# final check after the k_merge_wait griddepcontrol.wait change: full GPU suite, smoke, default bench line, reference arm
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r6a_pytest.log 2>&1; echo pytest $?; tail -3 gpurun_out/r6a_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/r6a_bench.json 2> gpurun_out/r6a_bench.err; echo bench $?; python -c "
import json; d=json.loads(open('gpurun_out/r6a_bench.json').read().strip().splitlines()[-1]); print(d['value'], d['ms_per_step'], d['roofline'], d['e2e'], d['cpu_baseline']['value'], d['time_to_p1']['value'], d['clocks'], d['gpu_launches'])"
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r6a_ref.json 2>gpurun_out/r6a_ref.err; echo ref $?; tail -c 600 gpurun_out/r6a_ref.json
