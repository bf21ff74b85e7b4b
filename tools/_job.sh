python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1
b() { tag=$1; shift; env "$@" timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > gpurun_out/h20_$tag.json 2>/dev/null; python -c "import json; d=json.load(open('gpurun_out/h20_$tag.json')); print('$tag', d['value'], d['ms_per_step'])"; }
b fold1 X=1
b nofold ASGD_K0_FOLD=0
b fold2 X=1
b nofold2 ASGD_K0_FOLD=0
timeout 300 python tools/ab_step.py --tag fold_k5w 2>/dev/null | cut -c1-100
ASGD_K0_FOLD=0 timeout 300 python tools/ab_step.py --tag nofold_k5w 2>/dev/null | cut -c1-100
