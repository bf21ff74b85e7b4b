python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1 || echo "build failed"
timeout 1200 python -m pytest tests/test_gpu_large.py -k "amazoncat or amazon670k or delicious" -m gpu -q -p no:cacheprovider -x > gpurun_out/h24_pytest.log 2>&1; echo "pytest $?"; tail -3 gpurun_out/h24_pytest.log
b() { tag=$1; shift; env "$@" timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 "${EXTRA[@]}" > gpurun_out/h24_$tag.json 2>gpurun_out/h24_$tag.err; python -c "import json; d=json.load(open('gpurun_out/h24_$tag.json')); print('$tag', d['config']['workload'], d['value'], d['ms_per_step'])" || tail -3 gpurun_out/h24_$tag.err; }
EXTRA=(--config amazoncat13k)
b acat_g4_eg2 X=1
b acat_g1_eg2 ASGD_STEP_GROUP=1
b acat_g4_eg1 ASGD_K3_EG=1
b acat_g1_eg1 ASGD_STEP_GROUP=1 ASGD_K3_EG=1
EXTRA=(--config amazon670k)
b a670_eg2 X=1
b a670_eg1 ASGD_K3_EG=1
EXTRA=(--config wiki10_31k)
b wiki_g4 X=1
b wiki_g1 ASGD_STEP_GROUP=1
