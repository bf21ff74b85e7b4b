python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1 || echo "build failed"
b() { tag=$1; shift; env "$@" timeout 600 python bench.py --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 "${EXTRA[@]}" > gpurun_out/h32_$tag.json 2>gpurun_out/h32_$tag.err; python -c "import json; d=json.load(open('gpurun_out/h32_$tag.json')); print('$tag', d['config']['workload'], d['dtype'], d['value'], d['ms_per_step'])" || tail -3 gpurun_out/h32_$tag.err; }
EXTRA=(); b base X=1; b after ASGD_K0_AFTER=1; b base2 X=1; b after2 ASGD_K0_AFTER=1
EXTRA=(--precision fp32); b f32base X=1; b f32after ASGD_K0_AFTER=1
