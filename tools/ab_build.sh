# A/B of compile-time switches on the GPU box: bash tools/ab_build.sh TAG "FLAGS" [bench args...]
# rebuilds libasgd.so with ASGD_NVCC_EXTRA=FLAGS, runs one bench line, restores the default build
T=$1; FL=$2; shift 2
mkdir -p gpurun_out
ASGD_NVCC_EXTRA="$FL" python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1 || { echo "build $FL failed"; exit 1; }
timeout 900 python bench.py --no-cpu-baseline --ttp-megabatches 0 "$@" > gpurun_out/${T}.json 2> gpurun_out/${T}.err
echo "$T [$FL] $*"; python tools/bench_brief.py gpurun_out/${T}.json | head -2
python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1
