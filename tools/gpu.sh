# One runner for the GPU-box jobs (run through gpurun from the repo root):
#   bash tools/gpu.sh TAG JOB [JOB ...]
# Outputs go to gpurun_out/TAG_*.  Jobs:
#   build            rebuild libasgd.so (sm_100a) on the box
#   suite            pytest -m gpu (parity log: gpurun_out/TAG_parity.jsonl)
#   smoke            __graft_entry__.smoke()
#   bench            default bench line (EURLex-4K, bf16)            -> TAG_bench.json
#   bench:CFG[:PREC] bench line of another workload / precision        -> TAG_bench_CFG_PREC.json
#   launches:CFG     ncu launch list of one bench mega-batch (--metrics gpu__time_duration.sum)
#   full:CFG:REGEX   ncu --set full capture of the kernels matching REGEX (one step)
#   sanitize         compute-sanitizer memcheck / racecheck / synccheck on tiny + EURLex steps
#   sass             per-kernel SASS census of libasgd.so (UTC*MMA, UTMALDG, LDTM ...)
#   timeline:CFG[:PREC]  live per-kernel timeline of one local step (-DASGD_TIMELINE build)
#   ab:NAME:FLAGS    bench line with libasgd rebuilt with ASGD_NVCC_EXTRA=FLAGS     -> TAG_ab_NAME.json
T=$1; shift
mkdir -p gpurun_out
export ASGD_PARITY_LOG=$PWD/gpurun_out/${T}_parity.jsonl
for J in "$@"; do
  IFS=: read -r JOB A B <<< "$J"
  case $JOB in
  build)
    python -m paper_conf_ipps_marws22_b200.build --force > gpurun_out/${T}_build.log 2>&1; echo "build $?" ;;
  suite)
    timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/${T}_pytest.log 2>&1
    echo "suite $?"; grep -E "passed|failed|Error" gpurun_out/${T}_pytest.log | tail -8 ;;
  smoke)
    timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2 ;;
  bench)
    if [[ -z $A ]]; then
      O=gpurun_out/${T}_bench.json
      timeout 900 python bench.py > $O 2> ${O%.json}.err
    else
      O=gpurun_out/${T}_bench_${A}_${B:-bf16}.json
      timeout 900 python bench.py --config $A --precision ${B:-bf16} --ttp-megabatches 0 > $O 2> ${O%.json}.err
    fi
    echo "bench $A $B $?"; python tools/bench_brief.py $O ;;
  launches)
    timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_" -c 2500 --csv \
      --log-file gpurun_out/${T}_launches_${A}.csv python bench.py --config $A --steps 1 --warmup 1 \
      --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > /dev/null 2>&1; echo "launches $A $?" ;;
  full)
    timeout 1500 ncu --set full --cache-control none --clock-control none --import-source on -k regex:"$B" \
      -s 400 -c 12 -o gpurun_out/${T}_full_${A} python bench.py --config $A --steps 1 --warmup 1 \
      --no-cpu-baseline --ttp-megabatches 0 --e2e-steps 0 > /dev/null 2>&1; echo "full $A $?" ;;
  sanitize)
    for tool in memcheck racecheck synccheck; do
      timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_steps.py \
        > gpurun_out/${T}_san_${tool}.log 2>&1; echo "sanitize $tool $?"; tail -2 gpurun_out/${T}_san_${tool}.log
    done ;;
  timeline)
    ASGD_NVCC_EXTRA=-DASGD_TIMELINE python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1
    timeout 600 python tools/timeline.py --config $A --precision ${B:-bf16} --out gpurun_out/${T}_tl_${A}_${B:-bf16}.json \
      > gpurun_out/${T}_tl_${A}_${B:-bf16}.txt 2>&1; echo "timeline $A $?"; cat gpurun_out/${T}_tl_${A}_${B:-bf16}.txt
    python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1 ;;
  ab)
    ASGD_NVCC_EXTRA="$B" python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1 || echo "build $B failed"
    O=gpurun_out/${T}_ab_${A}.json
    timeout 900 python bench.py --no-cpu-baseline --ttp-megabatches 0 > $O 2> ${O%.json}.err
    echo "ab $A [$B] $?"; python tools/bench_brief.py $O
    python -m paper_conf_ipps_marws22_b200.build --force > /dev/null 2>&1 ;;
  sass)
    python tools/sass_census.py > gpurun_out/${T}_sass.md; echo "sass $?" ;;
  *)
    echo "unknown job $JOB" ;;
  esac
done
