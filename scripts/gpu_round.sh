# The one GPU-box measurement recipe (run through gpurun; every output lands in gpurun_out/).
#
#   bash scripts/gpu_round.sh <TAG> <step> [args...]
#
# steps (combine several with repeated invocations in one gpurun command):
#   tests [pytest args]     full `pytest -m gpu` suite, per-test timeout      -> <TAG>_gpu_tests.log
#   bench <wl> [args]       bench.py line for one workload (default K/W)       -> <TAG>_bench_<wl>.log
#   solo <wl> <P>           SOLO per-rank compute of rank 0 of a P-way split,
#                           with the per-stage timeline (scripts/papers_rank.py) -> <TAG>_solo.jsonl (appended)
#   profile <wl>            launch list + ncu --set full of the top kernels
#                           (scripts/profile_round.sh; summarise here with
#                           scripts/summarize_profiles.py <TAG> <wl>)
#   sanitize                compute-sanitizer memcheck / racecheck / synccheck of scripts/sanitize.py
#   ablations [args]        scripts/ablations.py (NEXT-3 workloads)          -> <TAG>_ablations.jsonl
set -u
TAG=$1; STEP=$2; shift 2
mkdir -p gpurun_out
case $STEP in
  tests)
    timeout -s KILL 3000 python -m pytest tests -m gpu -q --timeout 900 "$@" > gpurun_out/${TAG}_gpu_tests.log 2>&1
    echo "gpu tests rc=$?"; tail -30 gpurun_out/${TAG}_gpu_tests.log ;;
  bench)
    WL=${1:-reddit}; shift || true
    nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
    timeout -s KILL 1200 python bench.py --workload $WL "$@" > gpurun_out/${TAG}_bench_${WL}.log 2>&1
    echo "bench $WL rc=$?"; tail -1 gpurun_out/${TAG}_bench_${WL}.log | cut -c1-400 ;;
  solo)
    WL=$1; P=$2
    timeout -s KILL 900 python scripts/papers_rank.py --workload $WL --parts $P --rank 0 --steps 10 --warmup 3 \
      --timeline 2>&1 | grep '^{' >> gpurun_out/${TAG}_solo.jsonl
    echo "solo $WL P=$P rc=$?" ;;
  profile)
    bash scripts/profile_round.sh $TAG ${1:-reddit} ;;
  sanitize)
    for tool in memcheck racecheck synccheck initcheck; do
      timeout -s KILL 1500 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 \
        python scripts/sanitize.py > gpurun_out/${TAG}_sanitize_$tool.log 2>&1
      echo "$tool rc=$?"; grep -E "ERROR SUMMARY" gpurun_out/${TAG}_sanitize_$tool.log | tail -1
    done ;;
  ablations)
    timeout -s KILL 2400 python scripts/ablations.py "$@" > gpurun_out/${TAG}_ablations.jsonl 2> gpurun_out/${TAG}_ablations.err
    echo "ablations rc=$?" ;;
  *) echo "unknown step $STEP"; exit 2 ;;
esac
