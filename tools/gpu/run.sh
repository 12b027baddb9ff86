#!/bin/bash
# One parameterised GPU-box job (run under gpurun from the repo root):
#   tools/gpu/run.sh <what> [args...]
# what:
#   tests [pytest args]       pytest -m gpu (default -x -q), log -> gpurun_out/tests.log
#   bench [bench args]        bench.py, JSON line -> gpurun_out/bench.json, stderr -> bench.log
#   launches [bench args]     ncu launch list of one bench step (cold-cache, serialised: shares only)
#   ncu <kernel-regex> [n] [bench args]   ncu --set full of the n-th launch matching the regex
#   sanitize <tool>           compute-sanitizer <tool> over tools/sanitize_run.py (RMAT-16, every kernel)
#   py <script> [args]        any python script, stdout -> gpurun_out/<script basename>.out
#   ab <pytest -k expr> <algos> <variants>   GPU tests matching the expression, then tools/kernel_ab.py
#                             over development-switch variants ("name:ENV=V;name2:..."; "" = the build as is)
#   ncuk <kernel-regex> <n> <algos>   ncu --set full of the n-th launch of a kernel in a bench run of <algos>
#   microbench                tools/microbench.cu (primitive rates) -> gpurun_out/microbench.txt
#   abso <algos> <alt.so>...  compile-time A/B: tools/kernel_ab.py with the in-tree libgts.so, then with
#                             each alternative build swapped in (the in-tree library is restored after)
set -u
cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out
mkdir -p $O
what=${1:-tests}; shift || true
case "$what" in
  tests)
    [ $# -eq 0 ] && set -- -x -q
    timeout 3000 python -m pytest -m gpu "$@" > $O/tests.log 2>&1; echo "pytest rc=$?"; tail -5 $O/tests.log ;;
  bench)
    timeout 1500 python bench.py "$@" > $O/bench.json 2> $O/bench.log; echo "bench rc=$?"; tail -c 3000 $O/bench.json ;;
  launches)
    timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv \
      python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e "$@" > /dev/null 2> $O/launches.log
    echo "ncu rc=$?"; python tools/launch_summary.py $O/launches.csv > $O/launches.txt; head -40 $O/launches.txt ;;
  ncu)
    k=$1; shift; c=${1:-1}; shift || true
    timeout 2400 ncu --set full --clock-control none --import-source on -k "regex:$k" -s $((c - 1)) -c 1 \
      -o $O/ncu_full -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e "$@" > $O/ncu.log 2>&1
    echo "ncu rc=$?"; tail -3 $O/ncu.log ;;
  sanitize)
    tool=${1:-memcheck}
    timeout ${SAN_TIMEOUT:-2400} compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_run.py > $O/sanitize_$tool.log 2>&1
    echo "sanitizer rc=$?"; tail -8 $O/sanitize_$tool.log ;;
  py)
    s=$1; shift
    timeout 3000 python "$s" "$@" > $O/$(basename "$s" .py).out 2>&1; echo "py rc=$?"; tail -40 $O/$(basename "$s" .py).out ;;
  ab)
    k=$1; algos=$2; variants=${3:-}
    timeout 1200 python -m pytest -m gpu -x -q -k "$k" tests > $O/ab_tests.log 2>&1; echo "tests rc=$?"; tail -2 $O/ab_tests.log
    timeout 1500 python tools/kernel_ab.py --scale ${AB_SCALE:-27} --algos $algos --reps ${AB_REPS:-5} --variants "$variants" \
      > $O/ab.jsonl 2> $O/ab.log; echo "ab rc=$?"; cut -c1-300 $O/ab.jsonl ;;
  ncuk)
    k=$1; c=$2; algos=$3
    timeout 1200 ncu --set full --clock-control none --import-source on -k "regex:$k" -s $((c - 1)) -c 1 \
      -o $O/ncu_${k}_$c -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-streamed \
      --algos $algos > $O/ncu_${k}_$c.log 2>&1
    echo "ncu $k $c rc=$?" ;;
  microbench)
    nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/microbench tools/microbench.cu && \
      timeout 300 /tmp/microbench > $O/microbench.txt 2>&1; echo "microbench rc=$?"; cat $O/microbench.txt ;;
  abso)
    algos=$1; shift
    L=paper_conf_sigmod_0002apsk16_b200/lib/libgts.so
    cp $L /tmp/libgts_base.so
    for so in base "$@"; do
      [ "$so" != base ] && cp "$so" $L
      timeout 1500 python tools/kernel_ab.py --scale ${AB_SCALE:-27} --algos $algos --reps ${AB_REPS:-5} \
        --tag "$(basename $so)" >> $O/abso.jsonl 2>> $O/abso.log; echo "ab $so rc=$?"
      cp /tmp/libgts_base.so $L
    done
    cut -c1-260 $O/abso.jsonl ;;
  *) echo "unknown job $what"; exit 2 ;;
esac
