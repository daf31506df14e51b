#!/bin/bash
# One GPU session (run under gpurun): smoke, pytest -m gpu, bench lines for every
# config, the C4 ncu launch list and one `ncu --set full` capture of the solver.
#   gpurun --timeout 3000 -- 'bash tools/gpu_round.sh TAG [parts...]'
# parts: any of smoke pytest bench ncu (default: all).  Output: gpurun_out/TAG/.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
TAG=${1:-run}; shift
PARTS=${*:-smoke pytest bench ncu}
O=gpurun_out/$TAG
mkdir -p "$O"
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > "$O/gpu.txt" 2>&1
python -c "import __graft_entry__ as g; g.build()" > "$O/build.log" 2>&1
has() { [[ " $PARTS " == *" $1 "* ]]; }
if has smoke; then
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > "$O/smoke.log" 2>&1; echo "exit $?" >> "$O/smoke.log"
fi
if has pytest; then
  timeout 1800 python -m pytest tests/ -q -m gpu -x > "$O/pytest_gpu.log" 2>&1; echo "exit $?" >> "$O/pytest_gpu.log"
fi
if has bench; then
  timeout 900 python bench.py --steps 5 --warmup 3 > "$O/bench_c4.json" 2> "$O/bench_c4.err"
  for W in C1 C2 C3; do
    timeout 600 python bench.py --workload $W --steps 5 --warmup 3 --no-cpu-baseline > "$O/bench_${W,,}.json" 2> "$O/bench_${W,,}.err"
  done
  timeout 900 python bench.py --workload C5 --steps 3 --warmup 3 > "$O/bench_c5.json" 2> "$O/bench_c5.err"
  timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > "$O/bench_ref_c4.json" 2> "$O/bench_ref_c4.err"
fi
if has ncu; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file "$O/launches_c4.csv" \
    python bench.py --steps 1 --warmup 3 --no-cpu-baseline --sweep "" > "$O/ncu_launch.log" 2>&1
  # one forced-k (20 iterations) C4 solve: skip the converged solve that exp_iter runs first
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:spcg_ -s 1 -c 1 -f -o "$O/prof_c4" \
    python tools/exp_iter.py aniso_layered 4096 4096 4 --k 20 --modes alg2 --reps 1 > "$O/ncu_full.log" 2>&1
  # the report itself is ~50 MB (over gpurun's copy-back limit): export the pages, keep the report off gpurun_out
  if [ -f "$O/prof_c4.ncu-rep" ]; then
    ncu -i "$O/prof_c4.ncu-rep" --page raw --csv > "$O/prof_c4_raw.csv" 2>/dev/null
    ncu -i "$O/prof_c4.ncu-rep" --page details --csv > "$O/prof_c4_details.csv" 2>/dev/null
    ncu -i "$O/prof_c4.ncu-rep" --page source --csv --print-source sass > "$O/prof_c4_sass.csv" 2>/dev/null
    gzip -f "$O/prof_c4_sass.csv"
    mv "$O/prof_c4.ncu-rep" /tmp/prof_c4.ncu-rep
  fi
fi
echo done > "$O/DONE"
