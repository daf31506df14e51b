# HEAD verification: build, GPU parity, smoke, default bench (C2), C4 bench, C2 ncu launch list + full capture
O=gpurun_out/r01e; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build rc=$?"
timeout 1500 python -m pytest tests -x -q -m gpu > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 600 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err; echo "c2 rc=$?"
timeout 900 python bench.py --workload C4 > $O/bench_c4.json 2> $O/bench_c4.err; echo "c4 rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_c2.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > $O/ncu_launch_c2.log 2>&1; echo "ncu launches rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:spcg_pcg_kernel --launch-skip 3 --launch-count 1 -o $O/prof_c2 -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline > $O/ncu_full_c2.log 2>&1; echo "ncu full c2 rc=$?"
