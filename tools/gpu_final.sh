# Final round bench set: parity tests, smoke, every config's bench line, reference arm, ncu (C2 default + C4)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err; echo "c2 rc=$?"
timeout 300 python bench.py --workload C1 > gpurun_out/bench_c1.json 2> gpurun_out/bench_c1.err; echo "c1 rc=$?"
timeout 1500 python bench.py --workload C3 --steps 3 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; echo "c3 rc=$?"
timeout 1500 python bench.py --workload C4 --steps 3 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err; echo "c4 rc=$?"
timeout 1200 python bench.py --workload C5 --steps 2 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err; echo "c5 rc=$?"
timeout 600 python bench.py --impl reference --steps 2 --warmup 0 > gpurun_out/bench_ref_c2.json 2> gpurun_out/bench_ref_c2.err; echo "ref rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_launch_c2.log 2>&1; echo "ncu launches rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:spcg_pcg_kernel --launch-skip 3 --launch-count 1 -o gpurun_out/prof_c2 -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full_c2.log 2>&1; echo "ncu full c2 rc=$?"
timeout 900 ncu --set full --clock-control none -k regex:spcg_pcg_kernel --launch-skip 1 --launch-count 1 -o gpurun_out/prof_c4 -f python tools/exp_iter.py aniso_layered 4096 4096 4 --k 20 --modes alg2 --reps 1 > gpurun_out/ncu_full_c4.log 2>&1; echo "ncu full c4 rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c4.csv python bench.py --workload C4 --steps 1 --warmup 1 --no-cpu-baseline --sweep "" > gpurun_out/ncu_launch_c4.log 2>&1; echo "ncu launches c4 rc=$?"
