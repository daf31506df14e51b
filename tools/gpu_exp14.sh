python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 1500 python bench.py --workload C3 --steps 3 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; echo "c3 rc=$?"
timeout 900 ncu --set full --clock-control none -k regex:spcg_pcg_kernel --launch-skip 1 --launch-count 1 -o gpurun_out/prof_c3 -f python tools/exp_iter.py fem_q1 128 128 128 3 --K 2 --k 5 --modes alg2 --reps 1 > gpurun_out/ncu_full_c3.log 2>&1; echo "ncu c3 rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3.csv python bench.py --workload C3 --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_launch_c3.log 2>&1; echo "ncu launches c3 rc=$?"
