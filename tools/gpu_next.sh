python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 1200 python bench.py --workload C5 --steps 2 > gpurun_out/bench_c5_dyn.json 2> gpurun_out/bench_c5_dyn.err; echo "c5 rc=$?"
timeout 1800 python tools/ratio_sweep.py > gpurun_out/ratio_sweep.log 2>&1; echo "sweep rc=$?"
