python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
timeout 300 python tools/exp_iter.py fem_q1 48 48 48 3 --K 2 --k 10 --modes alg2 >> gpurun_out/exp24.jsonl 2>>gpurun_out/exp24.err
timeout 1500 python bench.py --workload C3 --steps 3 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; echo "c3 rc=$?"
