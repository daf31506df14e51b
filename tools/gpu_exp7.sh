python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
for p in 64 96 148; do timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2 --parts $p >> gpurun_out/exp7.jsonl 2>>gpurun_out/exp7.err; done
timeout 1200 python bench.py --workload C5 --steps 2 --lanes 4 > gpurun_out/bench_c5_l4.json 2> gpurun_out/bench_c5_l4.err; echo "c5 l4 rc=$?"
timeout 1200 python bench.py --workload C5 --steps 2 --lanes 8 > gpurun_out/bench_c5_l8.json 2> gpurun_out/bench_c5_l8.err; echo "c5 l8 rc=$?"
