python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
for ex in level syncfree; do timeout 300 python tools/exp_iter.py fem_q1 48 48 48 3 --K 2 --k 10 --modes alg2 --sptrsv $ex --tag $ex >> gpurun_out/exp12.jsonl 2>>gpurun_out/exp12.err; done
timeout 1500 python bench.py --workload C3 --steps 3 --sptrsv syncfree --no-cpu-baseline > gpurun_out/bench_c3_sf.json 2> gpurun_out/bench_c3_sf.err; echo "c3 sf rc=$?"
timeout 1200 python bench.py --workload C5 --steps 2 > gpurun_out/bench_c5_dyn.json 2> gpurun_out/bench_c5_dyn.err; echo "c5 rc=$?"
