O=gpurun_out/r01h; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build rc=$?"
timeout 300 python bench.py --workload C1 > $O/bench_c1.json 2> $O/bench_c1.err; echo "c1 rc=$?"
timeout 600 python bench.py > $O/bench_c2.json 2> $O/bench_c2.err; echo "c2 rc=$?"
