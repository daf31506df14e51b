O=gpurun_out/r01m; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build rc=$?"
timeout 1500 python bench.py --workload C5 --steps 2 > $O/bench_c5.json 2> $O/bench_c5.err; echo "c5 rc=$?"; tail -3 $O/bench_c5.err
