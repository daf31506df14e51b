python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for L in 2 3 6; do timeout 1200 python bench.py --workload C5 --steps 2 --warmup 1 --lanes $L > gpurun_out/bench_c5_l$L.json 2> gpurun_out/bench_c5_l$L.err; echo "c5 l$L rc=$?"; done
