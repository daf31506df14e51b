O=gpurun_out/r01e_resncu; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build rc=$?"
timeout 600 ncu --set full --import-source on --clock-control none -k regex:spcg_resident_kernel --launch-skip 3 --launch-count 1 -o $O/prof_c1 -f python bench.py --workload C1 --sptrsv resident --steps 1 --warmup 3 --no-cpu-baseline > $O/ncu_c1.log 2>&1; echo "ncu rc=$?"
