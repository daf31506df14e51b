python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:spcg_pcg_kernel --launch-skip 1 --launch-count 1 \
  -o gpurun_out/aniso2048c -f python tools/exp_iter.py aniso_layered 2048 2048 4 --k 10 --modes alg2 --reps 1 > gpurun_out/ncu_aniso.log 2>&1
echo "ncu rc=$?"; tail -3 gpurun_out/ncu_aniso.log
