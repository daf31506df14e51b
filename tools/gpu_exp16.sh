python tools/build_variants.py small2:-DSPCG_BLOCK=128,-DSPCG_NCHUNK_SLOTS=4,-DSPCG_NPOLL=0 p0:-DSPCG_NPOLL=0 > gpurun_out/build.log 2>&1
for v in libspcg.so libspcg_small2.so libspcg_p0.so; do
export SPCG_LIB=$PWD/paper_conf_sc_maacsh25_b200/$v
timeout 300 python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30 --modes alg2 >> gpurun_out/exp16.jsonl 2>>gpurun_out/exp16.err
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2 >> gpurun_out/exp16.jsonl 2>>gpurun_out/exp16.err
done
export SPCG_LIB=$PWD/paper_conf_sc_maacsh25_b200/libspcg_small2.so
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "pcg_matches or operators" > gpurun_out/pytest_small2.log 2>&1; echo "pytest small2 rc=$?"; tail -2 gpurun_out/pytest_small2.log
