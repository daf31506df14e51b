python tools/build_variants.py ck8:-DSPCG_CHUNK_KB=8,-DSPCG_RING_MAX=8192 r8k:-DSPCG_RING_MAX=8192 > gpurun_out/build.log 2>&1
for v in libspcg.so libspcg_ck8.so libspcg_r8k.so; do
export SPCG_LIB=$PWD/paper_conf_sc_maacsh25_b200/$v
timeout 300 python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30 --modes alg2,none >> gpurun_out/exp25.jsonl 2>>gpurun_out/exp25.err
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2,none >> gpurun_out/exp25.jsonl 2>>gpurun_out/exp25.err
done
export SPCG_LIB=$PWD/paper_conf_sc_maacsh25_b200/libspcg_ck8.so
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "chunked" > gpurun_out/pytest_ck8.log 2>&1; echo "pytest ck8 rc=$?"; tail -2 gpurun_out/pytest_ck8.log
