python tools/build_variants.py ns4:-DSPCG_NSOLVER_WARPS=4 ns2:-DSPCG_NSOLVER_WARPS=2 > gpurun_out/build.log 2>&1
for v in ns4; do
export SPCG_LIB=$PWD/paper_conf_sc_maacsh25_b200/libspcg_$v.so
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "chunked or async or degenerate or determin" > gpurun_out/pytest_$v.log 2>&1; echo "pytest $v rc=$?"; tail -2 gpurun_out/pytest_$v.log
done
for v in libspcg.so libspcg_ns2.so libspcg_ns4.so; do
export SPCG_LIB=$PWD/paper_conf_sc_maacsh25_b200/$v
timeout 300 python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30 --modes alg2,none >> gpurun_out/exp20.jsonl 2>>gpurun_out/exp20.err
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2 >> gpurun_out/exp20.jsonl 2>>gpurun_out/exp20.err
timeout 300 python tools/exp_iter.py poisson2d 1024 1024 --k 30 --modes alg2 >> gpurun_out/exp20.jsonl 2>>gpurun_out/exp20.err
done
