python tools/build_variants.py nodefer:-DSPCG_DEFER_STORE=0 > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
for v in libspcg.so libspcg_nodefer.so; do
export SPCG_LIB=$PWD/paper_conf_sc_maacsh25_b200/$v
timeout 300 python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30 --modes alg2,none >> gpurun_out/exp21.jsonl 2>>gpurun_out/exp21.err
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2 >> gpurun_out/exp21.jsonl 2>>gpurun_out/exp21.err
timeout 300 python tools/exp_iter.py poisson2d 1024 1024 --k 30 --modes alg2 >> gpurun_out/exp21.jsonl 2>>gpurun_out/exp21.err
done
