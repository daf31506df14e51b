python tools/build_variants.py small:-DSPCG_BLOCK=128,-DSPCG_NCHUNK_SLOTS=4 > gpurun_out/build.log 2>&1
export SPCG_LIB=$PWD/paper_conf_sc_maacsh25_b200/libspcg_small.so
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > gpurun_out/pytest_small.log 2>&1; echo "pytest small rc=$?"; tail -3 gpurun_out/pytest_small.log
for v in libspcg.so libspcg_small.so; do
export SPCG_LIB=$PWD/paper_conf_sc_maacsh25_b200/$v
timeout 300 python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30 --modes alg2,none >> gpurun_out/exp11.jsonl 2>>gpurun_out/exp11.err
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2 >> gpurun_out/exp11.jsonl 2>>gpurun_out/exp11.err
timeout 300 python tools/exp_iter.py fem_q1 48 48 48 3 --K 2 --k 10 --modes alg2 >> gpurun_out/exp11.jsonl 2>>gpurun_out/exp11.err
timeout 600 python tools/exp_iter.py aniso_layered 4096 4096 4 --k 20 --modes alg2 --reps 3 >> gpurun_out/exp11.jsonl 2>>gpurun_out/exp11.err
done
