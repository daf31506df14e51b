python tools/build_variants.py ck8:-DSPCG_CHUNK_KB=8,-DSPCG_RING_MAX=8192 ck8r4:-DSPCG_CHUNK_KB=8,-DSPCG_RING_MAX=4096 ck16s4:-DSPCG_CHUNK_KB=16,-DSPCG_NCHUNK_SLOTS=4,-DSPCG_RING_MAX=4096 ck8s6:-DSPCG_CHUNK_KB=8,-DSPCG_NCHUNK_SLOTS=6,-DSPCG_RING_MAX=8192 > gpurun_out/build.log 2>&1
for v in libspcg_ck8.so libspcg_ck8r4.so libspcg_ck16s4.so libspcg_ck8s6.so; do
export SPCG_LIB=$PWD/paper_conf_sc_maacsh25_b200/$v
timeout 300 python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30 --modes alg2,none >> gpurun_out/exp26.jsonl 2>>gpurun_out/exp26.err
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2,none >> gpurun_out/exp26.jsonl 2>>gpurun_out/exp26.err
timeout 300 python tools/exp_iter.py poisson2d 1024 1024 --k 30 --modes alg2 >> gpurun_out/exp26.jsonl 2>>gpurun_out/exp26.err
done
