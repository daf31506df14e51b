python tools/build_variants.py ck8:-DSPCG_CHUNK_KB=8,-DSPCG_RING_MAX=8192 ck8r4:-DSPCG_CHUNK_KB=8,-DSPCG_RING_MAX=4096 > gpurun_out/build.log 2>&1
for v in libspcg.so libspcg_ck8.so libspcg_ck8r4.so; do
export SPCG_LIB=$PWD/paper_conf_sc_maacsh25_b200/$v
timeout 900 python tools/exp_iter.py aniso_layered 4096 4096 4 --k 20 --modes alg2,none --reps 3 >> gpurun_out/exp27.jsonl 2>>gpurun_out/exp27.err
done
