python tools/build_variants.py vg2:-DSPCG_VGROUP=2 vg8:-DSPCG_VGROUP=8 pa4:-DSPCG_POLL_AHEAD=4 pa24:-DSPCG_POLL_AHEAD=24 > gpurun_out/build.log 2>&1
for v in libspcg.so libspcg_vg2.so libspcg_vg8.so libspcg_pa4.so libspcg_pa24.so; do
export SPCG_LIB=$PWD/paper_conf_sc_maacsh25_b200/$v
timeout 300 python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30 --modes alg2 >> gpurun_out/exp23.jsonl 2>>gpurun_out/exp23.err
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2,none >> gpurun_out/exp23.jsonl 2>>gpurun_out/exp23.err
done
