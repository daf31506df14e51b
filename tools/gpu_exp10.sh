python tools/build_variants.py tree:-DSPCG_SOLVER_TREE=1 > gpurun_out/build.log 2>&1
for v in libspcg.so libspcg_tree.so; do
export SPCG_LIB=$PWD/paper_conf_sc_maacsh25_b200/$v
timeout 300 python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30 --modes alg2 >> gpurun_out/exp10.jsonl 2>>gpurun_out/exp10.err
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2 >> gpurun_out/exp10.jsonl 2>>gpurun_out/exp10.err
done
