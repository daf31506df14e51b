# A/B of the vector-warp grouping + executor choice on mid-size matrices (experiment, not the bench)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python -c "
from paper_conf_sc_maacsh25_b200 import _build as b
b.build(defines=['-DSPCG_VGROUP=1'], out=b.LIB.replace('libspcg.so','libspcg_vg1.so'))" >> gpurun_out/build.log 2>&1
python -c "import paper_conf_sc_maacsh25_b200 as s, json; print(json.dumps(s.calibrate(0)))" > gpurun_out/calib.json 2>&1
for lib in libspcg.so libspcg_vg1.so; do
  export SPCG_LIB=$PWD/paper_conf_sc_maacsh25_b200/$lib
  timeout 300 python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30 >> gpurun_out/exp1.jsonl 2>>gpurun_out/exp1.err
  timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 >> gpurun_out/exp1.jsonl 2>>gpurun_out/exp1.err
  timeout 300 python tools/exp_iter.py fem_q1 48 48 48 3 --K 2 --k 10 >> gpurun_out/exp1.jsonl 2>>gpurun_out/exp1.err
done
unset SPCG_LIB
for ex in level syncfree; do
  timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --sptrsv $ex --tag $ex >> gpurun_out/exp1.jsonl 2>>gpurun_out/exp1.err
  timeout 300 python tools/exp_iter.py fem_q1 48 48 48 3 --K 2 --k 10 --sptrsv $ex --tag $ex >> gpurun_out/exp1.jsonl 2>>gpurun_out/exp1.err
  timeout 300 python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30 --sptrsv $ex --tag $ex >> gpurun_out/exp1.jsonl 2>>gpurun_out/exp1.err
done
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
