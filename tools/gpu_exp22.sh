python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
for tag in defer nodefer; do
if [ $tag = nodefer ]; then export SPCG_NO_DEFER=1; fi
timeout 300 python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30 --modes alg2,none --tag $tag >> gpurun_out/exp22.jsonl 2>>gpurun_out/exp22.err
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2 --tag $tag >> gpurun_out/exp22.jsonl 2>>gpurun_out/exp22.err
timeout 300 python tools/exp_iter.py poisson2d 1024 1024 --k 30 --modes alg2 --tag $tag >> gpurun_out/exp22.jsonl 2>>gpurun_out/exp22.err
done
