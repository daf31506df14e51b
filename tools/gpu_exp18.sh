python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2,none --tag auto >> gpurun_out/exp18.jsonl 2>>gpurun_out/exp18.err
timeout 300 python tools/exp_iter.py poisson2d 1024 1024 --k 30 --modes alg2,none --tag auto >> gpurun_out/exp18.jsonl 2>>gpurun_out/exp18.err
SPCG_PART=contiguous timeout 300 python tools/exp_iter.py poisson2d 1024 1024 --k 30 --modes alg2 --tag contiguous >> gpurun_out/exp18.jsonl 2>>gpurun_out/exp18.err
timeout 300 python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30 --modes alg2,none --tag auto >> gpurun_out/exp18.jsonl 2>>gpurun_out/exp18.err
timeout 300 python tools/exp_iter.py poisson3d 102 102 102 --k 20 --modes alg2 --tag auto >> gpurun_out/exp18.jsonl 2>>gpurun_out/exp18.err
SPCG_PART=strided timeout 300 python tools/exp_iter.py poisson3d 102 102 102 --k 20 --modes alg2 --tag strided >> gpurun_out/exp18.jsonl 2>>gpurun_out/exp18.err
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
