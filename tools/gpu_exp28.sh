python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
timeout 300 python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30 --modes alg2,none >> gpurun_out/exp28.jsonl 2>>gpurun_out/exp28.err
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2,none >> gpurun_out/exp28.jsonl 2>>gpurun_out/exp28.err
timeout 300 python tools/exp_iter.py poisson2d 1024 1024 --k 30 --modes alg2,none >> gpurun_out/exp28.jsonl 2>>gpurun_out/exp28.err
timeout 900 python tools/exp_iter.py aniso_layered 4096 4096 4 --k 20 --modes alg2,none --reps 3 >> gpurun_out/exp28.jsonl 2>>gpurun_out/exp28.err
