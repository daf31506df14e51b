python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30 >> gpurun_out/exp3.jsonl 2>>gpurun_out/exp3.err
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 >> gpurun_out/exp3.jsonl 2>>gpurun_out/exp3.err
timeout 300 python tools/exp_iter.py fem_q1 48 48 48 3 --K 2 --k 10 --modes alg2 >> gpurun_out/exp3.jsonl 2>>gpurun_out/exp3.err
timeout 600 python tools/exp_iter.py aniso_layered 4096 4096 4 --k 20 --modes alg2 --reps 3 >> gpurun_out/exp3.jsonl 2>>gpurun_out/exp3.err
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
