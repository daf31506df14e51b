python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python -c "import paper_conf_sc_maacsh25_b200 as s, json; print(json.dumps(s.calibrate(0)))" > gpurun_out/calib.json 2>&1
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
timeout 300 python tools/exp_iter.py fem_q1 48 48 48 3 --K 2 --k 10 --modes alg2 >> gpurun_out/exp6.jsonl 2>>gpurun_out/exp6.err
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2 >> gpurun_out/exp6.jsonl 2>>gpurun_out/exp6.err
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2 --sptrsv level --tag level >> gpurun_out/exp6.jsonl 2>>gpurun_out/exp6.err
