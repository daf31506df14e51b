python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python tools/diag.py aniso_layered 2048 2048 4 --k 10 >> gpurun_out/diag.jsonl 2>>gpurun_out/diag.err
timeout 300 python tools/diag.py poisson3d 64 64 64 --k 10 >> gpurun_out/diag.jsonl 2>>gpurun_out/diag.err
timeout 300 python tools/diag.py fem_q1 48 48 48 3 --K 2 --k 4 >> gpurun_out/diag.jsonl 2>>gpurun_out/diag.err
python -c "import paper_conf_sc_maacsh25_b200 as s, json; print(json.dumps(s.calibrate(0)))" > gpurun_out/calib.json 2>&1
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
