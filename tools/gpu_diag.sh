python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python tools/diag.py aniso_layered 2048 2048 4 --k 10 >> gpurun_out/diag.jsonl 2>>gpurun_out/diag.err
timeout 300 python tools/diag.py poisson3d 64 64 64 --k 10 >> gpurun_out/diag.jsonl 2>>gpurun_out/diag.err
