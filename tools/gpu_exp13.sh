python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
export SPCG_WIDE_MIN=0
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2 --sptrsv syncfree --tag sfwide >> gpurun_out/exp13.jsonl 2>>gpurun_out/exp13.err
timeout 300 python tools/exp_iter.py aniso_layered 2048 2048 4 --k 30 --modes alg2,none --sptrsv syncfree --tag sfwide >> gpurun_out/exp13.jsonl 2>>gpurun_out/exp13.err
timeout 300 python tools/exp_iter.py poisson2d 1024 1024 --k 30 --modes alg2 --sptrsv syncfree --tag sfwide >> gpurun_out/exp13.jsonl 2>>gpurun_out/exp13.err
timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2 --sptrsv level --tag lvwide >> gpurun_out/exp13.jsonl 2>>gpurun_out/exp13.err
unset SPCG_WIDE_MIN
timeout 300 python tools/exp_iter.py poisson2d 1024 1024 --k 30 --modes alg2 --tag chunked >> gpurun_out/exp13.jsonl 2>>gpurun_out/exp13.err
