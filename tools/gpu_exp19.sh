python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for part in auto strided; do
  if [ $part = auto ]; then unset SPCG_PART; else export SPCG_PART=$part; fi
  timeout 300 python tools/exp_iter.py poisson3d 102 102 102 --k 20 --modes alg2 --tag $part >> gpurun_out/exp19.jsonl 2>>gpurun_out/exp19.err
  timeout 300 python tools/exp_iter.py poisson3d 48 48 48 --k 30 --modes alg2 --tag $part >> gpurun_out/exp19.jsonl 2>>gpurun_out/exp19.err
  timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2 --tag $part >> gpurun_out/exp19.jsonl 2>>gpurun_out/exp19.err
done
