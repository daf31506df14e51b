python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for part in strided tiles contiguous; do
SPCG_PART=$part timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --modes alg2,none --tag $part >> gpurun_out/exp17.jsonl 2>>gpurun_out/exp17.err
done
