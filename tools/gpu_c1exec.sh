# C1 / small-system executor comparison (1 CTA): chunked vs level vs syncfree
O=gpurun_out/r01e_c1; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build rc=$?"
for s in chunked level syncfree; do
  timeout 300 python bench.py --workload C1 --sptrsv $s --no-cpu-baseline > $O/bench_c1_$s.json 2> $O/bench_c1_$s.err; echo "c1 $s rc=$?"
  python -c "import json;d=json.loads(open('$O/bench_c1_$s.json').read().strip().splitlines()[-1]);print('$s',d['value'],d['ms_per_iter'],d['pcg']['ms_per_iter'])"
done
