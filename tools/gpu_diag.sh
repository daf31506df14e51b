cd $GRAFT_REPO_ROOT; O=gpurun_out/r02b; mkdir -p $O
./tools/micro/lat > $O/lat.txt 2>&1
for c in "aniso_layered 4096 4096 4" "aniso_layered 2048 2048 4" "poisson3d 64 64 64" "poisson2d 32 32" "poisson2d 1024 1024"; do
  SPCG_LIB=paper_conf_sc_maacsh25_b200/libspcg_prof.so K=10 timeout 300 python tools/chain_prof.py $c alg2 >> $O/chain_prof.jsonl 2>> $O/chain_prof.err
done
for ex in wchain chunked; do
  timeout 300 python tools/exp_iter.py poisson3d 64 64 64 --k 30 --sptrsv $ex >> $O/c2_exec.jsonl 2>>$O/exp.err
  timeout 300 python tools/exp_iter.py poisson2d 1024 1024 --k 30 --sptrsv $ex >> $O/p2d1024_exec.jsonl 2>>$O/exp.err
done
for ex in wchain resident; do
  timeout 300 python tools/exp_iter.py poisson2d 32 32 --k 30 --sptrsv $ex >> $O/c1_exec.jsonl 2>>$O/exp.err
  timeout 300 python tools/exp_iter.py poisson2d 64 64 --k 30 --sptrsv $ex >> $O/c1_exec.jsonl 2>>$O/exp.err
done
timeout 300 python -m pytest tests/test_gpu_parity.py -q -k "ll_flags" > $O/ll_stress.log 2>&1
timeout 300 python -c "
import paper_conf_sc_maacsh25_b200 as l, json
for ns,r in ((64,20000),(4096,2000),(1<<20,20)): print(json.dumps(dict(nslots=ns, rounds=r, **l.ll_stress(0,ns,r))))" >> $O/ll_stress.log 2>&1
for tool in memcheck synccheck racecheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize.py > $O/sanitize_$tool.log 2>&1; echo "exit $?" >> $O/sanitize_$tool.log
done
echo done > $O/DONE
