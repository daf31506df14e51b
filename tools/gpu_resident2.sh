O=gpurun_out/r01e_res5; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo "build rc=$?"
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "resident" > $O/pytest_parity.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_parity.log
timeout 600 python tools/res_cmp.py > $O/res_cmp.jsonl 2> $O/res_cmp.err; echo "cmp rc=$?"; cat $O/res_cmp.jsonl
