cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 2400 python -m pytest tests/ -q -m gpu -x > gpurun_out/g11_pytest.log 2>&1
echo "exit $?" >> gpurun_out/g11_pytest.log
timeout 1200 python bench.py --steps 5 --warmup 3 > gpurun_out/g11_bench.log 2>&1
echo "exit $?" >> gpurun_out/g11_bench.log
