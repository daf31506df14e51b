#!/bin/bash
# Quick GPU check (run under gpurun): the named pytest files, then optional commands.
#   gpurun -- 'bash tools/gpu_quick.sh TAG "tests/a.py tests/b.py" "cmd1" "cmd2" ...'
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
TAG=$1; TESTS=$2; shift 2
O=gpurun_out/$TAG; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
if [ -n "$TESTS" ]; then timeout 1500 python -m pytest $TESTS -q -x -m gpu > $O/pytest.log 2>&1; echo "exit $?" >> $O/pytest.log; fi
i=0
for c in "$@"; do i=$((i+1)); timeout 1200 bash -c "$c" > $O/cmd$i.log 2>&1; echo "exit $?" >> $O/cmd$i.log; done
echo done > $O/DONE
