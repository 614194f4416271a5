#!/bin/bash
# TMEM streamed-state path: parity + star25 exploration
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python -m pytest tests/test_gpu_tmem.py -m gpu -q -x --timeout 300 -p no:cacheprovider > gpurun_out/pytest_tmem.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_tmem.log
timeout -k 10 900 python tools/explore.py --settings tools/star25_tmem_explore.json --reps 10 > gpurun_out/explore_tmem.log 2>&1
echo done
