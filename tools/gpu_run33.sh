#!/bin/bash
# hypterm TMEM (late ring) over larger tiles
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python -m pytest tests/test_gpu_tmem.py -m gpu -q --timeout 300 -p no:cacheprovider > gpurun_out/pytest_tmem.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_tmem.log
timeout -k 10 1200 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_tmem_big_explore.json --reps 5 > gpurun_out/explore_hyp_big.log 2>&1
echo done
