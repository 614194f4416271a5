#!/bin/bash
# hypterm TMEM: split x/b partial sums; one-barrier-per-two-planes A/B (CST_HYP_SYNC2)
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python -m pytest tests/test_gpu_tmem.py -m gpu -q --timeout 400 -p no:cacheprovider > gpurun_out/pytest_sync.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_sync.log
CST_NVRTC_DEFINES="-DCST_HYP_SYNC2=1" timeout -k 10 900 python -m pytest tests/test_gpu_tmem.py -m gpu -q --timeout 400 -p no:cacheprovider -k hyp >> gpurun_out/pytest_sync.log 2>&1
echo "rc sync2=$?" >> gpurun_out/pytest_sync.log
timeout -k 10 900 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_sync_explore.json --reps 10 > gpurun_out/explore_sync0.log 2>&1
CST_NVRTC_DEFINES="-DCST_HYP_SYNC2=1" timeout -k 10 900 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_sync_explore.json --reps 10 > gpurun_out/explore_sync1.log 2>&1
timeout -k 10 900 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_sync_explore.json --reps 10 > gpurun_out/explore_sync0b.log 2>&1
echo done
