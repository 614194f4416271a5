#!/bin/bash
# TMEM hypterm: per-warp slot release (CST_HYP_EMPTY) A/B, parity
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
CST_NVRTC_DEFINES="-DCST_HYP_EMPTY=1" timeout -k 10 600 python -m pytest tests/test_gpu_tmem.py -m gpu -q --timeout 200 -p no:cacheprovider -k hyp > gpurun_out/pytest_empty.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_empty.log
for rep in 1 2; do
timeout -k 10 600 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_empty_explore.json --reps 10 > gpurun_out/explore_empty0_$rep.log 2>&1
CST_NVRTC_DEFINES="-DCST_HYP_EMPTY=1" timeout -k 10 600 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_empty_explore.json --reps 10 > gpurun_out/explore_empty1_$rep.log 2>&1
done
echo done
