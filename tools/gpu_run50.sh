#!/bin/bash
# TMEM hypterm: per-lane x weights selected once per thread (CST_HYP_WXPRE) A/B + parity
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 600 python -m pytest tests/test_gpu_tmem.py tests/test_gpu_fullsize.py -m gpu -q --timeout 300 -p no:cacheprovider -k "hyp or full" > gpurun_out/pytest_wx.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_wx.log
for rep in 1 2 3; do
timeout -k 10 600 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_empty_explore.json --reps 10 > gpurun_out/wx1_$rep.log 2>&1
CST_NVRTC_DEFINES="-DCST_HYP_WXPRE=0" timeout -k 10 600 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_empty_explore.json --reps 10 > gpurun_out/wx0_$rep.log 2>&1
done
echo done
