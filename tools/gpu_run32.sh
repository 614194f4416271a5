#!/bin/bash
# hypterm TMEM ring loaded late (fewer registers, 16 warps/SM) vs early
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
CST_NVRTC_DEFINES="-DCST_TM_LATE=1" timeout -k 10 900 python -m pytest tests/test_gpu_tmem.py -m gpu -q -k hypterm --timeout 300 -p no:cacheprovider > gpurun_out/pytest_tmem_late.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_tmem_late.log
CST_NVRTC_DEFINES="-DCST_TM_LATE=1" timeout -k 10 900 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_tmem_late_explore.json --reps 5 > gpurun_out/explore_hyp_late.log 2>&1
timeout -k 10 900 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_tmem_late_explore.json --reps 5 > gpurun_out/explore_hyp_early.log 2>&1
echo done
