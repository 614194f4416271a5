#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for mode in 1 0; do
  export CST_NVRTC_DEFINES="-DCST_HYP_SCALAR=$mode"
  timeout -k 10 900 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_explore4.json --reps 5 > gpurun_out/hs_$mode.log 2>&1
done
export CST_NVRTC_DEFINES="-DCST_HYP_SCALAR=1"
timeout -k 10 600 python -m pytest tests/test_gpu_sweep.py -m gpu -q -k "3-4 or hyp" --timeout 300 -p no:cacheprovider > gpurun_out/pytest_hs.log 2>&1
echo done
