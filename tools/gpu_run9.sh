#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for mode in 0 1; do
  export CST_NVRTC_DEFINES="-DCST_EMPTY_BARRIERS=$mode"
  timeout -k 10 600 python tools/explore.py --settings tools/star25_explore4.json > gpurun_out/ab_star_$mode.log 2>&1
  timeout -k 10 600 python tools/explore.py --kind 2 --order 1 --settings tools/box_explore2.json > gpurun_out/ab_box_$mode.log 2>&1
  timeout -k 10 600 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_explore3.json --reps 5 > gpurun_out/ab_hyp_$mode.log 2>&1
done
echo done
