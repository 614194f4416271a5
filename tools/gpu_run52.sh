#!/bin/bash
# star25: register blocking BM_y = 4 on the register path (fewer y-window wavefronts per point)
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python tools/explore.py --kind 1 --order 4 --settings tools/star25_bmy4_explore.json --reps 20 > gpurun_out/explore_star_bmy4.log 2>&1
echo done
