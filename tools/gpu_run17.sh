#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python tools/explore.py --kind 1 --order 1 --nsteps 8 --settings tools/tb_explore_star.json --reps 5 > gpurun_out/explore_tb_star1.log 2>&1
timeout -k 10 900 python tools/explore.py --kind 1 --order 2 --nsteps 8 --settings tools/tb_explore_star.json --reps 5 > gpurun_out/explore_tb_star2.log 2>&1
echo done
