#!/bin/bash
# session 4: interleaved A/B re-timing of the hill-climb's proposals
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 600 python tools/explore.py --kind 1 --order 4 --settings tools/star25_sb_ab.json --reps 20 > gpurun_out/ab_star25.log 2>&1
timeout -k 10 900 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_refine_ab.json --reps 20 > gpurun_out/ab_hyp.log 2>&1
echo done
