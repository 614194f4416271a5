#!/bin/bash
# session 4: second interleaved A/B round around the adopted hypterm setting
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_refine_ab2.json --reps 20 > gpurun_out/ab_hyp2.log 2>&1
nvidia-smi -q -d PERFORMANCE,POWER,TEMPERATURE > gpurun_out/smi_after.txt 2>&1
echo done
