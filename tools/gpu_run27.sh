#!/bin/bash
# persistent unit scheduling: full GPU suite, then A/B (CST_PERSIST=0/1) explores
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 2400 python -m pytest tests -m gpu -q -x --timeout 900 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_gpu.log
for ps in 0 1; do
  CST_PERSIST=$ps timeout -k 10 600 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_persist_explore.json --reps 5 > gpurun_out/explore_hyp_p$ps.log 2>&1
  CST_PERSIST=$ps timeout -k 10 600 python tools/explore.py --settings tools/star25_persist_explore.json --reps 10 > gpurun_out/explore_star_p$ps.log 2>&1
  CST_PERSIST=$ps timeout -k 10 600 python tools/explore.py --kind 2 --order 1 --settings tools/box_persist_explore.json --reps 10 > gpurun_out/explore_box_p$ps.log 2>&1
done
echo done
