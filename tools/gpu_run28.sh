#!/bin/bash
# after reverting persistent units: full GPU suite + quick bench + explores
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 2400 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_gpu.log
timeout -k 10 600 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_persist_explore.json --reps 5 > gpurun_out/explore_hyp.log 2>&1
timeout -k 10 600 python tools/explore.py --settings tools/star25_persist_explore.json --reps 10 > gpurun_out/explore_star.log 2>&1
echo done
