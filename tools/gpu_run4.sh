#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout -k 10 900 python tools/explore.py --settings tools/star25_explore3.json > gpurun_out/explore3.log 2>&1
timeout -k 10 900 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_explore2.json --reps 5 > gpurun_out/explore_hyp2.log 2>&1
echo done
