#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python -m pytest tests/test_gpu_tblock.py -m gpu -q --timeout 600 -p no:cacheprovider > gpurun_out/pytest_tblock.log 2>&1
timeout -k 10 900 python tools/explore.py --kind 2 --order 1 --nsteps 8 --settings tools/tb_explore_box.json --reps 5 > gpurun_out/explore_tb_box.log 2>&1
echo done
