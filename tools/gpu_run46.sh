#!/bin/bash
# compact hypterm weight bank (CST_MAX_COEF back to 27): GPU suite, smoke, bench, tile explore
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout -k 10 1500 python -m pytest tests -m gpu -q --timeout 400 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout -k 10 900 python bench.py > gpurun_out/bench.log 2>&1
timeout -k 10 900 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_tile_explore.json --reps 10 > gpurun_out/explore_tile.log 2>&1
echo done
