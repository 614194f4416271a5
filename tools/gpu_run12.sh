#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out tuned
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 1200 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout -k 10 600 python tools/explore.py --kind 4 --order 2 --n 320 320 320 --settings tools/rhs4_explore.json --reps 5 > gpurun_out/explore_rhs4.log 2>&1
timeout -k 10 600 python tools/tune.py --config rhs4 --budget 200 > gpurun_out/tune_rhs4.log 2>&1
cp tuned/rhs4_320.json gpurun_out/ 2>/dev/null; mkdir -p gpurun_out/tune_logs; cp tuned/logs/rhs4_seed1.json gpurun_out/tune_logs/ 2>/dev/null
timeout -k 10 600 python bench.py > gpurun_out/bench.log 2>&1
echo done
