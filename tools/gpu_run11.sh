#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out tuned
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 1200 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout -k 10 900 python tools/tune.py --config star25 --budget 300 > gpurun_out/tune_star25.log 2>&1
cp tuned/star25_512.json gpurun_out/ 2>/dev/null; mkdir -p gpurun_out/tune_logs; cp tuned/logs/star25_seed1.json gpurun_out/tune_logs/ 2>/dev/null
timeout -k 10 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.log 2>&1
echo done
