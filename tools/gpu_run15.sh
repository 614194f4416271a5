#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python tools/tune.py --config rhs4 --budget 240 > gpurun_out/tune_rhs4.log 2>&1
cp tuned/rhs4_320.json gpurun_out/ 2>/dev/null; mkdir -p gpurun_out/logs; cp tuned/logs/rhs4_seed1.json gpurun_out/logs/ 2>/dev/null
timeout -k 10 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
timeout -k 10 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1
timeout -k 10 900 python bench.py > gpurun_out/bench.log 2>&1
echo done
