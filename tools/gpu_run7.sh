#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out tuned
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout -k 10 900 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_explore2.json --reps 5 > gpurun_out/explore_hyp3.log 2>&1
for c in star25 box27 hypterm; do
  timeout -k 10 900 python tools/tune.py --config $c --budget 240 > gpurun_out/tune_$c.log 2>&1
done
cp tuned/*.json gpurun_out/ 2>/dev/null; mkdir -p gpurun_out/tune_logs; cp tuned/logs/*.json gpurun_out/tune_logs/ 2>/dev/null
timeout -k 10 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.log 2>&1
echo done
