#!/bin/bash
# session 4: is the bimodal per-step time (≈20 % of steps ~1.2x median) caused by the NVML poll?
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for rep in 1 2; do
 for p in 2 50 1000; do
  CST_BENCH_CLOCK_POLL_MS=$p timeout -k 10 300 python bench.py --no-cpu-baseline --e2e-steps 0 --no-other-configs > gpurun_out/poll_${p}_$rep.log 2>&1
 done
done
echo done
