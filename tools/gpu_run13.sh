#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
CST_BENCH_CLOCK_POLL_MS=20 timeout -k 10 600 python bench.py --no-cpu-baseline --no-other-configs --e2e-steps 0 > gpurun_out/bench_poll20.log 2>&1
CST_BENCH_CLOCK_POLL_MS=1000 timeout -k 10 600 python bench.py --no-cpu-baseline --no-other-configs --e2e-steps 0 > gpurun_out/bench_poll1000.log 2>&1
timeout -k 10 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-other-configs --e2e-steps 0 > gpurun_out/bench_20.log 2>&1
timeout -k 10 600 python tools/explore.py --kind 4 --order 2 --n 320 320 320 --settings tools/rhs4_explore.json --reps 5 > gpurun_out/explore_rhs4.log 2>&1
timeout -k 10 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 --no-other-configs > gpurun_out/ncu_launches.log 2>&1
timeout -k 10 600 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 5 -c 1 -o gpurun_out/prof_bench python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 --no-other-configs > gpurun_out/ncu_full.log 2>&1
echo done
