#!/bin/bash
# session 4: hill-climbed settings -> full-size parity, bench, ncu capture of the bench kernel
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout -k 10 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q --timeout 400 -p no:cacheprovider > gpurun_out/pytest_fullsize.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_fullsize.log
timeout -k 10 600 python bench.py > gpurun_out/bench.log 2>&1
echo "bench rc=$?" >> gpurun_out/bench.log
timeout -k 10 600 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 4 -c 1 -o gpurun_out/prof_bench_s4 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 --no-other-configs > gpurun_out/ncu_full.log 2>&1
timeout -k 10 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 --no-other-configs > gpurun_out/ncu_launch.log 2>&1
echo done
