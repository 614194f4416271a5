#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python -m pytest tests/test_gpu_p2p.py tests/test_gpu_dist.py -m gpu -q --timeout 300 -p no:cacheprovider > gpurun_out/pytest_p2p.log 2>&1
timeout -k 10 600 python bench.py --no-cpu-baseline --no-other-configs --e2e-steps 0 > gpurun_out/bench_quick.log 2>&1
timeout -k 10 600 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 5 -c 1 -o gpurun_out/prof_bench python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 --no-other-configs > gpurun_out/ncu_full.log 2>&1
timeout -k 10 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 --no-other-configs > gpurun_out/ncu_launches.log 2>&1
timeout -k 10 3600 python tools/tuning_quality.py --out gpurun_out/r01_tuning_quality.json > gpurun_out/tuning_quality.log 2>&1
echo done
