#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out tuned
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python -c "import torch; from paper_conf_cluster_sunlyjldlq21_b200 import cst as C; print(C.version())" > gpurun_out/version.log 2>&1
timeout -k 10 900 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout -k 10 900 python tools/explore.py --settings tools/star25_explore3.json > gpurun_out/explore3.log 2>&1
timeout -k 10 900 python tools/tune.py --config star25 --budget 300 > gpurun_out/tune_star25.log 2>&1
cp tuned/star25_512.json gpurun_out/ 2>/dev/null; cp -r tuned/logs gpurun_out/tune_logs 2>/dev/null
timeout -k 10 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench.log 2>&1
timeout -k 10 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_launches.log 2>&1
timeout -k 10 600 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 5 -c 1 -o gpurun_out/prof_bench python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_full.log 2>&1
echo done
