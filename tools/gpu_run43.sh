#!/bin/bash
# round-1 session-3 pass: GPU suite, smoke, hypterm re-tune, bench, launch list, bench ncu
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
nvidia-smi > gpurun_out/smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout -k 10 1500 python -m pytest tests -m gpu -q --timeout 400 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout -k 10 900 python tools/tune.py --config hypterm --budget 240 > gpurun_out/tune_hyp.log 2>&1
cp tuned/hypterm_512.json gpurun_out/hypterm_512.json; cp tuned/logs/hypterm_seed1.json gpurun_out/hypterm_seed1.json
timeout -k 10 900 python bench.py > gpurun_out/bench.log 2>&1
timeout -k 10 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_ncu_launches.log 2>&1
timeout -k 10 900 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 5 -c 1 -o gpurun_out/prof_bench python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 0 --no-other-configs > gpurun_out/bench_ncu_full.log 2>&1
timeout -k 10 600 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 2 -c 1 -o gpurun_out/prof_hyp_tuned python tools/prof_one.py 3 4 512x512x512 1 tuned/hypterm_512.json > gpurun_out/ncu_hyp.log 2>&1
echo done
