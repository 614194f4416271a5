#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python -m pytest tests/test_gpu_sweep.py -m gpu -q -k "rhs4 or 4-2" --timeout 600 -p no:cacheprovider > gpurun_out/pytest_rhs4.log 2>&1
timeout -k 10 1200 python -m pytest tests/test_gpu_fullsize.py -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest_fullsize.log 2>&1
timeout -k 10 900 python tools/explore.py --kind 4 --order 2 --n 320 320 320 --settings tools/rhs4_explore3.json --reps 5 > gpurun_out/explore_rhs4c.log 2>&1

timeout -k 10 600 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 2 -c 1 -o gpurun_out/prof_hyp python tools/prof_one.py 3 4 512x512x512 1 tuned/hypterm_512.json > gpurun_out/ncu_hyp.log 2>&1
echo done
