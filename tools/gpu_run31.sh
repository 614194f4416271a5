#!/bin/bash
# paired b-rows (star y-windows, hypterm b-lines) + TMEM star full prefetch: tests + explore
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 1200 python -m pytest tests/test_gpu_sweep.py tests/test_gpu_tmem.py -m gpu -q --timeout 600 -p no:cacheprovider > gpurun_out/pytest_pair.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_pair.log
timeout -k 10 900 python tools/explore.py --settings tools/star25_pair_explore.json --reps 10 > gpurun_out/explore_star_pair.log 2>&1
timeout -k 10 900 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_pair_explore.json --reps 5 > gpurun_out/explore_hyp_pair.log 2>&1
echo done
