#!/bin/bash
# hypterm TMEM two-point: early ring fetch A/B, parity, profile
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python -m pytest tests/test_gpu_tmem.py -m gpu -q --timeout 400 -p no:cacheprovider > gpurun_out/pytest_early.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_early.log
timeout -k 10 900 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_bmb2_explore.json --reps 10 > gpurun_out/explore_early1.log 2>&1
CST_NVRTC_DEFINES="-DCST_TM_EARLY=0" timeout -k 10 900 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_bmb2_explore.json --reps 10 > gpurun_out/explore_early0.log 2>&1
B='{"tb_x":16,"tb_y":8,"bm_y":2,"sb":256,"prefetch":3,"qstore":2,"use_constant":2}'
timeout -k 10 600 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 2 -c 1 -o gpurun_out/hyp_early python tools/prof_one.py 3 4 512x512x512 1 "$B" > gpurun_out/ncu_full.log 2>&1
echo done
