#!/bin/bash
# hypterm TMEM with two points along b (BM_b = 2): parity, explore, ncu of one variant
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python -m pytest tests/test_gpu_tmem.py tests/test_gpu_sweep.py -m gpu -q --timeout 400 -p no:cacheprovider -k "hyp or random" > gpurun_out/pytest_bmb.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_bmb.log
timeout -k 10 1200 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_bmb_explore.json --reps 10 > gpurun_out/explore_bmb.log 2>&1
B='{"tb_x":32,"tb_y":4,"bm_y":2,"sb":256,"prefetch":3,"qstore":2,"use_constant":2}'
timeout -k 10 600 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 2 -c 1 -o gpurun_out/hyp_bmb python tools/prof_one.py 3 4 512x512x512 1 "$B" > gpurun_out/ncu_full.log 2>&1
B='{"tb_x":32,"tb_y":8,"sb":256,"prefetch":3,"qstore":2,"use_constant":2}'
timeout -k 10 600 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 2 -c 1 -o gpurun_out/hyp_rows32 python tools/prof_one.py 3 4 512x512x512 1 "$B" >> gpurun_out/ncu_full.log 2>&1
echo done
