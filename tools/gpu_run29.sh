#!/bin/bash
# hypterm TMEM path: tests + exploration + ncu of the best guess
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python -m pytest tests/test_gpu_tmem.py -m gpu -q --timeout 300 -p no:cacheprovider > gpurun_out/pytest_tmem.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_tmem.log
timeout -k 10 900 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_tmem_explore.json --reps 5 > gpurun_out/explore_hyp_tmem.log 2>&1
N="ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 2 -c 1"
timeout -k 10 600 $N -o gpurun_out/prof_hyp_tmem python tools/prof_one.py 3 4 512x512x512 1 '{"tb_x":16,"tb_y":1,"tb_z":8,"staging":3,"use_constant":2,"use_streaming":2,"sd":2,"sb":512,"uf_x":1,"uf_y":1,"uf_z":1,"cm_x":1,"cm_y":1,"cm_z":1,"bm_x":1,"bm_y":1,"bm_z":1,"use_retiming":2,"prefetch":3,"bt":1,"qstore":2}' > gpurun_out/ncu_hyp_tmem.log 2>&1
python tools/ncu_summary.py gpurun_out/prof_hyp_tmem.ncu-rep gpurun_out/prof_hyp_tmem_sum
echo done
