#!/bin/bash
# TMEM path tests + ncu captures: tuned hypterm (y streaming), star25 register vs TMEM
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python -m pytest tests/test_gpu_tmem.py -m gpu -q --timeout 300 -p no:cacheprovider > gpurun_out/pytest_tmem.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_tmem.log
N="ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 2 -c 1"
timeout -k 10 600 $N -o gpurun_out/prof_hyp_tuned python tools/prof_one.py 3 4 512x512x512 1 tuned/hypterm_512.json > gpurun_out/ncu_hyp.log 2>&1
timeout -k 10 600 $N -o gpurun_out/prof_star_tm python tools/prof_one.py 1 4 512x512x512 1 '{"tb_x":32,"tb_y":4,"tb_z":1,"staging":3,"use_constant":1,"use_streaming":2,"sd":3,"sb":128,"uf_x":1,"uf_y":1,"uf_z":1,"cm_x":1,"cm_y":1,"cm_z":1,"bm_x":2,"bm_y":4,"bm_z":1,"use_retiming":2,"prefetch":4,"bt":1,"qstore":2}' > gpurun_out/ncu_star_tm.log 2>&1
for f in prof_hyp_tuned prof_star_tm; do python tools/ncu_summary.py gpurun_out/$f.ncu-rep gpurun_out/${f}_sum; done
timeout -k 10 900 python tools/explore.py --settings tools/star25_tmem_explore.json --reps 10 > gpurun_out/explore_tmem.log 2>&1
echo done
