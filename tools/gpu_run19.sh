#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
TB='{"tb_x":32,"tb_y":8,"tb_z":1,"staging":3,"use_constant":1,"use_streaming":2,"sd":3,"sb":128,"uf_x":1,"uf_y":1,"uf_z":1,"cm_x":1,"cm_y":1,"cm_z":1,"bm_x":2,"bm_y":2,"bm_z":1,"use_retiming":2,"prefetch":2,"bt":2}'
timeout -k 10 600 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 2 -c 1 -o gpurun_out/prof_tblock python tools/prof_one.py 1 1 512x512x512 8 "$TB" > gpurun_out/ncu_tblock.log 2>&1
timeout -k 10 600 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 2 -c 1 -o gpurun_out/prof_rhs4 python tools/prof_one.py 4 2 320x320x320 1 tuned/rhs4_320.json > gpurun_out/ncu_rhs4.log 2>&1
timeout -k 10 2400 python tools/tuning_quality.py --out gpurun_out/r01_tuning_quality.json > gpurun_out/tuning_quality.log 2>&1
echo done
