#!/bin/bash
# tile raster order A/B (CST_RASTER_W): hypterm / star25 / box27 best settings, time + DRAM bytes
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 600 python -m pytest tests/test_gpu_sweep.py tests/test_gpu_tmem.py -m gpu -q --timeout 400 -p no:cacheprovider -k "ragged or random" > gpurun_out/pytest_raster.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_raster.log
H='[{"tb_x":16,"tb_y":16,"sb":256,"prefetch":3,"uf_z":2,"qstore":2,"use_constant":2},{"tb_x":16,"tb_y":16,"sb":256,"prefetch":2,"qstore":2,"use_constant":2},{"tb_x":16,"tb_y":16,"sb":512,"prefetch":3,"uf_z":2,"qstore":2,"use_constant":2}]'
echo "$H" > /tmp/h.json
python -c "import json; d=json.load(open('tuned/star25_512.json'))['setting']; print(json.dumps([d, dict(d, sb=256), dict(d, sb=512)]))" > /tmp/s.json
python -c "import json; d=json.load(open('tuned/box27_512.json'))['setting']; print(json.dumps([d, dict(d, sb=256), dict(d, sb=512)]))" > /tmp/b.json
for W in 0 4 8 16; do
  CST_NVRTC_DEFINES="-DCST_RASTER_W=$W" timeout -k 10 600 python tools/explore.py --kind 3 --order 4 --settings /tmp/h.json --reps 10 > gpurun_out/raster_hyp_W$W.log 2>&1
  CST_NVRTC_DEFINES="-DCST_RASTER_W=$W" timeout -k 10 600 python tools/explore.py --kind 1 --order 4 --settings /tmp/s.json --reps 20 > gpurun_out/raster_star_W$W.log 2>&1
  CST_NVRTC_DEFINES="-DCST_RASTER_W=$W" timeout -k 10 600 python tools/explore.py --kind 2 --order 1 --settings /tmp/b.json --reps 20 > gpurun_out/raster_box_W$W.log 2>&1
  CST_NVRTC_DEFINES="-DCST_RASTER_W=$W" timeout -k 10 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:cst_kernel -s 2 -c 1 --csv python tools/prof_one.py 3 4 512x512x512 1 '{"tb_x":16,"tb_y":16,"sb":256,"prefetch":3,"uf_z":2,"qstore":2,"use_constant":2}' > gpurun_out/raster_ncu_hyp_W$W.log 2>&1
  CST_NVRTC_DEFINES="-DCST_RASTER_W=$W" timeout -k 10 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:cst_kernel -s 2 -c 1 --csv python tools/prof_one.py 1 4 512x512x512 1 tuned/star25_512.json > gpurun_out/raster_ncu_star_W$W.log 2>&1
done
echo done
