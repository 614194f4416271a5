#!/bin/bash
# tile dispatch order A/B (CST_TILE_BMAJOR): hypterm / star25 time + DRAM bytes
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct
for B in 0 1 0 1; do
  for S in tuned/hypterm_512.json '{"tb_x":32,"tb_y":8,"bm_y":2,"sb":256,"prefetch":3,"qstore":2,"use_constant":2,"uf_y":2,"uf_z":2}'; do
    echo "B=$B $S" >> gpurun_out/bmajor_ncu.log
    CST_NVRTC_DEFINES="-DCST_TILE_BMAJOR=$B" timeout -k 10 300 ncu --metrics $M --clock-control none -k regex:cst_kernel -s 2 -c 1 --csv python tools/prof_one.py 3 4 512x512x512 1 "$S" >> gpurun_out/bmajor_ncu.log 2>&1
  done
  echo "B=$B star" >> gpurun_out/bmajor_ncu.log
  CST_NVRTC_DEFINES="-DCST_TILE_BMAJOR=$B" timeout -k 10 300 ncu --metrics $M --clock-control none -k regex:cst_kernel -s 2 -c 1 --csv python tools/prof_one.py 1 4 512x512x512 1 tuned/star25_512.json >> gpurun_out/bmajor_ncu.log 2>&1
  CST_NVRTC_DEFINES="-DCST_TILE_BMAJOR=$B" timeout -k 10 600 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_empty_explore.json --reps 10 > gpurun_out/bmajor_hyp_$B.log 2>&1
done
echo done
