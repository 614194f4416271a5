#!/bin/bash
# hypterm TMEM: full ncu capture of the best setting + DRAM/L2 counters over tile shapes
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
B='{"tb_x":32,"tb_y":1,"tb_z":8,"sd":2,"sb":256,"prefetch":2,"qstore":2,"use_constant":2,"staging":3,"use_streaming":2,"use_retiming":2}'
timeout -k 10 600 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 2 -c 1 -o gpurun_out/hyp_tmem_best python tools/prof_one.py 3 4 512x512x512 1 "$B" > gpurun_out/ncu_full.log 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,smsp__inst_executed.sum,sm__warps_active.avg.pct_of_peak_sustained_active
for S in \
 '{"tb_x":32,"tb_y":1,"tb_z":8,"sd":2,"sb":256,"prefetch":2,"qstore":2,"use_constant":2}' \
 '{"tb_x":32,"tb_y":1,"tb_z":8,"sd":2,"sb":512,"prefetch":2,"qstore":2,"use_constant":2}' \
 '{"tb_x":32,"tb_y":8,"sd":3,"sb":256,"prefetch":2,"qstore":2,"use_constant":2}' \
 '{"tb_x":16,"tb_y":1,"tb_z":16,"sd":2,"sb":256,"prefetch":2,"qstore":2,"use_constant":2}' \
 '{"tb_x":32,"tb_y":1,"tb_z":16,"sd":2,"sb":256,"prefetch":2,"qstore":2,"use_constant":2}' \
 '{"tb_x":64,"tb_y":4,"sb":256,"prefetch":2,"qstore":2,"use_constant":2}' \
 '{"tb_x":16,"tb_y":1,"tb_z":16,"sd":2,"sb":256,"prefetch":3,"use_constant":2}' ; do
  echo "SETTING $S" >> gpurun_out/ncu_dram.log
  timeout -k 10 300 ncu --metrics $M --clock-control none -k regex:cst_kernel -s 2 -c 1 --csv python tools/prof_one.py 3 4 512x512x512 1 "$(python -c "import json,sys; d=dict(staging=3,use_streaming=2,use_retiming=2,tb_z=1,sd=3); d.update(json.loads(sys.argv[1])); print(json.dumps(d))" "$S")" >> gpurun_out/ncu_dram.log 2>&1
done
echo done
