#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
D='{"tb_x":32,"tb_y":4,"tb_z":1,"staging":3,"use_constant":1,"use_streaming":2,"sd":3,"sb":16,"uf_x":1,"uf_y":1,"uf_z":1,"cm_x":1,"cm_y":1,"cm_z":1,"bm_x":1,"bm_y":2,"bm_z":1,"use_retiming":2,"prefetch":3}'
timeout 120 python tools/run_one.py 1 1 33x20x17 default > gpurun_out/dbg_default.log 2>&1
timeout 300 compute-sanitizer --tool memcheck python tools/run_one.py 1 1 33x20x17 default > gpurun_out/dbg_memcheck.log 2>&1
for v in '"staging":2' '"prefetch":1' '"bm_y":1' '"use_retiming":1' '"sb":8'; do
  DD=$(echo $D | python -c "import json,sys; d=json.load(sys.stdin); d.update(json.loads('{'+sys.argv[1]+'}')); print(json.dumps(d))" "$v")
  echo "== $v" >> gpurun_out/dbg_vary.log
  timeout 120 python tools/run_one.py 1 1 33x20x17 "$DD" >> gpurun_out/dbg_vary.log 2>&1
done
for rr in 2 3; do echo "== r=$rr" >> gpurun_out/dbg_vary.log; timeout 120 python tools/run_one.py 1 $rr 33x20x17 default >> gpurun_out/dbg_vary.log 2>&1; done
echo '[{"tb_x": 64, "tb_y": 2, "bm_y": 4, "sb": 128}]' > /tmp/one.json
timeout 600 ncu --set full --import-source on -k regex:cst_kernel -s 3 -c 1 -o gpurun_out/prof_star25 python tools/explore.py --settings /tmp/one.json --reps 3 > gpurun_out/ncu1.log 2>&1
echo done
