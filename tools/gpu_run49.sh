#!/bin/bash
# box27 best-of-tuned per staging mode (none / smem ld-st / TMA) + ncu; bench
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out/c3
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for m in 1 2 3; do
  timeout -k 10 600 python tools/tune.py --config box27 --budget 120 --fix staging=$m > gpurun_out/c3/tune_staging$m.log 2>&1
  cp tuned/box27_512_staging$m.json gpurun_out/c3/ 2>/dev/null
  cp tuned/logs/box27_staging${m}_seed1.json gpurun_out/c3/ 2>/dev/null
  timeout -k 10 600 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 2 -c 1 -o gpurun_out/c3/box27_staging$m python tools/prof_one.py 2 1 512x512x512 1 tuned/box27_512_staging$m.json > gpurun_out/c3/ncu_staging$m.log 2>&1
done
timeout -k 10 900 python bench.py > gpurun_out/bench.log 2>&1
echo done
