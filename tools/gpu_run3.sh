#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python -m pytest tests -m gpu -q --timeout 300 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout -k 10 900 python tools/explore.py --kind 2 --order 1 --settings tools/box_explore.json > gpurun_out/explore_box.log 2>&1
timeout -k 10 1200 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_explore.json --reps 5 > gpurun_out/explore_hyp.log 2>&1
echo '[{"tb_x": 32, "tb_y": 4, "bm_x": 2, "bm_y": 2, "sb": 128, "prefetch": 3}]' > /tmp/one.json
timeout 600 ncu --set full --import-source on -k regex:cst_kernel -s 3 -c 1 -o gpurun_out/prof_star25_b python tools/explore.py --settings /tmp/one.json --reps 3 > gpurun_out/ncu2.log 2>&1
echo done
