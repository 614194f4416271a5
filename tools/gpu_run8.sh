#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python -m pytest tests -m gpu -q -x --timeout 300 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout -k 10 600 python tools/explore.py --settings tools/star25_explore4.json > gpurun_out/explore_star4.log 2>&1
timeout -k 10 600 python tools/explore.py --kind 2 --order 1 --settings tools/box_explore2.json > gpurun_out/explore_box2.log 2>&1
timeout -k 10 600 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_explore3.json --reps 5 > gpurun_out/explore_hyp4.log 2>&1
echo '[{"tb_x": 32, "tb_y": 8, "sb": 256, "prefetch": 3, "use_retiming": 2, "staging": 3}]' > /tmp/h1.json
timeout -k 10 600 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 2 -c 1 -o gpurun_out/prof_hyp python tools/explore.py --kind 3 --order 4 --settings /tmp/h1.json --reps 1 > gpurun_out/ncu_hyp.log 2>&1
echo done
