#!/bin/bash
# star/box: 16-B stores of x-adjacent output pairs (CST_STORE_VEC) A/B + parity
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 900 python -m pytest tests/test_gpu_sweep.py tests/test_gpu_dist.py tests/test_gpu_p2p.py tests/test_gpu_fullsize.py -m gpu -q --timeout 300 -p no:cacheprovider > gpurun_out/pytest_stvec.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_stvec.log
python -c "import json; d=json.load(open('tuned/star25_512.json'))['setting']; print(json.dumps([d, dict(d, sb=256)]))" > /tmp/s.json
python -c "import json; d=json.load(open('tuned/box27_512.json'))['setting']; print(json.dumps([d]))" > /tmp/b.json
for rep in 1 2 3; do
for V in 1 0; do
  CST_NVRTC_DEFINES="-DCST_STORE_VEC=$V" timeout -k 10 600 python tools/explore.py --kind 1 --order 4 --settings /tmp/s.json --reps 30 > gpurun_out/stvec_star_${V}_$rep.log 2>&1
  CST_NVRTC_DEFINES="-DCST_STORE_VEC=$V" timeout -k 10 600 python tools/explore.py --kind 2 --order 1 --settings /tmp/b.json --reps 30 > gpurun_out/stvec_box_${V}_$rep.log 2>&1
done
done
timeout -k 10 600 ncu --set full --import-source on --clock-control none -k regex:cst_kernel -s 2 -c 1 -o gpurun_out/star_stvec python tools/prof_one.py 1 4 512x512x512 1 tuned/star25_512.json > gpurun_out/ncu_stvec.log 2>&1
echo done
