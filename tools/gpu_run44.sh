#!/bin/bash
# A/B: TMA L2 promotion (CST_TMA_PROMO) on hypterm / star25 / box27; hypterm x-walk split
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python -c "import json; d=json.load(open('tuned/star25_512.json'))['setting']; print(json.dumps([d]))" > /tmp/s.json
python -c "import json; d=json.load(open('tuned/box27_512.json'))['setting']; print(json.dumps([d]))" > /tmp/b.json
for rep in 1 2; do
for P in 3 0 1 2; do
  CST_TMA_PROMO=$P timeout -k 10 600 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_final_explore.json --reps 10 > gpurun_out/promo_hyp_P${P}_$rep.log 2>&1
  CST_TMA_PROMO=$P timeout -k 10 600 python tools/explore.py --kind 1 --order 4 --settings /tmp/s.json --reps 30 > gpurun_out/promo_star_P${P}_$rep.log 2>&1
  CST_TMA_PROMO=$P timeout -k 10 600 python tools/explore.py --kind 2 --order 1 --settings /tmp/b.json --reps 30 > gpurun_out/promo_box_P${P}_$rep.log 2>&1
done
CST_NVRTC_DEFINES="-DCST_HYP_XSPLIT=1" timeout -k 10 600 python tools/explore.py --kind 3 --order 4 --settings tools/hyp_final_explore.json --reps 10 > gpurun_out/xsplit1_$rep.log 2>&1
done
CST_NVRTC_DEFINES="-DCST_HYP_XSPLIT=1" timeout -k 10 600 python -m pytest tests/test_gpu_tmem.py -m gpu -q --timeout 300 -p no:cacheprovider -k hyp > gpurun_out/pytest_xsplit.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_xsplit.log
echo done
