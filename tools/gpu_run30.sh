#!/bin/bash
# re-tune the three 512^3 configs over the extended space (qstore); results to gpurun_out
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out/tuned
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout -k 10 600 python -m pytest tests/test_gpu_tmem.py -m gpu -q --timeout 300 -p no:cacheprovider > gpurun_out/pytest_tmem.log 2>&1
for c in star25 hypterm box27; do
  timeout -k 10 900 python tools/tune.py --config $c --budget 240 --seed 2 --out gpurun_out/tuned/${c}_512.json > gpurun_out/tune_$c.log 2>&1
done
cp -r tuned/logs gpurun_out/tuned/ 2>/dev/null
echo done
