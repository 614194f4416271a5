#!/bin/bash
# tuning wall time with a cold and a warm cubin cache (100 s budget)
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out/tunetime
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
export CST_CACHE_DIR=/tmp/cst_cache_tunetime_$$
rm -rf $CST_CACHE_DIR
for cfg in star25 hypterm; do
  timeout -k 10 900 python tools/tune.py --config $cfg --budget 100 --seed 3 --out gpurun_out/tunetime/${cfg}_cold.json > gpurun_out/tunetime/${cfg}_cold.log 2>&1
  timeout -k 10 900 python tools/tune.py --config $cfg --budget 100 --seed 3 --out gpurun_out/tunetime/${cfg}_warm.json > gpurun_out/tunetime/${cfg}_warm.log 2>&1
done
cp tuned/logs/star25_seed3.json tuned/logs/hypterm_seed3.json gpurun_out/tunetime/ 2>/dev/null
echo done
