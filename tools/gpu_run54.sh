#!/bin/bash
# star25 / box27 / hypterm: cst_tune (300 s) + neighbour refinement of the winner; bench after
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out/retune
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for cfg in star25 box27 hypterm; do
  timeout -k 10 1200 python tools/tune.py --config $cfg --budget 300 --seed 4 --refine --out gpurun_out/retune/${cfg}_512.json > gpurun_out/retune/$cfg.log 2>&1
  cp tuned/logs/${cfg}_seed4.json gpurun_out/retune/ 2>/dev/null
done
echo done
