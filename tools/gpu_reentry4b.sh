#!/bin/bash
# session 4: full-neighbourhood hill climb from the tuned settings (tools/tune.py --start)
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out/tuned
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for c in hypterm star25 box27; do
  timeout -k 10 900 python tools/tune.py --config $c --start tuned/${c}_512.json --refine-all \
     --out gpurun_out/tuned/${c}_512_refined.json > gpurun_out/refine_$c.log 2>&1
  echo "$c rc=$?" >> gpurun_out/refine_$c.log
done
echo done
