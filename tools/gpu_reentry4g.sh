#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for i in 3; do timeout -k 10 300 python tools/step_series.py > gpurun_out/series_$i.json 2> gpurun_out/series_$i.err; done
echo done
