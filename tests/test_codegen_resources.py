"""Code generation resource check (CPU, no GPU): the sm_100a variants the bench and the
default settings use compile to cubins with no stack frame and no local memory (rule R13,
"only non-spilled parameter settings are explored").  A regression here shows up on
the GPU as R13 rejections (e.g. of the fused-halo twin in the z-slab sweep), so it is caught
here first by reading the cubins' resource usage with cuobjdump."""
import json
import os
import re
import shutil
import subprocess
import sys
import textwrap

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = textwrap.dedent("""
    import json, os, sys, glob
    sys.path.insert(0, %(root)r)
    from paper_conf_cluster_sunlyjldlq21_b200 import cst as C
    out = []
    for kind, r, n, setting, remote in json.loads(sys.argv[1]):
        os.environ["CST_NVRTC_DEFINES"] = "-DCST_REMOTE=1" if remote else ""
        nc = {1: 6 * r + 1, 2: 27, 3: 7, 4: 3}[kind]
        h = C.cst_stencil_create(kind, r, [0.5] * nc, C.make_grid(*n, r))
        s = C.cst_setting_default(h) if setting is None else C.cst_setting.from_dict(
            dict(C.cst_setting_default(h).as_dict(), **setting))
        before = set(os.listdir(os.environ["CST_CACHE_DIR"]))
        C.cst_variant_compile(h, s)
        new = sorted(set(os.listdir(os.environ["CST_CACHE_DIR"])) - before)
        out.append([json.dumps([kind, r, n, s.as_dict(), remote]), new])
        C.cst_stencil_destroy(h)
    print(json.dumps(out))
""")

CASES = [
    (1, 4, (512, 512, 512), None, False),                      # star25 default
    (1, 4, (64, 40, 16), dict(tb_x=32, tb_y=4, bm_x=2, bm_y=2, sb=8, prefetch=2), False),
    (1, 4, (64, 40, 16), dict(tb_x=32, tb_y=4, bm_x=2, bm_y=2, sb=8, prefetch=2), True),
    (2, 1, (512, 512, 512), None, False),                      # box27 default
    (3, 4, (512, 512, 512), None, False),                      # hypterm default (TMEM)
    (3, 4, (512, 512, 512), dict(qstore=1, bm_y=1, tb_y=8, prefetch=3), False),
    (4, 2, (320, 320, 320), None, False),                      # rhs4 default
    # hypterm register path with ld/st staging (tests/test_gpu_sweep.py "ldst-z")
    (3, 4, (37, 29, 26), dict(tb_x=32, tb_y=4, bm_y=1, qstore=1, staging=2, prefetch=1,
                              sb=8, use_constant=1), False),
]


def _tuned(name):
    with open(os.path.join(ROOT, "tuned", name)) as f:
        return json.load(f)["setting"]


# the settings bench.py times (tuned/*.json), and the fused-halo twin of the star25 one on
# bench's configs[4] slab (its p2p line)
CASES += [
    (1, 4, (512, 512, 512), _tuned("star25_512.json"), False),
    (1, 4, (1024, 1024, 256), _tuned("star25_512.json"), True),
    (2, 1, (512, 512, 512), _tuned("box27_512.json"), False),
    (3, 4, (512, 512, 512), _tuned("hypterm_512.json"), False),
    (4, 2, (320, 320, 320), _tuned("rhs4_320.json"), False),
]


@pytest.mark.skipif(shutil.which("cuobjdump") is None, reason="cuobjdump not found")
def test_default_and_bench_variants_have_no_stack_or_local(tmp_path):
    env = dict(os.environ, CST_CACHE_DIR=str(tmp_path))
    res = subprocess.run([sys.executable, "-c", CHILD % {"root": ROOT}, json.dumps(CASES)],
                         env=env, capture_output=True, text=True, timeout=900)
    assert res.returncode == 0, res.stderr[-2000:]
    files = json.loads(res.stdout.strip().splitlines()[-1])
    seen = {}
    for case, (key, new) in zip(CASES, files):
        if not new and key in seen:   # same variant as an earlier case (e.g. default == tuned)
            new = seen[key]
        assert len(new) == 1, (case, new)
        seen[key] = new
        usage = subprocess.run(["cuobjdump", "--dump-resource-usage", str(tmp_path / new[0])],
                               capture_output=True, text=True, check=True).stdout
        m = re.search(r"REG:(\d+) STACK:(\d+) SHARED:\d+ LOCAL:(\d+)", usage)
        assert m, usage
        regs, stack, local = (int(v) for v in m.groups())
        assert stack == 0 and local == 0, (case, usage.strip())
        assert regs <= 255, (case, regs)
