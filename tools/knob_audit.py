"""knob_audit.py — does every tuning field change the generated code? (CPU, no GPU)

For a set of base settings (one or more per kernel path) and every field, the valid
one-step neighbours (previous / next value of the field's range) are compiled with NVRTC
and their SASS (cuobjdump -sass) is compared with the base's.  A neighbour whose SASS is
byte-identical to the base's — and whose launch geometry is the same — is a dead knob: the
space would hold two settings that are one kernel.  Prints the dead pairs (JSON lines).

    python tools/knob_audit.py [--grid 64] [--jobs 8] [--only NAME]
"""
from __future__ import annotations

import argparse
import concurrent.futures as cf
import hashlib
import json
import os
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_cluster_sunlyjldlq21_b200 import cst as C  # noqa: E402

FIELDS = C.cst_setting.FIELDS if hasattr(C.cst_setting, "FIELDS") else None

STAR = dict(tb_x=32, tb_y=4, tb_z=1, staging=3, use_constant=1, use_streaming=2, sd=3, sb=32,
            uf_x=1, uf_y=1, uf_z=1, cm_x=1, cm_y=1, cm_z=1, bm_x=2, bm_y=2, bm_z=1,
            use_retiming=2, prefetch=3, bt=1, qstore=1)
# (name, kind, order, base setting overrides)
BASES = [
    ("star4_tma_ret", 1, 4, {}),
    ("star4_tma_gather", 1, 4, dict(use_retiming=1)),
    ("star4_l1", 1, 4, dict(staging=1, prefetch=1)),
    ("star4_ldst", 1, 4, dict(staging=2, prefetch=2)),
    ("star4_ystream", 1, 4, dict(sd=2, tb_y=1, tb_z=4, bm_y=1, bm_z=2)),
    ("star4_tmem", 1, 4, dict(qstore=2)),
    ("star4_generic", 1, 4, dict(tb_y=2, tb_z=2, bm_z=2, uf_z=2)),
    ("star4_tile3d", 1, 4, dict(use_streaming=1, sd=1, sb=1, prefetch=1, tb_y=2, tb_z=2,
                                bm_z=2, uf_z=2)),
    ("star1_tblock", 1, 1, dict(bt=2, prefetch=2)),
    ("box_tma_ret", 2, 1, dict(prefetch=2)),
    ("box_l1", 2, 1, dict(staging=1, prefetch=1)),
    ("hyp_tmem", 3, 4, dict(bm_x=1, bm_y=2, qstore=2, use_constant=2)),
    ("hyp_reg", 3, 4, dict(bm_x=1, bm_y=1, tb_y=8)),
    ("rhs4_generic", 4, 2, dict(tb_x=16, tb_y=8, bm_x=1, bm_y=1, prefetch=2, use_retiming=1)),
    ("star4_generic_l1", 1, 4, dict(tb_y=2, tb_z=2, bm_z=2, uf_z=2, staging=1, prefetch=1)),
    ("star4_generic_ldst", 1, 4, dict(tb_y=2, tb_z=2, bm_z=2, staging=2, prefetch=2)),
    ("hyp_reg_l1", 3, 4, dict(bm_x=1, bm_y=1, tb_y=8, staging=1, prefetch=1)),
    ("hyp_reg_ldst", 3, 4, dict(bm_x=1, bm_y=1, tb_y=8, staging=2, prefetch=2)),
    ("rhs4_l1", 4, 2, dict(tb_x=16, tb_y=8, bm_x=1, bm_y=1, staging=1, prefetch=1,
                                 use_retiming=1)),
    ("rhs4_bmz2", 4, 2, dict(tb_x=16, tb_y=8, bm_x=1, bm_y=1, bm_z=2, uf_z=2, prefetch=2,
                                   use_retiming=1)),
    ("box_ldst", 2, 1, dict(staging=2, prefetch=1)),
    ("rhs4_ret", 4, 2, dict(tb_x=16, tb_y=8, bm_x=1, bm_y=1, prefetch=2, use_retiming=2)),
    ("rhs4_ret_pair", 4, 2, dict(tb_x=8, tb_y=8, bm_x=2, bm_y=1, prefetch=2, use_retiming=2)),
    ("star2_tma_ret", 1, 2, {}),
]

NC = {1: lambda r: 6 * r + 1, 2: lambda r: 27, 3: lambda r: 7, 4: lambda r: 3}


def values(field, M):
    p2 = lambda hi: [1 << k for k in range(12) if (1 << k) <= hi]
    if field in ("tb_x", "tb_y"):
        return p2(1024)
    if field == "tb_z":
        return p2(64)
    if field == "staging":
        return [1, 2, 3]
    if field in ("use_constant", "use_streaming", "use_retiming", "qstore"):
        return [1, 2]
    if field == "sd":
        return [1, 2, 3]
    if field == "prefetch":
        return [1, 2, 3, 4]
    if field == "bt":
        return [1, 2, 4]
    return p2(max(M))


def sass_digest(cubin: bytes, tmpdir: str) -> str:
    fd, p = tempfile.mkstemp(suffix=".cubin", dir=tmpdir)
    with os.fdopen(fd, "wb") as f:
        f.write(cubin)
    out = subprocess.run(["cuobjdump", "-sass", p], capture_output=True, text=True, check=True).stdout
    os.unlink(p)
    body = [ln for ln in out.splitlines() if ln.strip().startswith("/*")]
    return hashlib.sha256("\n".join(body).encode()).hexdigest()


def geometry(d, M):
    T = [d["tb_" + a] * d["bm_" + a] * d["cm_" + a] for a in "xyz"]
    if d["use_streaming"] == 2:
        sd = d["sd"] - 1
        a, b = [k for k in range(3) if k != sd]
        return (-(-M[a] // T[a]), -(-M[b] // T[b]), -(-M[sd] // d["sb"]))
    return tuple(-(-M[k] // T[k]) for k in range(3))


def neighbours(h, base, M):
    for f in base:
        vals = values(f, M)
        i = vals.index(base[f])
        for j in (i - 1, i + 1):
            if 0 <= j < len(vals):
                d = dict(base, **{f: vals[j]})
                s = C.cst_setting.from_dict(d)
                try:
                    C.cst_setting_check(h, s)
                except C.CstError:
                    continue
                yield f, d


def audit(bases, n, jobs, tmpdir):
    M = (n, n, n)
    dead, checked = [], 0
    for name, kind, r, over in bases:
        h = C.cst_stencil_create(kind, r, [0.5] * NC[kind](r), C.make_grid(n, n, n, r))
        base = dict(STAR, **over)
        C.cst_setting_check(h, C.cst_setting.from_dict(base))
        todo = [("base", base)] + list(neighbours(h, base, M))

        def dig(item):
            return sass_digest(C.cst_variant_cubin(h, C.cst_setting.from_dict(item[1])), tmpdir)

        with cf.ThreadPoolExecutor(jobs) as ex:
            digs = list(ex.map(dig, todo))
        for (f, d), g in zip(todo[1:], digs[1:]):
            checked += 1
            if g == digs[0] and geometry(d, M) == geometry(base, M):
                dead.append(dict(path=name, field=f, base=base[f], neighbour=d[f]))
                print(json.dumps(dead[-1]), flush=True)
        C.cst_stencil_destroy(h)
    return dead, checked


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--grid", type=int, default=64)
    ap.add_argument("--jobs", type=int, default=os.cpu_count() or 4)
    ap.add_argument("--only", default=None)
    a = ap.parse_args()
    bases = [b for b in BASES if a.only is None or b[0] == a.only]
    with tempfile.TemporaryDirectory() as td:
        dead, checked = audit(bases, a.grid, a.jobs, td)
    print(json.dumps({"checked_pairs": checked, "dead_pairs": len(dead)}))


if __name__ == "__main__":
    main()
