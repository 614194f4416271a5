"""The C-ABI library on CPU: it loads, exports every symbol include/cst.h declares,
validates arguments, enumerates the parameter space bit-exactly like the oracle, and
generates + compiles (NVRTC, sm_100a) kernel variants without a GPU.  No compute calls."""
import json
import os
import random
import re

import pytest

from paper_conf_cluster_sunlyjldlq21_b200 import cst as C
from oracle import space as S
from cst_testutil import ROOT, gpu_available

HDR = os.path.join(ROOT, "include", "cst.h")
GOLD = os.path.join(ROOT, "tests", "golden")


def header_functions():
    txt = open(HDR).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    names = re.findall(r"\b(cst_[a-z0-9_]+)\s*\(", txt)
    return sorted(set(n for n in names if not n.endswith("_fn")))


def test_exports_every_declared_symbol():
    names = header_functions()
    assert len(names) >= 25
    for n in names:
        assert hasattr(C.lib(), n), n
    assert C.version().startswith("cst")


def coeffs_for(kind, r):
    return {C.CST_STAR: [1.0] * (6 * r + 1), C.CST_BOX: [1.0] * 27, C.CST_HYPTERM: [1.0] * 7,
            C.CST_RHS4: [1.0] * 3}[kind]


def handle(kind, r, n=(8, 8, 8), halo=None):
    g = C.make_grid(*n, halo if halo is not None else r)
    return C.cst_stencil_create(kind, r, coeffs_for(kind, r), g)


def test_create_validation():
    g = C.make_grid(8, 8, 8, 2)
    with pytest.raises(C.CstError) as e:
        C.cst_stencil_create(C.CST_STAR, 4, [1.0] * 25, g)          # halo < order
    assert e.value.status == C.CST_E_INVALID
    with pytest.raises(C.CstError) as e:
        C.cst_stencil_create(C.CST_BOX, 2, [1.0] * 125, C.make_grid(8, 8, 8, 2))
    assert e.value.status == C.CST_E_UNSUPPORTED
    with pytest.raises(C.CstError) as e:
        C.cst_stencil_create(C.CST_STAR, 2, [1.0] * 12, g)          # wrong coefficient count
    assert e.value.status == C.CST_E_INVALID
    bad = C.make_grid(8, 8, 8, 2)
    bad.pitch_x += 1                                                  # odd pitch
    with pytest.raises(C.CstError):
        C.cst_stencil_create(C.CST_STAR, 2, [1.0] * 13, bad)
    h = C.cst_stencil_create(C.CST_STAR, 2, [1.0] * 13, g)
    C.cst_stencil_destroy(h)


@pytest.mark.parametrize("kind,r", [(1, 2), (1, 4), (2, 1), (3, 4), (4, 2)])
def test_space_4cubed_matches_oracle_stream(kind, r):
    gold = json.load(open(os.path.join(GOLD, "space.json")))["spaces"]
    g = [e for e in gold if e["M"] == [4, 4, 4] and e["kind"] == kind and e["order"] == r][0]
    h = handle(kind, r, (4, 4, 4))
    n = C.cst_space_count(h)
    assert n == g["count"]
    tuples = [C.cst_space_at(h, i).as_tuple() for i in range(n)]
    settings = [dict(zip(S.FIELDS, t)) for t in tuples]
    cnt, fnv = S.fnv1a64_stream(settings)
    assert hex(fnv) == g["fnv1a64"]
    for i in range(0, n, 37):
        assert C.cst_space_rank(h, C.cst_space_at(h, i)) == i
    C.cst_stencil_destroy(h)


@pytest.mark.parametrize("kind,r", [(1, 4), (3, 4)])
def test_space_8cubed_counts_and_spot_positions(kind, r):
    gold = json.load(open(os.path.join(GOLD, "space.json")))["spaces"]
    g = [e for e in gold if e["M"] == [8, 8, 8] and e["kind"] == kind and e["order"] == r][0]
    h = handle(kind, r, (8, 8, 8))
    assert C.cst_space_count(h) == g["count"]
    if kind == 3:                       # small enough to compare positions with the oracle
        seq = [S.as_tuple(s) for s in S.enumerate_space(kind, r, (8, 8, 8))]
        rng = random.Random(5)
        for i in [0, len(seq) - 1] + [rng.randrange(len(seq)) for _ in range(200)]:
            assert C.cst_space_at(h, i).as_tuple() == seq[i]
    C.cst_stencil_destroy(h)


def test_rank_unrank_roundtrip_512():
    h = handle(1, 4, (512, 512, 512))
    n = C.cst_space_count(h)
    assert n > 10**7      # 2.35e7 after the canonical-UF rules (R6/R9/R16); literal Table I: 7.4e13
    rng = random.Random(11)
    for _ in range(300):
        i = rng.randrange(n)
        s = C.cst_space_at(h, i)
        C.cst_setting_check(h, s)
        assert C.cst_space_rank(h, s) == i
    prev = C.cst_space_at(h, 0).as_tuple()
    for i in range(1, 2000):                        # locally ascending
        cur = C.cst_space_at(h, i).as_tuple()
        assert cur > prev
        prev = cur
    C.cst_stencil_destroy(h)


def test_rules_agree_with_oracle_on_random_tuples():
    rng = random.Random(3)
    p2 = lambda hi: [1 << k for k in range(hi.bit_length()) if (1 << k) <= hi]
    for kind, r, M in [(1, 4, (64, 32, 128)), (2, 1, (32, 64, 16)), (3, 4, (64, 64, 64)),
                       (4, 2, (32, 32, 64))]:
        h = handle(kind, r, M)
        agree_valid = 0
        for _ in range(3000):
            d = dict(tb_x=rng.choice(p2(1024)), tb_y=rng.choice(p2(1024)), tb_z=rng.choice(p2(64)),
                     staging=rng.randint(1, 3), use_constant=rng.randint(1, 2),
                     use_streaming=rng.randint(1, 2), use_retiming=rng.randint(1, 2),
                     prefetch=rng.randint(1, 4))
            if d["use_streaming"] == 1:
                d["sd"], d["sb"] = 1, 1
                if rng.random() < 0.8:
                    d["prefetch"] = 1
            else:
                d["sd"] = rng.randint(1, 3)
                d["sb"] = rng.choice(p2(M[d["sd"] - 1]))
            for i, ax in enumerate("xyz"):
                d["uf_" + ax] = rng.choice(p2(M[i])[:4])
                d["cm_" + ax] = rng.choice(p2(M[i])[:3])
                d["bm_" + ax] = rng.choice(p2(M[i])[:4])
            d["bt"] = rng.choice([1, 1, 2, 4])
            if rng.random() < 0.3:              # the temporally blocked path's shape (R14)
                d.update(use_streaming=2, sd=3, staging=3, use_retiming=2, tb_z=1, bm_z=1,
                         bt=rng.choice([2, 4]), sb=rng.choice(p2(M[2])))
                for ax in "xyz":
                    d["cm_" + ax] = d["uf_" + ax] = 1
                d["bm_x"], d["bm_y"] = rng.choice([1, 2]), rng.choice([1, 2])
                d["tb_x"], d["tb_y"] = rng.choice([8, 16, 32, 64]), rng.choice([1, 2, 4, 8])
            d["qstore"] = rng.choice([1, 1, 2])
            if rng.random() < 0.3:              # the TMEM streamed-state path's shape (R15)
                d.update(use_streaming=2, sd=rng.choice([2, 3]), staging=3, use_retiming=2,
                         bt=1, qstore=2)
                d["sb"] = rng.choice(p2(M[d["sd"] - 1]))
                sa = "xyz"[d["sd"] - 1]
                d["tb_" + sa] = d["bm_" + sa] = d["cm_" + sa] = 1
                d["bm_x"] = rng.choice([1, 2, 4])
                d["tb_x"], d["tb_y" if sa == "z" else "tb_z"] = rng.choice([16, 32, 64]), rng.choice([1, 2, 4, 8])
            want = S.check(kind, r, M, d)
            s = C.cst_setting.from_dict(d)
            try:
                C.cst_setting_check(h, s)
                got = None
            except C.CstError as e:
                assert e.status == C.CST_E_CONSTRAINT
                got = str(e).split("violates ")[-1]
            assert got == want, (d, got, want)
            agree_valid += got is None
        n = C.cst_space_count(h)               # and every enumerated member is valid there
        for _ in range(200):
            assert S.check(kind, r, M, C.cst_space_at(h, rng.randrange(n)).as_dict()) is None
        C.cst_stencil_destroy(h)


def test_default_setting_valid():
    for kind, r, n in [(1, 2, (64, 64, 64)), (1, 4, (512, 512, 512)), (2, 1, (512, 512, 512)),
                       (3, 4, (512, 512, 512)), (1, 2, (4, 4, 4)), (3, 4, (8, 8, 8)),
                       (4, 2, (320, 320, 320))]:
        h = handle(kind, r, n)
        s = C.cst_setting_default(h)
        C.cst_setting_check(h, s)
        C.cst_stencil_destroy(h)


@pytest.mark.parametrize("kind,r", [(1, 4), (1, 2), (2, 1), (3, 4), (4, 2)])
def test_variants_compile_without_gpu(kind, r, tmp_path, monkeypatch):
    """Code generation + NVRTC for sm_100a of the default setting and random valid settings
    drawn from the canonical space (every path: streaming fast/generic, 3-D tiles)."""
    monkeypatch.setenv("CST_CACHE_DIR", str(tmp_path))
    h = handle(kind, r, (64, 64, 64))
    n = C.cst_space_count(h)
    rng = random.Random(kind * 10 + r)
    settings = [C.cst_setting_default(h)] + [C.cst_space_at(h, rng.randrange(n)) for _ in range(3)]
    for s in settings:
        t = C.cst_variant_compile(h, s)
        assert t > 0.0
        assert C.cst_variant_compile(h, s) == 0.0          # cache hit
    C.cst_stencil_destroy(h)


@pytest.mark.skipif(gpu_available(), reason="checks the no-GPU behaviour")
def test_compute_calls_fail_loudly_without_gpu():
    h = handle(1, 2, (8, 8, 8))
    s = C.cst_setting_default(h)
    with pytest.raises(C.CstError) as e:
        C.cst_sweep(h, s, [256], [1 << 20])
    assert e.value.status == C.CST_E_CUDA
    C.cst_stencil_destroy(h)
