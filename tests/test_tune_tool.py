"""tools/tune.py hill-climb neighbourhood (host logic, no GPU)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))

import tune  # noqa: E402


def _start():
    with open(os.path.join(ROOT, "tuned", "star25_512.json")) as f:
        return json.load(f)["setting"]


def test_sb_prefetch_neighbourhood():
    cur = _start()
    nb = tune.neighbours(cur)
    changed = sorted((k, d[k]) for d in nb for k in d if d[k] != cur[k])
    assert changed == sorted([("sb", cur["sb"] // 2), ("sb", cur["sb"] * 2),
                              ("prefetch", cur["prefetch"] - 1), ("prefetch", cur["prefetch"] + 1)])


def test_full_neighbourhood_one_field_one_step():
    cur = _start()
    nb = tune.neighbours(cur, fixed={"staging"}, full=True)
    assert len({json.dumps(d, sort_keys=True) for d in nb}) == len(nb)
    for d in nb:
        diff = [k for k in d if d[k] != cur[k]]
        assert len(diff) == 1 and diff[0] != "staging"
        k = diff[0]
        if k in tune.SIZE_FIELDS:
            assert d[k] in (cur[k] // 2, cur[k] * 2) and d[k] >= 1
        else:
            assert abs(d[k] - cur[k]) == 1 and d[k] >= 0
    # every field but the fixed one moves at least one way
    assert {k for d in nb for k in d if d[k] != cur[k]} == set(cur) - {"staging"}
