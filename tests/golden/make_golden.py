"""Writes the regression fixtures under tests/golden/ that come from the oracle.
Calls only oracle/ (never the CUDA path).  Run: python tests/golden/make_golden.py"""
import json
import os
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, os.path.dirname(os.path.dirname(HERE)))

from oracle import space as S  # noqa: E402
from oracle import tuner as T  # noqa: E402


def main():
    with open(os.path.join(HERE, "sampler.json"), "w") as f:
        json.dump({"source": "oracle.tuner.sample_ranks", "seed": 12345, "count": 1220000000,
                   "ranks": T.sample_ranks(12345, 1220000000, 16)}, f, indent=1)
    spaces = []
    for M in [(4, 4, 4), (8, 8, 8)]:
        for kind, r in [(1, 2), (1, 4), (2, 1), (3, 4), (4, 2)]:
            n, h = S.fnv1a64_stream(S.enumerate_space(kind, r, M))
            spaces.append({"M": list(M), "kind": kind, "order": r, "count": n, "fnv1a64": hex(h)})
    with open(os.path.join(HERE, "space.json"), "w") as f:
        json.dump({"source": "oracle.space.enumerate_space + fnv1a64_stream", "spaces": spaces}, f,
                  indent=1)


if __name__ == "__main__":
    main()
