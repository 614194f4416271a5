"""oracle.tuner — the csTuner method written out step by step, plain Python/numpy.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  The C++ tuner in libcst
(csrc/tuner) must reproduce: the sampled dataset indices, the CVs and groups
(Algorithm 1), the PCCs and metric collections (Algorithm 2), the PMNF fits (predictions
and RSE within 1e-10 relative), the kept (sampled) space up to borderline settings, and
the re-index tables.  The GA itself is pinned by properties, not matched.

Readings (restated in DESIGN.md §2):
* Q8  pair CV from the dataset only: for each value v of P_a present in the dataset
      (ascending), VS_ab[v] = encoded P_b of the best row with P_a = v (ties: lower rank).
* Q9  encoding: log2 for power-of-two parameters, raw value for bool/enum;
      population sigma (Eq. 1); CV := 0 when sigma == 0.
* Q6  Algorithm 1, text reading: alternate popleft / popright starting with
      popleft; left pops run the pair branch, right pops the singleton branch.
* Q10 Eq. 2 = standard Pearson r, deque ascending |r|; r := 0 for a constant metric.
* Q11 Algorithm 2: pop right; new collection while fewer than numCollections; a pair with
      exactly one collected metric joins that metric's collection; otherwise skipped.
* Q12 PMNF (Eq. 3): f = sum_k c_k prod_{l in G_k} P_l^i log2(P_l)^j, raw values, no
      intercept; least squares; RSE = sqrt(SSR / (m - rank)); min RSE over I x J.
* Q13 thresholds: one common order-statistic index t over a quantile sample of the space
      (the smallest t whose pass fraction is >= the sampling ratio); the sampled space is
      then every setting of the whole valid space that passes (sampled_space), and the GA's
      gene tables are its per-group projections (gene_tables).
"""
from __future__ import annotations

import math
from collections import deque

import numpy as np

from . import space as S

# fields whose values are powers of two (encoded by log2 for CV)
POW2_FIELDS = {"tb_x", "tb_y", "tb_z", "sb", "uf_x", "uf_y", "uf_z", "cm_x", "cm_y", "cm_z",
               "bm_x", "bm_y", "bm_z"}

MASK64 = (1 << 64) - 1


def _splitmix64(x: int) -> int:
    z = (x + 0x9E3779B97F4A7C15) & MASK64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31)


def sample_ranks(seed: int, count: int, n: int) -> list[int]:
    """Dataset sampler ("randomly sample 128 settings"): distinct ranks
    idx_i = (u_i * count) >> 64, u_i = splitmix64(splitmix64(seed) + i), duplicates
    rejected, in draw order.  If count <= n the whole space is returned in rank order."""
    if count <= n:
        return list(range(count))
    base = _splitmix64(seed & MASK64)
    seen, out, i = set(), [], 0
    while len(out) < n:
        u = _splitmix64((base + i) & MASK64)
        idx = (u * count) >> 64
        if idx not in seen:
            seen.add(idx)
            out.append(idx)
        i += 1
    return out


def encode(field: str, v: int) -> float:
    return math.log2(v) if field in POW2_FIELDS else float(v)


def cv(values) -> float:
    """Eq. 1: population standard deviation over mean; 0 when sigma == 0.
    Plain sequential sums (the C++ tuner sums in the same order)."""
    x = [float(v) for v in values]
    n = float(len(x))
    s = 0.0
    for v in x:
        s += v
    mu = s / n
    q = 0.0
    for v in x:
        q += (v - mu) * (v - mu)
    sigma = math.sqrt(q / n)
    if sigma == 0.0:
        return 0.0
    return sigma / mu


def pair_cvs(rows, fitness, fields=S.FIELDS):
    """All N(N-1) ordered pair CVs (Q7, Q8).  rows: list of dict settings in
    dataset order with their ranks; fitness: higher is better.
    Returns list of ((a, b), cv) in (a, b) field-index order."""
    out = []
    n = len(fields)
    for ia in range(n):
        a = fields[ia]
        for ib in range(n):
            if ib == ia:
                continue
            b = fields[ib]
            vs = []
            for v in sorted({r[a] for r, _ in rows}):
                best = None
                for (r, rank), f in zip(rows, fitness):
                    if r[a] != v:
                        continue
                    if best is None or f > best[0] or (f == best[0] and rank < best[1]):
                        best = (f, rank, r)
                vs.append(encode(b, best[2][b]))
            out.append(((ia, ib), cv(vs)))
    return out


def ascending_deque(pairs_with_score, key=lambda s: s):
    """Deque ordered by ascending score; ties keep the input (pair-index) order."""
    order = sorted(range(len(pairs_with_score)), key=lambda i: (key(pairs_with_score[i][1]), i))
    return deque(pairs_with_score[i][0] for i in order)


def group_parameters(dq: deque) -> list[list[int]]:
    """Algorithm 1, text reading (Q6)."""
    dq = deque(dq)
    groups: list[list[int]] = []

    def where(p):
        for gi, g in enumerate(groups):
            if p in g:
                return gi
        return -1

    n = len(dq)
    for i in range(n):
        if i % 2 == 0:                       # leftmost (lowest CV): pair branch
            a, b = dq.popleft()
            ga, gb = where(a), where(b)
            if ga < 0 and gb < 0:
                groups.append([a, b])
            elif ga >= 0 and gb >= 0:
                continue
            elif ga >= 0:
                groups[ga].append(b)
            else:
                groups[gb].append(a)
        else:                                # rightmost (highest CV): singleton branch
            a, b = dq.pop()
            if where(a) >= 0 and where(b) >= 0:
                continue
            if where(a) < 0:
                groups.append([a])
            if where(b) < 0:
                groups.append([b])
    return groups


def pcc(x, y) -> float:
    """Eq. 2 (garbled; Q10): the standard Pearson correlation coefficient
    (sequential sums)."""
    x = [float(v) for v in x]
    y = [float(v) for v in y]
    n = float(len(x))
    sx = sy = 0.0
    for a, b in zip(x, y):
        sx += a
        sy += b
    mx, my = sx / n, sy / n
    sxy = sxx = syy = 0.0
    for a, b in zip(x, y):
        dx, dy = a - mx, b - my
        sxy += dx * dy
        sxx += dx * dx
        syy += dy * dy
    ax, ay = math.sqrt(sxx), math.sqrt(syy)
    if ax == 0.0 or ay == 0.0:
        return 0.0
    return sxy / (ax * ay)


def metric_pairs(metrics: np.ndarray):
    """metrics: rows x M.  All unordered pairs (i < j) with their PCC, in (i, j) order."""
    M = metrics.shape[1]
    return [((i, j), pcc(metrics[:, i], metrics[:, j])) for i in range(M) for j in range(i + 1, M)]


def combine_metrics(dq: deque, num_collections: int) -> list[list[int]]:
    """Algorithm 2 (Q11): pop rightmost (highest |PCC|) until empty."""
    dq = deque(dq)
    cols: list[list[int]] = []

    def where(m):
        for ci, c in enumerate(cols):
            if m in c:
                return ci
        return -1

    while dq:
        a, b = dq.pop()
        ca, cb = where(a), where(b)
        if ca < 0 and cb < 0:
            if len(cols) < num_collections:
                cols.append([a, b])
            continue
        if ca >= 0 and cb >= 0:
            continue
        if ca >= 0:
            cols[ca].append(b)
        else:
            cols[cb].append(a)
    return cols


def select_metrics(cols, metrics: np.ndarray, times: np.ndarray) -> list[int]:
    """From each collection the metric with the highest |PCC| with execution time."""
    out = []
    for c in cols:
        best, bv = None, -1.0
        for m in c:
            v = abs(pcc(metrics[:, m], times))
            if v > bv:
                best, bv = m, v
        out.append(best)
    return out


IJ = [(i, j) for i in (0, 1, 2) for j in (0, 1)]


def pmnf_features(groups, X: np.ndarray, i: int, j: int) -> np.ndarray:
    """Eq. 3 design matrix: column k = prod_{l in G_k} P_l^i * log2(P_l)^j.
    X: rows x N raw (unencoded, >= 1) parameter values."""
    cols = []
    for g in groups:
        col = np.ones(X.shape[0])
        for l in g:
            p = X[:, l].astype(np.float64)
            col = col * (p ** i) * (np.log2(p) ** j)
        cols.append(col)
    return np.stack(cols, axis=1)


def lstsq_rank(A: np.ndarray, y: np.ndarray):
    """Least squares with numerical rank (numpy/LAPACK SVD, rcond = max(m,n)*eps)."""
    m, n = A.shape
    coef, _, rank, sv = np.linalg.lstsq(A, y, rcond=None)
    return coef, int(rank)


def pmnf_fit(groups, X: np.ndarray, y: np.ndarray):
    """Fit every (i, j) in I x J; return list of (i, j, coef, rse) and the index of the
    min-RSE hypothesis (first on ties)."""
    fits = []
    m = X.shape[0]
    for (i, j) in IJ:
        A = pmnf_features(groups, X, i, j)
        coef, rank = lstsq_rank(A, y)
        resid = y - A @ coef
        ssr = 0.0
        for e in resid:
            ssr += float(e) * float(e)
        dof = m - rank
        rse = math.sqrt(ssr / dof) if dof > 0 else float("inf")
        fits.append((i, j, coef, rse))
    best = min(range(len(fits)), key=lambda k: (fits[k][3], k))
    return fits, best


def pmnf_predict(groups, X: np.ndarray, fit) -> np.ndarray:
    i, j, coef, _ = fit
    return pmnf_features(groups, X, i, j) @ coef


def threshold_filter(preds: np.ndarray, directions, ratio: float):
    """Q13: preds = settings x K predicted metrics over the quantile sample; directions[k]
    = +1 if the metric correlates positively with time (smaller is better) else -1.
    Smallest order-statistic index t such that the fraction of settings passing every
    metric (pred <= asc_k[t], resp. >= desc_k[t]) is >= ratio.  Returns (t, thresholds)."""
    n, K = preds.shape
    asc = [np.sort(preds[:, k]) for k in range(K)]

    def thr(t):
        return [asc[k][t] if directions[k] > 0 else asc[k][n - 1 - t] for k in range(K)]

    def frac(t):
        th = thr(t)
        ok = np.ones(n, bool)
        for k in range(K):
            ok &= (preds[:, k] <= th[k]) if directions[k] > 0 else (preds[:, k] >= th[k])
        return ok.mean()

    lo, hi = 0, n - 1                     # frac(n-1) == 1
    while lo < hi:
        mid = (lo + hi) // 2
        if frac(mid) >= ratio:
            hi = mid
        else:
            lo = mid + 1
    return lo, thr(lo)


def sampled_space(X: np.ndarray, groups, chosen_fits, directions, th) -> np.ndarray:
    """P:290-292 ("filter out inappropriate parameter settings during the sampling
    process"), reading Q13: every setting of the WHOLE valid space (rows of X, raw values)
    whose predicted selected metrics all pass their thresholds (pred <= th for a metric
    that grows with time, >= th otherwise).  Returns the boolean keep mask."""
    keep = np.ones(X.shape[0], bool)
    for fit, d, t in zip(chosen_fits, directions, th):
        p = pmnf_predict(groups, X, fit)
        keep &= (p <= t) if d > 0 else (p >= t)
    return keep


def gene_tables(groups, X_kept: np.ndarray):
    """P:308-310 / Fig. 7: per group, the distinct value tuples of its fields over the
    sampled space, in ascending order (index = re-indexed gene value)."""
    return [sorted(set(tuple(int(v) for v in row) for row in X_kept[:, g])) for g in groups]


def passes(pred_row, directions, th) -> bool:
    return all((p <= t) if d > 0 else (p >= t) for p, d, t in zip(pred_row, directions, th))


def reindex(value_tuples) -> dict:
    """P:308-310 / Fig. 7: distinct valid value tuples of a group -> ascending index."""
    return {t: i for i, t in enumerate(sorted(set(value_tuples)))}
