"""oracle.space — brute-force enumeration of the csTuner parameter space.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  Plain nested loops in canonical field
order (Table I row order; values ascending), every rule checked as soon as the
fields it reads are fixed.  The C++ enumerator in libcst (csrc/space) must reproduce the
count, the ordered tuple stream (FNV-1a-64) and rank/unrank bit-exactly.

Space (readings Q14/Q15 of SURVEY.md §8(c)):

  #   field          range                          note
  1-3 TB_x,TB_y,TB_z p2[1,1024], p2[1,1024], p2[1,64] Table I
  4   staging        {1 none, 2 smem ld/st, 3 TMA}  useShared {1,2} + B200 TMA
  5   use_constant   {1,2}
  6   use_streaming  {1,2}
  7   SD             {1 x, 2 y, 3 z}                P:141; canonical 1 if streaming off
  8   SB             p2[1, M_SD]                    P:142; canonical 1 if streaming off
  9-11 UF_x,y,z      p2[1, M_d]
  12-14 CM_x,y,z     p2[1, M_d]
  15-17 BM_x,y,z     p2[1, M_d]
  18  use_retiming   {1,2}
  19  prefetch       {1 off, 2, 3, 4 stages}        usePrefetching {1,2} + depth
  20  bt             {1, 2, 4}                      temporal blocking degree: sweeps fused
                                                    per pass (B200 extension, SURVEY §8(f)
                                                    NEXT-2; "more optimization parameters",
                                                    P:127 / P:419)
  21  qstore         {1 registers, 2 TMEM}          where the streamed-direction state of the
                                                    retimed sweep lives (B200
                                                    extension: tensor memory)

Rules: paper R1 prod TB <= 1024; R2 SD=SB=1 when streaming off; R3 UF_SD <= SB when
streaming on.  Ours (Q15): R4 prod TB >= 32; R5 T_d = TB_d*BM_d*CM_d <= E_d (E_d = M_d,
E_SD = SB when streaming); R6 UF_d <= trip_d, the trip count of the loop the kernel path
unrolls along d (uf_trip; 1 where there is none); R7 prod(BM*CM) <= 16; R8 streaming =>
SD != 1; R9 prefetch > 1 => streaming with staging (nothing to prefetch into otherwise);
R10 modelled smem <= SMEM_LIMIT; R11 modelled registers <= 255; R12 smem staging (TMA or ld/st):
T_x even (16-B aligned rows; round 2 extended it to ld/st staging); TMA box: T_x even and
every box extent <= 256; R14 bt > 1 only for the temporally blocked path: star / box,
streaming along z with T_SD = 1, TMA staging, retimed accumulators, no cyclic merging,
BM_x, BM_y <= 2, every UF = 1 (reading Q23); R15 qstore = 2 only for the
TMEM path: star or hypterm (hypterm: one point along x, BM_b <= 2 along the other in-plane
dim, no cyclic merging), streaming with T_SD = 1, TMA staging, retimed, bt = 1, and
ceil(threads/128) * points per thread * (4r star, 20r hypterm) <= 512 TMEM columns;
R16 rhs4: use_retiming = 2 only for the retimed column walk (r4ret_path: streaming with
T_SD = 1, TMA, bt = 1, CM = 1, BM_b = 1, BM_x <= 2; qstore 2 puts its s-window queue in TMEM,
R15: ceil(threads/128) * points * 10(2r+1) <= 512 columns).  R6/R9/R16 keep every
field a kernel path does not read at its canonical value (round 2; tools/knob_audit.py).
"""
from __future__ import annotations

import math

FIELDS = ("tb_x", "tb_y", "tb_z", "staging", "use_constant", "use_streaming", "sd", "sb",
          "uf_x", "uf_y", "uf_z", "cm_x", "cm_y", "cm_z", "bm_x", "bm_y", "bm_z",
          "use_retiming", "prefetch", "bt", "qstore")

STAR, BOX, HYPTERM, RHS4 = 1, 2, 3, 4
SMEM_LIMIT = 227 * 1024 - 1024      # data bytes; 1 KiB kept for mbarriers / alignment
REG_LIMIT = 255


def p2(lo: int, hi: int):
    v, out = 1, []
    while v <= hi:
        if v >= lo:
            out.append(v)
        v *= 2
    return out


def n_arrays(kind: int) -> int:
    return {HYPTERM: 8, RHS4: 5}.get(kind, 1)


def live_doubles_per_point(kind: int, r: int) -> int:
    return {STAR: 2 * r + 2, BOX: 12, HYPTERM: 50, RHS4: 24}[kind]


def retention(kind: int, r: int) -> int:
    """Planes the gather (non-retimed) streaming path must keep after loading (T_SD == 1)."""
    return 2 * r if kind == BOX else r


def tiles(s: dict):
    return [s["tb_x"] * s["bm_x"] * s["cm_x"], s["tb_y"] * s["bm_y"] * s["cm_y"],
            s["tb_z"] * s["bm_z"] * s["cm_z"]]


def xr(r: int) -> int:
    """x half-width of a staged halo: r rounded up to even (16-B aligned TMA box rows)."""
    return r + (r & 1)


def tb_extent(r: int, s: dict, level: int):
    """(x, y) extents of level `level` of a temporally blocked CTA (level 0 = the TMA input
    box, level bt = the output tile): T + 2 (bt - level) * halo per side."""
    T = tiles(s)
    k = s["bt"] - level
    return T[0] + 2 * xr(r) * k, T[1] + 2 * r * k


def tb_blocks_per_thread(r: int, s: dict, level: int) -> int:
    ex, ey = tb_extent(r, s, level)
    nthr = s["tb_x"] * s["tb_y"] * s["tb_z"]
    return -(-((ex // s["bm_x"]) * (ey // s["bm_y"])) // nthr)


def r4ret_path(kind: int, s: dict) -> bool:
    """R16: the setting selects rhs4's retimed column walk (use_retiming = 2): streaming with
    T_SD = 1, TMA staging, bt = 1, no cyclic merging, one point along the in-plane non-x dim
    b, BM_x <= 2; its s-window queue in registers / shared memory (qstore 1) or TMEM (2)."""
    if kind != RHS4 or s["use_retiming"] != 2:
        return False
    if not (s["use_streaming"] == 2 and s["staging"] == 3 and s["bt"] == 1):
        return False
    sd = "xyz"[s["sd"] - 1]
    b = "y" if sd == "z" else "z"
    if any(s["cm_" + d] != 1 for d in "xyz"):
        return False
    return s["tb_" + sd] == 1 and s["bm_" + sd] == 1 and s["bm_" + b] == 1 and s["bm_x"] <= 2


def plane_geometry(kind: int, r: int, s: dict):
    """(in-plane elements P, ring planes NP) of the smem staging for a streaming setting;
    (box elements, 1) for a non-streaming one."""
    T = tiles(s)
    if s["use_streaming"] == 1:
        return (T[0] + 2 * r) * (T[1] + 2 * r) * (T[2] + 2 * r), 1
    sd = s["sd"] - 1
    a, b = [d for d in range(3) if d != sd]
    P = (T[a] + 2 * r) * (T[b] + 2 * r)
    D = s["prefetch"]
    if T[sd] == 1 and r4ret_path(kind, s):
        NP = D + 2 * r          # planes c-2 .. c+2 + prefetch (+ 6 product planes, smem_bytes)
    elif T[sd] == 1:
        NP = D + (0 if s["use_retiming"] == 2 else retention(kind, r))
    else:
        NP = D * T[sd] + 2 * r
    return P, NP


def smem_bytes(kind: int, r: int, s: dict) -> int:
    if s["staging"] == 1:
        return 0
    if s["bt"] > 1:
        # prefetch ring of input planes + two slots per intermediate level
        rnd = lambda e: -(-(e * 8) // 128) * 128
        e0 = tb_extent(r, s, 0)
        e1 = tb_extent(r, s, 1)
        return s["prefetch"] * rnd(e0[0] * e0[1]) + (s["bt"] - 1) * 2 * rnd(e1[0] * e1[1])
    P, NP = plane_geometry(kind, r, s)
    plane = -(-(P * 8) // 128) * 128
    return ((n_arrays(kind) * NP + (6 if r4ret_path(kind, s) else 0)) * plane
            + hyp_xprod_bytes(kind, r, s))


def hyp_xprod_bytes(kind: int, r: int, s: dict) -> int:
    """x-product planes of the TMEM hypterm kernel (round 2): two buffers of the 5 products
    E^x_f over the tile and its (even) x-halo."""
    if kind != HYPTERM or s["qstore"] != 2 or s["use_streaming"] != 2:
        return 0
    T = tiles(s)
    b = 1 if s["sd"] == 3 else 2
    return 2 * 5 * (-(-((T[0] + 2 * xr(r)) * T[b] * 8) // 128) * 128)


def points_per_thread(s: dict) -> int:
    ppt = 1
    for d in "xyz":
        ppt *= s["bm_" + d] * s["cm_" + d]
    return ppt


def tmem_columns(r: int, s: dict, kind: int = STAR) -> int:
    """TMEM columns of one CTA of the qstore = 2 path: warps are spread over the 4 lane
    quarters (ceil(threads/128) share one), each thread keeps 4r columns per point (star:
    r (value, partial) pairs) or 20r (hypterm: r slots of 5 products + r of 5 partials)."""
    nthr = s["tb_x"] * s["tb_y"] * s["tb_z"]
    if kind == RHS4:      # rhs4 retimed: 5 arrays x (2r+1) planes of the s-window, 2 columns each
        per = 10 * (2 * r + 1)
    else:
        per = (20 if kind == HYPTERM else 4) * r
    return (nthr // 32 + 3) // 4 * points_per_thread(s) * per


def qs_path_ok(kind: int, r: int, s: dict) -> bool:
    """R15: the TMEM streamed-state path's structural and capacity requirements (rhs4: the
    retimed column walk with its s-window queue in TMEM)."""
    if kind == RHS4:
        return r4ret_path(kind, s) and tmem_columns(r, s, kind) <= 512
    if not (kind in (STAR, HYPTERM) and s["use_streaming"] == 2 and s["staging"] == 3
            and s["use_retiming"] == 2 and s["bt"] == 1):
        return False
    if tiles(s)[s["sd"] - 1] != 1:
        return False
    if kind == HYPTERM:
        # one point along a (x), up to two stacked along b (the in-plane non-x dim)
        b = "y" if s["sd"] == 3 else "z"
        for d in "xyz":
            if s["cm_" + d] != 1 or s["bm_" + d] > 2 or (d != b and s["bm_" + d] != 1):
                return False
    return tmem_columns(r, s, kind) <= 512


def est_regs(kind: int, r: int, s: dict) -> int:
    if r4ret_path(kind, s):
        # s-window queue (5 arrays x 5 planes; 3 arrays when BM_x = 2), 5 x 3 pending
        # outputs, ~20 operands in flight, per point
        return 32 + 2 * s["bm_x"] * (60 if s["bm_x"] == 1 else 50)
    if s["qstore"] == 2 and kind == HYPTERM:
        # products, partial fluxes, the ring of one point, the in-plane row values
        return 32 + 2 * (5 * (r + 1) + 10 * points_per_thread(s) + 30)
    if s["qstore"] == 2:
        # in-plane part + centre per point, one point's ring, the block's column windows
        return 32 + 2 * (2 * points_per_thread(s) + (r + 1) + 2 * r)
    if s["bt"] > 1:
        # 2r+1 rotating accumulators per point of every level + one operand window
        pts = sum(tb_blocks_per_thread(r, s, lv) for lv in range(1, s["bt"] + 1))
        pts *= s["bm_x"] * s["bm_y"]
        win = (s["bm_y"] + 2 * r) * (s["bm_x"] + 2 * xr(r))
        return 32 + 2 * ((2 * r + 1) * pts + win)
    ppt = 1
    for d in "xyz":
        ppt *= s["bm_" + d] * s["cm_" + d]
    nthr = s["tb_x"] * s["tb_y"] * s["tb_z"]
    pf = 0
    if s["staging"] == 2 and s["prefetch"] > 1:
        P, _ = plane_geometry(kind, r, s)
        T = tiles(s)
        per_step = T[s["sd"] - 1] if s["use_streaming"] == 2 else 1
        pf = (s["prefetch"] - 1) * -(-(n_arrays(kind) * P * per_step) // nthr)
    return 32 + 2 * ppt * live_doubles_per_point(kind, r) + 2 * pf


def uf_trip(kind: int, s: dict, d: int) -> int:
    """R6: trip count of the per-thread loop that the setting's kernel path unrolls along
    dim d (loop unrolling), 1 where that path has no such loop (UF_d then stays at
    its canonical 1, so no two settings generate the same code — tools/knob_audit.py):
      streaming off (3-D tiles) and generic streaming (T_SD > 1, or rhs4): the merged-point
        loop, BM_d * CM_d;
      fast streaming paths (star / box / hypterm, T_SD = 1): no in-plane loop (the block is
        register-unrolled); along SD the plane loop, SB planes, which the compiler unrolls
        for star / box with TMA or no staging (not ld/st staging, not the hypterm, TMEM or
        temporally blocked kernels)."""
    a = "xyz"[d]
    bmcm = s["bm_" + a] * s["cm_" + a]
    if s["use_streaming"] == 1:
        return bmcm
    sd = s["sd"] - 1
    if r4ret_path(kind, s):
        return 1        # rhs4 retimed: the x pair runs in lockstep, the plane loop stays rolled
    if not (kind in (STAR, BOX, HYPTERM) and tiles(s)[sd] == 1):
        return bmcm
    if d != sd:
        return 1
    if kind in (STAR, BOX) and s["qstore"] == 1 and s["bt"] == 1 and s["staging"] != 2:
        return s["sb"]
    return 1


def tma_ok(r: int, s: dict) -> bool:
    T = tiles(s)
    if T[0] % 2:
        return False
    if s["bt"] > 1:
        return all(e <= 256 for e in tb_extent(r, s, 0))
    if s["use_streaming"] == 1:
        ext = [t + 2 * r for t in T]
    else:
        sd = s["sd"] - 1
        ext = [T[d] + 2 * r if d != sd else T[d] for d in range(3)]
    return all(e <= 256 for e in ext)


def check(kind: int, r: int, M, s: dict):
    """Return None if valid else the name of the first failing rule (R1..R12)."""
    tb = s["tb_x"] * s["tb_y"] * s["tb_z"]
    if tb > 1024:
        return "R1"
    stream = s["use_streaming"] == 2
    if not stream and (s["sd"] != 1 or s["sb"] != 1):
        return "R2"
    if stream and s["sd"] == 1:
        return "R8"
    if tb < 32:
        return "R4"
    T = tiles(s)
    sd = s["sd"] - 1
    for d in range(3):
        E = s["sb"] if (stream and d == sd) else M[d]
        if T[d] > E:
            return "R5"
    if stream and s["uf_" + "xyz"[sd]] > s["sb"]:
        return "R3"
    for d in range(3):
        if s["uf_" + "xyz"[d]] > uf_trip(kind, s, d):
            return "R6"
    ppt = 1
    for d in "xyz":
        ppt *= s["bm_" + d] * s["cm_" + d]
    if ppt > 16:
        return "R7"
    if s["prefetch"] > 1 and (not stream or s["staging"] == 1):
        return "R9"
    if s["bt"] > 1 and not tb_path_ok(kind, s):
        return "R14"
    if s["qstore"] == 2 and not qs_path_ok(kind, r, s):
        return "R15"
    if kind == RHS4 and s["use_retiming"] == 2 and not r4ret_path(kind, s):
        return "R16"
    if smem_bytes(kind, r, s) > SMEM_LIMIT:
        return "R10"
    if est_regs(kind, r, s) > REG_LIMIT:
        return "R11"
    if s["staging"] == 3 and not tma_ok(r, s):
        return "R12"
    if s["staging"] == 2 and T[0] % 2:       # ld/st rows are read as 16-B pairs as well
        return "R12"
    return None


def tb_path_ok(kind: int, s: dict) -> bool:
    """R14: the temporally blocked kernel's structural requirements."""
    return (kind in (STAR, BOX) and s["use_streaming"] == 2 and s["sd"] == 3
            and s["staging"] == 3 and s["use_retiming"] == 2
            and s["tb_z"] == 1 and s["bm_z"] == 1
            and s["cm_x"] == 1 and s["cm_y"] == 1 and s["cm_z"] == 1
            and s["bm_x"] <= 2 and s["bm_y"] <= 2
            and s["uf_x"] == 1 and s["uf_y"] == 1 and s["uf_z"] == 1)


def enumerate_space(kind: int, r: int, M):
    """Yield every valid setting (dict) in canonical order, by nested loops.  Rules that
    only read already-fixed fields are checked early purely to prune; the final `check`
    call decides validity."""
    Mx, My, Mz = M
    for tbx in p2(1, 1024):
        if tbx > Mx:
            continue
        for tby in p2(1, 1024):
            if tby > My or tbx * tby > 1024:
                continue
            for tbz in p2(1, 64):
                if tbz > Mz or tbx * tby * tbz > 1024 or tbx * tby * tbz < 32:
                    continue
                for stg in (1, 2, 3):
                    for uc in (1, 2):
                        for st in (1, 2):
                            for sd in (1, 2, 3):
                                if st == 1 and sd != 1:
                                    continue
                                if st == 2 and sd == 1:
                                    continue
                                sbs = p2(1, M[sd - 1]) if st == 2 else [1]
                                for sb in sbs:
                                    yield from _inner(kind, r, M, dict(
                                        tb_x=tbx, tb_y=tby, tb_z=tbz, staging=stg,
                                        use_constant=uc, use_streaming=st, sd=sd, sb=sb))


def _inner(kind, r, M, s):
    """Valid completions of the outer prefix `s`.  The loops run CM/BM before UF so that
    R7 can prune; the completions are then sorted into canonical (UF, CM, BM, ...) order.
    The outer prefix fields precede every inner field, so this yields the global order."""
    found = []
    for cmx in p2(1, M[0]):
        for cmy in p2(1, M[1]):
            for cmz in p2(1, M[2]):
                if cmx * cmy * cmz > 16:
                    continue
                for bmx in p2(1, M[0]):
                    for bmy in p2(1, M[1]):
                        for bmz in p2(1, M[2]):
                            if cmx * cmy * cmz * bmx * bmy * bmz > 16:
                                continue
                            T = tiles(dict(s, bm_x=bmx, bm_y=bmy, bm_z=bmz, cm_x=cmx,
                                           cm_y=cmy, cm_z=cmz))
                            if any(T[d] > M[d] for d in range(3)):
                                continue      # implied by R5 (SB <= M_SD)
                            # UF_d <= max(BM_d*CM_d, SB) is implied by R3/R6 (prune only)
                            bnd = [bmx * cmx, bmy * cmy, bmz * cmz]
                            if s["use_streaming"] == 2:
                                bnd[s["sd"] - 1] = s["sb"]
                            for ufx in p2(1, bnd[0]):
                                for ufy in p2(1, bnd[1]):
                                    for ufz in p2(1, bnd[2]):
                                        for ret in (1, 2):
                                            for pf in (1, 2, 3, 4):
                                                for bt in (1, 2, 4):
                                                    for qs in (1, 2):
                                                        t = dict(s, uf_x=ufx, uf_y=ufy, uf_z=ufz,
                                                                 cm_x=cmx, cm_y=cmy, cm_z=cmz,
                                                                 bm_x=bmx, bm_y=bmy, bm_z=bmz,
                                                                 use_retiming=ret, prefetch=pf,
                                                                 bt=bt, qstore=qs)
                                                        if check(kind, r, M, t) is None:
                                                            found.append(t)
    found.sort(key=as_tuple)
    yield from found


def as_tuple(s: dict):
    return tuple(s[f] for f in FIELDS)


FNV_OFFSET = 0xCBF29CE484222325
FNV_PRIME = 0x100000001B3


def fnv1a64_stream(settings) -> tuple[int, int]:
    """(count, FNV-1a-64 over the little-endian int32 encoding of every tuple in order)."""
    h, n = FNV_OFFSET, 0
    for s in settings:
        for v in as_tuple(s):
            for byte in int(v).to_bytes(4, "little", signed=True):
                h ^= byte
                h = (h * FNV_PRIME) & 0xFFFFFFFFFFFFFFFF
        n += 1
    return n, h


def literal_table1_count(M) -> int:
    """Size of the literal Table I space (useShared, usePrefetching in {1,2}) under the
    paper's explicit rules only (R1, R2, R3), by closed-form product counting."""
    Mx, My, Mz = M
    nlog = lambda m: int(math.floor(math.log2(m))) + 1
    ntb = sum(1 for a in p2(1, 1024) for b in p2(1, 1024) for c in p2(1, 64) if a * b * c <= 1024)
    per_dim = [nlog(m) for m in M]
    uf_cm_bm_all = 1
    for n in per_dim:
        uf_cm_bm_all *= n ** 3
    base = ntb * 2 * 2 * 2 * 2          # TB, useShared, useConstant, useRetiming, usePrefetching
    off = uf_cm_bm_all                  # streaming off: SD = SB = 1 canonical
    on = 0
    for sd in range(3):
        for sb in p2(1, M[sd]):
            nuf_sd = sum(1 for u in p2(1, M[sd]) if u <= sb)
            rest = uf_cm_bm_all // per_dim[sd] * nuf_sd
            on += rest
    return base * (off + on)
