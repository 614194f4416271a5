"""ctypes binding of libcst (include/cst.h) — argument marshalling only.

Every step of the sweep / tuner runs inside libcst.so (hand-written sm_100a CUDA + host
C++).  PyTorch is used by callers for device memory, streams and process groups only.
There is no CPU fallback: if libcst.so is missing this module raises at import time, and
without a GPU every compute call raises CstError(CST_E_CUDA).

Names follow the C ABI (cst_stencil_create, cst_sweep, cst_tune, ...).
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libcst.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} is missing: build it with `python paper_conf_cluster_sunlyjldlq21_b200/build.py`"
        " (there is no fallback implementation)")

_lib = ctypes.CDLL(LIB_PATH)

CST_OK, CST_E_INVALID, CST_E_UNSUPPORTED, CST_E_CONSTRAINT, CST_E_CUDA, CST_E_NVRTC, \
    CST_E_NCCL, CST_E_OOM, CST_E_INTERNAL = range(9)
CST_STAR, CST_BOX, CST_HYPTERM, CST_RHS4 = 1, 2, 3, 4
N_IN = {CST_STAR: 1, CST_BOX: 1, CST_HYPTERM: 8, CST_RHS4: 5}
N_OUT = {CST_STAR: 1, CST_BOX: 1, CST_HYPTERM: 5, CST_RHS4: 3}

FIELDS = ("tb_x", "tb_y", "tb_z", "staging", "use_constant", "use_streaming", "sd", "sb",
          "uf_x", "uf_y", "uf_z", "cm_x", "cm_y", "cm_z", "bm_x", "bm_y", "bm_z",
          "use_retiming", "prefetch", "bt", "qstore")


class CstError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{_lib.cst_status_str(status).decode()}: {msg}")
        self.status = status


class cst_stencil_desc(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("order", ctypes.c_int32), ("n_inputs", ctypes.c_int32),
                ("n_outputs", ctypes.c_int32), ("coeffs", ctypes.POINTER(ctypes.c_double)),
                ("n_coeffs", ctypes.c_int32)]


class cst_grid(ctypes.Structure):
    _fields_ = [("nx", ctypes.c_int64), ("ny", ctypes.c_int64), ("nz", ctypes.c_int64),
                ("halo", ctypes.c_int32), ("lead_x", ctypes.c_int32), ("pitch_x", ctypes.c_int64),
                ("pitch_y", ctypes.c_int64)]

    @property
    def numel(self) -> int:
        return (self.nz + 2 * self.halo) * self.pitch_y * self.pitch_x

    def offset(self, x, y, z) -> int:
        return ((z + self.halo) * self.pitch_y + (y + self.halo)) * self.pitch_x + self.lead_x + x


class cst_setting(ctypes.Structure):
    _fields_ = [("tb", ctypes.c_int32 * 3), ("staging", ctypes.c_int32),
                ("use_constant", ctypes.c_int32), ("use_streaming", ctypes.c_int32),
                ("sd", ctypes.c_int32), ("sb", ctypes.c_int32), ("uf", ctypes.c_int32 * 3),
                ("cm", ctypes.c_int32 * 3), ("bm", ctypes.c_int32 * 3),
                ("use_retiming", ctypes.c_int32), ("prefetch", ctypes.c_int32),
                ("bt", ctypes.c_int32), ("qstore", ctypes.c_int32)]

    def as_dict(self) -> dict:
        d = {}
        for i, ax in enumerate("xyz"):
            d["tb_" + ax] = self.tb[i]
            d["uf_" + ax] = self.uf[i]
            d["cm_" + ax] = self.cm[i]
            d["bm_" + ax] = self.bm[i]
        for f in ("staging", "use_constant", "use_streaming", "sd", "sb", "use_retiming",
                  "prefetch", "bt", "qstore"):
            d[f] = getattr(self, f)
        return {k: d[k] for k in FIELDS}

    def as_tuple(self):
        d = self.as_dict()
        return tuple(d[f] for f in FIELDS)

    @classmethod
    def from_dict(cls, d: dict) -> "cst_setting":
        s = cls()
        for i, ax in enumerate("xyz"):
            s.tb[i] = d["tb_" + ax]
            s.uf[i] = d["uf_" + ax]
            s.cm[i] = d["cm_" + ax]
            s.bm[i] = d["bm_" + ax]
        for f in ("staging", "use_constant", "use_streaming", "sd", "sb", "use_retiming",
                  "prefetch"):
            setattr(s, f, d[f])
        s.bt = d.get("bt", 1)   # field 20 (temporal blocking); older records predate it
        s.qstore = d.get("qstore", 1)  # field 21 (streamed state in TMEM); likewise
        return s

    def __repr__(self):
        return f"cst_setting({self.as_dict()})"


class cst_kernel_info(ctypes.Structure):
    _fields_ = [("registers", ctypes.c_int32), ("local_bytes", ctypes.c_int32),
                ("smem_bytes", ctypes.c_int32), ("threads", ctypes.c_int32),
                ("ctas_per_sm", ctypes.c_int32), ("grid_ctas", ctypes.c_int64),
                ("compile_s", ctypes.c_double)]


class cst_tune_opts(ctypes.Structure):
    _fields_ = [("seed", ctypes.c_uint64), ("dataset_size", ctypes.c_int32),
                ("sampling_ratio", ctypes.c_double), ("n_subpops", ctypes.c_int32),
                ("subpop_size", ctypes.c_int32), ("crossover", ctypes.c_double),
                ("mutation", ctypes.c_double), ("top_n", ctypes.c_int32),
                ("cv_threshold", ctypes.c_double), ("max_generations", ctypes.c_int32),
                ("num_collections", ctypes.c_int32), ("time_budget_s", ctypes.c_double),
                ("reps", ctypes.c_int32), ("warmup", ctypes.c_int32), ("log_path", ctypes.c_char_p),
                ("n_user_metrics", ctypes.c_int32), ("quantile_sample", ctypes.c_int32),
                ("warm_start", ctypes.c_int32), ("metrics_mode", ctypes.c_int32),
                ("nsteps", ctypes.c_int32), ("noise_reps", ctypes.c_int32),
                ("filter_threads", ctypes.c_int32), ("cool_ms", ctypes.c_int32)]


class cst_tune_report(ctypes.Structure):
    _fields_ = [("best_ms", ctypes.c_double), ("best_gstencils", ctypes.c_double),
                ("space_count", ctypes.c_uint64), ("sampled_count", ctypes.c_uint64),
                ("evaluations", ctypes.c_uint64), ("jit_compiles", ctypes.c_uint64),
                ("wall_s", ctypes.c_double), ("eval_s", ctypes.c_double), ("jit_s", ctypes.c_double),
                ("preproc_s", ctypes.c_double), ("n_groups", ctypes.c_int32),
                ("generations", ctypes.c_int32), ("phases_cv_stop", ctypes.c_int32),
                ("noise_cv", ctypes.c_double), ("cv_threshold_used", ctypes.c_double)]


class cst_halo_xfer(ctypes.Structure):
    _fields_ = [("peer", ctypes.c_int32), ("is_send", ctypes.c_int32),
                ("plane_begin", ctypes.c_int64), ("nplanes", ctypes.c_int64)]


EVAL_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.POINTER(cst_setting),
                           ctypes.c_int32, ctypes.POINTER(ctypes.c_double),
                           ctypes.POINTER(ctypes.c_double))

BCAST_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64,
                            ctypes.c_int32)
ALLGATHER_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                ctypes.c_int64)


class cst_collectives(ctypes.Structure):
    _fields_ = [("user", ctypes.c_void_p), ("bcast", BCAST_FN), ("allgather", ALLGATHER_FN)]


_P = ctypes.c_void_p
_PP = ctypes.POINTER(ctypes.c_void_p)
_S = ctypes.c_int  # cst_status


def _decl(name, res, *args):
    f = getattr(_lib, name)
    f.restype = res
    f.argtypes = list(args)
    return f


_decl("cst_status_str", ctypes.c_char_p, ctypes.c_int)
_decl("cst_last_error", ctypes.c_char_p)
_decl("cst_version", ctypes.c_char_p)
_decl("cst_stencil_create", _S, ctypes.POINTER(cst_stencil_desc), ctypes.POINTER(cst_grid),
      ctypes.c_int, ctypes.POINTER(_P))
_decl("cst_stencil_destroy", None, _P)
_decl("cst_setting_check", _S, _P, ctypes.POINTER(cst_setting))
_decl("cst_setting_default", _S, _P, ctypes.POINTER(cst_setting))
_decl("cst_space_count", _S, _P, ctypes.POINTER(ctypes.c_uint64))
_decl("cst_space_at", _S, _P, ctypes.c_uint64, ctypes.POINTER(cst_setting))
_decl("cst_space_rank", _S, _P, ctypes.POINTER(cst_setting), ctypes.POINTER(ctypes.c_uint64))
_decl("cst_kernel_info_get", _S, _P, ctypes.POINTER(cst_setting), ctypes.POINTER(cst_kernel_info))
_decl("cst_variant_compile", _S, _P, ctypes.POINTER(cst_setting), ctypes.POINTER(ctypes.c_double))
_decl("cst_variant_cubin", _S, _P, ctypes.POINTER(cst_setting), ctypes.c_int32, _P, ctypes.c_int64,
      ctypes.POINTER(ctypes.c_int64))
_decl("cst_sweep", _S, _P, ctypes.POINTER(cst_setting), _PP, _PP, ctypes.c_int32, _P)
_decl("cst_sweep_host", _S, _P, ctypes.POINTER(cst_setting), _PP, _PP, ctypes.c_int32)
_decl("cst_sync", _S, _P)
_decl("cst_last_launch_count", ctypes.c_int64, _P)
_decl("cst_fill_uniform", _S, ctypes.POINTER(cst_grid), _P, ctypes.c_uint64, ctypes.c_uint64,
      ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_double, _P)
_decl("cst_time_setting", _S, _P, ctypes.POINTER(cst_setting), _PP, _PP, ctypes.c_int32,
      ctypes.c_int32, ctypes.c_int32, _P, ctypes.POINTER(ctypes.c_double))
_decl("cst_collect_metrics", _S, _P, ctypes.POINTER(cst_setting), _PP, _PP,
      ctypes.POINTER(ctypes.c_char_p), ctypes.c_int32, ctypes.POINTER(ctypes.c_double))
_decl("cst_fp64_peak", _S, ctypes.c_int, ctypes.POINTER(ctypes.c_double),
      ctypes.POINTER(ctypes.c_double))
_decl("cst_tune_opts_default", None, ctypes.POINTER(cst_tune_opts))
_decl("cst_tune", _S, _P, ctypes.POINTER(cst_tune_opts), _PP, _PP, EVAL_FN, _P,
      ctypes.POINTER(cst_setting), ctypes.POINTER(cst_tune_report))
_decl("cst_dist_halo_plan", _S, ctypes.c_int32, ctypes.c_int32, ctypes.c_int64, ctypes.c_int32,
      ctypes.POINTER(cst_halo_xfer), ctypes.POINTER(ctypes.c_int32))
_decl("cst_dist_create", _S, _P, ctypes.c_int32, ctypes.c_int32, _P, ctypes.POINTER(_P))
_decl("cst_dist_create_host", _S, _P, ctypes.c_int32, ctypes.c_int32,
      ctypes.POINTER(cst_collectives), ctypes.POINTER(_P))
_decl("cst_dist_tune", _S, _P, ctypes.POINTER(cst_tune_opts), _PP, _PP, EVAL_FN, _P,
      ctypes.POINTER(cst_setting), ctypes.POINTER(cst_tune_report))
_decl("cst_dist_nccl_unique_id", _S, _P)
_decl("cst_dist_sweep", _S, _P, ctypes.POINTER(cst_setting), _PP, _PP, ctypes.c_int32, _P)
_decl("cst_dist_sweep_loopback", _S, _P, ctypes.c_int32, ctypes.POINTER(cst_setting), _PP, _PP,
      ctypes.c_int32, _P)
_decl("cst_dist_destroy", None, _P)
_decl("cst_dist_p2p_export", _S, _P, _PP, _PP, _P)
_decl("cst_dist_p2p_import", _S, _P, ctypes.c_int32, _P)
P2P_BLOB_BYTES = 2048

EXPORTS = [n for n in dir(_lib) if n.startswith("cst_")]


def check(status: int) -> None:
    if status != CST_OK:
        raise CstError(status, _lib.cst_last_error().decode(errors="replace"))


def lib():
    return _lib


def version() -> str:
    return _lib.cst_version().decode()


def _ptrs(ptrs):
    arr = (ctypes.c_void_p * len(ptrs))(*[ctypes.c_void_p(int(p)) for p in ptrs])
    return ctypes.cast(arr, _PP), arr


def make_grid(nx: int, ny: int, nz: int, halo: int, lead_x: int | None = None,
              align: int = 16) -> cst_grid:
    """Grid with interior x=0 on a 128-B boundary and rows padded to `align` doubles."""
    if lead_x is None:
        lead_x = max(16, -(-halo // 16) * 16)
    pitch_x = -(-(lead_x + nx + halo) // align) * align
    return cst_grid(nx, ny, nz, halo, lead_x, pitch_x, ny + 2 * halo)


# ------------------------------------------------------------------ C-ABI mirrors
def cst_stencil_create(kind: int, order: int, coeffs, grid: cst_grid, device: int = 0):
    c = (ctypes.c_double * len(coeffs))(*[float(v) for v in coeffs])
    desc = cst_stencil_desc(kind, order, N_IN[kind], N_OUT[kind], c, len(coeffs))
    h = ctypes.c_void_p()
    check(_lib.cst_stencil_create(ctypes.byref(desc), ctypes.byref(grid), device, ctypes.byref(h)))
    return h


def cst_stencil_destroy(h) -> None:
    _lib.cst_stencil_destroy(h)


def cst_setting_check(h, s: cst_setting) -> None:
    check(_lib.cst_setting_check(h, ctypes.byref(s)))


def cst_setting_default(h) -> cst_setting:
    s = cst_setting()
    check(_lib.cst_setting_default(h, ctypes.byref(s)))
    return s


def cst_space_count(h) -> int:
    n = ctypes.c_uint64()
    check(_lib.cst_space_count(h, ctypes.byref(n)))
    return n.value


def cst_space_at(h, rank: int) -> cst_setting:
    s = cst_setting()
    check(_lib.cst_space_at(h, rank, ctypes.byref(s)))
    return s


def cst_space_rank(h, s: cst_setting) -> int:
    r = ctypes.c_uint64()
    check(_lib.cst_space_rank(h, ctypes.byref(s), ctypes.byref(r)))
    return r.value


def cst_kernel_info_get(h, s: cst_setting) -> cst_kernel_info:
    i = cst_kernel_info()
    check(_lib.cst_kernel_info_get(h, ctypes.byref(s), ctypes.byref(i)))
    return i


def cst_variant_compile(h, s: cst_setting) -> float:
    t = ctypes.c_double()
    check(_lib.cst_variant_compile(h, ctypes.byref(s), ctypes.byref(t)))
    return t.value


def cst_variant_cubin(h, s: cst_setting, remote: bool = False) -> bytes:
    n = ctypes.c_int64()
    rc = _lib.cst_variant_cubin(h, ctypes.byref(s), int(remote), None, 0, ctypes.byref(n))
    if rc not in (0, 1) or n.value == 0:
        check(rc)
    buf = ctypes.create_string_buffer(n.value)
    check(_lib.cst_variant_cubin(h, ctypes.byref(s), int(remote), buf, n.value, ctypes.byref(n)))
    return buf.raw[:n.value]


def cst_sweep(h, s: cst_setting, in_ptrs, out_ptrs, nsteps: int = 1, stream: int = 0) -> None:
    pi, _a = _ptrs(in_ptrs)
    po, _b = _ptrs(out_ptrs)
    check(_lib.cst_sweep(h, ctypes.byref(s), pi, po, nsteps, ctypes.c_void_p(stream)))


def cst_sweep_host(h, s: cst_setting, in_ptrs, out_ptrs, nsteps: int = 1) -> None:
    pi, _a = _ptrs(in_ptrs)
    po, _b = _ptrs(out_ptrs)
    check(_lib.cst_sweep_host(h, ctypes.byref(s), pi, po, nsteps))


def cst_sync(h) -> None:
    check(_lib.cst_sync(h))


def cst_last_launch_count(h) -> int:
    return int(_lib.cst_last_launch_count(h))


def cst_fill_uniform(grid: cst_grid, dev_ptr: int, seed: int, array_id: int, nx_global=None,
                     ny_global=None, z0: int = 0, pad_value: float = float("nan"),
                     stream: int = 0) -> None:
    check(_lib.cst_fill_uniform(ctypes.byref(grid), ctypes.c_void_p(dev_ptr), seed, array_id,
                                grid.nx if nx_global is None else nx_global,
                                grid.ny if ny_global is None else ny_global, z0, pad_value,
                                ctypes.c_void_p(stream)))


def cst_time_setting(h, s: cst_setting, in_ptrs, out_ptrs, warmup=2, reps=5, stream=0,
                     nsteps=1) -> float:
    """Median ms PER STEP of `reps` timed cst_sweep calls of `nsteps` steps."""
    pi, _a = _ptrs(in_ptrs)
    po, _b = _ptrs(out_ptrs)
    ms = ctypes.c_double()
    check(_lib.cst_time_setting(h, ctypes.byref(s), pi, po, nsteps, warmup, reps,
                                ctypes.c_void_p(stream), ctypes.byref(ms)))
    return ms.value


def cst_collect_metrics(h, s: cst_setting, in_ptrs, out_ptrs, names):
    """{metric name: value} of one sweep from the CUPTI range profiler."""
    pi, _a = _ptrs(in_ptrs)
    po, _b = _ptrs(out_ptrs)
    arr = (ctypes.c_char_p * len(names))(*[n.encode() for n in names])
    vals = (ctypes.c_double * len(names))()
    check(_lib.cst_collect_metrics(h, ctypes.byref(s), pi, po, arr, len(names), vals))
    return dict(zip(names, list(vals)))


def cst_fp64_peak(device: int = 0):
    """(TFLOP/s, max SM clock GHz) from the DFMA-chain microbenchmark."""
    t, g = ctypes.c_double(), ctypes.c_double()
    check(_lib.cst_fp64_peak(device, ctypes.byref(t), ctypes.byref(g)))
    return t.value, g.value


def cst_tune_opts_default() -> cst_tune_opts:
    o = cst_tune_opts()
    _lib.cst_tune_opts_default(ctypes.byref(o))
    return o


def _eval_cb(eval_fn, nm):
    if eval_fn is None:
        return EVAL_FN()

    def _cb(user, settings, n, ms, metrics):
        try:
            res = eval_fn([settings[i] for i in range(n)])
            times, mets = (res if nm > 0 else (res, None))
            for i in range(n):
                ms[i] = float(times[i])
                for k in range(nm):
                    metrics[i * nm + k] = float(mets[i][k])
            return 0
        except Exception:
            import traceback
            traceback.print_exc()
            return 1
    return EVAL_FN(_cb)


def cst_dist_create_host(h, nranks: int, rank: int, bcast, allgather):
    """Tuning-only cst_dist whose collectives are Python callables:
    bcast(bytearray-like memoryview, root) in place; allgather(bytes) -> bytes (rank order).
    Returns (handle, keepalive) — keep the second object alive with the handle."""
    def _b(user, buf, nbytes, root):
        try:
            mv = (ctypes.c_char * nbytes).from_address(buf)
            out = bcast(bytes(mv), root)
            ctypes.memmove(buf, out, nbytes)
            return 0
        except Exception:
            import traceback
            traceback.print_exc()
            return 1

    def _g(user, send, recv, nbytes):
        try:
            data = allgather(ctypes.string_at(send, nbytes))
            assert len(data) == nbytes * nranks
            ctypes.memmove(recv, data, len(data))
            return 0
        except Exception:
            import traceback
            traceback.print_exc()
            return 1

    coll = cst_collectives(None, BCAST_FN(_b), ALLGATHER_FN(_g))
    d = ctypes.c_void_p()
    check(_lib.cst_dist_create_host(h, nranks, rank, ctypes.byref(coll), ctypes.byref(d)))
    return d, (coll, _b, _g)


def cst_dist_tune(d, opts: cst_tune_opts, in_ptrs, scratch_out_ptrs, local_eval=None):
    """Collective population-parallel cst_tune (include/cst.h).  local_eval: as cst_tune's
    eval_fn, for this rank's share only (None = built-in GPU timing on in/scratch_out)."""
    pi, _a = _ptrs(in_ptrs)
    po, _b = _ptrs(scratch_out_ptrs)
    best, rep = cst_setting(), cst_tune_report()
    cb = _eval_cb(local_eval, opts.n_user_metrics)
    check(_lib.cst_dist_tune(d, ctypes.byref(opts), pi, po, cb, None, ctypes.byref(best),
                             ctypes.byref(rep)))
    return best, rep


def cst_tune(h, opts: cst_tune_opts, in_ptrs, scratch_out_ptrs, eval_fn=None):
    """eval_fn(list[cst_setting]) -> list[float ms], or (ms list, metrics rows) when
    opts.n_user_metrics > 0 (optional: population-parallel / synthetic evaluation)."""
    pi, _a = _ptrs(in_ptrs)
    po, _b = _ptrs(scratch_out_ptrs)
    best, rep = cst_setting(), cst_tune_report()
    if eval_fn is not None:
        nm = opts.n_user_metrics

        def _cb(user, settings, n, ms, metrics):
            try:
                res = eval_fn([settings[i] for i in range(n)])
                times, mets = (res if nm > 0 else (res, None))
                for i in range(n):
                    ms[i] = float(times[i])
                    for k in range(nm):
                        metrics[i * nm + k] = float(mets[i][k])
                return 0
            except Exception:
                import traceback
                traceback.print_exc()
                return 1
        cb = EVAL_FN(_cb)
    else:
        cb = EVAL_FN()
    check(_lib.cst_tune(h, ctypes.byref(opts), pi, po, cb, None, ctypes.byref(best),
                        ctypes.byref(rep)))
    return best, rep


def cst_dist_halo_plan(nranks: int, rank: int, nz: int, r: int):
    """[(peer, is_send, plane_begin, nplanes), ...] of this rank's halo exchange."""
    xs = (cst_halo_xfer * 4)()
    n = ctypes.c_int32()
    check(_lib.cst_dist_halo_plan(nranks, rank, nz, r, xs, ctypes.byref(n)))
    return [(x.peer, x.is_send, x.plane_begin, x.nplanes) for x in xs[:n.value]]


def cst_dist_nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    check(_lib.cst_dist_nccl_unique_id(buf))
    return buf.raw


def cst_dist_create(h, nranks: int, rank: int, unique_id: bytes | None):
    d = ctypes.c_void_p()
    uid = None if unique_id is None else ctypes.create_string_buffer(unique_id, 128)
    check(_lib.cst_dist_create(h, nranks, rank, uid, ctypes.byref(d)))
    return d


def cst_dist_sweep(d, s: cst_setting, in_ptrs, out_ptrs, nsteps: int = 1, stream: int = 0):
    pi, _a = _ptrs(in_ptrs)
    po, _b = _ptrs(out_ptrs)
    check(_lib.cst_dist_sweep(d, ctypes.byref(s), pi, po, nsteps, ctypes.c_void_p(stream)))


def cst_dist_sweep_loopback(h, nslabs: int, s: cst_setting, in_ptrs, out_ptrs, nsteps: int = 1,
                            stream: int = 0):
    pi, _a = _ptrs(in_ptrs)
    po, _b = _ptrs(out_ptrs)
    check(_lib.cst_dist_sweep_loopback(h, nslabs, ctypes.byref(s), pi, po, nsteps,
                                       ctypes.c_void_p(stream)))


def cst_dist_destroy(d) -> None:
    _lib.cst_dist_destroy(d)


def cst_dist_p2p_export(d, a_ptrs, b_ptrs) -> bytes:
    """IPC description of my ping-pong buffer sets (a, b) and flag words (peer transport)."""
    pa, _a = _ptrs(a_ptrs)
    pb, _b = _ptrs(b_ptrs)
    blob = ctypes.create_string_buffer(P2P_BLOB_BYTES)
    check(_lib.cst_dist_p2p_export(d, pa, pb, blob))
    return blob.raw


def cst_dist_p2p_import(d, peer: int, blob: bytes) -> None:
    buf = ctypes.create_string_buffer(bytes(blob), P2P_BLOB_BYTES)
    check(_lib.cst_dist_p2p_import(d, peer, buf))


def cst_dist_p2p_setup(d, rank: int, world: int, a_ptrs, b_ptrs, group=None) -> None:
    """Export my buffers, all-gather the blobs over torch.distributed (any backend), import
    both neighbours: the fused peer-memory halo transport is then ready."""
    import torch.distributed as dist
    mine = cst_dist_p2p_export(d, a_ptrs, b_ptrs)
    blobs = [None] * world
    dist.all_gather_object(blobs, mine, group=group)
    for peer in (rank - 1, rank + 1):
        if 0 <= peer < world:
            cst_dist_p2p_import(d, peer, blobs[peer])
