"""Thin ctypes binding over libdysel.so (include/dysel.h).

Argument marshalling only: every step of DySel runs inside libdysel.so.
PyTorch supplies device memory (tensors -> data_ptr), the current CUDA stream
and process groups.  There is no CPU fallback: importing this module without
the built library raises.
"""
from __future__ import annotations

import ctypes
import os
import weakref

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
# DYSEL_LIB: an experimental build of the same library (scripts/build_exp.py)
LIB_PATH = os.environ.get("DYSEL_LIB") or os.path.join(_HERE, "libdysel.so")
if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} not built: run `python -m paper_conf_asplos_changkh16_b200.build` "
                      "(or __graft_entry__.build()); there is no fallback path")
_lib = ctypes.CDLL(LIB_PATH)

# ---------------------------------------------------------------- constants
OK, ERR_INVALID, ERR_UNSUPPORTED, ERR_NOMEM, ERR_CUDA, ERR_NOT_FOUND, ERR_NCCL = range(7)
FULLY, HYBRID, SWAP, AUTO = 0, 1, 2, 3
SYNC, ASYNC = 0, 4
NO_PROFILE, HOST_ORCH, FORCE_PROFILE, CONTIGUOUS, SCORE_CYCLES = 8, 16, 32, 64, 128
SCORE_MAKESPAN, NO_ABORT, SEQUENTIAL = 256, 1024, 2048
DEFAULT_MODE = FULLY | ASYNC
V_ATOMICS, V_NONUNIFORM = 1, 2
ROLE_PRODUCTIVE, ROLE_SANDBOX, ROLE_BATCH, ROLE_PRIVATE, ROLE_EAGER = range(5)
MAX_VARIANTS = 16
SPMV_CSR_SCALAR, SPMV_CSR_VECTOR, SPMV_ELL, SPMV_JDS, SPMV_CSR_STREAM, SPMV_CSR_TMA = range(6)
SPMV_NVARIANTS = 6
SPMV_NAMES = ["csr_scalar", "csr_vector", "ell", "jds", "csr_stream", "csr_tma"]
FMT_ELL, FMT_JDS, FMT_STREAM, FMT_TMA = 1, 2, 4, 8
FMT_ALL = FMT_ELL | FMT_JDS | FMT_STREAM | FMT_TMA
# default pool: CSR-T (bulk-staged data-placement variant) is opt-in
FMT_DEFAULT = FMT_ELL | FMT_JDS | FMT_STREAM
SPMV_DEFAULT_AUTO = -1
SGEMM_S64, SGEMM_S128, SGEMM_T128x64, SGEMM_T128x128 = range(4)
SGEMM_NAMES = ["simt64x64", "simt128x128", "tc3xtf32_128x64", "tc3xtf32_128x128"]
STENCIL_NAMES = ["base", "zmarch64", "tma128x8x16"]
SPMTV_NAMES = ["scatter_thread", "scatter_warp", "scatter_segment"]
STENCIL_BASE, STENCIL_ZMARCH, STENCIL_TILED = range(3)
PLACE_LDG, PLACE_L2, PLACE_SMEM, PLACE_PERSIST = range(4)
PLACE_NAMES = ["x_ldg", "x_l2", "x_smem", "x_persist"]
JDSG_PLAIN, JDSG_UNROLL, JDSG_PREFETCH, JDSG_UNROLL_PREFETCH = range(4)
JDSG_NAMES = ["jds_plain", "jds_unroll", "jds_prefetch", "jds_unroll_prefetch"]

c_void_p, c_int, c_float, c_u32, c_u64, c_i64, c_size = (ctypes.c_void_p, ctypes.c_int, ctypes.c_float,
                                                        ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int64,
                                                        ctypes.c_size_t)


class SliceRec(ctypes.Structure):
    _fields_ = [("granule_begin", c_u64), ("granule_count", c_u64), ("granule_stride", c_u64),
                ("variant", ctypes.c_int32), ("role", ctypes.c_int32)]


class Report(ctypes.Structure):
    _fields_ = [("mode_used", ctypes.c_int32), ("profiled", ctypes.c_int32), ("selected", ctypes.c_int32),
                ("n_variants", ctypes.c_int32), ("c", c_u64), ("n_granules", c_u64),
                ("score", c_u64 * MAX_VARIANTS), ("makespan_ns", c_u64 * MAX_VARIANTS),
                ("units", c_u64 * MAX_VARIANTS), ("cycles", c_u64 * MAX_VARIANTS),
                ("busy_ns", c_u64 * MAX_VARIANTS), ("aborted", c_u64 * MAX_VARIANTS), ("tail_units", c_u64),
                ("eager_units", c_u64), ("host_ns", c_u64), ("slices", ctypes.POINTER(SliceRec)),
                ("slices_cap", ctypes.c_int32), ("n_slices", ctypes.c_int32),
                ("unit_variant", ctypes.POINTER(ctypes.c_uint8)), ("unit_variant_cap", c_u64),
                ("timeline_ns", c_u64 * 8), ("sandbox_buffers", c_u32), ("pad_", c_u32), ("sandbox_bytes", c_u64)]


class PlanInfo(ctypes.Structure):
    _fields_ = [("n_rows", c_i64), ("n_cols", c_i64), ("nnz", c_i64), ("n_variants", ctypes.c_int32),
                ("variant_ids", ctypes.c_int32 * SPMV_NVARIANTS), ("ell_width", ctypes.c_int32), ("uniform", ctypes.c_int32),
                ("max_row_len", ctypes.c_int32), ("prep_ns", c_u64), ("ell_bytes", c_u64), ("jds_bytes", c_u64),
                ("default_variant", ctypes.c_int32), ("n_heavy", ctypes.c_int32), ("n_light", ctypes.c_int32)]


def _sig(name, res, *args):
    f = getattr(_lib, name)
    f.restype = res
    f.argtypes = list(args)
    return f


P = c_void_p
dysel_status_str = _sig("dysel_status_str", ctypes.c_char_p, c_int)
dysel_create = _sig("dysel_create", c_int, c_int, ctypes.POINTER(c_void_p))
dysel_destroy = _sig("dysel_destroy", None, P)
dysel_last_error = _sig("dysel_last_error", ctypes.c_char_p, P)
dysel_device_info = _sig("dysel_device_info", c_int, P, ctypes.POINTER(c_int), ctypes.POINTER(c_u64),
                         ctypes.POINTER(c_u64))
dysel_register_variants = _sig("dysel_register_variants", c_int, P, ctypes.c_char_p, P, c_int, c_int)
dysel_launch = _sig("dysel_launch", c_int, P, ctypes.c_char_p, ctypes.POINTER(c_u64), c_float, c_u32,
                    ctypes.POINTER(c_void_p), c_int, ctypes.POINTER(c_size), P, ctypes.POINTER(Report))
dysel_get_selection = _sig("dysel_get_selection", c_int, P, ctypes.c_char_p, ctypes.POINTER(c_int))
dysel_set_selection = _sig("dysel_set_selection", c_int, P, ctypes.c_char_p, c_int)
dysel_reset_selection = _sig("dysel_reset_selection", c_int, P, ctypes.c_char_p)
dysel_spmv_prepare = _sig("dysel_spmv_prepare", c_int, P, c_i64, c_i64, c_i64, P, P, P, c_u32, c_int, P,
                          ctypes.POINTER(c_void_p))
dysel_spmv_plan_get_info = _sig("dysel_spmv_plan_get_info", c_int, P, ctypes.POINTER(PlanInfo))
dysel_spmv_plan_destroy = _sig("dysel_spmv_plan_destroy", None, P)
dysel_spmv_plan_copy_array = _sig("dysel_spmv_plan_copy_array", c_int, P, c_int, P, ctypes.POINTER(c_size))
dysel_spmv = _sig("dysel_spmv", c_int, P, P, P, P, c_float, c_u32, P, ctypes.POINTER(Report))
dysel_spmv_host = _sig("dysel_spmv_host", c_int, P, P, P, P, P, P, c_float, c_u32, P, ctypes.POINTER(Report))
dysel_spmv_variant = _sig("dysel_spmv_variant", c_int, P, P, c_int, P, P, P)
dysel_spmv_gather_probe = _sig("dysel_spmv_gather_probe", c_int, P, P, c_int, P, P, P)
dysel_sgemm = _sig("dysel_sgemm", c_int, P, c_int, c_int, c_int, c_float, P, c_int, P, c_int, c_float, P, c_int,
                   c_float, c_u32, P, ctypes.POINTER(Report))
dysel_sgemm_variant = _sig("dysel_sgemm_variant", c_int, P, c_int, c_int, c_int, c_int, c_float, P, c_int, P, c_int,
                           c_float, P, c_int, P)
dysel_comm_unique_id = _sig("dysel_comm_unique_id", c_int, P)
dysel_comm_init = _sig("dysel_comm_init", c_int, P, P, c_int, c_int)
dysel_partition_rows = _sig("dysel_partition_rows", c_int, P, c_i64, c_int, P)
dysel_allgather_chunk = _sig("dysel_allgather_chunk", c_int, c_i64, c_int, P, P)
dysel_spmv_sharded = _sig("dysel_spmv_sharded", c_int, P, P, P, P, P, c_float, c_u32, P, ctypes.POINTER(Report))
dysel_stencil = _sig("dysel_stencil", c_int, P, c_int, c_int, c_int, c_float, c_float, P, P, c_float, c_u32, P,
                     ctypes.POINTER(Report))
dysel_spmtv = _sig("dysel_spmtv", c_int, P, P, P, P, c_float, c_u32, P, ctypes.POINTER(Report))
dysel_spmtv_variant = _sig("dysel_spmtv_variant", c_int, P, P, c_int, P, P, P)
dysel_stencil_variant = _sig("dysel_stencil_variant", c_int, P, c_int, c_int, c_int, c_int, c_float, c_float, P, P, P)
dysel_spmv_power = _sig("dysel_spmv_power", c_int, P, P, P, P, c_int, c_int, c_float, c_u32, P, P,
                        ctypes.POINTER(Report))
dysel_spmv_power_sharded = _sig("dysel_spmv_power_sharded", c_int, P, P, P, P, P, c_i64, c_int, c_int, c_float, c_u32,
                                P, P, ctypes.POINTER(Report))
dysel_comm_broadcast = _sig("dysel_comm_broadcast", c_int, P, P, c_size, c_int, P)
dysel_sgemm_sharded = _sig("dysel_sgemm_sharded", c_int, P, c_int, c_int, c_int, c_float, P, c_int, P, c_int, c_float,
                           P, c_int, c_float, c_u32, P, ctypes.POINTER(Report))
dysel_sgemm_shard_rows = _sig("dysel_sgemm_shard_rows", c_int, c_int, c_int, c_int, ctypes.POINTER(c_int),
                              ctypes.POINTER(c_int))
dysel_spmv_sharded_loopback = _sig("dysel_spmv_sharded_loopback", c_int, P, c_int, ctypes.POINTER(c_void_p), P, P, P,
                                   c_float, c_u32, P, P)
dysel_spmv_placement = _sig("dysel_spmv_placement", c_int, P, P, P, P, c_float, c_u32, P, ctypes.POINTER(Report))
dysel_spmv_placement_variant = _sig("dysel_spmv_placement_variant", c_int, P, P, c_int, P, P, P)
dysel_spmv_placement_windows = _sig("dysel_spmv_placement_windows", c_int, P, P, c_size)
dysel_spmv_jds_prepare = _sig("dysel_spmv_jds_prepare", c_int, P, c_i64, c_i64, c_i64, P, P, P, P,
                              ctypes.POINTER(c_void_p))
dysel_spmv_jds = _sig("dysel_spmv_jds", c_int, P, P, P, P, c_float, c_u32, P, ctypes.POINTER(Report))
dysel_spmv_jds_variant = _sig("dysel_spmv_jds_variant", c_int, P, P, c_int, P, P, P)
dysel_spmv_jds_copy_array = _sig("dysel_spmv_jds_copy_array", c_int, P, c_int, P, ctypes.POINTER(c_size))
dysel_spmv_jds_plan_destroy = _sig("dysel_spmv_jds_plan_destroy", None, P)
dysel_kernel_launches = _sig("dysel_kernel_launches", c_u64, P)
dysel_timer_calibrate = _sig("dysel_timer_calibrate", c_int, P, c_u64, c_u64, ctypes.POINTER(c_u64),
                             ctypes.POINTER(ctypes.c_double))
dysel_register_spin_variants = _sig("dysel_register_spin_variants", c_int, P, ctypes.c_char_p,
                                    ctypes.POINTER(c_u32), c_int, c_int)

EXPORTS = [n for n in dir() if n.startswith("dysel_")]


class DyselError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{dysel_status_str(status).decode()}: {msg}")
        self.status = status


def _hptr(t):
    """Host pointer of a CPU tensor (pinned for asynchronous copies)."""
    if not isinstance(t, torch.Tensor) or t.is_cuda:
        raise ValueError("host tensor expected")
    if not t.is_contiguous():
        raise ValueError("contiguous host tensor expected")
    return ctypes.c_void_p(t.data_ptr())


def _ptr(t):
    if t is None:
        return None
    if isinstance(t, torch.Tensor):
        if not t.is_cuda:
            raise ValueError("device tensor expected (libdysel takes device pointers)")
        return ctypes.c_void_p(t.data_ptr())
    return t


def _stream(stream):
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def report_dict(rep: Report, names=None, uv=None):
    K = rep.n_variants
    d = dict(mode_used=rep.mode_used, profiled=bool(rep.profiled), selected=rep.selected, n_variants=K,
             c=rep.c, n_granules=rep.n_granules, eager_units=rep.eager_units, host_ns=rep.host_ns,
             score=list(rep.score[:MAX_VARIANTS]), makespan_ns=list(rep.makespan_ns[:MAX_VARIANTS]),
             units=list(rep.units[:MAX_VARIANTS]), cycles=list(rep.cycles[:MAX_VARIANTS]),
             busy_ns=list(rep.busy_ns[:MAX_VARIANTS]), aborted=list(rep.aborted[:MAX_VARIANTS]),
             tail_units=rep.tail_units, n_slices=rep.n_slices, sandbox_buffers=rep.sandbox_buffers,
             sandbox_bytes=rep.sandbox_bytes,
             timeline_ns=[None if t == 2 ** 64 - 1 else int(t) for t in rep.timeline_ns])
    if rep.slices and rep.slices_cap:
        d["slices"] = [dict(begin=rep.slices[i].granule_begin, count=rep.slices[i].granule_count,
                            stride=rep.slices[i].granule_stride, variant=rep.slices[i].variant,
                            role=rep.slices[i].role) for i in range(min(rep.n_slices, rep.slices_cap))]
    if uv is not None:
        d["unit_variant"] = uv
    if names:
        d["selected_name"] = names[rep.selected] if 0 <= rep.selected < len(names) else None
    return d


def _make_report(unit_cap=0, slices_cap=64):
    rep = Report()
    sl = (SliceRec * slices_cap)()
    rep.slices = ctypes.cast(sl, ctypes.POINTER(SliceRec))
    rep.slices_cap = slices_cap
    uv = None
    if unit_cap:
        uv = (ctypes.c_uint8 * unit_cap)()
        rep.unit_variant = ctypes.cast(uv, ctypes.POINTER(ctypes.c_uint8))
        rep.unit_variant_cap = unit_cap
    return rep, sl, uv


class SpmvPlan:
    def __init__(self, ctx, handle, tensors):
        self.ctx = ctx
        self.handle = handle
        self._keep = tensors   # the plan holds non-owning CSR pointers
        info = PlanInfo()
        ctx._check(dysel_spmv_plan_get_info(handle, ctypes.byref(info)))
        self.info = info
        self.variant_ids = list(info.variant_ids[:info.n_variants])
        self.n_units = (info.n_rows + 255) // 256

    _ARRAYS = {"ell_col": (0, "int32"), "ell_val": (1, "float32"), "perm": (2, "int32"), "jds_len": (3, "int32"),
               "blk_off": (4, "int64"), "jd_off": (5, "int64"), "jd_ptr": (6, "int32"), "jds_col": (7, "int32"),
               "jds_val": (8, "float32"), "seq": (9, "int32")}

    def array(self, name):
        """Copy a format array of the plan to a host numpy array (tests)."""
        import numpy as np
        which, dt = self._ARRAYS[name]
        n = c_size(0)
        st = dysel_spmv_plan_copy_array(self.handle, which, None, ctypes.byref(n))
        if st == ERR_NOT_FOUND:
            return None
        self.ctx._check(st)
        out = np.empty(n.value // np.dtype(dt).itemsize, dt)
        self.ctx._check(dysel_spmv_plan_copy_array(self.handle, which, out.ctypes.data_as(c_void_p),
                                                   ctypes.byref(n)))
        return out

    def destroy(self):
        # a plan must die before its context (it unregisters from it)
        if self.handle and self.ctx is not None and self.ctx.h:
            dysel_spmv_plan_destroy(self.handle)
        self.handle = None

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass


class JdsPlan:
    """Global-sort JDS pool of one matrix (dysel_spmv_jds_plan, f-2 Case III)."""
    _ARRAYS = {"perm": (0, "int32"), "len": (1, "int32"), "jd_ptr": (2, "int32"), "col": (3, "int32"),
               "val": (4, "float32")}

    def __init__(self, ctx, handle, n_rows):
        self.ctx, self.handle, self.n_rows = ctx, handle, n_rows
        self.n_units = (n_rows + 255) // 256

    def array(self, name):
        import numpy as np
        which, dt = self._ARRAYS[name]
        n = c_size(0)
        self.ctx._check(dysel_spmv_jds_copy_array(self.handle, which, None, ctypes.byref(n)))
        out = np.empty(n.value // np.dtype(dt).itemsize, dt)
        self.ctx._check(dysel_spmv_jds_copy_array(self.handle, which, out.ctypes.data_as(c_void_p), ctypes.byref(n)))
        return out

    def destroy(self):
        if self.handle and self.ctx is not None and self.ctx.h:
            dysel_spmv_jds_plan_destroy(self.handle)
        self.handle = None

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass


class Context:
    """dysel_ctx on one CUDA device."""

    def __init__(self, device: int = 0):
        h = ctypes.c_void_p()
        torch.cuda.init()
        st = dysel_create(int(device), ctypes.byref(h))
        if st != OK:
            raise DyselError(st, "dysel_create failed")
        self.h = h
        self.device = device
        self._plans = weakref.WeakSet()
        n_sm, tick, l2 = c_int(), c_u64(), c_u64()
        dysel_device_info(h, ctypes.byref(n_sm), ctypes.byref(tick), ctypes.byref(l2))
        self.n_sm, self.globaltimer_tick_ns, self.l2_bytes = n_sm.value, tick.value, l2.value
        self.rank, self.world = 0, 1

    def _check(self, st):
        if st != OK:
            raise DyselError(st, dysel_last_error(self.h).decode())

    def close(self):
        for p in list(self._plans):
            p.destroy()
        if self.h:
            dysel_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def kernel_launches(self) -> int:
        return int(dysel_kernel_launches(self.h))

    # ------------------------------------------------------------- SpMV
    def spmv_prepare(self, row_ptr, col, val, n_cols, formats=FMT_DEFAULT, default=SPMV_CSR_VECTOR,
                     stream=None) -> SpmvPlan:
        n = row_ptr.numel() - 1
        nnz = col.numel()
        assert row_ptr.dtype == torch.int32 and col.dtype == torch.int32 and val.dtype == torch.float32
        h = ctypes.c_void_p()
        self._check(dysel_spmv_prepare(self.h, n, int(n_cols), nnz, _ptr(row_ptr), _ptr(col), _ptr(val),
                                       formats, default, _stream(stream), ctypes.byref(h)))
        plan = SpmvPlan(self, h, (row_ptr, col, val))
        self._plans.add(plan)
        return plan

    def spmv(self, plan, x, y, f=0.02, mode=DEFAULT_MODE, report=False, unit_map=False, stream=None):
        rep, keep, uv = (_make_report(plan.n_units if unit_map else 0) if report else (None, None, None))
        self._check(dysel_spmv(self.h, plan.handle, _ptr(x), _ptr(y), float(f), int(mode), _stream(stream),
                               ctypes.byref(rep) if rep is not None else None))
        if rep is None:
            return None
        return report_dict(rep, SPMV_NAMES, bytes(uv) if uv is not None else None)

    def spmv_host(self, plan, h_x, h_y, d_x, d_y, f=0.02, mode=DEFAULT_MODE, report=False, stream=None):
        """dysel_spmv_host: pinned host x in, host y out (chunked copy-out overlapped with the SpMV);
        d_x / d_y are the device staging buffers.  Stream-ordered: h_y is valid once `stream` is done."""
        rep, keep, uv = (_make_report(0) if report else (None, None, None))
        self._check(dysel_spmv_host(self.h, plan.handle, _hptr(h_x), _hptr(h_y), _ptr(d_x), _ptr(d_y), float(f),
                                    int(mode), _stream(stream), ctypes.byref(rep) if rep is not None else None))
        if rep is None:
            return None
        return report_dict(rep, SPMV_NAMES, None)

    def spmv_power(self, plan, x, y, n_iter, profile_every=0, f=0.02, mode=DEFAULT_MODE, norms=None, report=False,
                   stream=None):
        """Power iteration x <- A x / ||A x|| (dysel_spmv_power); x in/out, y = A x of the last iteration,
        norms: optional device float64 [n_iter] receiving ||A x_k||."""
        rep, keep, uv = (_make_report(0) if report else (None, None, None))
        self._check(dysel_spmv_power(self.h, plan.handle, _ptr(x), _ptr(y), int(n_iter), int(profile_every), float(f),
                                     int(mode), _stream(stream), _ptr(norms) if norms is not None else None,
                                     ctypes.byref(rep) if rep is not None else None))
        return report_dict(rep, SPMV_NAMES) if rep is not None else None

    def spmv_variant(self, plan, variant_id, x, y, stream=None):
        self._check(dysel_spmv_variant(self.h, plan.handle, int(variant_id), _ptr(x), _ptr(y), _stream(stream)))

    def spmtv(self, plan, x, y, f=0.02, mode=AUTO, report=False, unit_map=False, stream=None):
        """y += A^T x through the atomic scatter pool (dysel_spmtv; AUTO -> swap mode; ASYNC only on
        the additive device swap, not with HOST_ORCH: include/dysel.h, DESIGN A-47b)."""
        rep, keep, uv = (_make_report(plan.n_units if unit_map else 0) if report else (None, None, None))
        self._check(dysel_spmtv(self.h, plan.handle, _ptr(x), _ptr(y), float(f), int(mode), _stream(stream),
                                ctypes.byref(rep) if rep is not None else None))
        if rep is None:
            return None
        return report_dict(rep, SPMTV_NAMES, bytes(uv) if uv is not None else None)

    def spmtv_variant(self, plan, variant_id, x, y, stream=None):
        self._check(dysel_spmtv_variant(self.h, plan.handle, int(variant_id), _ptr(x), _ptr(y), _stream(stream)))

    def spmv_gather_probe(self, plan, flavour, x, out, stream=None):
        """Measurement only: the plan's CSR traffic with no row structure (include/dysel.h)."""
        self._check(dysel_spmv_gather_probe(self.h, plan.handle, int(flavour), _ptr(x), _ptr(out), _stream(stream)))

    # ----------------------------------------------------- SpMV f-2 pools
    def spmv_placement(self, plan, x, y, f=0.02, mode=DEFAULT_MODE, report=False, unit_map=False, stream=None):
        """y = A x through the x data-placement pool (Case II, f-2)."""
        rep, keep, uv = (_make_report(plan.n_units if unit_map else 0) if report else (None, None, None))
        self._check(dysel_spmv_placement(self.h, plan.handle, _ptr(x), _ptr(y), float(f), int(mode), _stream(stream),
                                         ctypes.byref(rep) if rep is not None else None))
        if rep is None:
            return None
        return report_dict(rep, PLACE_NAMES, bytes(uv) if uv is not None else None)

    def spmv_placement_variant(self, plan, variant_id, x, y, stream=None):
        self._check(dysel_spmv_placement_variant(self.h, plan.handle, int(variant_id), _ptr(x), _ptr(y),
                                                 _stream(stream)))

    def spmv_placement_windows(self, plan):
        import numpy as np
        out = np.empty((plan.n_units, 2), np.int32)
        st = dysel_spmv_placement_windows(plan.handle, out.ctypes.data_as(c_void_p), plan.n_units)
        if st == ERR_NOT_FOUND:
            return None
        self._check(st)
        return out

    def spmv_jds_prepare(self, row_ptr, col, val, n_cols, stream=None) -> JdsPlan:
        n = row_ptr.numel() - 1
        h = ctypes.c_void_p()
        self._check(dysel_spmv_jds_prepare(self.h, n, int(n_cols), col.numel(), _ptr(row_ptr), _ptr(col), _ptr(val),
                                           _stream(stream), ctypes.byref(h)))
        plan = JdsPlan(self, h, n)
        self._plans.add(plan)
        return plan

    def spmv_jds(self, plan, x, y, f=0.02, mode=DEFAULT_MODE, report=False, unit_map=False, stream=None):
        """y = A x through the global-sort JDS pool (Case III, f-2)."""
        rep, keep, uv = (_make_report(plan.n_units if unit_map else 0) if report else (None, None, None))
        self._check(dysel_spmv_jds(self.h, plan.handle, _ptr(x), _ptr(y), float(f), int(mode), _stream(stream),
                                   ctypes.byref(rep) if rep is not None else None))
        if rep is None:
            return None
        return report_dict(rep, JDSG_NAMES, bytes(uv) if uv is not None else None)

    def spmv_jds_variant(self, plan, variant_id, x, y, stream=None):
        self._check(dysel_spmv_jds_variant(self.h, plan.handle, int(variant_id), _ptr(x), _ptr(y), _stream(stream)))

    # ------------------------------------------------------------ SGEMM
    def sgemm(self, A, B, C, alpha=1.0, beta=0.0, f=0.02, mode=DEFAULT_MODE, report=False, unit_map=False,
              stream=None):
        M, K = A.shape
        N = B.shape[1]
        G = ((N + 31) // 32 + 3) // 4 * (((M + 31) // 32 + 3) // 4)
        rep, keep, uv = (_make_report(G if unit_map else 0) if report else (None, None, None))
        self._check(dysel_sgemm(self.h, M, N, K, float(alpha), _ptr(A), A.stride(0), _ptr(B), B.stride(0),
                                float(beta), _ptr(C), C.stride(0), float(f), int(mode), _stream(stream),
                                ctypes.byref(rep) if rep is not None else None))
        if rep is None:
            return None
        return report_dict(rep, SGEMM_NAMES, bytes(uv) if uv is not None else None)

    def sgemm_variant(self, variant_id, A, B, C, alpha=1.0, beta=0.0, stream=None):
        M, K = A.shape
        N = B.shape[1]
        self._check(dysel_sgemm_variant(self.h, int(variant_id), M, N, K, float(alpha), _ptr(A), A.stride(0),
                                        _ptr(B), B.stride(0), float(beta), _ptr(C), C.stride(0), _stream(stream)))

    # ---------------------------------------------------------- generic
    def register_spin_variants(self, sig, costs_ns, default=0):
        arr = (c_u32 * len(costs_ns))(*costs_ns)
        self._check(dysel_register_spin_variants(self.h, sig.encode(), arr, len(costs_ns), default))

    def launch(self, sig, ndrange, args, f=0.02, mode=DEFAULT_MODE, sandbox_bytes=None, report=False,
               unit_map=0, stream=None):
        U = (c_u64 * 3)(*(list(ndrange) + [1] * (3 - len(ndrange))))
        a = (c_void_p * max(1, len(args)))(*[(_ptr(t).value if isinstance(t, torch.Tensor) else t) for t in args])
        sb = (c_size * max(1, len(sandbox_bytes or [])))(*(sandbox_bytes or []))
        rep, keep, uv = (_make_report(unit_map) if report else (None, None, None))
        self._check(dysel_launch(self.h, sig.encode(), U, float(f), int(mode), a, len(args),
                                 sb if sandbox_bytes else None, _stream(stream),
                                 ctypes.byref(rep) if rep is not None else None))
        if rep is None:
            return None
        return report_dict(rep, None, bytes(uv) if uv is not None else None)

    def get_selection(self, key):
        v = c_int()
        st = dysel_get_selection(self.h, key.encode(), ctypes.byref(v))
        if st == ERR_NOT_FOUND:
            return None
        self._check(st)
        return v.value

    def set_selection(self, key, v):
        self._check(dysel_set_selection(self.h, key.encode(), int(v)))

    def reset_selection(self, key=None):
        self._check(dysel_reset_selection(self.h, key.encode() if key else None))

    def timer_calibrate(self, samples=1 << 20, spin_ns=200000):
        t, c = c_u64(), ctypes.c_double()
        self._check(dysel_timer_calibrate(self.h, samples, spin_ns, ctypes.byref(t), ctypes.byref(c)))
        return t.value, c.value

    # ------------------------------------------------------------ stencil
    def stencil(self, inp, out, c0, c1, f=0.02, mode=DEFAULT_MODE, report=False, unit_map=False, stream=None):
        """One 7-point Jacobi step out = c1 * (6-neighbour sum) - c0 * in (boundary copied); inp/out [nz, ny, nx]."""
        nz, ny, nx = inp.shape
        G = ((nx + 31) // 32 + 1) // 2 * ((ny + 3) // 4) * ((nz + 63) // 64)
        rep, keep, uv = (_make_report(G if unit_map else 0) if report else (None, None, None))
        self._check(dysel_stencil(self.h, nx, ny, nz, float(c0), float(c1), _ptr(inp), _ptr(out), float(f), int(mode),
                                  _stream(stream), ctypes.byref(rep) if rep is not None else None))
        if rep is None:
            return None
        return report_dict(rep, STENCIL_NAMES, bytes(uv) if uv is not None else None)

    def stencil_variant(self, variant_id, inp, out, c0, c1, stream=None):
        nz, ny, nx = inp.shape
        self._check(dysel_stencil_variant(self.h, int(variant_id), nx, ny, nz, float(c0), float(c1), _ptr(inp),
                                          _ptr(out), _stream(stream)))

    # -------------------------------------------------------- multi-GPU
    def comm_init(self, rank, world, uid: bytes):
        buf = ctypes.create_string_buffer(uid, 128)
        self._check(dysel_comm_init(self.h, buf, int(rank), int(world)))
        self.rank, self.world = int(rank), int(world)

    def spmv_sharded(self, local_plan, bounds, x, y, f=0.02, mode=DEFAULT_MODE, report=False, stream=None):
        b = (c_i64 * len(bounds))(*bounds)
        rep, keep, uv = (_make_report(0) if report else (None, None, None))
        self._check(dysel_spmv_sharded(self.h, local_plan.handle, b, _ptr(x), _ptr(y), float(f), int(mode),
                                       _stream(stream), ctypes.byref(rep) if rep is not None else None))
        return report_dict(rep, SPMV_NAMES) if rep is not None else None

    def spmv_power_sharded(self, local_plan, bounds, x, y, n_iter, profile_every=0, f=0.02, mode=DEFAULT_MODE,
                           norms=None, report=False, stream=None):
        b = (c_i64 * len(bounds))(*bounds)
        rep, keep, uv = (_make_report(0) if report else (None, None, None))
        self._check(dysel_spmv_power_sharded(self.h, local_plan.handle, b, _ptr(x), _ptr(y), int(bounds[-1]),
                                             int(n_iter), int(profile_every), float(f), int(mode), _stream(stream),
                                             _ptr(norms) if norms is not None else None,
                                             ctypes.byref(rep) if rep is not None else None))
        return report_dict(rep, SPMV_NAMES) if rep is not None else None

    def sgemm_sharded(self, A_local, B, C, alpha=1.0, beta=0.0, f=0.02, mode=DEFAULT_MODE, report=False,
                      stream=None):
        """C (full M x N on every rank) with rows [m0, m1) = alpha A_local B + beta C there, then allgathered;
        A_local = this rank's rows of A only (see sgemm_shard_rows)."""
        M, N = C.shape
        K = B.shape[0]
        m0, m1 = sgemm_shard_rows(M, self.world, self.rank)
        assert A_local.shape[0] == m1 - m0 and A_local.shape[1] == K
        rep, keep, uv = (_make_report(0) if report else (None, None, None))
        self._check(dysel_sgemm_sharded(self.h, M, N, K, float(alpha), _ptr(A_local), max(1, A_local.stride(0)),
                                        _ptr(B), B.stride(0), float(beta), _ptr(C), C.stride(0), float(f), int(mode),
                                        _stream(stream), ctypes.byref(rep) if rep is not None else None))
        return report_dict(rep, SGEMM_NAMES) if rep is not None else None

    def spmv_sharded_loopback(self, plans, bounds, x, y, f=0.02, mode=DEFAULT_MODE, report=False, stream=None):
        """1-GPU loopback of the row-sharded SpMV: plans[g] = shard g's plan (rebased row_ptr); y full length."""
        G = len(plans)
        arr = (c_void_p * G)(*[p.handle for p in plans])
        b = (c_i64 * len(bounds))(*bounds)
        reps = (Report * G)() if report else None
        self._check(dysel_spmv_sharded_loopback(self.h, G, arr, b, _ptr(x), _ptr(y), float(f), int(mode),
                                                _stream(stream), ctypes.cast(reps, c_void_p) if reps is not None else None))
        return [report_dict(reps[g], SPMV_NAMES) for g in range(G)] if reps is not None else None

    def comm_broadcast(self, t, root, stream=None):
        self._check(dysel_comm_broadcast(self.h, _ptr(t), t.numel(), int(root), _stream(stream)))


def comm_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    st = dysel_comm_unique_id(buf)
    if st != OK:
        raise DyselError(st, "ncclGetUniqueId failed")
    return buf.raw


def sgemm_shard_rows(M, world, rank):
    a, b = c_int(), c_int()
    st = dysel_sgemm_shard_rows(int(M), int(world), int(rank), ctypes.byref(a), ctypes.byref(b))
    if st != OK:
        raise DyselError(st, "dysel_sgemm_shard_rows")
    return a.value, b.value


def allgather_chunk(rows, k):
    """Rows [begin, end) of chunk k of a shard in the overlapped allgather."""
    a, e = c_i64(0), c_i64(0)
    st = dysel_allgather_chunk(int(rows), int(k), ctypes.byref(a), ctypes.byref(e))
    if st != OK:
        raise DyselError(st, "dysel_allgather_chunk")
    return a.value, e.value


def partition_rows(row_ptr_host, world):
    import numpy as np
    rp = np.ascontiguousarray(row_ptr_host, np.int32)
    out = (c_i64 * (world + 1))()
    st = dysel_partition_rows(rp.ctypes.data_as(c_void_p), rp.shape[0] - 1, int(world), out)
    if st != OK:
        raise DyselError(st, "dysel_partition_rows")
    return list(out)
