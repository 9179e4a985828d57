"""paper_conf_ipps_sandesm11_b200 -- B200-native CUDAlign 2.0 Stage 1.

Thin ctypes binding (argument marshalling only) over the C ABI declared in
``include/cudalign_b200.h`` and implemented by ``libcudalign_b200.so``
(csrc/sw_api.cu, csrc/sw_fill.cuh).  Every step of the path runs in the
library's sm_100a kernels; there is no CPU fallback -- if the shared library
is missing or no CUDA device is usable, the calls raise.

Paper: Sandes & de Melo, "Smith-Waterman Alignment of Huge Sequences with GPU
in Linear Space", IPDPS 2011 (``P:<line>`` = /root/reference/PAPER.md).
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

from . import build as _build

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SWB_LIB") or os.path.join(_HERE, "libcudalign_b200.so")

SW_OK = 0
SW_EINVAL = -1
SW_EALPHABET = -2
SW_ERANGE = -3
SW_ENOMEM = -4
SW_ECUDA = -5
SW_EABORTED = -6
SW_ENOTFOUND = -7

EXPORTED = [
    "sw_init",
    "sw_align_stage1",
    "sw_align_stage1_dev",
    "sw_reverse_goal",
    "sw_reverse_goal_dev",
    "sw_stage2",
    "sw_stage2_dev",
    "sw_align",
    "sw_row_granularity",
    "sw_band_height",
    "sw_set_kernel",
    "sw_set_patch",
    "sw_set_virtual_stripes",
    "sw_set_grid",
    "sw_set_tail",
    "sw_set_row_budget",
    "sw_set_multi_gpu",
    "sw_device_count",
    "sw_combine_best",
    "sw_stripe_epoch",
    "sw_plan",
    "sw_cyclic_export",
    "sw_cyclic_connect",
    "sw_cyclic_epoch",
    "sw_align_stage1_cyclic",
    "sw_stripe_export",
    "sw_stripe_connect",
    "sw_align_stage1_stripe",
    "sw_special_row_interval_for_budget",
    "sw_get_stats",
    "sw_shutdown",
    "sw_strerror",
    "sw_last_error",
]


class SwError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{msg} (code {code})")
        self.code = code


class _Result(ctypes.Structure):
    _fields_ = [("score", ctypes.c_int32), ("i", ctypes.c_int64), ("j", ctypes.c_int64)]


class _Crosspoint(ctypes.Structure):
    _fields_ = [("i", ctypes.c_int64), ("j", ctypes.c_int64), ("score", ctypes.c_int32), ("type", ctypes.c_int32)]


class _Gap(ctypes.Structure):
    _fields_ = [("i", ctypes.c_int64), ("j", ctypes.c_int64), ("len", ctypes.c_int64)]


class _Alignment(ctypes.Structure):
    _fields_ = [("score", ctypes.c_int32), ("i0", ctypes.c_int64), ("j0", ctypes.c_int64), ("i1", ctypes.c_int64),
                ("j1", ctypes.c_int64), ("n_gap1", ctypes.c_int64), ("n_gap2", ctypes.c_int64),
                ("partitions", ctypes.c_int64), ("mm_levels", ctypes.c_int64), ("ms_stage1", ctypes.c_double),
                ("ms_stage2", ctypes.c_double), ("ms_mm", ctypes.c_double), ("ms_stage5", ctypes.c_double)]


class Stats(ctypes.Structure):
    _fields_ = [
        ("total_ms", ctypes.c_double),
        ("upload_ms", ctypes.c_double),
        ("encode_ms", ctypes.c_double),
        ("fill_ms", ctypes.c_double),
        ("reduce_ms", ctypes.c_double),
        ("kernel_launches", ctypes.c_int64),
        ("replays", ctypes.c_int64),
        ("special_rows", ctypes.c_int64),
        ("special_bytes_d2h", ctypes.c_int64),
        ("alpha", ctypes.c_int32),
        ("warps", ctypes.c_int32),
        ("width", ctypes.c_int32),
        ("grid", ctypes.c_int32),
        ("patched", ctypes.c_int32),
        ("devices", ctypes.c_int32),
        ("sp_slots", ctypes.c_int32),
        ("tail_alpha", ctypes.c_int32),
        ("tail_warps", ctypes.c_int32),
        ("tail_grid", ctypes.c_int32),
        ("tail_rows", ctypes.c_int64),
    ]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


SINK = ctypes.CFUNCTYPE(
    ctypes.c_int,
    ctypes.c_void_p,
    ctypes.c_int64,
    ctypes.POINTER(ctypes.c_int32),
    ctypes.POINTER(ctypes.c_int32),
    ctypes.c_int64,
)

_lib = None


def load_library(path: str = LIB_PATH):
    """Load libcudalign_b200.so (raises if it is missing: no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError(f"{path} not built; run __graft_entry__.build() or python -m paper_conf_ipps_sandesm11_b200.build")
    lib = ctypes.CDLL(path)
    i32, i64, vp, cp = ctypes.c_int32, ctypes.c_int64, ctypes.c_void_p, ctypes.c_char_p
    R = ctypes.POINTER(_Result)
    lib.sw_init.argtypes = [ctypes.POINTER(ctypes.c_int), ctypes.c_int, ctypes.POINTER(vp)]
    lib.sw_init.restype = ctypes.c_int
    lib.sw_align_stage1.argtypes = [vp, vp, i64, vp, i64, i32, i32, i32, i32, i64, SINK, vp, R]
    lib.sw_align_stage1.restype = ctypes.c_int
    lib.sw_align_stage1_dev.argtypes = [vp, vp, i64, vp, i64, i32, i32, i32, i32, i64, SINK, vp, vp, R]
    lib.sw_align_stage1_dev.restype = ctypes.c_int
    lib.sw_reverse_goal.argtypes = [vp, vp, i64, vp, i64, i32, i32, i32, i32, i32, R]
    lib.sw_reverse_goal.restype = ctypes.c_int
    lib.sw_reverse_goal_dev.argtypes = [vp, vp, i64, vp, i64, i32, i32, i32, i32, i32, vp, R]
    lib.sw_reverse_goal_dev.restype = ctypes.c_int
    CP = ctypes.POINTER(_Crosspoint)
    lib.sw_stage2.argtypes = [vp, vp, i64, vp, i64, i32, i32, i32, i32, i64, R, CP, i64, ctypes.POINTER(i64)]
    lib.sw_stage2.restype = ctypes.c_int
    lib.sw_stage2_dev.argtypes = [vp, vp, i64, vp, i64, i32, i32, i32, i32, i64, R, vp, CP, i64, ctypes.POINTER(i64)]
    lib.sw_stage2_dev.restype = ctypes.c_int
    lib.sw_align.argtypes = [vp, vp, i64, vp, i64, i32, i32, i32, i32, i64, ctypes.POINTER(_Alignment),
                             ctypes.POINTER(_Gap), i64, ctypes.POINTER(_Gap), i64]
    lib.sw_align.restype = ctypes.c_int
    lib.sw_row_granularity.argtypes = [vp]
    lib.sw_row_granularity.restype = i64
    lib.sw_band_height.argtypes = [vp]
    lib.sw_band_height.restype = i64
    lib.sw_set_kernel.argtypes = [vp, ctypes.c_int, ctypes.c_int]
    lib.sw_set_kernel.restype = ctypes.c_int
    lib.sw_set_patch.argtypes = [vp, ctypes.c_int]
    lib.sw_set_patch.restype = ctypes.c_int
    lib.sw_set_virtual_stripes.argtypes = [vp, ctypes.c_int]
    lib.sw_set_virtual_stripes.restype = ctypes.c_int
    lib.sw_set_grid.argtypes = [vp, ctypes.c_int]
    lib.sw_set_grid.restype = ctypes.c_int
    lib.sw_set_tail.argtypes = [vp, ctypes.c_int]
    lib.sw_set_tail.restype = ctypes.c_int
    lib.sw_set_row_budget.argtypes = [vp, i64]
    lib.sw_set_row_budget.restype = ctypes.c_int
    lib.sw_set_multi_gpu.argtypes = [vp, ctypes.c_int]
    lib.sw_set_multi_gpu.restype = ctypes.c_int
    lib.sw_device_count.argtypes = [vp]
    lib.sw_device_count.restype = ctypes.c_int
    lib.sw_combine_best.argtypes = [R, ctypes.c_int, R]
    lib.sw_combine_best.restype = ctypes.c_int
    lib.sw_stripe_epoch.argtypes = [vp]
    lib.sw_stripe_epoch.restype = i32
    lib.sw_plan.argtypes = [vp, i64, i64, i32, i32, i32, i32, i64, i32, ctypes.POINTER(i32), ctypes.POINTER(i32)]
    lib.sw_plan.restype = ctypes.c_int
    lib.sw_cyclic_export.argtypes = [vp, i64, i64, vp]
    lib.sw_cyclic_export.restype = ctypes.c_int
    lib.sw_cyclic_connect.argtypes = [vp, vp, i64, i64]
    lib.sw_cyclic_connect.restype = ctypes.c_int
    lib.sw_cyclic_epoch.argtypes = [vp]
    lib.sw_cyclic_epoch.restype = i32
    lib.sw_align_stage1_cyclic.argtypes = [vp, vp, i64, vp, i64, i32, i32, i32, i32, i32, i32, i32, i64, SINK, vp, vp, R]
    lib.sw_align_stage1_cyclic.restype = ctypes.c_int
    lib.sw_stripe_export.argtypes = [vp, i64, vp]
    lib.sw_stripe_export.restype = ctypes.c_int
    lib.sw_stripe_connect.argtypes = [vp, vp, i64]
    lib.sw_stripe_connect.restype = ctypes.c_int
    lib.sw_align_stage1_stripe.argtypes = [vp, vp, i64, vp, i64, i64, i64, i32, i32, i32, i32, i32, i64, SINK, vp, vp, R]
    lib.sw_align_stage1_stripe.restype = ctypes.c_int
    lib.sw_special_row_interval_for_budget.argtypes = [i64, i64, i64, i64]
    lib.sw_special_row_interval_for_budget.restype = i64
    lib.sw_get_stats.argtypes = [vp, ctypes.POINTER(Stats)]
    lib.sw_get_stats.restype = ctypes.c_int
    lib.sw_shutdown.argtypes = [vp]
    lib.sw_shutdown.restype = None
    lib.sw_strerror.argtypes = [ctypes.c_int]
    lib.sw_strerror.restype = cp
    lib.sw_last_error.argtypes = [vp]
    lib.sw_last_error.restype = cp
    _lib = lib
    return lib


def special_row_interval_for_budget(m: int, n: int, bh: int, sra_bytes: int) -> int:
    """Flush-interval rule of P:178 (computed in the library)."""
    return int(load_library().sw_special_row_interval_for_budget(m, n, bh, sra_bytes))


def _as_bytes_ptr(x):
    """(pointer, length, keepalive) for bytes / str / numpy uint8 host sequences."""
    if isinstance(x, str):
        x = x.encode("ascii")
    if isinstance(x, (bytes, bytearray)):
        arr = np.frombuffer(bytes(x), dtype=np.uint8)
    else:
        arr = np.ascontiguousarray(x, dtype=np.uint8)
    return arr.ctypes.data, arr.size, arr


@dataclass
class Result:
    score: int
    i: int
    j: int

    def astuple(self):
        return (self.score, self.i, self.j)


def combine_best(results) -> tuple:
    """The library's total order of best cells (sw_combine_best) over (score, i, j) triples."""
    lib = load_library()
    rs = list(results)
    arr = (_Result * max(1, len(rs)))(*[_Result(int(a), int(b), int(c)) for a, b, c in rs])
    out = _Result()
    rc = lib.sw_combine_best(arr, len(rs), ctypes.byref(out))
    if rc != SW_OK:
        raise SwError(rc, "sw_combine_best")
    return (out.score, out.i, out.j)


class Context:
    """One engine context on one CUDA device (one process per GPU), or on
    several devices (``devices=[0, 1, ...]``: Stage 1 runs as one band pipeline
    across them)."""

    def __init__(self, device: int = 0, devices=None):
        self._lib = load_library()
        self._h = ctypes.c_void_p()
        ids_list = list(devices) if devices is not None else [device]
        ids = (ctypes.c_int * len(ids_list))(*ids_list)
        rc = self._lib.sw_init(ids, len(ids_list), ctypes.byref(self._h))
        if rc != SW_OK:
            raise SwError(rc, f"sw_init(devices={ids_list}) failed: {self._lib.sw_strerror(rc).decode()}")
        self.device = ids_list[0]
        self.devices = ids_list

    # ------------------------------------------------------------------ helpers
    def _check(self, rc, what):
        if rc != SW_OK:
            detail = self._lib.sw_last_error(self._h).decode()
            raise SwError(rc, f"{what}: {self._lib.sw_strerror(rc).decode()}" + (f" [{detail}]" if detail else ""))

    @staticmethod
    def _make_sink(sink, keep_rows, rows):
        def _cb(_user, row, H, F, n):
            try:
                h = np.ctypeslib.as_array(H, shape=(n,))
                f = np.ctypeslib.as_array(F, shape=(n,))
                if keep_rows:
                    rows.append((int(row), h.copy(), f.copy()))
                if sink is not None:
                    return 1 if sink(int(row), h, f) else 0
                return 0
            except Exception:  # never let an exception cross the C boundary
                return 1

        return SINK(_cb)

    # ------------------------------------------------------------------ API
    def align_stage1(self, A, B, match=1, mismatch=-3, gap_open=3, gap_ext=2, k=0, sink=None, keep_rows=False):
        """Stage 1 on host sequences.  Returns (Result, rows) where rows is the
        list of (row, H, F) if keep_rows.  ``sink(row, H, F)`` (views valid only
        during the call) may return True to abort."""
        pa, m, ka = _as_bytes_ptr(A)
        pb, n, kb = _as_bytes_ptr(B)
        rows = []
        cb = self._make_sink(sink, keep_rows, rows) if k > 0 else SINK()
        out = _Result()
        rc = self._lib.sw_align_stage1(self._h, pa, m, pb, n, match, mismatch, gap_open, gap_ext, k, cb, None, ctypes.byref(out))
        self._check(rc, "sw_align_stage1")
        return Result(out.score, out.i, out.j), rows

    def align_stage1_dev(self, dA_ptr: int, m: int, dB_ptr: int, n: int, match=1, mismatch=-3, gap_open=3, gap_ext=2,
                         k=0, sink=None, keep_rows=False, stream: int = 0):
        """Stage 1 on DEVICE byte buffers (e.g. torch uint8 cuda tensors' data_ptr())."""
        rows = []
        cb = self._make_sink(sink, keep_rows, rows) if k > 0 else SINK()
        out = _Result()
        rc = self._lib.sw_align_stage1_dev(self._h, dA_ptr, m, dB_ptr, n, match, mismatch, gap_open, gap_ext, k, cb,
                                           None, stream or None, ctypes.byref(out))
        self._check(rc, "sw_align_stage1_dev")
        return Result(out.score, out.i, out.j), rows

    def reverse_goal(self, A, i_end, B, j_end, goal, match=1, mismatch=-3, gap_open=3, gap_ext=2):
        """Start cell of the alignment ending at (i_end, j_end) with score goal."""
        pa, m, ka = _as_bytes_ptr(A)
        pb, n, kb = _as_bytes_ptr(B)
        if i_end > m or j_end > n:
            raise ValueError("end cell outside the sequences")
        out = _Result()
        rc = self._lib.sw_reverse_goal(self._h, pa, i_end, pb, j_end, match, mismatch, gap_open, gap_ext, goal, ctypes.byref(out))
        self._check(rc, "sw_reverse_goal")
        return Result(out.score, out.i, out.j)

    def reverse_goal_dev(self, dA_ptr, i_end, dB_ptr, j_end, goal, match=1, mismatch=-3, gap_open=3, gap_ext=2,
                         stream: int = 0):
        out = _Result()
        rc = self._lib.sw_reverse_goal_dev(self._h, dA_ptr, i_end, dB_ptr, j_end, match, mismatch, gap_open, gap_ext,
                                           goal, stream or None, ctypes.byref(out))
        self._check(rc, "sw_reverse_goal_dev")
        return Result(out.score, out.i, out.j)

    def _stage2_call(self, fn, args, cap):
        while True:
            buf = (_Crosspoint * max(1, cap))()
            cnt = ctypes.c_int64(0)
            rc = fn(*args, buf, cap, ctypes.byref(cnt))
            if rc == SW_ERANGE and cnt.value > cap:
                cap = cnt.value
                continue
            self._check(rc, fn.__name__)
            return [(c.i, c.j, c.score, c.type) for c in buf[: cnt.value]]

    def stage2(self, A, B, match=1, mismatch=-3, gap_open=3, gap_ext=2, k=0, end=None):
        """Stage 2 crosspoint list L_2 (ascending, start point first) from the end
        point `end` (a Result / (score, i, j)) against the special rows kept from
        the last align_stage1 call with the same inputs, k and scoring."""
        pa, m, ka = _as_bytes_ptr(A)
        pb, n, kb = _as_bytes_ptr(B)
        e = end if isinstance(end, tuple) else end.astuple()
        r = _Result(e[0], e[1], e[2])
        # at most one crosspoint per special row, plus the start and end points
        return self._stage2_call(self._lib.sw_stage2, (self._h, pa, m, pb, n, match, mismatch, gap_open, gap_ext, k,
                                                       ctypes.byref(r)), (m // k if k > 0 else 0) + 2)

    def stage2_dev(self, dA_ptr, m, dB_ptr, n, match=1, mismatch=-3, gap_open=3, gap_ext=2, k=0, end=None,
                   stream: int = 0):
        e = end if isinstance(end, tuple) else end.astuple()
        r = _Result(e[0], e[1], e[2])
        return self._stage2_call(self._lib.sw_stage2_dev, (self._h, dA_ptr, m, dB_ptr, n, match, mismatch, gap_open,
                                                           gap_ext, k, ctypes.byref(r), stream or None),
                                 (m // k if k > 0 else 0) + 2)

    def align(self, A, B, match=1, mismatch=-3, gap_open=3, gap_ext=2, k=0):
        """Stages 1-5: the full optimal local alignment (sw_align).  Returns a dict:
        score, start (i0, j0), end (i1, j1), gap1 / gap2 lists of (i, j, len)
        (P:281), partitions, mm_levels."""
        pa, m, ka = _as_bytes_ptr(A)
        pb, n, kb = _as_bytes_ptr(B)
        # gap-run buffers sized for typical alignments (a run every >= 64 columns),
        # so the call is not repeated; sw_align reports SW_ERANGE with the counts
        # if they are too small, and the call is retried with exact sizes
        cap1 = cap2 = max(1024, min(m, n) // 64)
        while True:
            g1 = (_Gap * cap1)()
            g2 = (_Gap * cap2)()
            out = _Alignment()
            rc = self._lib.sw_align(self._h, pa, m, pb, n, match, mismatch, gap_open, gap_ext, k, ctypes.byref(out),
                                    g1, cap1, g2, cap2)
            if rc == -3 and (out.n_gap1 > cap1 or out.n_gap2 > cap2):
                cap1, cap2 = max(cap1, out.n_gap1), max(cap2, out.n_gap2)
                continue
            self._check(rc, "sw_align")
            break
        return {"score": out.score, "start": (out.i0, out.j0), "end": (out.i1, out.j1),
                "gap1": [(g.i, g.j, g.len) for g in g1[: out.n_gap1]],
                "gap2": [(g.i, g.j, g.len) for g in g2[: out.n_gap2]],
                "partitions": out.partitions, "mm_levels": out.mm_levels,
                "ms": {"stage1": out.ms_stage1, "stage2": out.ms_stage2, "stages3_4": out.ms_mm,
                       "stage5": out.ms_stage5}}

    def row_granularity(self) -> int:
        return int(self._lib.sw_row_granularity(self._h))

    def band_height(self) -> int:
        return int(self._lib.sw_band_height(self._h))

    def set_kernel(self, variant: int = -1, packed: bool = True):
        """variant -1: automatic; 0..14: fixed geometry (8..14 packed-only); packed: allow the 16x2 kernel."""
        self._check(self._lib.sw_set_kernel(self._h, variant, int(bool(packed))), "sw_set_kernel")

    def set_patch(self, on: bool = True):
        """Run the packed kernel with the gap penalties patched in as immediates
        (default) or read from registers; results are identical."""
        self._check(self._lib.sw_set_patch(self._h, int(bool(on))), "sw_set_patch")

    def set_virtual_stripes(self, nstripes: int):
        """Split the next Stage-1 calls into `nstripes` column stripes on this GPU
        (the multi-GPU border protocol, run inside one launch)."""
        self._check(self._lib.sw_set_virtual_stripes(self._h, nstripes), "sw_set_virtual_stripes")

    def set_tail(self, mode: int = -1):
        """Tail segment: -1 automatic, 0 off, v + 1 force packed geometry v (testing)."""
        self._check(self._lib.sw_set_tail(self._h, mode), "sw_set_tail")

    def set_row_budget(self, nbytes: int = 0):
        """Device bytes for the special-row ring (0: default); smaller budgets
        stream the rows through a ring with back-pressure."""
        self._check(self._lib.sw_set_row_budget(self._h, nbytes), "sw_set_row_budget")

    def set_multi_gpu(self, cyclic: bool = True):
        """Multi-device Stage 1: band-cyclic (default) or column stripes on the first device."""
        self._check(self._lib.sw_set_multi_gpu(self._h, int(bool(cyclic))), "sw_set_multi_gpu")

    def device_count(self) -> int:
        return int(self._lib.sw_device_count(self._h))

    def set_grid(self, ctas: int = 0):
        """Cap the CTAs of every fill launch (0: resident capacity), so bands
        outnumber CTAs and the multi-wave band pipeline runs on small inputs."""
        self._check(self._lib.sw_set_grid(self._h, ctas), "sw_set_grid")

    def stripe_epoch(self) -> int:
        """Highest epoch this context ran a stripe call with (sw_stripe_epoch)."""
        return int(self._lib.sw_stripe_epoch(self._h))

    def plan(self, m, n, match=1, mismatch=-3, gap_open=3, gap_ext=2, k=0, world=0):
        """(alpha, warps) of the geometry the next rank call would run (alpha < 0:
        packed); world 0: a column-stripe rank, else a band-cyclic group of `world`."""
        a, w = ctypes.c_int32(0), ctypes.c_int32(0)
        self._check(self._lib.sw_plan(self._h, m, n, match, mismatch, gap_open, gap_ext, k, world, ctypes.byref(a),
                                      ctypes.byref(w)), "sw_plan")
        return (a.value, w.value)

    def cyclic_epoch(self) -> int:
        return int(self._lib.sw_cyclic_epoch(self._h))

    def cyclic_export(self, max_rows: int, max_cols: int) -> bytes:
        """Allocate this rank's incoming band-cyclic area; returns its 64-byte CUDA IPC handle."""
        buf = ctypes.create_string_buffer(64)
        self._check(self._lib.sw_cyclic_export(self._h, max_rows, max_cols, buf), "sw_cyclic_export")
        return buf.raw

    def cyclic_connect(self, next_handle, max_rows: int, max_cols: int):
        """Map the next rank's band-cyclic area."""
        h = ctypes.create_string_buffer(bytes(next_handle), 64)
        self._check(self._lib.sw_cyclic_connect(self._h, h, max_rows, max_cols), "sw_cyclic_connect")

    def align_stage1_cyclic(self, dA_ptr, m, dB_ptr, n, rank, world, epoch, match=1, mismatch=-3, gap_open=3,
                            gap_ext=2, k=0, sink=None, keep_rows=False, stream: int = 0):
        """This rank's bands (rank, rank + world, ...) of Stage 1 (device sequences)."""
        rows = []
        cb = self._make_sink(sink, keep_rows, rows) if k > 0 else SINK()
        out = _Result()
        rc = self._lib.sw_align_stage1_cyclic(self._h, dA_ptr, m, dB_ptr, n, rank, world, epoch, match, mismatch,
                                              gap_open, gap_ext, k, cb, None, stream or None, ctypes.byref(out))
        self._check(rc, "sw_align_stage1_cyclic")
        return Result(out.score, out.i, out.j), rows

    def stripe_export(self, max_rows: int) -> bytes:
        """Allocate this rank's left-border receive area; returns its 64-byte CUDA IPC handle."""
        buf = ctypes.create_string_buffer(64)
        self._check(self._lib.sw_stripe_export(self._h, max_rows, buf), "sw_stripe_export")
        return buf.raw

    def stripe_connect(self, right_handle, max_rows: int):
        """Map the right neighbour's receive area (None for the last stripe)."""
        h = ctypes.create_string_buffer(bytes(right_handle), 64) if right_handle is not None else None
        self._check(self._lib.sw_stripe_connect(self._h, h, max_rows), "sw_stripe_connect")

    def align_stage1_stripe(self, dA_ptr, m, dB_ptr, n, c_lo, c_hi, epoch, match=1, mismatch=-3, gap_open=3,
                            gap_ext=2, k=0, sink=None, keep_rows=False, stream: int = 0):
        """This rank's stripe [c_lo, c_hi) of Stage 1 (device sequences, whole A and B)."""
        rows = []
        cb = self._make_sink(sink, keep_rows, rows) if k > 0 else SINK()
        out = _Result()
        rc = self._lib.sw_align_stage1_stripe(self._h, dA_ptr, m, dB_ptr, n, c_lo, c_hi, epoch, match, mismatch,
                                              gap_open, gap_ext, k, cb, None, stream or None, ctypes.byref(out))
        self._check(rc, "sw_align_stage1_stripe")
        return Result(out.score, out.i, out.j), rows

    def stats(self) -> dict:
        s = Stats()
        self._check(self._lib.sw_get_stats(self._h, ctypes.byref(s)), "sw_get_stats")
        return s.as_dict()

    def close(self):
        if self._h:
            self._lib.sw_shutdown(self._h)
            self._h = ctypes.c_void_p()

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
