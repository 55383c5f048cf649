"""Python binding of libpsim (include/psim.h): argument marshalling only.

Every step of the simulation runs in the library's CUDA kernels; this module
never computes anything itself and has no CPU fallback.  If libpsim.so is
missing the import fails loudly (build it with ``python -m
paper_conf_sc_pandeylfhl22_b200.build`` or ``__graft_entry__.build()``).

Names follow the C ABI: load_trace, partition, load_model, simulate,
total_cycles.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("PSIM_LIB") or os.path.join(_HERE, "libpsim.so")   # PSIM_LIB: A/B experiments only

OK, ERR_ARG, ERR_STATE, ERR_CUDA, ERR_NCCL, ERR_OOM, ERR_UNSUPPORTED = 0, -1, -2, -3, -4, -5, -6
FP32, BF16 = 0, 1
ARCH = {"M2": 1, "C3": 2, "RB7": 3}
RECORD_ROWS = 1
PROFILE = 2
FORCE_PREDICT = 4
LAYERWISE = 8
SPARSE24 = 16
FC1_PAIR = 32
MAX_CAP = 110
MAX_INTERVAL = 262144   # PSIM_MAX_INTERVAL
NATTR = 47


class PsimError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"psim error {code}: {msg}")
        self.code = code


class _Opts(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("rank", ctypes.c_int), ("world_size", ctypes.c_int),
                ("nccl_id", ctypes.c_void_p), ("queue_cap", ctypes.c_uint32), ("precision", ctypes.c_uint32),
                ("chunk_steps", ctypes.c_uint64), ("stream", ctypes.c_void_p), ("flags", ctypes.c_uint32),
                ("correction_limit", ctypes.c_uint32), ("interval", ctypes.c_uint32)]


class _ModelDesc(ctypes.Structure):
    _fields_ = [("arch", ctypes.c_uint32), ("rows", ctypes.c_uint32), ("features", ctypes.c_uint32),
                ("reserved", ctypes.c_uint32)]


class Stats(ctypes.Structure):
    _fields_ = [("k_hist", ctypes.c_uint64 * 112), ("stalls", ctypes.c_uint64), ("steps", ctypes.c_uint64),
                ("simulated", ctypes.c_uint64), ("counted", ctypes.c_uint64), ("subtraces", ctypes.c_uint64),
                ("h2d_bytes", ctypes.c_uint64), ("gpu_launches", ctypes.c_uint64), ("sim_ms", ctypes.c_double),
                ("load_ms", ctypes.c_double), ("local_cycles", ctypes.c_int64), ("trace_mode", ctypes.c_int32),
                ("comm_ranks", ctypes.c_int32), ("kernel_ms", ctypes.c_double * 8), ("kernel_launches", ctypes.c_uint64 * 8),
                ("layer_m", ctypes.c_uint64 * 4), ("layer_n", ctypes.c_uint32 * 4), ("layer_k", ctypes.c_uint32 * 4),
                ("corrected", ctypes.c_uint64), ("corr_steps", ctypes.c_uint64)]

    def as_dict(self):
        d = {f: getattr(self, f) for f, _ in self._fields_}
        for f in ("k_hist", "kernel_ms", "kernel_launches", "layer_m", "layer_n", "layer_k"):
            d[f] = list(d[f])
        d["kernel_names"] = [lib().psim_kernel_class_name(i).decode() for i in range(8)]
        return d


EXPORTS = ["psim_create", "psim_destroy", "psim_load_trace", "psim_partition", "psim_load_model",
           "psim_simulate", "psim_total_cycles", "psim_last_error", "psim_force_latencies", "psim_get_rows",
           "psim_get_subtrace_cycles", "psim_rank_range", "psim_get_stats", "psim_cnn_forward", "psim_version",
           "psim_partition_range", "psim_kernel_class_name", "psim_nccl_unique_id", "psim_get_corrections",
           "psim_get_corrected_rows", "psim_get_interval_metrics", "psim_get_outputs"]

_lib = None


def lib():
    """Load libpsim.so (raises ImportError if it was not built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run `python -m paper_conf_sc_pandeylfhl22_b200.build` "
                              "(there is no CPU fallback)")
        L = ctypes.CDLL(LIB_PATH)
        c, P = ctypes, ctypes.c_void_p
        L.psim_create.argtypes = [c.POINTER(_Opts), c.POINTER(P)]
        L.psim_destroy.argtypes = [P]
        L.psim_destroy.restype = None
        L.psim_load_trace.argtypes = [P, P, c.c_uint64, c.c_uint64, c.c_uint64, c.c_uint32, c.c_uint64]
        L.psim_partition.argtypes = [P, c.c_uint64, c.c_uint64]
        L.psim_load_model.argtypes = [P, c.POINTER(_ModelDesc), P, c.c_uint64]
        L.psim_simulate.argtypes = [P]
        L.psim_total_cycles.argtypes = [P, c.POINTER(c.c_int64)]
        L.psim_last_error.argtypes = [P]
        L.psim_last_error.restype = c.c_char_p
        L.psim_force_latencies.argtypes = [P, P, c.c_uint64]
        L.psim_get_rows.argtypes = [P, c.c_uint64, c.c_uint64, P, P, P]
        L.psim_get_outputs.argtypes = [P, c.c_uint64, c.c_uint64, P]
        L.psim_get_subtrace_cycles.argtypes = [P, c.c_uint64, c.c_uint64, P]
        L.psim_get_corrections.argtypes = [P, c.c_uint64, c.c_uint64, P, P]
        L.psim_get_corrected_rows.argtypes = [P, c.c_uint64, c.c_uint64, P, P]
        L.psim_get_interval_metrics.argtypes = [P, c.c_uint64, c.c_uint64, P, P, P, P]
        L.psim_rank_range.argtypes = [P, c.POINTER(c.c_uint64), c.POINTER(c.c_uint64), c.POINTER(c.c_uint64),
                                      c.POINTER(c.c_uint64)]
        L.psim_get_stats.argtypes = [P, c.POINTER(Stats)]
        L.psim_cnn_forward.argtypes = [P, P, c.c_uint64, P]
        L.psim_version.restype = c.c_char_p
        U = c.POINTER(c.c_uint64)
        L.psim_kernel_class_name.argtypes = [c.c_int]
        L.psim_kernel_class_name.restype = c.c_char_p
        L.psim_nccl_unique_id.argtypes = [P]
        L.psim_partition_range.argtypes = [c.c_uint64, c.c_uint64, c.c_uint64, c.c_int, c.c_int, U, U, U, U, U]
        _lib = L
    return _lib


def version() -> str:
    return lib().psim_version().decode()


def _ptr(a):
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return a.ctypes.data_as(ctypes.c_void_p)
    # torch tensor (device or pinned host): raw data pointer
    return ctypes.c_void_p(a.data_ptr())


@dataclass
class RankRange:
    j0: int
    j1: int
    row_lo: int
    row_hi: int
    steps: int = 0


def partition_range(L: int, N: int, W: int, rank: int = 0, world_size: int = 1) -> RankRange:
    """Host-only: rank's sub-trace block, trace rows and step count (no GPU needed)."""
    v = [ctypes.c_uint64() for _ in range(5)]
    rc = lib().psim_partition_range(L, N, W, rank, world_size, *[ctypes.byref(x) for x in v])
    if rc != OK:
        raise PsimError(rc, "bad partition arguments")
    return RankRange(*[int(x.value) for x in v])


def nccl_unique_id() -> bytes:
    """128-byte ncclUniqueId (rank 0), to broadcast with torch.distributed."""
    buf = ctypes.create_string_buffer(128)
    rc = lib().psim_nccl_unique_id(buf)
    if rc != OK:
        raise PsimError(rc, "NCCL unavailable")
    return buf.raw


def all_reduce_total(local_total: int, group=None) -> int:
    """Sum per-rank totals over a torch.distributed group (used when the context
    was created without an NCCL id, e.g. gloo on CPU)."""
    import torch
    import torch.distributed as dist
    t = torch.tensor([local_total], dtype=torch.int64)
    dist.all_reduce(t, group=group)
    return int(t.item())


class Simulator:
    """One context = one GPU (one process per GPU)."""

    def __init__(self, device: int = 0, precision: str = "bf16", queue_cap: int = MAX_CAP,
                 rank: int = 0, world_size: int = 1, nccl_id: bytes | None = None,
                 stream=None, record_rows: bool = False, chunk_steps: int = 0, profile: bool = False,
                 force_predict: bool = False, layerwise: bool = False, correction_limit: int = 0,
                 interval: int = 0, sparse24: bool = False, fc1_pair: bool = False):
        self._keep = []
        idbuf = None
        if nccl_id is not None:
            idbuf = ctypes.create_string_buffer(bytes(nccl_id), 128)
            self._keep.append(idbuf)
        o = _Opts(device=device, rank=rank, world_size=world_size,
                  nccl_id=ctypes.cast(idbuf, ctypes.c_void_p) if idbuf is not None else None,
                  queue_cap=queue_cap, precision=BF16 if precision == "bf16" else FP32,
                  chunk_steps=chunk_steps,
                  stream=ctypes.c_void_p(int(stream)) if stream is not None else None,
                  flags=(RECORD_ROWS if record_rows else 0) | (PROFILE if profile else 0)
                  | (FORCE_PREDICT if force_predict else 0) | (LAYERWISE if layerwise else 0)
                  | (SPARSE24 if sparse24 else 0) | (FC1_PAIR if fc1_pair else 0),
                  correction_limit=correction_limit, interval=interval)
        h = ctypes.c_void_p()
        rc = lib().psim_create(ctypes.byref(o), ctypes.byref(h))
        if rc != OK:
            raise PsimError(rc, "psim_create failed")
        self._h = h
        self.world_size = world_size
        self._interval = interval
        self._L = 0

    def close(self):
        if getattr(self, "_h", None):
            lib().psim_destroy(self._h)
            self._h = None

    def __del__(self):
        self.close()

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def _check(self, rc):
        if rc != OK:
            raise PsimError(rc, lib().psim_last_error(self._h).decode())

    # ------------------------------------------------------------- the ABI
    def load_trace(self, attrs, n_instr: int | None = None, first_row: int = 0):
        """attrs: numpy uint8 [rows][stride] (host) or torch uint8 tensor (device or pinned host)."""
        rows, stride = int(attrs.shape[0]), int(attrs.shape[1])
        n_instr = rows + first_row if n_instr is None else n_instr
        self._trace_ref = attrs     # the library borrows the buffer until simulate returns
        self._L = n_instr
        self._check(lib().psim_load_trace(self._h, _ptr(attrs), n_instr, first_row, rows, NATTR, stride))

    def partition(self, n_subtraces: int, warmup: int):
        self._check(lib().psim_partition(self._h, n_subtraces, warmup))

    def load_model(self, arch: str, weights: np.ndarray):
        w = np.ascontiguousarray(weights, dtype=np.float32)
        d = _ModelDesc(arch=ARCH[arch], rows=112, features=50, reserved=0)
        self._check(lib().psim_load_model(self._h, ctypes.byref(d), _ptr(w), w.size))

    def simulate(self):
        self._check(lib().psim_simulate(self._h))

    def total_cycles(self) -> int:
        v = ctypes.c_int64()
        self._check(lib().psim_total_cycles(self._h, ctypes.byref(v)))
        return int(v.value)

    # ------------------------------------------------------------- diagnostics
    def force_latencies(self, lat3):
        if lat3 is None:
            self._check(lib().psim_force_latencies(self._h, None, 0))
            return
        a = np.ascontiguousarray(lat3, dtype=np.uint16)
        self._check(lib().psim_force_latencies(self._h, _ptr(a), a.shape[0]))

    def rank_range(self) -> RankRange:
        v = [ctypes.c_uint64() for _ in range(4)]
        self._check(lib().psim_rank_range(self._h, *[ctypes.byref(x) for x in v]))
        return RankRange(*[int(x.value) for x in v])

    def get_rows(self, first: int, n: int):
        lat = np.zeros((n, 3), np.uint16)
        k = np.zeros(n, np.int32)
        clk = np.zeros(n, np.int64)
        self._check(lib().psim_get_rows(self._h, first, n, _ptr(lat), _ptr(k), _ptr(clk)))
        return lat, k, clk

    def get_outputs(self, first: int, n: int) -> np.ndarray:
        """Raw fp32 CNN outputs [n][3] the hot path computed for real rows [first, first+n)."""
        y = np.zeros((max(n, 1), 3), np.float32)
        self._check(lib().psim_get_outputs(self._h, first, n, _ptr(y)))
        return y[:n]

    def subtrace_cycles(self, first: int = 0, n: int | None = None) -> np.ndarray:
        rr = self.rank_range()
        n = (rr.j1 - rr.j0 - first) if n is None else n
        out = np.zeros(max(n, 1), np.int64)
        self._check(lib().psim_get_subtrace_cycles(self._h, first, n, _ptr(out)))
        return out[:n]

    def corrections(self, first: int = 0, n: int | None = None):
        """(corr_len, cycles1) of local sub-traces [first, first+n): rows re-simulated by the
        predecessor and the first-pass cycles (post-error correction)."""
        rr = self.rank_range()
        n = (rr.j1 - rr.j0 - first) if n is None else n
        cl = np.zeros(max(n, 1), np.int32)
        c1 = np.zeros(max(n, 1), np.int64)
        self._check(lib().psim_get_corrections(self._h, first, n, _ptr(cl), _ptr(c1)))
        return cl[:n], c1[:n]

    def get_corrected_rows(self, first: int, n: int):
        lat = np.zeros((n, 3), np.uint16)
        k = np.zeros(n, np.int32)
        self._check(lib().psim_get_corrected_rows(self._h, first, n, _ptr(lat), _ptr(k)))
        return lat, k

    def interval_metrics(self, first: int = 0, n: int | None = None) -> dict:
        """Interval metrics of the last simulate (interval > 0, R20):
        int64 arrays cycles / retired / retired_st / mem_bytes for global intervals
        [first, first+n) (default: all), plus cpi = cycles / retired and bw = mem_bytes /
        cycles (bytes per cycle) where defined."""
        if n is None:
            n = max(0, -(-self._L // self._interval) - first) if getattr(self, "_interval", 0) else 0
        out = [np.zeros(max(n, 1), np.int64) for _ in range(4)]
        self._check(lib().psim_get_interval_metrics(self._h, first, n, *[_ptr(x) for x in out]))
        cyc, ret, ret_st, mb = (x[:n] for x in out)
        with np.errstate(divide="ignore", invalid="ignore"):
            cpi = np.where(ret > 0, cyc / np.maximum(ret, 1), np.nan)
            bw = np.where(cyc > 0, mb / np.maximum(cyc, 1), np.nan)
        return dict(cycles=cyc, retired=ret, retired_st=ret_st, mem_bytes=mb, cpi=cpi, bw=bw)

    def stats(self) -> dict:
        s = Stats()
        self._check(lib().psim_get_stats(self._h, ctypes.byref(s)))
        return s.as_dict()

    def cnn_forward(self, X: np.ndarray) -> np.ndarray:
        X = np.ascontiguousarray(X, dtype=np.float32).reshape(-1, 112, 50)
        Y = np.zeros((X.shape[0], 3), np.float32)
        self._check(lib().psim_cnn_forward(self._h, _ptr(X), X.shape[0], _ptr(Y)))
        return Y
