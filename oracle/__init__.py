"""ctypes wrapper of the CPU oracle (oracle/oracle.c).

TEST INFRASTRUCTURE ONLY: only tests/, ``__graft_entry__.smoke()`` and
bench.py's ``cpu_baseline`` / ``--impl reference`` legs may import this.  The
product package (paper_conf_sc_pandeylfhl22_b200) never imports it and shares
no code with it.

Every function documents the PAPER.md passage it follows; see oracle.c.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

ROWS = 112
FEAT = 50
NATTR = 47
FP64 = 0
BF16 = 1
ARCH = {"M2": 1, "C3": 2, "RB7": 3}


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (plain C, -O2, no intrinsics, no BLAS)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".{os.getpid()}.tmp"
        subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-fPIC", "-shared", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        c = ctypes
        P = c.c_void_p
        _lib.oracle_arch_nparams.restype = c.c_long
        _lib.oracle_arch_nparams.argtypes = [c.c_int]
        _lib.oracle_cnn_forward.restype = c.c_int
        _lib.oracle_cnn_forward.argtypes = [c.c_int, c.c_int, P, c.c_long, P, P]
        _lib.oracle_round_latency.restype = c.c_int
        _lib.oracle_round_latency.argtypes = [c.c_double]
        _lib.oracle_queue_new.restype = P
        _lib.oracle_queue_new.argtypes = [c.c_int, c.c_int64]
        _lib.oracle_queue_free.argtypes = [P]
        _lib.oracle_queue_clock.restype = c.c_int64
        _lib.oracle_queue_clock.argtypes = [P]
        _lib.oracle_queue_stalls.restype = c.c_int64
        _lib.oracle_queue_stalls.argtypes = [P]
        _lib.oracle_queue_size.restype = c.c_int
        _lib.oracle_queue_size.argtypes = [P]
        _lib.oracle_queue_entries.restype = c.c_int
        _lib.oracle_queue_entries.argtypes = [P, P, P, P, P]
        _lib.oracle_build_input.restype = c.c_int
        _lib.oracle_build_input.argtypes = [P, P, c.c_long, c.c_long, P]
        _lib.oracle_queue_update.restype = c.c_int
        _lib.oracle_queue_update.argtypes = [P, c.c_long, c.c_int, c.c_int, c.c_int, P, P, P]
        _lib.oracle_partition.restype = c.c_int
        _lib.oracle_partition.argtypes = [c.c_long, c.c_long, c.c_long, P, P, P]
        _lib.oracle_simulate.restype = c.c_int
        _lib.oracle_simulate.argtypes = [
            c.c_int, c.c_int, P, c.c_long,      # arch, mode, weights, n
            P, c.c_long, c.c_long, c.c_long, c.c_long, c.c_int,  # trace, stride, L, N, W, cap
            P, c.c_long, c.c_long, c.c_int64,   # forced, j0, nj, clock0
            P, P, P, P, P, P, P]                # cycles, boundary, lat, y, k, clock, stalls
        _lib.oracle_simulate_pec.restype = c.c_int
        _lib.oracle_simulate_pec.argtypes = [
            c.c_int, c.c_int, P, c.c_long,      # arch, mode, weights, n
            P, c.c_long, c.c_long, c.c_long, c.c_long, c.c_int,  # trace, stride, L, N, W, cap
            P, c.c_long, c.c_long, c.c_long, c.c_long,   # forced, j0, nj, G, limit
            P, P, P, P,                         # cycles, cycles1, boundary, corr_len
            P, P, P, P, P, P]                   # lat, k, clock, corr_lat, corr_k, stalls
        _lib.oracle_simulate_metrics.restype = c.c_int
        _lib.oracle_simulate_metrics.argtypes = [
            c.c_int, c.c_int, P, c.c_long,      # arch, mode, weights, n
            P, c.c_long, c.c_long, c.c_long, c.c_long, c.c_int,  # trace, stride, L, N, W, cap
            P, c.c_long, c.c_long, c.c_long,    # forced, j0, nj, interval
            P, P, P, P]                         # cycles, retired, retired_st, mem_bytes
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def nparams(arch: str) -> int:
    return int(lib().oracle_arch_nparams(ARCH[arch]))


def cnn_forward(arch: str, weights: np.ndarray, X: np.ndarray, mode: int = FP64) -> np.ndarray:
    """y = CNN(X) for one [112][50] input (PAPER.md:93 step 3; model per R11)."""
    w = np.ascontiguousarray(weights, dtype=np.float32)
    X = np.ascontiguousarray(X, dtype=np.float64).reshape(ROWS, FEAT)
    y = np.zeros(3, np.float64)
    rc = lib().oracle_cnn_forward(ARCH[arch], mode, _ptr(w), w.size, _ptr(X), _ptr(y))
    if rc != 0:
        raise ValueError(f"oracle_cnn_forward rc={rc}")
    return y


def round_latency(y: float) -> int:
    """rint(float(y)) clamped to [0, 4095], NaN -> 0 (R7)."""
    return int(lib().oracle_round_latency(float(y)))


class Queue:
    """The instruction queue with Clock and per-entry retire clock."""

    def __init__(self, cap: int, clock0: int = 0):
        self._q = lib().oracle_queue_new(cap, clock0)
        if not self._q:
            raise ValueError("bad capacity")
        self.cap = cap

    def __del__(self):
        if getattr(self, "_q", None):
            lib().oracle_queue_free(self._q)
            self._q = None

    @property
    def clock(self) -> int:
        return int(lib().oracle_queue_clock(self._q))

    @property
    def stalls(self) -> int:
        return int(lib().oracle_queue_stalls(self._q))

    def entries(self):
        n = lib().oracle_queue_size(self._q)
        a = [np.zeros(max(n, 1), np.int64) for _ in range(4)]
        lib().oracle_queue_entries(self._q, *[_ptr(x) for x in a])
        return [tuple(int(x[i]) for x in a) for i in range(n)]  # (seq, fetch, complete, retire)

    def build_input(self, trace: np.ndarray, i: int):
        X = np.zeros((ROWS, FEAT), np.float64)
        k = lib().oracle_build_input(self._q, _ptr(trace), trace.shape[1], i, _ptr(X))
        return X, int(k)

    def update(self, i: int, f: int, c: int, s: int):
        log_seq = np.zeros(self.cap + 2, np.int64)
        log_ret = np.zeros(self.cap + 2, np.int64)
        st = ctypes.c_int(0)
        n = lib().oracle_queue_update(self._q, i, f, c, s, _ptr(log_seq), _ptr(log_ret), ctypes.byref(st))
        return [(int(log_seq[k]), int(log_ret[k])) for k in range(n)], bool(st.value)


def partition(L: int, N: int, W: int):
    """s_j = floor(jL/N), e_j = s_{j+1}, ws_j = max(0, s_j - W) (R8, R9)."""
    s = np.zeros(N, np.int64); e = np.zeros(N, np.int64); ws = np.zeros(N, np.int64)
    if lib().oracle_partition(L, N, W, _ptr(s), _ptr(e), _ptr(ws)) != 0:
        raise ValueError("bad partition arguments")
    return s, e, ws


def simulate(trace: np.ndarray, N: int, W: int, *, arch: str = "C3", weights=None,
             mode: int = FP64, cap: int = 110, forced_lat=None, j0: int = 0, nj=None,
             clock0: int = 0, want_rows: bool = True, L: int | None = None, row_offset: int = 0):
    """Simulate sub-traces [j0, j0+nj) of the N-way partition.

    ``trace`` holds rows [row_offset, row_offset + len(trace)) of an L-row trace
    (default: the whole trace).  Returns dict(cycles, boundary, total, stalls,
    and per-row lat/y/k/clock over all L rows if want_rows).
    """
    trace = np.ascontiguousarray(trace, dtype=np.uint8)
    L = trace.shape[0] + row_offset if L is None else L
    nj = N - j0 if nj is None else nj
    w = None if weights is None else np.ascontiguousarray(weights, dtype=np.float32)
    forced = None if forced_lat is None else np.ascontiguousarray(forced_lat, dtype=np.uint16)
    cycles = np.zeros(max(nj, 1), np.int64)
    boundary = np.zeros(max(nj, 1), np.int64)
    lat = y = k = clk = None
    if want_rows:
        lat = np.zeros((L, 3), np.uint16)
        y = np.zeros((L, 3), np.float32)
        k = np.full(L, -1, np.int32)
        clk = np.zeros(L, np.int64)
    stalls = ctypes.c_int64(0)
    rc = lib().oracle_simulate(
        ARCH.get(arch, 0), mode, _ptr(w), 0 if w is None else w.size,
        ctypes.c_void_p(trace.ctypes.data - row_offset * trace.shape[1]), trace.shape[1], L, N, W, cap,
        _ptr(forced), j0, nj, clock0,
        _ptr(cycles), _ptr(boundary), _ptr(lat), _ptr(y), _ptr(k), _ptr(clk), ctypes.byref(stalls))
    if rc != 0:
        raise ValueError(f"oracle_simulate rc={rc}")
    out = dict(cycles=cycles[:nj], boundary=boundary[:nj], total=int(cycles[:nj].sum()),
               stalls=int(stalls.value))
    if want_rows:
        out.update(lat=lat, y=y, k=k, clock=clk)
    return out


def simulate_pec(trace: np.ndarray, N: int, W: int, *, limit: int = 100, G: int = 1, arch: str = "C3",
                 weights=None, mode: int = FP64, cap: int = 110, forced_lat=None, j0: int = 0, nj=None,
                 want_rows: bool = True, L: int | None = None, row_offset: int = 0):
    """Simulate with post-error correction (Fig. 9; R19).

    Same arguments as simulate() plus ``limit`` (max re-simulated rows per
    sub-trace, PAPER.md:291 uses 100) and ``G`` (ranks: the first sub-trace of
    each rank is not corrected).  Returns dict(cycles (corrected), cycles1
    (first pass), boundary, corr_len, total, total1, stalls, and per-row
    lat/k/clock (first pass) and corr_lat/corr_k (re-simulated rows, k = -1
    elsewhere) over all L rows if want_rows).
    """
    trace = np.ascontiguousarray(trace, dtype=np.uint8)
    L = trace.shape[0] + row_offset if L is None else L
    nj = N - j0 if nj is None else nj
    w = None if weights is None else np.ascontiguousarray(weights, dtype=np.float32)
    forced = None if forced_lat is None else np.ascontiguousarray(forced_lat, dtype=np.uint16)
    m = max(nj, 1)
    cycles, cycles1, boundary = (np.zeros(m, np.int64) for _ in range(3))
    corr_len = np.zeros(m, np.int32)
    lat = k = clk = clat = ck = None
    if want_rows:
        lat = np.zeros((L, 3), np.uint16)
        k = np.full(L, -1, np.int32)
        clk = np.zeros(L, np.int64)
        clat = np.zeros((L, 3), np.uint16)
        ck = np.full(L, -1, np.int32)
    stalls = ctypes.c_int64(0)
    rc = lib().oracle_simulate_pec(
        ARCH.get(arch, 0), mode, _ptr(w), 0 if w is None else w.size,
        ctypes.c_void_p(trace.ctypes.data - row_offset * trace.shape[1]), trace.shape[1], L, N, W, cap,
        _ptr(forced), j0, nj, G, limit,
        _ptr(cycles), _ptr(cycles1), _ptr(boundary), _ptr(corr_len),
        _ptr(lat), _ptr(k), _ptr(clk), _ptr(clat), _ptr(ck), ctypes.byref(stalls))
    if rc != 0:
        raise ValueError(f"oracle_simulate_pec rc={rc}")
    out = dict(cycles=cycles[:nj], cycles1=cycles1[:nj], boundary=boundary[:nj], corr_len=corr_len[:nj],
               total=int(cycles[:nj].sum()), total1=int(cycles1[:nj].sum()), stalls=int(stalls.value))
    if want_rows:
        out.update(lat=lat, k=k, clock=clk, corr_lat=clat, corr_k=ck)
    return out


def simulate_metrics(trace: np.ndarray, N: int, W: int, interval: int, *, arch: str = "C3", weights=None,
                     mode: int = FP64, cap: int = 110, forced_lat=None, j0: int = 0, nj=None,
                     L: int | None = None, row_offset: int = 0):
    """Interval metrics of the partitioned simulation (PAPER.md:310-318 [VI-E]; R20).

    For the counted rows of sub-traces [j0, j0+nj), per interval g of
    ``interval`` global rows: cycles (Clock advance of the steps of its rows),
    retired (queue entries retired in those steps), retired_st (of which
    stores), mem_bytes (data of its loads/stores served by memory).  Returns
    dict of int64 arrays of length ceil(L / interval) plus cpi and bw
    (bytes/cycle) where defined.
    """
    trace = np.ascontiguousarray(trace, dtype=np.uint8)
    L = trace.shape[0] + row_offset if L is None else L
    nj = N - j0 if nj is None else nj
    w = None if weights is None else np.ascontiguousarray(weights, dtype=np.float32)
    forced = None if forced_lat is None else np.ascontiguousarray(forced_lat, dtype=np.uint16)
    if interval < 1:
        raise ValueError("interval must be >= 1")
    ng = (L + interval - 1) // interval
    cyc, ret, ret_st, mb = (np.zeros(ng, np.int64) for _ in range(4))
    rc = lib().oracle_simulate_metrics(
        ARCH.get(arch, 0), mode, _ptr(w), 0 if w is None else w.size,
        ctypes.c_void_p(trace.ctypes.data - row_offset * trace.shape[1]), trace.shape[1], L, N, W, cap,
        _ptr(forced), j0, nj, interval, _ptr(cyc), _ptr(ret), _ptr(ret_st), _ptr(mb))
    if rc != 0:
        raise ValueError(f"oracle_simulate_metrics rc={rc}")
    with np.errstate(divide="ignore", invalid="ignore"):
        cpi = np.where(ret > 0, cyc / np.maximum(ret, 1), np.nan)
        bw = np.where(cyc > 0, mb / np.maximum(cyc, 1), np.nan)
    return dict(cycles=cyc, retired=ret, retired_st=ret_st, mem_bytes=mb, cpi=cpi, bw=bw)
