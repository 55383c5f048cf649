"""Seeded synthetic inputs shared by the oracle tests and the product path.

This module holds NONE of the method's arithmetic (no queue, clock, gather or
CNN forward).  It only draws:

* instruction traces shaped like the paper's SPEC-like workloads
  (``trace``; PAPER.md:87-89 encoding, SURVEY.md Appendix C recipe; C code in
  trace_gen.c, counter based so any row range regenerates identically);
* random-init SimNet-style CNN weights (``weights``; Kaiming-uniform from a
  splitmix64 counter stream, per-feature input scales folded into conv1, and
  the fc2 head scaled/biased by the committed constants in calibration.json,
  which tools/calibrate.py derives by running the oracle);
* teacher-forced latency triples for the bit-exact stage S1 (``teacher_latencies``).

Weight layout is PyTorch's (conv.weight [Cout][Cin][k], bias, linear.weight
[out][in], bias), layers in order; FC1 columns are position-major (p*C + c).
"""
from __future__ import annotations

import ctypes
import json
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "trace_gen.c")
_LIB = os.path.join(_HERE, "libsynth.so")
ROW_BYTES = 48
NATTR = 47
TRACE_SEED_BASE = 20221113   # trace seed = base + config id
WEIGHT_SEED = 42


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".{os.getpid()}.tmp"
        subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-fPIC", "-shared", "-fopenmp",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def _L():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        _lib.synth_trace.restype = ctypes.c_int
        _lib.synth_trace.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_int64,
                                     ctypes.c_void_p, ctypes.c_long]
    return _lib


def trace_into(out: np.ndarray, seed: int, r0: int = 0) -> np.ndarray:
    """Fill ``out`` ([rows][>=48] uint8, C-contiguous; may be pinned host memory
    viewed through numpy) with trace rows [r0, r0 + rows)."""
    assert out.dtype == np.uint8 and out.ndim == 2 and out.flags.c_contiguous and out.shape[1] >= 48
    rc = _L().synth_trace(seed, r0, r0 + out.shape[0], out.ctypes.data, out.shape[1])
    if rc != 0:
        raise ValueError("synth_trace failed")
    return out


def trace(L: int, seed: int, r0: int = 0) -> np.ndarray:
    """Rows [r0, r0+L) of the synthetic trace with this seed, uint8 [L][48]."""
    return trace_into(np.empty((L, ROW_BYTES), np.uint8), seed, r0)


# ----------------------------------------------------------------------------
# Model shapes (R11).  (kind, cin, cout, k)
# ----------------------------------------------------------------------------
ARCHS = {
    "M2": [("conv", 50, 64, 2), ("conv", 64, 64, 2), ("linear", 28 * 64, 256, 0), ("linear", 256, 3, 0)],
    "C3": [("conv", 50, 64, 2), ("conv", 64, 128, 2), ("conv", 128, 128, 2),
           ("linear", 14 * 128, 256, 0), ("linear", 256, 3, 0)],
    "RB7": [("conv", 50, 64, 2)] + [("conv", 64, 64, 3)] * 6 + [("linear", 56 * 64, 256, 0), ("linear", 256, 3, 0)],
}


def layer_shapes(arch: str):
    """[(weight_shape, bias_shape)] in file order."""
    out = []
    for kind, cin, cout, k in ARCHS[arch]:
        out.append(((cout, cin, k) if kind == "conv" else (cout, cin), (cout,)))
    return out


def nparams(arch: str) -> int:
    return int(sum(np.prod(w) + np.prod(b) for w, b in layer_shapes(arch)))


_M64 = (1 << 64) - 1


def _splitmix_uniform(seed: int, stream: int, n: int) -> np.ndarray:
    """u_i = splitmix64(seed, stream, i) / 2^64 in [0,1), vectorised."""
    base = (seed * 0x9E3779B97F4A7C15 + stream * 0xD1B54A32D192ED03) & _M64
    with np.errstate(over="ignore"):
        z = np.uint64(base) + (np.arange(1, n + 1, dtype=np.uint64) * np.uint64(0x9E3779B97F4A7C15))
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return (z >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)


# Typical magnitude of each of the 50 input columns; its inverse is folded into
# conv1 so the random network sees O(1) inputs (columns 0-2: time features).
FEATURE_SCALE = np.array(
    [16.0, 16.0, 16.0,          # age, rem_complete, rem_retire
     8.0] + [1.0] * 10 +         # op class, 10 flags
    [2.0, 2.0, 1.0, 2.0, 2.0, 1.0, 4.0] +   # fetch lvl, itlb, fwb, data lvl, dtlb, dwb, st-ld dist
    [48.0] * 14 +                # 8 src + 6 dst registers
    [1.0, 1.0, 2.0] + [1.0] * 12, dtype=np.float64)
assert FEATURE_SCALE.size == 50


# Completion-latency floor of the synthetic head (R21): the completion row of
# fc2 is drawn non-negative and its bias is COMPLETE_BIAS > 0.5, so y_c = COMPLETE_BIAS +
# a sum of non-negative terms (ReLU outputs x non-negative weights) and every rounded
# completion latency is >= 1.  Every pushed entry then lives at least one cycle, so a
# Clock that does not advance grows the queue by one entry per instruction and the
# ROB-full stall (R5) advances it within Context_length instructions: the random-weight
# model has no frozen-Clock fixed point (round 1 found one at row ~3.3M of the config-4
# trace: f = c = s = 0 with an unchanging context for millions of rows).
# Applied to the models of the long-running configs (C3: configs 2-4, RB7: config 5).  M2
# (config 1: 10k rows, one sub-trace) keeps a signed completion row: with the floor its
# small network has a positive feedback through the time features (completions run away
# to the 4095 clamp within ~1k rows), and config 1 is short.
FLOOR_OUTPUT = 1
COMPLETE_BIAS = 0.75
FLOOR_ARCHS = ("C3", "RB7")


def calibration(arch: str):
    path = os.path.join(_HERE, "calibration.json")
    if os.path.exists(path):
        with open(path) as f:
            cal = json.load(f)
        if arch in cal:
            return np.array(cal[arch]["gain"], np.float64), np.array(cal[arch]["bias"], np.float64)
    return np.ones(3), np.zeros(3)


def prune24(w: np.ndarray, kind: str) -> np.ndarray:
    """2:4 magnitude pruning of one tensor-core layer (R22; the paper prunes its
    trained model for 2:4 structured sparsity): in every group of 4
    consecutive inputs along the reduction dimension -- input channels of one conv tap
    (PyTorch [Cout][Cin][k]: w[o, 4g:4g+4, t]), or 4 consecutive flattened inputs of a
    linear layer -- keep the 2 largest magnitudes (ties: the lower index), zero the rest.
    This is model preparation (an input both the oracle and the GPU load unchanged), not
    part of the simulation."""
    w = np.array(w, dtype=np.float64, copy=True)
    if kind == "conv":
        cout, cin, k = w.shape
        v = np.moveaxis(w, 2, 1)                      # [Cout][k][Cin]
    else:
        cout, cin = w.shape
        v = w[:, None, :]                             # [Cout][1][Cin]
    pad = (-cin) % 4
    vp = np.concatenate([v, np.zeros(v.shape[:2] + (pad,))], axis=2) if pad else v
    g = vp.reshape(vp.shape[0], vp.shape[1], -1, 4)
    order = np.argsort(-np.abs(g), axis=3, kind="stable")
    keep = np.zeros_like(g, dtype=bool)
    np.put_along_axis(keep, order[..., :2], True, axis=3)
    g = np.where(keep, g, 0.0)
    vp = g.reshape(vp.shape)[:, :, :cin]
    return np.moveaxis(vp, 1, 2) if kind == "conv" else vp[:, 0, :]


def weights(arch: str = "C3", seed: int = WEIGHT_SEED, *, gain=None, bias=None, sparse24: bool = False) -> np.ndarray:
    """Flat fp32 weight vector for ``arch`` (PyTorch layouts, layers in order).  With
    ``sparse24`` every tensor-core layer (all but the fc2 head) is 2:4 magnitude-pruned
    (prune24) and the head uses its own calibration entry ``<arch>:24``."""
    if gain is None or bias is None:
        g0, b0 = calibration(arch + (":24" if sparse24 else ""))
        gain = g0 if gain is None else np.asarray(gain, np.float64)
        bias = b0 if bias is None else np.asarray(bias, np.float64)
    parts = []
    shapes = layer_shapes(arch)
    for li, (ws, bs) in enumerate(shapes):
        fan_in = int(np.prod(ws[1:]))
        bound = np.sqrt(6.0 / fan_in)                       # Kaiming-uniform, ReLU gain
        w = (2.0 * _splitmix_uniform(seed, 2 * li, int(np.prod(ws))) - 1.0) * bound
        w = w.reshape(ws)
        b = (2.0 * _splitmix_uniform(seed, 2 * li + 1, bs[0]) - 1.0) / np.sqrt(fan_in)
        if li == 0:
            w = w / FEATURE_SCALE[None, :, None]
        if sparse24 and li < len(shapes) - 1:                # tensor-core layers only (not the fc2 head)
            w = prune24(w, "conv" if len(ws) == 3 else "linear")
        if li == len(shapes) - 1:                            # calibrated head
            if arch in FLOOR_ARCHS:
                w[FLOOR_OUTPUT] = np.abs(w[FLOOR_OUTPUT])    # completion row non-negative (R21)
            w = w * gain[:, None] / np.sqrt(3.0)
            b = bias.copy()
            if arch in FLOOR_ARCHS:
                b[FLOOR_OUTPUT] = COMPLETE_BIAS
        parts += [w.ravel(), b.ravel()]
    out = np.concatenate(parts).astype(np.float32)
    assert out.size == nparams(arch)
    return out


def teacher_latencies(L: int, seed: int, *, f_mean: float = 1.0, c_mean: float = 20.0,
                      s_mean: float = 2.0, big: float = 0.0) -> np.ndarray:
    """Seeded (f, c, s) uint16 [L][3] for teacher forcing (stage S1).

    Geometric-ish draws; ``big`` > 0 sprinkles latencies up to 4095 to
    exercise clamps and long-lived entries."""
    u = _splitmix_uniform(seed, 777, 4 * L).reshape(L, 4)
    f = np.floor(-np.log1p(-u[:, 0]) * f_mean)
    c = np.floor(-np.log1p(-u[:, 1]) * c_mean)
    s = np.floor(-np.log1p(-u[:, 2]) * s_mean)
    if big > 0:
        m = u[:, 3] < big
        c = np.where(m, np.floor(u[:, 3] / big * 4095), c)
    lat = np.stack([f, c, s], 1)
    return np.clip(lat, 0, 4095).astype(np.uint16)
