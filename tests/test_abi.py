"""The C-ABI library loads and exports every symbol include/psim.h declares
(no compute calls: this runs on the CPU-only box), and the host-only
partition helper agrees with the oracle's partition."""
import ctypes
import os
import re

import numpy as np
import pytest

import oracle
import paper_conf_sc_pandeylfhl22_b200 as P

HEADER = os.path.join(os.path.dirname(__file__), "..", "include", "psim.h")


def declared():
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(psim_[a-z_]+)\s*\(", txt)))


def test_header_symbols_exported():
    lib = ctypes.CDLL(P.LIB_PATH)
    names = declared()
    assert len(names) >= 15
    for n in names:
        assert hasattr(lib, n), n
    assert set(names) == set(P.EXPORTS)


def test_library_is_sm100a():
    out = os.popen(f"cuobjdump --list-elf {P.LIB_PATH} 2>&1").read()
    assert "sm_100a" in out


def test_version_and_create_without_gpu():
    assert "sm_100a" in P.version()
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(P.PsimError):        # fails loudly: no device, no fallback
        P.Simulator()


@pytest.mark.parametrize("L,N,W,G", [(1000, 7, 13, 3), (100, 100, 5, 4), (10**8, 65536, 110, 8),
                                      (10**6, 1024, 1000, 2), (50, 3, 0, 1)])
def test_partition_range_matches_oracle(L, N, W, G):
    s, e, ws = oracle.partition(L, N, W) if L <= 10**7 else (None, None, None)
    covered = 0
    for g in range(G):
        rr = P.partition_range(L, N, W, g, G)
        assert rr.j0 == g * N // G and rr.j1 == (g + 1) * N // G
        covered += rr.j1 - rr.j0
        if s is not None and rr.j1 > rr.j0:
            assert rr.row_lo == ws[rr.j0:rr.j1].min() and rr.row_hi == e[rr.j1 - 1]
            assert rr.steps == int((e[rr.j0:rr.j1] - ws[rr.j0:rr.j1]).max())
    assert covered == N


def test_partition_range_errors():
    with pytest.raises(P.PsimError):
        P.partition_range(10, 0, 0)
    with pytest.raises(P.PsimError):
        P.partition_range(10, 11, 0)
