"""Partition pins (Fig. 5; warm-up :197; R8/R9)."""
import numpy as np
import pytest

import oracle


def test_fig5_six_instructions_three_subtraces():
    # "the six-instruction trace is partitioned into three sub-traces with two
    # instructions in each partition"
    s, e, ws = oracle.partition(6, 3, 0)
    assert list(zip(s, e)) == [(0, 2), (2, 4), (4, 6)]
    assert list(ws) == [0, 2, 4]
    s, e, ws = oracle.partition(6, 3, 1)          # W = 1: one warm-up row before each
    assert list(ws) == [0, 1, 3]


@pytest.mark.parametrize("L,N,W", [(10, 3, 4), (1000003, 65536, 110), (17, 17, 0), (5, 1, 9),
                                    (10**8, 65536, 1000)])
def test_partition_covers_disjoint_balanced(L, N, W):
    s, e, ws = oracle.partition(L, N, W)
    assert s[0] == 0 and e[-1] == L
    assert np.all(e[:-1] == s[1:])                 # disjoint, contiguous
    sizes = e - s
    assert sizes.min() >= 1 and sizes.max() - sizes.min() <= 1
    assert np.all(ws == np.maximum(0, s - W)) and ws[0] == 0


def test_partition_errors():
    with pytest.raises(ValueError):
        oracle.partition(10, 0, 0)
    with pytest.raises(ValueError):
        oracle.partition(10, 11, 0)
    with pytest.raises(ValueError):
        oracle.partition(10, 2, -1)
