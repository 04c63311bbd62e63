"""Pins for the oracle's reaching-distance index map.

The hand table (tests/golden/index_map.txt) is derived from the paper's text,
not from code; the properties are the ones the paper's rule implies."""
import os

import numpy as np
import pytest

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "index_map.txt")


def _rows():
    out = []
    for line in open(GOLDEN):
        line = line.split("#")[0].strip()
        if line:
            v = [int(t) for t in line.split()]
            out.append((v[0], v[1], v[2:]))
    return out


@pytest.mark.parametrize("r,d,expect", _rows())
def test_hand_table(O, r, d, expect):
    m = O.index_map(r, d)
    assert list(m[r:]) == expect
    assert list(m[:r + 1]) == [-v for v in expect[::-1]]


@pytest.mark.parametrize("r", range(0, 9))
@pytest.mark.parametrize("d", range(0, 11))
def test_properties(O, r, d):
    m = O.index_map(r, d)
    i = np.arange(-r, r + 1)
    # "neighbors, whose distances from the accessed element are less than [or
    # equal to] the reaching distance, will not be accessed" (L1202-1208, S2)
    assert np.all(np.abs(m - i) <= d)
    assert m[r] == 0                          # the centre is accessed (L1198-1202)
    assert np.all(m[::-1] == -m)              # symmetric tile
    assert np.all(m[m + r] == m)              # an accessed element stands for itself
    assert np.all(np.abs(m) <= r)             # stays inside the tile
    if d == 0:
        assert np.all(m == i)                 # reach 0 = exact
    if d >= r:
        assert np.all(m == 0)                 # full collapse onto the centre
    # monotone: a farther neighbour never maps closer to the centre
    assert np.all(np.diff(m) >= 0)


def test_reach_saturates(O):
    for r in range(0, 6):
        assert list(O.index_map(r, r + 3)) == list(O.index_map(r, max(r, 0)))


def test_scheme_reaches(O):
    assert O.scheme_reaches("exact", 3) == (0, 0)
    assert O.scheme_reaches("row", 2) == (2, 0)
    assert O.scheme_reaches("col", 2) == (0, 2)
    assert O.scheme_reaches("center", 1) == (1, 1)


def test_rejects_bad_args(O):
    with pytest.raises(ValueError):
        O.index_map(-1, 0)
    with pytest.raises(ValueError):
        O.index_map(2, -1)
