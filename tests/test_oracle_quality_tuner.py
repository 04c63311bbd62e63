"""Pins for the oracle's quality metrics and TOQ tuner.

Quality: closed forms (A = E(1+delta) -> MRE = L2 = delta; A = E -> 1; PSNR
of a constant offset).  Tuner: the candidate order against the hand-derived
golden table, and decisions fixed by construction (T-pins 1-3)."""
import math
import os

import numpy as np
import pytest

import workloads as W
from workloads import filters as F

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "tune_order.txt")


@pytest.mark.parametrize("delta", [0.0, 0.01, 0.1, 0.37])
def test_quality_closed_forms(O, delta):
    rng = np.random.default_rng(0)
    e = rng.uniform(16, 235, size=1000)
    a = e * (1.0 + delta)
    assert O.quality(e, a, "mre") == pytest.approx(1.0 - delta, abs=1e-14)
    assert O.quality(e, a, "l2") == pytest.approx(1.0 - delta, abs=1e-14)
    # sign-alternating error: same MRE, same L2
    a2 = e * (1.0 + delta * np.where(np.arange(1000) % 2 == 0, 1, -1))
    assert O.quality(e, a2, "mre") == pytest.approx(1.0 - delta, abs=1e-14)
    assert O.quality(e, a2, "l2") == pytest.approx(1.0 - delta, abs=1e-14)


def test_quality_mre_mixed_and_zero_guard(O):
    e = np.array([10.0, 20.0, 0.0, 0.0])
    a = np.array([11.0, 18.0, 0.0, 5.0])
    # terms 0.1, 0.1, 0 (A = E = 0), 1 (E = 0, A != 0)  -> mean 0.3
    assert O.quality(e, a, "mre") == pytest.approx(0.7, abs=1e-15)
    # L2: sqrt((1 + 4 + 0 + 25) / (100 + 400))
    assert O.quality(e, a, "l2") == pytest.approx(1.0 - math.sqrt(30 / 500), abs=1e-15)


def test_psnr(O):
    e = np.full(100, 50.0)
    for c in (1.0, 2.5, 10.0):
        assert O.quality(e, e + c, "psnr") == pytest.approx(20 * math.log10(255.0 / c), abs=1e-12)
    assert O.quality(e, e, "psnr") == math.inf


def _golden():
    out = []
    for line in open(GOLDEN):
        line = line.split("#")[0].strip()
        if not line:
            continue
        head, tail = line.split(":", 1)
        ky, kx, sep = (int(t) for t in head.split())
        order = [(t.split(":")[0], int(t.split(":")[1])) for t in tail.split()]
        out.append((ky, kx, bool(sep), order))
    return out


@pytest.mark.parametrize("ky,kx,sep,order", _golden())
def test_candidate_order(O, ky, kx, sep, order):
    assert O.tune_candidates(ky, kx, sep) == order


def test_candidates_1d_filters(O):
    # a 1 x K filter has no rows to substitute: only one axis is approximable
    c = O.tune_candidates(1, 5)
    assert [s for s, _ in c] == ["center", "center"]
    assert O.tune_candidates(1, 1) == []


@pytest.mark.parametrize("k", [3, 5, 9])
def test_tpin1_y_constant_picks_row(O, k):
    """y-constant image that varies in x: only row schemes reproduce the exact
    output, so the answer is (row, r), right after the centre full collapse."""
    x = np.repeat(W.image(1, 64, 3), 48, axis=0)[None]
    x = np.concatenate([x, np.repeat(W.image(1, 64, 4), 48, axis=0)[None]])
    w = F.gaussian(k) if k != 9 else F.conv(9)
    r = k // 2
    res = O.tune(x, w, toq=1.0 - 1e-6, metric="mre")
    assert (res["scheme"], res["reach"]) == ("row", r)
    assert res["quality"] >= 1.0 - 1e-6


@pytest.mark.parametrize("k", [3, 5, 9])
def test_tpin2_constant_picks_full_collapse(O, k):
    x = np.full((2, 32, 32), 120.0, dtype=np.float32)
    w = F.gaussian(k) if k != 9 else F.conv(9)
    res = O.tune(x, w, toq=1.0 - 1e-6, metric="l2")
    assert (res["scheme"], res["reach"]) == ("center", k // 2)


@pytest.mark.parametrize("w,metric", [(F.gaussian(3), "mre"), (F.mean(5), "mre"), (F.conv(9), "l2")])
def test_tpin3_noise_falls_back_to_exact(O, w, metric):
    x = W.uniform_noise(128, 128, 5)[None]
    res = O.tune(x, w, toq=0.95, metric=metric, all_qualities=True)
    assert res["scheme"] == "exact" and res["reach"] == 0 and res["quality"] == 1.0
    assert max(res["qualities"]) < 0.95


def test_tuner_monotone_in_toq(O):
    """A stricter TOQ never picks a candidate earlier in cost order."""
    x = W.frames(2, 96, 96, 11)
    w = F.mean(5)
    order = [("center", 2), ("row", 2), ("col", 2), ("center", 1), ("row", 1), ("col", 1)]
    pos = []
    for toq in (0.5, 0.8, 0.9, 0.95, 0.99, 0.999):
        r = O.tune(x, w, toq=toq, metric="mre")
        pos.append(len(order) if r["scheme"] == "exact" else order.index((r["scheme"], r["reach"])))
        assert r["quality"] >= toq
    assert pos == sorted(pos)


def test_tuner_reports_first_passing(O):
    x = W.frames(2, 64, 64, 20)
    w = F.mean(5)
    r = O.tune(x, w, toq=0.9, metric="mre", all_qualities=True)
    qs = r["qualities"]
    cands = O.tune_candidates(5, 5)
    k = next(i for i, q in enumerate(qs) if q >= 0.9)
    assert (r["scheme"], r["reach"]) == cands[k]
    assert r["quality"] == qs[k]
