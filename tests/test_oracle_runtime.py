"""Pins of the oracle's runtime-loop model (NEXT-2; §2:
"checks the output quality periodically ... If the quality drops below the
TOQ, it uses a less aggressive approximation"; §5: a check every
40-50 invocations).  The ladder and schedule are DESIGN.md's readings R1-R4;
the tables below are worked by hand from those rules, and the image cases
follow from closed forms (constant images: every candidate is exact;
checkerboards: no approximation keeps 90 %)."""
import numpy as np
import pytest

import workloads as W
from workloads import filters as F

EX = -1  # EXACT in the oracle's ladder

# (training qualities in cost order, TOQ) -> ladder, worked by hand from R1-R2
LADDERS = [
    ([0.85, 0.93, 0.91, 0.97, 0.96, 0.99], 0.90, [1, 3, 5, EX]),   # skip the failing head, keep rises only
    ([0.80, 0.70, 0.89], 0.90, [EX]),                              # nothing passes: exact alone
    ([0.95, 0.95, 0.95], 0.90, [0, EX]),                           # equal is not "less aggressive"
    ([0.50, 0.995, 0.999, 0.998, 1.0], 0.99, [1, 2, 4, EX]),
    ([0.90, 0.89, 0.905], 0.90, [0, 2, EX]),                       # q == TOQ passes (S14)
    ([], 0.90, [EX]),                                              # no candidate (1x1 filter)
]


@pytest.mark.parametrize("q,toq,want", LADDERS)
def test_ladder_hand_table(O, q, toq, want):
    assert O.runtime_ladder(q, toq) == want


def test_trace_hand_table(O):
    # 3 rungs (two approximations + exact), a check every 2nd invocation:
    # t0 checked on rung 0 (0.95 ok); t2 checked on rung 0 (0.85 < 0.9) -> rung 1;
    # t4 checked on rung 1 (0.88) -> exact; exact is never checked again
    q = [[0.95, 0.97, 1], [0.10, 0.10, 1], [0.85, 0.97, 1], [0.10, 0.10, 1],
         [0.50, 0.88, 1], [0.10, 0.10, 1], [0.10, 0.10, 1], [0.10, 0.10, 1]]
    tr = O.runtime_trace(q, 2, 0.90)
    assert tr["rungs"] == [0, 0, 0, 1, 1, 2, 2, 2]
    assert tr["checked"] == [1, 0, 1, 0, 1, 0, 0, 0]
    assert (tr["checks"], tr["backoffs"]) == (3, 2)


def test_trace_special_cases(O):
    q = np.full((10, 4), 0.5)
    q[:, 3] = 1.0
    # no checks: the first rung forever
    tr = O.runtime_trace(q, 0, 0.9)
    assert tr["rungs"] == [0] * 10 and tr["checks"] == 0
    # every invocation checked, every approximation failing: one rung per check
    tr = O.runtime_trace(q, 1, 0.9)
    assert tr["rungs"] == [0, 1, 2] + [3] * 7 and (tr["checks"], tr["backoffs"]) == (3, 3)
    # all passing: never moves, checked on the schedule
    tr = O.runtime_trace(np.ones((9, 4)), 4, 0.9)
    assert tr["rungs"] == [0] * 9 and tr["checked"] == [1, 0, 0, 0, 1, 0, 0, 0, 1] and tr["backoffs"] == 0
    # a failing check at the last approximate rung lands on exact and stays
    q = np.array([[0.1, 1.0]] * 5)
    assert O.runtime_trace(q, 3, 0.9)["rungs"] == [0, 1, 1, 1, 1]


def test_simulate_constant_image_keeps_the_first_candidate(O):
    # a constant image is a fixed point of every normalised candidate: all
    # training qualities are 1, so the ladder is (first candidate, exact) and
    # a check never fails
    train = np.full((2, 40, 48), 120.0, np.float32)
    sim = O.runtime_simulate(train, train, F.mean(5), 0.95, "mre", check_every=1)
    assert [r[:2] for r in sim["ladder"]] == [O.tune_candidates(5, 5)[0], ("exact", 0)]
    assert sim["trace"]["rungs"] == [0, 0] and sim["trace"]["backoffs"] == 0


def test_simulate_checkerboard_backs_off_to_exact(O):
    # natural training frames give a multi-rung ladder; a 16/235 checkerboard
    # breaks the adjacent-similarity premise: every approximate
    # rung's MRE is large, so each check moves one rung down to exact
    train = W.frames(3, 96, 128, 0)
    yy, xx = np.mgrid[0:64, 0:64]
    board = (16.0 + 219.0 * ((yy + xx) % 2)).astype(np.float32)
    frames = np.stack([board] * 8)
    sim = O.runtime_simulate(train, frames, F.mean(5), 0.90, "mre", check_every=1)
    n = len(sim["ladder"])
    assert n >= 3, sim["ladder"]
    q = np.array(sim["q"])
    assert np.all(q[:, :-1] < 0.9)
    assert sim["trace"]["rungs"][:n] == list(range(n)) and sim["trace"]["backoffs"] == n - 1
    # the ladder rises in training quality and starts at the TOQ
    tq = [r[2] for r in sim["ladder"]]
    assert tq[0] >= 0.9 and all(a < b for a, b in zip(tq, tq[1:]))
