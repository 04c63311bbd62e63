"""Full-size parity of the tuner (row a5) and the quality reduction (row a4)
on the training sets the bench itself tunes on (bench.py: `W.frames(tn, th,
tw, 0)` at rank 0 -- c2 10 x 4096^2 mean 5x5 MRE, c3 10 x 2160x3840 separable
7x7 L2, c4 2 x 4096^2 conv 9x9 L2).

At these sizes every level of the GPU reduction runs: the fused tile
kernels walk several bounded-persistence waves (c2: 20 480 tiles against
~7 100 per wave), each CTA writes one partial pair, and the partial pairs
(41 k at c2) pass through the fold level of `launch_quality_final` before the
final CTA.  Three comparisons per workload:

1. per-candidate quality from the fused tuner partials vs the oracle tuner's
   qualities (`oracle.tune(..., all_qualities=True)`: fp64 stencils rounded
   to fp32, fp64 quality) within QTOL, and the decisions at TOQ 0.80, 0.90,
   0.95, 0.99 identical (train on the first 10 runs and
   keep the first kernel meeting the TOQ; L572-592);
2. the same fused partials vs `oracle.quality` on the GPU's own stored fp32
   outputs (exact and candidate) within RTOL_REDUCTION: isolates the
   reduction, whose only difference from the oracle is the fp64 summation
   order (a tree on the GPU, rows in sequence in the oracle: typically
   sqrt(N) 2^-53 ~ 1e-12 relative at N = 8.3e7 - 1.7e8 terms; measured
   1.26e-12 on c3's L2), so RTOL_REDUCTION = 1e-11;
3. `paraprox_quality` (the unfused a4 kernel) vs `oracle.quality` on the same
   stored outputs within RTOL_REDUCTION.

QTOL: the two sides do not compute the same fp32 outputs.  The GPU applies
the plan's folded weights w' = fp32(sum of the substituted taps), each
rounded once (relative error <= 2^-24, the same sign at every pixel, so it
does not average out), and sums taps in fp32; the oracle substitutes
literally in fp64 and rounds the output once.  Measured on these training
sets (r02): 1.3e-9 (c2), 2.6e-9 (c3), 1.9e-9 (c4), in line with SURVEY
8(c)'s 1e-10 - 2e-9 at 256^2.  QTOL = 1e-8 bounds that with margin; a
decision can flip only when |q - TOQ| < QTOL; the minimum margin is printed)."""
import numpy as np
import pytest
import torch

import workloads as W
from workloads import filters as F

pytestmark = pytest.mark.gpu

QTOL = 1e-8
RTOL_REDUCTION = 1e-11
TOQS = (0.80, 0.90, 0.95, 0.99)

# name: (frames, h, w, filter, metric) -- bench.py WORKLOADS / tuner training set
CASES = {
    "c2": (10, 4096, 4096, "mean5", "mre"),
    "c3": (10, 2160, 3840, "sep7", "l2"),
    "c4": (2, 4096, 4096, "conv9", "l2"),
}


@pytest.fixture(scope="module")
def P():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_asplos_samadijlm14_b200 as pkg

    return pkg.paraprox


def _filter(P, name):
    kind, w = F.named(name)
    return (P.Filter(wy=w[0], wx=w[1]) if kind == "sep" else P.Filter(w)), (tuple(w) if kind == "sep" else w)


def _decide(cands, qs, toq):
    """The tuner's rule on a list of qualities in cost order."""
    for c, q in zip(cands, qs):
        if q >= toq:
            return c
    return ("exact", 0)


@pytest.mark.parametrize("cfg", sorted(CASES))
def test_tuner_and_quality_at_bench_size(P, O, cfg):
    n, h, w, fname, metric = CASES[cfg]
    x = W.frames(n, h, w, 0)
    f, warr = _filter(P, fname)
    xd = torch.from_numpy(x).cuda()
    cands = P.tune_candidates(f)

    # (1) fused tuner partials vs the oracle tuner
    parts = P.tune_partials(xd, f, metric)
    qg = [P.quality_from_partials(parts[3 * k:3 * k + 3], metric) for k in range(len(cands))]
    ref = O.tune(x, warr, 0.90, metric, all_qualities=True)
    qo = ref["qualities"]
    assert len(qo) == len(cands)
    assert O.tune_candidates(f.ky, f.kx, f.separable) == cands
    dq = np.abs(np.array(qg) - np.array(qo))
    margin = min(abs(q - t) for q in qo for t in TOQS)
    print(f"{cfg}: max |q_gpu - q_oracle| = {dq.max():.3e} over {len(cands)} candidates; "
          f"min |q - TOQ| = {margin:.3e}")
    assert dq.max() <= QTOL, (cfg, list(zip(cands, qg, qo)))
    assert P.tune(xd, f, 0.90, metric)[:2] == (ref["scheme"], ref["reach"])
    for toq in TOQS:
        got = P.tune(xd, f, toq, metric)
        assert got[:2] == _decide(cands, qo, toq), (cfg, toq, got)
        assert P.tune_decide(f, parts, toq, metric) == got

    # (2) + (3) the reduction alone, on the GPU's stored outputs
    e = P.stencil_exact(xd, f)
    en = e.cpu().numpy()
    for k, (scheme, reach) in enumerate(cands):
        a = P.stencil_approx(xd, f, scheme, reach)
        an = a.cpu().numpy()
        q_or = O.quality(en, an, metric)
        assert abs(qg[k] - q_or) <= RTOL_REDUCTION * max(1.0, abs(q_or)), (cfg, scheme, reach, qg[k], q_or)
        if k in (0, len(cands) - 1):  # the unfused a4 kernel, fold level included
            q_un = P.quality(e, a, metric)
            assert abs(q_un - q_or) <= RTOL_REDUCTION * max(1.0, abs(q_or)), (cfg, scheme, reach, q_un, q_or)
        del a, an
