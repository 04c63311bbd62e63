"""Multi-GPU orchestration of the stencil hot path (DESIGN.md
"Multi-GPU").  One process per GPU, torch.distributed (NCCL over NVLink /
NVSwitch) for the plumbing.  The paper is single-device; the decompositions
below are this build's.

* P1 frame sharding: independent frames split across ranks, no data-path
  collective (``frame_shard``).  Pooled tuning / quality all-reduce three fp64
  partial sums per candidate (``tune_pooled``, ``quality_pooled``), so every
  rank reaches the identical decision with no broadcast.
* P2 row stripes of one large image: rank k owns rows [r0, r1) and keeps
  ``halo`` rows above and below; one halo exchange per step with the two
  neighbours (``exchange_halos``, batch_isend_irecv) overlapped with the
  interior rows, then the two boundary bands (``stencil_stripe``).  The
  approximation shrinks the halo to the largest accessed row offset h_y; the
  row and centre schemes at full reach have h_y = 0 and need no exchange.
  Edge ranks clamp at the true image edge (halo_top / halo_bottom = 0).

All compute goes through the C ABI binding (``paraprox``); the ``compute``
hook of ``stencil_stripe`` exists only so the exchange logic can be tested on
CPU with the gloo backend against the oracle (tests/test_dist_gloo.py).
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np
import torch
import torch.distributed as dist


def frame_shard(n: int, world: int, rank: int):
    """Frames [f0, f1) of rank `rank` (contiguous, sizes differ by <= 1)."""
    f0 = n * rank // world
    f1 = n * (rank + 1) // world
    return f0, f1


@dataclass
class Stripe:
    r0: int          # first owned row (global)
    r1: int          # one past the last owned row
    cap: int         # halo capacity allocated above and below
    h: int           # global image rows

    @property
    def rows(self) -> int:
        return self.r1 - self.r0

    def halo_top(self, hy: int) -> int:
        """Valid halo rows above the stripe for a plan with halo hy."""
        return min(hy, self.r0)

    def halo_bottom(self, hy: int) -> int:
        return min(hy, self.h - self.r1)


def stripe_of(h: int, world: int, rank: int, cap: int) -> Stripe:
    r0 = h * rank // world
    r1 = h * (rank + 1) // world
    return Stripe(r0, r1, cap, h)


def alloc_stripe(s: Stripe, w: int, device=None, dtype=torch.float32) -> torch.Tensor:
    """[cap + rows + cap, w] buffer; owned rows at [cap, cap + rows)."""
    return torch.empty((s.cap + s.rows + s.cap, w), dtype=dtype, device=device)


def exchange_halos(buf: torch.Tensor, s: Stripe, hy: int, group=None, async_op: bool = False):
    """Send the top hy owned rows to rank-1 and the bottom hy owned rows to
    rank+1; receive their boundary rows into this stripe's halos.  Rows are
    contiguous, so every message is one contiguous tensor (no pack kernel).
    Returns the list of requests (async_op) or waits for them."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    if hy <= 0 or world == 1:
        return []
    if hy > s.cap:
        raise ValueError("halo larger than the allocated capacity")
    if s.rows < hy:
        raise ValueError("stripe thinner than the halo")
    c, n = s.cap, s.rows
    if buf.is_cuda and dist.get_backend(group) == "gloo":
        # gloo moves host tensors only: stage the halo rows through host memory
        # (the multi-process tests on single-GPU boxes); NCCL sends device rows
        host = buf.new_empty(buf.shape, device="cpu")
        for r0, r1 in ((c, c + hy), (c + n - hy, c + n)):
            host[r0:r1].copy_(buf[r0:r1])
        exchange_halos(host, s, hy, group, async_op=False)
        if rank > 0:
            buf[c - hy:c].copy_(host[c - hy:c])
        if rank < world - 1:
            buf[c + n:c + n + hy].copy_(host[c + n:c + n + hy])
        return []
    ops = []
    if rank > 0:
        peer = dist.get_global_rank(group, rank - 1) if group is not None else rank - 1
        ops.append(dist.P2POp(dist.isend, buf[c:c + hy], peer, group))
        ops.append(dist.P2POp(dist.irecv, buf[c - hy:c], peer, group))
    if rank < world - 1:
        peer = dist.get_global_rank(group, rank + 1) if group is not None else rank + 1
        ops.append(dist.P2POp(dist.isend, buf[c + n - hy:c + n], peer, group))
        ops.append(dist.P2POp(dist.irecv, buf[c + n:c + n + hy], peer, group))
    reqs = dist.batch_isend_irecv(ops)
    if async_op:
        return reqs
    for r in reqs:
        r.wait()
    return []


def _band(buf, s: Stripe, y0: int, y1: int, top: int, bottom: int):
    """View of owned rows [y0, y1) with `top` valid rows above and `bottom`
    below, as (tensor including halos, halo_top, halo_bottom)."""
    c = s.cap
    return buf[c + y0 - top:c + y1 + bottom], top, bottom


def scheme_xy(scheme, reach: int):
    """Per-axis reaches (d_y, d_x) of a scheme (O4)."""
    dy = {"exact": 0, "row": reach, "col": 0, "center": reach, "centre": reach}[scheme]
    dx = {"exact": 0, "row": 0, "col": reach, "center": reach, "centre": reach}[scheme]
    return dy, dx


def stencil_stripe(buf: torch.Tensor, s: Stripe, f, scheme, reach: int, out: torch.Tensor,
                   group=None, compute=None, hy: int | None = None):
    """One row-stripe step: halo exchange overlapped with the interior rows,
    then the boundary bands.  `out` is [rows, w].  `compute(band, ht, hb,
    out_rows)` defaults to the CUDA stencil through the C ABI."""
    if compute is None:
        from . import paraprox as P

        def compute(band, ht, hb, o):
            P.stencil_approx(band, f, scheme, reach, out=o, halo_top=ht, halo_bottom=hb)
    if hy is None:
        hy = f.plan_info(*scheme_xy(scheme, reach))["halo_y"]
    n = s.rows
    ht, hb = s.halo_top(hy), s.halo_bottom(hy)
    if hy == 0 or n <= 2 * hy:
        exchange_halos(buf, s, hy, group)
        band, t, b = _band(buf, s, 0, n, ht, hb)
        compute(band, t, b, out)
        return out
    reqs = exchange_halos(buf, s, hy, group, async_op=True)
    # interior rows [hy, n - hy): every input row they read is owned
    band, t, b = _band(buf, s, hy, n - hy, hy, hy)
    compute(band, t, b, out[hy:n - hy])
    for r in reqs:
        r.wait()
    # boundary bands: the top hy rows read the received top halo, and so on
    band, t, b = _band(buf, s, 0, hy, ht, min(hy, n - hy))
    compute(band, t, b, out[0:hy])
    band, t, b = _band(buf, s, n - hy, n, min(hy, n - hy), hb)
    compute(band, t, b, out[n - hy:n])
    return out


def hotspot_stripes(bufs, power: torch.Tensor, s: Stripe, params, scheme, reach: int, iterations: int,
                    group=None, compute=None):
    """`iterations` HotSpot steps (NEXT-4) of a row-striped grid: before each
    step the stripe exchanges the h_y halo rows of the current temperature
    with its neighbours (exact and column schemes read the north/south
    neighbours: h_y = 1; the row and centre schemes at reach >= 1 read only
    the centre row: h_y = 0, no exchange at all), overlapped with the interior
    rows; then the boundary rows.  `bufs` = two [cap + rows + cap, w] buffers,
    the initial temperature in bufs[0]'s owned rows; `power` = [rows, w].
    Returns the buffer holding the final owned rows.  `compute(band, ht, hb,
    power_rows, out_rows)` defaults to one paraprox_hotspot step."""
    if compute is None:
        from . import paraprox as P

        def compute(band, ht, hb, pw, o):
            P.hotspot(band, pw, params, scheme, reach, 1, out=o, halo_top=ht, halo_bottom=hb)
    hy = 1 if (scheme == "exact" or reach == 0 or scheme in ("col", "column")) else 0
    n, c = s.rows, s.cap
    ht, hb = s.halo_top(hy), s.halo_bottom(hy)
    cur, nxt = bufs
    for _ in range(iterations):
        out = nxt[c:c + n]
        if hy == 0 or n <= 2 * hy:
            exchange_halos(cur, s, hy, group)
            band, t, b = _band(cur, s, 0, n, ht, hb)
            compute(band, t, b, power, out)
        else:
            reqs = exchange_halos(cur, s, hy, group, async_op=True)
            band, t, b = _band(cur, s, hy, n - hy, hy, hy)
            compute(band, t, b, power[hy:n - hy], out[hy:n - hy])
            for r in reqs:
                r.wait()
            band, t, b = _band(cur, s, 0, hy, ht, min(hy, n - hy))
            compute(band, t, b, power[0:hy], out[0:hy])
            band, t, b = _band(cur, s, n - hy, n, min(hy, n - hy), hb)
            compute(band, t, b, power[n - hy:n], out[n - hy:n])
        cur, nxt = nxt, cur
    return cur


class PeerStripe:
    """A row stripe whose neighbours' boundary rows are read inside the
    stencil kernel through CUDA IPC mappings of their buffers (NVLink P2P on
    one node) -- the halo exchange without a separate collective (§8(e)).

    Every rank allocates its owned rows `buf` ([rows, w], device), exports it,
    and opens the handles of ranks k-1 and k+1 (handles travel once through
    torch.distributed's object collectives).  After the ranks have written
    their inputs, one barrier orders those writes before the reads;
    `stencil()` then needs no communication at all."""

    def __init__(self, s: Stripe, w: int, device, group=None):
        from . import paraprox as P
        self.P = P
        self.s = s
        self.w = w
        self.buf = torch.empty((s.rows, w), dtype=torch.float32, device=device)
        handle, off = P.ipc_export(self.buf)
        world = dist.get_world_size(group)
        rank = dist.get_rank(group)
        infos = [None] * world
        dist.all_gather_object(infos, (handle, off, s.rows, self.buf.stride(0)), group=group)
        self._opened = []
        self.top = self.bot = None
        self.top_rows = self.bot_rows = 0
        self.top_pitch = self.bot_pitch = w
        if rank > 0:
            h, o, rows, pitch = infos[rank - 1]
            base = P.ipc_open(h)
            self._opened.append(base)
            self.top, self.top_rows, self.top_pitch = base + o, rows, pitch
        if rank < world - 1:
            h, o, rows, pitch = infos[rank + 1]
            base = P.ipc_open(h)
            self._opened.append(base)
            self.bot, self.bot_rows, self.bot_pitch = base + o, rows, pitch
        if self.top_pitch != self.bot_pitch and self.top is not None and self.bot is not None:
            raise ValueError("neighbour pitches differ")
        self.group = group

    def ready(self):
        """Order every rank's writes of its `buf` before the peers' reads."""
        torch.cuda.synchronize()
        dist.barrier(group=self.group)

    def stencil(self, f, scheme, reach: int, out: torch.Tensor):
        pitch = self.top_pitch if self.top is not None else self.bot_pitch
        hy = f.plan_info(*scheme_xy(scheme, reach))["halo_y"]
        for rows in (self.top_rows, self.bot_rows):
            if 0 < rows < hy:
                raise ValueError("stripe thinner than the halo")
        return self.P.stencil_peer(self.buf, f, scheme, reach, out=out, top=self.top, top_rows=self.top_rows,
                                   bot=self.bot, bot_rows=self.bot_rows, src_pitch=pitch)

    def close(self):
        # every rank's kernels that read a neighbour's buf over the mapping
        # finish before any rank unmaps or frees
        torch.cuda.synchronize()
        dist.barrier(group=self.group)
        for base in self._opened:
            self.P.ipc_close(base)
        self._opened = []


class HotspotPeerStripes:
    """HotSpot (NEXT-4) on row stripes with the halo exchange inside the
    kernel: each rank keeps two temperature buffers, its power rows and a
    pass counter in CUDA-IPC-exported memory.  A pass of up to 8 steps reads
    the neighbours' boundary rows (8 x h_y of them) straight from their
    buffers over NVLink, after a device-side wait for their previous pass
    (paraprox_flag_wait on the neighbours' counters), then publishes its own
    counter -- no host synchronisation and no collective between passes.
    The ordering rule: before pass q every rank waits until its neighbours
    have finished pass q - 1, which both makes their rows ready and keeps
    them from overwriting rows still being read."""

    def __init__(self, s: Stripe, w: int, device, group=None):
        from . import paraprox as P
        self.P = P
        self.s = s
        self.w = w
        self.group = group
        self.T = [torch.empty((s.rows, w), dtype=torch.float32, device=device) for _ in range(2)]
        self.Pw = torch.empty((s.rows, w), dtype=torch.float32, device=device)
        self.flag = torch.zeros(2, dtype=torch.int64, device=device)
        mine = [P.ipc_export(t) for t in (self.T[0], self.T[1], self.Pw, self.flag)]
        world = dist.get_world_size(group)
        rank = dist.get_rank(group)
        infos = [None] * world
        dist.all_gather_object(infos, (mine, s.rows, self.T[0].stride(0)), group=group)
        self._opened = []
        self.nb = {}
        for side, peer in (("top", rank - 1), ("bot", rank + 1)):
            if 0 <= peer < world:
                handles, rows, pitch = infos[peer]
                ptrs = []
                for h, off in handles:
                    base = P.ipc_open(h)
                    self._opened.append(base)
                    ptrs.append(base + off)
                self.nb[side] = dict(T=ptrs[:2], P=ptrs[2], flag=ptrs[3], rows=rows, pitch=pitch)
        self.passes = 0

    def load(self, temp_rows: torch.Tensor, power_rows: torch.Tensor):
        """Owned rows of the initial temperature and the power; then every
        rank's writes are ordered before the peers' reads."""
        self.T[0].copy_(temp_rows)
        self.Pw.copy_(power_rows)
        self.flag.zero_()
        self.passes = 0
        torch.cuda.synchronize()
        dist.barrier(group=self.group)

    def run(self, params, scheme, reach: int, iterations: int):
        """`iterations` steps; returns the buffer holding the result."""
        P = self.P
        left = iterations
        while left > 0:
            steps = min(8, left)
            q = self.passes
            for nb in self.nb.values():
                P.flag_wait(nb["flag"], q)
            kw = {}
            pitch = self.w
            if "top" in self.nb:
                t = self.nb["top"]
                kw.update(top_t=t["T"][q % 2], top_p=t["P"], top_rows=t["rows"])
                pitch = t["pitch"]
            if "bot" in self.nb:
                b = self.nb["bot"]
                kw.update(bot_t=b["T"][q % 2], bot_p=b["P"], bot_rows=b["rows"])
                pitch = b["pitch"]
            P.hotspot_peer(self.T[q % 2], self.Pw, params, scheme, reach, steps, self.T[(q + 1) % 2],
                           src_pitch=pitch, **kw)
            P.flag_set(self.flag.data_ptr(), q + 1)
            self.passes += 1
            left -= steps
        return self.T[self.passes % 2]

    def close(self):
        torch.cuda.synchronize()
        dist.barrier(group=self.group)
        for base in self._opened:
            self.P.ipc_close(base)
        self._opened = []


def _allreduce_np(a: np.ndarray, device, group=None) -> np.ndarray:
    t = torch.from_numpy(np.ascontiguousarray(a, dtype=np.float64)).to(device)
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return t.cpu().numpy()


def tune_pooled(frames_local, f, toq: float, metric="mre", group=None, partials=None):
    """The TOQ tuner over the union of every rank's training frames: per-rank
    candidate partials (paraprox_tune_partials), one all-reduce of 3 fp64 per
    candidate, then the host-only decision (paraprox_tune_decide).  Every rank
    holds the same sums and takes the same decision."""
    from . import paraprox as P
    if partials is None:
        partials = P.tune_partials(frames_local, f, metric)
    dev = frames_local.device if isinstance(frames_local, torch.Tensor) else "cpu"
    summed = _allreduce_np(partials, dev if dist.get_backend(group) == "nccl" else "cpu", group)
    return P.tune_decide(f, summed, toq, metric)


def quality_pooled(exact, approx, metric="mre", group=None, partials=None) -> float:
    from . import paraprox as P
    if partials is None:
        partials = P.quality_partials(exact, approx, metric)
    dev = exact.device if dist.get_backend(group) == "nccl" else "cpu"
    summed = _allreduce_np(partials, dev, group)
    return P.quality_from_partials(summed, metric)
