"""Row stripes whose halo rows are read inside the stencil kernel from peer
pointers (§8(e); paraprox_stencil_peer, dist.PeerStripe): the stripe output
equals the whole-image output bit for bit -- in one process (pointers into
the same tensor), through the staging fallback, and across two processes
sharing the GPU through CUDA IPC (the path NVLink peers take on one node)."""
import os
import socket

import numpy as np
import pytest
import torch

import workloads as W
from workloads import filters as F

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def P():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_asplos_samadijlm14_b200 as pkg

    return pkg.paraprox


def mkf(P, w):
    return P.Filter(wy=w[0], wx=w[1]) if isinstance(w, tuple) else P.Filter(w)


CASES = [("conv9", F.conv(9)), ("mean5", F.mean(5)), ("sep7", F.separable(7)), ("rect3x7", F.conv(7, seed=11, ky=3))]
SCHEMES = [("exact", 0), ("row", 1), ("col", 2), ("center", 1), ("row", 4)]


@pytest.mark.parametrize("name,w", CASES, ids=[c[0] for c in CASES])
def test_peer_pointers_single_process(P, name, w):
    f = mkf(P, w)
    x = torch.from_numpy(W.image(300, 260, 5)).cuda()
    for scheme, reach in SCHEMES:
        full = P.stencil_approx(x, f, scheme, reach)
        for r0, r1 in ((0, 90), (90, 200), (200, 300), (37, 41)):
            stripe = x[r0:r1].clone()  # its own allocation, like a rank's buffer
            top = x[r0 - 6].data_ptr() if r0 >= 6 else (x.data_ptr() if r0 > 0 else None)
            top_rows = 6 if r0 >= 6 else r0
            bot = x[r1].data_ptr() if r1 < 300 else None
            bot_rows = min(6, 300 - r1)
            got = P.stencil_peer(stripe, f, scheme, reach, top=top, top_rows=top_rows, bot=bot, bot_rows=bot_rows,
                                 src_pitch=x.stride(0))
            assert torch.equal(got, full[r0:r1]), (name, scheme, reach, r0, r1, P.last_kernel())


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _ipc_worker(rank, world, port, q):
    try:
        import sys
        sys.path.insert(0, ROOT)
        import torch.distributed as dist
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        import paper_conf_asplos_samadijlm14_b200 as pkg
        from paper_conf_asplos_samadijlm14_b200 import dist as D
        P = pkg.paraprox
        h, w = 333, 300
        x = torch.from_numpy(W.image(h, w, 7)).cuda()
        s = D.stripe_of(h, world, rank, cap=4)
        ps = D.PeerStripe(s, w, "cuda")
        ps.buf.copy_(x[s.r0:s.r1])
        ps.ready()
        for wts in (F.conv(9), F.mean(5)):
            f = P.Filter(wts)
            for scheme, reach in SCHEMES:
                out = torch.empty((s.rows, w), device="cuda")
                ps.stencil(f, scheme, reach, out)
                full = P.stencil_approx(x, f, scheme, reach)
                assert torch.equal(out, full[s.r0:s.r1]), (rank, scheme, reach)
        dist.barrier()
        ps.close()
        q.put((rank, "ok"))
    except Exception:  # pragma: no cover
        import traceback
        q.put((rank, traceback.format_exc()))


@pytest.mark.parametrize("world", [2, 3])
def test_peer_stripes_ipc_two_processes(world):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ipc_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert res[r] == "ok", res[r]


def _hotspot_worker(rank, world, port, q):
    try:
        import sys
        sys.path.insert(0, ROOT)
        import torch.distributed as dist
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        import paper_conf_asplos_samadijlm14_b200 as pkg
        from paper_conf_asplos_samadijlm14_b200 import dist as D
        from workloads import hotspot as H
        P = pkg.paraprox
        h, w = 150, 260
        t, p = H.frames(1, h, w, 3)
        td, pd = torch.from_numpy(t[0]).cuda(), torch.from_numpy(p[0]).cuda()
        s = D.stripe_of(h, world, rank, cap=8)
        hs = D.HotspotPeerStripes(s, w, "cuda")
        for scheme, reach in (("exact", 0), ("col", 1), ("row", 1), ("center", 1)):
            for iters in (1, 8, 19):
                hs.load(td[s.r0:s.r1], pd[s.r0:s.r1])
                got = hs.run(H.PARAMS, scheme, reach, iters)
                full = P.hotspot(td, pd, H.PARAMS, scheme, reach, iters)
                torch.cuda.synchronize()
                assert torch.equal(got, full[s.r0:s.r1]), (rank, scheme, iters, float((got - full[s.r0:s.r1]).abs().max()))
        hs.close()
        q.put((rank, "ok"))
    except Exception:  # pragma: no cover
        import traceback
        q.put((rank, traceback.format_exc()))


@pytest.mark.parametrize("world", [2, 3])
def test_hotspot_peer_stripes_ipc(world):
    """HotSpot passes of a striped grid with in-kernel peer halos and
    device-side pass ordering: bit-identical to the whole grid."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_hotspot_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert res[r] == "ok", res[r]


def test_peer_neighbour_thinner_than_halo_is_refused(P):
    """A neighbour stripe with fewer rows than the plan's h_y cannot supply the
    halo (its first row is not the image edge): INVALID_ARG, no launch."""
    f = mkf(P, F.conv(9))  # exact: h_y = 4
    x = torch.from_numpy(W.image(40, 64, 6)).cuda()
    stripe = x[10:30].clone()
    with pytest.raises(P.ParaproxError):
        P.stencil_peer(stripe, f, "exact", 0, top=x[8].data_ptr(), top_rows=2, bot=x[30].data_ptr(), bot_rows=4,
                       src_pitch=x.stride(0))
    # h_y = 0 (row scheme at full reach): any neighbour is fine, nothing is read
    got = P.stencil_peer(stripe, f, "row", 4, top=x[8].data_ptr(), top_rows=2, bot=x[30].data_ptr(), bot_rows=1,
                         src_pitch=x.stride(0))
    assert torch.equal(got, P.stencil_approx(x, f, "row", 4)[10:30])
