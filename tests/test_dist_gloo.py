"""Multi-process (world_size 2 and 3, gloo on CPU) checks of the multi-GPU
orchestration in paper_conf_asplos_samadijlm14_b200/dist.py: frame sharding,
the row-stripe halo exchange, the interior/boundary split of a stripe step and
the pooled tuner decision.  The stencil itself is the oracle here (the CUDA
path is covered by tests/test_parity_gpu.py::test_stripes_with_halos_bitwise);
what is tested is that the decomposition reproduces the whole-image result."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _init(rank, world, port):
    import sys
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)


def _worker_stripes(rank, world, port, q):
    try:
        _init(rank, world, port)
        import oracle as O
        import paper_conf_asplos_samadijlm14_b200 as pkg
        from paper_conf_asplos_samadijlm14_b200 import dist as D
        import workloads as W
        from workloads import filters as F
        P = pkg.paraprox
        h, w = 61, 45
        x = W.image(h, w, 3)
        for wts in (F.conv(9), F.mean(5), F.gaussian(3)):
            f = P.Filter(wts)
            r = wts.shape[0] // 2
            s = D.stripe_of(h, world, rank, cap=r)
            for scheme in ("exact", "row", "col", "center"):
                for reach in (1, 2, r):
                    dy, dx = O.scheme_reaches(scheme, reach)
                    full = O.stencil_approx_xy(x, wts, dy, dx)
                    buf = D.alloc_stripe(s, w, dtype=torch.float64)
                    buf.fill_(float("nan"))  # halos must come from the exchange
                    buf[s.cap:s.cap + s.rows] = torch.from_numpy(x[s.r0:s.r1].astype(np.float64))
                    out = torch.empty((s.rows, w), dtype=torch.float64)

                    def compute(band, ht, hb, o):
                        b = band.numpy()
                        assert not np.isnan(b).any(), "read an unexchanged halo row"
                        res = O.stencil_approx_xy(b.astype(np.float32), wts, dy, dx)
                        o.copy_(torch.from_numpy(res[ht:ht + o.shape[0]]))

                    D.stencil_stripe(buf, s, f, scheme, reach, out, compute=compute)
                    assert np.array_equal(out.numpy(), full[s.r0:s.r1]), (rank, scheme, reach)
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        import traceback
        q.put((rank, traceback.format_exc()))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


def _worker_hotspot(rank, world, port, q):
    try:
        _init(rank, world, port)
        import oracle as O
        from paper_conf_asplos_samadijlm14_b200 import dist as D
        from workloads import hotspot as H
        h, w, iters = 37, 23, 5
        t, p = H.frames(1, h, w, 4)
        t, p = t[0], p[0]
        prm = H.PARAMS
        s = D.stripe_of(h, world, rank, cap=1)
        for scheme, reach, dd in (("exact", 0, (0, 0)), ("row", 1, (1, 0)), ("col", 1, (0, 1)),
                                  ("center", 1, (1, 1))):
            full = O.hotspot(t, p, prm, dd[0], dd[1], iters)
            bufs = [D.alloc_stripe(s, w, dtype=torch.float64) for _ in range(2)]
            for b in bufs:
                b.fill_(float("nan"))
            bufs[0][s.cap:s.cap + s.rows] = torch.from_numpy(t[s.r0:s.r1].astype(np.float64))
            pw = torch.from_numpy(p[s.r0:s.r1].astype(np.float64))

            def compute(band, ht, hb, pwr, o):
                bnd = band.numpy()
                assert not np.isnan(bnd).any(), "read an unexchanged halo row"
                res = O.hotspot(bnd.astype(np.float32), np.pad(pwr.numpy(), ((ht, hb), (0, 0))).astype(np.float32),
                                prm, dd[0], dd[1], 1)
                o.copy_(torch.from_numpy(res[ht:ht + o.shape[0]]))

            fin = D.hotspot_stripes(bufs, pw, s, prm, scheme, reach, iters, compute=compute)
            got = fin[s.cap:s.cap + s.rows].numpy()
            # the oracle band steps round the state to fp32 between steps: compare at fp32 precision
            assert np.allclose(got, full[s.r0:s.r1], rtol=1e-6, atol=0), (rank, scheme)
        q.put((rank, "ok"))
    except Exception:  # pragma: no cover
        import traceback
        q.put((rank, traceback.format_exc()))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


def _worker_exchange(rank, world, port, q):
    try:
        _init(rank, world, port)
        from paper_conf_asplos_samadijlm14_b200 import dist as D
        h, w = 40, 7
        img = torch.arange(h * w, dtype=torch.float32).view(h, w)
        s = D.stripe_of(h, world, rank, cap=4)
        for hy in (0, 1, 3, 4):
            buf = D.alloc_stripe(s, w).fill_(-1)
            buf[4:4 + s.rows] = img[s.r0:s.r1]
            D.exchange_halos(buf, s, hy)
            ht, hb = s.halo_top(hy), s.halo_bottom(hy)
            assert torch.equal(buf[4 - ht:4], img[s.r0 - ht:s.r0])
            assert torch.equal(buf[4 + s.rows:4 + s.rows + hb], img[s.r1:s.r1 + hb])
            # rows beyond the valid halos are untouched
            assert torch.all(buf[:4 - ht] == -1) and torch.all(buf[4 + s.rows + hb:] == -1)
        q.put((rank, "ok"))
    except Exception:
        import traceback
        q.put((rank, traceback.format_exc()))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


def _mre_partials(e, a):
    e = e.astype(np.float64).ravel()
    a = a.astype(np.float64).ravel()
    return np.array([np.sum(np.abs(a - e) / np.abs(e)), float(e.size), 0.0])


def _worker_tune(rank, world, port, q):
    try:
        _init(rank, world, port)
        import oracle as O
        import paper_conf_asplos_samadijlm14_b200 as pkg
        from paper_conf_asplos_samadijlm14_b200 import dist as D
        import workloads as W
        from workloads import filters as F
        P = pkg.paraprox
        wts = F.mean(5)
        f = P.Filter(wts)
        frames = W.frames(6, 64, 80, 40)
        f0, f1 = D.frame_shard(6, world, rank)
        mine = frames[f0:f1]
        e = O.stencil_exact(mine, wts).astype(np.float32)
        parts = []
        for scheme, reach in P.tune_candidates(f):
            a = O.stencil_approx(mine, wts, scheme, reach).astype(np.float32)
            parts.append(_mre_partials(e, a))
        parts = np.concatenate(parts)
        for toq in (0.8, 0.9, 0.95, 0.99):
            got = D.tune_pooled(torch.from_numpy(mine), f, toq, "mre", partials=parts)
            ref = O.tune(frames, wts, toq, "mre")
            assert got[:2] == (ref["scheme"], ref["reach"]), (toq, got, ref)
            assert abs(got[2] - ref["quality"]) < 1e-12
        q.put((rank, "ok"))
    except Exception:
        import traceback
        q.put((rank, traceback.format_exc()))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


def _run(worker, world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert res[r] == "ok", res[r]


@pytest.mark.parametrize("world", [2, 3])
def test_halo_exchange(world):
    _run(_worker_exchange, world)


@pytest.mark.parametrize("world", [2, 3])
def test_row_stripes_reproduce_whole_image(world):
    _run(_worker_stripes, world)


def test_pooled_tuning_matches_single_process(O):
    _run(_worker_tune, 2)


def test_frame_shard_covers():
    from paper_conf_asplos_samadijlm14_b200 import dist as D
    for n in (1, 7, 256):
        for world in (1, 2, 3, 8):
            got = [D.frame_shard(n, world, r) for r in range(world)]
            assert got[0][0] == 0 and got[-1][1] == n
            assert all(got[i][1] == got[i + 1][0] for i in range(world - 1))
            assert max(b - a for a, b in got) - min(b - a for a, b in got) <= 1


@pytest.mark.parametrize("world", [2, 3])
def test_hotspot_stripes_reproduce_whole_grid(world):
    _run(_worker_hotspot, world)
