"""Multi-GPU host logic on CPU with the gloo backend (world sizes 2-4): slab partition, the
library's halo-exchange schedule (mbir_halo_plan, the same plan the NCCL exchange posts) driven
with torch.distributed point-to-point on CPU tensors, and the NCCL unique-id bootstrap."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ppopp_sabnewkbrm17_b200 import dist as D


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _exchange(x, plan):
    """Execute a halo plan with gloo point-to-point ops; x is [nz_local + 2, ...] storage."""
    reqs = []
    for peer, kind, slice_ in plan:
        if kind == D.SEND:
            reqs.append(dist.isend(x[slice_].contiguous(), peer))
    bufs = []
    for peer, kind, slice_ in plan:
        if kind == D.RECV:
            b = torch.empty_like(x[slice_])
            reqs.append(dist.irecv(b, peer))
            bufs.append((slice_, b))
    for r in reqs:
        r.wait()
    for slice_, b in bufs:
        x[slice_] = b


def _worker(rank, world, port, nz_total, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        z0, nzl = D.slab(nz_total, world, rank)
        x = torch.full((nzl + 2, 3, 3), -1.0)

        def fill(stamp, parity=None):  # owned slice z holds 1000*stamp + z
            for l in range(nzl):
                z = z0 + l
                if parity is None or z % 2 == parity:
                    x[l + 1] = 1000.0 * stamp + z

        def check_halos(expect_stamp_of):
            if rank > 0:
                z = z0 - 1
                assert torch.all(x[0] == 1000.0 * expect_stamp_of(z) + z), (rank, "lower", x[0, 0, 0])
            if rank < world - 1:
                z = z0 + nzl
                assert torch.all(x[nzl + 1] == 1000.0 * expect_stamp_of(z) + z), (rank, "upper")

        # full exchange after set_image
        fill(1)
        _exchange(x, D.halo_plan(z0, nzl, rank, world, -1))
        check_halos(lambda z: 1)
        # iterations: update the even half, exchange it, then the odd half, exchange it
        for it in range(2, 5):
            fill(it, parity=0)
            _exchange(x, D.halo_plan(z0, nzl, rank, world, 0))
            check_halos(lambda z: it if z % 2 == 0 else it - 1)
            fill(it, parity=1)
            _exchange(x, D.halo_plan(z0, nzl, rank, world, 1))
            check_halos(lambda z: it)
        # NCCL unique-id bootstrap over the process group: every rank gets rank 0's id
        nid = D.broadcast_nccl_id()
        ids = [None] * world
        dist.all_gather_object(ids, nid)
        assert len(nid) == 128 and all(i == ids[0] for i in ids)
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,nz_total", [(2, 8), (3, 10), (4, 16)])
def test_halo_exchange_gloo(world, nz_total):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, nz_total, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert all(v == "ok" for v in res.values()), res


def test_slab_partition_covers_volume():
    for nz in (8, 10, 64):
        for world in (1, 2, 3, 4, 8):
            if world > nz:
                continue
            spans = [D.slab(nz, world, r) for r in range(world)]
            z = 0
            for z0, n in spans:
                assert z0 == z and n >= 1
                z += n
            assert z == nz


def test_halo_plan_edges():
    # single rank: nothing to exchange; first / last rank only talk to one neighbour
    assert D.halo_plan(0, 8, 0, 1, -1) == []
    # rank 0 owns z 0..3, rank 1 owns z 4..7: after the even half only z=4 moves (1 -> 0),
    # after the odd half only z=3 moves (0 -> 1)
    assert D.halo_plan(0, 4, 0, 2, 0) == [(1, D.RECV, 5)]
    assert D.halo_plan(0, 4, 0, 2, 1) == [(1, D.SEND, 4)]
    assert D.halo_plan(0, 4, 0, 2, -1) == [(1, D.SEND, 4), (1, D.RECV, 5)]
    assert D.halo_plan(4, 4, 1, 2, 0) == [(0, D.SEND, 1)]
    assert D.halo_plan(4, 4, 1, 2, 1) == [(0, D.RECV, 0)]
    with pytest.raises(Exception):
        D.halo_plan(0, 0, 0, 1, 0)
