"""Multi-GPU plumbing for the z-slab partition: slab assignment, the
library's halo schedule (``mbir_halo_plan``), and the NCCL unique-id broadcast over a
``torch.distributed`` process group.  The halo exchange itself runs inside libmbir over NCCL;
this module only exposes its host-side schedule (for tests) and bootstraps the communicator."""
from __future__ import annotations

import ctypes as C

import numpy as np

from . import _lib as L

SEND, RECV = 1, 0


def slab(nz_total: int, world: int, rank: int):
    """Contiguous slab of rank `rank`: (z_offset, nz_local); the first nz % world ranks get one
    extra slice."""
    if world < 1 or not 0 <= rank < world or nz_total < world:
        raise ValueError("need 1 <= world <= nz_total and 0 <= rank < world")
    base, extra = divmod(nz_total, world)
    z0 = rank * base + min(rank, extra)
    return z0, base + (1 if rank < extra else 0)


def halo_plan(z_offset: int, nz_local: int, rank: int, nranks: int, parity: int):
    """The library's exchange schedule: list of (peer, SEND/RECV, local storage slice)."""
    ops = np.zeros((4, 3), np.int32)
    n = L.load().mbir_halo_plan(z_offset, nz_local, rank, nranks, parity, ops.ctypes.data)
    L.check(n if n < 0 else 0, None, "mbir_halo_plan")
    return [tuple(int(v) for v in ops[i]) for i in range(n)]


def broadcast_nccl_id(group=None) -> bytes:
    """Rank 0 creates the NCCL unique id (``mbir_nccl_unique_id``) and every rank receives it
    through the torch process group (any backend)."""
    import torch
    import torch.distributed as dist

    buf = torch.zeros(128, dtype=torch.uint8)
    if dist.get_rank(group) == 0:
        raw = (C.c_char * 128)()
        L.check(L.load().mbir_nccl_unique_id(raw), None, "mbir_nccl_unique_id")
        buf.copy_(torch.frombuffer(bytearray(bytes(raw)), dtype=torch.uint8))
    if dist.get_backend(group) == "nccl":
        dev = torch.device("cuda", torch.cuda.current_device())
        b = buf.to(dev)
        dist.broadcast(b, 0, group=group)
        buf = b.cpu()
    else:
        dist.broadcast(buf, 0, group=group)
    return bytes(buf.numpy().tobytes())
