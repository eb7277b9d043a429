"""Bootstrap of the library's distributed handle (include/louvain.h
"multi-GPU").  Plumbing only: the vertex-sharded sweep, the per-bucket exchange
of moves, the all-reduce of Eq. (1)'s partial L change, the stop tests and the
contraction all run inside liblouvain.so (csrc/lv_dist.cu, csrc/lv_engine.cu).

Two transports are bootstrapped here through torch.distributed:
  * NCCL: rank 0 asks the library for a unique id, which is broadcast to the
    other ranks (broadcast_object_list); the library then drives NCCL itself on
    the handle's stream;
  * host: a pair of ctypes callbacks (all-gather of bytes, sum of uint64) over any
    process group -- gloo in the CPU/one-GPU tests, where NCCL cannot run (NCCL
    refuses two ranks on one GPU).
"""
from __future__ import annotations

import ctypes

import numpy as np


def nccl_unique_id(rank: int, group=None) -> ctypes.Array:
    """A 128-byte NCCL unique id made on rank 0 and shared with every rank."""
    import torch.distributed as dist
    from . import _check, lib
    buf = (ctypes.c_uint8 * 128)()
    obj = [None]
    if rank == 0:
        _check(lib().louvain_dist_unique_id(buf))
        obj = [bytes(buf)]
    dist.broadcast_object_list(obj, src=0, group=group)
    ctypes.memmove(buf, obj[0], 128)
    return buf


def host_comm(group=None):
    """louvain_host_comm_t over torch.distributed (CPU tensors; e.g. gloo).  The
    returned structure keeps its callbacks alive and must outlive the handle."""
    import torch
    import torch.distributed as dist
    from . import HOST_ALLGATHER, HOST_ALLREDUCE, HostComm

    world = dist.get_world_size(group)

    def allgather(user, send, recv, nbytes):
        try:
            n = int(nbytes)
            if n:
                mine = torch.frombuffer(bytearray(ctypes.string_at(send, n)), dtype=torch.uint8)
            else:
                mine = torch.zeros(0, dtype=torch.uint8)
            outs = [torch.empty(n, dtype=torch.uint8) for _ in range(world)]
            dist.all_gather(outs, mine, group=group)
            if n:
                flat = torch.cat(outs).numpy()
                ctypes.memmove(recv, flat.ctypes.data, n * world)
            return 0
        except Exception:  # noqa: BLE001 -- reported to the library as a failed collective
            return -1

    def allreduce(user, data, count):
        try:
            c = int(count)
            arr = np.ctypeslib.as_array(ctypes.cast(data, ctypes.POINTER(ctypes.c_int64)), shape=(c,))
            t = torch.from_numpy(arr.copy())
            dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)  # int64 two's complement = uint64 mod 2^64
            arr[:] = t.numpy()
            return 0
        except Exception:  # noqa: BLE001
            return -1

    hc = HostComm(None, HOST_ALLGATHER(allgather), HOST_ALLREDUCE(allreduce))
    hc._py = (allgather, allreduce)
    return hc


def edge_balanced_ranges(rowptr, world: int) -> list[tuple[int, int]]:
    """Contiguous vertex ranges [v_r, v_{r+1}) with rowptr[v_r] ~ r * nnz / world
    (the library's own split, louvain_dist_ranges; host-only, no GPU needed)."""
    from . import dist_ranges
    return dist_ranges(np.ascontiguousarray(rowptr, dtype=np.int64), world)


def local_rows(rowptr, col, w, lo: int, hi: int):
    """This rank's rows [lo, hi) of a full CSR as (rowptr_local starting at 0, col, w)."""
    e0, e1 = int(rowptr[lo]), int(rowptr[hi])
    rl = rowptr[lo:hi + 1] - rowptr[lo]
    return rl, col[e0:e1], (None if w is None else w[e0:e1])
