"""Bootstrap of a sharded log (include/ffm.h "Sharded logs").

Plumbing only.  The library runs the whole sharded step inside the collective
``ffm_dedup_run`` -- H1..H4 per rank, the all-gather of class representatives, the
peer-memory byte verify over NVLink, the labels and the all-reduce of the per-site
sums -- on the log's stream, over its own NCCL communicator.  This module only hands
it the world: rank 0's ``ncclUniqueId`` broadcast through a torch.distributed group,
or, where NCCL cannot connect the ranks (several ranks sharing one GPU in tests), a
host transport built from that group's gloo collectives (``HostComm``).
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch
import torch.distributed as dist

from . import ALLGATHER_FN, ALLREDUCE_FN, FfmCommOps, FfmLog, ffm_nccl_unique_id


class HostComm:
    """ffm_comm_ops over a torch.distributed group (host buffers; gloo).  Collective
    callbacks the library invokes from inside ffm_log_create / ffm_dedup_run."""

    def __init__(self, group=None):
        self.group = group
        self.world = dist.get_world_size(group)
        self.error = None
        self._ag = ALLGATHER_FN(self._allgather)
        self._ar = ALLREDUCE_FN(self._allreduce)
        self.ops = FfmCommOps(None, self._ag, self._ar)

    def allgather(self, send: np.ndarray) -> np.ndarray:
        """recv[world * bytes] = every rank's send (uint8), rank-major."""
        t = torch.from_numpy(np.ascontiguousarray(send, np.uint8))
        parts = [torch.empty_like(t) for _ in range(self.world)]
        dist.all_gather(parts, t, group=self.group)
        return torch.cat(parts).numpy()

    def allreduce_u64(self, buf: np.ndarray) -> np.ndarray:
        """Elementwise sum mod 2^64 (int64 two's complement sums wrap identically)."""
        t = torch.from_numpy(np.ascontiguousarray(buf, np.uint64).view(np.int64).copy())
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=self.group)
        return t.numpy().view(np.uint64)

    def _allgather(self, ctx, send, recv, nbytes):
        try:
            src = np.ctypeslib.as_array((ctypes.c_uint8 * max(nbytes, 1)).from_address(send))[:nbytes] \
                if nbytes else np.empty(0, np.uint8)
            out = self.allgather(src)
            if out.size:
                ctypes.memmove(recv, out.ctypes.data, out.size)
            return 0
        except Exception as e:          # never raise through the C ABI
            self.error = e
            return -1

    def _allreduce(self, ctx, buf, n):
        try:
            a = np.ctypeslib.as_array((ctypes.c_uint64 * n).from_address(buf))
            a[:] = self.allreduce_u64(a)
            return 0
        except Exception as e:
            self.error = e
            return -1


def create_sharded_log(n_sites: int, device: int, *, group=None, transport: str = "nccl", **kw) -> FfmLog:
    """A log for this rank of a sharded world (collective over `group`).
    transport "nccl": the library's own NCCL communicator (one GPU per rank);
    "host": HostComm over the group (gloo; ranks may share a GPU)."""
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    if transport == "nccl":
        uid = [ffm_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=dist.get_global_rank(group, 0) if group else 0, group=group)
        return FfmLog(n_sites, device, rank=rank, world=world, nccl_id=uid[0], **kw)
    if transport == "host":
        hc = HostComm(group)
        log = FfmLog(n_sites, device, rank=rank, world=world, comm=hc.ops, **kw)
        log.host_comm = hc
        return log
    raise ValueError(f"transport {transport!r}: 'nccl' or 'host'")
