"""Multi-GPU orchestration of a sharded log (include/ffm.h "Sharded logs").

Plumbing only: torch.distributed moves the representative tuples and the benefit
partials (NCCL over NVLink / NVSwitch on GPUs; gloo with host staging when NCCL is
unavailable, e.g. several ranks sharing one GPU in tests).  Every step of the hot
path -- H1..H4, the global group-by, the peer-memory byte verify and the labels --
runs in libffm's kernels.
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

from . import (REP_WORDS, ffm_log_count, ffm_shard_ipc_handle, ffm_shard_local, ffm_shard_merge,
               ffm_shard_open_peer, ffm_site_duplicate_counts)


def _on_nccl(group=None) -> bool:
    return dist.get_backend(group) == "nccl"


def exchange_handles(log, group=None):
    """Map every peer's HBM arena (CUDA IPC).  Call after the last append."""
    world = dist.get_world_size(group)
    mine = ffm_shard_ipc_handle(log.h)
    allh = [None] * world
    dist.all_gather_object(allh, mine, group=group)
    for r, hb in enumerate(allh):
        ffm_shard_open_peer(log.h, r, hb)


def allgather_reps(local: torch.Tensor, group=None):
    """local: int64 [n, REP_WORDS] (any device).  Returns (all reps rank-major on
    local.device, counts list)."""
    world = dist.get_world_size(group)
    comm_dev = local.device if _on_nccl(group) else torch.device("cpu")
    n = torch.tensor([local.shape[0]], dtype=torch.int64, device=comm_dev)
    counts_t = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(counts_t, n, group=group)
    counts = [int(c.item()) for c in counts_t]
    mx = max(counts) if counts else 0
    if mx == 0:
        return local.new_empty((0, REP_WORDS)), counts
    pad = torch.zeros((mx, REP_WORDS), dtype=torch.int64, device=comm_dev)
    pad[: local.shape[0]] = local.to(comm_dev)
    out = torch.empty((world * mx, REP_WORDS), dtype=torch.int64, device=comm_dev)
    dist.all_gather_into_tensor(out, pad, group=group)
    parts = [out[r * mx: r * mx + counts[r]] for r in range(world)]
    return torch.cat(parts).to(local.device).contiguous(), counts


def allreduce_benefit(ben: torch.Tensor, group=None) -> torch.Tensor:
    """Sum int64 (two's complement == uint64 mod 2^64) partial benefits over ranks."""
    if _on_nccl(group) or ben.device.type == "cpu":
        dist.all_reduce(ben, op=dist.ReduceOp.SUM, group=group)
        return ben
    h = ben.cpu()
    dist.all_reduce(h, op=dist.ReduceOp.SUM, group=group)
    ben.copy_(h)
    return ben


def site_counts_sharded(log, device, group=None) -> torch.Tensor:
    """All-reduced duplicates per call site of the last sharded run (int64 [n_sites])."""
    c = torch.empty(log.n_sites, dtype=torch.int64, device=device)
    ffm_site_duplicate_counts(log.h, log.n_sites, c)
    return allreduce_benefit(c, group)


def dedup_sharded(log, device, group=None, duplicate_of=None, benefit=None, reps_buf=None):
    """One sharded run.  Returns (duplicate_of for this rank's records [global gids],
    global benefit_ns as int64 [n_sites]); both on `device` unless given."""
    n = ffm_log_count(log.h)
    if reps_buf is None or reps_buf.shape[0] < max(n, 1):
        reps_buf = torch.empty((max(n, 1), REP_WORDS), dtype=torch.int64, device=device)
    n_reps = ffm_shard_local(log.h, reps_buf, reps_buf.shape[0])
    # the exchange's device work (NCCL, padding, concatenation) is ordered on the
    # library's stream, which the merge kernels then read from
    dev = torch.device(device)
    if dev.type == "cuda" and log.stream:
        with torch.cuda.stream(torch.cuda.ExternalStream(log.stream, device=dev)):
            all_reps, counts = allgather_reps(reps_buf[:n_reps], group)
    else:
        all_reps, counts = allgather_reps(reps_buf[:n_reps], group)
    if duplicate_of is None:
        duplicate_of = torch.empty(max(n, 1), dtype=torch.int64, device=device)
    if benefit is None:
        benefit = torch.empty(log.n_sites, dtype=torch.int64, device=device)
    if all_reps.shape[0] == 0:
        all_reps = torch.empty((1, REP_WORDS), dtype=torch.int64, device=device)
    ffm_shard_merge(log.h, all_reps, np.asarray(counts, np.uint64), duplicate_of, benefit)
    allreduce_benefit(benefit, group)
    return duplicate_of[:n], benefit
