"""Host-side logic of the multi-GPU path, on CPU: the shard planner (C ABI, host only)
and the torch.distributed exchange steps at world_size 2 over gloo."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import loggen
import paper_conf_sc_weltonm19_b200 as ffm
from paper_conf_sc_weltonm19_b200 import sharded


def test_plan_site_affinity_keeps_sites_whole_and_balances():
    lg = loggen.gen_config(5, n_scale=0.01, size_scale=1 / 16)
    for world in (2, 4, 8):
        ranks = ffm.ffm_shard_plan(lg.site, lg.size, lg.n_sites, world, ffm.FFM_SHARD_SITE_LPT)
        assert ranks.min() >= 0 and ranks.max() < world
        for s in np.unique(lg.site):
            assert len(np.unique(ranks[lg.site == s])) == 1          # a site never straddles shards
        load = np.bincount(ranks, weights=lg.size.astype(np.float64) + 1, minlength=world)
        big = max(np.bincount(lg.site, weights=lg.size.astype(np.float64) + 1))
        assert load.max() - load.min() <= big + 1                    # LPT bound: within one site


def test_plan_contiguous_is_ordered_and_balanced():
    lg = loggen.gen_config(2, n_scale=0.01)
    for world in (1, 2, 3, 8):
        r = ffm.ffm_shard_plan(lg.site, lg.size, lg.n_sites, world, ffm.FFM_SHARD_CONTIGUOUS)
        assert np.all(np.diff(r) >= 0) and r[0] == 0 and r[-1] == world - 1
        load = np.bincount(r, weights=lg.size.astype(np.float64), minlength=world)
        assert load.max() <= lg.total_bytes / world + lg.size.max() + 1


def test_plan_errors():
    with pytest.raises(ffm.FfmError):
        ffm.ffm_shard_plan([0, 5], [1, 1], 2, 2)
    with pytest.raises(ffm.FfmError):
        ffm.ffm_shard_plan([0], [1], 1, 0)
    assert ffm.ffm_shard_plan([], [], 1, 4).tolist() == []


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_dir):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # ragged counts, one rank empty when world > 2
        n = [3, 0, 5][rank] if world == 3 else [3, 5][rank]
        local = torch.arange(n * ffm.REP_WORDS, dtype=torch.int64).reshape(n, ffm.REP_WORDS) + 1000 * rank
        allr, counts = sharded.allgather_reps(local)
        ben = torch.tensor([rank + 1, -1, (1 << 62)], dtype=torch.int64)   # -1 == 2^64-1 as u64
        sharded.allreduce_benefit(ben)
        torch.save({"all": allr, "counts": counts, "ben": ben}, os.path.join(out_dir, f"r{rank}.pt"))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_exchange_steps_gloo(tmp_path, world):
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    res = [torch.load(tmp_path / f"r{r}.pt") for r in range(world)]
    ns = [3, 0, 5] if world == 3 else [3, 5]
    want = torch.cat([torch.arange(n * ffm.REP_WORDS, dtype=torch.int64).reshape(n, ffm.REP_WORDS) + 1000 * r
                      for r, n in enumerate(ns)])
    for r in res:
        assert r["counts"] == ns
        assert torch.equal(r["all"], want)                 # rank-major, padding stripped
        u = r["ben"].numpy().view(np.uint64)
        assert u[0] == sum(range(1, world + 1))
        assert u[1] == (world * ((1 << 64) - 1)) % (1 << 64)   # wraps mod 2^64 like the u64 sums
        assert u[2] == (world * (1 << 62)) % (1 << 64)
