"""Host-side logic of the multi-GPU path, on CPU: the shard planner (C ABI, host only),
the host exchange transport of a sharded log at world_size 2 / 3 over gloo, config checks."""
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
    import ctypes
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        hc = sharded.HostComm()
        # the library's calls, through the same C function pointers it receives
        send = (np.arange(40, dtype=np.uint8) + 50 * rank).astype(np.uint8)
        recv = np.zeros(40 * world, np.uint8)
        rc1 = hc.ops.allgather(None, send.ctypes.data, recv.ctypes.data, 40)
        rc0 = hc.ops.allgather(None, None, None, 0)                  # an empty block
        ben = np.array([rank + 1, 2**64 - 1, 1 << 62], np.uint64)    # wraps mod 2^64
        rc2 = hc.ops.allreduce_u64(None, ben.ctypes.data, 3)
        np.savez(os.path.join(out_dir, f"r{rank}.npz"), recv=recv, ben=ben, rc=[rc0, rc1, rc2])
        del ctypes
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_host_transport_gloo(tmp_path, world):
    """The ffm_comm_ops transport of a sharded log (sharded.HostComm) over gloo, world 2/3."""
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    want = np.concatenate([(np.arange(40, dtype=np.uint8) + 50 * r).astype(np.uint8) for r in range(world)])
    for r in range(world):
        z = np.load(tmp_path / f"r{r}.npz")
        assert z["rc"].tolist() == [0, 0, 0]
        np.testing.assert_array_equal(z["recv"], want)               # rank-major blocks
        u = z["ben"]
        assert int(u[0]) == sum(range(1, world + 1))
        assert int(u[1]) == (world * (2**64 - 1)) % 2**64
        assert int(u[2]) == (world * (1 << 62)) % 2**64


def test_sharded_config_validation():
    """world > 1 needs exactly one exchange transport (checked before any device work)."""
    c = ffm.ffm_config_init()
    c.world, c.rank, c.n_sites = 2, 0, 4
    with pytest.raises(ffm.FfmError) as e:
        ffm.ffm_log_create(c)
    assert e.value.code == ffm.FFM_E_INVAL


def test_nccl_unique_id_host_only():
    """ffm_nccl_unique_id opens the process's libnccl.so.2 (torch's) and returns a 128-byte
    ncclUniqueId without any GPU work."""
    import torch  # noqa: F401  (loads torch's NCCL)
    a, b = ffm.ffm_nccl_unique_id(), ffm.ffm_nccl_unique_id()
    assert len(a) == 128 and len(b) == 128 and a != b
