"""Sharded (multi-rank) parity on the GPU through the collective ffm_dedup_run: P
processes share cuda:0 (NCCL refuses two ranks on one device, so the library's exchange
runs over the host transport -- sharded.HostComm on gloo; peer arenas are CUDA-IPC
mapped exactly as across NVLink).  Every rank's duplicate_of (global gids), the global
benefit and the duplicate counts must equal the single-log oracle bit-exactly, for both
shard planners, P in {2, 3, 4, 8} and with forced digest collisions (slow segments)."""
import os
import socket

import numpy as np
import pytest

import loggen
import oracle

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


CASES = {
    "c5": dict(k=5, n_scale=0.004, size_scale=1 / 32),
    "c4": dict(k=4, n_scale=0.1, size_scale=1 / 64),
    "c3": dict(k=3, n_scale=0.02, size_scale=1 / 32),
    "c2": dict(k=2, n_scale=0.005, size_scale=1.0),
}


def _make(case):
    c = CASES[case.replace("+ch", "")]
    lg = loggen.gen_config(c["k"], n_scale=c["n_scale"], size_scale=c["size_scale"])
    if case.endswith("+ch"):        # destination-aware variant (S8(f) #3)
        lg.channel = np.random.default_rng(3).integers(0, 2, lg.n).astype(np.uint64)
    return lg


def _worker(rank, world, port, out_dir, case, policy, digest_bits, device_payloads, refine_bits=64):
    import torch
    import torch.distributed as dist
    import paper_conf_sc_weltonm19_b200 as ffm
    from paper_conf_sc_weltonm19_b200 import sharded

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        lg = _make(case)
        ranks = ffm.ffm_shard_plan(lg.site, lg.size, lg.n_sites, world, policy)
        idx = np.nonzero(ranks == rank)[0]
        log = sharded.create_sharded_log(lg.n_sites, 0, transport="host", digest_bits=digest_bits,
                                         refine_bits=refine_bits, chunk_bytes=4096, timing=True)
        if device_payloads:
            buf = torch.from_numpy(lg.materialize()).cuda()
            ptrs = (lg.c_off[lg.content] + np.uint64(buf.data_ptr())).astype(np.uint64)
            log.append_log(lg, ptrs=ptrs, payload_kind=ffm.FFM_PAYLOAD_DEVICE, gids=idx, idx=idx)
        else:
            log.append_log(lg, gids=idx, idx=idx)
        outs = []
        for _ in range(2):                                   # re-runnable
            dup, ben = log.run()
            outs.append((dup.copy(), ben.copy()))
        st = log.stats()
        cnt = log.site_counts()
        np.savez(os.path.join(out_dir, f"r{rank}.npz"), idx=idx, dup=outs[0][0], ben=outs[0][1],
                 dup2=outs[1][0], ben2=outs[1][1], cnt=cnt, n_slow=st["n_slow"], syncs=st["host_syncs"],
                 bx=st["remote_verify_bytes"], reps=st["n_reps_global"])
        log.close()
    finally:
        dist.destroy_process_group()


def _run(tmp_path, world, case, policy, digest_bits=64, device_payloads=False, refine_bits=64):
    import torch.multiprocessing as mp
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path), case, policy, digest_bits, device_payloads,
                            refine_bits), nprocs=world, join=True)
    lg = _make(case)
    want_dup, want_ben = oracle.dedup(lg)
    got = np.full(lg.n, -7, np.int64)
    for r in range(world):
        z = np.load(tmp_path / f"r{r}.npz")
        got[z["idx"]] = z["dup"]
        np.testing.assert_array_equal(z["ben"], want_ben)
        np.testing.assert_array_equal(z["dup2"], z["dup"])
        np.testing.assert_array_equal(z["ben2"], z["ben"])
    np.testing.assert_array_equal(got, want_dup)
    want_cnt = np.bincount(lg.site[want_dup >= 0].astype(np.int64), minlength=lg.n_sites)
    for r in range(world):
        np.testing.assert_array_equal(np.load(tmp_path / f"r{r}.npz")["cnt"], want_cnt)
    return lg, got


@pytest.mark.parametrize("case", ["c5", "c4", "c3", "c2"])
@pytest.mark.parametrize("policy", [0, 1])
def test_two_ranks(tmp_path, case, policy):
    lg, got = _run(tmp_path, 2, case, policy)
    assert (got >= 0).any()


def test_cross_shard_duplicates_exist_under_contiguous(tmp_path):
    import paper_conf_sc_weltonm19_b200 as ffm
    lg, got = _run(tmp_path, 3, "c4", 1)
    ranks = ffm.ffm_shard_plan(lg.site, lg.size, lg.n_sites, 3, 1)
    m = got >= 0
    assert (ranks[got[m]] != ranks[m]).sum() > 10


@pytest.mark.parametrize("digest_bits", [0, 8])
def test_forced_collisions_sharded(tmp_path, digest_bits):
    _run(tmp_path, 3, "c3", 1, digest_bits=digest_bits)


def test_four_ranks_device_payloads(tmp_path):
    _run(tmp_path, 4, "c5", 0, device_payloads=True)


@pytest.mark.parametrize("digest_bits", [64, 0])
def test_sharded_with_channels(tmp_path, digest_bits):
    _run(tmp_path, 3, "c5+ch", 1, digest_bits=digest_bits)


@pytest.mark.parametrize("case,policy", [("c5", 0), ("c5", 1), ("c4", 1)])
def test_eight_ranks(tmp_path, case, policy):
    """P = 8 through the collective run."""
    lg, got = _run(tmp_path, 8, case, policy)
    assert (got >= 0).any()
    z = [np.load(tmp_path / f"r{r}.npz") for r in range(8)]
    assert len({int(x["reps"]) for x in z}) == 1                 # one global table on every rank


def test_eight_ranks_forced_collisions(tmp_path):
    """Every representative of a size in one key (digest_bits 0) and no digest pruning
    (refine_bits 0): the same-key segment scan resolves every cross-rank class."""
    _run(tmp_path, 8, "c3", 1, digest_bits=0, refine_bits=0)
    assert sum(int(np.load(tmp_path / f"r{r}.npz")["n_slow"]) for r in range(8)) > 0


def test_two_host_syncs_without_collisions(tmp_path):
    """The collective run synchronises the host twice when no rank has digest collisions
    (the host transport's own staging copies aside, which NCCL does not need)."""
    lg, got = _run(tmp_path, 2, "c5", 0)
    for r in range(2):
        z = np.load(tmp_path / f"r{r}.npz")
        assert int(z["syncs"]) == 2, int(z["syncs"])


def test_nccl_world_of_one():
    """The collective run over the library's own NCCL communicator (ncclCommInitRank,
    ncclAllGather of the headers and representatives, ncclAllReduce of the per-site sums,
    all on the log's stream) in a world of one: the NCCL data plane on a single GPU."""
    import torch  # noqa: F401  (the process's NCCL is torch's)
    import paper_conf_sc_weltonm19_b200 as ffm
    lg = loggen.gen_config(5, n_scale=0.004, size_scale=1 / 32)
    want_dup, want_ben = oracle.dedup(lg)
    with ffm.FfmLog(lg.n_sites, rank=0, world=1, nccl_id=ffm.ffm_nccl_unique_id(), chunk_bytes=4096) as log:
        log.append_log(lg)
        for _ in range(2):
            dup, ben = log.run()
            np.testing.assert_array_equal(dup, want_dup)
            np.testing.assert_array_equal(ben, want_ben)
        st = log.stats()
        assert st["exchange_bytes"] > 0 and st["host_syncs"] == 2
        assert st["n_reps_local"] == st["n_reps_global"] > 0
        np.testing.assert_array_equal(log.site_counts(),
                                      np.bincount(lg.site[want_dup >= 0].astype(np.int64), minlength=lg.n_sites))
