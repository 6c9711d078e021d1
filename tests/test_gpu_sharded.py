"""Sharded (multi-rank) parity on the GPU: P processes share cuda:0 (NCCL refuses two
ranks on one device, so the tuple exchange uses gloo with host staging; peer arenas
are CUDA-IPC mapped exactly as across NVLink).  Every rank's duplicate_of (global
gids) and the all-reduced benefit must equal the single-log oracle bit-exactly, for
both shard planners and with forced digest collisions (slow merge path)."""
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


def _worker(rank, world, port, out_dir, case, policy, digest_bits, device_payloads):
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
        log = ffm.FfmLog(lg.n_sites, device=0, rank=rank, world=world, digest_bits=digest_bits,
                         chunk_bytes=4096, timing=True)
        if device_payloads:
            buf = torch.from_numpy(lg.materialize()).cuda()
            ptrs = (lg.c_off[lg.content] + np.uint64(buf.data_ptr())).astype(np.uint64)
            log.append_log(lg, ptrs=ptrs, payload_kind=ffm.FFM_PAYLOAD_DEVICE, gids=idx, idx=idx)
        else:
            log.append_log(lg, gids=idx, idx=idx)
        sharded.exchange_handles(log)
        outs = []
        for _ in range(2):                                   # re-runnable
            dup, ben = sharded.dedup_sharded(log, torch.device("cuda", 0))
            outs.append((dup.cpu().numpy().copy(), ben.cpu().numpy().view(np.uint64).copy()))
        cnt = sharded.site_counts_sharded(log, torch.device("cuda", 0)).cpu().numpy()
        dist.barrier()            # peers must not unmap while others still read their arenas
        np.savez(os.path.join(out_dir, f"r{rank}.npz"), idx=idx, dup=outs[0][0], ben=outs[0][1],
                 dup2=outs[1][0], ben2=outs[1][1], cnt=cnt)
        dist.barrier()
        log.close()
    finally:
        dist.destroy_process_group()


def _run(tmp_path, world, case, policy, digest_bits=64, device_payloads=False):
    import torch.multiprocessing as mp
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path), case, policy, digest_bits, device_payloads),
             nprocs=world, join=True)
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
