"""Small logs through every kernel (fused and two-pass round 0 incl. the TMA-pipelined k_fused_fx in
hash and verify mode with pieces split from 64 KiB chunks and groups of > 64 members, pre-filter,
collision resolve, online windows, the collective sharded merge, device-payload gather), for
compute-sanitizer memcheck /
racecheck / synccheck."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import loggen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_sc_weltonm19_b200 as ffm  # noqa: E402

class LonelyWorld:
    """ffm_comm_ops of a world of 2 whose rank 1 has no records (peer blocks are zeros)."""

    def __init__(self):
        import ctypes
        self._ag = ffm.ALLGATHER_FN(self._allgather)
        self._ar = ffm.ALLREDUCE_FN(lambda ctx, buf, n: 0)
        self.ops = ffm.FfmCommOps(None, self._ag, self._ar)
        self._ct = ctypes

    def _allgather(self, ctx, send, recv, nbytes):
        if nbytes:
            self._ct.memmove(recv, send, nbytes)
            self._ct.memset(recv + nbytes, 0, nbytes)
        return 0


for k, ns, ss in [(5, 0.001, 1 / 64), (3, 0.003, 1 / 64), (3, 0.012, 1 / 128), (4, 0.04, 1 / 512), (2, 0.001, 1.0)]:
    lg = loggen.gen_config(k, n_scale=ns, size_scale=ss)
    want = oracle.dedup(lg)
    for db, rb, dev, extra in [(64, 64, False, {}), (0, 64, True, {}), (0, 0, False, {}),
                               (64, 64, False, {"two_pass": True}), (64, 64, False, {"prefilter": True}),
                               (8, 64, True, {"fused": True}), (0, 64, False, {"chunk": 65536})]:
        chunk = extra.pop("chunk", 4096)
        with ffm.FfmLog(lg.n_sites, digest_bits=db, refine_bits=rb, chunk_bytes=chunk, small_bytes=1024,
                        **extra) as log:
            if dev:
                buf = torch.from_numpy(lg.materialize()).cuda()
                ptrs = (lg.c_off[lg.content] + np.uint64(buf.data_ptr())).astype(np.uint64)
                log.append_log(lg, ptrs=ptrs, payload_kind=ffm.FFM_PAYLOAD_DEVICE)
            else:
                log.append_log(lg)
            d, b = log.run()
            assert np.array_equal(d, want[0]) and np.array_equal(b, want[1]), (k, db, rb, extra)
    # online windows: fused (metadata uploaded by the step / at append time), append-time
    # hashing (two-pass steps); host outputs (direct launches) and device outputs (the
    # captured window step, replayed for equal windows, residual fix-up with digest_bits 0)
    for kw in ({}, {"online": True}, {"online": True, "append_hash": True}):
        for db, dev_out in ((8, False), (0, True)):
            with ffm.FfmLog(lg.n_sites, digest_bits=db, chunk_bytes=4096, **kw) as log:
                ptrs = lg.payload_ptrs()
                got = []
                w = max(1, lg.n // 4)
                dd = torch.empty(w + 1, dtype=torch.int64, device="cuda") if dev_out else None
                bb = torch.empty(lg.n_sites, dtype=torch.int64, device="cuda") if dev_out else None
                for a in range(0, lg.n, w):
                    e = min(lg.n, a + w)
                    log.append_batch(lg.site[a:e], lg.size[a:e], ptrs[a:e], lg.dur[a:e])
                    if dev_out:
                        log.online_step(dd, bb)
                        got.append(dd[:e - a].cpu().numpy().copy())
                    else:
                        got.append(log.online_step()[0].copy())
                assert np.array_equal(np.concatenate(got), want[0]), ("online", k, kw, db)
    # the collective sharded run in one process: a world of 2 whose other rank is empty
    # (header, export, all-gather, merge incl. the same-key segment scan, all-reduce)
    for db in (64, 0):
        w = LonelyWorld()
        with ffm.FfmLog(lg.n_sites, rank=0, world=2, comm=w.ops, digest_bits=db, chunk_bytes=4096) as log:
            log.append_log(lg, gids=np.arange(lg.n))
            d, b = log.run()
            assert np.array_equal(d, want[0]) and np.array_equal(b, want[1]), ("sharded", k, db)
print("sanitize smoke ok")
