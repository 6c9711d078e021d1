"""Config 2: wall / event time of ffm_dedup_run with pinned-host vs device outputs, graph
on / off (the speculative D2H of duplicate_of overlapping H3)."""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import loggen  # noqa: E402
import paper_conf_sc_weltonm19_b200 as ffm  # noqa: E402

k = int(sys.argv[1]) if len(sys.argv) > 1 else 2
lg = loggen.gen_config(k)
lg.materialize(nthreads=0)
content = torch.from_numpy(lg.buf).cuda()
ptrs = (lg.c_off[lg.content] + np.uint64(content.data_ptr())).astype(np.uint64)
for graph in (True, False):
    log = ffm.FfmLog(lg.n_sites, arena_bytes=lg.total_bytes + 128 * lg.n + (1 << 20), max_records=lg.n, graph=graph)
    log.append_log(lg, ptrs=ptrs, payload_kind=ffm.FFM_PAYLOAD_DEVICE)
    dh = torch.empty(lg.n, dtype=torch.int64).pin_memory()
    bh = torch.empty(lg.n_sites, dtype=torch.int64).pin_memory()
    dd = torch.empty(lg.n, dtype=torch.int64, device="cuda")
    bd = torch.empty(lg.n_sites, dtype=torch.int64, device="cuda")
    dp = np.empty(lg.n, np.int64)
    st = torch.cuda.ExternalStream(log.stream)
    for name, d, b in (("pinned", dh.numpy(), bh.numpy().view(np.uint64)), ("device", dd, bd),
                       ("pageable", dp, bh.numpy().view(np.uint64))):
        for _ in range(5):
            log.run(d, b)
        torch.cuda.synchronize()
        ts = []
        for _ in range(20):
            t0 = time.perf_counter()
            log.run(d, b)
            ts.append(time.perf_counter() - t0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for _ in range(20):
            log.run(d, b)
        e1.record(st)
        torch.cuda.synchronize()
        print(f"graph={graph} {name:8s} wall median {np.median(ts) * 1e3:.3f} ms  events {e0.elapsed_time(e1) / 20:.3f} ms "
              f"syncs {log.stats()['host_syncs']}", flush=True)
    log.close()
