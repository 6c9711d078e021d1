"""Host cost of ffm_log_append_batch for device-resident payloads (config 2), by flag:
where do ~17 ns per record go (staging descriptors, metadata upload at append)?"""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import loggen  # noqa: E402
import paper_conf_sc_weltonm19_b200 as ffm  # noqa: E402

if os.environ.get("PROBE_LIB"):
    ffm.set_library_path(os.environ["PROBE_LIB"])

lg = loggen.gen_config(2)
lg.materialize(nthreads=0)
content = torch.from_numpy(lg.buf).cuda()
ptrs = (lg.c_off[lg.content] + np.uint64(content.data_ptr())).astype(np.uint64)
w = 262144
for online in (False, True):
    with ffm.FfmLog(lg.n_sites, online=online, arena_bytes=lg.total_bytes + 128 * lg.n + (1 << 20),
                    max_records=lg.n) as log:
        for rep in range(2):
            log.reset()
            torch.cuda.synchronize()
            ts = []
            for a in range(0, lg.n - w + 1, w):
                e = a + w
                t0 = time.perf_counter()
                log.append_batch(lg.site[a:e], lg.size[a:e], ptrs[a:e], lg.dur[a:e], payload_kind=ffm.FFM_PAYLOAD_DEVICE)
                t1 = time.perf_counter()
                torch.cuda.synchronize()
                t2 = time.perf_counter()
                ts.append((t1 - t0, t2 - t0))
            if rep:
                print(f"online={online}: append call {np.median([t[0] for t in ts]) * 1e3:.3f} ms, "
                      f"+ device work {np.median([t[1] for t in ts]) * 1e3:.3f} ms per {w} records", flush=True)
    # the binding's own marshalling
    t0 = time.perf_counter()
    for _ in range(10):
        a = np.ascontiguousarray(lg.site[:w], np.uint32)
        b = np.ascontiguousarray(lg.size[:w], np.uint64)
        c = np.ascontiguousarray(ptrs[:w], np.uint64)
        d = np.ascontiguousarray(lg.dur[:w], np.uint64)
    print(f"numpy marshalling {(time.perf_counter() - t0) / 10 * 1e3:.3f} ms", flush=True)
