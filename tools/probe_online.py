"""Online mode: per-step wall time split for one window size (config 2), for profiling
under ncu (launch list) -- where a step's time goes (kernels vs host)."""
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

w = int(sys.argv[1]) if len(sys.argv) > 1 else 65536
nwin = int(sys.argv[2]) if len(sys.argv) > 2 else 8
append_hash = (sys.argv[3] == "append_hash") if len(sys.argv) > 3 else True
timing = len(sys.argv) > 4 and sys.argv[4] == "timing"
lg = loggen.gen_config(2)
lg.materialize(nthreads=0)
content = torch.from_numpy(lg.buf).cuda()
ptrs = (lg.c_off[lg.content] + np.uint64(content.data_ptr())).astype(np.uint64)
dup = torch.empty(w, dtype=torch.int64, device="cuda")
ben = torch.empty(lg.n_sites, dtype=torch.int64, device="cuda")
with ffm.FfmLog(lg.n_sites, online=True, append_hash=append_hash, timing=timing, arena_bytes=lg.total_bytes + 128 * lg.n + (1 << 20), max_records=lg.n) as log:
    for rep in range(2):
        log.reset()
        ta, ts = [], []
        for a in range(0, min(lg.n, nwin * w), w):
            e = min(lg.n, a + w)
            t0 = time.perf_counter()
            log.append_batch(lg.site[a:e], lg.size[a:e], ptrs[a:e], lg.dur[a:e], payload_kind=ffm.FFM_PAYLOAD_DEVICE)
            torch.cuda.synchronize()
            t1 = time.perf_counter()
            log.online_step(dup, ben)
            t2 = time.perf_counter()
            ta.append(t1 - t0)
            ts.append(t2 - t1)
            if timing and rep == 1:
                st = log.stats()
                print({k: round(v, 4) for k, v in st.items() if k.startswith("ms_") or k in ("host_syncs", "kernel_launches", "n_residual", "resolve_rounds")}, flush=True)
        print(f"rep {rep} window {w}: append+hash median {np.median(ta) * 1e3:.3f} ms, step median {np.median(ts) * 1e3:.3f} ms "
              f"stats {log.stats()['host_syncs']} syncs", flush=True)
