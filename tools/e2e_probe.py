"""Time the phases of one end-to-end step (create / append / run / destroy) from pinned
host memory, for the H0 staging design.  Not part of the product; run under gpurun."""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import loggen  # noqa: E402
import paper_conf_sc_weltonm19_b200 as ffm  # noqa: E402

k = int(sys.argv[1]) if len(sys.argv) > 1 else 5
lg = loggen.gen_config(k)
buf = lg.materialize()
t = time.time()
rc = torch.cuda.cudart().cudaHostRegister(buf.ctypes.data, buf.nbytes, 0)
print("register", rc, time.time() - t, flush=True)
ptrs = lg.payload_ptrs()
dup = torch.empty(lg.n, dtype=torch.int64).pin_memory()
ben = torch.empty(lg.n_sites, dtype=torch.int64).pin_memory()
for it in range(3):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    log = ffm.FfmLog(lg.n_sites, arena_bytes=lg.total_bytes + 128 * lg.n + (1 << 20), max_records=lg.n)
    t1 = time.perf_counter()
    log.append_batch(lg.site, lg.size, ptrs, lg.dur, payload_kind=ffm.FFM_PAYLOAD_HOST_PINNED)
    t2 = time.perf_counter()
    log.run(dup.numpy(), ben.numpy().view(np.uint64))
    t3 = time.perf_counter()
    log.close()
    t4 = time.perf_counter()
    print(f"it{it}: create {t1-t0:.3f}s append {t2-t1:.3f}s ({lg.total_bytes/(t2-t1)/1e9:.1f} GB/s) "
          f"run {t3-t2:.3f}s destroy {t4-t3:.3f}s total {t4-t0:.3f}s",
          flush=True)
