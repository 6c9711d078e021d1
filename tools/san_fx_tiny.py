"""A handful of large records through k_fused_fx (hash + verify mode) for racecheck with
synchronisation tracing.  usage: san_fx_tiny.py [libffm.so]"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import loggen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_sc_weltonm19_b200 as ffm  # noqa: E402

if len(sys.argv) > 1:
    ffm.set_library_path(sys.argv[1])
pay = [bytes([i % 7]) * 20000 for i in range(6)] + [bytes([1]) * 20000, bytes([3]) * 20000]
lg = loggen.from_payloads(pay, [0] * len(pay), None, 1)
want = oracle.dedup(lg)
with ffm.FfmLog(1, chunk_bytes=4096, small_bytes=1024, fused=True) as log:
    log.append_log(lg)
    d, b = log.run()
    assert np.array_equal(d, want[0]) and np.array_equal(b, want[1])
print("san fx tiny ok", d.tolist(), flush=True)
