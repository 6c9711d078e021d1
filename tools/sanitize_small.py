"""Racecheck companion of sanitize_smoke.py: logs whose payloads are all <= small_bytes
(no k_fused_fx launch), so that every other kernel's shared-memory accesses are checked
without the pipelined pass's mbarrier-ordered hazards filling the report."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import loggen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_sc_weltonm19_b200 as ffm  # noqa: E402

for k, ns, ss in [(2, 0.002, 1.0), (5, 0.001, 1 / 64)]:
    lg = loggen.gen_config(k, n_scale=ns, size_scale=ss)
    want = oracle.dedup(lg)
    for db, extra in [(64, {}), (0, {}), (64, {"two_pass": True}), (8, {"fused": True})]:
        with ffm.FfmLog(lg.n_sites, digest_bits=db, small_bytes=1 << 20, chunk_bytes=1 << 20, **extra) as log:
            log.append_log(lg)
            d, b = log.run()
            assert np.array_equal(d, want[0]) and np.array_equal(b, want[1]), (k, db, extra)
print("sanitize small ok")
