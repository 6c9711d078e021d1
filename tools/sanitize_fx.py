"""Large payloads only, for compute-sanitizer racecheck of the TMA-pipelined fused pass
(k_fused_fx in hash and verify mode; groups of > 64 members; 64 KiB chunks split into
pieces).  A few hundred records: racecheck instruments every shared-memory access."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import loggen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_sc_weltonm19_b200 as ffm  # noqa: E402

for k, ns, ss in [(4, 0.02, 1 / 512), (3, 0.008, 1 / 128)]:
    lg = loggen.gen_config(k, n_scale=ns, size_scale=ss)
    want = oracle.dedup(lg)
    for extra in ({"fused": True}, {"two_pass": True}, {"fused": True, "chunk_bytes": 65536}):
        with ffm.FfmLog(lg.n_sites, small_bytes=1024, **dict({"chunk_bytes": 4096}, **extra)) as log:
            log.append_log(lg)
            d, b = log.run()
            assert np.array_equal(d, want[0]) and np.array_equal(b, want[1]), (k, extra)
print("sanitize fx ok", flush=True)
