"""Debug driver: one sharded case (3 ranks sharing a GPU, host transport) under several
digest_bits / refine_bits / round-0 modes, result vs the oracle -- the harness that found the
legacy-stream memset race of the slow-path segment arrays.  usage: debug_sharded_case.py [libffm.so]"""
import os, sys, tempfile, pathlib, traceback
sys.path.insert(0, os.getcwd()); sys.path.insert(0, os.path.join(os.getcwd(), "tests"))
import numpy as np
import test_gpu_sharded as t
import torch.multiprocessing as mp
import loggen, oracle

def worker(rank, world, port, out_dir, case, policy, digest_bits, refine_bits, extra):
    import torch, torch.distributed as dist
    import paper_conf_sc_weltonm19_b200 as ffm
    if len(sys.argv) > 1:
        ffm.set_library_path(sys.argv[1])
    from paper_conf_sc_weltonm19_b200 import sharded
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    lg = t._make(case)
    ranks = ffm.ffm_shard_plan(lg.site, lg.size, lg.n_sites, world, policy)
    idx = np.nonzero(ranks == rank)[0]
    log = sharded.create_sharded_log(lg.n_sites, 0, transport="host", digest_bits=digest_bits,
                                     refine_bits=refine_bits, chunk_bytes=4096, **extra)
    log.append_log(lg, gids=idx, idx=idx)
    dup, ben = log.run()
    st = log.stats()
    np.savez(os.path.join(out_dir, f"r{rank}.npz"), idx=idx, dup=dup.copy(), ben=ben.copy(), nslow=st["n_slow"])
    log.close()
    dist.destroy_process_group()

if __name__ == "__main__":
    case = "c5+ch"
    lg = t._make(case)
    want_d, want_b = oracle.dedup(lg)
    for name, db, rb, extra in [("db0", 0, 64, {}), ("db0 rb0", 0, 0, {}), ("db0 two_pass", 0, 64, {"two_pass": True}),
                                ("db64", 64, 64, {}), ("db8", 8, 64, {})]:
        d = tempfile.mkdtemp()
        mp.spawn(worker, args=(3, t._free_port(), d, case, 1, db, rb, extra), nprocs=3, join=True)
        got = np.full(lg.n, -7, np.int64); ok_b = True; ns = 0
        for r in range(3):
            z = np.load(os.path.join(d, f"r{r}.npz")); got[z["idx"]] = z["dup"]; ok_b &= np.array_equal(z["ben"], want_b); ns += int(z["nslow"])
        bad = np.nonzero(got != want_d)[0]
        print(name, "dup ok" if len(bad) == 0 else f"dup BAD {len(bad)} e.g. {bad[:5]} got {got[bad[:5]]} want {want_d[bad[:5]]} sizes {lg.size[bad[:5]]}", "ben ok" if ok_b else "ben BAD", "n_slow", ns, flush=True)
