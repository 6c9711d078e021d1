#!/usr/bin/env python3
"""bench.py -- payload GB/s deduplicated on B200, with roofline and CPU-oracle baselines.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload 5] [--impl ours|reference]

--gpus N > 1 without a torchrun environment re-launches itself as N ranks (one per
GPU) under torch.distributed.run; ffm_dedup_run is then collective over the library's
own NCCL communicator.

A step = one ffm_dedup_run over the whole log (H1 hash .. H7 labels/benefit, all
of SURVEY.md 8(a)) with the payloads already resident in HBM.  Default workload
= BASELINE config 5 (the ~64 GB mixed application-shaped log, 2 M transfers,
10k call sites) on one GPU; inputs (63 GB) are far larger than L2 (126 MB).

  value    = sum of payload bytes / time per step (CUDA events on the library's
             stream, max over ranks), GB/s (1e9); every run writes duplicate_of /
             benefit_ns into pinned HOST arrays (the D2H is inside the step, SURVEY.md
             8(d) T_run); value_device_outputs keeps them in HBM.
  e2e      = the same metric through the public C ABI from pinned HOST buffers:
             ffm_log_create + ffm_log_append_batch (H2D of every payload) +
             ffm_dedup_run + D2H of duplicate_of / benefit_ns, per step.
  roofline = the dominant kernel's algorithmic bytes / its CUDA-event time vs
             the measured HBM copy bandwidth (MEASURED_PEAKS.json).
  cpu_baseline = the CPU oracle (oracle/) on a bounded gid-prefix sample, 1 core.

--impl reference times the oracle (the only "reference" this tier has) on the
host cores, on this arm's config / metric / unit.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "payload GB/s deduplicated (1/2/4/8 B200) and % of HBM roofline"
UNIT = "GB/s"
WORKLOADS = {
    1: "config1: 1,000 transfers 4 KB-1 MB, 30% planted dups, 50 sites",
    2: "config2: 1M small transfers 256 B-4 KB, 60% re-uploads, 256 sites",
    3: "config3: 10,000 x 1 MiB near-duplicates, single-byte differences",
    4: "config4: 1,000 large transfers 16-64 MiB, 20 solver arrays x 50 iterations",
    5: "config5: mixed application-shaped log, 2M transfers, ~64 GB, 10k call sites",
}


def log_msg(*a):
    print(*a, file=sys.stderr, flush=True)


def dist_env():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), \
        int(os.environ.get("LOCAL_RANK", 0))


def load_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons during the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device):
        self.device = device
        self.proc = None
        self.path = f"/tmp/ffm_clocks_{os.getpid()}.csv"

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=open(self.path, "w"), stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return None
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], 0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in open(self.path):
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = max(mx, float(f[2]))
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return None
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def make_log(workload, n_scale, size_scale, shard=(0, 1)):
    """The workload's log; with shard=(rank, world) > 1 only that rank's records'
    contents are materialised (site-affinity LPT plan) -- lg.shard_idx lists them."""
    import loggen
    import paper_conf_sc_weltonm19_b200 as ffm
    t = time.time()
    lg = loggen.gen_config(workload, n_scale=n_scale, size_scale=size_scale)
    rank, world = shard
    if world > 1:
        ranks = ffm.ffm_shard_plan(lg.site, lg.size, lg.n_sites, world, ffm.FFM_SHARD_SITE_LPT)
        lg.shard_idx = np.nonzero(ranks == rank)[0]
        lg.materialize(nthreads=0, records=lg.shard_idx)
    else:
        lg.shard_idx = np.arange(lg.n)
        lg.materialize(nthreads=0)
    log_msg(f"[bench] generated {lg.name}: {lg.n} records, {lg.total_bytes / 1e9:.2f} GB payload, "
            f"{lg.distinct_bytes / 1e9:.2f} GB distinct, {time.time() - t:.1f}s")
    return lg


def alg_bytes(lg, idx, dup, small_bytes, chunk=32768, two_pass=False, prefix=4096):
    """Algorithmic bytes per kernel for this rank's records idx: every
    payload byte is hashed once; a member payload's bytes are compared once against its
    leader, whose bytes are read once per class.
      prefix (k_prefix_hash):  sum over large payloads of p0 = min(size, prefix)
      fused  (k_fused_fx):  sum over large (size - p0) + members' p0 + their leaders' p0
                            (a group's first pieces are compared from byte 0)
      small  (k_fused_small): small sizes + leaders of small members
    two-pass: k_hash_large hashes every large byte, then members and their class leaders
    are read once more (verify); small: k_hash_small, then k_verify_small (side stream,
    concurrent with the large verify).
    dup: this rank's duplicate_of (global gids)."""
    size = lg.size[idx].astype(np.int64)
    n = len(size)
    small = size <= small_bytes
    member = dup >= 0
    leaders = np.zeros(n, bool)
    if member.any():
        pos = np.full(lg.n, -1, np.int64)
        pos[idx] = np.arange(n)
        lp = pos[dup[member]]
        leaders[lp[lp >= 0]] = True
    big = ~small
    p0 = np.minimum(size, prefix)
    units = int(((size[big] + chunk - 1) // chunk).sum())
    out = {
        "small": int(size[small].sum()) + int(size[small & leaders].sum()) + 40 * int(small.sum()),
        "prefix": int(p0[big].sum()) + 40 * int(big.sum()),
        "fused": int((size[big] - p0[big]).sum()) + int(p0[big & member].sum()) + int(p0[big & leaders].sum())
        + 32 * units,
    }
    if two_pass:
        out["small"] = int(size[small].sum()) + 32 * int(small.sum())      # k_hash_small only
        out["verify_small"] = int(size[small & member].sum()) + int(size[small & leaders].sum())
        out["prefix"] = int(size[big].sum()) + 40 * units
        out["fused"] = int(size[big & member].sum()) + int(size[big & leaders].sum())
    out["path"] = sum(out.values()) + 64 * n    # + group-by / label metadata
    return out


def ncu_traffic(kernel, capture):
    """dram bytes per launch of `kernel` from the committed ncu --set full capture of the
    same workload and round-0 mode (profiles/ncu_summary.json), else None."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        d = json.load(open(p))
        k = d["captures"][capture]["kernels"].get(kernel)
        return None if k is None else float(k["dram_bytes_per_launch"])
    except Exception:
        return None


def make_ffm_log(args, lg, n_records, my_bytes, rank, world, local, **kw):
    """This rank's log: one GPU, or a sharded world (collective: the library's NCCL
    communicator across GPUs; the host transport when ranks share a GPU)."""
    import paper_conf_sc_weltonm19_b200 as ffm
    from paper_conf_sc_weltonm19_b200 import sharded
    opts = dict(arena_bytes=my_bytes + 128 * n_records + (1 << 20), max_records=n_records, **kw)
    if world == 1 and args.collective:     # the collective path (library NCCL) in a world of one
        return ffm.FfmLog(lg.n_sites, device=local, nccl_id=ffm.ffm_nccl_unique_id(), **opts)
    if world == 1:
        return ffm.FfmLog(lg.n_sites, device=local, **opts)
    return sharded.create_sharded_log(lg.n_sites, local, transport="host" if args.same_device else "nccl", **opts)


def run_ours(args):
    import torch
    import torch.distributed as dist

    rank, world, local = dist_env()
    if args.same_device:                 # test hook: several ranks on one GPU
        local = 0
    elif world > 1 and torch.cuda.device_count() < world:
        raise SystemExit(f"bench: {world} ranks but {torch.cuda.device_count()} visible GPUs "
                         "(--same-device runs them on one GPU, host transport)")
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        # bootstrap / host-side timing reduction only; the data plane is the library's
        # own NCCL communicator (or its host transport under --same-device)
        dist.init_process_group("gloo")
    lg = make_log(args.workload, args.n_scale, args.size_scale, shard=(rank, world))
    idx = lg.shard_idx
    total = lg.total_bytes                      # the whole job's payload (strong scaling)
    my_bytes = int(lg.size[idx].sum())

    # ---- device-resident log: this rank's distinct contents uploaded once, records
    # snapshotted into the library's HBM arena
    t = time.time()
    content = torch.from_numpy(lg.buf).to(dev)
    ptrs = (lg.c_off[lg.content] + np.uint64(content.data_ptr())).astype(np.uint64)
    import paper_conf_sc_weltonm19_b200 as ffm
    log = make_ffm_log(args, lg, len(idx), my_bytes, rank, world, local, timing=True,
                       prefilter=args.prefilter and world == 1, digest_bits=args.digest_bits,
                       two_pass=args.two_pass)
    log.append_log(lg, ptrs=ptrs, payload_kind=ffm.FFM_PAYLOAD_DEVICE,
                   gids=idx if world > 1 else None, idx=idx if world > 1 else None)
    del content
    torch.cuda.synchronize()
    torch.cuda.empty_cache()
    log_msg(f"[bench] rank {rank}: staged {my_bytes / 1e9:.2f} GB ({len(idx)} records) into HBM "
            f"in {time.time() - t:.1f}s")

    n = len(idx)
    # outputs: host (pinned) arrays -- the D2H of duplicate_of / benefit_ns is inside the
    # timed run (SURVEY.md 8(d) T_run); device arrays for the kernel-side figure
    dup_h = torch.empty(max(n, 1), dtype=torch.int64).pin_memory()
    ben_h = torch.empty(lg.n_sites, dtype=torch.int64).pin_memory()
    dup_hn, ben_hn = dup_h.numpy(), ben_h.numpy().view(np.uint64)
    dup_d = torch.empty(max(n, 1), dtype=torch.int64, device=dev)
    ben_d = torch.empty(lg.n_sites, dtype=torch.int64, device=dev)

    def step(host=True):
        if host:
            log.run(dup_hn, ben_hn)
        else:
            log.run(dup_d, ben_d)

    def max_over_ranks(x):
        if world == 1:
            return x
        t_ = torch.tensor([x], dtype=torch.float64)
        dist.all_reduce(t_, op=dist.ReduceOp.MAX)
        return float(t_.item())

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()

    stream = torch.cuda.ExternalStream(log.stream, device=dev)
    for _ in range(args.warmup):
        step()
    barrier()
    clocks = ClockSampler(local) if rank == 0 else None
    if clocks:
        clocks.start()
        time.sleep(0.3)
    # measured steps: production runs (CUDA-graph replay, no per-stage events), events on
    # the library's stream (every kernel, collective and output copy of a run is on it)
    log.set_timing(False)
    step()

    def timed(host):
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.steps):
            step(host)
        e1.record(stream)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / args.steps

    ms_local = timed(True)
    ms = max_over_ranks(ms_local)
    ms_dev_local = timed(False)
    ms_dev = max_over_ranks(ms_dev_local)
    clk = clocks.stop() if clocks else None
    launches = int(log.stats()["kernel_launches"]) * args.steps
    # instrumented steps (per-stage CUDA events on the library's stream) for the kernel
    # roofline: same kernels, launched directly
    log.set_timing(True)
    acc = {}
    n_instr = max(3, min(args.steps, 5))
    for _ in range(n_instr):
        step(False)
        for k, v in log.stats().items():
            acc[k] = acc.get(k, 0) + v
    st = {k: v / n_instr for k, v in acc.items()}
    value = total / (ms * 1e-3) / 1e9

    # algorithmic bytes and the dominant kernel on this rank (rank 0 reports)
    dup_np = dup_d[:n].cpu().numpy()
    ab = alg_bytes(lg, idx, dup_np, 4096, two_pass=args.two_pass or st.get("two_pass", 0) >= 0.5)
    if args.prefilter and world == 1:
        # only the bytes the pre-filtered path must read: the library reports the bytes it
        # hashed beyond first chunks (prefix-unique payloads skip theirs)
        sz = lg.size[idx].astype(np.int64)
        big = sz > 4096
        mem = dup_np >= 0
        p0 = np.minimum(sz, 4096)
        ab["fused"] = int(st["prefilter_rest_bytes"]) + int(p0[big & mem].sum()) + 32 * int(((sz[big] + 32767) // 32768).sum())
        ab["path"] = sum(v for k, v in ab.items() if k != "path") + 64 * n
    peak, peak_src = load_peak()
    kern_ms = {"small": st["ms_hash_small"], "prefix": st["ms_hash_large"], "fused": st["ms_fused"]}
    dom = max(kern_ms, key=lambda k: kern_ms[k])
    dom_ms = kern_ms[dom]
    achieved = ab[dom] / (dom_ms * 1e-3) / 1e9 if dom_ms > 0 else 0.0
    two_pass = args.two_pass or st.get("two_pass", 0) >= 0.5
    kname = {"small": "k_hash_small" if two_pass else "k_fused_small",
             "prefix": "k_hash_large" if two_pass else "k_prefix_hash",
             "fused": "k_fused_fx"}[dom]
    mode = "two-pass" if two_pass else "fused"
    capture = f"config{args.workload}/{mode}" + ("/prefilter" if args.prefilter else "") + \
        (f"/digest_bits{args.digest_bits}" if args.digest_bits < 64 else "")
    traffic = ncu_traffic(kname, capture) if world == 1 and args.n_scale == 1 and args.size_scale == 1 else None
    roofline = {"bound": "hbm", "kernel": kname, "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                "frac": round(achieved / peak, 4), "traffic": traffic, "alg_bytes": ab[dom],
                "ms": round(dom_ms, 4), "peak_source": peak_src,
                "read_stream_ceiling_gbs": read_ceiling(),
                "note": "peak is the driver's copy (read+write) figure; the kernel is a pure read stream, "
                        "so frac > 1 is possible -- read_stream_ceiling_gbs is the measured 256-bit read ceiling",
                "traffic_source": f"profiles/ncu_summary.json captures[{capture}] (ncu --set full of the same "
                                  "workload and mode; committed capture, not measured in this run)"
                if traffic is not None else "no committed ncu capture of this workload/mode"}
    path_gbs = ab["path"] / (ms_dev * 1e-3) / 1e9

    # per-rank terms of the scaling cost model: local time, B_x, exchange
    mine = {"rank": rank, "ms": round(ms_local, 4), "ms_device_outputs": round(ms_dev_local, 4),
            "records": n, "payload_bytes": my_bytes,
            "reps_local": int(st.get("n_reps_local", 0)), "reps_global": int(st.get("n_reps_global", 0)),
            "remote_verify_bytes": int(st.get("remote_verify_bytes", 0)),
            "exchange_bytes": int(st.get("exchange_bytes", 0)), "slow_reps": int(st.get("n_slow", 0)),
            "host_syncs": int(st.get("host_syncs", 0)), "ms_exchange": round(st.get("ms_exchange", 0.0), 4)}
    per_rank = [mine]
    if world > 1:
        per_rank = [None] * world
        dist.all_gather_object(per_rank, mine)

    parity = None
    if args.check:
        parity = check_parity(lg, args, idx, dup_np, ben_d.cpu().numpy().view(np.uint64), rank, world)

    e2e = None
    if args.e2e_steps > 0:
        del log
        torch.cuda.empty_cache()
        e2e = run_e2e(args, lg, local, rank, world)
    cpu = cpu_baseline(lg, args.cpu_seconds) if (args.cpu_seconds > 0 and world == 1) else None
    if world > 1:
        dist.barrier()
    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return
    out = {
        "metric": METRIC, "value": round(value, 2), "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(ms, 4), "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": {"workload": WORKLOADS[args.workload], "records": lg.n, "payload_bytes": total,
                   "n_sites": lg.n_sites, "seed": "0x5C19D1000%d" % args.workload,
                   "n_scale": args.n_scale, "size_scale": args.size_scale,
                   "l2": "inputs larger than L2 (payload %.1f GB >> 126 MB L2)" % (total / 1e9),
                   "parallelism": ("single GPU, collective path (library NCCL communicator, world of one)"
                                   if args.collective else "single GPU") if world == 1 else
                   f"{world} shards (site-affinity LPT), collective ffm_dedup_run: "
                   + ("host transport, ranks sharing one GPU (test hook)" if args.same_device else
                      "library-owned NCCL all-gather of class representatives + all-reduce of per-site sums, "
                      "in-kernel peer byte verify over NVLink"),
                   "outputs": "host (pinned): duplicate_of / benefit_ns D2H inside every timed run",
                   "chunk_bytes": 32768, "small_bytes": 4096, "prefilter": bool(args.prefilter and world == 1),
                   "digest_bits": args.digest_bits,
                   "round0": "two-pass (forced)" if args.two_pass else
                   ("two-pass (adaptive)" if st.get("two_pass", 0) >= 0.5 else "fused")},
        "value_device_outputs": round(total / (ms_dev * 1e-3) / 1e9, 2),
        "ms_per_step_device_outputs": round(ms_dev, 4),
        "pct_hbm_roofline_path": round(path_gbs / peak, 4),
        "path_alg_gbs": round(path_gbs, 1),
        "stage_ms": {k: round(st[k], 4) for k in ("ms_hash_small", "ms_hash_large", "ms_group", "ms_verify",
                                                  "ms_fused", "ms_resolve", "ms_label", "ms_output", "ms_total",
                                                  "ms_exchange")},
        "clocks": clk, "gpu_launches": launches, "roofline": roofline, "e2e": e2e, "cpu_baseline": cpu,
        "per_rank": per_rank, "parity": parity,
        "duplicates_rank0": int((dup_np >= 0).sum()),
        "collisions": {"residual_members": int(round(st["n_residual"])), "resolve_rounds": int(round(st["resolve_rounds"]))},
    }
    print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


def run_online(args):
    """S8(f) #2 measurement: the log streamed through ffm_online_step in fixed windows
    (FFM_FLAG_ONLINE; FFM_FLAG_APPEND_HASH: each append hashes its records on the hashing stream), against the
    batch run of the same log.  Per window size: median step latency (host wall clock of
    the synchronous ffm_online_step) and streamed throughput = payload / (sum of append +
    step times); appends snapshot device-resident payloads (D2D)."""
    import torch
    import paper_conf_sc_weltonm19_b200 as ffm
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    lg = make_log(args.workload, args.n_scale, args.size_scale)
    content = torch.from_numpy(lg.buf).to(dev)
    ptrs = (lg.c_off[lg.content] + np.uint64(content.data_ptr())).astype(np.uint64)
    want = None
    if args.check:
        import oracle
        want = oracle.dedup(lg)
    opts = dict(arena_bytes=lg.total_bytes + 128 * lg.n + (1 << 20), max_records=lg.n)
    # batch reference: the same log in one ffm_dedup_run (device outputs)
    with ffm.FfmLog(lg.n_sites, **opts) as log:
        log.append_log(lg, ptrs=ptrs, payload_kind=ffm.FFM_PAYLOAD_DEVICE)
        d = torch.empty(lg.n, dtype=torch.int64, device=dev)
        b = torch.empty(lg.n_sites, dtype=torch.int64, device=dev)
        for _ in range(args.warmup):
            log.run(d, b)
        torch.cuda.synchronize()
        t = time.perf_counter()
        for _ in range(args.steps):
            log.run(d, b)
        torch.cuda.synchronize()
        batch_s = (time.perf_counter() - t) / args.steps
    rows = []
    for (mode, append_hash), w in [(m, int(x)) for m in (("fused", False), ("append_hash", True))
                                   for x in args.online.split(",")]:
        # both modes are online logs (FFM_FLAG_ONLINE: appends upload their metadata);
        # append_hash also hashes at append time (FFM_FLAG_APPEND_HASH)
        n_win = (lg.n + w - 1) // w
        if n_win > args.online_max_windows:          # latency only, over a bounded prefix
            n_win = args.online_max_windows
        end = min(lg.n, n_win * w)
        dup = torch.empty(max(w, 1), dtype=torch.int64, device=dev)
        ben = torch.empty(lg.n_sites, dtype=torch.int64, device=dev)
        got = np.empty(end, np.int64) if want is not None else None
        t_app, t_step = [], []
        with ffm.FfmLog(lg.n_sites, online=True, append_hash=append_hash, **opts) as log:
            for rep in range(2):                     # rep 0 warms up (allocations), rep 1 is measured
                log.reset()
                t_app.clear()
                t_step.clear()
                torch.cuda.synchronize()
                for a in range(0, end, w):
                    e = min(end, a + w)
                    t0 = time.perf_counter()
                    log.append_batch(lg.site[a:e], lg.size[a:e], ptrs[a:e], lg.dur[a:e],
                                     payload_kind=ffm.FFM_PAYLOAD_DEVICE)
                    t1 = time.perf_counter()
                    log.online_step(dup, ben)
                    t2 = time.perf_counter()
                    t_app.append(t1 - t0)
                    t_step.append(t2 - t1)
                    if got is not None and rep == 1:
                        got[a:e] = dup[:e - a].cpu().numpy()
        byts = int(lg.size[:end].sum())
        row = {"mode": mode, "window": w, "windows": len(t_step), "records": end, "payload_bytes": byts,
               "step_ms_median": round(statistics.median(t_step) * 1e3, 4),
               "step_ms_p90": round(float(np.percentile(t_step, 90)) * 1e3, 4),
               "append_ms_median": round(statistics.median(t_app) * 1e3, 4),
               "streamed_gbs": round(byts / (sum(t_app) + sum(t_step)) / 1e9, 2),
               "steps_only_gbs": round(byts / sum(t_step) / 1e9, 2)}
        if got is not None:
            row["parity"] = "ok" if np.array_equal(got, want[0][:end]) else "MISMATCH"
        rows.append(row)
        log_msg(f"[bench] online window {w}: {row}")
    out = {"metric": METRIC, "mode": "online (S8(f) #2)", "workload": WORKLOADS[args.workload],
           "records": lg.n, "payload_bytes": lg.total_bytes, "n_scale": args.n_scale,
           "batch_ms": round(batch_s * 1e3, 4), "batch_gbs": round(lg.total_bytes / batch_s / 1e9, 2),
           "windows": rows,
           "note": "host wall clock; appends snapshot device-resident payloads; mode fused: each step runs the "
                   "fused round 0 on its window (batch record order built on the device); mode append_hash: "
                   "appends queue the window's hashing (FFM_FLAG_APPEND_HASH), the step verifies two-pass; each step "
                   "is synchronous (labels in device memory)"}
    print(json.dumps(out), flush=True)


def check_parity(lg, args, idx, dup, ben, rank, world):
    """Every rank's duplicate_of (global gids) and the global benefit against the CPU
    oracle on the whole log (rank 0; small logs)."""
    import oracle
    import loggen
    import torch.distributed as dist
    parts = [(idx, dup)]
    if world > 1:
        parts = [None] * world
        dist.all_gather_object(parts, (idx, dup))
    if rank != 0:
        return None
    full = loggen.gen_config(args.workload, n_scale=args.n_scale, size_scale=args.size_scale)
    want_d, want_b = oracle.dedup(full)
    got = np.full(full.n, -7, np.int64)
    for i, d in parts:
        got[i] = d
    ok = bool(np.array_equal(got, want_d) and np.array_equal(ben, want_b))
    return {"oracle": "ok" if ok else "MISMATCH", "records": int(full.n),
            "mismatched_records": int((got != want_d).sum())}


def read_ceiling():
    try:
        for line in open(os.path.join(ROOT, "profiles", "r01_hbm_ceiling.json")):
            d = json.loads(line)
            if d.get("test") == "read_stream_256b":
                return d["gbs"]
    except Exception:
        return None


def run_e2e(args, lg, local, rank=0, world=1):
    """The metric end to end through the public C ABI, per step: ffm_log_reset +
    ffm_log_append_batch of every payload from HOST memory (H2D inside the step) +
    ffm_dedup_run with host output arrays (D2H inside).  Pinned source buffers (the
    copy engines / k_gather read them in place) and pageable ones (staged through the
    library's pinned ring), each over args.e2e_steps steps after one warm-up step."""
    import torch
    import torch.distributed as dist
    import paper_conf_sc_weltonm19_b200 as ffm
    buf = lg.buf
    idx = lg.shard_idx
    ptrs = lg.payload_ptrs()[idx]
    n = len(idx)
    my_bytes = int(lg.size[idx].sum())
    dup_pin = torch.empty(max(n, 1), dtype=torch.int64).pin_memory()
    ben_pin = torch.empty(lg.n_sites, dtype=torch.int64).pin_memory()
    # one long-lived log (allocated once, like any buffer); every step empties it
    # (ffm_log_reset keeps the HBM allocations)
    log = make_ffm_log(args, lg, n, my_bytes, rank, world, local)
    cudart = torch.cuda.cudart()

    def measure(kind, steps):
        times, phases = [], []
        for step in range(steps + 1):
            torch.cuda.synchronize()
            if world > 1:
                dist.barrier()
            t0 = time.perf_counter()
            log.reset()
            t1 = time.perf_counter()
            log.append_batch(lg.site[idx], lg.size[idx], ptrs, lg.dur[idx], gids=idx if world > 1 else None,
                             payload_kind=kind)
            t2 = time.perf_counter()
            log.run(dup_pin.numpy(), ben_pin.numpy().view(np.uint64))
            t3 = time.perf_counter()
            sec = t3 - t0
            if world > 1:
                tt = torch.tensor([sec], dtype=torch.float64)
                dist.all_reduce(tt, op=dist.ReduceOp.MAX)
                sec = float(tt.item())
            if step > 0:                     # the first step warms up
                times.append(sec)
                phases.append((t1 - t0, t2 - t1, t3 - t2))
        sec = statistics.median(times)
        return {"value": round(lg.total_bytes / sec / 1e9, 3), "steps": len(times), "s_per_step": round(sec, 4),
                "phases_s": dict(zip(("reset", "append_h2d", "run_d2h"),
                                     [round(statistics.median(p), 4) for p in zip(*phases)]))}

    reg = -1
    try:
        reg = int(cudart.cudaHostRegister(buf.ctypes.data, buf.nbytes, 0))
    except Exception:
        pass
    pinned = measure(ffm.FFM_PAYLOAD_HOST_PINNED if reg == 0 else ffm.FFM_PAYLOAD_HOST, args.e2e_steps)
    if reg == 0:
        cudart.cudaHostUnregister(buf.ctypes.data)
    pageable = measure(ffm.FFM_PAYLOAD_HOST, args.e2e_steps) if args.e2e_pageable else None
    log.close()
    meta = lg.n * (4 + 8 + 8 + 8)
    out = {"value": pinned["value"], "unit": UNIT,
           "h2d_bytes_per_step": int(lg.total_bytes + meta), "d2h_bytes_per_step": int(8 * lg.n + 8 * lg.n_sites * world),
           "steps": pinned["steps"], "s_per_step": pinned["s_per_step"], "phases_s": pinned["phases_s"],
           "source": "pinned host buffers (cudaHostRegister)" if reg == 0 else "pageable host buffers",
           "note": "wall clock per step, max over ranks, median: ffm_log_reset + append (host -> HBM) + "
                   "ffm_dedup_run with host output arrays (D2H of duplicate_of / benefit_ns)"}
    if pageable:
        out["pageable"] = dict(pageable, unit=UNIT, source="pageable host buffers (library's pinned staging ring)")
    return out


def oracle_sample(lg, seconds_budget):
    """gid-prefix of the log whose oracle time is ~seconds_budget (calibrated)."""
    import oracle
    n = lg.n
    csum = np.cumsum(lg.size.astype(np.int64))
    # calibrate on a small prefix
    k = int(np.searchsorted(csum, min(csum[-1], 200_000_000))) + 1
    k = max(1, min(k, n))
    t = time.perf_counter()
    oracle.dedup(lg.subset(np.arange(k)))
    dt = max(time.perf_counter() - t, 1e-6)
    rate = csum[k - 1] / dt
    want = rate * seconds_budget
    k2 = int(np.searchsorted(csum, want)) + 1
    return max(1, min(k2, n)), rate


def cpu_baseline(lg, seconds):
    import oracle
    try:
        os.sched_setaffinity(0, {sorted(os.sched_getaffinity(0))[0]})
        cores = 1
    except Exception:
        cores = 1
    k, _ = oracle_sample(lg, seconds)
    sub = lg.subset(np.arange(k))
    t = time.perf_counter()
    oracle.dedup(sub)
    dt = time.perf_counter() - t
    b = int(lg.size[:k].sum())
    return {"value": round(b / dt / 1e9, 3), "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"gid prefix of {k} of {lg.n} records ({b / 1e9:.2f} GB of {lg.total_bytes / 1e9:.2f} GB), "
                      f"{dt:.1f}s on 1 of {os.cpu_count()} host cores"}


def run_reference(args):
    """The reference arm of this tier: the CPU oracle as it stands, 1 core, on this arm's
    workload -- the whole log per timed step when K of them fit args.ref_budget seconds
    (else the largest gid prefix that does, said in `sample`).  Warm-up steps run the
    oracle on a small prefix (it keeps no state between calls)."""
    rank, world, _ = dist_env()
    if rank != 0:
        return
    import oracle
    lg = make_log(args.workload, args.n_scale, args.size_scale)
    os.sched_setaffinity(0, {sorted(os.sched_getaffinity(0))[0]})
    k_cal, rate = oracle_sample(lg, 1.0)
    t_full = lg.total_bytes / rate
    if args.steps * t_full <= args.ref_budget:
        k = lg.n
    else:
        k, _ = oracle_sample(lg, args.ref_budget / args.steps)
    sub = lg.subset(np.arange(k))
    warm = lg.subset(np.arange(k_cal))
    b = int(lg.size[:k].sum())
    for _ in range(args.warmup):
        oracle.dedup(warm)
    ts = []
    for _ in range(args.steps):
        t = time.perf_counter()
        oracle.dedup(sub)
        ts.append(time.perf_counter() - t)
    sec = sum(ts) / len(ts)
    v = round(b / sec / 1e9, 3)
    sample = (f"the whole log ({lg.n} records, {b / 1e9:.2f} GB) per step" if k == lg.n else
              f"gid prefix of {k} of {lg.n} records ({b / 1e9:.2f} GB) per step") + \
        f"; warm-up steps on a {k_cal}-record prefix; 1 of {os.cpu_count()} host cores"
    out = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": world,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(sec * 1e3, 3),
           "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u8",
           "data": "synthetic",
           "config": {"workload": WORKLOADS[args.workload], "records": lg.n, "payload_bytes": lg.total_bytes,
                      "n_sites": lg.n_sites, "n_scale": args.n_scale, "size_scale": args.size_scale,
                      "whole_log_per_step": k == lg.n},
           "cpu_baseline": {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample},
           "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


def spawn_ranks(args):
    """--gpus N without a torchrun environment: launch N ranks of this script (one per
    GPU) under torch.distributed.run and return its exit code."""
    import socket
    import torch
    if not args.same_device and torch.cuda.device_count() < args.gpus:
        log_msg(f"[bench] --gpus {args.gpus} but {torch.cuda.device_count()} GPUs are visible "
                "(--same-device runs the ranks on one GPU over the host transport)")
        return 2
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    log_msg("[bench] " + " ".join(cmd))
    return subprocess.run(cmd).returncode


def main():
    import faulthandler
    faulthandler.enable()          # a native crash prints a stack instead of dying silently
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--workload", type=int, default=5, choices=[1, 2, 3, 4, 5])
    ap.add_argument("--n-scale", type=float, default=1.0)
    ap.add_argument("--size-scale", type=float, default=1.0)
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--e2e-pageable", type=int, default=1, help="also measure e2e from pageable host memory")
    ap.add_argument("--cpu-seconds", type=float, default=30.0)
    ap.add_argument("--ref-budget", type=float, default=400.0,
                    help="reference arm: seconds of timed oracle steps; the whole log per step if it fits")
    ap.add_argument("--same-device", action="store_true",
                    help="test hook: run the N ranks on one GPU (host exchange transport instead of NCCL)")
    ap.add_argument("--check", action="store_true", help="check the result against the CPU oracle (small logs)")
    ap.add_argument("--collective", action="store_true",
                    help="--gpus 1: run the collective (sharded) path over the library's NCCL in a world of one")
    ap.add_argument("--lib", default=None, help="load another build of libffm.so (tools/build_variants.sh)")
    ap.add_argument("--online", default=None,
                    help="comma-separated window sizes: measure online mode (ffm_online_step) instead")
    ap.add_argument("--online-max-windows", type=int, default=3000,
                    help="online: at most this many windows per size (small windows: latency over a prefix)")
    ap.add_argument("--digest-bits", type=int, default=64,
                    help="< 64 truncates the group-by digest (forced collisions, verify stress; config 3)")
    ap.add_argument("--two-pass", action="store_true",
                    help="round 0 as hash-all then verify (better for near-duplicate-heavy logs, config 3)")
    ap.add_argument("--prefilter", action="store_true",
                    help="S8(f) #4 size/prefix pre-filter (opt-in; single GPU); roofline counts bytes required")
    args = ap.parse_args()
    if args.warmup < 3:
        log_msg("[bench] warmup raised to 3 (timing rules)")
        args.warmup = 3
    if args.lib:
        import paper_conf_sc_weltonm19_b200 as ffm
        ffm.set_library_path(args.lib)
    if args.impl == "reference":
        run_reference(args)
    elif args.online:
        run_online(args)
    elif args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(spawn_ranks(args))
    else:
        if int(os.environ.get("WORLD_SIZE", 1)) != args.gpus:
            raise SystemExit(f"bench: --gpus {args.gpus} but WORLD_SIZE={os.environ.get('WORLD_SIZE')}")
        run_ours(args)


if __name__ == "__main__":
    main()
