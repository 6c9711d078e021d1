"""loggen -- seeded synthetic transfer logs shaped like the paper's workloads.

Shared INPUT infrastructure: it feeds both the CPU
oracle (``oracle/``) and the CUDA path, and holds none of the deduplication
method's arithmetic -- no payload hashing, grouping or comparison.  A log is a
list of records (call_site, size, duration_ns, content id); a content is a
descriptor (kind, seed, size, base content, byte flips) that ``fill.c``
turns into bytes with a counter-based generator.

Planted ground truth: the planner gives two records the same content id iff it
made them byte-identical on purpose.  Distinct ids are distinct bytes by
construction (fresh random/smooth seeds are unique; zero contents are keyed
by size; a near-duplicate xors >= 1 byte of its base with a non-zero value and
(base, flips) keys are de-duplicated).  ``planted_duplicate_of`` is derived
from the ids alone -- an independent check on the oracle (tests/test_oracle_pins.py).

Workload shapes (BASELINE.json configs 1-5):
  cumf_als re-sends the same data every loop iteration (PAPER.md P:1194-1197,
  P:1222-1226); cuIBM issues > 75 M small CUDA calls.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field

import numpy as np

KIND_RANDOM, KIND_ZERO, KIND_SMOOTH = 0, 1, 2
KiB, MiB = 1 << 10, 1 << 20
_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "libloggen.so")
_lib = None


def build(verbose: bool = False) -> str:
    """Compile fill.c -> libloggen.so (gcc, OpenMP)."""
    src = os.path.join(_HERE, "fill.c")
    if not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(src):
        cmd = f"gcc -O3 -march=x86-64-v3 -fopenmp -shared -fPIC -o {_LIB} {src}"
        if verbose:
            print(cmd)
        if os.system(cmd) != 0:
            raise RuntimeError("building libloggen.so failed")
    return _LIB


def _get_lib():
    global _lib
    if _lib is None:
        build()
        _lib = ctypes.CDLL(_LIB)
        _lib.loggen_materialize.restype = ctypes.c_int
    return _lib


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


@dataclass
class Log:
    """A planned transfer log.  Records are in gid (program) order."""
    n_sites: int
    site: np.ndarray            # uint32 [N]
    size: np.ndarray            # uint64 [N]
    dur: np.ndarray             # uint64 [N]   duration_ns of the transfer call
    content: np.ndarray         # int64  [N]   content id
    c_kind: np.ndarray          # int32  [M]
    c_seed: np.ndarray          # uint64 [M]
    c_size: np.ndarray          # uint64 [M]
    c_base: np.ndarray          # int64  [M]   -1 or base content id (< own id)
    c_flip_start: np.ndarray    # int64  [M+1]
    flip_pos: np.ndarray        # uint64 [F]
    flip_xor: np.ndarray        # uint8  [F]
    name: str = ""
    buf: np.ndarray | None = field(default=None, repr=False)   # materialised bytes
    channel: np.ndarray | None = None   # uint64 [N] direction/destination id (S8(f) #3), or None
    c_off: np.ndarray | None = field(default=None, repr=False)

    @property
    def n(self) -> int:
        return int(self.site.shape[0])

    @property
    def total_bytes(self) -> int:
        return int(self.size.sum())

    @property
    def distinct_bytes(self) -> int:
        return int(self.c_size.sum())

    # ---- materialisation -------------------------------------------------
    def needed_contents(self, records: np.ndarray) -> np.ndarray:
        """Content ids used by `records`, closed under derivation bases."""
        need = np.zeros(len(self.c_size), bool)
        need[np.unique(self.content[records])] = True
        for c in range(len(self.c_base) - 1, -1, -1):       # bases have smaller ids
            if need[c] and self.c_base[c] >= 0:
                need[self.c_base[c]] = True
        return need

    def materialize(self, nthreads: int = 0, buf: np.ndarray | None = None,
                    records: np.ndarray | None = None) -> np.ndarray:
        """Fill the contents into one host buffer (16-B aligned slots).  With
        `records`, only the contents those records use (one shard's share)."""
        if self.buf is not None:
            return self.buf
        sz = self.c_size.astype(np.uint64)
        if records is not None:
            sz = np.where(self.needed_contents(records), sz, np.uint64(0)).astype(np.uint64)
        slot = (sz + np.uint64(15)) // np.uint64(16) * np.uint64(16)
        off = np.zeros(len(sz), dtype=np.uint64)
        if len(sz) > 1:
            off[1:] = np.cumsum(slot[:-1], dtype=np.uint64)
        total = int(slot.sum()) if len(sz) else 0
        if buf is None:
            buf = np.zeros(max(total, 16), dtype=np.uint8)   # calloc: padding deterministic
        elif buf.nbytes < total:
            raise ValueError("buffer too small")
        lib = _get_lib()
        rc = lib.loggen_materialize(
            ctypes.c_int64(len(sz)), _ptr(self.c_kind), _ptr(self.c_seed), _ptr(sz),
            _ptr(self.c_base), _ptr(self.c_flip_start), _ptr(self.flip_pos),
            _ptr(self.flip_xor), _ptr(off), _ptr(buf), ctypes.c_int(nthreads))
        if rc != 0:
            raise RuntimeError("loggen_materialize: inconsistent content table")
        self.buf, self.c_off = buf, off
        return buf

    def payload_ptrs(self) -> np.ndarray:
        """Host address of each record's payload (records share content buffers)."""
        self.materialize()
        base = np.uint64(self.buf.ctypes.data)
        return (self.c_off[self.content] + base).astype(np.uint64)

    def payload(self, i: int) -> bytes:
        self.materialize()
        c = int(self.content[i])
        o = int(self.c_off[c])
        return self.buf[o:o + int(self.c_size[c])].tobytes()

    def content_bytes(self, c: int) -> np.ndarray:
        self.materialize()
        o = int(self.c_off[c])
        return self.buf[o:o + int(self.c_size[c])]

    # ---- planted ground truth ---------------------------------------------
    def planted_duplicate_of(self) -> np.ndarray:
        """dup_of from content ids (and channels, if any) alone: first earlier record
        with the same id."""
        first: dict = {}
        out = np.full(self.n, -1, dtype=np.int64)
        keys = self.content.tolist() if self.channel is None else \
            list(zip(self.content.tolist(), self.channel.tolist()))
        for i, c in enumerate(keys):
            j = first.get(c)
            if j is None:
                first[c] = i
            else:
                out[i] = j
        return out

    def planted_benefit(self) -> np.ndarray:
        d = self.planted_duplicate_of()
        b = np.zeros(self.n_sites, dtype=np.uint64)
        m = d >= 0
        np.add.at(b, self.site[m].astype(np.int64), self.dur[m])
        return b

    def subset(self, idx: np.ndarray, name: str | None = None) -> "Log":
        """Records idx (in the given order) with the same content table."""
        lg = Log(self.n_sites, self.site[idx], self.size[idx], self.dur[idx], self.content[idx],
                 self.c_kind, self.c_seed, self.c_size, self.c_base, self.c_flip_start,
                 self.flip_pos, self.flip_xor, name or self.name + "/subset")
        lg.buf, lg.c_off = self.buf, self.c_off
        lg.channel = None if self.channel is None else self.channel[idx]
        return lg


class _Planner:
    """Accumulates contents and records; guarantees distinct ids => distinct bytes."""

    def __init__(self, seed: int, n_sites: int):
        self.rng = np.random.default_rng(seed)
        self.seed_ctr = (seed * 0x9E3779B97F4A7C15) & 0xFFFFFFFFFFFFFFFF
        self.n_sites = n_sites
        self.kind: list[int] = []
        self.cseed: list[int] = []
        self.csize: list[int] = []
        self.base: list[int] = []
        self.flips: list[list[tuple[int, int]]] = []
        self.zero_by_size: dict[int, int] = {}
        self.derived: dict[tuple, int] = {}
        self.r_site: list[int] = []
        self.r_content: list[int] = []
        lat = self.rng.integers(4000, 12001, size=n_sites)   # per-site launch latency, ns
        self.site_lat = lat.astype(np.int64)

    def _next_seed(self) -> int:
        self.seed_ctr = (self.seed_ctr + 0x9E3779B97F4A7C15) & 0xFFFFFFFFFFFFFFFF
        return self.seed_ctr

    def fresh(self, size: int, kind: int | None = None) -> int:
        if kind is None:
            u = self.rng.random()
            kind = KIND_RANDOM if u < 0.85 else (KIND_SMOOTH if u < 0.97 else KIND_ZERO)
        if kind == KIND_SMOOTH and size < 8:
            kind = KIND_RANDOM
        if kind == KIND_ZERO:
            return self.zero(size)
        self.kind.append(kind)
        self.cseed.append(self._next_seed())
        self.csize.append(size)
        self.base.append(-1)
        self.flips.append([])
        return len(self.kind) - 1

    def zero(self, size: int) -> int:
        c = self.zero_by_size.get(size)
        if c is None:
            self.kind.append(KIND_ZERO)
            self.cseed.append(0)
            self.csize.append(size)
            self.base.append(-1)
            self.flips.append([])
            c = len(self.kind) - 1
            self.zero_by_size[size] = c
        return c

    def derive(self, base: int, flips: list[tuple[int, int]]) -> int:
        """base content with bytes xored; flips: distinct positions, non-zero xor."""
        pos = [p for p, _ in flips]
        assert len(set(pos)) == len(pos) and all(x != 0 for _, x in flips)
        key = (base, tuple(sorted(flips)))
        c = self.derived.get(key)
        if c is None:
            # the kind of a derived content is its base's (materialised from base)
            self.kind.append(self.kind[base])
            self.cseed.append(0)
            self.csize.append(self.csize[base])
            self.base.append(base)
            self.flips.append(sorted(flips))
            c = len(self.kind) - 1
            self.derived[key] = c
        return c

    def record(self, site: int, content: int):
        self.r_site.append(site)
        self.r_content.append(content)

    def finish(self, name: str) -> Log:
        rng = self.rng
        content = np.asarray(self.r_content, dtype=np.int64)
        csize = np.asarray(self.csize, dtype=np.uint64)
        site = np.asarray(self.r_site, dtype=np.uint32)
        size = csize[content] if len(content) else np.zeros(0, np.uint64)
        # dur = site latency + size at 12 GB/s (12 B/ns) + jitter U[0, 10%]
        base = self.site_lat[site.astype(np.int64)] + (size // np.uint64(12)).astype(np.int64)
        jit = np.floor(rng.random(len(site)) * 0.1 * base).astype(np.int64)
        dur = (base + jit).astype(np.uint64)
        fs = np.zeros(len(self.flips) + 1, dtype=np.int64)
        fs[1:] = np.cumsum([len(f) for f in self.flips])
        fpos = np.asarray([p for f in self.flips for p, _ in f], dtype=np.uint64)
        fx = np.asarray([x for f in self.flips for _, x in f], dtype=np.uint8)
        return Log(self.n_sites, site, size.astype(np.uint64), dur, content,
                   np.asarray(self.kind, dtype=np.int32), np.asarray(self.cseed, dtype=np.uint64),
                   csize, np.asarray(self.base, dtype=np.int64), fs, fpos, fx, name)


def _loguniform(rng, lo: float, hi: float, n=None):
    return np.exp(rng.uniform(np.log(lo), np.log(hi), size=n))


def _shape_size(rng, raw: float, lo: int) -> int:
    """90% of sizes are multiples of 8, 10% arbitrary (tail handling)."""
    s = max(int(raw), lo)
    if rng.random() < 0.9:
        s = max(8, s - s % 8)
    return s


def _zipf_choice(rng, n: int, s: float, size: int) -> np.ndarray:
    p = 1.0 / np.arange(1, n + 1, dtype=np.float64) ** s
    p /= p.sum()
    return rng.choice(n, size=size, p=p)


def config1(seed: int | None = None, n_scale: float = 1.0, size_scale: float = 1.0) -> Log:
    """1,000 transfers of 4 KB-1 MB, 30% planted exact duplicates, 50 sites (BJ configs[0])."""
    seed = 0x5C19D10000 + 1 if seed is None else seed
    N = max(4, int(round(1000 * n_scale)))
    P = _Planner(seed, 50)
    rng = P.rng
    zs = _zipf_choice(rng, 50, 1.1, N)
    lo, hi = max(16, int(4 * KiB * size_scale)), max(32, int(1 * MiB * size_scale))
    for i in range(N):
        if i > 0 and rng.random() < 0.3:
            src = int(rng.integers(0, i))
            site = P.r_site[src] if rng.random() < 0.7 else int(zs[i])
            P.record(site, P.r_content[src])
        else:
            sz = _shape_size(rng, _loguniform(rng, lo, hi), 1)
            P.record(int(zs[i]), P.fresh(sz))
    return P.finish("config1")


def config2(seed: int | None = None, n_scale: float = 1.0, size_scale: float = 1.0) -> Log:
    """1 M small transfers 256 B-4 KB, 60% re-uploads (cudaMemcpy-in-loop), 256 sites."""
    seed = 0x5C19D10000 + 2 if seed is None else seed
    N = max(4, int(round(1_000_000 * n_scale)))
    S = 256
    P = _Planner(seed, S)
    rng = P.rng
    lo, hi = max(8, int(256 * size_scale)), max(16, int(4 * KiB * size_scale))
    site_size = [_shape_size(rng, v, 1) for v in _loguniform(rng, lo, hi, S)]
    sites = _zipf_choice(rng, S, 1.0, N)
    u1, u2, u3 = rng.random(N), rng.random(N), rng.random(N)
    versions: list[list[int]] = [[] for _ in range(S)]
    for i in range(N):
        s = int(sites[i])
        v = versions[s]
        if v and u1[i] < 0.6:
            if len(v) > 1 and u2[i] < 0.05:
                c = v[int(u3[i] * (len(v) - 1))]      # revert to an older version
            else:
                c = v[-1]
        else:
            c = P.fresh(site_size[s])
            v.append(c)
        P.record(s, c)
    return P.finish("config2")


def config3(seed: int | None = None, n_scale: float = 1.0, size_scale: float = 1.0,
            chunk: int = 16 * KiB) -> Log:
    """10,000 x 1 MiB near-duplicates with single-byte differences (verify stress)."""
    seed = 0x5C19D10000 + 3 if seed is None else seed
    N = max(4, int(round(10_000 * n_scale)))
    size = max(64, int(MiB * size_scale))
    NB = 64
    P = _Planner(seed, NB)
    rng = P.rng
    bases = [P.fresh(size, KIND_RANDOM if b % 8 else KIND_SMOOTH) for b in range(NB)]
    special = [0, size - 1] + [p for c in range(1, size // chunk + 1)
                               for p in (c * chunk - 1, c * chunk) if p < size]
    near: list[tuple[int, int]] = []     # (site, content) of planted near-duplicates
    for i in range(N):
        b = int(rng.integers(0, NB))
        u = rng.random()
        if u < 0.25:
            P.record(b, bases[b])
        elif u < 0.75 or not near:
            pos = int(special[int(rng.integers(0, len(special)))]) if rng.random() < 0.1 \
                else int(rng.integers(0, size))
            x = 1 + int(rng.integers(0, 1 << 30)) % 255
            c = P.derive(bases[b], [(pos, x)])
            near.append((b, c))
            P.record(b, c)
        else:
            s, c = near[int(rng.integers(0, len(near)))]
            P.record(s, c)
    return P.finish("config3")


def config4(seed: int | None = None, n_scale: float = 1.0, size_scale: float = 1.0) -> Log:
    """1,000 large transfers 16-64 MB: 20 solver arrays x 50 iterations (~34 GiB)."""
    seed = 0x5C19D10000 + 4 if seed is None else seed
    iters = max(2, int(round(50 * n_scale)))
    A = 20
    P = _Planner(seed, A)
    rng = P.rng
    page = max(64, int(4 * KiB * size_scale))
    sizes = []
    for v in _loguniform(rng, 16 * MiB * size_scale, 64 * MiB * size_scale, A):
        s = max(page, int(v) // page * page)
        sizes.append(s)
    cur = [P.fresh(sizes[a], KIND_RANDOM if a % 3 else KIND_SMOOTH) for a in range(A)]
    first = list(cur)
    revert_cycle = 0
    for it in range(iters):
        if it > 0:
            for a in range(12, 16):                       # fully regenerated
                cur[a] = P.fresh(sizes[a], KIND_RANDOM)
            for a in range(16, 20):                       # 1% of pages rewritten
                npages = sizes[a] // page
                k = max(1, npages // 100)
                pages = rng.choice(npages, size=k, replace=False)
                flips = [(int(p) * page + int(rng.integers(0, page)), 1 + int(rng.integers(0, 255)))
                         for p in pages]
                cur[a] = P.derive(cur[a], flips)
            if it % 10 == 0:                              # a far-back duplicate
                a = 12 + revert_cycle % 8
                revert_cycle += 1
                cur[a] = first[a]
        for a in range(A):
            P.record(a, cur[a])
    return P.finish("config4")


def config5(seed: int | None = None, n_scale: float = 1.0, size_scale: float = 1.0,
            n_sites: int = 10_000) -> Log:
    """Mixed application-shaped log: ~64 GB, 2 M transfers, 10k call sites."""
    seed = 0x5C19D10000 + 5 if seed is None else seed
    N = max(16, int(round(2_000_000 * n_scale)))
    n_large = max(1, n_sites // 100)
    n_med = max(1, (n_sites * 9) // 100)
    n_small = max(1, n_sites - n_large - n_med)
    S = n_small + n_med + n_large
    P = _Planner(seed, S)
    rng = P.rng
    T = 12
    small_sz = [_shape_size(rng, v, 1) for v in
                _loguniform(rng, max(8, 256 * size_scale), max(16, 4 * KiB * size_scale), n_small)]
    med_sz = [_shape_size(rng, v, 1) for v in
              _loguniform(rng, max(16, 4 * KiB * size_scale), max(32, MiB * size_scale), n_med)]
    pg = max(64, int(4 * KiB * size_scale))
    large_sz = [max(pg, int(v) // pg * pg) for v in
                _loguniform(rng, 16 * MiB * size_scale, 64 * MiB * size_scale, n_large)]
    site_size = small_sz + med_sz + large_sz
    cur: list[int] = [-1] * S
    fresh_log: list[tuple[int, int]] = []               # (site, content) first sends
    n_sm = N - n_large * T
    per_it = [n_sm // T + (1 if t < n_sm % T else 0) for t in range(T)]
    frac_small = 0.9506
    for t in range(T):
        m = per_it[t]
        is_small = rng.random(m) < frac_small
        ss = _zipf_choice(rng, n_small, 1.1, m)
        ms = _zipf_choice(rng, n_med, 1.1, m) + n_small
        sites = np.where(is_small, ss, ms)
        u_zero, u_dup, u_cross = rng.random(m), rng.random(m), rng.random(m)
        slots = sorted(rng.choice(m + n_large, size=n_large, replace=False).tolist())
        large_order = rng.permutation(n_large) + n_small + n_med
        j = 0
        li = 0
        for k in range(m + n_large):
            if li < n_large and k == slots[li]:
                s = int(large_order[li])
                li += 1
                if cur[s] >= 0 and rng.random() < 0.6:
                    c = cur[s]
                else:
                    c = P.fresh(site_size[s], KIND_RANDOM if rng.random() < 0.8 else KIND_SMOOTH)
                    cur[s] = c
                    fresh_log.append((s, c))
                P.record(s, c)
                continue
            s = int(sites[j])
            p_re = 0.6 if is_small[j] else 0.3
            if u_zero[j] < 0.03:
                c = P.zero(site_size[s])
            elif cur[s] >= 0 and u_dup[j] < p_re:
                if u_cross[j] < 0.05 and fresh_log:
                    # cross-site shared content: data first sent by another site
                    c = fresh_log[int(rng.integers(0, len(fresh_log)))][1]
                else:
                    c = cur[s]
            else:
                c = P.fresh(site_size[s])
                cur[s] = c
                fresh_log.append((s, c))
            P.record(s, c)
            j += 1
    return P.finish("config5")


CONFIGS = {1: config1, 2: config2, 3: config3, 4: config4, 5: config5}


def gen_config(k: int, seed: int | None = None, n_scale: float = 1.0, size_scale: float = 1.0) -> Log:
    return CONFIGS[k](seed=seed, n_scale=n_scale, size_scale=size_scale)


def from_payloads(payloads: list[bytes], sites=None, durs=None, n_sites: int | None = None,
                  channels=None) -> Log:
    """A log from explicit byte strings (tiny / adversarial tests).  Content ids
    are assigned by exact byte equality, so planted truth is exact."""
    n = len(payloads)
    ids: dict[bytes, int] = {}
    content = []
    for p in payloads:
        content.append(ids.setdefault(bytes(p), len(ids)))
    uniq = sorted(ids.items(), key=lambda kv: kv[1])
    sites = np.zeros(n, np.uint32) if sites is None else np.asarray(sites, np.uint32)
    durs = np.arange(1, n + 1, dtype=np.uint64) * 10 if durs is None else np.asarray(durs, np.uint64)
    ns = int(sites.max()) + 1 if (n_sites is None and n) else (n_sites or 1)
    m = len(uniq)
    csize = np.asarray([len(b) for b, _ in uniq], np.uint64)
    lg = Log(ns, sites, csize[np.asarray(content, np.int64)] if n else np.zeros(0, np.uint64),
             durs, np.asarray(content, np.int64),
             np.zeros(m, np.int32), np.zeros(m, np.uint64), csize, np.full(m, -1, np.int64),
             np.zeros(m + 1, np.int64), np.zeros(0, np.uint64), np.zeros(0, np.uint8), "explicit")
    slot = (csize + np.uint64(15)) // np.uint64(16) * np.uint64(16)
    off = np.zeros(m, np.uint64)
    if m > 1:
        off[1:] = np.cumsum(slot[:-1], dtype=np.uint64)
    buf = np.zeros(max(16, int(slot.sum()) if m else 16), np.uint8)
    for (b, c) in uniq:
        o = int(off[c])
        buf[o:o + len(b)] = np.frombuffer(b, np.uint8) if len(b) else buf[o:o]
    lg.buf, lg.c_off = buf, off
    lg.channel = None if channels is None else np.asarray(channels, np.uint64)
    return lg
