"""paper_conf_sc_weltonm19_b200 -- B200-native duplicate memory-transfer detection.

Thin ctypes binding over ``libffm.so`` (include/ffm.h).  Argument marshalling
only: every step of the hot path runs in the library's sm_100a kernels.  There
is no CPU fallback -- if the CUDA library is missing or no device is present,
the calls raise.

Raw functions keep the C names (``ffm_log_create``, ``ffm_log_append``,
``ffm_log_append_batch``, ``ffm_dedup_run``, ...); ``FfmLog`` is a small
convenience wrapper used by the tests and bench.py.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from ._build import LIB as _LIB_DEFAULT

_LIB_PATH = _LIB_DEFAULT


def set_library_path(path: str) -> None:
    """Load another build of the same sources (a tuning variant from
    tools/build_variants.sh) instead of the in-tree libffm.so; call before the first
    use of the library."""
    global _LIB_PATH
    if _lib is not None:
        raise RuntimeError("libffm.so is already loaded")
    _LIB_PATH = path

FFM_OK, FFM_E_INVAL, FFM_E_RANGE, FFM_E_NOMEM, FFM_E_CUDA, FFM_E_COMM, FFM_E_STATE, FFM_E_NODEV = \
    0, -1, -2, -3, -4, -5, -6, -7
FFM_PAYLOAD_AUTO, FFM_PAYLOAD_HOST, FFM_PAYLOAD_DEVICE, FFM_PAYLOAD_HOST_PINNED = 0, 1, 2, 3
FFM_FLAG_TIMING = 1
FFM_FLAG_PREFILTER = 2
FFM_FLAG_TWO_PASS = 4
FFM_FLAG_FUSED = 8
FFM_FLAG_NO_GRAPH = 16
FFM_FLAG_ONLINE = 32
FFM_FLAG_APPEND_HASH = 64

# every symbol include/ffm.h declares (checked by tests/test_abi.py)
EXPORTS = ["ffm_config_init", "ffm_log_create", "ffm_log_append", "ffm_log_append_batch", "ffm_log_append_batch_ex",
           "ffm_dedup_run", "ffm_log_count", "ffm_log_payload_bytes", "ffm_log_stream",
           "ffm_last_run_stats", "ffm_debug_digests", "ffm_log_destroy", "ffm_strerror",
           "ffm_last_error", "ffm_version", "ffm_shard_plan", "ffm_nccl_unique_id",
           "ffm_site_duplicate_counts", "ffm_fold_sites",
           "ffm_online_step", "ffm_online_done", "ffm_log_reset", "ffm_log_set_flags"]
FFM_SHARD_SITE_LPT, FFM_SHARD_CONTIGUOUS = 0, 1

# ffm_comm_ops callbacks (host buffers)
ALLGATHER_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64)
ALLREDUCE_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64)


class FfmCommOps(ctypes.Structure):
    _fields_ = [("ctx", ctypes.c_void_p), ("allgather", ALLGATHER_FN), ("allreduce_u64", ALLREDUCE_FN)]


class FfmConfig(ctypes.Structure):
    _fields_ = [("n_sites", ctypes.c_uint32), ("device", ctypes.c_int32), ("rank", ctypes.c_int32),
                ("world", ctypes.c_int32), ("arena_bytes", ctypes.c_uint64),
                ("max_records", ctypes.c_uint64), ("digest_bits", ctypes.c_uint32),
                ("refine_bits", ctypes.c_uint32), ("chunk_bytes", ctypes.c_uint32),
                ("small_bytes", ctypes.c_uint32), ("flags", ctypes.c_uint32),
                ("reserved0", ctypes.c_uint32), ("stream", ctypes.c_void_p),
                ("nccl_id", ctypes.c_void_p), ("comm", ctypes.POINTER(FfmCommOps))]


class FfmRunStats(ctypes.Structure):
    _fields_ = [(k, ctypes.c_double) for k in ("ms_total", "ms_hash", "ms_group", "ms_verify", "ms_resolve",
                                                 "ms_label", "ms_output", "ms_hash_large", "ms_hash_small")] + \
               [(k, ctypes.c_uint64) for k in ("n_records", "payload_bytes", "n_members", "n_residual",
                                                "resolve_rounds", "kernel_launches", "hash_items",
                                                "verify_items", "prefilter_rest_bytes")] + \
               [("ms_fused", ctypes.c_double), ("two_pass", ctypes.c_uint64), ("n_reread", ctypes.c_uint64)] + \
               [(k, ctypes.c_uint64) for k in ("n_reps_local", "n_reps_global", "exchange_bytes",
                                                "remote_verify_bytes", "n_slow", "host_syncs")] + \
               [("ms_exchange", ctypes.c_double)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class FfmError(RuntimeError):
    def __init__(self, code, msg=""):
        super().__init__(f"{ffm_strerror(code)} ({code}){': ' + msg if msg else ''}")
        self.code = code


_lib = None


def lib() -> ctypes.CDLL:
    """Load libffm.so (in-tree).  Raises if it is missing: there is no fallback."""
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise ImportError(f"{_LIB_PATH} is missing: run __graft_entry__.build() "
                              "(the CUDA library is the only implementation)")
        L = ctypes.CDLL(_LIB_PATH)
        vp, u64, u32, i32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
        L.ffm_config_init.argtypes = [ctypes.POINTER(FfmConfig)]
        L.ffm_config_init.restype = None
        L.ffm_log_create.argtypes = [ctypes.POINTER(FfmConfig), ctypes.POINTER(vp)]
        L.ffm_log_create.restype = i32
        L.ffm_log_append.argtypes = [vp, u32, u64, vp, u64]
        L.ffm_log_append.restype = i32
        L.ffm_log_append_batch.argtypes = [vp, u64, vp, vp, vp, vp, vp, i32]
        L.ffm_log_append_batch.restype = i32
        L.ffm_log_append_batch_ex.argtypes = [vp, u64, vp, vp, vp, vp, vp, vp, i32]
        L.ffm_log_append_batch_ex.restype = i32
        L.ffm_dedup_run.argtypes = [vp, vp, vp]
        L.ffm_dedup_run.restype = i32
        L.ffm_log_count.argtypes = [vp]
        L.ffm_log_count.restype = u64
        L.ffm_log_payload_bytes.argtypes = [vp]
        L.ffm_log_payload_bytes.restype = u64
        L.ffm_log_stream.argtypes = [vp]
        L.ffm_log_stream.restype = vp
        L.ffm_last_run_stats.argtypes = [vp, ctypes.POINTER(FfmRunStats)]
        L.ffm_last_run_stats.restype = i32
        L.ffm_debug_digests.argtypes = [vp, vp]
        L.ffm_debug_digests.restype = i32
        L.ffm_log_set_flags.argtypes = [vp, u32]
        L.ffm_log_set_flags.restype = i32
        L.ffm_log_reset.argtypes = [vp]
        L.ffm_log_reset.restype = i32
        L.ffm_log_destroy.argtypes = [vp]
        L.ffm_log_destroy.restype = i32
        L.ffm_strerror.argtypes = [i32]
        L.ffm_strerror.restype = ctypes.c_char_p
        L.ffm_last_error.argtypes = [vp]
        L.ffm_last_error.restype = ctypes.c_char_p
        L.ffm_version.argtypes = []
        L.ffm_version.restype = ctypes.c_char_p
        L.ffm_shard_plan.argtypes = [u64, vp, vp, u32, ctypes.c_int32, i32, vp]
        L.ffm_shard_plan.restype = i32
        L.ffm_nccl_unique_id.argtypes = [vp]
        L.ffm_nccl_unique_id.restype = i32
        L.ffm_site_duplicate_counts.argtypes = [vp, vp]
        L.ffm_site_duplicate_counts.restype = i32
        L.ffm_fold_sites.argtypes = [vp, vp, vp, u32, vp]
        L.ffm_fold_sites.restype = i32
        L.ffm_online_step.argtypes = [vp, vp, vp, ctypes.POINTER(u64)]
        L.ffm_online_step.restype = i32
        L.ffm_online_done.argtypes = [vp]
        L.ffm_online_done.restype = u64
        _lib = L
    return _lib


# ---- raw C-named wrappers (argument marshalling only) -----------------------
def ffm_config_init() -> FfmConfig:
    c = FfmConfig()
    lib().ffm_config_init(ctypes.byref(c))
    return c


def ffm_strerror(code: int) -> str:
    return lib().ffm_strerror(code).decode()


def ffm_version() -> str:
    return lib().ffm_version().decode()


def ffm_log_create(cfg: FfmConfig) -> int:
    h = ctypes.c_void_p()
    rc = lib().ffm_log_create(ctypes.byref(cfg), ctypes.byref(h))
    if rc != FFM_OK:
        raise FfmError(rc)
    return h.value


def ffm_last_error(h) -> str:
    return lib().ffm_last_error(h).decode()


def _check(h, rc):
    if rc != FFM_OK:
        raise FfmError(rc, ffm_last_error(h) if h else "")


def ffm_log_append(h, call_site: int, size: int, payload_ptr: int, duration_ns: int):
    _check(h, lib().ffm_log_append(h, call_site, size, payload_ptr, duration_ns))


def _addr(a):
    """Address of a numpy array or torch tensor (host or device)."""
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return a.ctypes.data
    if hasattr(a, "data_ptr"):
        return a.data_ptr()
    return int(a)


def ffm_log_append_batch(h, call_sites, sizes, payload_ptrs, durations_ns, gids=None,
                         payload_kind: int = FFM_PAYLOAD_AUTO):
    ffm_log_append_batch_ex(h, call_sites, sizes, payload_ptrs, durations_ns, gids, None, payload_kind)


def ffm_log_append_batch_ex(h, call_sites, sizes, payload_ptrs, durations_ns, gids=None, channels=None,
                            payload_kind: int = FFM_PAYLOAD_AUTO):
    sites = np.ascontiguousarray(call_sites, dtype=np.uint32)
    sz = np.ascontiguousarray(sizes, dtype=np.uint64)
    pp = np.ascontiguousarray(payload_ptrs, dtype=np.uint64)
    du = np.ascontiguousarray(durations_ns, dtype=np.uint64)
    g = None if gids is None else np.ascontiguousarray(gids, dtype=np.uint64)
    ch = None if channels is None else np.ascontiguousarray(channels, dtype=np.uint64)
    n = len(sites)
    if not (len(sz) == len(pp) == len(du) == n) or (g is not None and len(g) != n) or \
            (ch is not None and len(ch) != n):
        raise ValueError("array lengths differ")
    _check(h, lib().ffm_log_append_batch_ex(h, n, _addr(sites), _addr(sz), _addr(pp), _addr(du),
                                            _addr(g), _addr(ch), payload_kind))


def ffm_dedup_run(h, duplicate_of, benefit_ns):
    """duplicate_of / benefit_ns: numpy arrays (host) or torch CUDA tensors (device)."""
    _check(h, lib().ffm_dedup_run(h, _addr(duplicate_of), _addr(benefit_ns)))


def ffm_log_count(h) -> int:
    return int(lib().ffm_log_count(h))


def ffm_log_payload_bytes(h) -> int:
    return int(lib().ffm_log_payload_bytes(h))


def ffm_log_stream(h) -> int:
    return lib().ffm_log_stream(h) or 0


def ffm_last_run_stats(h) -> dict:
    s = FfmRunStats()
    _check(h, lib().ffm_last_run_stats(h, ctypes.byref(s)))
    return s.as_dict()


def ffm_debug_digests(h) -> np.ndarray:
    out = np.empty(max(1, ffm_log_count(h)), np.uint64)
    _check(h, lib().ffm_debug_digests(h, _addr(out)))
    return out[:ffm_log_count(h)]


def ffm_log_set_flags(h, flags: int):
    _check(h, lib().ffm_log_set_flags(h, flags))


def ffm_log_reset(h):
    _check(h, lib().ffm_log_reset(h))


def ffm_log_destroy(h):
    _check(None, lib().ffm_log_destroy(h))


def ffm_shard_plan(call_sites, sizes, n_sites: int, world: int, policy: int = FFM_SHARD_SITE_LPT) -> np.ndarray:
    """Host-only: rank of each record (site-affinity LPT or contiguous byte-balanced ranges)."""
    sites = np.ascontiguousarray(call_sites, dtype=np.uint32)
    sz = np.ascontiguousarray(sizes, dtype=np.uint64)
    out = np.empty(max(len(sites), 1), np.int32)
    rc = lib().ffm_shard_plan(len(sites), _addr(sites), _addr(sz), n_sites, world, policy, _addr(out))
    if rc != FFM_OK:
        raise FfmError(rc)
    return out[:len(sites)]


def ffm_nccl_unique_id() -> bytes:
    """128-byte ncclUniqueId for a new sharded world (call on one rank, broadcast it)."""
    buf = ctypes.create_string_buffer(128)
    rc = lib().ffm_nccl_unique_id(buf)
    if rc != FFM_OK:
        raise FfmError(rc, "libnccl.so.2 unavailable")
    return buf.raw


def ffm_site_duplicate_counts(h, n_sites: int, out=None):
    if out is None:
        out = np.empty(n_sites, np.uint64)
    _check(h, lib().ffm_site_duplicate_counts(h, _addr(out)))
    return out


def ffm_fold_sites(h, site_values, site_to_group, n_groups: int, out=None):
    sv = site_values if not isinstance(site_values, np.ndarray) else np.ascontiguousarray(site_values, np.uint64)
    mp = site_to_group if not isinstance(site_to_group, np.ndarray) else \
        np.ascontiguousarray(site_to_group, np.uint32)
    if out is None:
        out = np.empty(n_groups, np.uint64)
    _check(h, lib().ffm_fold_sites(h, _addr(sv), _addr(mp), n_groups, _addr(out)))
    return out


def ffm_online_step(h, duplicate_of, benefit_ns=None) -> int:
    """Label the records appended since the previous step; returns how many."""
    n = ctypes.c_uint64()
    _check(h, lib().ffm_online_step(h, _addr(duplicate_of), _addr(benefit_ns), ctypes.byref(n)))
    return int(n.value)


def ffm_online_done(h) -> int:
    return int(lib().ffm_online_done(h))


# ---- convenience wrapper ----------------------------------------------------
class FfmLog:
    """Owns one ffm_log handle."""

    def __init__(self, n_sites: int, device: int = 0, *, arena_bytes: int = 0, max_records: int = 0,
                 digest_bits: int = 64, refine_bits: int = 64, chunk_bytes: int = 0, small_bytes: int = 0,
                 timing: bool = False, stream: int = 0, rank: int = 0, world: int = 1,
                 prefilter: bool = False, two_pass: bool = False, fused: bool = False,
                 graph: bool = True, online: bool = False, append_hash: bool = False,
                 nccl_id: bytes | None = None,
                 comm: FfmCommOps | None = None):
        """world > 1 (collective): pass the world's nccl_id (ffm_nccl_unique_id) or a comm
        transport (FfmCommOps, e.g. sharded.HostComm)."""
        self.h = None
        cfg = ffm_config_init()
        cfg.n_sites, cfg.device, cfg.rank, cfg.world = n_sites, device, rank, world
        cfg.arena_bytes, cfg.max_records = arena_bytes, max_records
        cfg.digest_bits, cfg.refine_bits = digest_bits, refine_bits
        cfg.chunk_bytes, cfg.small_bytes = chunk_bytes, small_bytes
        cfg.flags = (FFM_FLAG_TIMING if timing else 0) | (FFM_FLAG_PREFILTER if prefilter else 0) | \
            (FFM_FLAG_TWO_PASS if two_pass else 0) | (FFM_FLAG_FUSED if fused else 0) | \
            (0 if graph else FFM_FLAG_NO_GRAPH) | (FFM_FLAG_ONLINE if online else 0) | \
            (FFM_FLAG_APPEND_HASH if append_hash else 0)
        cfg.stream = stream or None
        self._keep = (nccl_id, comm)     # alive while the library may use them
        if nccl_id is not None:
            self._id_buf = ctypes.create_string_buffer(bytes(nccl_id), 128)
            cfg.nccl_id = ctypes.cast(self._id_buf, ctypes.c_void_p)
        if comm is not None:
            cfg.comm = ctypes.pointer(comm)
        self.n_sites = n_sites
        self.rank, self.world = rank, world
        self.flags = cfg.flags
        self.h = ffm_log_create(cfg)

    def append(self, call_site, size, payload_ptr, duration_ns):
        ffm_log_append(self.h, call_site, size, payload_ptr, duration_ns)

    def append_batch(self, call_sites, sizes, payload_ptrs, durations_ns, gids=None,
                     payload_kind=FFM_PAYLOAD_AUTO, channels=None):
        ffm_log_append_batch_ex(self.h, call_sites, sizes, payload_ptrs, durations_ns, gids, channels,
                                payload_kind)

    def append_log(self, log, ptrs=None, payload_kind=FFM_PAYLOAD_HOST, gids=None, idx=None):
        """Append a log object with site/size/dur arrays and payload_ptrs() (host payloads by
        default, or the device addresses `ptrs`)."""
        p = log.payload_ptrs() if ptrs is None else ptrs
        ch = getattr(log, "channel", None)
        if idx is None:
            self.append_batch(log.site, log.size, p, log.dur, gids, payload_kind, ch)
        else:
            self.append_batch(log.site[idx], log.size[idx], np.asarray(p)[idx], log.dur[idx],
                              gids, payload_kind, None if ch is None else ch[idx])

    def run(self, duplicate_of=None, benefit_ns=None):
        n = self.count
        if duplicate_of is None:
            duplicate_of = np.empty(max(n, 1), np.int64)
        if benefit_ns is None:
            benefit_ns = np.empty(self.n_sites, np.uint64)
        ffm_dedup_run(self.h, duplicate_of, benefit_ns)
        return duplicate_of[:n] if isinstance(duplicate_of, np.ndarray) else duplicate_of, benefit_ns

    @property
    def count(self):
        return ffm_log_count(self.h)

    @property
    def payload_bytes(self):
        return ffm_log_payload_bytes(self.h)

    @property
    def stream(self):
        return ffm_log_stream(self.h)

    def stats(self):
        return ffm_last_run_stats(self.h)

    def digests(self):
        return ffm_debug_digests(self.h)

    def online_step(self, duplicate_of=None, benefit_ns=None):
        """Online mode: label the records appended since the last step."""
        pending = self.count - ffm_online_done(self.h)
        if duplicate_of is None:
            duplicate_of = np.empty(max(pending, 1), np.int64)
        if benefit_ns is None:
            benefit_ns = np.empty(self.n_sites, np.uint64)
        k = ffm_online_step(self.h, duplicate_of, benefit_ns)
        return (duplicate_of[:k] if isinstance(duplicate_of, np.ndarray) else duplicate_of), benefit_ns

    def site_counts(self, out=None):
        return ffm_site_duplicate_counts(self.h, self.n_sites, out)

    def fold(self, site_values, site_to_group, n_groups, out=None):
        return ffm_fold_sites(self.h, site_values, site_to_group, n_groups, out)

    def set_timing(self, on: bool):
        """Per-stage CUDA events on (direct launches) or off (graph replay)."""
        self.flags = (self.flags | FFM_FLAG_TIMING) if on else (self.flags & ~FFM_FLAG_TIMING)
        ffm_log_set_flags(self.h, self.flags)

    def reset(self):
        """Empty the log, keep its HBM allocations (ffm_log_reset)."""
        ffm_log_reset(self.h)

    def close(self):
        if self.h:
            ffm_log_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()
