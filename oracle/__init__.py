"""oracle -- CPU oracle for duplicate memory-transfer detection.

TEST INFRASTRUCTURE ONLY: tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / ``--impl reference`` legs are the only callers.  The product
package never imports this module; the two share no code.

* ``dedup``      -- ffm_oracle.c:oracle_dedup, the paper's procedure
  (Sec. 3.3.2; Fig. 5), sequential
  hash map of prior transfers + memcmp, in program order.
* ``brute``      -- ffm_oracle.c:oracle_brute, the plain definition (all pairs).
* ``brute_py``   -- the plain definition in pure Python, for tiny logs.
* ``dup_of_one`` -- the plain definition for one record (sampled parity).

Parity pins: tests/test_oracle_pins.py (brute force, exhaustive enumeration,
planted ground truth, closed forms, golden fixtures under tests/golden/).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "libffm_oracle.so")
_lib = None


def build(verbose: bool = False) -> str:
    src = os.path.join(_HERE, "ffm_oracle.c")
    if not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(src):
        cmd = f"gcc -O2 -std=c11 -Wall -shared -fPIC -o {_LIB} {src}"
        if verbose:
            print(cmd)
        if os.system(cmd) != 0:
            raise RuntimeError("building libffm_oracle.so failed")
    return _LIB


def _get():
    global _lib
    if _lib is None:
        build()
        _lib = ctypes.CDLL(_LIB)
        vp = ctypes.c_void_p
        _lib.oracle_dedup.argtypes = [ctypes.c_uint64, vp, vp, vp, vp, vp, ctypes.c_uint32,
                                      ctypes.c_int, vp, vp]
        _lib.oracle_dedup.restype = ctypes.c_int
        _lib.oracle_brute.argtypes = [ctypes.c_uint64, vp, vp, vp, vp, vp, ctypes.c_uint32, vp, vp]
        _lib.oracle_brute.restype = ctypes.c_int
        _lib.oracle_dup_of_one.argtypes = [ctypes.c_uint64, vp, vp, vp]
        _lib.oracle_dup_of_one.restype = ctypes.c_int64
    return _lib


def _arrays(log):
    site = np.ascontiguousarray(log.site, dtype=np.uint32)
    size = np.ascontiguousarray(log.size, dtype=np.uint64)
    dur = np.ascontiguousarray(log.dur, dtype=np.uint64)
    ptrs = np.ascontiguousarray(log.payload_ptrs(), dtype=np.uint64)
    return site, size, dur, ptrs


def _chan(log):
    ch = getattr(log, "channel", None)
    return None if ch is None else np.ascontiguousarray(ch, dtype=np.uint64)


def _p(a):
    return None if a is None else ctypes.c_void_p(a.ctypes.data)


def dedup(log, hash_bits: int = 64):
    """Run the oracle on a loggen.Log.  Returns (duplicate_of int64[N], benefit uint64[n_sites])."""
    site, size, dur, ptrs = _arrays(log)
    n = len(site)
    dup = np.empty(max(n, 1), np.int64)
    ben = np.empty(max(log.n_sites, 1), np.uint64)
    rc = _get().oracle_dedup(n, _p(site), _p(size), _p(ptrs), _p(dur), _p(_chan(log)), log.n_sites,
                             hash_bits, _p(dup), _p(ben))
    if rc != 0:
        raise ValueError(f"oracle_dedup failed: {rc}")
    return dup[:n], ben[:log.n_sites]


def dedup_raw(n, site, size, ptrs, dur, n_sites, hash_bits=64, channel=None):
    dup = np.empty(max(n, 1), np.int64)
    ben = np.empty(max(n_sites, 1), np.uint64)
    rc = _get().oracle_dedup(n, _p(site), _p(size), _p(ptrs), _p(dur), _p(channel), n_sites, hash_bits,
                             _p(dup), _p(ben))
    if rc != 0:
        raise ValueError(f"oracle_dedup failed: {rc}")
    return dup[:n], ben[:n_sites]


def brute(log):
    site, size, dur, ptrs = _arrays(log)
    n = len(site)
    dup = np.empty(max(n, 1), np.int64)
    ben = np.empty(max(log.n_sites, 1), np.uint64)
    rc = _get().oracle_brute(n, _p(site), _p(size), _p(ptrs), _p(dur), _p(_chan(log)), log.n_sites,
                             _p(dup), _p(ben))
    if rc != 0:
        raise ValueError(f"oracle_brute failed: {rc}")
    return dup[:n], ben[:log.n_sites]


def dup_of_one(log, i: int) -> int:
    _, size, _, ptrs = _arrays(log) if not hasattr(log, "_oracle_cache") else log._oracle_cache
    log._oracle_cache = (None, size, None, ptrs)
    return int(_get().oracle_dup_of_one(i, _p(size), _p(ptrs), _p(_chan(log))))


def brute_py(payloads, sites, durs, n_sites, channels=None):
    """The plain definition in pure Python (tiny logs only)."""
    n = len(payloads)
    ch = channels if channels is not None else [0] * n
    dup = [-1] * n
    ben = [0] * n_sites
    for i in range(n):
        for j in range(i):
            if len(payloads[j]) == len(payloads[i]) and ch[j] == ch[i] and payloads[j] == payloads[i]:
                dup[i] = j
                break
        if dup[i] >= 0:
            ben[sites[i]] = (ben[sites[i]] + durs[i]) % (1 << 64)
    return dup, ben
