"""Test-only scalar reference of the GPU digest as specified in DESIGN.md "Digest".

This pins an IMPLEMENTATION DETAIL (T6 in SURVEY.md 4.2): the digest is never
part of the result, but cross-rank consistency and the chunk-size invariance
rely on it being exactly this function of (bytes, size).  It is not the oracle
and the oracle does not use it.
"""
import numpy as np

M32 = 0xFFFFFFFF
M64 = (1 << 64) - 1


def _sm64(x):
    x = (x + 0x9E3779B97F4A7C15) & M64
    x = ((x ^ (x >> 30)) * 0xBF58476D1CE4E5B9) & M64
    x = ((x ^ (x >> 27)) * 0x94D049BB133111EB) & M64
    return x ^ (x >> 31)


def _keys():
    s = 0xD10E5E5FF1
    ka = np.zeros((16, 6), np.uint64)
    for g in range(16):
        for j in range(6):
            ka[g, j] = (_sm64(s) >> 16) & M32
            s += 1
    return ka


KA = _keys()
DA = np.array([0x9E3779B9, 0x7F4A7C15, 0xF39CC061, 0x5CEDC835, 0x1B873593, 0xCC9E2D51], np.uint64)


def fmix64(k):
    k ^= k >> 33
    k = (k * 0xff51afd7ed558ccd) & M64
    k ^= k >> 33
    k = (k * 0xc4ceb9fe1a85ec53) & M64
    k ^= k >> 33
    return k


def nh_sums(b: bytes):
    n = len(b)
    nw = (n + 15) // 16
    if nw == 0:
        return 0, 0
    buf = np.zeros(nw * 16, np.uint8)
    buf[:n] = np.frombuffer(b, np.uint8)
    w = buf.view("<u4").reshape(nw, 4).astype(np.uint64)
    q = np.arange(nw, dtype=np.uint64)
    g = (q % 16).astype(np.int64)
    s = q // np.uint64(16)
    k = [((KA[g, j] + s * DA[j]) & np.uint64(M32)) for j in range(6)]
    m = np.uint64(M32)
    with np.errstate(over="ignore"):
        a = ((w[:, 0] + k[0]) & m) * ((w[:, 1] + k[1]) & m) + ((w[:, 2] + k[2]) & m) * ((w[:, 3] + k[3]) & m)
        bb = ((w[:, 0] + k[2]) & m) * ((w[:, 1] + k[3]) & m) + ((w[:, 2] + k[4]) & m) * ((w[:, 3] + k[5]) & m)
        A = int(a.sum(dtype=np.uint64))
        B = int(bb.sum(dtype=np.uint64))
    return A, B


def digest(b: bytes) -> int:
    A, B = nh_sums(b)
    n = len(b)
    h = fmix64((B ^ ((n * 0x9E3779B97F4A7C15) & M64)) & M64)
    return fmix64(A ^ h)
