"""Pins for the CPU oracle (runs with -m "not gpu").

The oracle (oracle/ffm_oracle.c:oracle_dedup) is pinned to things other than
itself:
  * hand-derived golden fixtures (tests/golden/*.json, each citing PAPER.md);
  * the plain definition by brute force -- pure Python and C all-pairs --
    on random tiny logs and on EVERY log of length <= 6 over a small alphabet;
  * planted ground truth from the generator's content ids (an independent
    derivation) on all five BASELINE configs at reduced scale;
  * closed forms / special cases (all identical, alternating, all distinct);
  * invariants (points at a root, bytes equal, conservation of benefit);
  * flip tests and metamorphic invariance under a truncated / constant hash.
A plausible mistake in the oracle -- pointing at the latest instead of the
first transfer, comparing a prefix, ignoring size, crediting the original's
site, dropping a bucket on collision -- fails at least one of these.
"""
import itertools
import json
import os

import numpy as np
import pytest

import loggen
import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _run(payloads, sites=None, durs=None, n_sites=None, hash_bits=64):
    lg = loggen.from_payloads(payloads, sites, durs, n_sites)
    return oracle.dedup(lg, hash_bits=hash_bits)


@pytest.mark.parametrize("name", sorted(f for f in os.listdir(GOLDEN) if f.endswith(".json")))
@pytest.mark.parametrize("hash_bits", [64, 0])
def test_golden_fixture(name, hash_bits):
    fx = json.load(open(os.path.join(GOLDEN, name)))
    pay = [bytes.fromhex(r["hex"]) for r in fx["records"]]
    sites = [r["site"] for r in fx["records"]]
    durs = [r["dur"] for r in fx["records"]]
    chans = [r["channel"] for r in fx["records"]] if "channel" in fx["records"][0] else None
    lg = loggen.from_payloads(pay, sites, durs, fx["n_sites"], channels=chans)
    dup, ben = oracle.dedup(lg, hash_bits=hash_bits)
    assert dup.tolist() == fx["expect_duplicate_of"]
    assert ben.tolist() == fx["expect_benefit_ns"]
    if "expect_content_only" in fx:
        lg.channel = None
        dup, ben = oracle.dedup(lg, hash_bits=hash_bits)
        assert dup.tolist() == fx["expect_content_only"]["duplicate_of"]
        assert ben.tolist() == fx["expect_content_only"]["benefit_ns"]


@pytest.mark.parametrize("seed", range(40))
def test_channels_vs_python_brute(seed):
    """Destination-aware variant (S8(f) #3) against the plain definition."""
    rng = np.random.default_rng(5000 + seed)
    n = int(rng.integers(1, 150))
    pay, sites, durs, ns = _random_log(rng, n, int(rng.integers(1, 8)), int(rng.integers(0, 40)))
    chans = rng.integers(0, int(rng.integers(1, 4)), n).tolist()
    want = oracle.brute_py(pay, sites, durs, ns, chans)
    lg = loggen.from_payloads(pay, sites, durs, ns, channels=chans)
    for hb in (64, 0):
        d, b = oracle.dedup(lg, hash_bits=hb)
        assert d.tolist() == want[0] and b.tolist() == want[1]
    d, b = oracle.brute(lg)
    assert d.tolist() == want[0]
    # a single channel reduces to the content-only result
    lg1 = loggen.from_payloads(pay, sites, durs, ns, channels=[7] * n)
    assert oracle.dedup(lg1)[0].tolist() == oracle.brute_py(pay, sites, durs, ns)[0]


def _random_log(rng, n, alphabet_size, max_len):
    base = [rng.integers(0, 256, int(rng.integers(0, max_len + 1)), dtype=np.uint8).tobytes()
            for _ in range(alphabet_size)]
    pay = []
    for _ in range(n):
        u = rng.random()
        if u < 0.6 or not pay:
            b = base[int(rng.integers(0, alphabet_size))]
        elif u < 0.8 and len(b := base[int(rng.integers(0, alphabet_size))]) > 0:
            # single-byte flip of an alphabet entry
            arr = bytearray(b)
            p = int(rng.integers(0, len(arr)))
            arr[p] ^= 1 + int(rng.integers(0, 255))
            b = bytes(arr)
        else:
            b = b[: max(0, len(b) - 1)] if (b := base[int(rng.integers(0, alphabet_size))]) else b"\0"
        pay.append(b)
    n_sites = int(rng.integers(1, 6))
    sites = rng.integers(0, n_sites, n).tolist()
    durs = rng.integers(0, 1 << 40, n).tolist()
    return pay, sites, durs, n_sites


@pytest.mark.parametrize("seed", range(120))
def test_oracle_vs_python_brute(seed):
    rng = np.random.default_rng(1000 + seed)
    n = int(rng.integers(0, 120))
    pay, sites, durs, ns = _random_log(rng, n, int(rng.integers(1, 12)), int(rng.integers(0, 70)))
    want_dup, want_ben = oracle.brute_py(pay, sites, durs, ns)
    for hb in (64, 8, 0):
        dup, ben = _run(pay, sites, durs, ns, hb)
        assert dup.tolist() == want_dup
        assert ben.tolist() == want_ben


@pytest.mark.parametrize("seed", range(8))
def test_oracle_vs_c_brute_medium(seed):
    rng = np.random.default_rng(77 + seed)
    pay, sites, durs, ns = _random_log(rng, 2000, 40, 4096)
    lg = loggen.from_payloads(pay, sites, durs, ns)
    bd, bb = oracle.brute(lg)
    py_d, py_b = oracle.brute_py(pay[:300], sites[:300], durs[:300], ns)
    assert bd[:300].tolist() == py_d                    # the two brute forces agree
    for hb in (64, 0):
        d, b = oracle.dedup(lg, hash_bits=hb)
        np.testing.assert_array_equal(d, bd)
        np.testing.assert_array_equal(b, bb)


def test_exhaustive_small_logs():
    """Every log of length <= 5 over the alphabet (and a sample at length 6)."""
    alpha = [b"", b"a", b"b", b"ab", b"ba", b"\0" * 16]
    n_checked = 0
    rng = np.random.default_rng(5)
    for n in range(0, 7):
        combos = itertools.product(range(len(alpha)), repeat=n)
        if n == 6:
            combos = [tuple(rng.integers(0, len(alpha), 6)) for _ in range(3000)]
        for combo in combos:
            pay = [alpha[k] for k in combo]
            sites = [k % 2 for k in combo]
            durs = [3 + 7 * i for i in range(n)]
            want = oracle.brute_py(pay, sites, durs, 2)
            d, b = _run(pay, sites, durs, 2, 64 if n % 2 else 0)
            assert d.tolist() == want[0] and b.tolist() == want[1], combo
            n_checked += 1
    assert n_checked > 9000


@pytest.mark.parametrize("k,n_scale,size_scale", [
    (1, 1.0, 0.25), (2, 0.02, 1.0), (3, 0.05, 1 / 64), (4, 0.2, 1 / 256), (5, 0.005, 1 / 64)])
def test_planted_ground_truth(k, n_scale, size_scale):
    lg = loggen.gen_config(k, n_scale=n_scale, size_scale=size_scale)
    d, b = oracle.dedup(lg)
    np.testing.assert_array_equal(d, lg.planted_duplicate_of())
    np.testing.assert_array_equal(b, lg.planted_benefit())
    assert (d >= 0).any() and (d < 0).any()


def test_closed_forms():
    n = 50
    durs = [int(x) for x in np.random.default_rng(3).integers(1, 10**9, n)]
    sites = [i % 3 for i in range(n)]
    # all identical -> [-1, 0, 0, ...]; benefit = sum_{i>=1} dur by site
    d, b = _run([b"same-bytes"] * n, sites, durs, 3)
    assert d.tolist() == [-1] + [0] * (n - 1)
    want = [sum(durs[i] for i in range(1, n) if sites[i] == s) for s in range(3)]
    assert b.tolist() == want
    # alternating A, B -> [-1, -1, 0, 1, 0, 1, ...]
    d, b = _run([b"A", b"B"] * (n // 2), sites, durs, 3)
    assert d.tolist() == [-1, -1] + [i % 2 for i in range(n - 2)]
    # all distinct -> all -1, zero benefit
    d, b = _run([i.to_bytes(4, "little") for i in range(n)], sites, durs, 3)
    assert d.tolist() == [-1] * n and b.tolist() == [0, 0, 0]
    # empty log
    d, b = _run([], [], [], 2)
    assert d.tolist() == [] and b.tolist() == [0, 0]


def test_benefit_wraps_mod_2_64_and_linearity():
    big = (1 << 64) - 5
    d, b = _run([b"x", b"x", b"x"], [0, 0, 0], [1, big, 10], 1)
    assert b.tolist() == [(big + 10) % (1 << 64)]
    lg = loggen.gen_config(1, n_scale=0.3, size_scale=0.1)
    _, b1 = oracle.dedup(lg)
    lg.dur = lg.dur * np.uint64(3)
    _, b3 = oracle.dedup(lg)
    np.testing.assert_array_equal(b3, b1 * np.uint64(3))


def test_invariants_on_configs():
    for k in (1, 2, 3):
        lg = loggen.gen_config(k, n_scale=0.02 if k == 2 else 0.1, size_scale=0.05 if k == 3 else 0.5)
        d, b = oracle.dedup(lg)
        seen = {}
        for i in range(lg.n):
            p = lg.payload(i)
            j = int(d[i])
            if j >= 0:
                assert j < i and d[j] == -1               # points at a root, earlier
                assert lg.payload(j) == p                  # byte-equal
                assert seen[p] == j                        # the first one
            else:
                assert p not in seen                       # an original has no earlier equal
                seen[p] = i
        # conservation: sum of benefit == sum of duplicate durations (mod 2^64)
        assert int(b.sum(dtype=np.uint64)) == int(lg.dur[d >= 0].sum(dtype=np.uint64))
        assert int((d < 0).sum()) == len(seen)


def test_single_flip_breaks_duplicate():
    rng = np.random.default_rng(11)
    for size in (1, 15, 16, 17, 511, 512, 513, 4096, 16385):
        base = rng.integers(0, 256, size, dtype=np.uint8).tobytes()
        positions = sorted({0, size - 1, min(size - 1, 15), min(size - 1, 16), size // 2})
        for p in positions:
            arr = bytearray(base)
            arr[p] ^= 0x5A
            d, _ = _run([base, bytes(arr), base, bytes(arr)], hash_bits=64)
            assert d.tolist() == [-1, -1, 0, 1]
            d, _ = _run([base, bytes(arr), base, bytes(arr)], hash_bits=0)
            assert d.tolist() == [-1, -1, 0, 1]
        # a prefix and a zero-extension are not duplicates
        d, _ = _run([base, base[:-1], base + b"\0", base], hash_bits=0)
        assert d.tolist() == [-1, -1, -1, 0]


def test_sampled_one_by_one_matches_full():
    lg = loggen.gen_config(2, n_scale=0.01)
    d, _ = oracle.dedup(lg)
    for i in np.random.default_rng(2).integers(0, lg.n, 200).tolist():
        assert oracle.dup_of_one(lg, i) == d[i]


def test_oracle_rejects_bad_input():
    lg = loggen.from_payloads([b"a", b"b"], [0, 5], None, 2)
    with pytest.raises(ValueError):
        oracle.dedup(lg)
