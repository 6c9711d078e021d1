"""Parity of the CUDA path (through the C ABI) against the CPU oracle -- bit-exact.

All outputs are integers (gids and nanoseconds), so the bar is bit-exact equality
of duplicate_of and benefit_ns with oracle/ffm_oracle.c on the same seeded logs.
"""
import json
import os

import numpy as np
import pytest

import loggen
import oracle

pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


@pytest.fixture(scope="module")
def ffm():
    import torch
    assert torch.cuda.is_available(), "the -m gpu tests need a CUDA device"
    import paper_conf_sc_weltonm19_b200 as m
    return m


def gpu_dedup(ffm, lg, device_payloads=False, **kw):
    with ffm.FfmLog(lg.n_sites, device=0, timing=True, **kw) as log:
        if device_payloads:
            import torch
            buf = torch.from_numpy(lg.materialize()).cuda()
            ptrs = (lg.c_off[lg.content] + np.uint64(buf.data_ptr())).astype(np.uint64)
            log.append_log(lg, ptrs=ptrs, payload_kind=ffm.FFM_PAYLOAD_DEVICE)
            del buf
        else:
            log.append_log(lg)
        dup, ben = log.run()
        return dup.copy(), ben.copy(), log.stats()


def assert_same(lg, dup, ben, hash_bits=64):
    want_dup, want_ben = oracle.dedup(lg, hash_bits=hash_bits)
    np.testing.assert_array_equal(dup, want_dup)
    np.testing.assert_array_equal(ben, want_ben)


@pytest.mark.parametrize("name", sorted(f for f in os.listdir(GOLDEN) if f.endswith(".json")))
@pytest.mark.parametrize("digest_bits", [64, 0])
def test_golden(ffm, name, digest_bits):
    fx = json.load(open(os.path.join(GOLDEN, name)))
    lg = loggen.from_payloads([bytes.fromhex(r["hex"]) for r in fx["records"]],
                              [r["site"] for r in fx["records"]], [r["dur"] for r in fx["records"]],
                              fx["n_sites"])
    if "channel" in fx["records"][0]:
        lg.channel = np.asarray([r["channel"] for r in fx["records"]], np.uint64)
    dup, ben, _ = gpu_dedup(ffm, lg, digest_bits=digest_bits)
    assert dup.tolist() == fx["expect_duplicate_of"]
    assert ben.tolist() == fx["expect_benefit_ns"]


def _rand_log(seed, n, alphabet, max_len):
    rng = np.random.default_rng(seed)
    base = [rng.integers(0, 256, int(rng.integers(0, max_len + 1)), dtype=np.uint8).tobytes()
            for _ in range(alphabet)]
    pay = []
    for _ in range(n):
        b = base[int(rng.integers(0, alphabet))]
        u = rng.random()
        if u < 0.25 and b:
            a = bytearray(b)
            a[int(rng.integers(0, len(a)))] ^= 1 + int(rng.integers(0, 255))
            b = bytes(a)
        elif u < 0.3:
            b = b[:-1]
        pay.append(b)
    ns = int(rng.integers(1, 7))
    return loggen.from_payloads(pay, rng.integers(0, ns, n), rng.integers(0, 1 << 40, n), ns)


@pytest.mark.parametrize("seed", range(12))
@pytest.mark.parametrize("digest_bits,refine_bits", [(64, 64), (8, 64), (0, 64), (0, 0)])
def test_random_tiny_logs(ffm, seed, digest_bits, refine_bits):
    lg = _rand_log(seed, int(np.random.default_rng(seed).integers(1, 400)), 12, 700)
    dup, ben, st = gpu_dedup(ffm, lg, digest_bits=digest_bits, refine_bits=refine_bits,
                             chunk_bytes=1024, small_bytes=128)
    assert_same(lg, dup, ben)


@pytest.mark.parametrize("chunk,small", [(1024, 128), (4096, 4096), (32768, 4096), (65536, 16384)])
@pytest.mark.parametrize("device_payloads", [False, True])
def test_configs_reduced(ffm, chunk, small, device_payloads):
    for k, ns, ss in [(1, 0.3, 0.25), (2, 0.01, 1.0), (3, 0.03, 1 / 16), (4, 0.1, 1 / 64), (5, 0.003, 1 / 32)]:
        lg = loggen.gen_config(k, n_scale=ns, size_scale=ss)
        dup, ben, st = gpu_dedup(ffm, lg, device_payloads, chunk_bytes=chunk, small_bytes=small)
        assert_same(lg, dup, ben)
        np.testing.assert_array_equal(dup, lg.planted_duplicate_of())


@pytest.mark.parametrize("digest_bits,refine_bits", [(64, 64), (16, 64), (0, 64), (0, 0)])
def test_forced_collisions_config3(ffm, digest_bits, refine_bits):
    lg = loggen.gen_config(3, n_scale=0.02 if refine_bits else 0.006, size_scale=1 / 32)
    dup, ben, st = gpu_dedup(ffm, lg, digest_bits=digest_bits, refine_bits=refine_bits, chunk_bytes=4096)
    assert_same(lg, dup, ben)
    if digest_bits == 0:
        assert st["n_residual"] > 0 and st["resolve_rounds"] >= 1


def test_digest_spec_and_chunk_invariance(ffm):
    from digest_spec import digest
    rng = np.random.default_rng(9)
    sizes = [0, 1, 15, 16, 17, 31, 32, 33, 255, 256, 257, 4095, 4096, 4097, 32767, 32768, 32769,
             100000, (1 << 20) + 3]
    pay = [rng.integers(0, 256, s, dtype=np.uint8).tobytes() for s in sizes]
    lg = loggen.from_payloads(pay)
    want = [digest(p) for p in pay]
    for chunk, small in [(1024, 128), (32768, 4096), (65536, 0)]:
        with ffm.FfmLog(1, chunk_bytes=chunk, small_bytes=small) as log:
            log.append_log(lg)
            log.run()
            got = log.digests()
        assert [int(x) for x in got] == want, (chunk, small)


@pytest.mark.parametrize("small", [4096, 16384, 128])
def test_small_pass_variants(ffm, small):
    """Small payloads through the fused small pass (k_fused_small: full-block fast path,
    masked tail): labels, benefit and digests at three thresholds, with empty payloads,
    ragged tails, sizes at and next to the threshold, members with a flipped last or
    random byte and re-uploads of several contents."""
    from digest_spec import digest
    rng = np.random.default_rng(17 + small)
    bases = [rng.integers(0, 256, int(s), dtype=np.uint8).tobytes()
             for s in list(rng.integers(0, small + 1, 40)) + [0, 1, 31, 32, 33, small - 1, small]]
    pay = []
    for _ in range(3000):
        b = bases[int(rng.integers(0, len(bases)))]
        if b and rng.random() < 0.15:
            a = bytearray(b)
            a[-1 if rng.random() < 0.5 else int(rng.integers(0, len(a)))] ^= 0x5A
            b = bytes(a)
        pay.append(b)
    lg = loggen.from_payloads(pay, rng.integers(0, 5, len(pay)), rng.integers(0, 1 << 40, len(pay)), 5)
    for db in (64, 0):
        with ffm.FfmLog(lg.n_sites, small_bytes=small, chunk_bytes=max(1024, small), digest_bits=db) as log:
            log.append_log(lg)
            dup, ben = log.run()
            assert_same(lg, dup, ben)
            if db == 64:
                got = log.digests()
                assert all(int(got[i]) == digest(pay[i]) for i in range(0, len(pay), 7))


def test_flip_at_boundaries(ffm):
    rng = np.random.default_rng(4)
    size = 3 * 4096 + 77
    base = rng.integers(0, 256, size, dtype=np.uint8).tobytes()
    pay = [base]
    for p in [0, 15, 16, 31, 32, 1023, 1024, 4095, 4096, 8191, 8192, size - 1]:
        a = bytearray(base)
        a[p] ^= 0x80
        pay += [bytes(a), base]
    lg = loggen.from_payloads(pay)
    for chunk, small in [(1024, 128), (4096, 16384)]:
        for db in (64, 0):
            dup, ben, _ = gpu_dedup(ffm, lg, chunk_bytes=chunk, small_bytes=small, digest_bits=db)
            assert dup.tolist() == [-1] + [-1, 0] * 12


def test_repeat_runs_and_appends_after_run(ffm):
    lg = loggen.gen_config(2, n_scale=0.005)
    half = lg.n // 2
    with ffm.FfmLog(lg.n_sites) as log:
        ptrs = lg.payload_ptrs()
        log.append_batch(lg.site[:half], lg.size[:half], ptrs[:half], lg.dur[:half])
        d1, b1 = [x.copy() for x in log.run()]
        sub = lg.subset(np.arange(half))
        assert_same(sub, d1, b1)
        log.append_batch(lg.site[half:], lg.size[half:], ptrs[half:], lg.dur[half:])
        outs = [tuple(x.copy() for x in log.run()) for _ in range(3)]
    for d, b in outs:
        np.testing.assert_array_equal(d, outs[0][0])
        np.testing.assert_array_equal(b, outs[0][1])
    assert_same(lg, *outs[0])


def test_single_appends_mixed_host_device(ffm):
    import torch
    lg = loggen.gen_config(1, n_scale=0.1, size_scale=0.1)
    buf = torch.from_numpy(lg.materialize()).cuda()
    with ffm.FfmLog(lg.n_sites) as log:
        hp = lg.payload_ptrs()
        for i in range(lg.n):
            c = int(lg.content[i])
            p = int(hp[i]) if i % 2 else buf.data_ptr() + int(lg.c_off[c])
            log.append(int(lg.site[i]), int(lg.size[i]), p, int(lg.dur[i]))
        dup, ben = log.run()
    assert_same(lg, dup, ben)


def test_batch_mixed_pageable_pinned_device(ffm):
    """One AUTO batch interleaving pageable, pinned and device payloads (runs of each, runs
    spanning several ring windows): the parallel pageable staging closes its run
    before every record written by another path; pageable bytes are snapshotted."""
    import torch
    lg = loggen.gen_config(5, n_scale=0.003, size_scale=1 / 8)
    host = lg.materialize()
    pageable = host.copy()
    pinned = torch.from_numpy(host.copy()).pin_memory()
    dev = torch.from_numpy(host).cuda()
    bases = [pageable.ctypes.data, pinned.data_ptr(), dev.data_ptr()]
    rng = np.random.default_rng(7)
    kind = np.repeat(rng.integers(0, 3, lg.n // 40 + 1), 40)[:lg.n]   # runs of 40 records
    ptrs = np.array([lg.c_off[lg.content[i]] + np.uint64(bases[kind[i]]) for i in range(lg.n)], np.uint64)
    with ffm.FfmLog(lg.n_sites) as log:
        log.append_batch(lg.site, lg.size, ptrs, lg.dur, payload_kind=ffm.FFM_PAYLOAD_AUTO)
        pageable[:] = 0                      # snapshot taken: later writes are invisible
        pinned.zero_()
        dup, ben = log.run()
    assert_same(lg, dup, ben)
    # (ring windows are 32 MiB: some pageable run spans several, so records straddle windows)
    spans = [int(lg.size[i:i + 40].sum()) for i in range(0, lg.n, 40) if kind[i] == 0]
    assert max(spans) > (32 << 20)


@pytest.mark.parametrize("kind", ["pinned", "auto_pinned", "pageable"])
def test_host_payload_kinds(ffm, kind):
    import torch
    lg = loggen.gen_config(5, n_scale=0.002, size_scale=1 / 16)
    host = lg.materialize()
    if kind != "pageable":
        pinned = torch.from_numpy(host).pin_memory()
        base = pinned.data_ptr()
    else:
        pinned, base = None, host.ctypes.data
    ptrs = (lg.c_off[lg.content] + np.uint64(base)).astype(np.uint64)
    pk = {"pinned": ffm.FFM_PAYLOAD_HOST_PINNED, "auto_pinned": ffm.FFM_PAYLOAD_AUTO,
          "pageable": ffm.FFM_PAYLOAD_HOST}[kind]
    with ffm.FfmLog(lg.n_sites) as log:
        log.append_log(lg, ptrs=ptrs, payload_kind=pk)
        if pinned is not None:
            pinned.zero_()                       # snapshot taken: later writes are invisible
        dup, ben = log.run()
    assert_same(lg, dup, ben)


def test_device_outputs(ffm):
    import torch
    lg = loggen.gen_config(5, n_scale=0.002, size_scale=1 / 64)
    with ffm.FfmLog(lg.n_sites) as log:
        log.append_log(lg)
        d = torch.empty(lg.n, dtype=torch.int64, device="cuda")
        b = torch.empty(lg.n_sites, dtype=torch.int64, device="cuda")
        log.run(d, b)
        assert_same(lg, d.cpu().numpy(), b.cpu().numpy().view(np.uint64))


def test_snapshot_semantics(ffm):
    a = np.frombuffer(b"0123456789abcdef" * 4, np.uint8).copy()
    with ffm.FfmLog(1) as log:
        log.append(0, a.nbytes, a.ctypes.data, 5)
        a[3] ^= 1                                   # caller mutates after append
        log.append(0, a.nbytes, a.ctypes.data, 7)
        a[3] ^= 1
        log.append(0, a.nbytes, a.ctypes.data, 11)
        dup, ben = log.run()
    assert dup.tolist() == [-1, -1, 0] and ben.tolist() == [11]


def test_errors_leave_log_unchanged(ffm):
    x = np.zeros(64, np.uint8)
    with ffm.FfmLog(2) as log:
        log.append(1, 64, x.ctypes.data, 1)
        with pytest.raises(ffm.FfmError) as e:
            log.append(2, 64, x.ctypes.data, 1)
        assert e.value.code == ffm.FFM_E_RANGE
        with pytest.raises(ffm.FfmError) as e:
            log.append(0, 8, 0, 1)
        assert e.value.code == ffm.FFM_E_INVAL
        with pytest.raises(ffm.FfmError) as e:
            log.append_batch([0, 1], [64, 64], [x.ctypes.data] * 2, [1, 1], gids=[5, 5])
        assert e.value.code == ffm.FFM_E_RANGE
        log.append(0, 0, 0, 3)                      # size 0 with NULL is fine
        assert log.count == 2
        dup, ben = log.run()
        assert dup.tolist() == [-1, -1]


def test_gids_are_reported(ffm):
    x = np.frombuffer(b"abcdefgh" * 8, np.uint8).copy()
    with ffm.FfmLog(1) as log:
        log.append_batch([0, 0, 0], [64, 32, 64], [x.ctypes.data] * 3, [1, 2, 3], gids=[10, 20, 35])
        dup, ben = log.run()
    assert dup.tolist() == [-1, -1, 10] and ben.tolist() == [3]


@pytest.mark.parametrize("k", [1, 2, 3])
def test_full_size_configs_1_to_3(ffm, k):
    lg = loggen.gen_config(k)
    lg.materialize(nthreads=0)
    dup, ben, st = gpu_dedup(ffm, lg)
    assert_same(lg, dup, ben)
    if k == 3:
        dup0, ben0, st0 = gpu_dedup(ffm, lg, digest_bits=0)
        np.testing.assert_array_equal(dup0, dup)
        np.testing.assert_array_equal(ben0, ben)
        assert st0["n_residual"] > 0


def test_site_counts_and_fold(ffm):
    from paper_conf_sc_weltonm19_b200 import report
    lg = loggen.gen_config(5, n_scale=0.003, size_scale=1 / 32)
    want_dup, want_ben = oracle.dedup(lg)
    want_cnt = np.bincount(lg.site[want_dup >= 0].astype(np.int64), minlength=lg.n_sites).astype(np.uint64)
    rng = np.random.default_rng(1)
    gmap = rng.integers(0, 37, lg.n_sites).astype(np.uint32)
    with ffm.FfmLog(lg.n_sites) as log:
        log.append_log(lg)
        dup, ben = log.run()
        cnt = log.site_counts()
        np.testing.assert_array_equal(cnt, want_cnt)
        g = log.fold(ben, gmap, 37)
        np.testing.assert_array_equal(log.fold(ben, np.arange(lg.n_sites, dtype=np.uint32), lg.n_sites), ben)
        np.testing.assert_array_equal(log.fold(ben, np.zeros(lg.n_sites, np.uint32), 1),
                                      [int(ben.sum(dtype=np.uint64))])
        names = [f"site{s}" for s in range(lg.n_sites)]
        funcs = [f"ns::fn{s % 7}<T{s % 3}>(int)" for s in range(lg.n_sites)]
        rep = report.ranked_report(ben, names, cnt, funcs, fold=log.fold, exec_time_ns=10**12)
    want_g = np.zeros(37, np.uint64)
    np.add.at(want_g, gmap.astype(np.int64), want_ben)
    np.testing.assert_array_equal(g, want_g)
    assert rep["total"]["benefit_ns"] == int(want_ben.sum(dtype=np.uint64))
    assert len(rep["folded_function"]) <= 7
    assert sum(r["benefit_ns"] for r in rep["folded_function"]) == rep["total"]["benefit_ns"]


@pytest.mark.parametrize("k", [4, 5])
def test_full_size_configs_4_5(ffm, k):
    """Full BASELINE sizes (config 4: 40.9 GB, config 5: 63.4 GB) in bench.py's launch
    configuration (default chunk / small sizes, device-resident payloads), against
    the full oracle run on the host (~10-20 s single core)."""
    import torch
    lg = loggen.gen_config(k)
    buf_h = lg.materialize(nthreads=0)
    want_dup, want_ben = oracle.dedup(lg)
    dev = torch.from_numpy(buf_h).cuda()
    ptrs = (lg.c_off[lg.content] + np.uint64(dev.data_ptr())).astype(np.uint64)
    with ffm.FfmLog(lg.n_sites, arena_bytes=lg.total_bytes + 32 * lg.n + (1 << 20), max_records=lg.n) as log:
        log.append_log(lg, ptrs=ptrs, payload_kind=ffm.FFM_PAYLOAD_DEVICE)
        del dev
        torch.cuda.empty_cache()
        d = torch.empty(lg.n, dtype=torch.int64, device="cuda")
        b = torch.empty(lg.n_sites, dtype=torch.int64, device="cuda")
        log.run(d, b)
        dup = d.cpu().numpy()
        ben = b.cpu().numpy().view(np.uint64)
    np.testing.assert_array_equal(dup, want_dup)
    np.testing.assert_array_equal(ben, want_ben)
    np.testing.assert_array_equal(dup, lg.planted_duplicate_of())


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("digest_bits", [64, 0])
def test_channels_destination_aware(ffm, seed, digest_bits):
    """S8(f) #3: a record duplicates only an earlier one with equal bytes AND channel."""
    lg = _rand_log(100 + seed, 300, 10, 600)
    rng = np.random.default_rng(seed)
    lg.channel = rng.integers(0, 3, lg.n).astype(np.uint64)
    dup, ben, _ = gpu_dedup(ffm, lg, digest_bits=digest_bits, chunk_bytes=1024, small_bytes=128)
    assert_same(lg, dup, ben)
    big = loggen.gen_config(5, n_scale=0.002, size_scale=1 / 32)
    big.channel = (big.site.astype(np.uint64) * np.uint64(7) + rng.integers(0, 2, big.n).astype(np.uint64)) \
        % np.uint64(5)
    dup, ben, _ = gpu_dedup(ffm, big, digest_bits=digest_bits)
    assert_same(big, dup, ben)


@pytest.mark.parametrize("digest_bits", [64, 0])
def test_prefilter_same_results(ffm, digest_bits):
    """S8(f) #4: skipping the rest of payloads with a unique (size, first chunk) prefix
    changes no output -- near-duplicates (configs 3, 4) share prefixes and still resolve."""
    for k, ns, ss in [(1, 0.5, 0.25), (3, 0.03, 1 / 16), (4, 0.1, 1 / 64), (5, 0.003, 1 / 32)]:
        lg = loggen.gen_config(k, n_scale=ns, size_scale=ss)
        dup, ben, st = gpu_dedup(ffm, lg, prefilter=True, digest_bits=digest_bits, chunk_bytes=4096)
        assert_same(lg, dup, ben)
        large = lg.size > 4096
        assert st["prefilter_rest_bytes"] <= int((lg.size[large] - 4096).clip(0).sum())


def test_prefilter_full_size_config5(ffm):
    lg = loggen.gen_config(5)
    lg.materialize(nthreads=0)
    want_dup, want_ben = oracle.dedup(lg)
    dup, ben, st = gpu_dedup(ffm, lg, prefilter=True)
    np.testing.assert_array_equal(dup, want_dup)
    np.testing.assert_array_equal(ben, want_ben)
    assert st["prefilter_rest_bytes"] < 0.8 * lg.total_bytes


def test_reset_reuses_the_log(ffm):
    a = loggen.gen_config(5, n_scale=0.002, size_scale=1 / 32)
    b = loggen.gen_config(2, n_scale=0.003)
    b.n_sites = a.n_sites           # same site space for one log
    with ffm.FfmLog(a.n_sites) as log:
        log.append_log(a)
        d1, b1 = [x.copy() for x in log.run()]
        log.reset()
        assert log.count == 0
        log.append_log(b)
        d2, b2 = [x.copy() for x in log.run()]
        log.reset()
        log.append_log(a)
        d3, _ = log.online_step()
        d3 = d3.copy()
    assert_same(a, d1, b1)
    assert_same(b, d2, b2)
    np.testing.assert_array_equal(d3, d1)


@pytest.mark.parametrize("digest_bits", [64, 0])
def test_two_pass_round0(ffm, digest_bits):
    """FFM_FLAG_TWO_PASS (hash all, group by full digest, verify) gives the same results."""
    for k, ns, ss in [(3, 0.03, 1 / 16), (4, 0.1, 1 / 64), (5, 0.003, 1 / 32)]:
        lg = loggen.gen_config(k, n_scale=ns, size_scale=ss)
        dup, ben, st = gpu_dedup(ffm, lg, two_pass=True, digest_bits=digest_bits, chunk_bytes=4096)
        assert_same(lg, dup, ben)


def test_difference_lists_settle_near_duplicates(ffm):
    """Config 3 shape: single-byte near-duplicates share their first 4 KiB with a base, so
    they mismatch it in the fused pass; their re-uploads are then settled exactly through
    the difference lists against the base (no bytes re-read), and the log stays fused."""
    lg = loggen.gen_config(3, n_scale=0.05, size_scale=1 / 8)
    want = oracle.dedup(lg)
    with ffm.FfmLog(lg.n_sites, timing=True) as log:
        log.append_log(lg)
        d1, b1 = [x.copy() for x in log.run()]
        s1 = log.stats()
        d2, b2 = [x.copy() for x in log.run()]
        s2 = log.stats()
    assert s1["two_pass"] == 0 and s2["two_pass"] == 0
    assert s1["n_residual"] > 0 and s1["n_reread"] * 10 <= s1["n_residual"]
    for d, b in ((d1, b1), (d2, b2)):
        np.testing.assert_array_equal(d, want[0])
        np.testing.assert_array_equal(b, want[1])


def _many_word_near_dups(seed, n_bases=6, n_var=8, reps=4, size=64 * 1024 + 48, words=9):
    """Variants of a few bases, each differing from its base in `words` 16-byte words past
    the first 4 KiB (more than a difference list holds), each uploaded `reps` times."""
    rng = np.random.default_rng(seed)
    pay = []
    for _ in range(n_bases):
        base = rng.integers(0, 256, size, dtype=np.uint8)
        pay.append(base.tobytes())
        for _ in range(n_var):
            v = base.copy()
            for q in rng.choice(np.arange(4096 // 16 + 1, size // 16), words, replace=False):
                v[16 * q + int(rng.integers(0, 16))] ^= 0xA5
            pay += [v.tobytes()] * reps
    order = rng.permutation(len(pay))
    order = np.concatenate([[i for i in order if i % (n_var * reps + 1) == 0],
                            [i for i in order if i % (n_var * reps + 1) != 0]])   # bases first
    pay = [pay[i] for i in order]
    return loggen.from_payloads(pay, rng.integers(0, 3, len(pay)), rng.integers(0, 1 << 40, len(pay)), 3)


def test_adaptive_round0(ffm):
    """Near-duplicates whose difference lists overflow must be re-read in the resolve
    rounds: the log switches itself to two-pass after one run; outputs never change."""
    lg = _many_word_near_dups(5)
    want = oracle.dedup(lg)
    with ffm.FfmLog(lg.n_sites, timing=True, chunk_bytes=16384) as log:
        log.append_log(lg)
        d1, b1 = [x.copy() for x in log.run()]
        s1 = log.stats()
        d2, b2 = [x.copy() for x in log.run()]
        s2 = log.stats()
    assert s1["two_pass"] == 0 and s2["two_pass"] == 1
    assert 2 * s1["n_reread"] > s1["n_members"]
    for d, b in ((d1, b1), (d2, b2)):
        np.testing.assert_array_equal(d, want[0])
        np.testing.assert_array_equal(b, want[1])
    with ffm.FfmLog(lg.n_sites, fused=True) as log:       # forced: no adaptation
        log.append_log(lg)
        log.run()
        log.run()
        assert log.stats()["two_pass"] == 0


@pytest.mark.parametrize("words", [1, 3, 4, 5, 9])
@pytest.mark.parametrize("digest_bits", [64, 0])
def test_difference_list_sizes(ffm, words, digest_bits):
    """Variants differing from their base in 1..9 words (the list holds 4): settled
    through lists up to 4, re-read beyond; exact either way."""
    lg = _many_word_near_dups(11 + words, n_bases=3, n_var=5, reps=3, words=words)
    dup, ben, st = gpu_dedup(ffm, lg, digest_bits=digest_bits, chunk_bytes=16384, fused=True)
    assert_same(lg, dup, ben)
    if digest_bits == 64 and words <= 4:
        assert st["n_reread"] == 0 and st["n_residual"] > 0


def test_benefit_linear_in_durations(ffm):
    """Scaling every duration by k scales every per-site benefit by k (mod 2^64)."""
    lg = loggen.gen_config(5, n_scale=0.002, size_scale=1 / 32)
    _, b1, _ = gpu_dedup(ffm, lg)
    lg.dur = lg.dur * np.uint64(7)
    _, b7, _ = gpu_dedup(ffm, lg)
    np.testing.assert_array_equal(b7, b1 * np.uint64(7))


class _LonelyWorld:
    """An ffm_comm_ops transport for a world of 2 in which rank 1 never has records: the
    collective run can be driven from one process (peer blocks are zeros)."""

    def __init__(self, ffm, fail=False):
        self.fail, self.calls = fail, 0
        self._ag = ffm.ALLGATHER_FN(self._allgather)
        self._ar = ffm.ALLREDUCE_FN(lambda ctx, buf, n: 0)      # sum with an all-zero peer
        self.ops = ffm.FfmCommOps(None, self._ag, self._ar)

    def _allgather(self, ctx, send, recv, nbytes):
        import ctypes
        self.calls += 1
        if self.fail:
            return -1
        if nbytes:
            ctypes.memmove(recv, send, nbytes)
            ctypes.memset(recv + nbytes, 0, nbytes)
        return 0


def test_sharded_api_errors_and_lonely_world(ffm):
    """Sharded-log rules (include/ffm.h): gids are required and < 2^63; online mode is
    single-log; a failing exchange poisons the handle; a world whose other rank is empty
    gives the single-log result through the whole collective path (header, export,
    all-gather, merge, all-reduce)."""
    x = np.frombuffer(b"abcdefgh" * 8, np.uint8).copy()
    w = _LonelyWorld(ffm)
    with ffm.FfmLog(2, rank=0, world=2, comm=w.ops) as log:
        with pytest.raises(ffm.FfmError) as e:
            log.append_batch([0, 1], [64, 64], [x.ctypes.data] * 2, [1, 2])      # no gids
        assert e.value.code == ffm.FFM_E_INVAL
        with pytest.raises(ffm.FfmError) as e:
            log.append_batch([0], [64], [x.ctypes.data], [1], gids=[1 << 63])
        assert e.value.code == ffm.FFM_E_RANGE
        log.append_batch([0, 1], [64, 64], [x.ctypes.data] * 2, [1, 2], gids=[0, 3])
        with pytest.raises(ffm.FfmError) as e:
            log.online_step()
        assert e.value.code == ffm.FFM_E_STATE
        for _ in range(2):
            dup, ben = log.run()
            assert dup.tolist() == [-1, 0] and ben.tolist() == [0, 2]
        assert log.site_counts().tolist() == [0, 1]
        st = log.stats()
        assert st["n_reps_local"] == 1 and st["n_reps_global"] == 1 and st["host_syncs"] == 2
    lg = loggen.gen_config(5, n_scale=0.002, size_scale=1 / 32)
    want = oracle.dedup(lg)
    w = _LonelyWorld(ffm)
    with ffm.FfmLog(lg.n_sites, rank=0, world=2, comm=w.ops, chunk_bytes=4096) as log:
        log.append_log(lg, gids=np.arange(lg.n) * 3 + 5)
        dup, ben = log.run()
        np.testing.assert_array_equal(np.where(want[0] >= 0, want[0] * 3 + 5, -1), dup)
        np.testing.assert_array_equal(ben, want[1])
    bad = _LonelyWorld(ffm, fail=True)
    with ffm.FfmLog(2, rank=0, world=2, comm=bad.ops) as log:
        log.append_batch([0, 1], [64, 64], [x.ctypes.data] * 2, [1, 2], gids=[0, 3])
        with pytest.raises(ffm.FfmError) as e:
            log.run()
        assert e.value.code == ffm.FFM_E_COMM
        with pytest.raises(ffm.FfmError) as e:
            log.run()
        assert e.value.code == ffm.FFM_E_STATE                 # poisoned


def test_graph_replay_matches_direct_launches(ffm):
    """Runs replay a captured CUDA graph while the log is unchanged; appends, output
    buffer changes and mode changes re-capture.  Same results as direct launches."""
    import torch
    lg = loggen.gen_config(5, n_scale=0.002, size_scale=1 / 32)
    want = oracle.dedup(lg)
    half = lg.n // 2
    ptrs = lg.payload_ptrs()
    for graph in (True, False):
        with ffm.FfmLog(lg.n_sites, graph=graph, timing=True) as log:
            log.append_batch(lg.site[:half], lg.size[:half], ptrs[:half], lg.dur[:half])
            for _ in range(3):
                d, b = log.run()
            np.testing.assert_array_equal(d, oracle.dedup(lg.subset(np.arange(half)))[0])
            log.append_batch(lg.site[half:], lg.size[half:], ptrs[half:], lg.dur[half:])
            for _ in range(2):
                d, b = log.run()
                np.testing.assert_array_equal(d, want[0])
                np.testing.assert_array_equal(b, want[1])
            dd = torch.empty(lg.n, dtype=torch.int64, device="cuda")
            bb = torch.empty(lg.n_sites, dtype=torch.int64, device="cuda")
            for _ in range(2):
                log.run(dd, bb)
                np.testing.assert_array_equal(dd.cpu().numpy(), want[0])
                np.testing.assert_array_equal(bb.cpu().numpy().view(np.uint64), want[1])


def test_empty_log_and_all_empty_payloads(ffm):
    """Degenerate logs (S8(c) edge cases): no records at all -> empty duplicate_of, zero
    benefit; 5000 empty payloads over 7 sites (several thread blocks) -> each one after the
    first duplicates record 0 (reading R7), benefit = the sites' duration sums
    minus the first record's."""
    with ffm.FfmLog(3) as log:
        dup, ben = log.run()
    assert dup.tolist() == [] and ben.tolist() == [0, 0, 0]
    n = 5000
    sites = [i % 7 for i in range(n)]
    durs = [1000 + 3 * i for i in range(n)]
    with ffm.FfmLog(7) as log:
        log.append_batch(sites, [0] * n, [0] * n, durs)
        dup, ben = log.run()
    assert dup.tolist() == [-1] + [0] * (n - 1)
    want = [0] * 7
    for i in range(1, n):
        want[sites[i]] += durs[i]
    assert ben.tolist() == want


@pytest.mark.parametrize("kind", ["device", "pinned"])
def test_large_batch_parallel_staging(ffm, kind):
    """A batch of >= 65,536 device or page-locked payloads is classified and its gather
    descriptors written by the host threads in parallel; empty payloads and payloads
    above the gather limit (copy engines) mixed in; bytes snapshotted before return."""
    import torch
    lg = loggen.gen_config(2, n_scale=0.12)
    host = lg.materialize()
    buf = torch.from_numpy(host.copy()).cuda() if kind == "device" else torch.from_numpy(host.copy()).pin_memory()
    ptrs = (lg.c_off[lg.content] + np.uint64(buf.data_ptr())).astype(np.uint64)
    sizes = lg.size.copy()
    sizes[::997] = 0                                  # empty payloads (all equal, R7)
    big = np.zeros(3 << 20, np.uint8)                 # > the 1 MiB gather limit: copy engines
    big[::4099] = 7
    bt = torch.from_numpy(big).cuda() if kind == "device" else torch.from_numpy(big).pin_memory()
    sizes[5::20011] = big.size
    ptrs[5::20011] = bt.data_ptr()
    lg2 = loggen.from_payloads([host[lg.c_off[lg.content[i]]:lg.c_off[lg.content[i]] + sizes[i]].tobytes()
                                if ptrs[i] != bt.data_ptr() else big.tobytes() for i in range(lg.n)],
                               lg.site, lg.dur, lg.n_sites)
    pk = ffm.FFM_PAYLOAD_DEVICE if kind == "device" else ffm.FFM_PAYLOAD_HOST_PINNED
    with ffm.FfmLog(lg.n_sites) as log:
        log.append_batch(lg.site, sizes, ptrs, lg.dur, payload_kind=pk)
        buf.zero_()                                   # snapshot taken: later writes are invisible
        bt.zero_()
        dup, ben = log.run()
    want_d, want_b = oracle.dedup(lg2)
    np.testing.assert_array_equal(dup, want_d)
    np.testing.assert_array_equal(ben, want_b)


def test_large_batch_errors_leave_log_unchanged(ffm):
    """A batch of >= 65,536 records is planned by the host threads in parallel: the first
    offending record decides the error (as record-by-record checking would) and the log is
    left unchanged."""
    n = 100_000
    x = np.zeros(64, np.uint8)
    sites = np.zeros(n, np.uint32)
    sizes = np.full(n, 64, np.uint64)
    ptrs = np.full(n, x.ctypes.data, np.uint64)
    durs = np.ones(n, np.uint64)
    gids = np.arange(n, dtype=np.uint64) * 2
    with ffm.FfmLog(4) as log:
        s2 = sites.copy()
        s2[90_000] = 4                        # call_site out of range, later than ...
        g2 = gids.copy()
        g2[70_001] = g2[70_000]               # ... a gid that is not increasing: reported first
        with pytest.raises(ffm.FfmError) as e:
            log.append_batch(s2, sizes, ptrs, durs, gids=g2)
        assert e.value.code == ffm.FFM_E_RANGE and "increasing" in str(e.value)
        p2 = ptrs.copy()
        p2[66_000] = 0                        # NULL payload before the out-of-range site
        with pytest.raises(ffm.FfmError) as e:
            log.append_batch(s2, sizes, p2, durs, gids=gids)
        assert e.value.code == ffm.FFM_E_INVAL
        assert log.count == 0
        log.append_batch(sites, sizes, ptrs, durs, gids=gids)
        assert log.count == n
        dup, ben = log.run()
        assert dup[0] == -1 and (dup[1:] == 0).all() and int(ben[0]) == n - 1
