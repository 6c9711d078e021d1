"""Online (streaming) mode, S8(f) #2: labels produced window by window -- each window
compared with the stored representatives of all earlier transfers (PAPER.md
P:669-676) -- must equal the batch result and the oracle, bit for bit, for any
window split, including digest collisions across windows."""
import numpy as np
import pytest

import loggen
import oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ffm():
    import torch
    assert torch.cuda.is_available()
    import paper_conf_sc_weltonm19_b200 as m
    return m


def _online(ffm, lg, cuts, **kw):
    ptrs = lg.payload_ptrs()
    dups, bens = [], []
    with ffm.FfmLog(lg.n_sites, **kw) as log:
        prev = 0
        for c in list(cuts) + [lg.n]:
            if c > prev:
                sl = slice(prev, c)
                log.append_batch(lg.site[sl], lg.size[sl], ptrs[sl], lg.dur[sl],
                                 channels=None if lg.channel is None else lg.channel[sl])
            d, b = log.online_step()
            dups.append(d.copy())
            bens.append((c, b.copy()))
            prev = c
        batch_d, batch_b = log.run()
    return np.concatenate(dups), bens, batch_d, batch_b


MODES = {"step": {}, "online": {"online": True}, "append_hash": {"online": True, "append_hash": True}}


@pytest.mark.parametrize("k,ns,ss", [(1, 0.5, 0.25), (2, 0.01, 1.0), (3, 0.03, 1 / 32), (4, 0.1, 1 / 64),
                                     (5, 0.003, 1 / 32)])
@pytest.mark.parametrize("digest_bits", [64, 0])
@pytest.mark.parametrize("mode", list(MODES))
def test_online_equals_batch_and_oracle(ffm, k, ns, ss, digest_bits, mode):
    """step: the step uploads and processes its window (fused round 0); online: appends
    upload their metadata (FFM_FLAG_ONLINE), the step runs the fused round 0; append_hash:
    appends also hash (FFM_FLAG_APPEND_HASH), the step verifies two-pass."""
    lg = loggen.gen_config(k, n_scale=ns, size_scale=ss)
    rng = np.random.default_rng(k)
    cuts = sorted(set(rng.integers(1, lg.n, 6).tolist()))
    want_d, want_b = oracle.dedup(lg)
    got_d, bens, bd, bb = _online(ffm, lg, cuts, digest_bits=digest_bits, chunk_bytes=4096, **MODES[mode])
    np.testing.assert_array_equal(got_d, want_d)
    np.testing.assert_array_equal(bd, want_d)
    np.testing.assert_array_equal(bb, want_b)
    for end, b in bens:                       # cumulative benefit of every prefix
        np.testing.assert_array_equal(b, oracle.dedup(lg.subset(np.arange(end)))[1])


def test_online_single_record_windows_and_empty_steps(ffm):
    pay = [b"A", b"B", b"A", b"", b"", b"AB", b"A", b"B" * 40, b"B" * 40]
    lg = loggen.from_payloads(pay, [0, 1, 0, 1, 0, 1, 0, 1, 0], None, 2)
    got_d, bens, bd, bb = _online(ffm, lg, range(1, lg.n), digest_bits=0, refine_bits=0)
    want_d, want_b = oracle.dedup(lg)
    assert got_d.tolist() == want_d.tolist() == [-1, -1, 0, -1, 3, -1, 0, -1, 7]
    np.testing.assert_array_equal(bb, want_b)
    with ffm.FfmLog(2) as log:                # a step with nothing pending
        d, b = log.online_step()
        assert len(d) == 0 and b.tolist() == [0, 0]


def test_online_with_channels(ffm):
    lg = loggen.gen_config(2, n_scale=0.01)
    lg.channel = (lg.site.astype(np.uint64) % np.uint64(3))
    want_d, want_b = oracle.dedup(lg)
    got_d, bens, bd, bb = _online(ffm, lg, [100, 2000, 7000], digest_bits=8)
    np.testing.assert_array_equal(got_d, want_d)
    np.testing.assert_array_equal(bd, want_d)
    np.testing.assert_array_equal(bb, want_b)


@pytest.mark.parametrize("window", [1, 64, 4096])
@pytest.mark.parametrize("mode", ["online", "append_hash"])
def test_online_fixed_windows_grow_the_table(ffm, window, mode):
    """Fixed-size windows over a config-2-shaped log (many small transfers):
    the persistent table grows (rehash on doubling) across steps; the result never changes."""
    lg = loggen.gen_config(2, n_scale=0.004 if window == 1 else 0.02)
    cuts = list(range(window, lg.n, window))
    want_d, want_b = oracle.dedup(lg)
    got_d, bens, bd, bb = _online(ffm, lg, cuts, **MODES[mode])
    np.testing.assert_array_equal(got_d, want_d)
    np.testing.assert_array_equal(bens[-1][1], want_b)
    np.testing.assert_array_equal(bd, want_d)


@pytest.mark.parametrize("mode", ["online", "append_hash"])
def test_online_after_reset_and_forced_collisions_across_windows(ffm, mode):
    """ffm_log_reset empties the stored classes too; with digest_bits = refine_bits = 0
    every stored class of a size shares one chain (byte compares decide)."""
    lg = loggen.gen_config(3, n_scale=0.02, size_scale=1 / 64)
    want_d, want_b = oracle.dedup(lg)
    ptrs = lg.payload_ptrs()
    with ffm.FfmLog(lg.n_sites, digest_bits=0, refine_bits=0, **MODES[mode]) as log:
        for rep in range(2):
            dups = []
            for a in range(0, lg.n, 37):
                b = min(lg.n, a + 37)
                log.append_batch(lg.site[a:b], lg.size[a:b], ptrs[a:b], lg.dur[a:b])
                d, ben = log.online_step()
                dups.append(d.copy())
            np.testing.assert_array_equal(np.concatenate(dups), want_d)
            np.testing.assert_array_equal(ben, want_b)
            log.reset()


@pytest.mark.parametrize("mode", ["online", "append_hash"])
@pytest.mark.parametrize("digest_bits", [64, 0])
def test_online_device_payloads_and_outputs(ffm, mode, digest_bits):
    """Appends of device-resident payloads (hashed at append time with append_hash), labels
    written to device memory (the streaming shape of bench.py --online): fused windows of
    one size replay one captured step; digest_bits = 0 makes every window resolve residuals
    after its speculative labels (the fix-up path)."""
    import torch
    lg = loggen.gen_config(5, n_scale=0.002, size_scale=1 / 32)
    want_d, want_b = oracle.dedup(lg)
    buf = torch.from_numpy(lg.materialize()).cuda()
    ptrs = (lg.c_off[lg.content] + np.uint64(buf.data_ptr())).astype(np.uint64)
    dup = torch.empty(lg.n, dtype=torch.int64, device="cuda")
    ben = torch.empty(lg.n_sites, dtype=torch.int64, device="cuda")
    got = []
    with ffm.FfmLog(lg.n_sites, chunk_bytes=4096, digest_bits=digest_bits, **MODES[mode]) as log:
        for a in range(0, lg.n, 777):
            e = min(lg.n, a + 777)
            log.append_batch(lg.site[a:e], lg.size[a:e], ptrs[a:e], lg.dur[a:e], payload_kind=ffm.FFM_PAYLOAD_DEVICE)
            log.online_step(dup, ben)
            got.append(dup[:e - a].cpu().numpy().copy())
    np.testing.assert_array_equal(np.concatenate(got), want_d)
    np.testing.assert_array_equal(ben.cpu().numpy().view(np.uint64), want_b)


@pytest.mark.parametrize("digest_bits", [64, 0])
def test_online_pinned_host_outputs_and_table_growth(ffm, digest_bits):
    """Labels into pinned host memory (the captured window step copies into it), windows of
    one size long enough to replay the captured step several times while the stored-class
    table grows (rehash: the captured step must be re-made), a reset mid-stream, and a
    tail window of another size."""
    import torch
    lg = loggen.gen_config(2, n_scale=0.03)
    want_d, want_b = oracle.dedup(lg)
    ptrs = lg.payload_ptrs()
    dup = torch.empty(lg.n, dtype=torch.int64).pin_memory()
    ben = torch.empty(lg.n_sites, dtype=torch.int64).pin_memory()
    w = 997
    with ffm.FfmLog(lg.n_sites, digest_bits=digest_bits, online=True) as log:
        for rep in range(2):
            got = []
            for a in range(0, lg.n, w):
                e = min(lg.n, a + w)
                log.append_batch(lg.site[a:e], lg.size[a:e], ptrs[a:e], lg.dur[a:e])
                log.online_step(dup, ben)
                got.append(dup[:e - a].numpy().copy())
            np.testing.assert_array_equal(np.concatenate(got), want_d)
            np.testing.assert_array_equal(ben.numpy().view(np.uint64), want_b)
            log.reset()


@pytest.mark.parametrize("digest_bits", [64, 0])
def test_online_tiny_and_regular_windows_interleaved(ffm, digest_bits):
    """Windows of 1..12 records: the tiny ones (<= 8 small records) are labelled by one warp
    in order against the table, the others by the fused window step; both store classes the
    other finds (same digest, same table).  digest_bits = 0: every class of a size shares one
    chain; channels split equal bytes."""
    lg = loggen.gen_config(2, n_scale=0.004)
    lg.channel = (lg.site.astype(np.uint64) % np.uint64(2))
    want_d, want_b = oracle.dedup(lg)
    rng = np.random.default_rng(7)
    cuts, c = [], 0
    while c < lg.n:
        c += int(rng.integers(1, 13))
        cuts.append(min(c, lg.n))
    got_d, bens, bd, bb = _online(ffm, lg, cuts[:-1], digest_bits=digest_bits, online=True)
    np.testing.assert_array_equal(got_d, want_d)
    np.testing.assert_array_equal(bens[-1][1], want_b)
    for end, b in bens[::50]:
        np.testing.assert_array_equal(b, oracle.dedup(lg.subset(np.arange(end)))[1])
