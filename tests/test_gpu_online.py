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


@pytest.mark.parametrize("k,ns,ss", [(1, 0.5, 0.25), (2, 0.01, 1.0), (3, 0.03, 1 / 32), (4, 0.1, 1 / 64),
                                     (5, 0.003, 1 / 32)])
@pytest.mark.parametrize("digest_bits", [64, 0])
def test_online_equals_batch_and_oracle(ffm, k, ns, ss, digest_bits):
    lg = loggen.gen_config(k, n_scale=ns, size_scale=ss)
    rng = np.random.default_rng(k)
    cuts = sorted(set(rng.integers(1, lg.n, 6).tolist()))
    want_d, want_b = oracle.dedup(lg)
    got_d, bens, bd, bb = _online(ffm, lg, cuts, digest_bits=digest_bits, chunk_bytes=4096)
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
