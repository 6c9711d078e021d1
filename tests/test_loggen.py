"""The input generator: determinism and the planted-truth guarantees it claims."""
import numpy as np

import loggen


def test_materialize_is_deterministic_and_seeded():
    a = loggen.gen_config(1, n_scale=0.05, size_scale=0.1)
    b = loggen.gen_config(1, n_scale=0.05, size_scale=0.1)
    c = loggen.gen_config(1, seed=123, n_scale=0.05, size_scale=0.1)
    assert np.array_equal(a.materialize(), b.materialize())
    assert not np.array_equal(a.size, c.size) or not np.array_equal(a.materialize()[:1000], c.materialize()[:1000])


def test_derived_contents_differ_exactly_in_flips():
    lg = loggen.gen_config(3, n_scale=0.02, size_scale=1 / 32)
    lg.materialize()
    n_derived = 0
    for c in range(len(lg.c_base)):
        b = int(lg.c_base[c])
        if b < 0:
            continue
        n_derived += 1
        x = lg.content_bytes(c)
        y = lg.content_bytes(b)
        diff = np.nonzero(x != y)[0]
        fs, fe = int(lg.c_flip_start[c]), int(lg.c_flip_start[c + 1])
        assert sorted(diff.tolist()) == sorted(lg.flip_pos[fs:fe].tolist())
    assert n_derived > 10


def test_distinct_content_ids_have_distinct_bytes():
    for k in (1, 2, 3, 4, 5):
        lg = loggen.gen_config(k, n_scale=0.01 if k in (2, 5) else 0.1,
                               size_scale=1 / 64 if k >= 3 else 0.2)
        lg.materialize()
        seen = {}
        for c in range(len(lg.c_size)):
            key = lg.content_bytes(c).tobytes()
            assert key not in seen, (k, c, seen.get(key))
            seen[key] = c


def test_full_scale_shapes():
    # planning only (no materialisation): the BASELINE config shapes
    l2 = loggen.gen_config(2)
    assert l2.n == 1_000_000 and 256 <= int(l2.size.min()) and int(l2.size.max()) <= 4096
    d = l2.planted_duplicate_of()
    assert 0.55 < (d >= 0).mean() < 0.65
    l3 = loggen.gen_config(3)
    assert l3.n == 10_000 and set(l3.size.tolist()) == {1 << 20}
    l4 = loggen.gen_config(4)
    assert l4.n == 1000 and 16 << 20 <= int(l4.size.min()) and int(l4.size.max()) <= 64 << 20
