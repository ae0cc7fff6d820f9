"""Pins for the shared input generator (rwgen): torch int64 vs a numpy uint64 SplitMix64."""
import numpy as np

import rwgen


def np_mix64(z):
    z = z.astype(np.uint64)
    with np.errstate(over="ignore"):
        z = (z ^ (z >> np.uint64(30))) * np.uint64(rwgen.M1)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(rwgen.M2)
    return z ^ (z >> np.uint64(31))


def test_torch_generator_matches_numpy_uint64():
    seed = rwgen.seed_col(1, 0, 0)
    i = np.arange(1000, 2000, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = np.uint64(seed) + (i + np.uint64(1)) * np.uint64(rwgen.GOLDEN)
    ref = np_mix64(z)
    got = rwgen.raw64(seed, 1000, 1000).numpy().view(np.uint64)
    assert np.array_equal(got, ref)
    assert np.array_equal(rwgen.u32(seed, 1000, 1000).numpy(), (ref >> np.uint64(32)).astype(np.int64))


def test_stateless_row_ranges_concatenate():
    a = rwgen.uniform_u32_relation(2, 0, 4, 0, 3000)
    b = rwgen.uniform_u32_relation(2, 0, 4, 1000, 1000)
    for c in a:
        assert np.array_equal(a[c][1000:2000].numpy(), b[c].numpy())


def test_lineitem_ranges():
    li = rwgen.lineitem(4, 0, 20000)
    assert li["qty"].min() >= 100 and li["qty"].max() <= 5000
    assert li["disc"].min() >= 0 and li["disc"].max() <= 10
    assert li["tax"].min() >= 0 and li["tax"].max() <= 8
    assert set(li["rf"].unique().tolist()) <= {0, 1, 2}
    assert set(li["ls"].unique().tolist()) <= {0, 1}
    assert li["price"].max() <= 10495000 * 1
