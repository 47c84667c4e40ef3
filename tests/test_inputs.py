"""The seeded input generator (shared by both sides; holds no method arithmetic)."""
import numpy as np

from paper_conf_ipps_wurypgll25_b200 import inputs as I


def test_splitmix64_known_values():
    # splitmix64 reference outputs of the Vigna generator seeded with 0
    # (state advances by the golden gamma before mixing): first outputs.
    x = np.array([0, 0x9E3779B97F4A7C15], dtype=np.uint64)
    out = I.splitmix64(x)
    assert int(out[0]) == 0xE220A8397B1DCDAF
    assert int(out[1]) == 0x6E789E6AA1B965F4


def test_box_slicing_is_coordinate_based():
    """A sub-box equals the same slice of a bigger box (sharding-invariant)."""
    big = I.gen_f16(7, I.STREAM_K, 3, 0, 4, 0, 6, 0, 40, 128)
    sub = I.gen_f16(7, I.STREAM_K, 3, 2, 2, 1, 3, 17, 9, 128)
    assert np.array_equal(big[2:4, 1:4, 17:26], sub)


def test_distribution_and_outliers():
    v = I.gen_f16(I.seed_for_config(1), I.STREAM_V, 0, 0, 8, 0, 8, 0, 64, 128).astype(np.float64)
    assert abs(v.mean()) < 0.02 and abs(v.std() - 1.1547) < 0.02
    assert np.abs(v).max() <= 4.0
    k = I.gen_f16(I.seed_for_config(1), I.STREAM_K, 0, 0, 2, 0, 32, 0, 64, 128).astype(np.float64)
    mask = I.outlier_mask(I.seed_for_config(1), 0, np.arange(32)[:, None], np.arange(128)[None, :])
    frac = mask.mean()
    assert 0.003 < frac < 0.03
    ks = k.std(axis=(0, 2))                      # [head][chan]
    assert np.all(ks[mask] > 4.0) and np.all(ks[~mask] < 2.0)


def test_streams_and_layers_differ():
    a = I.gen_f16(1, I.STREAM_K, 0, 0, 1, 0, 1, 0, 4, 64)
    b = I.gen_f16(1, I.STREAM_V, 0, 0, 1, 0, 1, 0, 4, 64)
    c = I.gen_f16(1, I.STREAM_K, 1, 0, 1, 0, 1, 0, 4, 64)
    assert not np.array_equal(a, b) and not np.array_equal(a, c)
