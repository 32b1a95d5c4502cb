"""The seeded input generator (synth/): deterministic, shardable, right statistics."""
import numpy as np

import synth


def test_slab_is_bit_identical_to_full_rows():
    full = synth.noisy_rgba(96, 80, seed=4, sigma=0.13)
    slab = synth.noisy_rgba(96, 80, seed=4, sigma=0.13, row_begin=17, row_end=53)
    assert np.array_equal(full[17:53], slab)


def test_range_alpha_and_noise_std():
    img = synth.noisy_rgba(256, 256, seed=1, sigma=0.05)
    assert img.dtype == np.float32 and img.shape == (256, 256, 4)
    assert (img[..., :3] >= 0).all() and (img[..., :3] <= 1).all()
    assert (img[..., 3] == 1).all()
    # noise = image - clean; with sigma=0.05 and clean in [0.1, 0.9] nothing is clipped
    clean = synth.noisy_rgba(256, 256, seed=1, sigma=0.0)
    std = (img[..., :3] - clean[..., :3]).std()
    assert abs(std - 0.05) < 0.002


def test_seeds_differ_and_repeat():
    a = synth.noisy_rgba(32, 32, seed=1)
    assert np.array_equal(a, synth.noisy_rgba(32, 32, seed=1))
    assert not np.array_equal(a, synth.noisy_rgba(32, 32, seed=2))


def test_thermal_ranges():
    t0, p = synth.thermal_inputs(64, 48, seed=1)
    assert t0.dtype == np.float32 and p.dtype == np.float32
    assert t0.min() >= 323.15 and t0.max() < 343.16
    assert p.min() >= 0 and p.max() < 0.05
