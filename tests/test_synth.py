"""The shared seeded generators (synth/): determinism, shard independence,
BF16 representability.  CPU only."""
import numpy as np

import synth


def test_images_shard_regeneration():
    full = synth.images(0, 6, (3, 5, 4))
    part = synth.images(2, 3, (3, 5, 4))
    np.testing.assert_array_equal(full[2:5], part)
    assert full.dtype == np.float32
    assert full.min() >= -128 and full.max() <= 128


def test_bf16_rounding_is_rne_and_idempotent():
    one = np.float32(1.0)
    ulp = 2.0 ** -7                           # bf16 spacing at 1.0
    vals = np.array([1.0 + ulp / 2, 1.0 + 1.5 * ulp, 1.0 + 0.49 * ulp, -3.0], np.float32)
    r = synth.round_to_bf16(vals)
    np.testing.assert_array_equal(r, np.array([1.0, 1.0 + 2 * ulp, 1.0, -3.0], np.float32))
    x = synth.images(0, 2, (3, 8, 8))
    np.testing.assert_array_equal(synth.round_to_bf16(x), x)
    assert (x.view(np.uint32) & 0xFFFF == 0).all()
    assert one == synth.round_to_bf16(one)


def test_he_weights_statistics_and_determinism():
    w = synth.he_weights((64, 32, 3, 3), 32 * 9, 4)
    assert abs(w.std() - np.sqrt(2.0 / 288)) < 0.03 * np.sqrt(2.0 / 288)
    np.testing.assert_array_equal(w, synth.he_weights((64, 32, 3, 3), 32 * 9, 4))
    assert not np.array_equal(w, synth.he_weights((64, 32, 3, 3), 32 * 9, 5))


def test_net_params_shapes():
    net = synth.alexnet()
    ws, bs = synth.net_params(net)
    shapes = [None if w is None else w.shape for w in ws]
    assert shapes[0] == (96, 3, 11, 11)
    assert shapes[3] == (256, 48, 5, 5)
    assert shapes[10] == (4096, 9216)
    assert bs[12].shape == (1000,)


def test_planted_set_generator():
    """Planted-class images: deterministic by global index, label = index mod
    classes, image = its prototype plus small noise."""
    shp = (3, 40, 36)
    x1, l1 = synth.planted_images(5, 3, shp, 4)
    x2, l2 = synth.planted_images(5, 3, shp, 4)
    assert (x1 == x2).all() and list(l1) == [1, 2, 3]
    p = synth.prototypes(4, shp)
    d = np.abs(x1 - p[l1]).max(axis=(1, 2, 3))
    assert (d < 0.12 * 128 * 6).all() and (d > 0).all()
    assert np.abs(p[0] - p[1]).mean() > 20          # distinct prototypes
