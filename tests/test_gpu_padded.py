"""Padded-layout ("shifted window") conv mode (kernel K1 a_mode 2):
activations live on zero-haloed grids, one TMA row window per filter row
feeds all S taps.  Parity with the FP64 oracle, agreement with the im2col
mode, ragged tails, the rank-r variant and the SM budget on pm layers."""
import numpy as np
import pytest

from tests.helpers import (FLAG_CONV_LRN_EPILOGUE, FLAG_NARROW_SLABS, FLAG_NO_LRN_POOL_FUSION,
                           FLAG_NO_PADDED_LAYOUT, FLAG_PER_ROW_WINDOWS, FLAG_PERFORATION_IM2COL,
                           TOL, conv_layer, gpu_run, params, rel_err, small_inputs)

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


def vgg_like(hw=40, c1=64, c2=128, groups=1):
    """VGG-shaped blocks (3x3 / 1 / pad 1 convs + 2x2 pools) at a size whose
    halo overhead passes the 25% rule and whose M = B*(H+2)*(W+2) rows end
    in a ragged tile."""
    q = hw // 4
    return dict(in_shape=(3, hw, hw), layers=[
        conv_layer(c1, 3, 3, 1, 1), conv_layer(c1, 3, c1, 1, 1, groups),
        dict(kind="maxpool", k=2, stride=2),
        conv_layer(c2, 3, c1, 1, 1), conv_layer(c2, 3, c2, 1, 1, groups),
        dict(kind="maxpool", k=2, stride=2),
        dict(kind="fc", out=16, in_f=c2 * q * q, relu=False)])


PM_LAYERS = [0, 1, 3, 4]


@pytest.mark.parametrize("prec", ["tf32", "bf16"])
def test_padded_mode_matches_oracle(orc, prec):
    net = vgg_like()
    w, b = params(net, seed=21)
    x = small_inputs((3, 40, 40), 3, lo=-128, hi=128)
    ref = orc.run_net(net, w, b, x).reshape(3, -1)
    r = gpu_run(net, w, b, x, prec)
    infos = [r["net"].query_layer(i, 3) for i in range(len(net["layers"]))]
    assert [i for i, f in enumerate(infos) if f["a_mode"] == 2] == PM_LAYERS
    assert [(f["halo_in"], f["halo_out"]) for f in infos] == \
        [(1, 1), (1, 1), (1, 1), (1, 1), (1, 1), (1, 0), (0, 0)]
    assert rel_err(r["out"], ref) <= TOL[prec] / 2


@pytest.mark.parametrize("prec", ["tf32", "bf16"])
def test_padded_mode_agrees_with_im2col_mode(orc, prec):
    """Same products, different K order: the two A-addressing modes agree far
    inside the tolerance (and the zero halos never leak into the result)."""
    net = vgg_like(hw=36, c1=64, c2=64)
    w, b = params(net, seed=5)
    x = small_inputs((3, 36, 36), 5, lo=-128, hi=128)
    pm = gpu_run(net, w, b, x, prec)
    assert pm["net"].query_layer(1, 5)["a_mode"] == 2
    im = gpu_run(net, w, b, x, prec, flags=FLAG_NO_PADDED_LAYOUT)
    assert im["net"].query_layer(1, 5)["a_mode"] == 0
    assert rel_err(pm["out"], im["out"]) <= TOL[prec] / 4


def test_padded_mode_grouped_conv(orc):
    net = vgg_like(hw=40, c1=128, c2=128, groups=2)
    w, b = params(net, seed=8)
    x = small_inputs((3, 40, 40), 2, lo=-128, hi=128)
    ref = orc.run_net(net, w, b, x).reshape(2, -1)
    r = gpu_run(net, w, b, x, "bf16")
    assert r["net"].query_layer(1, 2)["a_mode"] == 2
    assert rel_err(r["out"], ref) <= TOL["bf16"] / 2


@pytest.mark.parametrize("prec", ["tf32", "bf16"])
def test_padded_mode_rank_variant(orc, prec):
    """Rank-r on a pm layer: both stages stay on the halo grid."""
    net = vgg_like()
    w, b = params(net, seed=21)
    x = small_inputs((3, 40, 40), 2, lo=-128, hi=128)
    for i, r in [(1, 24), (4, 48)]:
        ref = orc.run_net(net, w, b, x, ranks={i: r}).reshape(2, -1)
        res = gpu_run(net, w, b, x, prec, variants={i: ("rank", r)})
        assert res["net"].query_layer(i, 2)["a_mode"] == 2
        assert rel_err(res["out"], ref) <= TOL[prec] / 2, (prec, i, r)


def test_padded_mode_budget_bitwise():
    net = vgg_like()
    w, b = params(net, seed=21)
    x = small_inputs((3, 40, 40), 3, lo=-128, hi=128)
    base = gpu_run(net, w, b, x, "bf16")["out"]
    for n_sms in (2, 16, 74):
        r = gpu_run(net, w, b, x, "bf16", budgets={i: (n_sms, 0) for i in PM_LAYERS}, census=True)
        np.testing.assert_array_equal(r["out"], base)
        for i in PM_LAYERS:
            assert 0 < len(r["census"][i]) <= n_sms


def test_padded_mode_batch_one_and_max_batch(orc):
    """B = 1 (M smaller than one CTA pair's rows) and a net created for a
    larger max batch run at a smaller batch."""
    net = vgg_like(hw=24, c1=64, c2=64)
    w, b = params(net, seed=3)
    x = small_inputs((3, 24, 24), 1, lo=-128, hi=128)
    ref = orc.run_net(net, w, b, x).reshape(1, -1)
    r = gpu_run(net, w, b, x, "bf16", max_batch=7)
    assert r["net"].query_layer(1, 1)["a_mode"] == 2
    assert rel_err(r["out"], ref) <= TOL["bf16"] / 2


@pytest.mark.parametrize("cg", ["1", "2"])
@pytest.mark.parametrize("groups", [1, 2])
def test_padded_mode_two_subtiles_bitwise(orc, cg, groups):
    """msub = 2 (two 128-row M sub-tiles per CTA sharing every weight slab,
    two TMEM accumulators) computes each sub-tile with the same UMMA sequence
    as msub = 1: bitwise equal outputs, ragged last tile included."""
    net = vgg_like(hw=36, c1=64 * groups, c2=128, groups=groups)
    w, b = params(net, seed=13)
    x = small_inputs((3, 36, 36), 3, lo=-128, hi=128)
    ref = orc.run_net(net, w, b, x).reshape(3, -1)
    out = {}
    for ms in ("1", "2"):
        r = gpu_run(net, w, b, x, "bf16", plans={1: (int(cg), int(ms))})
        f = r["net"].query_layer(1, 3)
        assert f["a_mode"] == 2 and f["tile_m"] == 128 * int(cg) * int(ms)
        out[ms] = r["out"]
    np.testing.assert_array_equal(out["1"], out["2"])
    assert rel_err(out["2"], ref) <= TOL["bf16"] / 2


@pytest.mark.parametrize("prec", ["bf16", "tf32"])
def test_padded_mode_narrow_slabs(orc, prec):
    """PCNN_FLAG_NARROW_SLABS: a grouped conv with 48 channels per group (AlexNet
    conv2's input) stays unpadded and runs in padded-layout mode on SW32
    (BF16) / SW64 (TF32) slabs, each tap's window shifted by one narrow row."""
    net = dict(in_shape=(96, 27, 27), layers=[
        dict(kind="maxpool", k=1, stride=1),
        conv_layer(256, 5, 96, 1, 2, 2), dict(kind="maxpool", k=3, stride=2)])
    w, b = params(net, seed=12)
    x = small_inputs((96, 27, 27), 2, lo=-2, hi=2)
    ref = orc.run_net(net, w, b, x).reshape(2, -1)
    r = gpu_run(net, w, b, x, prec, flags=FLAG_NARROW_SLABS)
    assert r["net"].query_layer(1, 2)["a_mode"] == 2
    assert rel_err(r["out"], ref) <= TOL[prec] / 2


@pytest.mark.parametrize("prec", ["bf16", "tf32"])
def test_padded_mode_conv_lrn_fusion(orc, prec):
    """AlexNet conv1 -> norm1 -> pool1 shape (space-to-depth conv in padded-
    layout mode): LRN fused into the conv epilogue writes the halo layout the
    pool reads; agrees with the unfused kernels and the oracle."""
    net = dict(in_shape=(3, 67, 67), layers=[
        conv_layer(96, 11, 3, 4, 0, 1, relu=True),
        dict(kind="lrn", size=5, alpha=1e-4, beta=0.75, k=1.0),
        dict(kind="maxpool", k=3, stride=2)])
    w, b = params(net, seed=21)
    x = small_inputs((3, 67, 67), 2, lo=-128, hi=128)
    ref = orc.run_net(net, w, b, x).reshape(2, -1)
    fused = gpu_run(net, w, b, x, prec, flags=FLAG_CONV_LRN_EPILOGUE)
    assert fused["net"].query_layer(0, 2)["a_mode"] == 2
    pr = gpu_run(net, w, b, x, prec, flags=FLAG_NO_LRN_POOL_FUSION)
    plain = pr["out"]
    assert fused["net"].last_launch_count() < pr["net"].last_launch_count()
    assert rel_err(fused["out"], ref) <= TOL[prec] / 4
    assert rel_err(plain, ref) <= TOL[prec] / 4
    # last-place differences of the storage format (R16)
    ulp = 2.0 ** -8 if prec == "bf16" else 2.0 ** -10
    assert rel_err(fused["out"], plain) <= 2 * ulp


@pytest.mark.parametrize("prec", ["bf16", "tf32"])
def test_padded_mode_skips_channel_padding(orc, prec):
    """AlexNet conv2-shaped grouped conv (48 real channels per group stored
    as 64): the UMMAs that would only multiply the zero padding are skipped;
    the result matches the oracle and the narrow-slab plan (which has no
    padding to skip)."""
    net = dict(in_shape=(96, 27, 27), layers=[
        dict(kind="maxpool", k=1, stride=1),
        conv_layer(256, 5, 96, 1, 2, 2), dict(kind="maxpool", k=3, stride=2)])
    w, b = params(net, seed=12)
    x = small_inputs((96, 27, 27), 2, lo=-2, hi=2)
    fast = gpu_run(net, w, b, x, prec)
    assert fast["net"].query_layer(1, 2)["a_mode"] == 2
    ref = orc.run_net(net, w, b, x).reshape(2, -1)
    assert rel_err(fast["out"], ref) <= TOL[prec] / 2
    narrow = gpu_run(net, w, b, x, prec, flags=FLAG_NARROW_SLABS)["out"]
    assert rel_err(fast["out"], narrow) <= TOL[prec] / 8


@pytest.mark.parametrize("prec", ["bf16", "tf32"])
@pytest.mark.parametrize("shape,cout,k,groups,B", [
    ((256, 13, 13), 384, 3, 1, 16),     # AlexNet conv3 (14-wide shared-halo grid)
    ((384, 13, 13), 256, 3, 2, 16),     # conv5, grouped
    ((64, 23, 23), 96, 3, 1, 24),       # narrow N, several windows per image row
])
def test_whole_window_bitwise_equals_per_row_windows(orc, prec, shape, cout, k, groups, B):
    """Whole-slab A windows (one TMA window of 128 + (S-1)(wv+1) rows feeds
    all S x S taps) change only which shared-memory rows each tap's UMMA
    reads: the K order (slab, filter row, tap) is the per-row mode's, so the
    result is bitwise the same; and the oracle's tolerance."""
    C = shape[0]
    net = dict(in_shape=shape, layers=[dict(kind="maxpool", k=1, stride=1),
                                       conv_layer(cout, k, C, 1, k // 2, groups),
                                       dict(kind="maxpool", k=1, stride=1)])
    w, b = params(net, seed=31)
    x = small_inputs(shape, B, lo=-4, hi=4)
    ww = gpu_run(net, w, b, x, prec)
    pr = gpu_run(net, w, b, x, prec, flags=FLAG_PER_ROW_WINDOWS)
    fw, fr = ww["net"].query_layer(1, B), pr["net"].query_layer(1, B)
    assert fw["a_mode"] == 2 and fr["a_mode"] == 2
    assert fw["whole_window"] == 1 and fr["whole_window"] == 0
    np.testing.assert_array_equal(ww["out"], pr["out"])
    ref = orc.run_net(net, w, b, x[:2]).reshape(2, -1)
    assert rel_err(ww["out"][:2], ref) <= TOL[prec] / 4
