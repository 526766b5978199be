"""Perforation-interpolation conv variant (NEXT-1; Fig. 11; DESIGN.md
R13) through the C ABI against the FP64 oracle: the conv runs on the kept
sh x sw output grid (tcgen05 im2col mode with traversal strides sh, sw, on
zero-haloed inputs too) and an interpolation kernel fills every output
position from its nearest kept neighbour."""
import numpy as np
import pytest

import synth
from tests.helpers import (FLAG_CONV_LRN_EPILOGUE, FLAG_NARROW_SLABS, FLAG_NO_LRN_POOL_FUSION,
                           FLAG_NO_PADDED_LAYOUT, FLAG_PERFORATION_IM2COL, TOL, conv_layer,
                           gpu_run, params, rel_err, small_inputs)

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


def vgg_like(hw=36, c1=64, c2=128, groups=1):
    q = hw // 4
    return dict(in_shape=(3, hw, hw), layers=[
        conv_layer(c1, 3, 3, 1, 1), conv_layer(c1, 3, c1, 1, 1, groups),
        dict(kind="maxpool", k=2, stride=2),
        conv_layer(c2, 3, c1, 1, 1), conv_layer(c2, 3, c2, 1, 1, groups),
        dict(kind="maxpool", k=2, stride=2),
        dict(kind="fc", out=16, in_f=c2 * q * q, relu=False)])


@pytest.mark.parametrize("prec", ["tf32", "bf16"])
@pytest.mark.parametrize("steps", [(1, 2), (2, 2), (2, 3), (3, 1)])
def test_perforated_layers_match_oracle(orc, prec, steps):
    """Perforated padded-layout layers (input on a zero-haloed grid) inside a
    VGG-shaped net: every layer's kept-grid conv + interpolation, end to end."""
    net = vgg_like()
    w, b = params(net, seed=31)
    x = small_inputs((3, 36, 36), 3, lo=-128, hi=128)
    perf = {1: steps, 4: steps}
    ref = orc.run_net(net, w, b, x, perforation=perf).reshape(3, -1)
    r = gpu_run(net, w, b, x, prec, perforation=perf)
    assert rel_err(r["out"], ref) <= TOL[prec] / 2, (prec, steps)
    f = r["net"].query_layer(1, 3)
    kept = len(range(0, 36, steps[0])) * len(range(0, 36, steps[1]))
    assert abs(f["flops"] / f["flops_exact"] - kept / 36.0 ** 2) < 1e-12


def test_perforated_grouped_strided_layer(orc):
    """AlexNet-shaped grouped conv (conv2: 5x5 pad 2, groups 2) and a strided
    conv, perforated: layer outputs against the oracle."""
    net = dict(in_shape=(96, 27, 27), layers=[
        conv_layer(256, 5, 96, 1, 2, 2), dict(kind="maxpool", k=3, stride=2),
        conv_layer(64, 3, 256, 2, 1, 1)])
    w, b = params(net, seed=9)
    x = small_inputs((96, 27, 27), 2, lo=-2, hi=2)
    perf = {0: (2, 2), 2: (1, 2)}
    ref = orc.run_net(net, w, b, x, perforation=perf).reshape(2, -1)
    out = gpu_run(net, w, b, x, "bf16", perforation=perf)["out"]
    assert rel_err(out, ref) <= TOL["bf16"] / 2


def test_perforation_off_is_exact_bitwise(orc):
    """Steps (1, 1) restore the exact layer (same kernels, bitwise)."""
    net = vgg_like()
    w, b = params(net, seed=31)
    x = small_inputs((3, 36, 36), 2, lo=-128, hi=128)
    base = gpu_run(net, w, b, x, "bf16")["out"]
    r = gpu_run(net, w, b, x, "bf16", perforation={1: (1, 1), 4: (1, 1)})
    np.testing.assert_array_equal(r["out"], base)


def test_perforation_interpolation_structure():
    """Single perforated layer as the net output: every output column / row
    repeats its nearest kept one (R13), bit for bit on the GPU."""
    net = dict(in_shape=(16, 13, 11), layers=[conv_layer(32, 3, 16, 1, 1, 1)])
    w, b = params(net, seed=4)
    x = small_inputs((16, 13, 11), 2)
    sh, sw = 2, 3
    y = gpu_run(net, w, b, x, "bf16", perforation={0: (sh, sw)})["out"].reshape(2, 32, 13, 11)

    def src(p, s, n):
        lo, hi = p // s * s, p // s * s + s
        return hi if (hi < n and hi - p < p - lo) else lo
    for p in range(13):
        for q in range(11):
            np.testing.assert_array_equal(y[:, :, p, q], y[:, :, src(p, sh, 13), src(q, sw, 11)])


def test_perforation_rejections():
    import torch  # noqa: F401
    from paper_conf_hpca_songhcl17_b200 import pcnn
    net = synth.alexnet()
    w, b = params(net)
    n = pcnn.Net(net, w, b, 1, "bf16")
    with pytest.raises(pcnn.PcnnError):
        n.set_perforation(1, 2, 2)        # LRN layer
    with pytest.raises(pcnn.PcnnError):
        n.set_perforation(3, 5, 1)        # step out of range
    n.set_variant(3, "rank", 64)
    with pytest.raises(pcnn.PcnnError):
        n.set_perforation(3, 2, 2)        # rank-r layer
    n.set_variant(3, "exact")
    n.set_perforation(3, 2, 2)
    n.close()


@pytest.mark.parametrize("prec", ["bf16", "tf32"])
@pytest.mark.parametrize("sh", [2, 3])
def test_row_perforation_padded_layout(orc, prec, sh):
    """Row perforation (s_w = 1) of padded-layout layers runs the kept rows in
    padded-layout mode (row-strided 3-D TMA windows, segments of W + 2h + 2p
    rows): oracle parity, agreement with the im2col kept grid, and the
    AlexNet conv2 shape (5x5, groups 2) included."""
    net = vgg_like()
    w, b = params(net, seed=31)
    x = small_inputs((3, 36, 36), 3, lo=-128, hi=128)
    perf = {1: (sh, 1), 4: (sh, 1)}
    ref = orc.run_net(net, w, b, x, perforation=perf).reshape(3, -1)
    r = gpu_run(net, w, b, x, prec, perforation=perf)
    assert r["net"].query_layer(1, 3)["a_mode"] == 2
    assert rel_err(r["out"], ref) <= TOL[prec] / 2
    r2 = gpu_run(net, w, b, x, prec, perforation=perf, flags=FLAG_PERFORATION_IM2COL)
    assert r2["net"].query_layer(1, 3)["a_mode"] == 0
    assert rel_err(r["out"], r2["out"]) <= TOL[prec] / 4
    anet = dict(in_shape=(96, 27, 27), layers=[
        dict(kind="maxpool", k=1, stride=1), conv_layer(256, 5, 96, 1, 2, 2),
        dict(kind="maxpool", k=3, stride=2)])
    aw, ab = params(anet, seed=9)
    ax = small_inputs((96, 27, 27), 2, lo=-2, hi=2)
    aref = orc.run_net(anet, aw, ab, ax, perforation={1: (sh, 1)}).reshape(2, -1)
    ar = gpu_run(anet, aw, ab, ax, prec, perforation={1: (sh, 1)})
    assert ar["net"].query_layer(1, 2)["a_mode"] == 2
    assert rel_err(ar["out"], aref) <= TOL[prec] / 2


@pytest.mark.parametrize("sh", [2, 4])
def test_row_perforation_feeding_padded_conv(orc, sh):
    """A row-perforated padded-layout layer whose consumer is another
    padded-layout conv: the direct multi-row epilogue stores and the halo-row
    zeroing must leave exactly the zero border the consumer reads."""
    net = vgg_like()
    w, b = params(net, seed=33)
    x = small_inputs((3, 36, 36), 2, lo=-128, hi=128)
    perf = {3: (sh, 1)}                 # conv 3 feeds padded-layout conv 4
    ref = orc.run_net(net, w, b, x, perforation=perf).reshape(2, -1)
    r = gpu_run(net, w, b, x, "bf16", perforation=perf)
    assert r["net"].query_layer(3, 2)["a_mode"] == 2
    assert rel_err(r["out"], ref) <= TOL["bf16"] / 2
