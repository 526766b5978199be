"""The weight-streaming FC kernel (kernels_fc.cu, a6) against the FP64
oracle: every precision, ragged N (not a multiple of 128), batches from 1 to
past one 256-image chunk, K splits in a CTA cluster; bitwise invariance of an
image's outputs under the batch size and the SM budget (the K split depends
on the layer shape only)."""
import numpy as np
import pytest

import synth
from tests.helpers import TOL, gpu_run, rel_err

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


def fc_net(c, h, w, n_out, relu):
    return dict(name="fc", in_shape=(c, h, w), layers=[
        dict(kind="fc", out=n_out, in_f=c * h * w, relu=relu, name="fc")])


def _params(net, seed):
    return synth.net_params(net, seed=seed)


CASES = [
    # (C, H, W, N, B, relu)
    (256, 6, 6, 4096, 3, True),      # AlexNet fc6 shape, 8-way K split
    (64, 8, 8, 1000, 17, False),     # fc8-like ragged N, ragged batch
    (512, 1, 1, 100, 1, False),      # N < 128, one image
    (128, 2, 2, 384, 300, True),     # two 150-image chunks
]


@pytest.mark.parametrize("case", CASES)
@pytest.mark.parametrize("prec", ["bf16", "tf32"])
def test_fc_kernel_parity(orc, case, prec):
    c, h, w, n, B, relu = case
    net = fc_net(c, h, w, n, relu)
    wt, bs = _params(net, seed=40 + n)
    x = synth.images(0, B, net["in_shape"], lo=-2, hi=2)
    r = gpu_run(net, wt, bs, x, prec)
    info = r["net"].query_layer(0, B)
    assert info["a_mode"] == 3                          # the FC weight-stream kernel
    ref = orc.run_net(net, wt, bs, x)
    assert rel_err(r["out"], ref) <= TOL[prec] / 4
    if relu:
        assert (r["out"] >= 0).all()


def test_fc_kernel_batch_and_budget_bitwise():
    net = fc_net(256, 6, 6, 4096, True)
    wt, bs = _params(net, seed=7)
    x = synth.images(0, 300, net["in_shape"], lo=-2, hi=2)
    big = gpu_run(net, wt, bs, x, "bf16")
    assert big["net"].query_layer(0, 300)["splits"] > 1
    for sl in (slice(0, 1), slice(5, 22), slice(40, 296)):
        part = gpu_run(net, wt, bs, x[sl], "bf16")["out"]
        np.testing.assert_array_equal(part, big["out"][sl])
    for n_sms in (8, 37):
        r = gpu_run(net, wt, bs, x[:64], "bf16", budgets={0: (n_sms, 0)}, census=True)
        np.testing.assert_array_equal(r["out"], big["out"][:64])
        assert 0 < len(r["census"][0]) <= max(n_sms, 2 * big["net"].query_layer(0, 300)["splits"])


def test_alexnet_fc_layers_parity_b256(orc):
    """fc6 -> fc7 -> fc8 at the bench batch (256 images, one chunk, two
    accumulators per CTA): sampled images against the oracle."""
    net = dict(name="fc678", in_shape=(256, 6, 6), layers=[
        dict(kind="fc", out=4096, in_f=9216, relu=True, name="fc6"),
        dict(kind="fc", out=4096, in_f=4096, relu=True, name="fc7"),
        dict(kind="fc", out=1000, in_f=4096, relu=False, name="fc8")])
    wt, bs = synth.net_params(net, seed=11)
    x = synth.images(0, 256, net["in_shape"], lo=0, hi=4)
    r = gpu_run(net, wt, bs, x, "bf16")
    assert r["net"].query_layer(0, 256)["tile_m"] == 256
    idx = [0, 77, 255]
    ref = orc.run_net(net, wt, bs, x[idx])
    assert rel_err(r["out"][idx], ref) <= TOL["bf16"] / 2
