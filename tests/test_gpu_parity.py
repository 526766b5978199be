"""Parity of the CUDA path (through the C ABI) against the FP64 oracle on the
same seeded inputs.  Tolerances from north_star (R10):
max|err|/max|ref| <= 1e-4 (FP32 SIMT), 5e-3 (TF32), 2e-2 (BF16); max-pool
bitwise; top-1 identical (margin-aware on iid inputs)."""
import numpy as np
import pytest

import synth
from tests.helpers import (FLAG_NO_LRN_POOL_FUSION, FLAG_NO_PADDED_LAYOUT,
                           FLAG_NO_SPACE_TO_DEPTH, TOL, conv_layer, gpu_run, params, rel_err,
                           small_inputs)

pytestmark = pytest.mark.gpu
PRECS = ["fp32", "tf32", "bf16"]


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_hpca_songhcl17_b200 import pcnn  # noqa: F401  (fails loudly if unbuilt)


# ------------------------------------------------------------ config 0 (CIFAR-quick)
@pytest.mark.parametrize("prec", PRECS)
def test_cifar_quick_config0(orc, prec):
    net = synth.cifar_quick()
    w, b = params(net)
    x = synth.images(0, 1, net["in_shape"], lo=-1, hi=1)
    ref = orc.run_net(net, w, b, x).reshape(1, -1)
    out = gpu_run(net, w, b, x, prec)["out"]
    assert rel_err(out, ref) <= TOL[prec]
    assert (out >= 0).all()


# ------------------------------------------------------------ layer-isolated conv
CONV_CASES = [
    # (out, k, in_c, stride, pad, groups, H, W, B)
    (16, 5, 3, 1, 2, 1, 32, 32, 1),        # configs[0] geometry
    (96, 11, 3, 4, 0, 1, 67, 67, 2),       # AlexNet conv1 geometry, smaller image
    (256, 5, 96, 1, 2, 2, 27, 27, 1),      # AlexNet conv2 (groups 2, C/g = 48)
    (384, 3, 256, 1, 1, 1, 13, 13, 3),     # conv3: ragged M (507 rows), N = 384
    (192, 3, 192, 1, 1, 2, 13, 13, 2),     # conv4-like, groups 2
    (64, 3, 64, 1, 1, 1, 20, 18, 2),       # VGG conv1_2-like, ragged tiles
    (40, 3, 16, 2, 1, 1, 17, 15, 3),       # N not a tile multiple, stride 2
    (128, 1, 64, 1, 0, 1, 9, 9, 2),        # 1x1 conv
]


# first-layer staging (a1): 3-channel inputs staged as im2col rows (S <= 5)
# or space-to-depth (strided S = 11), in bands of output rows -- sizes that
# span several bands with ragged last bands, checked element by element so a
# single wrong tap in one band row cannot hide under the max-relative metric
STAGE_CASES = [
    # (out, k, stride, pad, H, W, B)
    (32, 3, 1, 1, 40, 40, 3),
    (16, 5, 1, 2, 45, 37, 2),
    (96, 11, 4, 0, 67, 71, 2),
    (64, 3, 1, 1, 23, 224, 1),
]


@pytest.mark.parametrize("prec", PRECS)
@pytest.mark.parametrize("case", STAGE_CASES, ids=lambda c: "x".join(map(str, c)))
def test_first_layer_staging_elementwise(orc, prec, case):
    out_c, k, st, pad, H, W, B = case
    net = dict(in_shape=(3, H, W), layers=[conv_layer(out_c, k, 3, st, pad, 1, relu=False)])
    w, b = params(net, seed=41)
    x = small_inputs((3, H, W), B, lo=-1, hi=1)
    ref = orc.run_net(net, w, b, x).reshape(B, out_c, -1)
    out = gpu_run(net, w, b, x, prec)["out"].reshape(B, out_c, -1)
    scale = np.abs(ref).max()
    # per output pixel: the worst channel's error, relative to the layer scale
    per_pix = np.abs(out - ref).max(axis=1) / scale
    assert per_pix.max() <= TOL[prec] / 4, np.argwhere(per_pix > TOL[prec] / 4)[:8]


@pytest.mark.parametrize("prec", PRECS)
@pytest.mark.parametrize("case", CONV_CASES, ids=lambda c: "x".join(map(str, c)))
def test_conv_layer_parity(orc, prec, case):
    out_c, k, in_c, st, pad, g, H, W, B = case
    net = dict(in_shape=(in_c, H, W),
               layers=[conv_layer(out_c, k, in_c, st, pad, g, relu=False)])
    w, b = params(net, seed=31)
    x = small_inputs((in_c, H, W), B)
    ref = orc.run_net(net, w, b, x).reshape(B, -1)
    out = gpu_run(net, w, b, x, prec)["out"]
    assert rel_err(out, ref) <= TOL[prec] / 4


@pytest.mark.parametrize("prec", PRECS)
def test_fc_layer_parity_and_chw_flatten(orc, prec):
    # FC directly on a spatial input: columns permuted CHW -> HWC at create.
    net = dict(in_shape=(16, 3, 5), layers=[dict(kind="fc", out=40, in_f=16 * 15, relu=False)])
    w, b = params(net, seed=5)
    x = small_inputs((16, 3, 5), 5)
    ref = orc.run_net(net, w, b, x)
    out = gpu_run(net, w, b, x, prec)["out"]
    assert rel_err(out, ref) <= TOL[prec] / 4
    # single-column probe: only input element (c=7, h=2, w=1) matters
    wp = np.zeros_like(w[0])
    col = 7 * 15 + 2 * 5 + 1
    wp[:, col] = synth.round_to_bf16(np.linspace(-1, 1, 40))
    out = gpu_run(net, [wp], [np.zeros(40, np.float32)], x, prec)["out"]
    np.testing.assert_allclose(out, x[:, 7, 2, 1][:, None] * wp[:, col][None, :],
                               rtol=1e-2 if prec == "bf16" else 1e-6, atol=1e-6)


@pytest.mark.parametrize("prec", PRECS)
def test_maxpool_bitwise(orc, prec):
    net = dict(in_shape=(24, 27, 27), layers=[dict(kind="maxpool", k=3, stride=2)])
    x = small_inputs((24, 27, 27), 3, lo=-100, hi=100)
    ref = orc.run_net(net, [None], [None], x).reshape(3, -1)
    out = gpu_run(net, [None], [None], x, prec)["out"]
    np.testing.assert_array_equal(out, ref.astype(np.float32))


@pytest.mark.parametrize("prec", PRECS)
def test_avgpool(orc, prec):
    net = dict(in_shape=(16, 14, 14), layers=[dict(kind="avgpool", k=2, stride=2)])
    x = small_inputs((16, 14, 14), 2)
    ref = orc.run_net(net, [None], [None], x).reshape(2, -1)
    out = gpu_run(net, [None], [None], x, prec)["out"]
    assert rel_err(out, ref) <= TOL[prec] / 4


@pytest.mark.parametrize("prec", PRECS)
def test_lrn_parity(orc, prec):
    # Caffe-scale inputs make the LRN term O(1) (reading R3), C = 96 like norm1
    L = dict(kind="lrn", size=5, alpha=1e-4, beta=0.75, k=1.0)
    net = dict(in_shape=(96, 9, 7), layers=[L])
    x = small_inputs((96, 9, 7), 2, lo=-128, hi=128)
    ref = orc.run_net(net, [None], [None], x).reshape(2, -1)
    out = gpu_run(net, [None], [None], x, prec)["out"]
    assert rel_err(out, ref) <= TOL[prec] / 4
    assert np.abs(ref - x.reshape(2, -1)).max() > 1.0      # LRN is active


# ------------------------------------------------------------ softmax + entropy
def test_softmax_entropy_parity(orc):
    net = synth.cifar_quick()
    net = dict(in_shape=(8, 4, 4), layers=[dict(kind="fc", out=1000, in_f=128, relu=False)])
    w, b = params(net, seed=9)
    x = small_inputs((8, 4, 4), 6, lo=-30, hi=30)
    r = gpu_run(net, w, b, x, "fp32", probs=True)
    p_ref, h_ref = orc.softmax_entropy(r["out"].astype(np.float64))
    np.testing.assert_allclose(r["probs"], p_ref, rtol=2e-5, atol=1e-9)
    np.testing.assert_allclose(r["entropy"], h_ref, rtol=2e-5, atol=2e-6)
    np.testing.assert_allclose(r["probs"].sum(1), 1.0, rtol=1e-5)


# ------------------------------------------------------------ end to end
def _top1_agreement(out, ref, tol):
    top_g, top_r = out.argmax(1), ref.argmax(1)
    srt = np.sort(ref, axis=1)
    margin = srt[:, -1] - srt[:, -2]
    near_tie = margin < 2 * tol * np.abs(ref).max()
    agree = (top_g == top_r) | near_tie
    return agree.mean(), (top_g == top_r).mean()


@pytest.mark.parametrize("prec", PRECS)
def test_alexnet_end_to_end(orc, prec):
    net = synth.alexnet()
    w, b = params(net)
    B = 4
    x = synth.images(0, B, net["in_shape"])
    ref = orc.run_net(net, w, b, x)
    r = gpu_run(net, w, b, x, prec, probs=True)
    err = rel_err(r["out"], ref)
    assert err <= TOL[prec], err
    aware, raw = _top1_agreement(r["out"], ref, TOL[prec])
    assert aware == 1.0
    p_ref, h_ref = orc.softmax_entropy(ref)
    assert np.abs(r["entropy"] - h_ref).max() < 0.05 + 10 * err


@pytest.mark.parametrize("prec", ["tf32", "bf16"])
def test_vgg16_end_to_end(orc, prec):
    net = synth.vgg16()
    w, b = params(net)
    x = synth.images(0, 2, net["in_shape"])
    ref = orc.run_net(net, w, b, x)
    out = gpu_run(net, w, b, x, prec)["out"]
    assert rel_err(out, ref) <= TOL[prec]
    aware, _ = _top1_agreement(out, ref, TOL[prec])
    assert aware == 1.0


def test_infer_host_matches_device(orc):
    import torch
    from paper_conf_hpca_songhcl17_b200 import pcnn
    net = synth.alexnet()
    w, b = params(net)
    x = synth.images(0, 3, net["in_shape"])
    n = pcnn.Net(net, w, b, 4, "bf16")
    xd = torch.from_numpy(x).cuda()
    out, _, _ = n.infer(xd)
    torch.cuda.synchronize()
    xh = torch.from_numpy(x).pin_memory()
    oh = torch.empty((3, 1000)).pin_memory()
    n.infer_host(xh, oh)
    np.testing.assert_array_equal(oh.numpy(), out.cpu().numpy())


# ------------------------------------------------------------ layout transforms
@pytest.mark.parametrize("shape", [(96, 27, 27), (96, 55, 55), (256, 27, 27), (48, 19, 71)])
def test_fused_lrn_pool_bitwise_equals_unfused(orc, shape):
    """norm -> pool fusion changes scheduling only: the LRN output is rounded
    to the storage precision before the max in both paths.  The fused pair
    runs the register-only walk kernel (3 x 3 / 2 max pool; strips of 30
    columns, 71 -> 3 strips), the unfused one the LRN kernel + the pooling
    kernel: bitwise equal."""
    net = dict(in_shape=shape, layers=[
        dict(kind="lrn", size=5, alpha=1e-4, beta=0.75, k=1.0),
        dict(kind="maxpool", k=3, stride=2)])
    x = small_inputs(shape, 3, lo=-128, hi=128)
    for prec in PRECS:
        fr = gpu_run(net, [None, None], [None, None], x, prec)
        fused = fr["out"]
        pr = gpu_run(net, [None, None], [None, None], x, prec, flags=FLAG_NO_LRN_POOL_FUSION)
        plain = pr["out"]
        assert fr["net"].last_launch_count() + 1 == pr["net"].last_launch_count()
        np.testing.assert_array_equal(fused, plain)
        ref = orc.run_net(net, [None, None], [None, None], x).reshape(3, -1)
        assert rel_err(fused, ref) <= TOL[prec] / 4


@pytest.mark.parametrize("prec", PRECS)
def test_space_to_depth_first_conv(orc, prec):
    """The strided first conv runs as a space-to-depth 3x3/1 conv; the plain
    channel-padded path must agree with it and with the oracle."""
    net = dict(in_shape=(3, 51, 47), layers=[conv_layer(32, 11, 3, 4, 2, 1, relu=True)])
    w, b = params(net, seed=3)
    x = small_inputs((3, 51, 47), 2, lo=-128, hi=128)
    ref = orc.run_net(net, w, b, x).reshape(2, -1)
    s2d = gpu_run(net, w, b, x, prec)["out"]
    plain = gpu_run(net, w, b, x, prec, flags=FLAG_NO_SPACE_TO_DEPTH)["out"]
    assert rel_err(s2d, ref) <= TOL[prec] / 4
    assert rel_err(plain, ref) <= TOL[prec] / 4


@pytest.mark.parametrize("prec", ["tf32", "bf16"])
def test_conv_lrn_epilogue_fusion(orc, prec):
    """conv -> LRN fused in the tcgen05 epilogue (AlexNet conv1 + norm1 shape,
    smaller image, im2col mode so the fusion is on by default): agrees with
    the stand-alone LRN kernel path and the oracle.  The fused epilogue rounds
    the conv output to the storage precision exactly like the stored
    activation and then runs the LRN kernel's arithmetic, but the compiler
    contracts its squared sum into FMAs differently, so the two paths differ
    by last-place roundings of the storage format (R16: <= 2 ulp of
    max|y|, 2^-9 x 2 x 2 for BF16 and 2^-11 x 2 x 2 for TF32)."""
    net = dict(in_shape=(3, 67, 67), layers=[
        conv_layer(96, 11, 3, 4, 0, 1, relu=True),
        dict(kind="lrn", size=5, alpha=1e-4, beta=0.75, k=1.0),
        dict(kind="maxpool", k=3, stride=2)])
    w, b = params(net, seed=21)
    x = small_inputs((3, 67, 67), 2, lo=-128, hi=128)
    ref = orc.run_net(net, w, b, x).reshape(2, -1)
    fr = gpu_run(net, w, b, x, prec, flags=FLAG_NO_PADDED_LAYOUT)
    pr = gpu_run(net, w, b, x, prec, flags=FLAG_NO_PADDED_LAYOUT | FLAG_NO_LRN_POOL_FUSION)
    fused, plain = fr["out"], pr["out"]
    # the fusion really happened: the conv+LRN epilogue saves the LRN launch
    assert fr["net"].last_launch_count() < pr["net"].last_launch_count()
    assert fr["net"].query_layer(0, 2)["tile_n"] >= 96          # one N tile holds all channels
    assert rel_err(fused, ref) <= TOL[prec] / 4
    assert rel_err(plain, ref) <= TOL[prec] / 4
    ulp = 2.0 ** -8 if prec == "bf16" else 2.0 ** -10
    assert rel_err(fused, plain) <= 2 * ulp
    assert np.mean(fused == plain) > 0.99


@pytest.mark.parametrize("shape", [(96, 55, 55), (256, 27, 27), (64, 13, 11)])
def test_lrn_pool_kernel_shapes(orc, shape):
    """norm -> pool with the LRN window in registers (lane shuffles for the
    neighbouring chunks, swizzled smem for C = 256) against the oracle:
    AlexNet norm1 / norm2 shapes and a 6-chunk case."""
    net = dict(in_shape=shape, layers=[
        dict(kind="lrn", size=5, alpha=1e-4, beta=0.75, k=1.0),
        dict(kind="maxpool", k=3, stride=2)])
    x = small_inputs(shape, 2, lo=-128, hi=128)
    ref = orc.run_net(net, [None, None], [None, None], x).reshape(2, -1)
    for prec in PRECS:
        reg = gpu_run(net, [None, None], [None, None], x, prec)["out"]
        assert rel_err(reg, ref) <= TOL[prec] / 4


def test_infer_host_pipelined_chunks(orc):
    """AlexNet at B = 64 through pcnn_infer_host takes the pipelined path (4
    chunks, copies overlapping inference): bitwise the device call's logits
    (the FC K split is batch-independent and no conv layer splits K at 16
    images), and the oracle's tolerance."""
    import torch
    from paper_conf_hpca_songhcl17_b200 import pcnn
    net = synth.alexnet()
    w, b = params(net)
    B = 64
    x = synth.images(0, B, net["in_shape"])
    n = pcnn.Net(net, w, b, B, "bf16")
    dev, _, _ = n.infer(torch.from_numpy(x).cuda())
    torch.cuda.synchronize()
    xh = torch.from_numpy(x).pin_memory()
    oh = torch.empty((B, 1000)).pin_memory()
    hh = torch.empty((B,)).pin_memory()
    n.infer_host(xh, oh, None, hh)
    d = dev.cpu().numpy()
    np.testing.assert_array_equal(oh.numpy(), d)
    ref = orc.run_net(net, w, b, x[:2])
    assert rel_err(oh.numpy()[:2], ref) <= TOL["bf16"]
    assert np.isfinite(hh.numpy()).all() and (hh.numpy() >= 0).all()


@pytest.mark.parametrize("name,B", [("alexnet", 64), ("tiny", 3)])
def test_infer_host_u8_equals_device_call(orc, name, B):
    """pcnn_infer_host_u8 (8-bit pixels over PCIe, (pixel - mean) * scale on
    the device): bitwise the device call on the converted float images.
    AlexNet B = 64 takes the pipelined 4-chunk path and the 16-pixel vector
    conversion; the tiny net (H*W = 63) the scalar conversion."""
    import torch
    from paper_conf_hpca_songhcl17_b200 import pcnn
    if name == "alexnet":
        net = synth.alexnet()
        mean, scale = [128.0, 117.0, 104.0], 1.0
    else:
        net = dict(in_shape=(3, 9, 7), layers=[conv_layer(16, 3, 3, 1, 1, 1, relu=True)])
        mean, scale = [120.5, 100.25, 90.0], 0.5
    w, b = params(net)
    px = synth.pixels(0, B, net["in_shape"])
    x = ((px.astype(np.float32) - np.array(mean, np.float32)[None, :, None, None]) *
         np.float32(scale)).astype(np.float32)
    n = pcnn.Net(net, w, b, B, "bf16")
    dev, _, _ = n.infer(torch.from_numpy(x).cuda())
    torch.cuda.synchronize()
    ph = torch.from_numpy(px).pin_memory()
    oh = torch.empty(tuple(dev.shape)).pin_memory()
    n.infer_host_u8(ph, oh, mean=mean, scale=scale)
    np.testing.assert_array_equal(oh.numpy(), dev.cpu().numpy())
    ref = orc.run_net(net, w, b, x[:2]).reshape(2, -1)
    assert rel_err(oh.numpy()[:2].reshape(2, -1), ref) <= TOL["bf16"]


# ------------------------------------------------------------ bench configurations, full size
@pytest.mark.parametrize("name,B,samples", [("alexnet", 256, (0, 131, 255)), ("vgg16", 64, (0, 63))])
def test_bench_workload_sampled_parity(orc, name, B, samples):
    """The workloads bench.py times (AlexNet B = 256, VGG-16 B = 64, BF16, the
    same launch plan and CUDA graph): sampled images against the oracle one by
    one, and properties that hold for every image of the batch (finite logits,
    softmax rows summing to 1, entropy in [0, ln 1000])."""
    net = synth.get_net(name)
    w, b = params(net)
    x = synth.images(0, B, net["in_shape"])
    r = gpu_run(net, w, b, x, "bf16", probs=True)
    out, probs, ent = r["out"], r["probs"], r["entropy"]
    assert np.isfinite(out).all()
    assert np.abs(probs.sum(1) - 1.0).max() < 1e-4
    assert (ent >= -1e-5).all() and (ent <= np.log(1000) + 1e-4).all()
    for i in samples:
        ref = orc.run_net(net, w, b, x[i:i + 1])
        assert rel_err(out[i:i + 1], ref) <= TOL["bf16"], (name, i)


def test_vgg16_tf32_bench_batch_sampled(orc):
    """VGG-16 TF32 (configs[3]'s second precision) at the bench batch: one
    sampled image against the oracle within the TF32 tolerance."""
    net = synth.vgg16()
    w, b = params(net)
    x = synth.images(0, 64, net["in_shape"])
    out = gpu_run(net, w, b, x, "tf32")["out"]
    assert np.isfinite(out).all()
    ref = orc.run_net(net, w, b, x[17:18])
    assert rel_err(out[17:18], ref) <= TOL["tf32"]


@pytest.mark.parametrize("name,B,half", [("alexnet", 64, 16), ("vgg16", 16, 8)])
def test_per_image_logits_bitwise_batch_independent(name, B, half):
    """configs[4]'s requirement: an image's logits do
    not depend on how many images share its launch -- the FC K split is fixed
    by the layer shape and no conv splits K once a tile shape fills the GPU --
    so the per-rank shards B / W reproduce the W = 1 run bit for bit."""
    net = synth.get_net(name)
    w, b = params(net)
    x = synth.images(0, B, net["in_shape"])
    full = gpu_run(net, w, b, x, "bf16")["out"]
    part = gpu_run(net, w, b, x[half:2 * half], "bf16")["out"]
    np.testing.assert_array_equal(part, full[half:2 * half])
