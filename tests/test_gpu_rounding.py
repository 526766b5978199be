"""Operand rounding of the CUDA path on values that are NOT BF16-representable
(R9).  Everywhere else the seeded inputs and weights are generated
BF16-representable so every precision sees identical operands; here they are
full FP32 values, so the path's own rounding is exercised:

* input staging: BF16 round-to-nearest-even / TF32 round-to-nearest (ties
  away, `cvt.rna.tf32`),
* weight packing at pcnn_create_net (same rules, on the host),
* the conv epilogue's rounding of stored activations.

Two checks per precision:
1. north_star: the end-to-end AlexNet error against the FP64 oracle on the
   raw FP32 operands is within the precision's tolerance;
2. sharp: a conv -> fc net matches the FP64 oracle run on operands rounded by
   the R9 rule (and with the stored conv activations rounded the same way) to
   accumulation-order accuracy -- far tighter than the difference that
   truncation instead of rounding makes (negative control below).
"""
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


def rna_tf32(a):
    """TF32 round to nearest, ties away from zero (reading R9)."""
    u = np.ascontiguousarray(np.asarray(a, dtype=np.float32)).view(np.uint32).astype(np.uint64)
    u = ((u + np.uint64(0x1000)) & np.uint64(0xFFFFE000)).astype(np.uint32)
    return u.view(np.float32)


def trunc_bf16(a):
    u = np.ascontiguousarray(np.asarray(a, dtype=np.float32)).view(np.uint32)
    return (u & np.uint32(0xFFFF0000)).view(np.float32)


def trunc_tf32(a):
    u = np.ascontiguousarray(np.asarray(a, dtype=np.float32)).view(np.uint32)
    return (u & np.uint32(0xFFFFE000)).view(np.float32)


ROUND = {"bf16": synth.round_to_bf16, "tf32": rna_tf32, "fp32": lambda a: np.asarray(a, np.float32)}
TRUNC = {"bf16": trunc_bf16, "tf32": trunc_tf32}
# accumulation-order bound of the sharp check: K <= 1024 FP32 products
SHARP = {"bf16": 2e-4, "tf32": 2e-4, "fp32": 2e-5}


def _conv_fc_net():
    return dict(name="conv_fc", in_shape=(64, 9, 9), layers=[
        dict(kind="conv", out=64, k=3, stride=1, pad=1, groups=1, relu=True, in_c=64, name="c"),
        dict(kind="fc", out=96, in_f=64 * 9 * 9, relu=False, name="f"),
    ])


def _raw_params(net):
    w, b = synth.net_params(net, bf16=False)
    x = synth.images(0, 3, net["in_shape"], lo=-1.0, hi=1.0, bf16=False)
    assert (synth.round_to_bf16(x) != x).mean() > 0.9      # really not BF16-representable
    assert (synth.round_to_bf16(w[0]) != w[0]).mean() > 0.9
    return w, b, x


def _oracle_rounded(orc, net, w, b, x, rnd):
    """FP64 oracle on R9-rounded operands, stored conv activations rounded."""
    L0, L1 = net["layers"]
    y = orc.conv2d(rnd(x), rnd(w[0]), b[0], L0["stride"], L0["pad"], 1, True)
    y = rnd(y).astype(np.float64)
    return orc.fc(y, rnd(w[1]), b[1], False)


@pytest.mark.parametrize("prec", ["bf16", "tf32", "fp32"])
def test_operand_rounding_sharp(orc, prec):
    net = _conv_fc_net()
    w, b, x = _raw_params(net)
    out = gpu_run(net, w, b, x, prec)["out"]
    ref = _oracle_rounded(orc, net, w, b, x, ROUND[prec])
    e = rel_err(out, ref)
    assert e <= SHARP[prec], e
    if prec in TRUNC:
        # negative control: truncating instead of rounding moves the result
        # by much more than the sharp bound, so a truncation bug would fail
        bad = _oracle_rounded(orc, net, w, b, x, TRUNC[prec])
        assert rel_err(bad, ref) > 5 * SHARP[prec]


@pytest.mark.parametrize("prec", ["bf16", "tf32"])
def test_alexnet_full_fp32_operands_within_tolerance(orc, prec):
    net = synth.alexnet()
    w, b = synth.net_params(net, bf16=False)
    x = synth.images(0, 2, net["in_shape"], bf16=False)
    out = gpu_run(net, w, b, x, prec)["out"]
    ref = orc.run_net(net, w, b, x)
    assert rel_err(out, ref) <= TOL[prec]
    # top-1 where the oracle's margin is outside the tolerance band (R10)
    srt = np.sort(ref, axis=1)
    clear = (srt[:, -1] - srt[:, -2]) > 2 * TOL[prec] * np.abs(ref).max()
    assert (out.argmax(1)[clear] == ref.argmax(1)[clear]).all()
