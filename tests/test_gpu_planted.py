"""Top-1 on the planted-class set (SURVEY.md §8(d) / DESIGN.md R10), where
top-1 is meaningful: images are noisy copies of class prototypes and fc8's
first rows are the normalised, centred FP64 fc7 features of those
prototypes (built here by the oracle).  north_star: identical top-1 on
>= 99.9% of images -- with 64 images that is all of them."""
import numpy as np
import pytest
import torch

import synth
from tests.helpers import TOL, gpu_run, params, rel_err

pytestmark = pytest.mark.gpu
N_CLASSES = 100


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


@pytest.fixture(scope="module")
def planted(orc):
    net = synth.alexnet()
    w, b = params(net)
    protos = synth.prototypes(N_CLASSES, net["in_shape"])
    _, outs = orc.run_net(net, w, b, protos, return_all=True)
    feats = np.asarray(outs[-2], dtype=np.float64)          # fc7 output [n, 4096]
    mean = feats.mean(0)
    F = feats - mean
    F /= np.linalg.norm(F, axis=1, keepdims=True)
    W8 = 0.1 * np.asarray(w[-1], dtype=np.float64)
    W8[:N_CLASSES] = F
    w = list(w)
    b = list(b)
    w[-1] = synth.round_to_bf16(W8)
    b[-1] = synth.round_to_bf16(-(W8 @ mean))
    return net, w, b


@pytest.mark.parametrize("prec", ["bf16", "tf32"])
def test_planted_top1(orc, planted, prec):
    net, w, b = planted
    x, labels = synth.planted_images(0, 64, net["in_shape"], N_CLASSES)
    out = gpu_run(net, w, b, x, prec)["out"]
    top1 = out.argmax(1)
    assert (top1 == labels).mean() >= 0.999, (top1 != labels).sum()
    ref = orc.run_net(net, w, b, x[:8])
    assert (ref.argmax(1) == labels[:8]).all()
    assert (top1[:8] == ref.argmax(1)).all()
    assert rel_err(out[:8], ref) <= TOL[prec]
