"""C-ABI boundary checks that need no GPU: the library loads, exports every
symbol include/pcnn.h declares, does host-only shape/FLOP accounting right,
and fails loudly (no CPU fallback) when no B200 is present."""
import json
import os
import re

import numpy as np
import pytest

import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def pcnn():
    from paper_conf_hpca_songhcl17_b200 import build
    build.build()
    from paper_conf_hpca_songhcl17_b200 import pcnn as p
    return p


def _declared_symbols():
    with open(os.path.join(ROOT, "include", "pcnn.h")) as f:
        src = f.read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(pcnn_[a-z0-9_]+)\s*\(", src)))


def test_every_declared_symbol_is_exported(pcnn):
    lib = pcnn.library()
    decl = _declared_symbols()
    assert len(decl) >= 15
    for name in decl:
        assert hasattr(lib, name), name
    assert set(decl) == set(pcnn.EXPORTED)


def test_version_and_status_strings(pcnn):
    assert "sm_100a" in pcnn.version()
    lib = pcnn.library()
    assert lib.pcnn_status_string(0) == b"ok"
    assert lib.pcnn_status_string(6) == b"batch too large"


def test_describe_alexnet_table_iv_dims(pcnn):
    """T4: per-group GEMM dims of Table IV from the library's own
    shape inference: conv2 128 x 729 (K = 1200), conv5 128 x 169 (K = 1728)."""
    infos = pcnn.describe_net(synth.alexnet(), batch=1)
    convs = [i for i in infos if i["kind"] == pcnn.CONV]
    assert [(c["gemm_n"], c["gemm_m"]) for c in convs] == [
        (96, 3025), (128, 729), (384, 169), (192, 169), (128, 169)]
    assert convs[1]["gemm_k"] == 5 * 5 * 48 and convs[4]["gemm_k"] == 3 * 3 * 192
    assert [c["groups"] for c in convs] == [1, 2, 1, 2, 2]
    fc6 = infos[10]
    assert fc6["gemm_k"] == 9216 and fc6["gemm_n"] == 4096
    assert (infos[-1]["out_c"], infos[-1]["out_h"]) == (1000, 1)


def test_describe_vgg_multiplications_p14(pcnn):
    """VGGNet needs 1.5e10 multiplications per image (eq. 1: 2 FLOPs per MAC)."""
    with open(os.path.join(ROOT, "tests", "golden", "paper_pins.json")) as f:
        pin = json.load(f)["vgg_multiplications"]
    infos = pcnn.describe_net(synth.vgg16(), batch=1)
    mults = sum(i["flops"] for i in infos) / 2
    assert abs(mults - pin["value"]) / pin["value"] < pin["rel_tol"]
    # flops scale linearly with batch
    infos8 = pcnn.describe_net(synth.vgg16(), batch=8)
    assert abs(sum(i["flops"] for i in infos8) - 8 * 2 * mults) < 1.0


def test_describe_rejects_bad_shapes(pcnn):
    bad = dict(in_shape=(3, 8, 8), layers=[dict(kind="conv", out=4, k=11, stride=1, pad=0,
                                                groups=1, relu=True, in_c=3)])
    with pytest.raises(pcnn.PcnnError) as e:
        pcnn.describe_net(bad)
    assert e.value.status == 2     # PCNN_ERR_SHAPE
    bad2 = dict(in_shape=(3, 8, 8), layers=[dict(kind="conv", out=4, k=3, stride=1, pad=1,
                                                 groups=2, relu=True, in_c=3)])
    with pytest.raises(pcnn.PcnnError):
        pcnn.describe_net(bad2)


def test_create_net_fails_loudly_without_gpu(pcnn):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    net = synth.cifar_quick()
    w = [np.zeros((16, 3, 5, 5), np.float32), None]
    b = [np.zeros(16, np.float32), None]
    with pytest.raises(pcnn.PcnnError) as e:
        pcnn.Net(net, w, b, max_batch=1, precision="fp32")
    assert e.value.status == 5        # PCNN_ERR_CUDA: no silent CPU fallback
    assert pcnn.device_sm_count(0) == 0
