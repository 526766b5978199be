"""NEXT-3 time model (eq. 12 on B200; R12): the
library's t = t_launch + nInvocations(n) x t_unit against measured per-layer
latency (live CUDA events, the same measurement the fit used) on n SMs and a
few batches; eq. 11's optSM keeps the modelled time."""
import numpy as np
import pytest
import torch

import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


def _layer_times(n, x, reps=10):
    n.infer(x)
    torch.cuda.synchronize()
    n.set_layer_timing(True)
    for _ in range(reps):
        n.infer(x)
    torch.cuda.synchronize()
    ms, k = n.read_layer_timing()
    n.set_layer_timing(False)
    return [m / k * 1000.0 for m in ms]


def test_eq12_model_tracks_measured_latency():
    from paper_conf_hpca_songhcl17_b200 import pcnn
    net = synth.alexnet()
    w, b = synth.net_params(net)
    gemm = [i for i, L in enumerate(net["layers"]) if L["kind"] in ("conv", "fc")]
    rel = []
    for B in (1, 64):
        x = torch.from_numpy(synth.images(0, B, net["in_shape"])).cuda()
        prev = None
        for nb in (18, 74, 148):
            n = pcnn.Net(net, w, b, B, "bf16")
            for i in gemm:
                n.set_sm_budget(i, nb, 0)
            t = _layer_times(n, x)
            model = [n.model_layer_time(i, B, nb) for i in gemm]
            for i, m in zip(gemm, model):
                rel.append(abs(m - t[i]) / t[i])
            if prev is not None:   # fewer SMs never model faster
                assert all(p >= m - 1e-9 for p, m in zip(prev, model))
            prev = model
            # eq. 11: optSM keeps nInvocations, hence the modelled time
            for i in gemm:
                bp = n.plan_budget(i, B)
                assert abs(n.model_layer_time(i, B, bp["opt_sm"]) - bp["t_model_us"]) < 1e-6
            n.close()
    rel = np.array(rel)
    assert np.median(rel) < 0.15, np.median(rel)
    assert (rel <= 0.25).mean() >= 0.8, (rel <= 0.25).mean()
