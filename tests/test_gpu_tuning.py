"""Entropy-guided greedy tuning + calibration (Fig. 12, eq. 14) on
the GPU: every candidate runs through libpcnn's kernels, its time from CUDA
events and CNN_entropy (eq. 2) from the fused softmax + entropy kernel."""
import math

import numpy as np
import pytest
import torch

import synth
from tests.helpers import params

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


def test_greedy_tuning_on_alexnet():
    from paper_conf_hpca_songhcl17_b200 import pcnn, tuning
    net = synth.alexnet()
    w, b = params(net)
    B = 32
    x = torch.from_numpy(synth.images(0, B, net["in_shape"])).cuda()
    n = pcnn.Net(net, w, b, B, "bf16")
    ladders = {3: [("exact",), ("rank", 64), ("perf", 2, 1)],
               6: [("exact",), ("rank", 192), ("rank", 96)],
               8: [("exact",), ("perf", 2, 1)]}
    measure = tuning.gpu_measure(n, ladders, x, reps=5)
    t0, h0 = measure({3: 0, 6: 0, 8: 0})
    threshold = h0 + 10.0          # permissive: every eligible rung may be taken
    path = tuning.greedy_tune(ladders, measure, threshold)
    assert path[0]["state"] == {3: 0, 6: 0, 8: 0}
    for a, c in zip(path, path[1:]):
        # one layer moves one rung per iteration, and only faster candidates
        diff = [l for l in ladders if c["state"][l] != a["state"][l]]
        assert len(diff) == 1 and c["state"][diff[0]] == a["state"][diff[0]] + 1
        assert c["time"] < a["time"] and c["entropy"] <= threshold
        assert c["te"] == math.inf or c["te"] > 0
    # calibration on the resulting path, re-measuring the entropy of
    # the inputs at every back-track step: a permissive threshold keeps the
    # current table after one measurement; a threshold below every table's
    # measured entropy walks back to the exact table, measuring each
    last = len(path) - 1
    observe = tuning.gpu_observe(n, ladders, path, x)
    idx, trace = tuning.calibrate(path, last, observe, threshold)
    assert idx == last and len(trace) == 1
    idx, trace = tuning.calibrate(path, last, observe, -1.0)
    assert idx == 0 and [t[0] for t in trace] == list(range(last, -1, -1))
    # the measured entropies reproduce the tuning-time ones (same inputs)
    for i, h in trace:
        assert abs(h - path[i]["entropy"]) < 1e-4
    # the tuned state programs the net and still infers finite probabilities
    tuning.apply_state(n, ladders, path[-1]["state"], batch=B)
    out, p, h = n.infer(x, probs=True, entropy=True)
    torch.cuda.synchronize()
    assert np.isfinite(out.cpu().numpy()).all()
    assert np.allclose(p.cpu().numpy().sum(1), 1.0, atol=1e-4)
