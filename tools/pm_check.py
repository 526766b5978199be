"""Padded-layout (shifted-window) conv mode vs the oracle on a small VGG-like
net, with and without PCNN_NO_PM (quick GPU check; the pytest version lives in
tests/test_gpu_parity.py)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import synth
from oracle import oracle as orc
from tests.helpers import TOL, conv_layer, gpu_run, params, rel_err, small_inputs

net = dict(in_shape=(3, 40, 40), layers=[
    conv_layer(64, 3, 3, 1, 1), conv_layer(64, 3, 64, 1, 1), dict(kind="maxpool", k=2, stride=2),
    conv_layer(128, 3, 64, 1, 1), conv_layer(128, 3, 128, 1, 1), dict(kind="maxpool", k=2, stride=2),
    dict(kind="fc", out=16, in_f=128 * 10 * 10, relu=False)])
w, b = params(net, seed=21)
x = small_inputs((3, 40, 40), 3, lo=-128, hi=128)
ref = orc.run_net(net, w, b, x).reshape(3, -1)
for prec in sys.argv[1:] or ["bf16", "tf32"]:
    r = gpu_run(net, w, b, x, prec)
    modes = [(r["net"].query_layer(i, 3)["a_mode"], r["net"].query_layer(i, 3)["halo_in"],
              r["net"].query_layer(i, 3)["halo_out"]) for i in range(len(net["layers"]))]
    print(prec, "modes/halos", modes, "err %.3g (tol %g)" % (rel_err(r["out"], ref), TOL[prec]))
