"""Quick GPU probe: one conv / FC layer per engine variant vs the oracle.
    PCNN_FORCE_CG=2 python tools/probe_tc.py
"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import synth
from oracle import oracle as orc
from tests.helpers import conv_layer, gpu_run, params, rel_err, small_inputs

cases = [(64, 3, 64, 1, 1, 1, 20, 18, 2), (256, 5, 96, 1, 2, 2, 27, 27, 1),
         (384, 3, 256, 1, 1, 1, 13, 13, 3)]
for prec in sys.argv[1:] or ["bf16", "tf32"]:
    for c in cases:
        out_c, k, in_c, st, pad, g, H, W, B = c
        net = dict(in_shape=(in_c, H, W), layers=[conv_layer(out_c, k, in_c, st, pad, g, relu=False)])
        w, b = params(net, seed=31)
        x = small_inputs((in_c, H, W), B)
        ref = orc.run_net(net, w, b, x).reshape(B, -1)
        t = time.time()
        r = gpu_run(net, w, b, x, prec)
        print(prec, c, "err %.3g" % rel_err(r["out"], ref), r["net"].query_layer(0, B), "%.2fs" % (time.time() - t), flush=True)
