import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np
from oracle import oracle as orc
from tests.helpers import conv_layer, gpu_run, params, small_inputs
for cg in ("1", "2"):
    os.environ["PCNN_FORCE_CG"] = cg
    net = dict(in_shape=(64, 20, 18), layers=[conv_layer(64, 3, 64, 1, 1, 1, relu=False)])
    w, b = params(net, seed=31)
    x = small_inputs((64, 20, 18), 2)
    ref = orc.run_net(net, w, b, x)            # [2, 64, 20, 18]
    r = gpu_run(net, w, b, x, "bf16")
    out = r["out"].reshape(2, 64, 20, 18)
    print("cg", cg, r["net"].query_layer(0, 2))
    bad = np.abs(out - ref) > 0.05 * np.abs(ref).max()
    idx = np.argwhere(bad)
    print("bad", bad.sum(), "of", bad.size)
    if len(idx):
        m = idx[:, 0] * 360 + idx[:, 2] * 18 + idx[:, 3]
        print(" rows m:", sorted(set(m.tolist()))[:40], "...", len(set(m.tolist())))
        print(" chans:", sorted(set(idx[:, 1].tolist())))
