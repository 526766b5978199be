import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth
from oracle import oracle as orc
from tests.helpers import gpu_run, rel_err
net = dict(name="conv_fc", in_shape=(64, 9, 9), layers=[
    dict(kind="conv", out=64, k=3, stride=1, pad=1, groups=1, relu=True, in_c=64, name="c"),
    dict(kind="fc", out=96, in_f=64 * 9 * 9, relu=False, name="f")])
w, b = synth.net_params(net, bf16=False)
x = synth.images(0, 3, net["in_shape"], lo=-1.0, hi=1.0, bf16=False)
for prec in ("bf16", "tf32", "fp32"):
    conv = dict(net, layers=net["layers"][:1])
    r = gpu_run(conv, w[:1], b[:1], x, prec)
    ref = orc.run_net(conv, w[:1], b[:1], x).reshape(3, -1)
    q = r["net"].query_layer(0, 3)
    print(prec, "conv only", rel_err(r["out"], ref), q["a_mode"], q["tile_m"], q["tile_n"], q["splits"], q["halo_in"], q["halo_out"])
    fc = dict(name="fc", in_shape=(64, 9, 9), layers=net["layers"][1:])
    r = gpu_run(fc, w[1:], b[1:], x, prec)
    ref = orc.run_net(fc, w[1:], b[1:], x)
    q = r["net"].query_layer(0, 3)
    print(prec, "fc only", rel_err(r["out"], ref), q["splits"], q["tile_n"])
    r = gpu_run(net, w, b, x, prec)
    ref = orc.run_net(net, w, b, x)
    print(prec, "both", rel_err(r["out"], ref), [r["net"].query_layer(i, 3)["splits"] for i in range(2)])
