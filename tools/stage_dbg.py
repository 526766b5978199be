"""Which output pixels of a staged first conv differ from the oracle (tf32)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
from oracle import oracle
from paper_conf_hpca_songhcl17_b200 import pcnn
prec = sys.argv[1] if len(sys.argv) > 1 else "tf32"
hw = 40
net = dict(in_shape=(3, hw, hw), layers=[
    dict(kind="conv", out=32, k=3, stride=1, pad=1, groups=1, relu=False, in_c=3),
    dict(kind="maxpool", k=1, stride=1)])
w, b = synth.net_params(net)
B = 2
x = synth.images(0, B, net["in_shape"], lo=-1, hi=1)
n = pcnn.Net(net, w, b, B, prec)
out, _, _ = n.infer(torch.from_numpy(x).cuda())
torch.cuda.synchronize()
got = out.cpu().numpy().reshape(B, 32, hw, hw)
ref = oracle.run_net(net, w, b, x).reshape(B, 32, hw, hw)
err = np.abs(got - ref)
print(prec, "max err", err.max(), "ref max", np.abs(ref).max(), "info", n.query_layer(0, B)["a_mode"], n.query_layer(0, B)["halo_in"])
bad = np.argwhere(err > 1e-2 * np.abs(ref).max())
print("bad count", len(bad))
if len(bad):
    print("channels", np.unique(bad[:, 1])[:40])
    print("rows", np.unique(bad[:, 2])[:50])
    print("cols", np.unique(bad[:, 3])[:50])
    print("images", np.unique(bad[:, 0]))
