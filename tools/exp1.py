"""Experiments: (1) VGG prefix vs isolated conv1_2 timing, input scale;
(2) per-CTA K-block cycles vs SM budget (chip-L2 vs per-SM operand limit)."""
import ctypes, os, sys
os.environ["PCNN_TC_PROFILE"] = os.environ.get("PCNN_TC_PROFILE", "0")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
from paper_conf_hpca_songhcl17_b200 import pcnn
from tools.one_layer import make_net


def timed(net, B, lo, hi, budget=None, li=None, reps=20):
    w, b = synth.net_params(net)
    n = pcnn.Net(net, w, b, B, "bf16")
    if budget:
        n.set_sm_budget(li, budget)
    x = torch.from_numpy(synth.images(0, B, net["in_shape"], lo=lo, hi=hi)).cuda()
    n.set_layer_timing(True)
    for _ in range(reps):
        n.infer(x)
    torch.cuda.synchronize()
    ms, k = n.read_layer_timing()
    n.close()
    return [round(v / k, 4) for v in ms]


vgg = synth.vgg16()
pre = dict(in_shape=vgg["in_shape"], layers=vgg["layers"][:3])
print("vgg prefix (conv1_1, conv1_2, pool1) +-128:", timed(pre, 64, -128, 128))
print("vgg prefix +-1:", timed(pre, 64, -1, 1))
_, net, li = make_net("vgg1_2+pm")
print("vgg1_2+pm +-1:", timed(net, 64, -1, 1))
print("vgg1_2+pm +-128:", timed(net, 64, -128, 128))
for name, B in (("conv3", 256), ("vgg3_2+pm", 64), ("conv2", 256)):
    _, net, li = make_net(name)
    for bud in (148, 74, 36):
        t = timed(net, B, -1, 1, budget=bud, li=li)
        print("%s budget %d: %s  (x budget/148 = %.4f)" % (name, bud, t, t[li] * bud / 148))
