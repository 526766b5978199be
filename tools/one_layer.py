"""Run one AlexNet/VGG layer shape in isolation (for ncu / timing).
    python tools/one_layer.py conv3 [batch] [reps] [precision]
"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
from paper_conf_hpca_songhcl17_b200 import pcnn

SHAPES = {  # name: (in_shape, layer)
    "conv1": ((3, 227, 227), dict(kind="conv", out=96, k=11, stride=4, pad=0, groups=1, relu=True, in_c=3)),
    "conv2": ((96, 27, 27), dict(kind="conv", out=256, k=5, stride=1, pad=2, groups=2, relu=True, in_c=96)),
    "conv3": ((256, 13, 13), dict(kind="conv", out=384, k=3, stride=1, pad=1, groups=1, relu=True, in_c=256)),
    "conv4": ((384, 13, 13), dict(kind="conv", out=384, k=3, stride=1, pad=1, groups=2, relu=True, in_c=384)),
    "conv5": ((384, 13, 13), dict(kind="conv", out=256, k=3, stride=1, pad=1, groups=2, relu=True, in_c=384)),
    "vgg3_2": ((256, 56, 56), dict(kind="conv", out=256, k=3, stride=1, pad=1, groups=1, relu=True, in_c=256)),
    "vgg4_2": ((512, 28, 28), dict(kind="conv", out=512, k=3, stride=1, pad=1, groups=1, relu=True, in_c=512)),
    "fc6": ((256, 6, 6), dict(kind="fc", out=4096, in_f=9216, relu=True)),
    "fc7": ((4096, 1, 1), dict(kind="fc", out=4096, in_f=4096, relu=True)),
    "fc8": ((4096, 1, 1), dict(kind="fc", out=1000, in_f=4096, relu=False)),
    "conv2p": ((128, 27, 27), dict(kind="conv", out=256, k=5, stride=1, pad=2, groups=2, relu=True, in_c=128)),
    "conv1p": ((64, 57, 57), dict(kind="conv", out=96, k=3, stride=1, pad=0, groups=1, relu=True, in_c=64)),
    "conv1s": ((48, 57, 57), dict(kind="conv", out=96, k=3, stride=1, pad=0, groups=1, relu=True, in_c=48)),
    "vgg1_2": ((64, 224, 224), dict(kind="conv", out=64, k=3, stride=1, pad=1, groups=1, relu=True, in_c=64)),
    "vgg1_1s": ((32, 224, 224), dict(kind="conv", out=64, k=1, stride=1, pad=0, groups=1, relu=True, in_c=32)),
    "rank2": ((128, 27, 27), dict(kind="conv", out=256, k=1, stride=1, pad=0, groups=2, relu=True, in_c=128)),
    "vgg2_2": ((128, 112, 112), dict(kind="conv", out=128, k=3, stride=1, pad=1, groups=1, relu=True, in_c=128)),
    "vgg5_2": ((512, 14, 14), dict(kind="conv", out=512, k=3, stride=1, pad=1, groups=1, relu=True, in_c=512)),
    "norm1pool1": ((96, 55, 55), [dict(kind="lrn", size=5, alpha=1e-4, beta=0.75, k=1.0), dict(kind="maxpool", k=3, stride=2)]),
    "pool5": ((256, 13, 13), dict(kind="maxpool", k=3, stride=2)),
    "norm2pool2": ((256, 27, 27), [dict(kind="lrn", size=5, alpha=1e-4, beta=0.75, k=1.0), dict(kind="maxpool", k=3, stride=2)]),
    "stage": ((3, 227, 227), dict(kind="maxpool", k=1, stride=1)),
}
def make_net(name):
    """name[+pm]: '+pm' wraps the conv between identity pools so the runtime
    may choose the padded-layout mode (it needs pool / pm-conv neighbours).
    'alexnet_head': AlexNet's conv1 -> norm1 -> pool1 as the full net runs them
    (space-to-depth staging, padded-layout conv1)."""
    if name == "alexnet_head":
        import synth
        net = synth.alexnet()
        return net["in_shape"], dict(in_shape=net["in_shape"], layers=net["layers"][:3]), 0
    wrap = name.endswith("+pm")
    shape, L = SHAPES[name[:-3] if wrap else name]
    layers = L if isinstance(L, list) else [L]
    if wrap:
        ident = dict(kind="maxpool", k=1, stride=1)
        layers = [ident] + layers + [ident]
    return shape, dict(in_shape=shape, layers=layers), (1 if wrap else 0)


def main():
    name = sys.argv[1]
    B = int(sys.argv[2]) if len(sys.argv) > 2 else 256
    reps = int(sys.argv[3]) if len(sys.argv) > 3 else 20
    prec = sys.argv[4] if len(sys.argv) > 4 else "bf16"
    shape, net, li = make_net(name)
    w, b = synth.net_params(net)
    n = pcnn.Net(net, w, b, B, prec)
    x = torch.from_numpy(synth.images(0, B, shape, lo=-1, hi=1)).cuda()
    n.set_layer_timing(True)
    for _ in range(reps):
        n.infer(x)
    torch.cuda.synchronize()
    ms, k = n.read_layer_timing()
    info = n.query_layer(li, B)
    t = sum(ms) / k
    if li:
        print("  per layer ms:", [round(v / k, 4) for v in ms], "a_mode", info.get("a_mode"))
    byt = sum(n.query_layer(i, B)["bytes"] for i in range(len(net["layers"])))
    print("%s B=%d %s: %.4f ms  %.1f TFLOP/s  %.0f GB/s  tile %dx%d grid %d splits %d" % (
        name, B, prec, t, info["flops"] / t / 1e9, byt / t / 1e6, info["tile_m"], info["tile_n"],
        info["grid"], info["splits"]))


if __name__ == "__main__":
    main()
