"""Per-layer time of AlexNet's variants (exact / rank-r / perforated) at one
batch, live CUDA events:  python tools/variant_layers.py [B]"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import synth  # noqa: E402
from paper_conf_hpca_songhcl17_b200 import pcnn  # noqa: E402

B = int(sys.argv[1]) if len(sys.argv) > 1 else 256
net = synth.alexnet()
w, b = synth.net_params(net)
x = torch.from_numpy(synth.images(0, B, net["in_shape"])).cuda()
names = [L.get("name", str(i)) for i, L in enumerate(net["layers"])]
for label, setup in [("exact", {}), ("rank conv2=64", {"rank": {3: 64}}),
                     ("rank conv2=32 conv3=96", {"rank": {3: 32, 6: 96}}),
                     ("perf conv2 2x2", {"perf": {3: (2, 2)}}),
                     ("perf conv2 2x1", {"perf": {3: (2, 1)}}),
                     ("perf conv2-5 2x1", {"perf": {3: (2, 1), 6: (2, 1), 7: (2, 1), 8: (2, 1)}}),
                     ("perf conv2-5 3x1", {"perf": {3: (3, 1), 6: (3, 1), 7: (3, 1), 8: (3, 1)}}),
                     ("perf conv3 2x2", {"perf": {6: (2, 2)}})]:
    n = pcnn.Net(net, w, b, B, "bf16")
    for i, r in setup.get("rank", {}).items():
        n.set_variant(i, "rank", r)
    for i, st in setup.get("perf", {}).items():
        n.set_perforation(i, *st)
    n.infer(x)
    torch.cuda.synchronize()
    n.set_layer_timing(True)
    for _ in range(20):
        n.infer(x)
    torch.cuda.synchronize()
    ms, k = n.read_layer_timing()
    sel = [3, 4, 6, 7]
    print("%-24s total %.4f ms | %s" % (label, sum(ms) / k, "  ".join(
        "%s %.4f" % (names[i], ms[i] / k) for i in sel)))
    for i in (3, 6):
        f = n.query_layer(i, B)
        print("     %s plan: tile %dx%d grid %d splits %d a_mode %d flops %.3g" % (
            names[i], f["tile_m"], f["tile_n"], f["grid"], f["splits"], f["a_mode"], f["flops"]))
    n.close()
