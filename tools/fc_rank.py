"""FC rank-r on AlexNet (configs[2] ladder extended to the classifier, where
P:429 puts most parameters): randomized top-r SVD factors of fc6 / fc7 from
numpy, installed through pcnn_set_variant_factors; per-layer time, img/s and
logit error / top-1 agreement against the exact CUDA path.
    python tools/fc_rank.py [B]"""
import json
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import synth  # noqa: E402
from paper_conf_hpca_songhcl17_b200 import pcnn  # noqa: E402

B = int(sys.argv[1]) if len(sys.argv) > 1 else 256
net = synth.alexnet()
w, b = synth.net_params(net)
names = [L.get("name", str(i)) for i, L in enumerate(net["layers"])]
fc = [i for i, L in enumerate(net["layers"]) if L["kind"] == "fc"]
x = torch.from_numpy(synth.images(0, B, net["in_shape"])).cuda()
rng = np.random.default_rng(0)


def top_r(W, r, iters=2):
    """Randomized range finder + small SVD (Halko et al.)."""
    Q = np.linalg.qr(W @ rng.standard_normal((W.shape[1], r + 16)))[0]
    for _ in range(iters):
        Q = np.linalg.qr(W @ (W.T @ Q))[0]
    Ub, S, Vt = np.linalg.svd(Q.T @ W, full_matrices=False)
    return (Q @ Ub)[:, :r] * S[:r], Vt[:r]


def run(ranks):
    n = pcnn.Net(net, w, b, B, "bf16")
    for i, r in ranks.items():
        A, Bf = top_r(np.asarray(w[i], dtype=np.float64), r)
        n.set_variant_factors(i, r, A, Bf)
    out, _, _ = n.infer(x)
    torch.cuda.synchronize()
    n.set_layer_timing(True)
    for _ in range(20):
        n.infer(x)
    torch.cuda.synchronize()
    ms, k = n.read_layer_timing()
    n.set_layer_timing(False)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(30):
        n.infer(x)
    e1.record()
    torch.cuda.synchronize()
    res = {"ranks": {names[i]: r for i, r in ranks.items()},
           "img_s": round(B * 30 / (e0.elapsed_time(e1) / 1000), 1),
           "fc_ms": {names[i]: round(ms[i] / k, 5) for i in fc},
           "fc_flops": {names[i]: n.query_layer(i, B)["flops"] for i in fc}}
    n.close()
    return res, out.cpu().numpy()


base, y0 = run({})
rows = [base]
for ranks in ({10: 512}, {10: 512, 11: 512}, {10: 256, 11: 256}, {10: 128, 11: 128}):
    r, y = run(ranks)
    r["err_vs_exact"] = float(np.abs(y - y0).max() / np.abs(y0).max())
    r["top1_agree_exact"] = float((y.argmax(1) == y0.argmax(1)).mean())
    rows.append(r)
print(json.dumps({"net": "alexnet", "batch": B, "precision": "bf16", "rows": rows}, indent=1))
