"""NEXT-3 (eq. 12): measure every AlexNet GEMM layer's latency
(live CUDA events, one launch per layer) on n SMs for n in {8, 18, 37, 74,
148} at B in {1, 64, 256}, next to the library's eq. 12 model
t = t_launch + nInvocations(n) x t_unit, and fit the two constants per kernel
class (tcgen05 conv, weight-streaming FC) by least squares on the relative
error.  Writes one JSON document (stdout) with the raw points, the fitted
constants and the relative errors of the model as compiled in.

    python tools/time_model_fit.py > profiles/r02_time_model_fit.json
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_songhcl17_b200 import pcnn  # noqa: E402

net = synth.alexnet()
w, b = synth.net_params(net)
names = [L.get("name", str(i)) for i, L in enumerate(net["layers"])]
gemm = [i for i, L in enumerate(net["layers"]) if L["kind"] in ("conv", "fc")]
BUDGETS = (8, 18, 37, 74, 148)


def layer_times(n, x, reps=20):
    n.infer(x)
    torch.cuda.synchronize()
    n.set_layer_timing(True)
    for _ in range(reps):
        n.infer(x)
    torch.cuda.synchronize()
    ms, k = n.read_layer_timing()
    n.set_layer_timing(False)
    return [m / k * 1000.0 for m in ms]


points = []
for B in (1, 64, 256):
    x = torch.from_numpy(synth.images(0, B, net["in_shape"])).cuda()
    for nb in BUDGETS:
        n = pcnn.Net(net, w, b, B, "bf16")
        for i in gemm:
            n.set_sm_budget(i, nb, 0)
        t = layer_times(n, x)
        for i in gemm:
            q = n.query_layer(i, B)
            bp = n.plan_budget(i, B)
            # eq. 8 at this budget, as the library evaluates it
            model = n.model_layer_time(i, B, nb)
            inv = round((model - bp["t_launch_us"]) / bp["t_unit_us"]) if bp["t_unit_us"] else 0
            points.append({"layer": names[i], "B": B, "n": nb, "measured_us": round(t[i], 3),
                           "model_us": round(model, 3), "t_launch_us": bp["t_launch_us"],
                           "t_unit_us": round(bp["t_unit_us"], 4), "inv": inv,
                           "class": "fc" if q["a_mode"] == 3 else "conv"})
        n.close()

fit = {}
for cls in ("conv", "fc"):
    P = [p for p in points if p["class"] == cls]
    # weighted least squares on relative error: minimise sum ((T0 + s*inv*u - m) / m)^2
    A = np.array([[1.0 / p["measured_us"], p["inv"] * p["t_unit_us"] / p["measured_us"]] for p in P])
    y = np.ones(len(P))
    (t0, sc), *_ = np.linalg.lstsq(A, y, rcond=None)
    pred = t0 + sc * np.array([p["inv"] * p["t_unit_us"] for p in P])
    meas = np.array([p["measured_us"] for p in P])
    rel = np.abs(pred - meas) / meas
    fit[cls] = {"t_launch_us": round(float(t0), 3), "unit_scale": round(float(sc), 4),
                "max_rel_err": round(float(rel.max()), 4), "median_rel_err": round(float(np.median(rel)), 4),
                "frac_within_25pct": round(float((rel <= 0.25).mean()), 4), "points": len(P)}
compiled = np.array([abs(p["model_us"] - p["measured_us"]) / p["measured_us"] for p in points])
print(json.dumps({"net": "alexnet", "precision": "bf16", "budgets": BUDGETS, "fit": fit,
                  "compiled_model": {"max_rel_err": round(float(compiled.max()), 4),
                                     "median_rel_err": round(float(np.median(compiled)), 4),
                                     "frac_within_25pct": round(float((compiled <= 0.25).mean()), 4)},
                  "points": points}, indent=1))
