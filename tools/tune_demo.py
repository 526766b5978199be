"""Run-time management demo: entropy-guided greedy tuning of
AlexNet (BF16, one batch of seeded images) over per-layer rank-r and
perforation ladders, then calibration along the tuning path.  Prints JSON:
the path (state, ms per pass, mean CNN_entropy, TE), each table's eq. 11
optSM per layer, and calibration decisions for a few observed entropies.

    python tools/tune_demo.py [B] [entropy_margin_nats] > profiles/r01_tuning_path.json
"""
import json
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import synth  # noqa: E402
from paper_conf_hpca_songhcl17_b200 import pcnn, tuning  # noqa: E402

B = int(sys.argv[1]) if len(sys.argv) > 1 else 64
margin = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5
net = synth.alexnet()
w, b = synth.net_params(net)
names = [L.get("name", str(i)) for i, L in enumerate(net["layers"])]
x = torch.from_numpy(synth.images(0, B, net["in_shape"])).cuda()
n = pcnn.Net(net, w, b, B, "bf16")
ladders = {3: [("exact",), ("perf", 2, 1), ("rank", 64), ("rank", 32)],
           6: [("exact",), ("rank", 192), ("rank", 96), ("perf", 2, 1)],
           7: [("exact",), ("rank", 96), ("rank", 48)],
           8: [("exact",), ("rank", 64), ("perf", 2, 1)]}
measure = tuning.gpu_measure(n, ladders, x, reps=10)
t0, h0 = measure({l: 0 for l in ladders})
threshold = h0 + margin
path = tuning.greedy_tune(ladders, measure, threshold)
out = {"net": "alexnet", "batch": B, "precision": "bf16", "threshold_nats": threshold,
       "ladders": {names[l]: [list(v) for v in r] for l, r in ladders.items()}, "path": []}
for step in path:
    tuning.apply_state(n, ladders, step["state"])
    plans = [n.plan_budget(i, B) for i in range(n.n_layers)]
    out["path"].append({
        "layer": names[step["layer"]] if step["layer"] is not None else None,
        "state": {names[l]: list(ladders[l][r]) for l, r in step["state"].items()},
        "ms": round(step["time"], 5), "entropy": round(step["entropy"], 5),
        "te": None if step["te"] is None else (str(step["te"]) if step["te"] == float("inf")
                                               else round(step["te"], 5)),
        "opt_sm": {names[i]: p["opt_sm"] for i, p in enumerate(plans) if p["grid_size"] > 0}})
# eq. 15 SoC of the first and last tables: board energy per pass over ~1 s
meter = tuning.EnergyMeter(0)


def energy_per_pass(state):
    tuning.apply_state(n, ladders, state)
    o, _, e = n.infer(x, entropy=True)
    torch.cuda.synchronize()
    import time
    j0, t0, k = meter.read_j(), time.perf_counter(), 0
    while time.perf_counter() - t0 < 1.0:
        for _ in range(10):
            n.infer(x, out=o, entropy=e)
        k += 10
        torch.cuda.synchronize()
    return (meter.read_j() - j0) / k


if meter.read_j() is not None:
    t_i, t_t = 0.5, 2.0          # ms: imperceptible / unusable bounds of this demo (R15)
    out["soc"] = []
    for idx in (0, len(path) - 1):
        ej = energy_per_pass(path[idx]["state"])
        out["soc"].append({"table": idx, "j_per_pass": round(ej, 5),
                           "soc": tuning.soc(path[idx]["time"], path[idx]["entropy"], ej,
                                             t_i, t_t, threshold),
                           "t_i_ms": t_i, "t_t_ms": t_t})
last = len(path) - 1
# calibration with re-measurement: new inputs (another image range)
# observed under the last table, stepping back while the measured entropy
# exceeds the threshold; and the shift estimator for comparison
x2 = torch.from_numpy(synth.images(4096, B, net["in_shape"], lo=-160, hi=160)).cuda()
idx, trace = tuning.calibrate(path, last, tuning.gpu_observe(n, ladders, path, x2), threshold)
out["calibration"] = {"new_inputs": "images 4096.. at U[-160, 160)", "final_table": idx,
                      "trace": [[i, round(h, 5)] for i, h in trace],
                      "estimate_only": {str(h): tuning.calibrate_estimate(path, last, h, threshold)
                                        for h in (path[last]["entropy"], threshold + 0.5, 1e9)}}
# a stricter requirement than at tuning time (a threshold below every table's
# entropy): calibration walks back along the path to the exact table,
# re-measuring the entropy after every step
tight = min(p["entropy"] for p in path) - 1e-3
idx, trace = tuning.calibrate(path, last, tuning.gpu_observe(n, ladders, path, x), tight)
out["calibration_tight"] = {"threshold_nats": round(tight, 5), "final_table": idx,
                            "trace": [[i, round(h, 5)] for i, h in trace]}
# NEXT-4: background-task batch (every conv layer at Util = 1, eq. 6) on this
# net's own tile plans, and eq. 13's rescaled batch for a 0.2 ms requirement
nb = pcnn.Net(net, w, b, 256, "bf16")
convs = [i for i, L in enumerate(net["layers"]) if L["kind"] == "conv"]
out["background_batch"] = tuning.background_batch(
    lambda l, bsz: nb.query_layer(l, bsz)["util"], convs, 256)
out["util_at_background_batch"] = {names[l]: round(nb.query_layer(l, out["background_batch"])["util"], 4)
                                   for l in convs}
t_model = sum(nb.plan_budget(i, B)["t_model_us"] for i in range(nb.n_layers)) / 1000
out["eq13"] = {"t_user_ms": 0.2, "t_model_ms": round(t_model, 5), "batch": B,
               "new_batch": tuning.rescale_batch(0.2, t_model, B)}
print(json.dumps(out, indent=1))
