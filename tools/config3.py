"""BASELINE.json configs[2]: AlexNet with rank-reduced conv variants per layer
(the accuracy-tuning ladder of SURVEY.md §8(d) config 3) and per-layer SM
budgets.  Writes one JSON document (stdout):

  budget_sweep[B][n] : per-GEMM-layer latency (ms, live CUDA events) with every
                       GEMM layer on n SMs, n in {148, 74, 37, 18, 8, "opt"}
                       ("opt" = each layer's eq. 11 optSM), plus eq. 12's
                       modelled time and eq. 11's optSM per layer
  ladder[B]          : img/s per ladder level, FLOP reduction, logit error of
                       the CUDA path vs the rank-r oracle and vs the exact
                       oracle, top-1 agreement with the exact oracle (4 images)

    python tools/config3.py > profiles/r01_config3_budget_rank.json
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from oracle import oracle as orc  # noqa: E402
from paper_conf_hpca_songhcl17_b200 import pcnn  # noqa: E402

net = synth.alexnet()
w, b = synth.net_params(net)
names = [L.get("name", str(i)) for i, L in enumerate(net["layers"])]
gemm = [i for i, L in enumerate(net["layers"]) if L["kind"] in ("conv", "fc")]
nsms = torch.cuda.get_device_properties(0).multi_processor_count
PERF_LADDER = [{}, {3: (2, 1)}, {3: (2, 1), 8: (2, 1)}, {3: (2, 1), 8: (2, 1), 7: (2, 1)},
               {3: (2, 1), 8: (2, 1), 7: (2, 1), 6: (2, 1)},
               {3: (3, 1), 8: (3, 1), 7: (3, 1), 6: (3, 1)},
               {3: (2, 2), 8: (2, 2), 7: (2, 2), 6: (2, 2)}]
LADDER = [{}, {3: 64}, {3: 64, 8: 64}, {3: 64, 8: 64, 7: 96}, {3: 64, 8: 64, 7: 96, 6: 192},
          {3: 32, 8: 32, 7: 48, 6: 96}, {3: 16, 8: 16, 7: 32, 6: 48}]


def layer_times(n, x, reps=20):
    n.infer(x)
    torch.cuda.synchronize()
    n.set_layer_timing(True)
    for _ in range(reps):
        n.infer(x)
    torch.cuda.synchronize()
    ms, k = n.read_layer_timing()
    n.set_layer_timing(False)
    return [m / k for m in ms]


def img_s(n, x, reps=30):
    for _ in range(3):
        n.infer(x)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        n.infer(x)
    e1.record()
    torch.cuda.synchronize()
    return x.shape[0] * reps / (e0.elapsed_time(e1) / 1000)


res = {"net": "alexnet", "precision": "bf16", "sms": nsms, "budget_sweep": {}, "ladder": {}}
for B in (1, 64, 256):
    x = torch.from_numpy(synth.images(0, B, net["in_shape"])).cuda()
    sweep = {}
    for nb in (nsms, 74, 37, 18, 8, "opt"):
        n = pcnn.Net(net, w, b, B, "bf16")
        plans = [n.plan_budget(i, B) for i in range(n.n_layers)]
        for i in gemm:
            n.set_sm_budget(i, plans[i]["opt_sm"] if nb == "opt" else nb, 0)
        t = layer_times(n, x)
        sweep[str(nb)] = {names[i]: round(t[i], 5) for i in gemm}
        sweep[str(nb)]["total_ms"] = round(sum(t), 5)
        if nb == "opt":
            sweep["model"] = {names[i]: {"opt_sm": plans[i]["opt_sm"],
                                         "grid_size": plans[i]["grid_size"],
                                         "n_invocations": plans[i]["n_invocations"],
                                         "t_model_ms": round(plans[i]["t_model_us"] / 1000, 5)}
                              for i in gemm}
        n.close()
    res["budget_sweep"][str(B)] = sweep

xs = synth.images(0, 4, net["in_shape"])
ref_exact = orc.run_net(net, w, b, xs)
for B in (64, 256):
    x = torch.from_numpy(synth.images(0, B, net["in_shape"])).cuda()
    rows = []
    for lvl, ranks in enumerate(LADDER):
        n = pcnn.Net(net, w, b, B, "bf16")
        for i, r in ranks.items():
            n.set_variant(i, "rank", r)
        fl = sum(n.query_layer(i, B)["flops"] for i in gemm)
        fe = sum(n.query_layer(i, B)["flops_exact"] for i in gemm)
        row = {"level": lvl, "ranks": {names[i]: r for i, r in ranks.items()},
               "img_s": round(img_s(n, x), 1), "flop_fraction": round(fl / fe, 4)}
        if B == 64:
            out, _, _ = n.infer(torch.from_numpy(xs).cuda())
            torch.cuda.synchronize()
            y = out.cpu().numpy()
            ref_r = orc.run_net(net, w, b, xs, ranks=ranks) if ranks else ref_exact
            row["err_vs_rank_oracle"] = float(np.abs(y - ref_r).max() / np.abs(ref_r).max())
            row["err_vs_exact_oracle"] = float(np.abs(y - ref_exact).max() / np.abs(ref_exact).max())
            row["top1_agree_exact"] = float((y.argmax(1) == ref_exact.argmax(1)).mean())
        rows.append(row)
        n.close()
    res["ladder"][str(B)] = rows
# NEXT-1: perforation ladder (R13 grid steps per layer)
res["perforation_ladder"] = {}
for B in (64, 256):
    x = torch.from_numpy(synth.images(0, B, net["in_shape"])).cuda()
    rows = []
    for lvl, perf in enumerate(PERF_LADDER):
        n = pcnn.Net(net, w, b, B, "bf16")
        for i, st in perf.items():
            n.set_perforation(i, *st)
        fl = sum(n.query_layer(i, B)["flops"] for i in gemm)
        fe = sum(n.query_layer(i, B)["flops_exact"] for i in gemm)
        row = {"level": lvl, "steps": {names[i]: list(st) for i, st in perf.items()},
               "img_s": round(img_s(n, x), 1), "flop_fraction": round(fl / fe, 4)}
        if B == 64:
            out, _, ent = n.infer(torch.from_numpy(xs).cuda(), entropy=True)
            torch.cuda.synchronize()
            y = out.cpu().numpy()
            ref_p = orc.run_net(net, w, b, xs, perforation=perf) if perf else ref_exact
            row["err_vs_perforated_oracle"] = float(np.abs(y - ref_p).max() / np.abs(ref_p).max())
            row["err_vs_exact_oracle"] = float(np.abs(y - ref_exact).max() / np.abs(ref_exact).max())
            row["top1_agree_exact"] = float((y.argmax(1) == ref_exact.argmax(1)).mean())
            row["mean_entropy"] = float(ent.mean().item())
        rows.append(row)
        n.close()
    res["perforation_ladder"][str(B)] = rows
print(json.dumps(res, indent=1))
