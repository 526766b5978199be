"""NEXT-3 demo ("we can release 3 SMs to perform other tasks"):
workload A = AlexNet at batch 1 (the latency-critical task) with every GEMM
layer on its eq. 11 optSM budget, workload B = AlexNet at batch 64 (a
background task) capped to the SMs A never needs (148 - max optSM of A).
Each runs alone, then both run concurrently on two streams; A's pass latency
and B's throughput are reported for every case, plus A on all SMs next to the
same background task for comparison.  Writes one JSON document (stdout).

    python tools/released_sms_demo.py > profiles/r02_released_sms_demo.json
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_hpca_songhcl17_b200 import pcnn  # noqa: E402

net = synth.alexnet()
w, b = synth.net_params(net)
nsms = torch.cuda.get_device_properties(0).multi_processor_count
sA, sB = torch.cuda.Stream(), torch.cuda.Stream()
xa = torch.from_numpy(synth.images(0, 1, net["in_shape"])).cuda()
xb = torch.from_numpy(synth.images(1, 64, net["in_shape"])).cuda()


def make_a(opt):
    n = pcnn.Net(net, w, b, 1, "bf16")
    plans = n.apply_opt_budgets(1) if opt else [n.plan_budget(i, 1) for i in range(n.n_layers)]
    return n, plans


def make_b(cap):
    n = pcnn.Net(net, w, b, 64, "bf16")
    if cap < nsms:
        for i in range(n.n_layers):
            n.set_sm_budget(i, cap, 0)
    return n


def run(na, nb, passes_a=400, passes_b=40):
    """Returns (A ms per pass, B img/s); either may be None."""
    oa = torch.empty((1, 1000), device="cuda")
    ob = torch.empty((64, 1000), device="cuda")
    for _ in range(3):
        if na:
            na.infer(xa, oa, stream=sA)
        if nb:
            nb.infer(xb, ob, stream=sB)
    torch.cuda.synchronize()
    ea0, ea1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    eb0, eb1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if na:
        ea0.record(sA)
    if nb:
        eb0.record(sB)
    ratio = passes_a // passes_b
    for i in range(passes_a):
        if na:
            na.infer(xa, oa, stream=sA)
        if nb and i % ratio == 0:
            nb.infer(xb, ob, stream=sB)
    if na:
        ea1.record(sA)
    if nb:
        eb1.record(sB)
    torch.cuda.synchronize()
    ta = ea0.elapsed_time(ea1) / passes_a if na else None
    tb = 64 * passes_b / (eb0.elapsed_time(eb1) / 1000) if nb else None
    return ta, tb


na_opt, plans = make_a(True)
opt = {net["layers"][i].get("name"): p["opt_sm"] for i, p in enumerate(plans) if p["grid_size"] > 0}
cap = nsms - max(opt.values())
na_all, _ = make_a(False)
nb = make_b(max(cap, 2))
res = {"sms": nsms, "A": "alexnet batch 1, bf16, every GEMM layer on its eq. 11 optSM",
       "B": "alexnet batch 64, bf16, every layer capped to %d SMs (148 - max optSM of A)" % cap,
       "opt_sm": opt, "b_cap_sms": cap}
res["A_alone_optSM_ms"] = round(run(na_opt, None)[0], 5)
res["A_alone_allSM_ms"] = round(run(na_all, None)[0], 5)
res["B_alone_img_s"] = round(run(None, nb)[1], 1)
ta, tb = run(na_opt, nb)
res["concurrent_optSM"] = {"A_ms": round(ta, 5), "B_img_s": round(tb, 1)}
ta, tb = run(na_all, nb)
res["concurrent_allSM"] = {"A_ms": round(ta, 5), "B_img_s": round(tb, 1)}
nb_free = make_b(nsms)
ta, tb = run(na_opt, nb_free)
res["concurrent_optSM_B_uncapped"] = {"A_ms": round(ta, 5), "B_img_s": round(tb, 1)}
print(json.dumps(res, indent=1))
