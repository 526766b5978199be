"""Shared test helpers: run a synth net through the CUDA path (C ABI) and the
oracle on the same seeded inputs, and compute the north_star error metric."""
import numpy as np

import synth

TOL = {"fp32": 1e-4, "tf32": 5e-3, "bf16": 2e-2}   # north_star, reading R10

# pcnn_net_flag (include/pcnn.h) -- layout choices compared by the tests
FLAG_NO_SPACE_TO_DEPTH = 1
FLAG_NO_PADDED_LAYOUT = 2
FLAG_NO_LRN_POOL_FUSION = 4
FLAG_CONV_LRN_EPILOGUE = 8
FLAG_PER_ROW_WINDOWS = 64
FLAG_NARROW_SLABS = 16
FLAG_PERFORATION_IM2COL = 32


def rel_err(y, ref):
    """max |y - ref| / max |ref| (R10)."""
    y = np.asarray(y, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    assert y.shape == ref.shape, (y.shape, ref.shape)
    den = np.abs(ref).max()
    return float(np.abs(y - ref).max() / (den if den > 0 else 1.0))


def gpu_run(net, weights, biases, x, precision, max_batch=None, probs=False,
            variants=None, budgets=None, census=False, perforation=None, flags=0,
            plans=None):
    """Build a libpcnn net, run x (numpy NCHW fp32) and return numpy outputs."""
    import torch
    from paper_conf_hpca_songhcl17_b200 import pcnn
    B = x.shape[0]
    n = pcnn.Net(net, weights, biases, max_batch or B, precision, flags=flags)
    for (i, (cg, ms)) in (plans or {}).items():
        n.set_layer_plan(i, cg, ms)
    for (i, (v, r)) in (variants or {}).items():
        n.set_variant(i, v, r)
    for (i, (sh, sw)) in (perforation or {}).items():
        n.set_perforation(i, sh, sw)
    for (i, (s, t)) in (budgets or {}).items():
        n.set_sm_budget(i, s, t)
    if census:
        n.enable_sm_census(True)
    xd = torch.from_numpy(np.ascontiguousarray(x, dtype=np.float32)).cuda()
    out, p, h = n.infer(xd, probs=probs, entropy=probs)
    torch.cuda.synchronize()
    res = {"out": out.cpu().numpy()}
    if probs:
        res["probs"] = p.cpu().numpy()
        res["entropy"] = h.cpu().numpy()
    if census:
        res["census"] = [n.sm_census(i) for i in range(len(net["layers"]))]
    res["net"] = n
    return res


def random_layer_net(layer, in_shape):
    return dict(name="one", in_shape=in_shape, layers=[layer])


def conv_layer(out, k, in_c, stride=1, pad=0, groups=1, relu=True):
    return dict(kind="conv", out=out, k=k, stride=stride, pad=pad, groups=groups,
                relu=relu, in_c=in_c)


def small_inputs(shape, B, seed=18, lo=-1.0, hi=1.0):
    return synth.images(0, B, shape, seed=seed, lo=lo, hi=hi)


def params(net, seed=17):
    return synth.net_params(net, seed)
