"""Per-layer SM budget (P:213 PSM, P:341 optSM x optTLP) and the rank-r
variant (north_star; R7) on the GPU, through the C ABI."""
import numpy as np
import pytest

import synth
from tests.helpers import TOL, conv_layer, gpu_run, params, rel_err, small_inputs

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")


@pytest.fixture(scope="module")
def alex():
    net = synth.alexnet()
    w, b = params(net)
    x = synth.images(0, 2, net["in_shape"])
    return net, w, b, x


# ------------------------------------------------------------------ SM budget
@pytest.mark.parametrize("prec", ["bf16", "fp32"])
def test_budget_is_bitwise_invariant_and_census_bounded(alex, prec):
    """R11: the budget changes placement only.  Every budget gives bitwise
    identical logits; the %smid census of each layer stays within the budget
    (tcgen05 CTA pairs round the budget up to 2 SMs, an FC layer's K-split
    cluster up to its `splits` SMs)."""
    net, w, b, x = alex
    gemm_layers = [i for i, L in enumerate(net["layers"]) if L["kind"] in ("conv", "fc")]
    base = gpu_run(net, w, b, x, prec)["out"]
    for n_sms, tlp in [(1, 0), (2, 0), (7, 1), (37, 2), (74, 0), (148, 0)]:
        budgets = {i: (n_sms, tlp) for i in range(len(net["layers"]))}
        r = gpu_run(net, w, b, x, prec, budgets=budgets, census=True)
        np.testing.assert_array_equal(r["out"], base, err_msg="budget %d/%d" % (n_sms, tlp))
        for i in gemm_layers:
            used = r["census"][i]
            # an FC layer's K split needs all its CTA pairs at once
            floor = 2 * r["net"].query_layer(i, x.shape[0])["splits"] \
                if net["layers"][i]["kind"] == "fc" else 2
            assert 0 < len(used) <= max(n_sms, floor), (i, n_sms, used)


def test_budget_simt_tlp_gating(alex):
    """SIMT kernels: CTAs admitted only on SMs with %smid < n, at most tlp
    CTAs each (Priority-SM packing, Fig. 7)."""
    net, w, b, x = alex
    r = gpu_run(net, w, b, x, "fp32", budgets={3: (4, 2)}, census=True)
    assert set(r["census"][3]) <= {0, 1, 2, 3}


def test_query_layer_reports_plan(alex):
    net, w, b, x = alex
    r = gpu_run(net, w, b, x, "bf16", budgets={6: (37, 0)})
    info = r["net"].query_layer(6, 64)
    assert info["engine"] == 1 and info["n_sms"] == 37
    assert 0 < info["util"] <= 1 and 0 < info["rec"] <= 1
    assert info["tiles"] >= 1 and info["grid"] <= 37
    assert info["flops"] == info["flops_exact"] == 2 * 64 * 13 * 13 * 384 * 9 * 256


# ------------------------------------------------------------------ rank-r variant
def test_rank_identity_factors_bitwise_fp32(alex):
    """Identity factorisation (A = I, B = W) reproduces the exact layer
    bitwise on the FP32 path: stage 1 sums the same K terms in the same order,
    stage 2 multiplies by exact ones and zeros."""
    net = dict(in_shape=(32, 13, 13), layers=[conv_layer(64, 3, 32, 1, 1, 2, relu=True)])
    w, b = params(net, seed=11)
    x = small_inputs((32, 13, 13), 3)
    import torch
    from paper_conf_hpca_songhcl17_b200 import pcnn
    n = pcnn.Net(net, w, b, 3, "fp32")
    xd = torch.from_numpy(x).cuda()
    exact = n.infer(xd)[0].cpu().numpy()
    g, Nfg = 2, 32
    A = np.stack([np.eye(Nfg, dtype=np.float32)] * g)             # [g][Nfg][r]
    B = w[0].reshape(g, Nfg, 16, 3, 3)                             # [g][r][C/g][S][S]
    n.set_variant_factors(0, Nfg, A, B)
    fact = n.infer(xd)[0].cpu().numpy()
    np.testing.assert_array_equal(fact, exact)
    n.set_variant(0, "exact")
    np.testing.assert_array_equal(n.infer(xd)[0].cpu().numpy(), exact)


@pytest.mark.parametrize("prec", ["fp32", "tf32", "bf16"])
def test_rank_r_conv_matches_rank_oracle(orc, prec):
    """The two-stage rank-r conv equals the oracle's W_r = U_r U_r^T W conv."""
    net = dict(in_shape=(48, 15, 15), layers=[conv_layer(64, 3, 48, 1, 1, 1, relu=True)])
    w, b = params(net, seed=13)
    x = small_inputs((48, 15, 15), 2)
    for r in (8, 24, 64):
        ref = orc.run_net(net, w, b, x, ranks={0: r}).reshape(2, -1)
        out = gpu_run(net, w, b, x, prec, variants={0: ("rank", r)})["out"]
        assert rel_err(out, ref) <= TOL[prec] / 2, (prec, r)
    # full rank == exact layer
    ref = orc.run_net(net, w, b, x).reshape(2, -1)
    out = gpu_run(net, w, b, x, prec, variants={0: ("rank", 64)})["out"]
    assert rel_err(out, ref) <= TOL[prec] / 2


@pytest.mark.parametrize("prec", ["tf32", "bf16"])
def test_alexnet_rank_ladder(orc, alex, prec):
    """configs[2]: the accuracy-tuning ladder -- each
    rung matches the rank-r oracle end to end."""
    net, w, b, x = alex
    ladder = [{}, {3: 64}, {3: 64, 8: 64}, {3: 64, 8: 64, 7: 96},
              {3: 64, 8: 64, 7: 96, 6: 192}]
    for rung in ladder[1:]:
        ref = orc.run_net(net, w, b, x, ranks=rung)
        out = gpu_run(net, w, b, x, prec,
                      variants={i: ("rank", r) for i, r in rung.items()})["out"]
        assert rel_err(out, ref) <= TOL[prec], (prec, rung)


def test_rank_variant_rejects_bad_requests(alex):
    net, w, b, x = alex
    from paper_conf_hpca_songhcl17_b200 import pcnn
    n = pcnn.Net(net, w, b, 2, "bf16")
    with pytest.raises(pcnn.PcnnError):
        n.set_variant(1, "rank", 8)         # LRN layer
    with pytest.raises(pcnn.PcnnError):
        n.set_variant(3, "rank", 0)
    with pytest.raises(pcnn.PcnnError):
        n.set_variant(3, "rank", 129)       # > min(N_f/g, K) = 128
    info = n.query_layer(3, 2)
    assert info["variant"] == 0
    n.set_variant(3, "rank", 32)
    info = n.query_layer(3, 2)
    assert info["variant"] == 1 and info["rank"] == 32
    assert info["flops"] < info["flops_exact"]


# ------------------------------------------------------------------ resource / time model (NEXT-3)
@pytest.mark.parametrize("prec,B", [("bf16", 1), ("bf16", 64), ("fp32", 2)])
def test_plan_budget_matches_oracle_eq11(orc, alex, prec, B):
    """pcnn_plan_budget's optSM is eq. 11 applied to the layer's
    own GridSize, TLP and SM count -- checked against the oracle's eq. 8 / 11
    helpers, which tests/test_oracle_pins.py pins to the paper's worked
    example -- and eq. 12's time is positive and scales with 1 / optSM."""
    import torch
    from paper_conf_hpca_songhcl17_b200 import pcnn
    net, w, b, _ = alex
    n = pcnn.Net(net, w, b, B, prec)
    nsms = torch.cuda.get_device_properties(0).multi_processor_count
    for i, L in enumerate(net["layers"]):
        p = n.plan_budget(i, B)
        if L["kind"] not in ("conv", "fc"):
            assert p["grid_size"] == 0 and p["opt_sm"] == nsms
            continue
        cg, G, tlp = p["cta_group"], p["grid_size"], p["opt_tlp"]
        info = n.query_layer(i, B)
        assert G == info["tiles"] * info["splits"]
        assert tlp == (1 if prec == "bf16" else max(1, info["tlp"]))
        assert p["n_invocations"] == orc.n_invocations(G, tlp, nsms // cg)
        assert p["opt_sm"] == cg * orc.opt_sm(G, tlp, nsms // cg), (i, p)
        assert p["opt_sm"] <= nsms and p["t_model_us"] > 0


def test_opt_budgets_keep_results_and_latency(alex):
    """Running every GEMM layer on its eq. 11 optSM changes placement only
    (bitwise identical logits, per-layer SM census within optSM) and keeps
    the number of invocations, so the whole pass stays within 25% of the
    unbudgeted latency (the paper's claim: 'release SMs' at the same
    nInvocations)."""
    import torch
    from paper_conf_hpca_songhcl17_b200 import pcnn
    net, w, b, _ = alex
    B = 8
    x = torch.from_numpy(synth.images(0, B, net["in_shape"])).cuda()

    def timed(n):
        n.infer(x)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(20):
            n.infer(x)
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / 20

    n0 = pcnn.Net(net, w, b, B, "bf16")
    base, _, _ = n0.infer(x)
    t0 = timed(n0)
    n1 = pcnn.Net(net, w, b, B, "bf16")
    plans = n1.apply_opt_budgets(B)
    n1.enable_sm_census(True)
    out, _, _ = n1.infer(x)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(out.cpu().numpy(), base.cpu().numpy())
    for i, p in enumerate(plans):
        if p["grid_size"] > 0:
            assert 0 < len(n1.sm_census(i)) <= p["opt_sm"], (i, p)
    assert sum(p["opt_sm"] < 148 for p in plans if p["grid_size"] > 0) >= 1   # SMs released
    n1.enable_sm_census(False)
    t1 = timed(n1)
    assert t1 <= 1.25 * t0, (t0, t1)


@pytest.mark.parametrize("prec", ["tf32", "bf16"])
def test_fc_rank_variant_factors(orc, prec):
    """FC rank-r: factors A = U_r S_r, B = V_r^T installed
    through pcnn_set_variant_factors (B's columns in the input's C,H,W order,
    so the CHW -> HWC permutation of the first FC applies) match the oracle's
    rank-r operator (its own SVD algorithm) end to end."""
    net = dict(in_shape=(16, 8, 8), layers=[
        conv_layer(32, 3, 16, 1, 1), dict(kind="maxpool", k=2, stride=2),
        dict(kind="fc", out=96, in_f=32 * 4 * 4, relu=True),
        dict(kind="fc", out=16, in_f=96, relu=False)])
    w, b = params(net, seed=41)
    x = small_inputs((16, 8, 8), 3, lo=-2, hi=2)
    ranks = {2: 32, 3: 8}
    ref = orc.run_net(net, w, b, x, ranks=ranks).reshape(3, -1)
    import torch
    from paper_conf_hpca_songhcl17_b200 import pcnn
    n = pcnn.Net(net, w, b, 3, prec)
    for i, r in ranks.items():
        U, S, Vt = np.linalg.svd(np.asarray(w[i], dtype=np.float64), full_matrices=False)
        n.set_variant_factors(i, r, U[:, :r] * S[:r], Vt[:r])
        f = n.query_layer(i, 3)
        assert f["rank"] == r and f["flops"] < f["flops_exact"]
    out, _, _ = n.infer(torch.from_numpy(x).cuda())
    torch.cuda.synchronize()
    assert rel_err(out.cpu().numpy(), ref) <= TOL[prec] / 2
    with pytest.raises(pcnn.PcnnError):
        n.set_variant_factors(3, 17, np.zeros((16, 17)), np.zeros((17, 96)))   # rank > min(N, K)
