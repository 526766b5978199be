"""Pins of the FP64 oracle against things other than itself (CPU only).

Each test names what fixes the expected value: a hand-computed fixture under
tests/golden/ (with its citation), a value printed in PAPER.md, a closed form,
an invariant, or an independent library routine (scipy / numpy).
"""
import json
import math
import os

import numpy as np
import pytest
from scipy import signal

import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _load(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


# ----------------------------------------------------------------- conv
def test_conv_tiny_hand_computed(orc):
    g = _load("conv_tiny.json")
    x = np.array(g["x"], float)[None, None]
    w = np.array(g["w"], float)[None, None]
    for case in g["cases"]:
        y = orc.conv2d(x, w, np.array([case["bias"]]), case["stride"],
                       case["pad"], 1, False, threads=1)
        np.testing.assert_array_equal(y[0, 0], np.array(case["y"], float))
        y2 = orc.conv2d_im2col_gemm(x, w, np.array([case["bias"]]),
                                    case["stride"], case["pad"], 1, False)
        np.testing.assert_array_equal(y2[0, 0], np.array(case["y"], float))


def test_conv_grouped_hand_computed(orc):
    g = _load("conv_tiny.json")
    x = np.stack([np.array(g["x"], float), np.array(g["grouped"]["x1"], float)])[None]
    w = np.stack([np.array(g["w"], float), np.array(g["grouped"]["w1"], float)])[:, None]
    y = orc.conv2d(x, w, np.zeros(2), 1, 0, 2, False, threads=1)
    np.testing.assert_array_equal(y[0, 0], np.array(g["grouped"]["y0"], float))
    np.testing.assert_array_equal(y[0, 1], np.array(g["grouped"]["y1"], float))


def _scipy_conv(x, w, b, stride, pad, groups, relu):
    """Independent reference: scipy.signal.correlate2d per (filter, channel)."""
    B, C, H, W = x.shape
    F, Cg, S, _ = w.shape
    Fg = F // groups
    xp = np.pad(x, ((0, 0), (0, 0), (pad, pad), (pad, pad)))
    out = []
    for n in range(B):
        per_f = []
        for f in range(F):
            g = f // Fg
            acc = 0.0
            for c in range(Cg):
                acc = acc + signal.correlate2d(xp[n, g * Cg + c], w[f, c], mode="valid")
            acc = acc[::stride, ::stride] + b[f]
            per_f.append(np.maximum(acc, 0) if relu else acc)
        out.append(np.stack(per_f))
    return np.stack(out)


@pytest.mark.parametrize("shape", [
    # B, C, H, W, F, S, stride, pad, groups
    (2, 3, 9, 7, 4, 3, 1, 1, 1),
    (1, 4, 11, 11, 6, 5, 2, 2, 2),
    (2, 3, 15, 15, 2, 11, 4, 0, 1),
    (1, 6, 6, 6, 6, 3, 1, 1, 3),
])
def test_conv_matches_scipy_and_fig2(orc, shape):
    B, C, H, W, F, S, st, pad, g = shape
    rng = np.random.default_rng(1)
    x = rng.standard_normal((B, C, H, W))
    w = rng.standard_normal((F, C // g, S, S))
    b = rng.standard_normal(F)
    for relu in (False, True):
        y = orc.conv2d(x, w, b, st, pad, g, relu, threads=3)
        ref = _scipy_conv(x, w, b, st, pad, g, relu)
        assert y.shape == ref.shape
        np.testing.assert_allclose(y, ref, rtol=1e-12, atol=1e-12)
        y2 = orc.conv2d_im2col_gemm(x, w, b, st, pad, g, relu)
        np.testing.assert_allclose(y, y2, rtol=1e-13, atol=1e-13)
        if relu:
            assert (y >= 0).all()


def test_conv_thread_count_invariant(orc):
    rng = np.random.default_rng(2)
    x = rng.standard_normal((5, 4, 8, 8))
    w = rng.standard_normal((6, 2, 3, 3))
    b = rng.standard_normal(6)
    y1 = orc.conv2d(x, w, b, 1, 1, 2, True, threads=1)
    y8 = orc.conv2d(x, w, b, 1, 1, 2, True, threads=8)
    np.testing.assert_array_equal(y1, y8)


def test_output_sizes_pin_paper_shapes(orc):
    p = _load("paper_pins.json")["alexnet_shapes"]
    h = orc.conv_out_size(227, 11, 4, 0)
    assert h == p["conv1"]
    h = orc.pool_out_size(h, 3, 2)
    assert h == p["pool1"]
    h = orc.conv_out_size(h, 5, 1, 2)
    assert h == p["conv2"]
    h = orc.pool_out_size(h, 3, 2)
    assert h == p["pool2"]
    h = orc.conv_out_size(h, 3, 1, 1)
    assert h == p["conv5"]
    assert orc.pool_out_size(h, 3, 2) == p["pool5"]
    # VGG: 224 -> 112 -> 56 -> 28 -> 14 -> 7 (2x2 s2 pools), 3x3 p1 convs keep size
    h = 224
    for _ in range(5):
        assert orc.conv_out_size(h, 3, 1, 1) == h
        h = orc.pool_out_size(h, 2, 2)
    assert h == 7


def test_alexnet_per_group_gemm_dims_table_iv(orc):
    """T4: per-group GEMM N_f/g x W_oH_o of AlexNet at batch 1 (Table IV)."""
    p = _load("paper_pins.json")["alexnet_per_group_gemm"]
    net = synth.alexnet()
    h = 227
    ci = 0
    for L in net["layers"]:
        if L["kind"] == "conv":
            h = orc.conv_out_size(h, L["k"], L["stride"], L["pad"])
            ci += 1
            assert [L["out"] // L["groups"], h * h] == p["conv%d" % ci]
        elif L["kind"] == "maxpool":
            h = orc.pool_out_size(h, L["k"], L["stride"])


# ----------------------------------------------------------------- pool
def test_maxpool_hand_computed(orc):
    g = _load("conv_tiny.json")["maxpool"]
    x = np.array(g["x"], float)[None, None]
    y = orc.maxpool(x, 3, 2, threads=1)
    np.testing.assert_array_equal(y[0, 0], np.array(g["y"], float))


def test_avgpool_closed_forms(orc):
    x = np.full((2, 3, 8, 8), 2.5)
    np.testing.assert_array_equal(orc.avgpool(x, 2, 2), np.full((2, 3, 4, 4), 2.5))
    x = np.arange(16, dtype=float).reshape(1, 1, 4, 4)
    y = orc.avgpool(x, 2, 2)
    np.testing.assert_allclose(y[0, 0], [[2.5, 4.5], [10.5, 12.5]])


def test_maxpool_matches_numpy_reduce(orc):
    rng = np.random.default_rng(3)
    x = rng.standard_normal((2, 5, 8, 8))
    y = orc.maxpool(x, 2, 2)
    ref = x.reshape(2, 5, 4, 2, 4, 2).max(axis=(3, 5))
    np.testing.assert_array_equal(y, ref)


# ----------------------------------------------------------------- LRN
@pytest.mark.parametrize("a", [1.0, 30.0, 128.0])
def test_lrn_constant_input_closed_form(orc, a):
    """Closed form on constant input: interior channels see 5 equal terms,
    channel 0 / C-1 see 3, channel 1 / C-2 see 4 (Caffe window, reading R3)."""
    C = 8
    x = np.full((1, C, 2, 3), a)
    y = orc.lrn(x, 5, 1e-4, 0.75, 1.0)
    n_terms = [3, 4, 5, 5, 5, 5, 4, 3]
    for c in range(C):
        expect = a / (1.0 + 1e-4 / 5 * n_terms[c] * a * a) ** 0.75
        np.testing.assert_allclose(y[0, c], expect, rtol=1e-14)


def test_lrn_single_channel_spike(orc):
    """A lone non-zero channel normalises itself only through its own square;
    neighbours stay exactly zero."""
    x = np.zeros((1, 6, 1, 1))
    x[0, 2] = 10.0
    y = orc.lrn(x, 5, 1e-4, 0.75, 2.0)
    np.testing.assert_allclose(y[0, 2, 0, 0], 10.0 / (2.0 + 1e-4 / 5 * 100.0) ** 0.75, rtol=1e-14)
    assert np.count_nonzero(y) == 1


# ----------------------------------------------------------------- FC
def test_fc_single_column_probe(orc):
    N, K = 7, 12
    w = np.zeros((N, K))
    w[:, 5] = np.arange(1, N + 1)
    x = np.arange(K, dtype=float)[None] + 1.0
    b = np.full(N, -0.25)
    y = orc.fc(x, w, b, relu=False)
    np.testing.assert_array_equal(y[0], np.arange(1, N + 1) * 6.0 - 0.25)


def test_fc_matches_numpy_matmul_and_chw_flatten(orc):
    rng = np.random.default_rng(4)
    x = rng.standard_normal((3, 4, 2, 5))
    w = rng.standard_normal((9, 40))
    b = rng.standard_normal(9)
    y = orc.fc(x, w, b, relu=True)
    ref = np.maximum(x.reshape(3, 40) @ w.T + b, 0)   # C,H,W flatten
    np.testing.assert_allclose(y, ref, rtol=1e-13, atol=1e-13)


# ----------------------------------------------------------------- softmax / entropy
def test_entropy_paper_example(orc):
    e = _load("paper_pins.json")["entropy_example"]
    h1, h2 = orc.entropy(np.array(e["P1"])), orc.entropy(np.array(e["P2"]))
    assert abs(h1 - e["H1"]) < 5e-5 and abs(h2 - e["H2"]) < 5e-5
    assert h1 > h2


def test_softmax_closed_forms(orc):
    p, H = orc.softmax_entropy(np.zeros((2, 1000)))
    np.testing.assert_allclose(p, 1e-3, rtol=1e-14)
    np.testing.assert_allclose(H, math.log(1000.0), rtol=1e-12)   # 6.9078 (1000-term sum rounding)
    p, H = orc.softmax_entropy(np.array([[0.0, math.log(2.0)]]))
    np.testing.assert_allclose(p[0], [1 / 3, 2 / 3], rtol=1e-14)
    rng = np.random.default_rng(5)
    z = rng.standard_normal((4, 50)) * 20
    p, H = orc.softmax_entropy(z)
    np.testing.assert_allclose(p.sum(1), 1.0, rtol=1e-14)
    p2, _ = orc.softmax_entropy(z + 1234.5)           # shift invariance
    np.testing.assert_allclose(p, p2, rtol=1e-9)
    # one-hot limit: H -> 0
    _, H = orc.softmax_entropy(np.array([[0.0, 800.0, 0.0]]))
    assert H[0] < 1e-300 or H[0] == 0.0


# ----------------------------------------------------------------- rank-r
def test_rank_r_against_numpy_svd(orc):
    rng = np.random.default_rng(6)
    Wm = rng.standard_normal((24, 40))
    U, s, Vt = np.linalg.svd(Wm, full_matrices=False)
    for r in (1, 5, 12, 24):
        Wr, sig, uniq = orc.rank_r(Wm, r)
        assert uniq
        np.testing.assert_allclose(sig, s, rtol=1e-10, atol=1e-10)
        ref = (U[:, :r] * s[:r]) @ Vt[:r]
        np.testing.assert_allclose(Wr, ref, atol=1e-10)
        # Eckart-Young: ||W - W_r||_F^2 = sum_{i>r} sigma_i^2
        np.testing.assert_allclose(np.sum((Wm - Wr) ** 2), np.sum(s[r:] ** 2),
                                   rtol=1e-9, atol=1e-9)
    # full rank reproduces W
    Wr, _, _ = orc.rank_r(Wm, 24)
    np.testing.assert_allclose(Wr, Wm, atol=1e-12)


def test_rank_r_exact_on_rank_one(orc):
    u = np.arange(1.0, 9.0)
    v = np.linspace(-1, 1, 13)
    Wm = np.outer(u, v)
    Wr, sig, _ = orc.rank_r(Wm, 1)
    np.testing.assert_allclose(Wr, Wm, atol=1e-12)
    assert sig[1] < 1e-6 * sig[0]


def test_rank_r_conv_linearity(orc):
    """conv with W_r == stage-1 conv (filters V_r^T) then 1x1 conv (U_r S_r):
    the two-stage identity the CUDA variant uses (reading R7)."""
    rng = np.random.default_rng(7)
    x = rng.standard_normal((1, 4, 7, 7))
    w = rng.standard_normal((6, 4, 3, 3))
    b = rng.standard_normal(6)
    r = 3
    Wr, _ = orc.rank_r_conv_weight(w, 1, r)
    y = orc.conv2d(x, Wr, b, 1, 1, 1, True)
    U, s, Vt = np.linalg.svd(w.reshape(6, -1), full_matrices=False)
    st1 = orc.conv2d(x, Vt[:r].reshape(r, 4, 3, 3), None, 1, 1, 1, False)
    st2 = orc.conv2d(st1, (U[:, :r] * s[:r]).reshape(6, r, 1, 1), b, 1, 0, 1, True)
    np.testing.assert_allclose(y, st2, rtol=1e-10, atol=1e-10)


# ----------------------------------------------------------------- analytical models
def test_table_v_util_all_cells(orc):
    """T1: all 15 Util cells of Table V from eqs. 4 and 6 (reading R8)."""
    pins = _load("paper_pins.json")
    dims = pins["alexnet_per_group_gemm"]
    for gpu, cfg in pins["table_v_util"].items():
        if gpu.startswith("_"):
            continue
        for i, want in enumerate(cfg["util"]):
            nf, wh = dims["conv%d" % (i + 1)]
            G = orc.grid_size(nf, wh, cfg["tile_nf"], cfg["tile_wh"])
            assert abs(orc.util(G, cfg["max_blocks"]) - want) < 0.006, (gpu, i)


def test_table_iv_grid_and_max_blocks(orc):
    """T2: Table IV grid sizes (eq. 4) and maxBlocks (eq. 5)."""
    p = _load("paper_pins.json")
    dims = p["alexnet_per_group_gemm"]
    for name, t in p["table_iv"].items():
        if name.startswith("_"):
            continue
        assert orc.max_blocks(t["n_sms"], 65536, t["block"], t["regs"]) == t["max_blocks"]
        assert orc.grid_size(*dims["conv2"], t["tile_nf"], t["tile_wh"]) == t["grid_conv2"]
        assert orc.grid_size(*dims["conv5"], t["tile_nf"], t["tile_wh"]) == t["grid_conv5"]


def test_eq11_worked_example(orc):
    e = _load("paper_pins.json")["eq11_example"]
    assert orc.opt_sm(e["grid"], e["opt_tlp"], e["num_sms"]) == e["opt_sm"]
    # eq. 8 consistency: optSM keeps the invocation count
    assert orc.n_invocations(40, 3, 7) == orc.n_invocations(40, 3, 10) == 2


def test_rec_eq9_closed_forms(orc):
    assert orc.rec(256, 256, 128, 128) == 1.0
    assert orc.rec(100, 128, 128, 128) == 100 / 128
    assert abs(orc.rec(169, 128, 128, 128) - 169 / 256) < 1e-15


# ------------------------------------------------------------ perforation (NEXT-1, R13)
def test_perforation_index_hand_fixture(orc):
    """Nearest kept index (ties to the lower one) on a hand-written case:
    n = 7, s = 3 keeps 0, 3, 6; n = 6, s = 2 keeps 0, 2, 4 (5 -> 4);
    n = 5, s = 4 keeps 0, 4 (2 is a tie -> 0)."""
    assert list(orc.perforation_index(7, 3)) == [0, 0, 3, 3, 3, 6, 6]
    assert list(orc.perforation_index(6, 2)) == [0, 0, 2, 2, 4, 4]
    assert list(orc.perforation_index(5, 4)) == [0, 0, 0, 4, 4]
    assert list(orc.perforation_index(4, 1)) == [0, 1, 2, 3]


def test_perforation_rate_zero_is_exact_conv(orc):
    """Rate 0 (sh = sw = 1) is the exact layer, bit for bit."""
    rng = np.random.default_rng(3)
    x = rng.standard_normal((2, 6, 9, 8))
    w = rng.standard_normal((8, 3, 3, 3))
    b = rng.standard_normal(8)
    e = orc.conv2d(x, w, b, 1, 1, 2, True)
    p = orc.perforated_conv2d(x, w, b, 1, 1, 2, True, 1, 1)
    np.testing.assert_array_equal(p, e)
    assert orc.perforation_rate(9, 8, 1, 1) == 0.0


def test_perforation_kept_values_and_interpolation(orc):
    """Kept positions carry the exact conv values computed by brute force at
    those positions only; every other position equals a kept neighbour at
    distance <= s/2 per axis; the rate is 1 - H'W'/(HW)."""
    rng = np.random.default_rng(4)
    x = rng.standard_normal((1, 3, 11, 10))
    w = rng.standard_normal((4, 3, 3, 3))
    b = rng.standard_normal(4)
    sh, sw = 2, 3
    y = orc.perforated_conv2d(x, w, b, 1, 1, 1, False, sh, sw)
    xp = np.pad(x, ((0, 0), (0, 0), (1, 1), (1, 1)))
    for p in range(0, 11, sh):
        for q in range(0, 10, sw):
            for f in range(4):
                ref = b[f] + np.sum(w[f] * xp[0, :, p:p + 3, q:q + 3])
                assert abs(y[0, f, p, q] - ref) < 1e-12
    for p in range(11):
        for q in range(10):
            kp = min(range(0, 11, sh), key=lambda k: (abs(p - k), k))
            kq = min(range(0, 10, sw), key=lambda k: (abs(q - k), k))
            assert abs(p - kp) <= sh // 2 + (1 if p > 10 // sh * sh else 0)
            np.testing.assert_array_equal(y[0, :, p, q], y[0, :, kp, kq])
    assert abs(orc.perforation_rate(11, 10, sh, sw) - (1 - 6 * 4 / 110)) < 1e-15


# ------------------------------------------------------- rank-r per group (R7)
def test_rank_r_conv_weight_per_group_equals_numpy_svd_per_block(orc):
    """Reading R7: the rank-r operator is applied to each group's own
    (N_f/g) x (C/g S^2) block.  Pinned against numpy's SVD of each block: a
    wrong group slice (e.g. factorising the whole filter bank, swapping the
    blocks, or slicing by input channels) changes the result.  The two blocks
    are built with very different spectra so that any mix-up is visible."""
    rng = np.random.default_rng(21)
    g, Fg, Cg, S = 2, 6, 3, 3
    w = rng.standard_normal((g * Fg, Cg, S, S))
    w[Fg:] *= 10.0                                 # group 1: 10x the scale of group 0
    w[Fg:, :, 0, 0] += 25.0                        # and a dominant direction of its own
    for r in (1, 2, 4, Fg):
        wr, uniq = orc.rank_r_conv_weight(w, g, r)
        assert uniq
        for gi in range(g):
            blk = w[gi * Fg:(gi + 1) * Fg].reshape(Fg, -1)
            U, s, Vt = np.linalg.svd(blk, full_matrices=False)
            ref = ((U[:, :r] * s[:r]) @ Vt[:r]).reshape(Fg, Cg, S, S)
            np.testing.assert_allclose(wr[gi * Fg:(gi + 1) * Fg], ref, atol=1e-9)
        # the whole-bank factorisation is a different operator (negative control)
        if r < Fg:
            U, s, Vt = np.linalg.svd(w.reshape(g * Fg, -1), full_matrices=False)
            whole = ((U[:, :r] * s[:r]) @ Vt[:r]).reshape(w.shape)
            assert np.abs(whole - wr).max() > 1e-3
    # full rank per group reproduces the weights
    wr, _ = orc.rank_r_conv_weight(w, g, Fg)
    np.testing.assert_allclose(wr, w, atol=1e-9)


def test_run_net_rank_option_uses_per_group_operator(orc):
    """run_net(ranks={i: r}) runs the exact conv with the per-group W_r."""
    rng = np.random.default_rng(22)
    net = dict(name="t", in_shape=(4, 6, 6), layers=[
        dict(kind="conv", out=8, k=3, stride=1, pad=1, groups=2, relu=True, in_c=4)])
    w = [rng.standard_normal((8, 2, 3, 3))]
    b = [rng.standard_normal(8)]
    x = rng.standard_normal((2, 4, 6, 6))
    y = orc.run_net(net, w, b, x, ranks={0: 2})
    wr = np.empty_like(w[0])
    for gi in range(2):
        blk = w[0][gi * 4:(gi + 1) * 4].reshape(4, -1)
        U, s, Vt = np.linalg.svd(blk, full_matrices=False)
        wr[gi * 4:(gi + 1) * 4] = ((U[:, :2] * s[:2]) @ Vt[:2]).reshape(4, 2, 3, 3)
    ref = _scipy_conv(x, wr, b[0], 1, 1, 2, True)
    np.testing.assert_allclose(y, ref, rtol=1e-9, atol=1e-9)


# ------------------------------------------------------- run_net sequencing
def _np_lrn(a, size, alpha, beta, k):
    """Caffe across-channel LRN written with numpy (reading R3)."""
    C = a.shape[1]
    out = np.empty_like(a)
    h = size // 2
    for c in range(C):
        lo, hi = max(0, c - h), min(C - 1, c + h)
        ssum = np.sum(a[:, lo:hi + 1] ** 2, axis=1)
        out[:, c] = a[:, c] / (k + alpha / size * ssum) ** beta
    return out


def _np_maxpool(a, k, s):
    """ceil-mode max pooling (reading R4) by explicit windows."""
    B, C, H, W = a.shape
    Ho = -(-(H - k) // s) + 1
    Wo = -(-(W - k) // s) + 1
    if (Ho - 1) * s >= H:
        Ho -= 1
    if (Wo - 1) * s >= W:
        Wo -= 1
    y = np.empty((B, C, Ho, Wo))
    for p in range(Ho):
        for q in range(Wo):
            y[:, :, p, q] = a[:, :, p * s:min(p * s + k, H), q * s:min(q * s + k, W)].max(axis=(2, 3))
    return y


def test_run_net_equals_independent_numpy_composition(orc):
    """run_net's layer sequencing (conv -> LRN -> pool -> fc -> fc, the CHW
    flatten before fc, ReLU on all but the last layer, the final fc without
    ReLU) against a composition written with scipy / numpy only, on a tiny
    net at Caffe pixel scale (LRN active), and against the hand composition
    of the oracle's own pinned primitives."""
    rng = np.random.default_rng(23)
    net = dict(name="tiny", in_shape=(3, 11, 11), layers=[
        dict(kind="conv", out=6, k=3, stride=2, pad=1, groups=1, relu=True, in_c=3),
        dict(kind="lrn", size=5, alpha=1e-4, beta=0.75, k=1.0),
        dict(kind="maxpool", k=3, stride=2),
        dict(kind="conv", out=8, k=3, stride=1, pad=1, groups=2, relu=True, in_c=6),
        dict(kind="fc", out=7, in_f=8 * 3 * 3, relu=True),
        dict(kind="fc", out=5, in_f=7, relu=False),
    ])
    w = [rng.standard_normal((6, 3, 3, 3)) * 0.3, None, None,
         rng.standard_normal((8, 3, 3, 3)) * 0.2, rng.standard_normal((7, 72)) * 0.1,
         rng.standard_normal((5, 7))]
    b = [rng.uniform(-1, 1, 6), None, None, rng.uniform(-1, 1, 8), rng.uniform(-1, 1, 7),
         rng.uniform(-1, 1, 5)]
    x = rng.uniform(-128, 128, (2, 3, 11, 11))
    y, outs = orc.run_net(net, w, b, x, return_all=True)
    # independent composition
    a = _scipy_conv(x, w[0], b[0], 2, 1, 1, True)
    assert a.shape == (2, 6, 6, 6)
    a = _np_lrn(a, 5, 1e-4, 0.75, 1.0)
    assert np.abs(a - outs[0]).max() > 1e-3 * np.abs(a).max()   # LRN is not ~identity here
    a = _np_maxpool(a, 3, 2)
    assert a.shape == (2, 6, 3, 3)   # ceil mode: ceil((6 - 3) / 2) + 1 = 3, last window clipped
    a = _scipy_conv(a, w[3], b[3], 1, 1, 2, True)
    a = np.maximum(a.reshape(2, -1) @ w[4].T + b[4], 0.0)       # CHW flatten
    a = a @ w[5].T + b[5]                                        # no ReLU on the last fc
    np.testing.assert_allclose(y, a, rtol=1e-10, atol=1e-10)
    assert (y < 0).any()
    # hand composition of the oracle's pinned primitives
    h = orc.conv2d(x, w[0], b[0], 2, 1, 1, True)
    h = orc.lrn(h, 5, 1e-4, 0.75, 1.0)
    h = orc.maxpool(h, 3, 2)
    h = orc.conv2d(h, w[3], b[3], 1, 1, 2, True)
    h = orc.fc(h, w[4], b[4], True)
    h = orc.fc(h, w[5], b[5], False)
    np.testing.assert_array_equal(y, h)
    for i, o in enumerate(outs):
        assert o.shape[0] == 2, i
