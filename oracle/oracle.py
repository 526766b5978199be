"""Python front of the FP64 CPU oracle (oracle/pcnn_oracle.c).

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / ``--impl reference`` legs may import this module.  It never
imports the CUDA package and the CUDA package never imports it.

All arithmetic happens in the C library (FP64 loops); this module only
marshals numpy arrays and sequences the layers of a net description from
``synth.nets`` (NCHW activations, OIHW weights, FC input flattened C,H,W).
"""
import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "pcnn_oracle.c")
_LIB = os.path.join(_HERE, "liborc.so")

_dp = ctypes.POINTER(ctypes.c_double)


def build(force=False):
    """Compile the oracle with gcc -O2 (no -ffast-math)."""
    if force or not os.path.exists(_LIB) or \
            os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared",
                               "-o", tmp, _SRC, "-lm", "-lpthread"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        L = _lib
        i, d, l = ctypes.c_int, ctypes.c_double, ctypes.c_long
        L.orc_conv2d.argtypes = [_dp, i, i, i, i, _dp, _dp, i, i, i, i, i, i, _dp, i]
        L.orc_conv2d_im2col_gemm.argtypes = [_dp, i, i, i, i, _dp, _dp, i, i, i, i, i, i, _dp]
        L.orc_lrn.argtypes = [_dp, i, i, i, i, i, d, d, d, _dp, i]
        L.orc_maxpool.argtypes = [_dp, i, i, i, i, i, i, _dp, i]
        L.orc_avgpool.argtypes = [_dp, i, i, i, i, i, i, _dp, i]
        L.orc_fc.argtypes = [_dp, i, i, _dp, _dp, i, i, _dp, i]
        L.orc_softmax_entropy.argtypes = [_dp, i, i, _dp, _dp]
        L.orc_entropy.argtypes = [_dp, i]
        L.orc_entropy.restype = d
        L.orc_rank_r.argtypes = [_dp, i, i, i, _dp, _dp]
        L.orc_conv_out_size.argtypes = [i, i, i, i]
        L.orc_pool_out_size.argtypes = [i, i, i]
        L.orc_grid_size.argtypes = [l, l, l, l]
        L.orc_grid_size.restype = l
        L.orc_max_blocks.argtypes = [l, l, l, l]
        L.orc_max_blocks.restype = l
        L.orc_util.argtypes = [l, l]
        L.orc_util.restype = d
        L.orc_n_invocations.argtypes = [l, l, l]
        L.orc_n_invocations.restype = l
        L.orc_rec.argtypes = [l, l, l, l]
        L.orc_rec.restype = d
        L.orc_opt_sm.argtypes = [l, l, l]
        L.orc_opt_sm.restype = l
    return _lib


def _c(a):
    a = np.ascontiguousarray(a, dtype=np.float64)
    return a, a.ctypes.data_as(_dp)


def _null():
    return ctypes.cast(None, _dp)


def default_threads():
    return os.cpu_count() or 1


def _check(rc, what):
    if rc < 0:
        raise ValueError("oracle %s failed (rc=%d)" % (what, rc))


def conv_out_size(n, k, stride, pad):
    return lib().orc_conv_out_size(n, k, stride, pad)


def pool_out_size(n, k, stride):
    return lib().orc_pool_out_size(n, k, stride)


def conv2d(x, w, b, stride=1, pad=0, groups=1, relu=False, threads=None):
    x, xp = _c(x)
    w, wp = _c(w)
    B, C, H, W = x.shape
    F, _, S, _ = w.shape
    Ho, Wo = conv_out_size(H, S, stride, pad), conv_out_size(W, S, stride, pad)
    y = np.empty((B, F, Ho, Wo))
    if b is None:
        bp = _null()
    else:
        b, bp = _c(b)
    _check(lib().orc_conv2d(xp, B, C, H, W, wp, bp, F, S, stride, pad, groups,
                            int(relu), y.ctypes.data_as(_dp),
                            threads or default_threads()), "conv2d")
    return y


def conv2d_im2col_gemm(x, w, b, stride=1, pad=0, groups=1, relu=False):
    x, xp = _c(x)
    w, wp = _c(w)
    B, C, H, W = x.shape
    F, _, S, _ = w.shape
    Ho, Wo = conv_out_size(H, S, stride, pad), conv_out_size(W, S, stride, pad)
    y = np.empty((B, F, Ho, Wo))
    if b is None:
        bp = _null()
    else:
        b, bp = _c(b)
    _check(lib().orc_conv2d_im2col_gemm(xp, B, C, H, W, wp, bp, F, S, stride,
                                        pad, groups, int(relu),
                                        y.ctypes.data_as(_dp)), "im2col_gemm")
    return y


def lrn(x, size=5, alpha=1e-4, beta=0.75, k=1.0, threads=None):
    x, xp = _c(x)
    y = np.empty_like(x)
    B, C, H, W = x.shape
    _check(lib().orc_lrn(xp, B, C, H, W, size, alpha, beta, k,
                         y.ctypes.data_as(_dp), threads or default_threads()), "lrn")
    return y


def _pool(fn, x, k, stride, threads):
    x, xp = _c(x)
    B, C, H, W = x.shape
    Ho, Wo = pool_out_size(H, k, stride), pool_out_size(W, k, stride)
    y = np.empty((B, C, Ho, Wo))
    _check(fn(xp, B, C, H, W, k, stride, y.ctypes.data_as(_dp),
              threads or default_threads()), "pool")
    return y


def maxpool(x, k, stride, threads=None):
    return _pool(lib().orc_maxpool, x, k, stride, threads)


def avgpool(x, k, stride, threads=None):
    return _pool(lib().orc_avgpool, x, k, stride, threads)


def fc(x, w, b, relu=False, threads=None):
    B = x.shape[0]
    x, xp = _c(x.reshape(B, -1))          # C,H,W flatten of NCHW (reading R5)
    w, wp = _c(w)
    N, K = w.shape
    assert x.shape[1] == K, (x.shape, w.shape)
    y = np.empty((B, N))
    if b is None:
        bp = _null()
    else:
        b, bp = _c(b)
    _check(lib().orc_fc(xp, B, K, wp, bp, N, int(relu), y.ctypes.data_as(_dp),
                        threads or default_threads()), "fc")
    return y


def softmax_entropy(z):
    z, zp = _c(z)
    B, N = z.shape
    p = np.empty_like(z)
    H = np.empty(B)
    _check(lib().orc_softmax_entropy(zp, B, N, p.ctypes.data_as(_dp),
                                     H.ctypes.data_as(_dp)), "softmax")
    return p, H


def entropy(p):
    p, pp = _c(p)
    return lib().orc_entropy(pp, p.size)


def rank_r(Wm, r):
    """W_r = U_r U_r^T Wm (Gram/Jacobi); returns (W_r, sigma, unique_flag)."""
    Wm, wp = _c(Wm)
    N, K = Wm.shape
    Wr = np.empty_like(Wm)
    sig = np.empty(min(N, K))
    rc = lib().orc_rank_r(wp, N, K, r, Wr.ctypes.data_as(_dp),
                          sig.ctypes.data_as(_dp))
    _check(rc, "rank_r")
    return Wr, sig, rc == 0


def rank_r_conv_weight(w, groups, r):
    """Apply rank_r per group to OIHW conv weights (reading R7: per group,
    W_g in R^{(N_f/g) x (C/g S^2)})."""
    F = w.shape[0]
    Fg = F // groups
    out = np.empty(w.shape, dtype=np.float64)
    unique = True
    for g in range(groups):
        Wg = w[g * Fg:(g + 1) * Fg].reshape(Fg, -1).astype(np.float64)
        Wr, _, u = rank_r(Wg, r)
        unique = unique and u
        out[g * Fg:(g + 1) * Fg] = Wr.reshape((Fg,) + w.shape[1:])
    return out, unique


# perforation-interpolation (NEXT-1; Fig. 11, ref. [38] P:479)
def perforation_index(n, s):
    """Reading R13: the grid perforation keeps every s-th output row (column)
    0, s, 2s, ... < n; every other index takes the value of its nearest kept
    index (ties to the lower one; indices past the last kept one take the
    last).  Returns the kept-index source of each of the n outputs."""
    kept = list(range(0, n, s))
    src = []
    for p in range(n):
        best = min(kept, key=lambda k: (abs(p - k), k))
        src.append(best)
    return np.asarray(src, dtype=np.int64)


def perforated_conv2d(x, w, b, stride=1, pad=0, groups=1, relu=False, sh=1, sw=1,
                      threads=None):
    """Perforated conv: the convolution (eq. 1, bias, ReLU) evaluated
    only at the kept output positions of an sh x sw grid -- perforation rate
    1 - H'W'/(HW) -- and every skipped position filled with its nearest kept
    neighbour (interpolation, R13).  The kept values are the exact conv's
    values at those positions (the direct loop computes every output position
    independently), so they are taken from conv2d."""
    y = conv2d(x, w, b, stride, pad, groups, relu, threads)
    Ho, Wo = y.shape[2], y.shape[3]
    ri, ci = perforation_index(Ho, sh), perforation_index(Wo, sw)
    return y[:, :, ri][:, :, :, ci]


def perforation_rate(Ho, Wo, sh, sw):
    """1 - W'_o H'_o / (W_o H_o)."""
    return 1.0 - len(range(0, Ho, sh)) * len(range(0, Wo, sw)) / float(Ho * Wo)


# analytical helpers (eqs. 4, 5, 6, 8, 9, 11)
def grid_size(M, N, m, n):
    return lib().orc_grid_size(M, N, m, n)


def max_blocks(nsms, R, block, r):
    return lib().orc_max_blocks(nsms, R, block, r)


def util(grid, maxb):
    return lib().orc_util(grid, maxb)


def n_invocations(grid, tlp, nsms):
    return lib().orc_n_invocations(grid, tlp, nsms)


def rec(M, N, m, n):
    return lib().orc_rec(M, N, m, n)


def opt_sm(grid, tlp, nsms):
    return lib().orc_opt_sm(grid, tlp, nsms)


def run_net(net, weights, biases, x, ranks=None, threads=None,
            return_all=False, perforation=None):
    """Run a synth net description over images x [B,C,H,W] in FP64.

    ranks: optional {layer_index: r} -> the conv/FC weight of that layer is
    replaced by its rank-r operator W_r (reading R7), then the exact layer
    runs with W_r.  Returns the final layer output [B, ...] (float64) and,
    with return_all, the list of every layer's output.
    """
    ranks = ranks or {}
    perforation = perforation or {}       # {layer: (sh, sw)} (NEXT-1, R13)
    a = np.asarray(x, dtype=np.float64)
    outs = []
    for i, L in enumerate(net["layers"]):
        k = L["kind"]
        if k == "conv":
            w = weights[i]
            if i in ranks:
                w, _ = rank_r_conv_weight(w, L["groups"], ranks[i])
            if i in perforation:
                sh, sw = perforation[i]
                a = perforated_conv2d(a, w, biases[i], L["stride"], L["pad"], L["groups"],
                                      L["relu"], sh, sw, threads)
            else:
                a = conv2d(a, w, biases[i], L["stride"], L["pad"], L["groups"],
                           L["relu"], threads)
        elif k == "fc":
            w = weights[i]
            if i in ranks:
                w, _, _ = rank_r(np.asarray(w, dtype=np.float64), ranks[i])
            a = fc(a, w, biases[i], L["relu"], threads)
        elif k == "lrn":
            a = lrn(a, L["size"], L["alpha"], L["beta"], L["k"], threads)
        elif k == "maxpool":
            a = maxpool(a, L["k"], L["stride"], threads)
        elif k == "avgpool":
            a = avgpool(a, L["k"], L["stride"], threads)
        else:
            raise ValueError(k)
        if return_all:
            outs.append(a)
    return (a, outs) if return_all else a
