"""Run-time management of P-CNN (Fig. 12): entropy-guided greedy
accuracy tuning over each layer's variant ladder, the tuning path it leaves
behind, and calibration by backtracking along that path.

This is host-side control logic over the C ABI: every candidate is executed
by libpcnn's kernels (the network's time comes from CUDA events, its
uncertainty CNN_entropy from the fused softmax + entropy kernel, eq. 2).

* A *ladder* per layer lists variants from exact to most aggressive, e.g.
  ``[("exact",), ("rank", 64), ("rank", 32)]`` or
  ``[("exact",), ("perf", 1, 2), ("perf", 2, 2)]`` (perforation).
* One greedy *iteration* (Fig. 12) tries, for every layer that has a further
  rung, that layer one rung further with all other layers unchanged, and
  scores it with eq. 14:  TE = (T_ori - T_layer) / (H_layer - H_ori);
  the candidate with the largest TE is adopted (a candidate that does not
  raise the entropy has TE = +inf: free speed).  Candidates whose entropy
  exceeds the user's threshold, or that are not faster, are not eligible.
* Tuning stops when no eligible candidate remains.  Each adopted state is a
  *tuning table*: the per-layer rungs plus every layer's optSM (eq. 11) for
  the run-time kernel scheduler.
* *Calibration* (P:345): at run time P-CNN monitors the output uncertainty;
  while it exceeds the threshold, it switches to the previous (slower, more
  precise) table of the tuning path and measures again, until the measured
  uncertainty is below the threshold or the exact table is reached.
* P:335's rEC rule: the perforation rungs are chosen so that the GEMM's M
  dimension (B x W'_o H'_o) is a multiple of the tile's M (eq. 9, rEC = 1).
"""
import math


def te_score(t_ori, h_ori, t_new, h_new):
    """eq. 14.  +inf when the candidate is faster without raising entropy."""
    dh = h_new - h_ori
    dt = t_ori - t_new
    if dh <= 0:
        return math.inf if dt > 0 else -math.inf
    return dt / dh


def greedy_tune(ladders, measure, threshold, max_iters=64):
    """Fig. 12.  ladders: {layer: [variant, ...]} (rung 0 = exact);
    measure(state) -> (time, entropy) for a state {layer: rung}.
    Returns the tuning path: a list of dicts {"state", "time", "entropy", "te",
    "layer"} starting with the all-exact state."""
    state = {l: 0 for l in ladders}
    t0, h0 = measure(dict(state))
    path = [{"state": dict(state), "time": t0, "entropy": h0, "te": None, "layer": None}]
    for _ in range(max_iters):
        t_ori, h_ori = path[-1]["time"], path[-1]["entropy"]
        best = None
        for l, rungs in ladders.items():
            if state[l] + 1 >= len(rungs):
                continue
            cand = dict(state)
            cand[l] += 1
            t, h = measure(cand)
            if h > threshold or t >= t_ori:
                continue
            te = te_score(t_ori, h_ori, t, h)
            if best is None or te > best[0] or (te == best[0] and l < best[1]):
                best = (te, l, cand, t, h)
        if best is None:
            break
        te, l, cand, t, h = best
        state = cand
        path.append({"state": dict(state), "time": t, "entropy": h, "te": te, "layer": l})
    return path


def calibrate(path, index, observe, threshold):
    """P:345 ("monitors the uncertainty of the output ... switches to a slower
    but more precise version ... by backtracking along the tuning path ...
    until the output uncertainty is less than the pre-defined threshold").

    observe(index) programs table `index` of the path and returns the
    CNN_entropy the current inputs produce under it (a measurement, eq. 2).
    Starting from the current table, while the measured entropy exceeds the
    threshold, step back one table and measure again.  Returns (index, trace)
    where trace lists every (index, measured entropy) visited."""
    h = observe(index)
    trace = [(index, h)]
    while h > threshold and index > 0:
        index -= 1
        h = observe(index)
        trace.append((index, h))
    return index, trace


def calibrate_estimate(path, index, observed_entropy, threshold):
    """Cheap predictor for calibrate (no re-measurement): shift the tuned
    entropies by (observed - tuned) at the current index and back-track while
    the shifted value exceeds the threshold."""
    shift = observed_entropy - path[index]["entropy"]
    while index > 0 and path[index]["entropy"] + shift > threshold:
        index -= 1
    return index


def perforation_ladder(out_h, out_w, batch, tile_m=128, max_step=4, rec_min=1.0):
    """Perforation rungs of one conv layer honouring P:335 ("make sure that
    W_o H_o ... is a multiple of n", reading R13 / eq. 9): the grid steps
    (sh, sw) in 1..max_step whose kept positions give a GEMM M = batch x
    ceil(H/sh) x ceil(W/sw) with rEC >= rec_min for the tile M, ordered from
    exact to the highest perforation rate (ties: fewer kept rows first kept).
    Returns [("exact",), ("perf", sh, sw), ...]."""
    cands = []
    for sh in range(1, max_step + 1):
        for sw in range(1, max_step + 1):
            if sh * sw == 1:
                continue
            kept = -(-out_h // sh) * -(-out_w // sw)
            m = batch * kept
            rec = m / (-(-m // tile_m) * tile_m)
            if rec >= rec_min - 1e-12:
                cands.append((kept, sh, sw))
    cands.sort(key=lambda c: (-c[0], c[1], c[2]))
    return [("exact",)] + [("perf", sh, sw) for _, sh, sw in cands]


def apply_state(net, ladders, state, batch=None):
    """Program a libpcnn Net with the rungs of `state` (and, given a batch,
    every GEMM layer's eq. 11 optSM budget)."""
    for l, rung in state.items():
        v = ladders[l][rung]
        net.set_variant(l, "exact")
        if v[0] == "rank":
            net.set_variant(l, "rank", v[1])
        elif v[0] == "perf":
            net.set_perforation(l, v[1], v[2])
    if batch is not None:
        net.apply_opt_budgets(batch)


def gpu_observe(net, ladders, path, images):
    """observe() for calibrate on the GPU: program table `index` of the path
    and return the mean CNN_entropy (eq. 2, the fused softmax + entropy
    kernel) of the current inputs."""
    def observe(index):
        apply_state(net, ladders, path[index]["state"])
        _, _, ent = net.infer(images, entropy=True)
        return float(ent.mean().item())
    return observe


def gpu_measure(net, ladders, images, reps=10):
    """measure() for greedy_tune on the GPU: mean time per pass (CUDA events)
    and mean CNN_entropy (eq. 2) of the calibration images."""
    import torch

    def measure(state):
        apply_state(net, ladders, state)
        out, _, ent = net.infer(images, entropy=True)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            net.infer(images, out=out, entropy=ent)
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / reps, float(ent.mean().item())
    return measure


# ---------------------------------------------------------------- batch selection (NEXT-4)
def background_batch(util_of_layer, layers, max_batch):
    """P:259 (background task): the optimal batch is the smallest one at which
    every GEMM layer -- in practice the last, least-utilised one (Table V) --
    reaches Util = 1 (eq. 6); beyond it throughput cannot grow.  util_of_layer
    (layer, batch) -> eq. 6 Util.  Returns max_batch when no batch reaches 1."""
    for bsz in range(1, max_batch + 1):
        if all(util_of_layer(l, bsz) >= 1.0 - 1e-9 for l in layers):
            return bsz
    return max_batch


def rescale_batch(t_user, t_model, batch):
    """eq. 13: new batch size = T_user / T x batch (floored, >= 1),
    applied when the modelled time T exceeds the user's requirement."""
    if t_model <= t_user:
        return batch
    return max(1, int(math.floor(t_user / t_model * batch)))


# ---------------------------------------------------------------- SoC (NEXT-4, eq. 15)
def soc_time(t, t_i, t_t):
    """P:69 / P:364: 1 in the imperceptible region (0, T_i], 0 in the
    unusable region (T_t, inf), linear in between (reading R15: linear from
    1 at T_i to 0 at T_t)."""
    if t <= t_i:
        return 1.0
    if t >= t_t:
        return 0.0
    return (t_t - t) / (t_t - t_i)


def soc_accuracy(entropy, threshold):
    """1 when CNN_entropy <= CNN_threshold, else threshold / entropy."""
    return 1.0 if entropy <= threshold else threshold / entropy


def soc(t, entropy, energy_j, t_i, t_t, threshold):
    """eq. 15: SoC = SoC_time x SoC_accuracy / energy consumption."""
    return soc_time(t, t_i, t_t) * soc_accuracy(entropy, threshold) / energy_j


class EnergyMeter:
    """Board energy from NVML's total-energy counter (mJ since driver load;
    SM power gating is not software-controllable on B200, so this is the
    board-level figure eq. 15 divides by).  Unavailable -> None."""

    def __init__(self, device=0):
        self.h = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self._nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device)
            pynvml.nvmlDeviceGetTotalEnergyConsumption(self.h)
        except Exception:
            self.h = None

    def read_j(self):
        if self.h is None:
            return None
        return self._nv.nvmlDeviceGetTotalEnergyConsumption(self.h) / 1000.0
