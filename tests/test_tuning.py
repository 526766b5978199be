"""Entropy-guided greedy accuracy tuning and calibration (Fig. 12,
eq. 14) on hand-made (time, entropy) tables whose outcome is worked out by
hand below -- host logic, no GPU."""
import math

from paper_conf_hpca_songhcl17_b200 import tuning


def table_measure(table):
    def measure(state):
        return table[tuple(sorted(state.items()))]
    return measure


def test_te_score_eq14():
    assert tuning.te_score(10.0, 1.0, 8.0, 1.5) == 4.0          # 2 / 0.5
    assert tuning.te_score(10.0, 1.0, 9.0, 1.0) == math.inf     # free speed-up
    assert tuning.te_score(10.0, 1.0, 11.0, 0.9) == -math.inf


def test_greedy_follows_fig12():
    """Two layers, two rungs each.  Iteration 1: layer A -> TE (10-8)/(1.2-1)
    = 10, layer B -> (10-9)/(1.05-1) = 20: B wins.  Iteration 2 from (0,1):
    A -> (9-6.5)/(1.3-1.05) = 10, B -> (9-8.9)/(1.06-1.05) = 10: tie -> the
    lower layer index (A).  Iteration 3 from (1,1): A's rung 2 exceeds the
    threshold 1.5 (1.6), B -> (6.5-6)/(1.4-1.3) = 5 -> (1,2).  Then A's last
    rung exceeds the threshold: stop."""
    T = {((0, 0), (1, 0)): (10.0, 1.00),
         ((0, 1), (1, 0)): (8.0, 1.20), ((0, 0), (1, 1)): (9.0, 1.05),
         ((0, 1), (1, 1)): (6.5, 1.30), ((0, 0), (1, 2)): (8.9, 1.06),
         ((0, 2), (1, 1)): (5.0, 1.60), ((0, 1), (1, 2)): (6.0, 1.40),
         ((0, 2), (1, 2)): (4.0, 1.70)}
    ladders = {0: [("exact",), ("rank", 64), ("rank", 32)],
               1: [("exact",), ("perf", 1, 2), ("perf", 2, 2)]}
    path = tuning.greedy_tune(ladders, table_measure(T), threshold=1.5)
    assert [p["layer"] for p in path] == [None, 1, 0, 1]
    assert [tuple(sorted(p["state"].items())) for p in path][-1] == ((0, 1), (1, 2))
    assert abs(path[1]["te"] - 20.0) < 1e-9 and abs(path[2]["te"] - 10.0) < 1e-9
    assert abs(path[3]["te"] - 5.0) < 1e-9


def test_calibration_backtracks_with_remeasurement():
    """measure, and while the measured uncertainty is above the
    threshold step back one table and measure AGAIN (hand-worked traces:
    the new inputs make every table 0.3 nats less certain than at tuning)."""
    path = [{"entropy": 1.0}, {"entropy": 1.2}, {"entropy": 1.4}]
    calls = []

    def observe(i):
        calls.append(i)
        return path[i]["entropy"] + 0.3
    idx, trace = tuning.calibrate(path, 2, observe, 1.5)
    assert idx == 1 and calls == [2, 1] and trace == [(2, 1.7), (1, 1.5)]
    # within the threshold: one measurement, stay
    calls.clear()
    idx, trace = tuning.calibrate(path, 2, lambda i: calls.append(i) or 1.45, 1.5)
    assert idx == 2 and calls == [2]
    # never satisfied: every table is measured down to exact, which is kept
    idx, trace = tuning.calibrate(path, 2, lambda i: 9.0, 1.5)
    assert idx == 0 and [t[0] for t in trace] == [2, 1, 0]
    # the shift estimator agrees on the first trace without measuring
    assert tuning.calibrate_estimate(path, 2, 1.6, 1.5) == 1
    assert tuning.calibrate_estimate(path, 2, 3.0, 1.5) == 0


def test_perforation_ladder_rec_rule():
    """W_o H_o (x batch: the GEMM M) a multiple of the tile's n.
    AlexNet conv2 27 x 27 at batch 128: kept grids 14 x 27 (sh = 2) ->
    128 x 378 = 48384 = 378 x 128 (rEC 1); 27 x 14 likewise; 9 x 27 ->
    128 x 243, a multiple of 128 too; every rung has rEC = 1."""
    lad = tuning.perforation_ladder(27, 27, 128)
    assert lad[0] == ("exact",)
    for r in lad[1:]:
        _, sh, sw = r
        kept = -(-27 // sh) * -(-27 // sw)
        assert (128 * kept) % 128 == 0
    # at batch 1 most grids are not multiples of 128: only rEC-1 ones remain
    lad1 = tuning.perforation_ladder(16, 16, 1)
    kept1 = [-(-16 // sh) * -(-16 // sw) for _, sh, sw in lad1[1:]]
    assert kept1 and all(k % 128 == 0 for k in kept1) and kept1 == sorted(kept1, reverse=True)
    assert ("perf", 1, 2) in lad1 and ("perf", 2, 2) not in lad1          # 128 kept vs 64


def test_background_batch_rule():
    """the smallest batch at which every layer's Util (eq. 6) is 1.
    Hand table: layer 0 saturates at 3, layer 1 (the 'last layer') at 5."""
    util = {0: lambda b: min(1.0, b / 3.0), 1: lambda b: min(1.0, b / 5.0)}
    assert tuning.background_batch(lambda l, b: util[l](b), [0, 1], 64) == 5
    assert tuning.background_batch(lambda l, b: 0.5, [0], 8) == 8


def test_eq13_rescale():
    assert tuning.rescale_batch(10.0, 40.0, 64) == 16      # T_user / T = 1/4
    assert tuning.rescale_batch(10.0, 5.0, 64) == 64       # already fast enough
    assert tuning.rescale_batch(1.0, 1000.0, 64) == 1


def test_soc_eq15():
    """eq. 15 and its two factors on hand-worked values."""
    assert tuning.soc_time(0.05, 0.1, 1.0) == 1.0
    assert abs(tuning.soc_time(0.55, 0.1, 1.0) - 0.5) < 1e-12
    assert tuning.soc_time(2.0, 0.1, 1.0) == 0.0
    assert tuning.soc_accuracy(0.4, 0.5) == 1.0
    assert tuning.soc_accuracy(1.0, 0.5) == 0.5
    assert abs(tuning.soc(0.55, 1.0, 2.0, 0.1, 1.0, 0.5) - 0.125) < 1e-12
