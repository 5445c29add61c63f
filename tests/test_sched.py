"""Incremental-retraining planning (include/adainf_sched.h) through the C-ABI, host-only
(no GPU needed): the spare-time split pinned to the paper's worked example and its formula, and the retraining
setting a time allocation affords (reading in DESIGN.md)."""
import json
import math
import os

import numpy as np

import pytest

from paper_conf_sigcomm_shubhas23_b200 import binding as B

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def _golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def test_spare_time_worked_example_p51():
    """a 400 ms SLO with 200 ms of inference leaves 200 ms of retraining; 300 ms leaves 100 ms
    (tests/golden/p51_incremental_retraining.json)."""
    g = _golden("p51_incremental_retraining.json")
    for c in g["cases"]:
        tr, alloc = B.time_split(g["slo_ms"], c["inference_ms"], [1.0])
        assert tr == c["retrain_ms"] and alloc == [c["retrain_ms"]]


def test_spare_time_sums_dag_inference_tasks():
    """T_r = L_s - sum_k l_k over all inference tasks of the job (detector + two classifiers)."""
    tr, _ = B.time_split(500.0, [120.0, 80.5, 60.25], [])
    assert tr == 500.0 - (120.0 + 80.5 + 60.25)


def test_split_by_impact_degree_p237():
    """T_r * d_j / sum_j d_j; vehicle 0.15 : person 0.09 (the P:86-90 accuracy losses) -> 5:3."""
    g = _golden("p237_impact_split.json")
    d, want = g["impact_degrees"], g["expected_alloc_ms"]
    tr, alloc = B.time_split(g["slo_ms"], g["inference_ms"], [d["vehicle_type"], d["person_activity"]])
    assert tr == g["expected_retrain_total_ms"]
    assert alloc[0] == pytest.approx(want["vehicle_type"], rel=1e-12)
    assert alloc[1] == pytest.approx(want["person_activity"], rel=1e-12)
    assert math.isclose(sum(alloc), tr, rel_tol=1e-12)
    # a model not impacted by drift gets no retraining time (Observation 2)
    _, alloc = B.time_split(400.0, [240.0], [0.15, 0.0])
    assert alloc == [160.0, 0.0]


def test_slo_shorter_than_inference_and_degenerate_cases():
    assert B.time_split(100.0, [150.0], [1.0]) == (0.0, [0.0])
    assert B.time_split(400.0, [200.0], [0.0, 0.0]) == (200.0, [0.0, 0.0])
    assert B.time_split(400.0, [], []) == (400.0, [])
    for bad in ([-1.0], [float("nan")]):
        with pytest.raises(B.AdaInfError) as ei:
            B.time_split(400.0, bad, [1.0])
        assert ei.value.code == B.ERR_INVALID
    with pytest.raises(B.AdaInfError):
        B.time_split(400.0, [1.0], [-0.5])


def test_retrain_setting_maximises_sample_visits():
    batches, ms = [128, 256, 512, 1024], [3.0, 5.0, 9.0, 17.0]
    # 40 ms: 13 x 128 = 1664, 8 x 256 = 2048, 4 x 512 = 2048 (tie -> larger batch), 2 x 1024 = 2048 (larger still)
    plan = B.retrain_setting(40.0, batches, ms, eligible=100000, max_batch=1024)
    assert plan == {"samples": 2048, "batch": 1024, "steps": 2, "epochs": 1, "est_ms": 34.0}
    # max_batch caps the choice; 35 ms: 11 x 128 = 1408, 7 x 256 = 1792, 3 x 512 = 1536
    plan = B.retrain_setting(35.0, batches, ms, eligible=100000, max_batch=512)
    assert (plan["batch"], plan["steps"], plan["samples"], plan["epochs"]) == (256, 7, 1792, 1)


def test_retrain_setting_epochs_when_pool_is_small_and_nothing_fits():
    plan = B.retrain_setting(100.0, [256], [5.0], eligible=1000, max_batch=1024)
    assert (plan["steps"], plan["samples"], plan["epochs"]) == (20, 1000, 6)  # 5120 visits over 1000 samples
    plan = B.retrain_setting(2.0, [256], [5.0], eligible=1000, max_batch=1024)
    assert plan["samples"] == 0 and plan["steps"] == 0
    plan = B.retrain_setting(100.0, [256], [5.0], eligible=100, max_batch=1024)  # fewer eligible than a batch
    assert plan["samples"] == 0


def test_drift_stop_rule_table2():
    """Table 2, S = 3%, 6%, ... of the retraining samples: the impacted set is {} at 3% (reading of
    the garbled cell), {Person} at 6%, {Person, Vehicle} from 9%; the process stops at 18% - the first S whose
    result equals the previous ones for 4 consecutive values - and not before."""
    g = _golden("table2_drift_stop.json")
    bit = {"Person": 1, "Vehicle": 2}
    seq = [sum(bit[m] for m in s) for s in g["impacted"]]
    stops = [B.drift_should_stop(seq[:i + 1], n=g["repeat_n"]) for i in range(len(seq))]
    first = g["S_percent"][stops.index(True)]
    assert first == g["stops_at_percent"]  # 3, 6, 9, 12, 15 -> continue; 18% -> stop
    assert not any(stops[:g["S_percent"].index(first)])
    assert seq[g["S_percent"].index(first)] == seq[-1]  # the same result as S = 100%
    assert not B.drift_should_stop([], n=4)
    assert B.drift_should_stop([5], n=1)
    assert not B.drift_should_stop([1, 1, 2, 1], n=2)


# ---- NEXT-4: batch size and structure from latency profiles ----
def _brute_batch(batches, ms, R):
    w = [(t * -(-R // b), b) for b, t in zip(batches, ms)]
    return min(w)[1], min(w)[0]


def test_pick_batch_worst_case_definition_and_brute_force():
    """W(b) = per-batch latency x number of batches; the batch minimising W, ties -> smaller."""
    from paper_conf_sigcomm_shubhas23_b200 import binding as B
    batches = [1, 2, 4, 8, 16, 32, 64]
    # a per-batch latency with a fixed launch cost and a linear part: W(b) = (a + c b) ceil(R / b)
    for a, c, R in ((2.0, 0.5, 100), (0.1, 1.0, 64), (5.0, 0.01, 1000), (1.0, 1.0, 1)):
        ms = [a + c * b for b in batches]
        got = B.pick_batch(batches, ms, R)
        assert got[0] == _brute_batch(batches, ms, R)[0]
        assert abs(got[1] - _brute_batch(batches, ms, R)[1]) < 1e-12
    # closed form: a = 3, c = 1, R = 64 -> W(b) = (3 + b) 64 / b for b | 64, minimised at the largest b
    b, w = B.pick_batch([4, 8, 16, 32, 64], [7.0, 11.0, 19.0, 35.0, 67.0], 64)
    assert b == 64 and w == 67.0
    # ragged last batch counts as a whole batch: R = 17 at b = 16 -> 2 batches
    b, w = B.pick_batch([16, 17], [1.0, 1.5], 17)
    assert b == 17 and w == 1.5
    # tie -> smaller batch
    assert B.pick_batch([8, 16], [2.0, 4.0], 16) == (8, 4.0)
    rng = np.random.default_rng(0)
    for _ in range(200):
        bs = sorted(set(rng.integers(1, 129, 6).tolist()))
        ms = rng.uniform(0.1, 10, len(bs)).tolist()
        R = int(rng.integers(1, 5000))
        gb, gw = B.pick_batch(bs, ms, R)
        eb, ew = _brute_batch(bs, ms, R)
        assert gb == eb and abs(gw - ew) < 1e-9 * ew


def test_pick_structure_rules():
    """no retraining task -> full structure; else the lowest per-batch latency among structures with
    accuracy >= A_m (at the job's batch), then the batch re-picked for that structure; none qualifies -> full."""
    from paper_conf_sigcomm_shubhas23_b200 import binding as B
    batches = [8, 16, 32]
    tables = [([8, 16, 32], [1.0, 1.5, 2.5]),    # truncate at exit 0: fastest, least accurate
              ([8, 16, 32], [1.6, 2.4, 4.2]),
              ([8, 16, 32], [2.0, 3.0, 5.0])]    # full structure
    acc = [0.70, 0.85, 0.90]
    # no retraining task: the full structure regardless of A_m
    s, b, w = B.pick_structure(tables, acc, 0.5, 0, 2, 16, 100)
    assert s == 2 and (b, w) == _brute_batch(batches, tables[2][1], 100)
    # A_m = 0.8: structures 1 and 2 qualify, 1 is faster at batch0
    s, b, w = B.pick_structure(tables, acc, 0.8, 1, 2, 16, 100)
    assert s == 1 and (b, w) == _brute_batch(batches, tables[1][1], 100)
    # A_m = 0.6: all qualify -> structure 0
    assert B.pick_structure(tables, acc, 0.6, 1, 2, 16, 100)[0] == 0
    # A_m above every accuracy: fall back to the full structure
    assert B.pick_structure(tables, acc, 0.95, 1, 2, 16, 100)[0] == 2
    # the choice is made at batch0: a structure faster at 8 but slower at 16 loses when batch0 = 16
    t2 = [([8, 16], [1.0, 5.0]), ([8, 16], [1.2, 2.0]), ([8, 16], [3.0, 6.0])]
    assert B.pick_structure(t2, [0.9, 0.9, 0.9], 0.5, 1, 2, 16, 64)[0] == 1
    assert B.pick_structure(t2, [0.9, 0.9, 0.9], 0.5, 1, 2, 8, 64)[0] == 0
    with pytest.raises(B.AdaInfError):
        B.pick_structure(tables, acc, 0.5, 1, 2, 12, 100)  # batch0 not profiled
    with pytest.raises(B.AdaInfError):
        B.pick_batch([4, 8], [1.0, -1.0], 10)


def test_app_placement_and_dp_rows():
    """BASELINE config 4: app i -> GPU i mod G, every application on exactly one GPU, loads within one
    application of each other; each retraining task's rows split index mod G, disjoint and covering."""
    from paper_conf_sigcomm_shubhas23_b200.driver import dp_rows, place_apps
    for world in (1, 2, 3, 4, 8):
        pl = place_apps(8, world)
        flat = sorted(a for r in pl for a in r)
        assert flat == list(range(8))
        assert max(map(len, pl)) - min(map(len, pl)) <= 1
        assert all(a % world == r for r, apps in enumerate(pl) for a in apps)
        for n in (1, 341, 640, 1024):
            rows = [dp_rows(n, r, world) for r in range(world)]
            assert sorted(x for rr in rows for x in rr) == list(range(n))
