"""Incremental-retraining planning (include/adainf_sched.h) through the C-ABI, host-only
(no GPU needed): the spare-time split pinned to the paper's worked example and its formula, and the retraining
setting a time allocation affords (reading in DESIGN.md)."""
import math

import pytest

from paper_conf_sigcomm_shubhas23_b200 import binding as B


def test_spare_time_worked_example_p51():
    """a 400 ms SLO with 200 ms of inference leaves 200 ms of retraining; 300 ms leaves 100 ms."""
    tr, alloc = B.time_split(400.0, [200.0], [1.0])
    assert tr == 200.0 and alloc == [200.0]
    tr, alloc = B.time_split(400.0, [300.0], [1.0])
    assert tr == 100.0 and alloc == [100.0]


def test_spare_time_sums_dag_inference_tasks():
    """T_r = L_s - sum_k l_k over all inference tasks of the job (detector + two classifiers)."""
    tr, _ = B.time_split(500.0, [120.0, 80.5, 60.25], [])
    assert tr == 500.0 - (120.0 + 80.5 + 60.25)


def test_split_by_impact_degree_p237():
    """T_r * d_j / sum_j d_j; vehicle 0.15 : person 0.09 (the P:86-90 accuracy losses) -> 5:3."""
    tr, alloc = B.time_split(400.0, [240.0], [0.15, 0.09])
    assert tr == 160.0
    assert alloc[0] == pytest.approx(100.0, rel=1e-12) and alloc[1] == pytest.approx(60.0, rel=1e-12)
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
    PERSON, VEHICLE = 1, 2
    seq = [0, PERSON, PERSON | VEHICLE, PERSON | VEHICLE, PERSON | VEHICLE, PERSON | VEHICLE]
    stops = [B.drift_should_stop(seq[:i + 1], n=4) for i in range(len(seq))]
    assert stops == [False, False, False, False, False, True]  # 3, 6, 9, 12, 15 -> continue; 18% -> stop
    assert not B.drift_should_stop([], n=4)
    assert B.drift_should_stop([5], n=1)
    assert not B.drift_should_stop([1, 1, 2, 1], n=2)
