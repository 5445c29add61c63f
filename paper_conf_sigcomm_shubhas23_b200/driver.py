"""Incremental-retraining job driver: one job of an application executed along its
retraining -> inference DAG (Fig. 15), every compute step a libadainf.so call:

  1. spare time T_r = L_s - sum_k l_k and its split by impact degree      adainf_time_split
  2. per retraining task: start from the mean of concurrent versions       adainf_model_average
  3. retraining setting the allocation affords under the measured profile adainf_retrain_setting
  4. the R most divergent eligible samples, then mark them used            adainf_select_retrain,
                                                                           adainf_mark_used
  5. SGD steps over batches of the selected samples                        adainf_gather_rows,
                                                                           adainf_retrain_step
  6. inference of the DAG with the retrained models                        adainf_infer_dag

The host only plans (no device read-back on the path: the number of eligible samples is tracked on the host
from the selection sizes it requested).  Latency profiles (NEXT-4) are measured with CUDA events on the
launching stream.
"""
from __future__ import annotations

from dataclasses import dataclass, field

from . import binding as B


def place_apps(n_apps: int, world: int):
    """Application placement (BASELINE config 4): app i -> GPU i mod G.  A DAG's models stay on one GPU,
    so routing never crosses devices (the B200 analogue of the paper's GPU-space division, done by placement
    instead of MPS percentages).  Returns, per rank, the list of its applications."""
    if n_apps < 0 or world < 1:
        raise ValueError("place_apps: n_apps >= 0, world >= 1")
    return [[i for i in range(n_apps) if i % world == r] for r in range(world)]


def dp_rows(n: int, rank: int, world: int):
    """Rows of a retraining task's n selected samples that rank `rank` trains on: index mod G (no sample is
    used by two replicas), gradients scaled by 1/n and all-reduced."""
    return list(range(rank, n, world))


@dataclass
class RetrainTask:
    model: "B.Model"
    impact: float                 # impact degree d_j = I_m - I'_m
    pool_x: object                # device bf16 [N][H][W][C] retraining pool (new samples of period T-1)
    pool_y: object                # device int32 [N] labels (reading Q25)
    emb: object                   # device bf16 [N][D] pool feature vectors (reading Q12)
    pca: object                   # device bf16 [D][P] or None
    ref: object                   # device fp32 [M][D] mean feature vector(s) of the old samples
    exclude: object               # device uint8 [N], shared by the jobs of the application
    eligible: int                 # host count of samples not yet used
    lr: float = 0.01
    versions: list = field(default_factory=list)  # concurrent versions of the model
    profile_batches: list = field(default_factory=list)
    profile_ms: list = field(default_factory=list)


def _elapsed(fn, reps, stream=None):
    import torch
    s = stream or torch.cuda.current_stream()
    fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(reps):
        fn()
    e1.record(s)
    e1.synchronize()
    return e0.elapsed_time(e1) / reps


def profile_retrain(model, x, y, batches, reps=3):
    """NEXT-4: measured ms per retrain_step at each batch size (lr 0: parameters unchanged)."""
    return [_elapsed(lambda b=b: model.retrain_step(x[:b], y[:b], n_global=b, lr=0.0), reps) for b in batches]


def profile_infer(app, x, taus, outs, reps=3):
    """NEXT-4: measured ms of one DAG inference call on batch x."""
    outs = outs if isinstance(outs, list) else [outs]
    return _elapsed(lambda: app.infer(x, taus, outs), reps)


def run_job(app, batch, taus, outs, slo_ms, infer_ms, tasks, sel_idx, sel_cnt, rt_x, rt_y):
    """Execute one job: retraining tasks (time split, version averaging, selection, SGD), then inference.
    sel_idx / sel_cnt / rt_x / rt_y are caller-owned device work buffers (capacity = the largest plan and
    batch).  Returns the plan and the device time the retraining took (CUDA events)."""
    import torch
    tr, alloc = B.time_split(slo_ms, infer_ms, [t.impact for t in tasks])
    report = {"spare_ms": tr, "alloc_ms": alloc, "plans": [], "retrain_ms": 0.0}
    s = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for t, a in zip(tasks, alloc):
        if t.versions:
            B.model_average(t.model, t.versions)
        plan = B.retrain_setting(a, t.profile_batches, t.profile_ms, t.eligible, t.model.max_batch)
        report["plans"].append(plan)
        R, b = plan["samples"], plan["batch"]
        if R == 0:
            continue
        idx = sel_idx[:R]
        B.select_retrain(t.emb, t.pca, t.ref, R, exclude=t.exclude, out_idx=idx, out_count=sel_cnt)
        B.mark_used(t.exclude, idx, sel_cnt)
        t.eligible -= R
        done = 0
        while done < plan["steps"]:
            for s0 in range(0, R, b):
                if done == plan["steps"]:
                    break
                n = min(b, R - s0)
                B.gather_rows(t.pool_x, idx[s0:s0 + n], None, n, rt_x)
                B.gather_rows(t.pool_y, idx[s0:s0 + n], None, n, rt_y)
                t.model.retrain_step(rt_x[:n], rt_y[:n], n_global=n, lr=t.lr)
                done += 1
    e1.record(s)
    app.infer(batch, taus, outs if isinstance(outs, list) else [outs])
    e1.synchronize()
    report["retrain_ms"] = e0.elapsed_time(e1)
    return report


@dataclass
class DriftModel:
    """One model of an application for the drift-impact check."""
    app: "B.App"                  # single-model app used for the full-structure inference
    model: "B.Model"
    initial_acc: float            # I_m, accuracy of the initially trained version
    emb: object                   # device bf16 [N][D] feature vectors of the new samples
    pca: object                   # device bf16 [D][P] or None
    ref: object                   # device fp32 [1][D] mean feature vector of the old training samples
    pool_x: object                # device bf16 [N][H][W][C] new samples
    pool_y: object                # device int32 [N] their labels (reading Q25)


def detect_drift(models, fractions=(0.03, 0.06, 0.09, 0.12, 0.15, 0.18, 0.21, 0.24, 0.27, 0.30), n_unchanged=4):
    """NEXT-2 (Table 2): for S = 3%, 6%, ... of the new samples, pick the S most divergent ones (cosine
    distance to the old mean after PCA, adainf_select_retrain), predict them with the model's FULL structure
    (every early exit disabled), accuracy I'_m (adainf_count_correct); model m is impacted iff
    I'_m < I_m.  Stop when the impacted set is unchanged for n consecutive values of S
    (adainf_drift_should_stop).  Returns the impacted bit set, the impact degrees I_m - I'_m at the last S, and
    the per-S trace.  Runs at scheduling time (once per period), so it reads the counts back to the host."""
    import torch
    trace, results = [], []
    degrees = [0.0] * len(models)
    for frac in fractions:
        mask = 0
        accs = []
        for j, dm in enumerate(models):
            N = dm.emb.shape[0]
            S = max(1, int(round(frac * N)))
            if S > dm.model.max_batch:
                raise ValueError("detect_drift: S exceeds the model's max_batch")
            idx, _, cnt = B.select_retrain(dm.emb, dm.pca, dm.ref, S)
            dev = dm.pool_x.device
            xs = torch.empty((S,) + tuple(dm.pool_x.shape[1:]), dtype=dm.pool_x.dtype, device=dev)
            ys = torch.empty(S, dtype=torch.int32, device=dev)
            B.gather_rows(dm.pool_x, idx, cnt, S, xs)
            B.gather_rows(dm.pool_y, idx, cnt, S, ys)
            outs = B.alloc_outs(dm.model, S)
            E = dm.model.num_exits
            dm.app.infer(xs, [2.0] * (E - 1), [outs])  # tau > 1 disables every early exit: the full structure
            correct = int(B.count_correct(outs["pred"][:S], ys).item())
            acc = correct / S
            accs.append(acc)
            degrees[j] = dm.initial_acc - acc
            if acc < dm.initial_acc:
                mask |= 1 << j
        results.append(mask)
        trace.append({"fraction": frac, "impacted": mask, "acc": accs})
        if B.drift_should_stop(results, n_unchanged):
            break
    return results[-1], degrees, trace


# ------------------------------------------------------------------------------------------------
# NEXT-4: B200 latency profiles of early-exit structures and the structure / batch-size choice (P:118-134,
# P:221-231).  Measurement is on the device (CUDA events); the choice is adainf_pick_structure / _pick_batch.
def early_exit_structures(num_exits):
    """The structures of an early-exit model as threshold vectors (reading Q2): "truncate at exit k" = tau_k = 0
    with the earlier exits disabled (tau > 1), k = 0..E-2, then the full structure (every exit disabled), which
    is the last entry (index E-1)."""
    E = num_exits
    out = []
    for k in range(E - 1):
        t = [2.0] * (E - 1)
        t[k] = 0.0
        out.append(t)
    out.append([2.0] * (E - 1))
    return out


def profile_structures(app, x, structures, batches, outs, reps=3):
    """Per-batch inference latency table [structure][batch] (ms, whole GPU, CUDA events on the stream): the
    offline profiling of P:221 / P:229 re-measured on this B200."""
    return [[profile_infer(app, x[:b], taus, outs, reps) for b in batches] for taus in structures]


def structure_accuracy(app, x, y, structures, outs):
    """Accuracy of each structure on labelled samples (stored accuracy, refreshed on the S new samples);
    correct predictions counted on the device (adainf_count_correct)."""
    n = x.shape[0]
    acc = []
    for taus in structures:
        app.infer(x, taus, [outs])
        acc.append(int(B.count_correct(outs["pred"][:n], y).item()) / n)
    return acc


def plan_inference(batches, tables, accuracy, a_min, has_retraining, requests):
    """Structure + request batch size for one inference task: batch0 from the full structure's table
    (the initial DAG, §3.3.1), then adainf_pick_structure (accuracy >= A_m, lowest per-batch latency at batch0;
    the batch re-picked for the chosen structure).  Returns (structure index, batch, worst-case ms)."""
    full = len(tables) - 1
    batch0, _ = B.pick_batch(batches, tables[full], requests)
    return B.pick_structure([(batches, t) for t in tables], accuracy, a_min, has_retraining, full, batch0, requests)
