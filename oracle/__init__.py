"""AdaInf hot-path ORACLE — TEST INFRASTRUCTURE ONLY.

ctypes binding of ``oracle/oracle.cpp`` (plain C++ direct loops, fp64 accumulation; see that file's
header).  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` leg may import this module.  It shares no code with the CUDA path
(``paper_conf_sigcomm_shubhas23_b200``) and never imports it; model descriptions arrive as plain
dicts (``specs``-style op lists) and are marshalled into the oracle's own ``or_op`` struct here.

Parity status per function (see DESIGN.md §Oracle pins): every function below is pinned by a
``-m "not gpu"`` test in ``tests/test_oracle_*.py``; the paper-level effects (accuracy gains,
finish rates) are OUT of scope and "parity unpinned".
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.cpp")
_lock = threading.Lock()
_lib = None

OR_CONV, OR_MAXPOOL, OR_BLOCK, OR_EXIT, OR_DET_HEAD, OR_SHUFFLE, OR_UPSAMPLE, OR_ROUTE = 0, 1, 2, 3, 4, 5, 6, 7
_KIND = {"conv": OR_CONV, "maxpool": OR_MAXPOOL, "block": OR_BLOCK, "exit": OR_EXIT, "det_head": OR_DET_HEAD,
         "shuffle": OR_SHUFFLE, "upsample": OR_UPSAMPLE, "route": OR_ROUTE}


class OrOp(C.Structure):
    _fields_ = [
        ("kind", C.c_int32), ("kh", C.c_int32), ("kw", C.c_int32), ("stride", C.c_int32),
        ("pad", C.c_int32), ("cout", C.c_int32), ("act", C.c_int32), ("residual", C.c_int32),
        ("num_classes", C.c_int32), ("loss_weight", C.c_float), ("anchors", C.c_int32),
        ("det_classes", C.c_int32), ("grid_stride", C.c_int32), ("anchor_wh", C.c_float * 16),
        ("groups", C.c_int32), ("pool", C.c_int32),
    ]


class OrModel(C.Structure):
    _fields_ = [("in_h", C.c_int32), ("in_w", C.c_int32), ("in_c", C.c_int32), ("n_ops", C.c_int32),
                ("ops", C.POINTER(OrOp))]


def build(force: bool = False) -> str:
    """Compile liboracle.so (plain g++, -O2, no fast-math, no FMA contraction, OpenMP)."""
    with _lock:
        if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < max(
                os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "oracle.h"))):
            cmd = ["g++", "-O2", "-std=c++17", "-fPIC", "-shared", "-fopenmp", "-ffp-contract=off",
                   "-fno-fast-math", "-o", _SO + ".tmp", _SRC]
            subprocess.check_call(cmd)
            os.replace(_SO + ".tmp", _SO)
    return _SO


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_SO)
        f32p, i32p, i8p, u8p, f64p = (C.POINTER(C.c_float), C.POINTER(C.c_int32), C.POINTER(C.c_int8),
                                      C.POINTER(C.c_uint8), C.POINTER(C.c_double))
        mp = C.POINTER(OrModel)
        L.or_bf16.restype = C.c_float
        L.or_bf16.argtypes = [C.c_float]
        L.or_bf16_array.argtypes = [f32p, f32p, C.c_int64]
        L.or_conv_acc.argtypes = [f32p, C.c_int, C.c_int, C.c_int, f32p, C.c_int, C.c_int, C.c_int, C.c_int,
                                  C.c_int, f32p, i32p, i32p]
        L.or_maxpool.argtypes = [f32p, C.c_int, C.c_int, C.c_int, C.c_int, C.c_int, C.c_int, f32p, i32p, i32p]
        L.or_exit_head.argtypes = [f32p, C.c_int, C.c_int, C.c_int, f32p, f32p, C.c_int, f32p, f32p, f32p,
                                   f32p, i32p]
        L.or_softmax_stats.argtypes = [f32p, C.c_int, f32p, f32p, i32p]
        L.or_num_params.restype = C.c_int64
        L.or_num_params.argtypes = [mp]
        L.or_num_exits.argtypes = [mp]
        L.or_tensor_shape.argtypes = [mp, C.c_int, i32p, i32p, i32p]
        L.or_forward.argtypes = [mp, f32p, f32p, C.c_int, f32p, f32p, i32p, f32p, f32p, f32p]
        L.or_exit_assign.argtypes = [f32p, C.c_int, C.c_int, f32p, i8p, i32p, i32p]
        L.or_detect.restype = C.c_int32
        L.or_detect.argtypes = [f32p, C.c_int, C.c_int, C.c_int, C.c_int, f32p, C.c_int, C.c_int, C.c_int,
                                C.c_float, f32p, C.c_int32]
        L.or_nms.restype = C.c_int32
        L.or_nms.argtypes = [f32p, C.c_int32, C.c_float, u8p]
        L.or_iou.restype = C.c_float
        L.or_iou.argtypes = [f32p, f32p]
        L.or_crop.argtypes = [f32p, C.c_int, C.c_int, C.c_int, C.c_float, C.c_float, C.c_float, C.c_float,
                              C.c_int, C.c_int, f32p]
        L.or_select.restype = C.c_int32
        L.or_select.argtypes = [f32p, C.c_int64, C.c_int, f32p, C.c_int, f32p, C.c_int, u8p, C.c_int32, f32p,
                                i32p, f32p]
        L.or_retrain_step.argtypes = [mp, f32p, f32p, f32p, i32p, C.c_int, C.c_int64, C.c_float, C.c_float,
                                      C.c_float, f32p, f64p]
        L.or_loss.restype = C.c_double
        L.or_loss.argtypes = [mp, f64p, f32p, i32p, C.c_int, C.c_int64, C.c_int]
        L.or_grad_exact.argtypes = [mp, f64p, f32p, i32p, C.c_int, C.c_int64, f64p]
        L.or_set_threads.argtypes = [C.c_int]
        L.or_get_threads.restype = C.c_int
        _lib = L
    return _lib


def _p(a, ct):
    return a.ctypes.data_as(C.POINTER(ct)) if a is not None else None


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


class Model:
    """Oracle model built from a spec dict {in_h,in_w,in_c,ops:[{kind:...}, ...]}."""

    def __init__(self, spec: dict):
        ops = spec["ops"]
        self._ops = (OrOp * len(ops))()
        for i, o in enumerate(ops):
            r = self._ops[i]
            r.kind = _KIND[o["kind"]]
            r.kh = o.get("kh", o.get("k", 1))
            r.kw = o.get("kw", o.get("k", 1))
            r.stride = o.get("stride", 1)
            r.pad = o.get("pad", 0)
            r.cout = o.get("cout", 0)
            r.act = o.get("act", 0)
            r.residual = int(o.get("residual", 0))
            r.num_classes = o.get("num_classes", 0)
            r.loss_weight = o.get("loss_weight", 1.0)
            r.anchors = o.get("anchors", 0)
            r.det_classes = o.get("det_classes", 0)
            r.grid_stride = o.get("grid_stride", 0)
            for j, v in enumerate(o.get("anchor_wh", [])):
                r.anchor_wh[j] = v
            r.groups = int(o.get("groups", 1))
            r.pool = int(o.get("pool", 0))
        self.m = OrModel(spec["in_h"], spec["in_w"], spec["in_c"], len(ops), self._ops)
        self.spec = spec
        L = lib()
        self.num_params = int(L.or_num_params(C.byref(self.m)))
        self.num_exits = int(L.or_num_exits(C.byref(self.m)))
        self.ncls = next((o["num_classes"] for o in ops if o["kind"] == "exit"), 0)

    def tensor_shape(self, op_idx):
        H, W, Cc = C.c_int32(), C.c_int32(), C.c_int32()
        rc = lib().or_tensor_shape(C.byref(self.m), op_idx, C.byref(H), C.byref(W), C.byref(Cc))
        assert rc == 0
        return H.value, W.value, Cc.value

    def forward(self, params, x, want_det=False):
        """Full-depth forward: returns dict conf[B,E], ent[B,E], pred[B,E], logits[B,E,ncls], pooled0."""
        params, x = _f32(params), _f32(x)
        B = x.shape[0]
        E, ncls = self.num_exits, self.ncls
        conf = np.zeros((B, E), np.float32)
        ent = np.zeros((B, E), np.float32)
        pred = np.zeros((B, E), np.int32)
        logits = np.zeros((B, E, ncls), np.float32)
        c0 = 0
        for i, o in enumerate(self.spec["ops"]):
            if o["kind"] == "exit":
                c0 = self.tensor_shape(i)[2]
                break
        pooled0 = np.zeros((B, max(c0, 1)), np.float32)
        det = None
        heads = []
        if want_det:
            heads = [self.tensor_shape(i) for i, o in enumerate(self.spec["ops"]) if o["kind"] == "det_head"]
            det = np.zeros((B, sum(G * G2 * CH for G, G2, CH in heads)), np.float32)
        rc = lib().or_forward(C.byref(self.m), _p(params, C.c_float), _p(x, C.c_float), B,
                              _p(conf, C.c_float), _p(ent, C.c_float), _p(pred, C.c_int32),
                              _p(logits, C.c_float), _p(pooled0, C.c_float), _p(det, C.c_float))
        assert rc == 0, rc
        if want_det:  # per head [B, G, G, A*(5+nc)], op order; a single head is returned as the array itself
            outs, o = [], 0
            for G, G2, CH in heads:
                outs.append(det[:, o:o + G * G2 * CH].reshape(B, G, G2, CH).copy())
                o += G * G2 * CH
            det = outs[0] if len(outs) == 1 else outs
        return dict(conf=conf, ent=ent, pred=pred, logits=logits, pooled0=pooled0, det=det)

    def retrain_step(self, params, mom, x, labels, n_global=None, lr=0.01, mu=0.9, wd=0.0):
        params = _f32(params).copy()
        mom = _f32(mom).copy()
        x = _f32(x)
        labels = np.ascontiguousarray(labels, np.int32)
        n = x.shape[0]
        grads = np.zeros(self.num_params, np.float32)
        loss = C.c_double()
        rc = lib().or_retrain_step(C.byref(self.m), _p(params, C.c_float), _p(mom, C.c_float), _p(x, C.c_float),
                                   _p(labels, C.c_int32), n, int(n_global or n), lr, mu, wd,
                                   _p(grads, C.c_float), C.byref(loss))
        assert rc == 0
        return params, mom, grads, loss.value

    def loss(self, params64, x, labels, n_global=None, exact=True):
        p = np.ascontiguousarray(params64, np.float64)
        x = _f32(x)
        labels = np.ascontiguousarray(labels, np.int32)
        return lib().or_loss(C.byref(self.m), _p(p, C.c_double), _p(x, C.c_float), _p(labels, C.c_int32),
                             x.shape[0], int(n_global or x.shape[0]), int(exact))

    def grad_exact(self, params64, x, labels, n_global=None):
        p = np.ascontiguousarray(params64, np.float64)
        x = _f32(x)
        labels = np.ascontiguousarray(labels, np.int32)
        g = np.zeros(self.num_params, np.float64)
        rc = lib().or_grad_exact(C.byref(self.m), _p(p, C.c_double), _p(x, C.c_float), _p(labels, C.c_int32),
                                 x.shape[0], int(n_global or x.shape[0]), _p(g, C.c_double))
        assert rc == 0
        return g


def bf16(x):
    x = _f32(x)
    y = np.empty_like(x)
    lib().or_bf16_array(_p(x, C.c_float), _p(y, C.c_float), x.size)
    return y


def conv_acc(x, w, stride, pad):
    """x: [H,W,C], w: [Co,KH,KW,C] -> fp32 acc [Ho,Wo,Co]."""
    x, w = _f32(x), _f32(w)
    H, W, Cc = x.shape
    Co, KH, KW, _ = w.shape
    Ho, Wo = (H + 2 * pad - KH) // stride + 1, (W + 2 * pad - KW) // stride + 1
    out = np.zeros((Ho, Wo, Co), np.float32)
    a, b = C.c_int32(), C.c_int32()
    lib().or_conv_acc(_p(x, C.c_float), H, W, Cc, _p(w, C.c_float), Co, KH, KW, stride, pad,
                      _p(out, C.c_float), C.byref(a), C.byref(b))
    return out


def maxpool(x, k, stride, pad):
    x = _f32(x)
    H, W, Cc = x.shape
    Ho, Wo = (H + 2 * pad - k) // stride + 1, (W + 2 * pad - k) // stride + 1
    out = np.zeros((Ho, Wo, Cc), np.float32)
    a, b = C.c_int32(), C.c_int32()
    lib().or_maxpool(_p(x, C.c_float), H, W, Cc, k, stride, pad, _p(out, C.c_float), C.byref(a), C.byref(b))
    return out


def exit_head(fmap, Wk, bk):
    fmap, Wk, bk = _f32(fmap), _f32(Wk), _f32(bk)
    H, W, Cc = fmap.shape
    ncls = bk.shape[0]
    pooled = np.zeros(Cc, np.float32)
    logits = np.zeros(ncls, np.float32)
    conf, ent, pred = C.c_float(), C.c_float(), C.c_int32()
    lib().or_exit_head(_p(fmap, C.c_float), H, W, Cc, _p(Wk, C.c_float), _p(bk, C.c_float), ncls,
                       _p(pooled, C.c_float), _p(logits, C.c_float), C.byref(conf), C.byref(ent), C.byref(pred))
    return pooled, logits, conf.value, ent.value, pred.value


def softmax_stats(logits):
    l = _f32(logits)
    conf, ent, pred = C.c_float(), C.c_float(), C.c_int32()
    lib().or_softmax_stats(_p(l, C.c_float), l.shape[0], C.byref(conf), C.byref(ent), C.byref(pred))
    return conf.value, ent.value, pred.value


def exit_assign(conf, tau):
    conf = _f32(conf)
    B, E = conf.shape
    tau = _f32(np.asarray(tau, np.float32).reshape(-1))
    exit_id = np.zeros(B, np.int8)
    surv = np.zeros((max(E - 1, 1), B), np.int32)
    counts = np.zeros(E, np.int32)
    lib().or_exit_assign(_p(conf, C.c_float), B, E, _p(tau, C.c_float), _p(exit_id, C.c_int8),
                         _p(surv, C.c_int32), _p(counts, C.c_int32))
    return exit_id, surv[:E - 1], counts


def detect(raw, anchors, nc, anchor_wh, stride, img_w, img_h, tau_det, max_det=1 << 20):
    raw = _f32(raw)
    B, G, _, _ = raw.shape
    aw = _f32(np.asarray(anchor_wh, np.float32).reshape(-1))
    det = np.zeros((max_det, 9), np.float32)
    n = lib().or_detect(_p(raw, C.c_float), B, G, anchors, nc, _p(aw, C.c_float), stride, img_w, img_h,
                        tau_det, _p(det, C.c_float), max_det)
    return det[:min(n, max_det)].copy(), int(n)


def detect_multi(raws, anchors, nc, anchor_whs, strides, img_w, img_h, tau_det, max_det=1 << 20):
    """Two-scale TinyYOLOv3 decode (NEXT-3, reading Q18c): each head decoded by or_detect on its own grid, the cell
    column re-based to the frame's concatenated cell space (head h's cells follow the G_i^2 cells of heads i < h),
    rows merged in ascending candidate index ((frame * sum_h G_h^2 + cell) * A + anchor): a stable sort as a step."""
    rows, off = [], 0
    cpf = sum(int(r.shape[1]) * int(r.shape[2]) for r in raws)
    total = 0
    for r, aw, st in zip(raws, anchor_whs, strides):
        d, n = detect(r, anchors, nc, aw, st, img_w, img_h, tau_det, max_det)
        total += n
        d = d.copy()
        d[:, 1] += off
        rows.append(d)
        off += int(r.shape[1]) * int(r.shape[2])
    det = np.concatenate(rows, 0) if rows else np.zeros((0, 9), np.float32)
    key = (det[:, 0].astype(np.int64) * cpf + det[:, 1].astype(np.int64)) * anchors + det[:, 2].astype(np.int64)
    order = np.argsort(key, kind="stable")
    return det[order][:max_det].copy(), int(total)


def nms(det, iou_thr):
    """Greedy per-(frame, class) NMS over or_detect rows; returns keep[n] (uint8) and the kept count."""
    det = _f32(det).reshape(-1, 9)
    keep = np.zeros(det.shape[0], np.uint8)
    k = lib().or_nms(_p(det, C.c_float), det.shape[0], float(iou_thr), _p(keep, C.c_uint8))
    return keep, int(k)


def iou(a, b):
    a, b = _f32(a), _f32(b)
    return float(lib().or_iou(_p(a, C.c_float), _p(b, C.c_float)))


def crop(frame, box, crop_h, crop_w):
    frame = _f32(frame)
    H, W, Cc = frame.shape
    out = np.zeros((crop_h, crop_w, Cc), np.float32)
    x0, y0, x1, y1 = [float(np.float32(v)) for v in box]
    lib().or_crop(_p(frame, C.c_float), H, W, Cc, x0, y0, x1, y1, crop_h, crop_w, _p(out, C.c_float))
    return out


def select(X, Wp, ref, k, exclude=None):
    X = _f32(X)
    N, D = X.shape
    Wp_ = _f32(Wp) if Wp is not None else None
    P = Wp_.shape[1] if Wp_ is not None else D
    ref = _f32(ref).reshape(-1, D)
    M = ref.shape[0]
    ex = np.ascontiguousarray(exclude, np.uint8) if exclude is not None else None
    dist = np.zeros(N, np.float32)
    idx = np.zeros(max(k, 1), np.int32)
    dd = np.zeros(max(k, 1), np.float32)
    cnt = lib().or_select(_p(X, C.c_float), N, D, _p(Wp_, C.c_float), P, _p(ref, C.c_float), M,
                          _p(ex, C.c_uint8), k, _p(dist, C.c_float), _p(idx, C.c_int32), _p(dd, C.c_float))
    return idx[:cnt].copy(), dd[:cnt].copy(), int(cnt), dist


def set_threads(n: int):
    lib().or_set_threads(int(n))


def get_threads() -> int:
    return int(lib().or_get_threads())
