"""Thin ctypes binding of libadainf.so (argument marshalling only; every step runs in the library's
sm_100a kernels).  Names mirror include/adainf.h.  There is no fallback: if the shared library is
missing or the device is not sm_100, calls raise AdaInfError.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

from . import specs as S

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libadainf.so")

OK, ERR_INVALID, ERR_SHAPE, ERR_CAPACITY, ERR_OOM, ERR_CUDA, ERR_NCCL, ERR_UNSUPPORTED = 0, -1, -2, -3, -4, -5, -6, -7
_OPKIND = {"conv": 0, "maxpool": 1, "block": 2, "exit": 3, "det_head": 4, "shuffle": 5, "upsample": 6, "route": 7}
ROUTE_DET_CROP, ROUTE_CLASS_WHOLE = 0, 1


class AdaInfError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"adainf status {code}: {msg}")
        self.code = code


class Op(C.Structure):
    _fields_ = [("kind", C.c_int32), ("kh", C.c_int32), ("kw", C.c_int32), ("stride", C.c_int32),
                ("pad", C.c_int32), ("cout", C.c_int32), ("act", C.c_int32), ("residual", C.c_int32),
                ("num_classes", C.c_int32), ("loss_weight", C.c_float), ("anchors", C.c_int32),
                ("det_classes", C.c_int32), ("grid_stride", C.c_int32), ("anchor_wh", C.c_float * 16),
                ("nms_iou", C.c_float), ("groups", C.c_int32), ("pool", C.c_int32)]


class ModelSpec(C.Structure):
    _fields_ = [("in_h", C.c_int32), ("in_w", C.c_int32), ("in_c", C.c_int32), ("max_batch", C.c_int32),
                ("n_ops", C.c_int32), ("ops", C.POINTER(Op)), ("momentum", C.c_float),
                ("weight_decay", C.c_float), ("seed", C.c_uint64), ("init_params", C.POINTER(C.c_float)),
                ("device", C.c_int32)]


class Edge(C.Structure):
    _fields_ = [("src_model", C.c_int32), ("dst_model", C.c_int32), ("kind", C.c_int32),
                ("src_class", C.c_int32), ("crop_h", C.c_int32), ("crop_w", C.c_int32)]


class AppSpec(C.Structure):
    _fields_ = [("n_models", C.c_int32), ("models", C.POINTER(C.c_void_p)), ("n_edges", C.c_int32),
                ("edges", C.POINTER(Edge)), ("max_routed_per_dst", C.c_int32)]


class ModelOut(C.Structure):
    _fields_ = [("exit_id", C.c_void_p), ("pred", C.c_void_p), ("conf", C.c_void_p), ("entropy", C.c_void_p),
                ("logits", C.c_void_p), ("exit_counts", C.c_void_p), ("surv_idx", C.c_void_p),
                ("embed", C.c_void_p), ("n_det", C.c_void_p), ("det_table", C.c_void_p), ("max_det", C.c_int32),
                ("route_idx", C.c_void_p), ("n_routed", C.c_void_p)]


class RetrainProfile(C.Structure):
    _fields_ = [("n", C.c_int32), ("batch", C.POINTER(C.c_int32)), ("step_ms", C.POINTER(C.c_double))]


class RetrainPlan(C.Structure):
    _fields_ = [("samples", C.c_int32), ("batch", C.c_int32), ("steps", C.c_int32), ("epochs", C.c_int32),
                ("est_ms", C.c_double)]


class LatencyProfile(C.Structure):
    _fields_ = [("n", C.c_int32), ("batch", C.POINTER(C.c_int32)), ("per_batch_ms", C.POINTER(C.c_double))]


class SelectIn(C.Structure):
    _fields_ = [("X_bf16", C.c_void_p), ("N", C.c_int64), ("D", C.c_int32), ("W_bf16", C.c_void_p),
                ("P", C.c_int32), ("ref", C.c_void_p), ("M", C.c_int32), ("exclude", C.c_void_p)]


_lib = None


def lib():
    """Load libadainf.so (fails loudly when absent: no fallback path exists)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise AdaInfError(ERR_UNSUPPORTED, f"{LIB_PATH} missing: run __graft_entry__.build()")
        L = C.CDLL(LIB_PATH)
        vp, i32, i64 = C.c_void_p, C.c_int32, C.c_int64
        L.adainf_last_error.restype = C.c_char_p
        L.adainf_version.restype = C.c_int32
        L.adainf_launch_count.restype = C.c_int64
        for name, args in {
            "adainf_model_create": [C.POINTER(ModelSpec), C.POINTER(vp)],
            "adainf_model_destroy": [vp],
            "adainf_model_num_params": [vp, C.POINTER(i64)],
            "adainf_model_num_exits": [vp, C.POINTER(i32)],
            "adainf_model_get_params": [vp, C.POINTER(C.c_float), i64],
            "adainf_model_set_params": [vp, C.POINTER(C.c_float), i64],
            "adainf_model_grad_ptr": [vp, C.POINTER(vp)],
            "adainf_model_get_grads": [vp, C.POINTER(C.c_float), i64],
            "adainf_app_create": [C.POINTER(AppSpec), C.POINTER(vp)],
            "adainf_app_destroy": [vp],
            "adainf_infer_dag": [vp, vp, i32, C.POINTER(C.c_float), i32, C.POINTER(ModelOut), vp],
            "adainf_select_retrain": [C.POINTER(SelectIn), i32, vp, vp, vp, vp, vp],
            "adainf_retrain_step": [vp, vp, vp, i32, i64, C.c_float, vp, vp],
            "adainf_retrain_step_rows": [vp, vp, i64, vp, vp, vp, i32, i64, C.c_float, vp, vp],
            "adainf_retrain_grad": [vp, vp, vp, i32, i64, vp, vp],
            "adainf_retrain_grad_rows": [vp, vp, i64, vp, vp, vp, i32, i64, vp, vp],
            "adainf_model_update": [vp, C.c_float, vp, vp],
            "adainf_app_poll": [vp, vp],
            "adainf_dbg_app_crops": [vp, i32, C.POINTER(vp)],
            "adainf_dbg_app_crop_layout": [vp, i32, C.POINTER(i32)],
            "adainf_dp_attach": [vp, vp, i32, i32],
            "adainf_select_merge": [vp, vp, vp, i32, i32, i64, i64, i64, i32, vp, vp, vp, vp],
            "adainf_nccl_unique_id": [vp],
            "adainf_gather_rows": [vp, vp, vp, i32, i64, vp, vp],
            "adainf_time_split": [C.c_double, C.POINTER(C.c_double), i32, C.POINTER(C.c_double), i32,
                                  C.POINTER(C.c_double), C.POINTER(C.c_double)],
            "adainf_retrain_setting": [C.c_double, C.POINTER(RetrainProfile), i64, i32, C.POINTER(RetrainPlan)],
            "adainf_model_average": [vp, C.POINTER(vp), i32, vp],
            "adainf_pick_batch": [C.POINTER(LatencyProfile), i64, C.POINTER(i32), C.POINTER(C.c_double)],
            "adainf_pick_structure": [i32, C.POINTER(LatencyProfile), C.POINTER(C.c_double), C.c_double, i32, i32,
                                      i32, i64, C.POINTER(i32), C.POINTER(i32), C.POINTER(C.c_double)],
            "adainf_dp_average": [vp, vp],
            "adainf_mark_used": [vp, vp, vp, i32, vp],
            "adainf_count_correct": [vp, vp, i32, vp, vp],
            "adainf_drift_should_stop": [C.POINTER(C.c_uint64), i32, i32, C.POINTER(i32)],
            "adainf_dbg_set_win_mode": [i32],
            "adainf_prof_enable": [i32],
            "adainf_prof_reset": [],
            "adainf_prof_query": [vp, i32, C.POINTER(i32)],
            "adainf_dbg_conv_fwd": [vp, i32, i32, i32, i32, vp, vp, i32, i32, i32, i32, i32, i32, vp, vp, i32, vp],
            "adainf_dbg_conv3_pool": [vp, i32, i32, i32, i32, i32, vp, vp, i32, i32, i32, vp, vp],
            "adainf_dbg_conv_dgrad": [vp, i32, i32, i32, i32, vp, i32, i32, i32, i32, i32, vp, vp, vp, i32, vp,
                                      vp],
            "adainf_dbg_conv_wgrad": [vp, vp, i32, i32, i32, i32, i32, i32, i32, i32, i32, vp, vp, vp],
            "adainf_dbg_stem_fwd": [vp, i32, i32, i32, i32, vp, vp, vp, vp, vp],
            "adainf_dbg_stem_wgrad": [vp, vp, i32, i32, i32, i32, vp, vp, vp],
        }.items():
            f = getattr(L, name, None)
            if f is not None:
                f.argtypes = args
                f.restype = C.c_int32
        _lib = L
    return _lib


def check(rc):
    if rc != OK:
        raise AdaInfError(rc, lib().adainf_last_error().decode(errors="replace"))


def ptr(t):
    """Device/host pointer of a torch tensor (or None)."""
    return None if t is None else C.c_void_p(t.data_ptr())


def stream_ptr(stream=None):
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return C.c_void_p(s.cuda_stream)


def make_ops(spec):
    ops = (Op * len(spec["ops"]))()
    for i, o in enumerate(spec["ops"]):
        r = ops[i]
        r.kind = _OPKIND[o["kind"]]
        r.kh = o.get("kh", 1)
        r.kw = o.get("kw", 1)
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
        r.nms_iou = float(o.get("nms_iou", 0.0))
        r.groups = int(o.get("groups", 1))
        r.pool = int(o.get("pool", 0))
    return ops


def _exit0_channels(spec):
    Cc = spec["in_c"]
    for o in spec["ops"]:
        if o["kind"] == "conv":
            Cc = o["cout"]
        elif o["kind"] == "exit":
            return Cc
    return 0


class _CudaArray:
    """__cuda_array_interface__ over a library-owned device buffer (zero-copy torch view)."""

    def __init__(self, p, shape, typestr):
        self.__cuda_array_interface__ = {"shape": tuple(shape), "typestr": typestr, "data": (int(p), False),
                                         "version": 2}


def _device_view(p, n, dtype, device, shape=None):
    import torch
    ts = {torch.float32: "<f4", torch.int16: "<i2", torch.int32: "<i4"}[dtype]
    return torch.as_tensor(_CudaArray(p, shape or (n,), ts), device=f"cuda:{device}")


class Model:
    """Owns an adainf_model_t."""

    def __init__(self, spec, max_batch, params=None, seed=0, momentum=0.9, weight_decay=0.0, device=0):
        self.spec = spec
        self._ops = make_ops(spec)
        self._params = None if params is None else np.ascontiguousarray(params, np.float32)
        ms = ModelSpec(spec["in_h"], spec["in_w"], spec["in_c"], max_batch, len(spec["ops"]), self._ops, momentum,
                       weight_decay, seed,
                       self._params.ctypes.data_as(C.POINTER(C.c_float)) if self._params is not None else None,
                       device)
        h = C.c_void_p()
        check(lib().adainf_model_create(C.byref(ms), C.byref(h)))
        self.h = h
        n = C.c_int64()
        check(lib().adainf_model_num_params(self.h, C.byref(n)))
        self.num_params = n.value
        e = C.c_int32()
        check(lib().adainf_model_num_exits(self.h, C.byref(e)))
        self.num_exits = e.value
        self.ncls = next((o["num_classes"] for o in spec["ops"] if o["kind"] == "exit"), 0)
        self.max_batch = max_batch
        self.device = device
        self.exit0_channels = _exit0_channels(spec)

    def get_params(self):
        out = np.zeros(self.num_params, np.float32)
        check(lib().adainf_model_get_params(self.h, out.ctypes.data_as(C.POINTER(C.c_float)), self.num_params))
        return out

    def set_params(self, p):
        p = np.ascontiguousarray(p, np.float32)
        check(lib().adainf_model_set_params(self.h, p.ctypes.data_as(C.POINTER(C.c_float)), self.num_params))

    def get_grads(self):
        out = np.zeros(self.num_params, np.float32)
        check(lib().adainf_model_get_grads(self.h, out.ctypes.data_as(C.POINTER(C.c_float)), self.num_params))
        return out

    def retrain_step(self, samples, labels, n_global=None, lr=0.01, stats=None, stream=None):
        check(lib().adainf_retrain_step(self.h, ptr(samples), ptr(labels), int(samples.shape[0]),
                                        int(n_global or samples.shape[0]), float(lr), ptr(stats),
                                        stream_ptr(stream)))

    def retrain_step_rows(self, pool, pool_labels, row_idx, n_global=None, lr=0.01, stats=None, stream=None,
                          count=None):
        """Retraining step on pool rows row_idx (device int32[n]) with labels pool_labels[row_idx]; rows past the
        device count (int32[1], optional) or outside the pool contribute nothing."""
        n = int(row_idx.shape[0])
        check(lib().adainf_retrain_step_rows(self.h, ptr(pool), int(pool.shape[0]), ptr(pool_labels), ptr(row_idx),
                                             ptr(count), n, int(n_global or n), float(lr), ptr(stats),
                                             stream_ptr(stream)))

    def retrain_grad(self, samples, labels, n_global=None, stats=None, stream=None):
        """Forward + backward only: this replica's 1/n_global-scaled gradient left in the gradient buffer."""
        check(lib().adainf_retrain_grad(self.h, ptr(samples), ptr(labels), int(samples.shape[0]),
                                        int(n_global or samples.shape[0]), ptr(stats), stream_ptr(stream)))

    def retrain_grad_rows(self, pool, pool_labels, row_idx, n_global=None, stats=None, stream=None, count=None):
        n = int(row_idx.shape[0])
        check(lib().adainf_retrain_grad_rows(self.h, ptr(pool), int(pool.shape[0]), ptr(pool_labels), ptr(row_idx),
                                             ptr(count), n, int(n_global or n), ptr(stats), stream_ptr(stream)))

    def update(self, lr=0.01, stats=None, stream=None):
        """SGD / momentum update on the current gradient buffer (all-reduced first over an attached communicator)."""
        check(lib().adainf_model_update(self.h, float(lr), ptr(stats), stream_ptr(stream)))

    def grad_tensor(self):
        """The device gradient buffer as a torch float32 tensor view (num_params), for callers reducing it."""
        import torch
        p = C.c_void_p()
        check(lib().adainf_model_grad_ptr(self.h, C.byref(p)))
        return _device_view(p.value, self.num_params, torch.float32, self.device)

    def dp_attach(self, uid: bytes, rank: int, world: int):
        buf = C.create_string_buffer(uid, 128)
        check(lib().adainf_dp_attach(self.h, buf, rank, world))

    def close(self):
        if getattr(self, "h", None):
            lib().adainf_model_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def alloc_outs(model, rows, max_det=0, n_out_edges=0, max_routed=0, device="cuda"):
    """Per-model output buffers of adainf_infer_dag as torch tensors (rows = input rows capacity)."""
    import torch
    E, NC = model.num_exits, model.ncls
    o = {}
    if E:
        o["exit_id"] = torch.full((rows,), -1, dtype=torch.int8, device=device)
        o["pred"] = torch.full((rows,), -1, dtype=torch.int32, device=device)
        o["conf"] = torch.zeros(rows, dtype=torch.float32, device=device)
        o["entropy"] = torch.zeros(rows, dtype=torch.float32, device=device)
        o["logits"] = torch.zeros((rows, NC), dtype=torch.float32, device=device)
        o["exit_counts"] = torch.zeros(E, dtype=torch.int32, device=device)
        o["surv_idx"] = torch.full((max(E - 1, 1), rows), -1, dtype=torch.int32, device=device)
        c0 = model.exit0_channels
        o["embed"] = torch.zeros((rows, c0), dtype=torch.float32, device=device)
    if max_det:
        o["n_det"] = torch.zeros(1, dtype=torch.int32, device=device)
        o["det_table"] = torch.zeros((max_det, 9), dtype=torch.float32, device=device)
    if n_out_edges:
        o["route_idx"] = torch.full((n_out_edges, max_routed), -1, dtype=torch.int32, device=device)
        o["n_routed"] = torch.zeros(n_out_edges, dtype=torch.int32, device=device)
    return o


def nccl_unique_id() -> bytes:
    buf = C.create_string_buffer(128)
    check(lib().adainf_nccl_unique_id(buf))
    return buf.raw


class App:
    """Owns an adainf_app_t over borrowed Models."""

    def __init__(self, models, edges=(), max_routed_per_dst=0):
        self.models = list(models)
        arr = (C.c_void_p * len(self.models))(*[m.h.value for m in self.models])
        self._arr = arr
        self._edges = (Edge * max(1, len(edges)))()
        for i, e in enumerate(edges):
            self._edges[i] = Edge(*e)
        self.edges = list(edges)
        spec = AppSpec(len(self.models), C.cast(arr, C.POINTER(C.c_void_p)), len(edges), self._edges,
                       max_routed_per_dst)
        h = C.c_void_p()
        check(lib().adainf_app_create(C.byref(spec), C.byref(h)))
        self.h = h
        self.max_routed = max_routed_per_dst

    def infer(self, batch, taus, outs, stream=None):
        """batch: cuda bf16/uint16 tensor [B,H,W,C]; taus: host list; outs: list of dicts of cuda tensors."""
        t = np.ascontiguousarray(np.asarray(taus, np.float32).reshape(-1))
        mo = (ModelOut * len(self.models))()
        for i, o in enumerate(outs):
            for k in ("exit_id", "pred", "conf", "entropy", "logits", "exit_counts", "surv_idx", "embed", "n_det",
                      "det_table", "route_idx", "n_routed"):
                if o.get(k) is not None:
                    setattr(mo[i], k, o[k].data_ptr())
            mo[i].max_det = int(o["det_table"].shape[0]) if o.get("det_table") is not None else 0
        check(lib().adainf_infer_dag(self.h, ptr(batch), int(batch.shape[0]),
                                     t.ctypes.data_as(C.POINTER(C.c_float)), int(t.size), mo, stream_ptr(stream)))

    def poll(self, stream=None):
        """Synchronize the stream; raise AdaInfError(ERR_CAPACITY) if a routing overflow happened since the last check."""
        check(lib().adainf_app_poll(self.h, stream_ptr(stream)))

    def crops(self, edge, rows):
        """Routed-crop batch of DET_CROP edge `edge` (debug view, bf16 bits as int16 [rows, H, W, C])."""
        import torch
        e = self.edges[edge]
        dst = self.models[e[1]].spec
        p = C.c_void_p()
        check(lib().adainf_dbg_app_crops(self.h, edge, C.byref(p)))
        s2d = C.c_int32()
        check(lib().adainf_dbg_app_crop_layout(self.h, edge, C.byref(s2d)))
        H, W, Cc = dst["in_h"], dst["in_w"], dst["in_c"]
        if not s2d.value:
            return _device_view(p.value, 0, torch.int16, self.models[e[1]].device, shape=(rows, H, W, Cc))
        # space-to-depth packed [rows][H/2][W/2][16], channel (bh*2 + bw)*4 + c: unpacked to NHWC for inspection
        s = _device_view(p.value, 0, torch.int16, self.models[e[1]].device, shape=(rows, H // 2, W // 2, 2, 2, 4))
        return s.permute(0, 1, 3, 2, 4, 5).reshape(rows, H, W, 4)[..., :Cc].contiguous()

    def close(self):
        if getattr(self, "h", None):
            lib().adainf_app_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def select_retrain(X, W, ref, k, exclude=None, out_idx=None, out_dist=None, out_count=None, dist_all=None,
                   stream=None):
    """X: cuda bf16 [N,D]; W: cuda bf16 [D,P] or None; ref: cuda fp32 [M,D]."""
    import torch
    N, D = X.shape
    P = W.shape[1] if W is not None else D
    si = SelectIn(X.data_ptr(), N, D, W.data_ptr() if W is not None else None, P, ref.data_ptr(),
                  ref.shape[0], exclude.data_ptr() if exclude is not None else None)
    dev = X.device
    out_idx = out_idx if out_idx is not None else torch.empty(k, dtype=torch.int32, device=dev)
    out_dist = out_dist if out_dist is not None else torch.empty(k, dtype=torch.float32, device=dev)
    out_count = out_count if out_count is not None else torch.empty(1, dtype=torch.int32, device=dev)
    check(lib().adainf_select_retrain(C.byref(si), int(k), ptr(out_idx), ptr(out_dist), ptr(out_count),
                                      ptr(dist_all), stream_ptr(stream)))
    return out_idx, out_dist, out_count


def select_merge(dist, idx, block_count, n_blocks, block_len, idx_mul, block_off, n_total, k, stream=None):
    """K12: global top-k from gathered per-shard top-k lists (device tensors [n_blocks * block_len])."""
    import torch
    dev = dist.device
    out_idx = torch.empty(k, dtype=torch.int32, device=dev)
    out_dist = torch.empty(k, dtype=torch.float32, device=dev)
    out_count = torch.empty(1, dtype=torch.int32, device=dev)
    check(lib().adainf_select_merge(ptr(dist), ptr(idx), ptr(block_count), int(n_blocks), int(block_len),
                                    int(idx_mul), int(block_off), int(n_total), int(k), ptr(out_idx), ptr(out_dist),
                                    ptr(out_count), stream_ptr(stream)))
    return out_idx, out_dist, out_count


def select_retrain_sharded(X_local, W, ref, k, group, exclude=None, mode="contiguous", n_total=None):
    """Selection over a pool sharded across the ranks of `group`: local exact top-k on this rank's
    rows (adainf_select_retrain), all-gather of (distance, local index, count) over the process group (NCCL on
    GPUs), exact merge on the device (adainf_select_merge).  mode "contiguous": rank r holds global rows
    [r * N_local, (r + 1) * N_local); "mod": rank r holds rows r, r + G, r + 2G, ... (P:243 disjoint shards)."""
    import torch
    import torch.distributed as dist
    G = dist.get_world_size(group)
    n_local = X_local.shape[0]
    idx, dd, cnt = select_retrain(X_local, W, ref, k, exclude=exclude)
    cat = torch.cat([dd.view(torch.int32), idx, cnt]).contiguous()
    gathered = [torch.empty_like(cat) for _ in range(G)]
    if dist.get_backend(group) == "gloo":
        g_cpu = [torch.empty_like(cat, device="cpu") for _ in range(G)]
        dist.all_gather(g_cpu, cat.cpu(), group=group)
        gathered = [t.to(X_local.device) for t in g_cpu]
    else:
        dist.all_gather(gathered, cat, group=group)
    st = torch.stack(gathered)  # [G][2k + 1]
    dists = st[:, :k].contiguous().view(torch.float32).reshape(-1)
    idxs = st[:, k:2 * k].contiguous().reshape(-1)
    cnts = st[:, 2 * k].contiguous()
    total = n_total or n_local * G
    mul, off = (1, n_local) if mode == "contiguous" else (G, 1)
    return select_merge(dists, idxs, cnts, G, k, mul, off, total, k)


def gather_rows(src, idx, count, n, dst, stream=None):
    """dst[r] = src[idx[r]] for r < min(count, n) (device count tensor or None)."""
    row_bytes = src[0].numel() * src.element_size()
    check(lib().adainf_gather_rows(ptr(src), ptr(idx), ptr(count), int(n), int(row_bytes), ptr(dst),
                                   stream_ptr(stream)))


class ProfEntry(C.Structure):
    _fields_ = [("name", C.c_char_p), ("launches", C.c_int64), ("total_ms", C.c_double)]


def launch_count() -> int:
    return int(lib().adainf_launch_count())


def prof_enable(on: bool):
    check(lib().adainf_prof_enable(int(on)))


def prof_reset():
    check(lib().adainf_prof_reset())


def prof_query():
    arr = (ProfEntry * 64)()
    n = C.c_int32()
    check(lib().adainf_prof_query(arr, 64, C.byref(n)))
    return {arr[i].name.decode(): (int(arr[i].launches), float(arr[i].total_ms)) for i in range(n.value)}


# ---- kernel-level (include/adainf_debug.h) ----
def dbg_set_win_mode(mode: int):
    check(lib().adainf_dbg_set_win_mode(int(mode)))


def dbg_conv_fwd(x, w, b, stride, pad, act=0, res=None, out_f32=False, stream=None):
    import torch
    n, H, W_, Cc = x.shape
    Co, KH, KW, _ = w.shape
    Ho, Wo = (H + 2 * pad - KH) // stride + 1, (W_ + 2 * pad - KW) // stride + 1
    out = torch.empty((n, Ho, Wo, Co), dtype=torch.float32 if out_f32 else torch.bfloat16, device=x.device)
    check(lib().adainf_dbg_conv_fwd(ptr(x), n, H, W_, Cc, ptr(w), ptr(b), Co, KH, KW, stride, pad, act, ptr(res),
                                    ptr(out), int(out_f32), stream_ptr(stream)))
    return out


def dbg_conv3_pool(x, w, b, act=0, first=False, cin_real=None, stream=None):
    """3x3/1 conv + bias + act + 2x2/2 max-pool in one kernel (include/adainf_debug.h)."""
    import torch
    n, H, W_, Cc = x.shape
    Co = w.shape[0]
    y = torch.empty((n, H // 2, W_ // 2, Co), dtype=torch.bfloat16, device=x.device)
    check(lib().adainf_dbg_conv3_pool(ptr(x), n, H, W_, Cc, Cc if cin_real is None else cin_real, ptr(w), ptr(b), Co,
                                      act, int(first), ptr(y), stream_ptr(stream)))
    return y


def dbg_conv_dgrad(dz, w, H, W_, stride, pad, bcast=None, sc=None, yact=None, mask_act=0, stream=None):
    import torch
    n = dz.shape[0]
    Co, KH, KW, Cc = w.shape
    dx = torch.empty((n, H, W_, Cc), dtype=torch.bfloat16, device=dz.device)
    check(lib().adainf_dbg_conv_dgrad(ptr(dz), n, H, W_, Cc, ptr(w), Co, KH, KW, stride, pad, ptr(bcast), ptr(sc),
                                      ptr(yact), mask_act, ptr(dx), stream_ptr(stream)))
    return dx


def dbg_stem_fwd(x, w, b, stream=None, want_argmax=True):
    """Space-to-depth stem: conv 7x7/2 pad 3 + bias + ReLU + maxpool 3x3/2 pad 1 (include/adainf_debug.h)."""
    import torch
    n, H, W_, cin = x.shape
    Hp, Wp = (H // 2 - 1) // 2 + 1, (W_ // 2 - 1) // 2 + 1
    pooled = torch.empty((n, Hp, Wp, 64), dtype=torch.bfloat16, device=x.device)
    am = torch.empty((n, Hp, Wp, 64), dtype=torch.uint8, device=x.device) if want_argmax else None
    check(lib().adainf_dbg_stem_fwd(ptr(x), n, H, W_, cin, ptr(w), ptr(b), ptr(pooled), ptr(am), stream_ptr(stream)))
    return pooled, am


def dbg_stem_wgrad(x, dz, stream=None):
    import torch
    n, H, W_, cin = x.shape
    dw = torch.empty((64, 7, 7, cin), dtype=torch.float32, device=x.device)
    db = torch.empty(64, dtype=torch.float32, device=x.device)
    check(lib().adainf_dbg_stem_wgrad(ptr(x), ptr(dz), n, H, W_, cin, ptr(dw), ptr(db), stream_ptr(stream)))
    return dw, db


def dbg_conv_wgrad(x, dz, KH, KW, stride, pad, stream=None):
    import torch
    n, H, W_, Cc = x.shape
    Co = dz.shape[-1]
    dw = torch.empty((Co, KH, KW, Cc), dtype=torch.float32, device=x.device)
    db = torch.empty(Co, dtype=torch.float32, device=x.device)
    check(lib().adainf_dbg_conv_wgrad(ptr(x), ptr(dz), n, H, W_, Cc, Co, KH, KW, stride, pad, ptr(dw), ptr(db),
                                      stream_ptr(stream)))
    return dw, db


# ---- incremental-retraining support (include/adainf_sched.h) ----
def time_split(slo_ms, infer_ms, impact):
    """T_r = max(0, L_s - sum l_k) and its split by impact degree.  Host arithmetic."""
    li = (C.c_double * max(1, len(infer_ms)))(*infer_ms)
    di = (C.c_double * max(1, len(impact)))(*impact)
    out = (C.c_double * max(1, len(impact)))()
    tr = C.c_double()
    check(lib().adainf_time_split(float(slo_ms), li, len(infer_ms), di, len(impact), C.byref(tr), out))
    return tr.value, [out[j] for j in range(len(impact))]


def retrain_setting(alloc_ms, batches, step_ms, eligible, max_batch):
    """Retraining setting a time allocation affords under a measured step profile."""
    bi = (C.c_int32 * len(batches))(*batches)
    ti = (C.c_double * len(step_ms))(*step_ms)
    prof = RetrainProfile(len(batches), bi, ti)
    out = RetrainPlan()
    check(lib().adainf_retrain_setting(float(alloc_ms), C.byref(prof), int(eligible), int(max_batch), C.byref(out)))
    return {"samples": out.samples, "batch": out.batch, "steps": out.steps, "epochs": out.epochs, "est_ms": out.est_ms}


def _latency_profile(batches, ms, keep):
    bi = (C.c_int32 * len(batches))(*batches)
    ti = (C.c_double * len(ms))(*ms)
    keep += [bi, ti]
    return LatencyProfile(len(batches), bi, ti)


def pick_batch(batches, per_batch_ms, requests):
    """NEXT-4: batch with the lowest worst-case latency per_batch_ms(b) * ceil(requests / b)."""
    keep = []
    prof = _latency_profile(batches, per_batch_ms, keep)
    b, w = C.c_int32(), C.c_double()
    check(lib().adainf_pick_batch(C.byref(prof), int(requests), C.byref(b), C.byref(w)))
    return b.value, w.value


def pick_structure(tables, accuracy, a_min, has_retraining, full_index, batch0, requests):
    """NEXT-4: tables = [(batches, per_batch_ms)] per structure; returns (structure, batch, worst_ms)."""
    keep = []
    arr = (LatencyProfile * len(tables))(*[_latency_profile(b, t, keep) for b, t in tables])
    acc = (C.c_double * len(accuracy))(*accuracy)
    s, b, w = C.c_int32(), C.c_int32(), C.c_double()
    check(lib().adainf_pick_structure(len(tables), arr, acc, float(a_min), int(has_retraining), int(full_index),
                                      int(batch0), int(requests), C.byref(s), C.byref(b), C.byref(w)))
    return s.value, b.value, w.value


def model_average(dst, versions, stream=None):
    """dst <- mean of the versions' fp32 parameters, momentum reset (reading Q23)."""
    arr = (C.c_void_p * len(versions))(*[v.h for v in versions])
    check(lib().adainf_model_average(dst.h, arr, len(versions), stream_ptr(stream)))


def dp_average(model, stream=None):
    check(lib().adainf_dp_average(model.h, stream_ptr(stream)))


def mark_used(exclude, idx, count=None, stream=None):
    """exclude[idx[:count]] = 1 (samples used by one job are not reused by another)."""
    check(lib().adainf_mark_used(ptr(exclude), ptr(idx), ptr(count), int(idx.numel()), stream_ptr(stream)))


def count_correct(pred, labels, stream=None):
    import torch
    out = torch.empty(1, dtype=torch.int32, device=pred.device)
    check(lib().adainf_count_correct(ptr(pred), ptr(labels), int(pred.numel()), ptr(out), stream_ptr(stream)))
    return out


def drift_should_stop(results, n=4):
    """Stop rule of the drift-impact detection (Table 2): the last n impacted-set results agree."""
    arr = (C.c_uint64 * max(1, len(results)))(*results)
    out = C.c_int32()
    check(lib().adainf_drift_should_stop(arr, len(results), int(n), C.byref(out)))
    return bool(out.value)
