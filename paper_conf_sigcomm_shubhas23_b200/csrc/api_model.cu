// C-ABI entry points (include/adainf.h): models, apps (DAG inference with on-device routing), selection,
// retraining step, data-parallel attach.
#include <cstring>
#include <vector>

#include "api_common.h"
#include "model.h"

namespace adainf {
void select_merge(const float* dist, const int32_t* idx, const int32_t* block_count, int n_blocks, int block_len,
                  long long idx_mul, long long block_off, long long n_total, int k, int32_t* out_idx, float* out_dist,
                  int32_t* out_count, cudaStream_t st);
void select_retrain(const adainf_select_in& in, int k, int32_t* out_idx, float* out_dist, int32_t* out_count,
                    float* dist_all, cudaStream_t st);
}

using namespace adainf;

#include "api_handles.h"

extern "C" adainf_status adainf_model_create(const adainf_model_spec* spec, adainf_model_t* out) {
  return guard([&] {
    if (!spec || !out) throw InvalidError("null argument");
    require_device();
    auto* h = new adainf_model();
    try {
      h->m.build(*spec);
    } catch (...) {
      delete h;
      throw;
    }
    *out = h;
  });
}

extern "C" adainf_status adainf_model_destroy(adainf_model_t m) {
  return guard([&] {
    if (!m) return;
#ifdef ADAINF_WITH_NCCL
    if (m->m.comm) ncclCommDestroy(m->m.comm);
#endif
    cudaDeviceSynchronize();
    delete m;
  });
}

extern "C" adainf_status adainf_model_num_params(adainf_model_t m, int64_t* n) {
  return guard([&] {
    if (!m || !n) throw InvalidError("null argument");
    *n = m->m.nparams;
  });
}
extern "C" adainf_status adainf_model_num_exits(adainf_model_t m, int32_t* n) {
  return guard([&] {
    if (!m || !n) throw InvalidError("null argument");
    *n = (int32_t)m->m.exits.size();
  });
}
extern "C" adainf_status adainf_model_get_params(adainf_model_t m, float* dst, int64_t n) {
  return guard([&] {
    if (!m || !dst || n != m->m.nparams) throw InvalidError("get_params: size mismatch");
    CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(dst, m->m.params.p, n * 4, cudaMemcpyDeviceToHost));
  });
}
extern "C" adainf_status adainf_model_set_params(adainf_model_t m, const float* src, int64_t n) {
  return guard([&] {
    if (!m || !src || n != m->m.nparams) throw InvalidError("set_params: size mismatch");
    CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(m->m.params.p, src, n * 4, cudaMemcpyHostToDevice));
    m->m.mom.zero();
    m->m.refresh_shadows(0);
    CK(cudaDeviceSynchronize());
  });
}
extern "C" adainf_status adainf_model_get_grads(adainf_model_t m, float* dst, int64_t n) {
  return guard([&] {
    if (!m || !dst || n != m->m.nparams) throw InvalidError("get_grads: size mismatch");
    CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(dst, m->m.grads.p, n * 4, cudaMemcpyDeviceToHost));
  });
}
extern "C" adainf_status adainf_model_grad_ptr(adainf_model_t m, float** p) {
  return guard([&] {
    if (!m || !p) throw InvalidError("null argument");
    *p = m->m.grads.as<float>();
  });
}

// ------------------------------------------------------------------------------------------------
namespace adainf {

struct AppModelScratch {
  DevBuf pred;                   // [rows]
  DevBuf n_det, route_idx, n_routed, cnt_clamped;  // detector out-edges
  DevBuf det_table;              // all candidates x 9
  DevBuf det_ws;
  std::vector<int> det_edges;    // app edge indices (DET_CROP) out of this model, local order
  int rows = 0;
};

struct AppImpl {
  std::vector<AppModelScratch> ms;
  std::vector<DevBuf> routed_in;  // per edge (DET_CROP)
  std::vector<char> crop_s2d;     // per edge: crops written straight into the destination's space-to-depth input
  DevBuf route_list, route_cnt;   // CLASS_WHOLE: [n_edges][cap], [n_edges]
  int32_t* cap_flag_host = nullptr;
  int32_t* cap_flag_dev = nullptr;
  std::vector<int> in_edge;       // per model: incoming edge (-1 for root)
};

}  // namespace adainf

struct AppHolder {
  App a;
  AppImpl impl;
  ~AppHolder() {
    if (impl.cap_flag_host) cudaFreeHost(impl.cap_flag_host);
  }
};

extern "C" adainf_status adainf_app_create(const adainf_app_spec* spec, adainf_app_t* out) {
  return guard([&] {
    if (!spec || !out || spec->n_models <= 0 || !spec->models) throw InvalidError("app: bad spec");
    require_device();
    auto* h = new AppHolder();
    try {
      App& a = h->a;
      AppImpl& I = h->impl;
      for (int i = 0; i < spec->n_models; ++i) {
        if (!spec->models[i]) throw InvalidError("app: null model");
        a.models.push_back(&spec->models[i]->m);
      }
      a.edges.assign(spec->edges, spec->edges + spec->n_edges);
      a.max_routed = spec->max_routed_per_dst;
      const int nm = (int)a.models.size();
      I.in_edge.assign(nm, -1);
      I.ms.resize(nm);
      for (size_t e = 0; e < a.edges.size(); ++e) {
        const adainf_edge& ed = a.edges[e];
        if (ed.src_model < 0 || ed.src_model >= nm || ed.dst_model <= ed.src_model || ed.dst_model >= nm)
          throw InvalidError("app: edges must go from a lower to a higher model index");
        if (I.in_edge[ed.dst_model] >= 0) throw InvalidError("app: a model may have only one incoming edge");
        I.in_edge[ed.dst_model] = (int)e;
        if (a.max_routed <= 0) throw InvalidError("app: max_routed_per_dst must be > 0 with edges");
        Model* src = a.models[ed.src_model];
        Model* dst = a.models[ed.dst_model];
        if (a.max_routed > dst->max_batch) throw ShapeError("app: max_routed_per_dst exceeds the dst max_batch");
        if (ed.kind == ADAINF_ROUTE_DET_CROP) {
          if (src->det.tensor < 0) throw InvalidError("app: DET_CROP edge from a non-detector");
          if (ed.crop_h != dst->in_h || ed.crop_w != dst->in_w || dst->in_c != src->in_c)
            throw ShapeError("app: crop size must equal the destination input");
          if (ed.src_class < 0 || ed.src_class >= src->det.classes) throw InvalidError("app: bad src_class");
          for (int q : I.ms[ed.src_model].det_edges)  // a detection goes to its class's one destination
            if (a.edges[q].src_class == ed.src_class) throw InvalidError("app: two DET_CROP edges for one class");
          I.ms[ed.src_model].det_edges.push_back((int)e);
        } else if (ed.kind == ADAINF_ROUTE_CLASS_WHOLE) {
          if (src->exits.empty()) throw InvalidError("app: CLASS_WHOLE edge from a model without exits");
          if (dst->in_h != src->in_h || dst->in_w != src->in_w || dst->in_c != src->in_c)
            throw ShapeError("app: CLASS_WHOLE destination input must equal the source input");
        } else {
          throw InvalidError("app: unknown edge kind");
        }
      }
      for (int i = 1; i < nm; ++i)
        if (I.in_edge[i] < 0) throw InvalidError("app: every non-root model needs an incoming edge");
      I.routed_in.resize(a.edges.size());
      I.crop_s2d.assign(a.edges.size(), 0);
      for (size_t e = 0; e < a.edges.size(); ++e)
        if (a.edges[e].kind == ADAINF_ROUTE_DET_CROP) {
          Model* dst = a.models[a.edges[e].dst_model];
          const adainf_edge& ed = a.edges[e];
          // a ResNet-stem destination takes its crops already space-to-depth packed (no packing pass)
          const bool s2d = dst->stem_s2d && dst->in_c <= 4 && ed.crop_h == dst->in_h && ed.crop_w == dst->in_w &&
                           getenv("ADAINF_CROP_S2D") == nullptr;
          I.crop_s2d[e] = s2d;
          I.routed_in[e].alloc((size_t)a.max_routed * dst->in_h * dst->in_w * (s2d ? 4 : dst->in_c) * 2);
        }
      I.route_list.alloc((size_t)std::max<size_t>(1, a.edges.size()) * std::max(1, a.max_routed) * 4);
      I.route_cnt.alloc((size_t)std::max<size_t>(1, a.edges.size()) * 4 + 16);
      I.route_cnt.zero();
      for (int i = 0; i < nm; ++i) {
        Model* m = a.models[i];
        AppModelScratch& S = I.ms[i];
        S.rows = i == 0 ? m->max_batch : a.max_routed;
        S.pred.alloc((size_t)m->max_batch * 4);
        if (m->det.tensor >= 0) {
          const TensorRt& D = m->T[m->det.tensor];
          const int cpf = D.H * D.W + (m->det.tensor2 >= 0 ? m->T[m->det.tensor2].H * m->T[m->det.tensor2].W : 0);
          const size_t ncand = (size_t)m->max_batch * cpf * m->det.anchors;
          S.det_table.alloc(ncand * 9 * 4);
          S.det_ws.alloc(det_route_ws_bytes(m->max_batch, cpf, m->det.anchors, m->det.nms_iou > 0.f));
          const int ne = std::max<int>(1, (int)S.det_edges.size());
          S.n_det.alloc(16);
          S.route_idx.alloc((size_t)ne * std::max(1, a.max_routed) * 4);
          S.n_routed.alloc((size_t)ne * 4 + 16);
          S.cnt_clamped.alloc((size_t)ne * 4 + 16);
        }
      }
      CK(cudaHostAlloc((void**)&I.cap_flag_host, 4, cudaHostAllocMapped));
      *I.cap_flag_host = 0;
      CK(cudaHostGetDevicePointer((void**)&I.cap_flag_dev, I.cap_flag_host, 0));
      CK(cudaDeviceSynchronize());
    } catch (...) {
      delete h;
      throw;
    }
    *out = (adainf_app_t)h;
  });
}

extern "C" adainf_status adainf_app_destroy(adainf_app_t app) {
  return guard([&] {
    if (!app) return;
    cudaDeviceSynchronize();
    delete (AppHolder*)app;
  });
}

extern "C" adainf_status adainf_infer_dag(adainf_app_t app, const void* batch, int32_t n, const float* taus,
                                          int32_t n_taus, adainf_model_out* outs, adainf_stream_t stream) {
  return guard([&] {
    if (!app || !batch || !outs) throw InvalidError("infer_dag: null argument");
    require_device();
    AppHolder* H = (AppHolder*)app;
    App& a = H->a;
    AppImpl& I = H->impl;
    cudaStream_t st = (cudaStream_t)stream;
    if (*I.cap_flag_host) {
      *I.cap_flag_host = 0;
      throw CapacityError("a previous infer_dag routed more crops than max_routed_per_dst (clamped in index order)");
    }
    const int nm = (int)a.models.size();
    if (n <= 0 || n > a.models[0]->max_batch) throw ShapeError("infer_dag: batch must be in 1..max_batch");
    // thresholds, concatenated in model order
    std::vector<const float*> tau_of(nm, nullptr);
    int need = 0;
    for (int i = 0; i < nm; ++i) {
      Model* m = a.models[i];
      const int c = m->exits.empty() ? 1 : (int)m->exits.size() - 1;
      if (taus) tau_of[i] = taus + need;
      need += c;
    }
    if (n_taus != need || (need > 0 && !taus)) throw InvalidError("infer_dag: expected " + std::to_string(need) + " thresholds");
    for (int i = 0; i < need; ++i)
      if (taus[i] != taus[i]) throw InvalidError("infer_dag: NaN threshold");
    for (int i = 0; i < nm; ++i) {
      Model* m = a.models[i];
      AppModelScratch& S = I.ms[i];
      adainf_model_out o = outs[i];
      if (!o.pred) o.pred = S.pred.as<int32_t>();
      // input of this model
      const bf16* x = (const bf16*)batch;
      const int* map = nullptr;
      const int* cnt = nullptr;
      int rows = n;
      bool padded = false;
      if (i > 0) {
        const int e = I.in_edge[i];
        const adainf_edge& ed = a.edges[e];
        rows = a.max_routed;
        cnt = I.route_cnt.as<int>() + e;
        if (ed.kind == ADAINF_ROUTE_DET_CROP) {
          x = I.routed_in[e].as<bf16>();  // crops in the destination's own input layout (ingested like a batch)
          padded = I.crop_s2d[e] != 0;     // ... or already in its packed space-to-depth layout
        } else {
          // whole-input routing: read the source model's own input rows through the route list
          if (ed.src_model != 0) throw UnsupportedError("CLASS_WHOLE routing from a routed model");
          map = I.route_list.as<int>() + (size_t)e * a.max_routed;
        }
      }
      m->infer(x, map, cnt, rows, tau_of[i], o, st, padded);
      // routing out of this model
      if (m->det.tensor >= 0) {
        const TensorRt& D = m->T[m->det.tensor];
        DetRouteArgs d{};
        d.raw = (const float*)D.buf;
        d.count = cnt;
        d.n_static = rows;
        d.G = D.H;
        d.A = m->det.anchors;
        d.NC = m->det.classes;
        d.stride = m->det.stride;
        d.img_w = m->in_w;
        d.img_h = m->in_h;
        memcpy(d.anchor_wh, m->det.anchor_wh, sizeof(d.anchor_wh));
        if (m->det.tensor2 >= 0) {  // second scale: its cells follow the first head's in each frame
          const TensorRt& D2 = m->T[m->det.tensor2];
          d.raw2 = (const float*)D2.buf;
          d.G2 = D2.H;
          d.stride2 = m->det.stride2;
          memcpy(d.anchor_wh2, m->det.anchor_wh2, sizeof(d.anchor_wh2));
        }
        d.tau = tau_of[i][0];
        d.n_edges = (int)S.det_edges.size();
        for (int q = 0; q < d.n_edges; ++q) d.edge_class[q] = a.edges[S.det_edges[q]].src_class;
        d.cap = std::max(1, a.max_routed);
        d.det_table = S.det_table.as<float>();
        d.user_table = o.det_table;
        d.user_max = o.max_det;
        d.n_det = o.n_det ? o.n_det : S.n_det.as<int32_t>();
        d.route_idx = S.route_idx.as<int32_t>();
        d.n_routed = S.n_routed.as<int32_t>();
        d.count_clamped = S.cnt_clamped.as<int32_t>();
        d.cap_flag = I.cap_flag_dev;
        d.nms_iou = m->det.nms_iou;
        launch_det_route(d, S.det_ws.p, st);
        for (int q = 0; q < d.n_edges; ++q) {
          const int e = S.det_edges[q];
          Model* dst = a.models[a.edges[e].dst_model];
          CK(cudaMemcpyAsync(I.route_cnt.as<int>() + e, S.cnt_clamped.as<int>() + q, 4, cudaMemcpyDeviceToDevice, st));
          launch_crops(x, m->in_h, m->in_w, m->in_c, S.det_table.as<float>(), S.route_idx.as<int32_t>(),
                       S.cnt_clamped.as<int32_t>(), q, d.cap, a.edges[e].crop_h, a.edges[e].crop_w, dst->in_c,
                       I.routed_in[e].as<bf16>(), st, I.crop_s2d[e] != 0);
        }
        if (o.route_idx && d.n_edges)
          CK(cudaMemcpyAsync(o.route_idx, S.route_idx.p, (size_t)d.n_edges * d.cap * 4, cudaMemcpyDeviceToDevice, st));
        if (o.n_routed && d.n_edges)
          CK(cudaMemcpyAsync(o.n_routed, S.n_routed.p, (size_t)d.n_edges * 4, cudaMemcpyDeviceToDevice, st));
      }
      int qn = 0;
      for (size_t e = 0; e < a.edges.size(); ++e) {
        const adainf_edge& ed = a.edges[e];
        if (ed.src_model != i || ed.kind != ADAINF_ROUTE_CLASS_WHOLE) continue;
        launch_route_class(o.pred, cnt, rows, ed.src_class, I.route_list.as<int32_t>() + e * a.max_routed,
                           I.route_cnt.as<int32_t>() + e, a.max_routed, I.cap_flag_dev, st);
        if (o.route_idx)
          CK(cudaMemcpyAsync(o.route_idx + (size_t)qn * a.max_routed, I.route_list.as<int32_t>() + e * a.max_routed,
                             (size_t)a.max_routed * 4, cudaMemcpyDeviceToDevice, st));
        if (o.n_routed)
          CK(cudaMemcpyAsync(o.n_routed + qn, I.route_cnt.as<int32_t>() + e, 4, cudaMemcpyDeviceToDevice, st));
        qn++;
      }
    }
  });
}

// ------------------------------------------------------------------------------------------------
extern "C" adainf_status adainf_select_retrain(const adainf_select_in* in, int32_t k, int32_t* out_idx, float* out_dist,
                                               int32_t* out_count, float* dist_all, adainf_stream_t stream) {
  return guard([&] {
    if (!in || !out_idx || !out_count) throw InvalidError("select: null argument");
    require_device();
    select_retrain(*in, k, out_idx, out_dist, out_count, dist_all, (cudaStream_t)stream);
  });
}

extern "C" adainf_status adainf_select_merge(const float* dist, const int32_t* idx, const int32_t* block_count,
                                             int32_t n_blocks, int32_t block_len, int64_t idx_mul, int64_t block_off,
                                             int64_t n_total, int32_t k, int32_t* out_idx, float* out_dist,
                                             int32_t* out_count, adainf_stream_t stream) {
  return guard([&] {
    if (!out_idx || !out_count) throw InvalidError("select_merge: null output");
    require_device();
    select_merge(dist, idx, block_count, n_blocks, block_len, idx_mul, block_off, n_total, k, out_idx, out_dist,
                 out_count, (cudaStream_t)stream);
  });
}

extern "C" adainf_status adainf_retrain_step(adainf_model_t m, const void* samples, const int32_t* labels,
                                             int32_t n_local, int64_t n_global, float lr, adainf_step_stats* stats,
                                             adainf_stream_t stream) {
  return guard([&] {
    if (!m || !samples || !labels) throw InvalidError("retrain: null argument");
    if (!(lr == lr)) throw InvalidError("retrain: NaN lr");
    require_device();
    m->m.train_step((const bf16*)samples, labels, n_local, n_global, lr, stats, (cudaStream_t)stream);
  });
}

extern "C" adainf_status adainf_retrain_step_rows(adainf_model_t m, const void* pool, int64_t pool_rows,
                                                  const int32_t* pool_labels, const int32_t* row_idx,
                                                  const int32_t* count, int32_t n_local, int64_t n_global, float lr,
                                                  adainf_step_stats* stats, adainf_stream_t stream) {
  return guard([&] {
    if (!m || !pool || !pool_labels || !row_idx) throw InvalidError("retrain_step_rows: null argument");
    if (!(lr == lr)) throw InvalidError("retrain: NaN lr");
    require_device();
    m->m.train_step_rows((const bf16*)pool, pool_rows, pool_labels, row_idx, count, n_local, n_global, lr, stats,
                         (cudaStream_t)stream);
  });
}

extern "C" adainf_status adainf_retrain_grad(adainf_model_t m, const void* samples, const int32_t* labels,
                                             int32_t n_local, int64_t n_global, adainf_step_stats* stats,
                                             adainf_stream_t stream) {
  return guard([&] {
    if (!m || !samples || !labels) throw InvalidError("retrain_grad: null argument");
    require_device();
    m->m.train_step((const bf16*)samples, labels, n_local, n_global, 0.f, stats, (cudaStream_t)stream, false);
  });
}

extern "C" adainf_status adainf_retrain_grad_rows(adainf_model_t m, const void* pool, int64_t pool_rows,
                                                  const int32_t* pool_labels, const int32_t* row_idx,
                                                  const int32_t* count, int32_t n_local, int64_t n_global,
                                                  adainf_step_stats* stats, adainf_stream_t stream) {
  return guard([&] {
    if (!m || !pool || !pool_labels || !row_idx) throw InvalidError("retrain_grad_rows: null argument");
    require_device();
    m->m.train_step_rows((const bf16*)pool, pool_rows, pool_labels, row_idx, count, n_local, n_global, 0.f, stats,
                         (cudaStream_t)stream, false);
  });
}

extern "C" adainf_status adainf_model_update(adainf_model_t m, float lr, adainf_step_stats* stats,
                                             adainf_stream_t stream) {
  return guard([&] {
    if (!m) throw InvalidError("update: null model");
    if (!(lr == lr)) throw InvalidError("update: NaN lr");
    require_device();
    m->m.update_impl(lr, stats, (cudaStream_t)stream);
  });
}

extern "C" adainf_status adainf_app_poll(adainf_app_t app, adainf_stream_t stream) {
  return guard([&] {
    if (!app) throw InvalidError("app_poll: null app");
    require_device();
    CK(cudaStreamSynchronize((cudaStream_t)stream));
    AppHolder* H = (AppHolder*)app;
    if (*H->impl.cap_flag_host) {
      *H->impl.cap_flag_host = 0;
      throw CapacityError("infer_dag routed more crops than max_routed_per_dst (clamped in index order)");
    }
  });
}

extern "C" adainf_status adainf_dbg_app_crops(adainf_app_t app, int32_t edge, const void** crops) {
  return guard([&] {
    if (!app || !crops) throw InvalidError("dbg_app_crops: null argument");
    AppHolder* H = (AppHolder*)app;
    if (edge < 0 || edge >= (int)H->a.edges.size() || H->a.edges[edge].kind != ADAINF_ROUTE_DET_CROP)
      throw InvalidError("dbg_app_crops: not a DET_CROP edge");
    *crops = H->impl.routed_in[edge].p;
  });
}

extern "C" adainf_status adainf_dbg_app_crop_layout(adainf_app_t app, int32_t edge, int32_t* s2d) {
  return guard([&] {
    if (!app || !s2d) throw InvalidError("dbg_app_crop_layout: null argument");
    AppHolder* H = (AppHolder*)app;
    if (edge < 0 || edge >= (int)H->a.edges.size() || H->a.edges[edge].kind != ADAINF_ROUTE_DET_CROP)
      throw InvalidError("dbg_app_crop_layout: not a DET_CROP edge");
    *s2d = H->impl.crop_s2d[edge];
  });
}

extern "C" adainf_status adainf_gather_rows(const void* src, const int32_t* idx, const int32_t* count, int32_t n,
                                            int64_t row_bytes, void* dst, adainf_stream_t stream) {
  return guard([&] {
    if (!src || !idx || !dst || n < 0 || row_bytes <= 0) throw InvalidError("gather_rows: bad argument");
    require_device();
    launch_gather_rows(src, idx, count, n, row_bytes, dst, (cudaStream_t)stream);
  });
}

extern "C" adainf_status adainf_nccl_unique_id(void* out128) {
  return guard([&] {
    if (!out128) throw InvalidError("null argument");
#ifdef ADAINF_WITH_NCCL
    ncclUniqueId id;
    if (ncclGetUniqueId(&id) != ncclSuccess) throw NcclError("ncclGetUniqueId failed");
    static_assert(sizeof(id) == 128, "ncclUniqueId is 128 bytes");
    memcpy(out128, &id, 128);
#else
    throw UnsupportedError("built without NCCL");
#endif
  });
}

extern "C" adainf_status adainf_dp_attach(adainf_model_t m, const void* uid, int32_t rank, int32_t world) {
  adainf_status s = guard([&] {
    if (!m) throw InvalidError("null model");
    if (world < 1 || rank < 0 || rank >= world) throw InvalidError("dp_attach: bad rank/world");
#ifdef ADAINF_WITH_NCCL
    if (m->m.comm) {
      ncclCommDestroy(m->m.comm);
      m->m.comm = nullptr;
    }
    m->m.dp_world = world;
    m->m.dp_rank = rank;
    if (world == 1) return;
    if (!uid) throw InvalidError("dp_attach: null unique id");
    ncclUniqueId id;
    memcpy(&id, uid, 128);
    CK(cudaSetDevice(m->m.device));
    ncclResult_t r = ncclCommInitRank(&m->m.comm, world, id, rank);
    if (r != ncclSuccess) throw NcclError(std::string("ncclCommInitRank: ") + ncclGetErrorString(r));
#else
    if (world > 1) throw UnsupportedError("built without NCCL");
#endif
  });
  return s;
}
