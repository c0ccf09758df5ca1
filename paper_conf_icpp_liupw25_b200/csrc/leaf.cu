// leaf.cu — (a)8 leaf values and (a)9 incremental prediction update,
// plus the export of the heap-indexed tree record.
#include "common.cuh"

namespace gbdtmo {

// leaf[h][k] = -lr * G_k / (H_k + lambda) for LEAF nodes (exact sums; MSE H = 2 count), else 0.
__global__ void k_leaf_values(gbdtmo_problem p, const float* __restrict__ scales, State s, double* __restrict__ leaf) {
  const int64_t NH = heap_nodes(p);
  const int d = p.d, V = channels(p);
  const bool softmax = p.loss == GBDTMO_LOSS_SOFTMAX;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < NH * d; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t h = e / d;
    const int k = (int)(e - h * d);
    double v = 0.0;
    if (s.node_state[h] == GBDTMO_NODE_LEAF) {
      const int64_t* S = s.node_sum + h * (V + 1);
      const double G = (double)S[k] * (double)scales[k];
      const double H = softmax ? (double)S[d + k] * (double)scales[d + k] : 2.0 * (double)S[V];
      v = -p.lr * G / (H + p.lambda);
    }
    leaf[e] = v;
  }
}

// pred[i][k] += leaf[nid[i]][k]: every instance reads its leaf directly (no traversal).
__global__ void k_update_pred(gbdtmo_problem p, State s, const double* __restrict__ leaf, double* __restrict__ pred) {
  const int d = p.d;
  const int64_t total = p.n * d;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = e / d;
    const int k = (int)(e - i * d);
    pred[e] += leaf[(int64_t)s.nid[i] * d + k];
  }
}

__global__ void k_tree_export(gbdtmo_problem p, State s, int32_t* node_state, int32_t* feature, int32_t* bin,
                              double* gain, int64_t* n_rows, int64_t* n_left, const float* __restrict__ cuts,
                              float* threshold) {
  const int64_t NH = heap_nodes(p);
  const int V = channels(p);
  for (int64_t h = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; h < NH; h += (int64_t)gridDim.x * blockDim.x) {
    int st = s.node_state[h];
    if (st == GBDTMO_NODE_ACTIVE) st = GBDTMO_NODE_LEAF;     // (only before a tree is finished)
    if (node_state) node_state[h] = st;
    if (feature) feature[h] = st == GBDTMO_NODE_SPLIT ? s.node_feat[h] : -1;
    if (bin) bin[h] = st == GBDTMO_NODE_SPLIT ? s.node_bin[h] : -1;
    if (gain) gain[h] = st == GBDTMO_NODE_SPLIT ? s.node_gain[h] : 0.0;
    if (n_rows) n_rows[h] = st != GBDTMO_NODE_NONE ? s.node_sum[h * (V + 1) + V] : 0;
    if (n_left) n_left[h] = st == GBDTMO_NODE_SPLIT ? s.node_nleft[h] : 0;
    if (threshold) {
      float t = 0.0f;
      const int fl = s.node_feat[h] - p.f_begin;
      if (st == GBDTMO_NODE_SPLIT && fl >= 0 && fl < p.m) t = cuts[(int64_t)fl * (p.B - 1) + s.node_bin[h]];
      threshold[h] = t;
    }
  }
}

// One warp per instance: all lanes walk the (uniform) path of each tree, lanes add the leaf's
// outputs (coalesced); trees in order so the sums match the training-time accumulation.
__global__ void k_predict(const float* __restrict__ X, int64_t n, int64_t ld_x, int T, int D, int d,
                          const int32_t* __restrict__ node_state, const int32_t* __restrict__ feature,
                          const float* __restrict__ threshold, const double* __restrict__ leaf,
                          double* __restrict__ pred) {
  const int lane = threadIdx.x & 31;
  const int64_t NH = (int64_t(1) << (D + 1)) - 1;
  const int64_t wpb = blockDim.x >> 5;
  for (int64_t i = blockIdx.x * wpb + (threadIdx.x >> 5); i < n; i += (int64_t)gridDim.x * wpb) {
    const float* xi = X + i * ld_x;
    double* pi = pred + i * d;
    for (int t = 0; t < T; ++t) {
      const int32_t* st = node_state + (int64_t)t * NH;
      int64_t h = 0;
      while (h < NH && st[h] == GBDTMO_NODE_SPLIT) {
        const int32_t f = feature[(int64_t)t * NH + h];
        h = (xi[f] < threshold[(int64_t)t * NH + h]) ? 2 * h + 1 : 2 * h + 2;
      }
      if (h < NH && st[h] == GBDTMO_NODE_LEAF) {
        const double* lv = leaf + ((int64_t)t * NH + h) * d;
        for (int k = lane; k < d; k += 32) pi[k] += lv[k];
      }
    }
  }
}

__global__ void k_rows_export(gbdtmo_problem p, State s, const int32_t* __restrict__ list, int32_t* rows,
                              int32_t* node_of_row, int32_t* node_begin, int32_t* node_end) {
  const int64_t NH = heap_nodes(p);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < p.n; i += (int64_t)gridDim.x * blockDim.x) {
    if (rows) rows[i] = list[i];
    if (node_of_row) node_of_row[i] = s.nid[i];
  }
  for (int64_t h = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; h < NH; h += (int64_t)gridDim.x * blockDim.x) {
    if (node_begin) node_begin[h] = s.node_begin[h];
    if (node_end) node_end[h] = s.node_end[h];
  }
}

}  // namespace gbdtmo

using namespace gbdtmo;

extern "C" gbdtmo_status gbdtmo_rows_export(gbdtmo_ctx c, const gbdtmo_problem* p, const void* state, int32_t level,
                                            int32_t* rows, int32_t* node_of_row, int32_t* node_begin,
                                            int32_t* node_end) {
  Ctx* ctx = (Ctx*)c;
  DeviceGuard device_guard_(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(state && level >= 0 && level <= p->D, "null state or level out of range [0, D]");
  State s = state_view(*p, const_cast<void*>(state));
  GB_LAUNCH(k_rows_export, ctx->num_sms, 256, 0, *p, s, (level & 1) ? s.rows1 : s.rows0, rows, node_of_row,
            node_begin, node_end);
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_leaf_values(gbdtmo_ctx c, const gbdtmo_problem* p, const float* scales,
                                            void* state, double* leaf) {
  Ctx* ctx = (Ctx*)c;
  DeviceGuard device_guard_(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(scales && state && leaf, "null pointer");
  State s = state_view(*p, state);
  GB_LAUNCH(k_leaf_values, 64, 256, 0, *p, scales, s, leaf);
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_update_pred(gbdtmo_ctx c, const gbdtmo_problem* p, const void* state,
                                            const double* leaf, double* pred) {
  Ctx* ctx = (Ctx*)c;
  DeviceGuard device_guard_(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(state && leaf && pred, "null pointer");
  State s = state_view(*p, const_cast<void*>(state));
  GB_LAUNCH(k_update_pred, ctx->num_sms * 8, 256, 0, *p, s, leaf, pred);
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_tree_export(gbdtmo_ctx c, const gbdtmo_problem* p, const void* state,
                                            int32_t* node_state, int32_t* feature, int32_t* bin, double* gain,
                                            int64_t* n_rows, int64_t* n_left, const float* cuts, float* threshold) {
  Ctx* ctx = (Ctx*)c;
  DeviceGuard device_guard_(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(state, "null pointer");
  GB_CHECK_ARG(!threshold || cuts, "threshold requires cuts");
  State s = state_view(*p, const_cast<void*>(state));
  GB_LAUNCH(k_tree_export, 16, 256, 0, *p, s, node_state, feature, bin, gain, n_rows, n_left, cuts, threshold);
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_predict(gbdtmo_ctx c, const float* X, int64_t n, int64_t ld_x, int32_t T, int32_t D,
                                        int32_t d, const int32_t* node_state, const int32_t* feature,
                                        const float* threshold, const double* leaf, double* pred) {
  Ctx* ctx = (Ctx*)c;
  DeviceGuard device_guard_(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  GB_CHECK_ARG(X && node_state && feature && threshold && leaf && pred, "null pointer");
  GB_CHECK_ARG(n >= 0 && T >= 0 && D >= 0 && D <= 20 && d >= 1, "bad shape");
  if (n == 0 || T == 0) return GBDTMO_OK;
  GB_LAUNCH(k_predict, ctx->num_sms * 8, 256, 0, X, n, ld_x, T, D, d, node_state, feature, threshold, leaf, pred);
  return GBDTMO_OK;
}
