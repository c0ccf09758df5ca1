// leaf.cu — (a)8 leaf values and (a)9 incremental prediction update,
// plus the export of the heap-indexed tree record.
#include "common.cuh"
#include "plan.cuh"

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

// Leaf values from fp64 node totals summed from the leaf's rows (reading R17; the oracle's
// definition), not from the 31-bit fixed-point sums: gbdtmo_grad keeps the fp64 g, h it quantises
// (gh), so a leaf whose rows all have tiny |g| (confident softmax rows: G ~ 1e-3 against a
// quantisation floor of n 2^-31) is exact to fp64 rounding.  Deterministic, in three steps:
//   k_leaf_plan     every leaf's segment of the final row list is cut into chunks of <= kLeafRows
//   k_leaf_partial  one block per chunk: warp w sums rows w, w + 8, ... in order, lanes over
//                   channels; the 8 warps' sums are added in warp order
//   k_leaf_final    one block per leaf: its chunks' partials added in chunk order, then Eq.
// The order depends only on the row list, so the result is identical on every rank and run.
constexpr int kLeafPartWarps = 8;

__global__ void k_leaf_plan(gbdtmo_problem p, State s) {
  const int64_t NH = heap_nodes(p);
  __shared__ int sh_base;
  if (threadIdx.x == 0) sh_base = 0;
  __syncthreads();
  for (int64_t h0 = 0; h0 < NH; h0 += blockDim.x) {
    const int64_t h = h0 + threadIdx.x;
    int nch = 0, b = 0, e = 0;
    if (h < NH && s.node_state[h] == GBDTMO_NODE_LEAF) {
      b = s.node_begin[h]; e = s.node_end[h];
      nch = (e - b + kLeafRows - 1) / kLeafRows;
    }
    int total;
    const int off = block_excl_scan_256(nch, &total) + sh_base;
    if (h < NH) s.leaf_c0[h] = off;
    for (int c = 0; c < nch; ++c) {
      const int cb = b + c * kLeafRows;
      s.leaf_chunk[off + c] = make_int4((int)h, cb, cb + kLeafRows < e ? cb + kLeafRows : e, 0);
    }
    __syncthreads();
    if (threadIdx.x == 0) sh_base += total;
    __syncthreads();
  }
  if (threadIdx.x == 0) s.leaf_c0[NH] = sh_base;
}

__global__ void __launch_bounds__(kLeafPartWarps * 32)
k_leaf_partial(gbdtmo_problem p, const double* __restrict__ gh, State s) {
  __shared__ double part[kLeafPartWarps][32];
  const int64_t NH = heap_nodes(p);
  const int V = channels(p);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int32_t* rl = (p.D & 1) ? s.rows1 : s.rows0;    // the list after the last level's partition
  const int nchunks = s.leaf_c0[NH];
  for (int ch = blockIdx.x; ch < nchunks; ch += gridDim.x) {
    const int4 c4 = s.leaf_chunk[ch];
    for (int c0 = 0; c0 < V; c0 += 32) {
      const int c = c0 + lane;
      double acc = 0.0;
      int pos = c4.y + warp;
      for (; pos + 3 * kLeafPartWarps < c4.z; pos += 4 * kLeafPartWarps) {   // 4 rows in flight, in order
        double v[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) v[u] = c < V ? gh[(int64_t)rl[pos + u * kLeafPartWarps] * V + c] : 0.0;
#pragma unroll
        for (int u = 0; u < 4; ++u) acc += v[u];
      }
      for (; pos < c4.z; pos += kLeafPartWarps)
        if (c < V) acc += gh[(int64_t)rl[pos] * V + c];
      part[warp][lane] = acc;
      __syncthreads();
      if (warp == 0 && c < V) {
        double t = 0.0;
#pragma unroll
        for (int w = 0; w < kLeafPartWarps; ++w) t += part[w][lane];
        s.leaf_part[(int64_t)ch * V + c] = t;
      }
      __syncthreads();
    }
  }
}

__global__ void k_leaf_final(gbdtmo_problem p, State s, double* __restrict__ leaf) {
  const int64_t h = blockIdx.x;
  const int d = p.d, V = channels(p);
  const bool softmax = p.loss == GBDTMO_LOSS_SOFTMAX;
  const bool is_leaf = s.node_state[h] == GBDTMO_NODE_LEAF;
  const int c0 = s.leaf_c0[h], c1 = is_leaf ? s.leaf_c0[h + 1] : c0;
  const double cntd = (double)s.node_sum[h * (V + 1) + V];
  for (int k = threadIdx.x; k < d; k += blockDim.x) {
    double v = 0.0;
    if (is_leaf) {
      double G = 0.0, H = 0.0;
      for (int ch = c0; ch < c1; ++ch) {
        G += s.leaf_part[(int64_t)ch * V + k];
        if (softmax) H += s.leaf_part[(int64_t)ch * V + d + k];
      }
      if (!softmax) H = 2.0 * cntd;                      // MSE: h = 2 for every row
      v = -p.lr * G / (H + p.lambda);
    }
    leaf[h * d + k] = v;
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
// Inference for unseen rows (instance-level and tree-level parallelism).
// A block owns a tile of RB rows at a time (persistent over tiles):
//   1. the tile's rows are staged in shared memory (coalesced; row stride mp = m | 1, so 32 rows
//      reading the same feature hit 32 different banks);
//   2. tree-level x instance-level walk: thread pairs (row r, tree t) of a chunk of TC trees walk
//      tree t from the root for row r (x < threshold -> left, reading R15) and park the leaf id
//      in shared memory; consecutive lanes take consecutive rows of the same tree, so node
//      loads are broadcast near the root;
//   3. lanes over (row, output) add the chunk's leaf values in tree order (fp64, the same
//      sequential order as the training path's update_pred, so predictions of training rows are
//      bit-identical to the training prediction).
// Without staging (rows wider than the shared-memory budget) the walk reads X from global memory.
constexpr int kPredThreads = 512;
constexpr int kPredW = 4;             // walks per thread in flight

__device__ __forceinline__ void cp_async4(float* dst, const float* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"((uint32_t)__cvta_generic_to_shared(dst)), "l"(src)
               : "memory");
}

__global__ void __launch_bounds__(kPredThreads)
k_predict_tiles(const float* __restrict__ X, int64_t n, int m, int64_t ld_x, int T, int D, int d, int lrb, int TC,
                int stage, const int32_t* __restrict__ node_state, const int32_t* __restrict__ feature,
                const float* __restrict__ threshold, const double* __restrict__ leaf, double* __restrict__ pred) {
  extern __shared__ __align__(16) unsigned char smp[];
  const int RB = 1 << lrb;
  const int mp = m | 1;
  float* const xs0 = reinterpret_cast<float*>(smp);
  const int bufw = stage ? RB * mp : 0;                  // floats per staging buffer
  int16_t* lh = reinterpret_cast<int16_t*>(smp + (stage ? (size_t)2 * RB * mp * 4 : 0));
  const int64_t NH = (int64_t(1) << (D + 1)) - 1;
  const int64_t ntiles = (n + RB - 1) >> lrb;
  // rows of a tile are copied asynchronously (cp.async, no register round trip) one tile ahead:
  // the next tile lands while this one is walked
  auto stage_tile = [&](int64_t tile, float* xs) {
    if (tile < ntiles) {
      const int64_t r0 = tile << lrb;
      const int rows = (int)min((int64_t)RB, n - r0);
      for (int r = 0; r < rows; ++r) {
        const float* src = X + (r0 + r) * ld_x;
        float* dst = xs + r * mp;
        for (int j = threadIdx.x; j < m; j += blockDim.x) cp_async4(dst + j, src + j);
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  int buf = 0;
  if (stage) stage_tile(blockIdx.x, xs0);
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t r0 = tile << lrb;
    const int rows = (int)min((int64_t)RB, n - r0);
    const float* xs = xs0 + buf * bufw;
    if (stage) {
      stage_tile(tile + gridDim.x, xs0 + (buf ^ 1) * bufw);
      asm volatile("cp.async.wait_group 1;" ::: "memory");
      __syncthreads();
    }
    for (int t0 = 0; t0 < T; t0 += TC) {
      const int tc = min(TC, T - t0);
      // kPredW (row, tree) walks per thread advance level by level together: the node loads of all
      // of them are in flight at once (memory-level parallelism for the latency-bound walk)
      for (int pq0 = threadIdx.x; pq0 < (tc << lrb); pq0 += kPredW * blockDim.x) {
        int64_t c[kPredW];
        int sc[kPredW], f[kPredW], r_[kPredW], t_[kPredW];
        float th[kPredW];
#pragma unroll
        for (int w = 0; w < kPredW; ++w) {
          const int pq = pq0 + w * blockDim.x;
          r_[w] = pq & (RB - 1);
          t_[w] = pq >> lrb;
          c[w] = 0;
          sc[w] = GBDTMO_NODE_NONE;
          if (pq < (tc << lrb) && r_[w] < rows) {
            const int64_t to = (int64_t)(t0 + t_[w]) * NH;
            sc[w] = __ldg(&node_state[to]);
            f[w] = __ldg(&feature[to]);
            th[w] = __ldg(&threshold[to]);
          }
        }
        for (int lv = 0; lv <= D; ++lv) {
          bool any = false;
#pragma unroll
          for (int w = 0; w < kPredW; ++w) {
            if (sc[w] != GBDTMO_NODE_SPLIT) continue;
            if ((unsigned)f[w] >= (unsigned)m) { sc[w] = GBDTMO_NODE_NONE; continue; }   // (malformed model)
            const float x = stage ? xs[r_[w] * mp + f[w]] : __ldg(&X[(r0 + r_[w]) * ld_x + f[w]]);
            c[w] = (x < th[w]) ? 2 * c[w] + 1 : 2 * c[w] + 2;
            if (c[w] >= NH) { sc[w] = GBDTMO_NODE_NONE; continue; }
            const int64_t o = (int64_t)(t0 + t_[w]) * NH + c[w];
            sc[w] = __ldg(&node_state[o]);
            f[w] = __ldg(&feature[o]);
            th[w] = __ldg(&threshold[o]);
            any = true;
          }
          if (!any) break;
        }
#pragma unroll
        for (int w = 0; w < kPredW; ++w) {
          const int pq = pq0 + w * blockDim.x;
          if (pq < (tc << lrb)) lh[(r_[w] * TC) + t_[w]] = (int16_t)(sc[w] == GBDTMO_NODE_LEAF ? (int)c[w] : -1);
        }
      }
      __syncthreads();
      for (int e = threadIdx.x; e < rows * d; e += blockDim.x) {
        const int r = e / d, k = e - r * d;
        double* pp = pred + (r0 + r) * d + k;
        double acc = *pp;
        const int16_t* hr = lh + r * TC;
        int t = 0;
        for (; t + 8 <= tc; t += 8) {                    // 8 leaf loads in flight, added in tree order
          double v[8];
#pragma unroll
          for (int u = 0; u < 8; ++u) {
            const int h = hr[t + u];
            v[u] = h >= 0 ? __ldg(&leaf[((int64_t)(t0 + t + u) * NH + h) * d + k]) : 0.0;
          }
#pragma unroll
          for (int u = 0; u < 8; ++u)
            if (hr[t + u] >= 0) acc += v[u];
        }
        for (; t < tc; ++t) {
          const int h = hr[t];
          if (h >= 0) acc += __ldg(&leaf[((int64_t)(t0 + t) * NH + h) * d + k]);
        }
        *pp = acc;
      }
      __syncthreads();
    }
    buf ^= 1;
  }
  asm volatile("cp.async.wait_group 0;" ::: "memory");
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
  GB_ENTRY(ctx);
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
                                            void* state, const double* gh, double* leaf) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(state && leaf, "null pointer");
  State s = state_view(*p, state);
  if (gh) {
    GB_LAUNCH(k_leaf_plan, 1, kPlanThreads, 0, *p, s);
    int64_t grid = ctx->num_sms * 8;
    if (grid > leaf_chunks_max(*p)) grid = leaf_chunks_max(*p);
    GB_LAUNCH(k_leaf_partial, (unsigned)grid, kLeafPartWarps * 32, 0, *p, gh, s);
    GB_LAUNCH(k_leaf_final, (unsigned)heap_nodes(*p), 128, 0, *p, s, leaf);
  } else {
    GB_CHECK_ARG(scales, "null scales");
    GB_LAUNCH(k_leaf_values, 64, 256, 0, *p, scales, s, leaf);
  }
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_update_pred(gbdtmo_ctx c, const gbdtmo_problem* p, const void* state,
                                            const double* leaf, double* pred) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
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
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(state, "null pointer");
  GB_CHECK_ARG(!threshold || cuts, "threshold requires cuts");
  State s = state_view(*p, const_cast<void*>(state));
  GB_LAUNCH(k_tree_export, 16, 256, 0, *p, s, node_state, feature, bin, gain, n_rows, n_left, cuts, threshold);
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_predict(gbdtmo_ctx c, const float* X, int64_t n, int32_t m, int64_t ld_x, int32_t T,
                                        int32_t D, int32_t d, const int32_t* node_state, const int32_t* feature,
                                        const float* threshold, const double* leaf, double* pred) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  GB_CHECK_ARG(X && node_state && feature && threshold && leaf && pred, "null pointer");
  GB_CHECK_ARG(n >= 0 && T >= 0 && m >= 1 && ld_x >= m && d >= 1, "bad shape");
  GB_CHECK_ARG(D >= 1 && D <= 12, "D out of range [1, 12]");
  if (n == 0 || T == 0) return GBDTMO_OK;
  // rows per tile: rows of <= 1024 features are staged in shared memory (two buffers of up to 32 KB:
  // the next tile is copied while this one is walked); wider rows are read from global memory
  // (L1 / L2: a walk touches D of the m values) with 32-row tiles, so a tile holds 32 T walks
  const int64_t row_bytes = 4 * (int64_t)(m | 1);
  int lrb = 6;
  while (lrb > 0 && (int64_t(1) << lrb) * row_bytes > 32 * 1024) --lrb;
  const int stage = m <= 1024 && (int64_t(1) << lrb) * row_bytes <= 32 * 1024;
  if (!stage) lrb = 5;
  const int RB = 1 << lrb;
  const int TC = T < 256 ? T : 256;
  const int smem = (stage ? 2 * (int)(RB * row_bytes) : 0) + RB * TC * 2;   // two staging buffers
  static unsigned long long attr_mask = 0;
  smem_optin_once(ctx, k_predict_tiles, attr_mask, 200 * 1024);
  const int64_t ntiles = (n + RB - 1) / RB;
  int per_sm = (int)(ctx->max_smem_optin / (smem + 1024));
  per_sm = per_sm < 1 ? 1 : per_sm > 4 ? 4 : per_sm;
  int64_t grid = (int64_t)ctx->num_sms * per_sm;
  if (grid > ntiles) grid = ntiles;
  GB_LAUNCH(k_predict_tiles, (unsigned)grid, kPredThreads, smem, X, n, m, ld_x, T, D, d, lrb, TC, stage, node_state,
            feature, threshold, leaf, pred);
  return GBDTMO_OK;
}
