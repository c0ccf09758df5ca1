// grad.cu — (a)2: per-output g/h (softmax reading R12), fixed-point
// quantisation, exact root sums, and tree initialisation.
#include "common.cuh"
#include "plan.cuh"

namespace gbdtmo {

__global__ void k_tree_reset(gbdtmo_problem p, State s) {
  const int64_t NH = heap_nodes(p), V = channels(p);
  for (int64_t h = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; h < NH; h += (int64_t)gridDim.x * blockDim.x) {
    s.node_begin[h] = 0; s.node_end[h] = 0; s.node_state[h] = GBDTMO_NODE_NONE; s.node_mode[h] = MODE_NONE;
    s.node_feat[h] = -1; s.node_bin[h] = -1; s.node_gain[h] = 0.0; s.node_nleft[h] = 0;
    for (int64_t c = 0; c <= V; ++c) s.node_sum[h * (V + 1) + c] = 0;
  }
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < V; c += (int64_t)gridDim.x * blockDim.x)
    s.scale_max[c] = 0ull;
}

// MSE pass 1: S_k = max_i |g_ik| with g = 2 (yhat - y) in fp64.
__global__ void k_mse_max(gbdtmo_problem p, const float* __restrict__ y, const double* __restrict__ pred, State s) {
  const int d = p.d;
  // block (32, 8): x = channel within a group of 32, y = row
  __shared__ double red[8][33];
  for (int c0 = 0; c0 < d; c0 += 32) {
    const int c = c0 + threadIdx.x;
    double mx = 0.0;
    if (c < d)
      for (int64_t i = blockIdx.x * 8 + threadIdx.y; i < p.n; i += (int64_t)gridDim.x * 8)
        mx = fmax(mx, fabs(2.0 * (pred[i * d + c] - (double)y[i * d + c])));
    red[threadIdx.y][threadIdx.x] = mx;
    __syncthreads();
    if (threadIdx.y == 0 && c < d) {
      for (int r = 1; r < 8; ++r) mx = fmax(mx, red[r][threadIdx.x]);
      if (mx > 0.0) atomicMax(&s.scale_max[c], (unsigned long long)__double_as_longlong(mx));
    }
    __syncthreads();
  }
}

// log2 of P = 2^ceil(log2 S) (S > 0); P = 1 for S = 0.
__device__ __forceinline__ int pow2_exponent(double S) {
  if (!(S > 0.0)) return 0;
  int e;
  double mant = frexp(S, &e);          // S = mant * 2^e, mant in [0.5, 1)
  return mant == 0.5 ? e - 1 : e;
}

// MSE pass 2: q = rint(g * 2^(30 - log2 P)), exact root sums.  block (32, 8): x = channel, y = row.
__global__ void k_mse_quantize(gbdtmo_problem p, const float* __restrict__ y, const double* __restrict__ pred,
                               int32_t* __restrict__ q, float* __restrict__ scales, State s, double* __restrict__ gh) {
  __shared__ long long red[8][33];
  const int d = p.d;
  for (int c0 = 0; c0 < d; c0 += 32) {
    const int c = c0 + threadIdx.x;
    const bool on = c < d;
    const int ex = on ? pow2_exponent(__longlong_as_double((long long)s.scale_max[c])) : 0;
    long long acc = 0;
    if (on) {
      for (int64_t i = blockIdx.x * 8 + threadIdx.y; i < p.n; i += (int64_t)gridDim.x * 8) {
        const double g = 2.0 * (pred[i * d + c] - (double)y[i * d + c]);
        if (gh) gh[i * d + c] = g;                      // fp64 g for the leaf values (R17)
        const int qi = __double2int_rn(ldexp(g, kQShift - ex));
        q[i * d + c] = qi;
        acc += qi;
      }
    }
    red[threadIdx.y][threadIdx.x] = acc;
    __syncthreads();
    if (threadIdx.y == 0 && on) {
      long long t = 0;
      for (int r = 0; r < 8; ++r) t += red[r][threadIdx.x];
      atomicAdd((unsigned long long*)&s.node_sum[c], (unsigned long long)t);
      if (blockIdx.x == 0) scales[c] = ldexpf(1.0f, ex - kQShift);
    }
    __syncthreads();
  }
}

// Softmax (fp64): one warp per row; p = softmax(yhat) (max-subtracted), g = p - y, h = p (1 - p);
// q_g = rint(g 2^30) (P = 1), q_h = rint(h 2^32) (P = 1/4).  Any d (lanes stride the outputs;
// exp is recomputed instead of held in registers).
__global__ void k_softmax_quantize(gbdtmo_problem p, const float* __restrict__ y, const double* __restrict__ pred,
                                   int32_t* __restrict__ q, float* __restrict__ scales, State s,
                                   double* __restrict__ gh) {
  const int d = p.d, V = 2 * d;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  for (int64_t i = blockIdx.x * (int64_t)nw + warp; i < p.n; i += (int64_t)gridDim.x * nw) {
    const double* pr = pred + i * d;
    double mx = -INFINITY;
    for (int c = lane; c < d; c += 32) mx = fmax(mx, pr[c]);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    double sum = 0.0;
    for (int c = lane; c < d; c += 32) sum += exp(pr[c] - mx);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
    for (int c = lane; c < d; c += 32) {
      const double pk = exp(pr[c] - mx) / sum;
      const double g = pk - (double)y[i * d + c];
      const double h = pk * (1.0 - pk);
      q[i * V + c] = __double2int_rn(ldexp(g, kQShift));
      q[i * V + d + c] = __double2int_rn(ldexp(h, kQShift + 2));
      if (gh) { gh[i * V + c] = g; gh[i * V + d + c] = h; }   // fp64 g, h for the leaf values (R17)
    }
  }
  if (blockIdx.x == 0) {
    for (int c = threadIdx.x; c < d; c += blockDim.x) {
      scales[c] = ldexpf(1.0f, -kQShift);
      scales[d + c] = ldexpf(1.0f, -kQShift - 2);
    }
  }
}

// Exact column sums of q (root node totals).  block (32, 8): x = column within a group of 32.
__global__ void k_qsum(gbdtmo_problem p, const int32_t* __restrict__ q, State s) {
  __shared__ long long red[8][33];
  const int V = channels(p);
  for (int c0 = 0; c0 < V; c0 += 32) {
    const int c = c0 + threadIdx.x;
    long long acc = 0;
    if (c < V)
      for (int64_t i = blockIdx.x * 8 + threadIdx.y; i < p.n; i += (int64_t)gridDim.x * 8) acc += q[i * V + c];
    red[threadIdx.y][threadIdx.x] = acc;
    __syncthreads();
    if (threadIdx.y == 0 && c < V) {
      long long t = 0;
      for (int r = 0; r < 8; ++r) t += red[r][threadIdx.x];
      atomicAdd((unsigned long long*)&s.node_sum[c], (unsigned long long)t);
    }
    __syncthreads();
  }
}

__global__ void k_rows_init(gbdtmo_problem p, State s) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < p.n; i += (int64_t)gridDim.x * blockDim.x) {
    s.rows0[i] = (int32_t)i;
    s.nid[i] = 0;
  }
}

__global__ void k_root_plan(gbdtmo_problem p, State s, int target_chunks, int64_t gmem_max_rows,
                            int64_t small_max_rows) {
  const int64_t V = channels(p);
  if (threadIdx.x == 0) {
    s.node_begin[0] = 0;
    s.node_end[0] = (int32_t)p.n;
    s.node_sum[V] = p.n;
    bool active = p.D >= 1 && p.n >= 2 * (int64_t)p.min_node;
    s.node_state[0] = active ? GBDTMO_NODE_ACTIVE : GBDTMO_NODE_LEAF;
    s.node_mode[0] = active ? (p.n <= small_max_rows ? MODE_SMALL : MODE_BUILD) : MODE_NONE;
  }
  __syncthreads();
  plan_level_chunks(p, s, 0, target_chunks, gmem_max_rows);
}

int target_chunks_for(const Ctx* ctx, const gbdtmo_problem& p) {
  HistCfg hc = ctx->hist_kernel == 1 ? hist_config_diag(p)
               : (ctx->hist_kernel == 2 && hist_tma_supported(p, nullptr)) ? hist_config_tma(p, ctx->max_smem_optin)
                                                                          : hist_config(p);
  int64_t tiles = (int64_t)hc.n_ft * hc.n_ct;
#ifndef GBDTMO_HIST_WAVES
#define GBDTMO_HIST_WAVES 2   // default work items wanted per level, in multiples of the SM count
#endif
  // fewer waves: fewer chunks per node, so more nodes are built by a single item per tile (plain
  // stores, no zeroing of the node's slot); more waves: better balance.  Per shape by measurement
  // (GBDTMO_OPT_HIST_WAVES from the variant table): C2 4.62 / 4.42 / 4.28 ms per tree at 4 / 2 / 1.
  const int64_t waves = ctx->hist_waves > 0 ? ctx->hist_waves : GBDTMO_HIST_WAVES;
  int64_t want = waves * ctx->num_sms * kHistCtas;
  int64_t t = (want + tiles - 1) / tiles;
  return (int)(t < 1 ? 1 : t);
}

}  // namespace gbdtmo

using namespace gbdtmo;

extern "C" gbdtmo_status gbdtmo_grad(gbdtmo_ctx c, const gbdtmo_problem* p, const float* y, const double* pred,
                                     int32_t* q, float* scales, void* state, double* gh) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(y && pred && q && scales && state, "null pointer");
  State s = state_view(*p, state);
  const int sms = ctx->num_sms;
  GB_LAUNCH(k_tree_reset, sms, 256, 0, *p, s);
  if (p->loss == GBDTMO_LOSS_MSE) {
    GB_LAUNCH(k_mse_max, sms * 4, dim3(32, 8), 0, *p, y, pred, s);
    GB_LAUNCH(k_mse_quantize, sms * 4, dim3(32, 8), 0, *p, y, pred, q, scales, s, gh);
  } else {
    GB_LAUNCH(k_softmax_quantize, sms * 4, 256, 0, *p, y, pred, q, scales, s, gh);
    GB_LAUNCH(k_qsum, sms * 4, dim3(32, 8), 0, *p, q, s);
  }
  GB_LAUNCH(k_rows_init, sms * 4, 256, 0, *p, s);
  GB_LAUNCH(k_root_plan, 1, kPlanThreads, 0, *p, s, target_chunks_for(ctx, *p), ctx->gmem_max_rows,
            small_rows(ctx, *p));
  return GBDTMO_OK;
}
