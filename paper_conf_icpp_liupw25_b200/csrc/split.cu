// split.cu — (a)4 sibling histogram by subtraction, (a)5 multi-output split search, and the
// (a)6 exchange payload (split records + row-direction bitmap).
//
// Split search: for node N, feature f, bin b (left = bins <= b):
//   G_L^k, H_L^k, C_L = prefix sums over bins (exact int64 fixed point, MSE: H = 2 C),
//   gain = 1/2 sum_k [G_L^2/(H_L+l) + G_R^2/(H_R+l) - G^2/(H+l)]   (Eq. 3, fp64),
// valid iff C_L, C_R >= min_node; best per node by an atomicMax on a packed 64-bit key.
#include "common.cuh"

namespace gbdtmo {

constexpr int kFsFeatures = 2;   // features per block (looped)
constexpr int kFsChunk = 8;      // channels (outputs) scanned together per pass

__device__ __forceinline__ uint64_t pack_key(double gain, int64_t fb) {
  return ((uint64_t)__double_as_longlong(gain) & ~0xFFFFFFull) | (uint64_t)(0xFFFFFF - fb);
}

// Block-wide inclusive scan over bins (thread = bin) of N int64 values per thread; also
// returns the grand totals.  ws: shared [32][N] scratch.
template <int N>
__device__ __forceinline__ void block_scan_bins(long long (&v)[N], long long (&tot)[N], long long* ws) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
#pragma unroll
    for (int k = 0; k < N; ++k) {
      const long long y = __shfl_up_sync(0xffffffffu, v[k], o);
      if (lane >= o) v[k] += y;
    }
  }
  if (lane == 31) {
#pragma unroll
    for (int k = 0; k < N; ++k) ws[warp * N + k] = v[k];
  }
  __syncthreads();
#pragma unroll
  for (int k = 0; k < N; ++k) {
    long long off = 0, t = 0;
    for (int w = 0; w < nw; ++w) {
      const long long x = ws[w * N + k];
      off += (w < warp) ? x : 0;
      t += x;
    }
    v[k] += off;
    tot[k] = t;
  }
  __syncthreads();
}

// One block per (node slot, kFsFeatures features); thread = bin.  For every channel chunk the
// bins' values (derived nodes: parent - sibling, written back when needed) are prefix-summed
// across the block; MSE accumulates sum_k G_L^2 and sum_k G_R^2 (H = 2 C is shared by all
// outputs, so only two divisions per bin are needed), softmax accumulates the Eq. (3) terms.
template <bool SOFTMAX>
__global__ void __launch_bounds__(256)
k_find_split(gbdtmo_problem p, int level, const int32_t* __restrict__ nbins, const float* __restrict__ scales,
             State s, int64_t* __restrict__ hist, int32_t* __restrict__ cnt,
             const int64_t* __restrict__ phist, const int32_t* __restrict__ pcnt,
             uint64_t* __restrict__ keys, int write_derived) {
  const int slot = blockIdx.y;
  const int64_t h = (int64_t(1) << level) - 1 + slot;
  if (s.node_state[h] != GBDTMO_NODE_ACTIVE) return;
  const bool derive = s.node_mode[h] == MODE_DERIVE;
  const bool store = derive && write_derived;
  const int V = channels(p), B = p.B, m = p.m, d = p.d;
  constexpr bool softmax = SOFTMAX;
  constexpr int NS = SOFTMAX ? 2 * kFsChunk : kFsChunk;   // scanned values per bin per pass
  const int b = threadIdx.x;                     // this thread's bin
  const bool bon = b < B;
  const int sib = slot ^ 1, par = slot >> 1;
  const double lam = p.lambda;
  __shared__ long long ws[32 * 2 * kFsChunk];
  __shared__ unsigned long long wbest[32];
  uint64_t best = 0;

  for (int fi = 0; fi < kFsFeatures; ++fi) {
    const int f = blockIdx.x * kFsFeatures + fi;
    if (f >= m) break;
    const int64_t row_cur = ((int64_t)slot * m + f) * B + b;
    const int64_t row_sib = ((int64_t)sib * m + f) * B + b;
    const int64_t row_par = ((int64_t)par * m + f) * B + b;
    // counts
    long long cv[1] = {0}, ct[1];
    if (bon) {
      if (derive) {
        const int x = pcnt[row_par] - cnt[row_sib];
        if (store) cnt[row_cur] = x;
        cv[0] = x;
      } else {
        cv[0] = cnt[row_cur];
      }
    }
    block_scan_bins<1>(cv, ct, ws);
    const long long cl = cv[0], ctot = ct[0];
    double accL = 0.0, accR = 0.0, P = 0.0;          // MSE: sums of squares; softmax: Eq. (3) terms
    const int64_t* hc = hist + row_cur * V;
    const int64_t* hs = hist + row_sib * V;
    const int64_t* hp = phist + row_par * V;
    int64_t* hw = hist + row_cur * V;
    for (int k0 = 0; k0 < d; k0 += kFsChunk) {
      long long gv[NS], gt[NS];
#pragma unroll
      for (int u = 0; u < kFsChunk; ++u) {
        const int k = k0 + u;
        long long x = 0, y = 0;
        if (bon && k < d) {
          if (derive) {
            x = hp[k] - hs[k];
            if (store) hw[k] = x;
            if (softmax) { y = hp[d + k] - hs[d + k]; if (store) hw[d + k] = y; }
          } else {
            x = hc[k];
            if (softmax) y = hc[d + k];
          }
        }
        gv[u] = x;
        if (SOFTMAX) gv[(kFsChunk + u) % NS] = y;
      }
      block_scan_bins<NS>(gv, gt, ws);
#pragma unroll
      for (int u = 0; u < kFsChunk; ++u) {
        const int k = k0 + u;
        if (k < d) {
          const double sg = (double)scales[k];
          const double GL = (double)gv[u] * sg, GR = (double)(gt[u] - gv[u]) * sg, G = (double)gt[u] * sg;
          if (!softmax) {
            accL = fma(GL, GL, accL);
            accR = fma(GR, GR, accR);
            P = fma(G, G, P);
          } else {
            const double sh = (double)scales[d + k];
            const int uh = (kFsChunk + u) % NS;
            const double HL = (double)gv[uh] * sh, H = (double)gt[uh] * sh;
            const double HR = (double)(gt[uh] - gv[uh]) * sh;
            accL += GL * GL / (HL + lam) + GR * GR / (HR + lam);
            P += G * G / (H + lam);
          }
        }
      }
    }
    if (bon && b <= nbins[f] - 2 && cl >= p.min_node && ctot - cl >= p.min_node) {
      double gain;
      if (!softmax) {
        gain = 0.5 * (accL / (2.0 * (double)cl + lam) + accR / (2.0 * (double)(ctot - cl) + lam) -
                      P / (2.0 * (double)ctot + lam));
      } else {
        gain = 0.5 * (accL - P);
      }
      if (gain > p.gamma) {
        const uint64_t key = pack_key(gain, (int64_t)(p.f_begin + f) * B + b);
        best = key > best ? key : best;
      }
    }
  }
  // block max of the packed keys -> one atomicMax per block
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const uint64_t y = __shfl_xor_sync(0xffffffffu, best, o);
    best = y > best ? y : best;
  }
  if (lane == 0) wbest[warp] = best;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint64_t bb = 0;
    for (int w = 0; w < nw; ++w) bb = wbest[w] > bb ? wbest[w] : bb;
    if (bb) atomicMax((unsigned long long*)&keys[slot], (unsigned long long)bb);
  }
}

__global__ void k_zero_u64(uint64_t* p, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) p[i] = 0;
}

// ---------------------------------------------------------------- exchange payload

__device__ __forceinline__ bool decode_local(const gbdtmo_problem& p, uint64_t key, int* fl, int* b, int* fg) {
  if (!key) return false;
  const int idx = 0xFFFFFF - (int)(key & 0xFFFFFFull);
  *fg = idx / p.B;
  *b = idx - *fg * p.B;
  *fl = *fg - p.f_begin;
  return *fl >= 0 && *fl < p.m;
}

// One block per slot: left sums at the winning (feature, bin) if the feature is local.
__global__ void k_split_record(gbdtmo_problem p, int level, State s, const int64_t* __restrict__ hist,
                               const int32_t* __restrict__ cnt, const int64_t* __restrict__ phist,
                               const int32_t* __restrict__ pcnt, const uint64_t* __restrict__ keys,
                               const float* __restrict__ scales, int64_t* __restrict__ xchg) {
  const int slot = blockIdx.x;
  const int64_t h = (int64_t(1) << level) - 1 + slot;
  const int V = channels(p), B = p.B, m = p.m;
  const int64_t RW = rec_words(p);
  int64_t* rec = xchg + slot * RW;
  int fl = 0, b = 0, fg = 0;
  const bool own = s.node_state[h] == GBDTMO_NODE_ACTIVE && decode_local(p, keys[slot], &fl, &b, &fg);
  if (!own) {
    for (int i = threadIdx.x; i < RW; i += blockDim.x) rec[i] = 0;
    return;
  }
  const bool derive = s.node_mode[h] == MODE_DERIVE;
  const int sib = slot ^ 1, par = slot >> 1;
  const int64_t rc = ((int64_t)slot * m + fl) * B, rs = ((int64_t)sib * m + fl) * B, rp = ((int64_t)par * m + fl) * B;
  for (int c = threadIdx.x; c < V; c += blockDim.x) {
    long long acc = 0;
    for (int bb = 0; bb <= b; ++bb)
      acc += derive ? (phist[(rp + bb) * V + c] - hist[(rs + bb) * V + c]) : hist[(rc + bb) * V + c];
    rec[c] = acc;
  }
  if (threadIdx.x == 0) {
    long long cl = 0;
    for (int bb = 0; bb <= b; ++bb) cl += derive ? (pcnt[rp + bb] - cnt[rs + bb]) : cnt[rc + bb];
    rec[V] = cl;
    rec[V + 1] = fg + 1;
    rec[V + 2] = b;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    // exact Eq. (3) at the winner from the exact sums (informational: the tree record's gain)
    const int d = p.d;
    const bool softmax = p.loss == GBDTMO_LOSS_SOFTMAX;
    const int64_t* S = s.node_sum + h * (V + 1);
    const long long ctot = S[V], cl = rec[V];
    double g = 0.0;
    for (int k = 0; k < d; ++k) {
      const double sg = (double)scales[k];
      const double GL = (double)rec[k] * sg, G = (double)S[k] * sg, GR = (double)(S[k] - rec[k]) * sg;
      double HL, H, HR;
      if (softmax) {
        const double sh = (double)scales[d + k];
        HL = (double)rec[d + k] * sh; H = (double)S[d + k] * sh; HR = (double)(S[d + k] - rec[d + k]) * sh;
      } else {
        HL = 2.0 * cl; H = 2.0 * ctot; HR = 2.0 * (ctot - cl);
      }
      g += GL * GL / (HL + p.lambda) + GR * GR / (HR + p.lambda) - G * G / (H + p.lambda);
    }
    rec[V + 3] = __double_as_longlong(0.5 * g);
  }
}

// Row-direction bitmap (owner's bits only): bit i = instance i is in a splitting node of this
// level whose winning feature is local, and bin(i, f*) <= b*.
__global__ void k_bitmap(gbdtmo_problem p, int level, const uint8_t* __restrict__ bins, State s,
                         const uint64_t* __restrict__ keys, int64_t* __restrict__ xchg) {
  extern __shared__ int sh_split[];   // [LN][2]: local feature (-1: none), bin
  const int64_t LN = int64_t(1) << level, first = LN - 1;
  for (int64_t i = threadIdx.x; i < LN; i += blockDim.x) {
    int fl = -1, b = 0, fg = 0;
    if (!(s.node_state[first + i] == GBDTMO_NODE_ACTIVE && decode_local(p, keys[i], &fl, &b, &fg))) fl = -1;
    sh_split[2 * i] = fl;
    sh_split[2 * i + 1] = b;
  }
  __syncthreads();
  uint32_t* bm = reinterpret_cast<uint32_t*>(xchg + bitmap_offset(p));
  const int64_t nwords32 = ((p.n + 63) / 64) * 2;
  const int lane = threadIdx.x & 31;
  for (int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; w < nwords32;
       w += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const int64_t i = w * 32 + lane;
    bool bit = false;
    if (i < p.n) {
      const int64_t sl = (int64_t)s.nid[i] - first;
      if (sl >= 0 && sl < LN) {
        const int fl = sh_split[2 * sl];
        if (fl >= 0) bit = bins[i * p.ld_bins + fl] <= sh_split[2 * sl + 1];
      }
    }
    const uint32_t word = __ballot_sync(0xffffffffu, bit);
    if (lane == 0) bm[w] = word;
  }
}

}  // namespace gbdtmo

using namespace gbdtmo;

extern "C" gbdtmo_status gbdtmo_find_split(gbdtmo_ctx c, const gbdtmo_problem* p, int32_t level,
                                           const int32_t* nbins, const float* scales, void* state,
                                           int64_t* hist, int32_t* cnt, const int64_t* parent_hist,
                                           const int32_t* parent_cnt, uint64_t* keys) {
  Ctx* ctx = (Ctx*)c;
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(level >= 0 && level < p->D, "level out of range [0, D)");
  GB_CHECK_ARG(nbins && scales && state && hist && cnt && keys, "null pointer");
  GB_CHECK_ARG(level == 0 || (parent_hist && parent_cnt), "parent histogram required for level > 0");
  State s = state_view(*p, state);
  const int64_t LN = int64_t(1) << level;
  GB_LAUNCH(k_zero_u64, 1, 256, 0, keys, LN);
  dim3 grid((p->m + kFsFeatures - 1) / kFsFeatures, (unsigned)LN);
  const int threads = ((p->B + 31) / 32) * 32;
  auto kern = p->loss == GBDTMO_LOSS_SOFTMAX ? k_find_split<true> : k_find_split<false>;
  GB_LAUNCH(kern, grid, threads, 0, *p, level, nbins, scales, s, hist, cnt,
            level > 0 ? parent_hist : hist, level > 0 ? parent_cnt : cnt, keys, level < p->D - 1 ? 1 : 0);
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_split_record(gbdtmo_ctx c, const gbdtmo_problem* p, int32_t level,
                                             const uint8_t* bins, const float* scales, void* state,
                                             const int64_t* hist, const int32_t* cnt,
                                             const int64_t* parent_hist, const int32_t* parent_cnt,
                                             const uint64_t* keys, int64_t* xchg) {
  Ctx* ctx = (Ctx*)c;
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(level >= 0 && level < p->D, "level out of range [0, D)");
  GB_CHECK_ARG(bins && state && hist && cnt && keys && xchg && scales, "null pointer");
  GB_CHECK_ARG(level == 0 || (parent_hist && parent_cnt), "parent histogram required for level > 0");
  State s = state_view(*p, state);
  const int64_t LN = int64_t(1) << level;
  GB_LAUNCH(k_split_record, (unsigned)LN, 256, 0, *p, level, s, hist, cnt, level > 0 ? parent_hist : hist,
            level > 0 ? parent_cnt : cnt, keys, scales, xchg);
  // zero the record words of the unused slots of this buffer (levels < D-1) so SUM-merging is clean
  const int64_t used = LN * rec_words(*p), cap = bitmap_offset(*p);
  if (cap > used) GB_LAUNCH(k_zero_u64, 64, 256, 0, reinterpret_cast<uint64_t*>(xchg + used), cap - used);
  GB_LAUNCH(k_bitmap, ctx->num_sms * 4, 256, (size_t)(2 * LN * sizeof(int)), *p, level, bins, s, keys, xchg);
  return GBDTMO_OK;
}
