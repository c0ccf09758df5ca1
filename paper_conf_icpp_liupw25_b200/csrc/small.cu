// small.cu — split search for deep, small nodes by sort-and-segment (the paper's "sort-and-
// reduce" approach, redesigned for B200; reading R27).
//
// Deep levels hold many nodes with few rows (C2 at depth 7: ~470 rows per node) against
// histograms of B x V entries per feature (C2: 40 KB per feature, 32 MB per node): building,
// subtracting and re-reading them in HBM costs far more than the rows themselves.  A node marked
// SMALL by the plan (both children of its parent fit GBDTMO_OPT_SMALL_MAX_ROWS) is searched
// directly from its rows instead, and never materialised:
//   - one CTA per (node, block of features) stages the node's row ids and q rows in shared memory;
//   - one warp per feature counting-sorts the node's rows by bin (shared counters, in-place
//     exclusive scan), then walks them in bin order with lanes = outputs, accumulating the exact
//     int64 G_L (and H_L) prefix sums from the staged q rows;
//   - at every bin boundary, i.e. only for bins present in the node (an empty bin gives the same
//     partition as its predecessor), each output lane writes its Eq. (3) term to a
//     kCand-candidate buffer; a full buffer is reduced with lanes = candidates (no shuffles on the
//     walk), and the best packed key per CTA is max-reduced into keys[slot] — the same key and
//     tie rule as k_find_split, so the chosen split is the same.
#include "common.cuh"

namespace gbdtmo {

constexpr int kSortWarps = 16;
constexpr int kCand = 16;            // candidates buffered per warp before a reduction

struct SmallLayout {
  int dp;                          // doubles per buffered candidate (d rounded up to odd: conflict-free reads)
  int o_qs, o_warps;               // CTA-shared: row ids [rc] i32 at 0, q rows [rc][V] i32 at o_qs
  int o_sidx, o_bk, o_sb, o_cand, o_cbin, warp_bytes;   // per-warp region offsets
  int bytes;                       // dynamic shared memory of one CTA
};

// rcap = largest node the CTA stages (rounded up to 8).  CTA: row ids, the node's q rows.  Per
// warp: counts[256] u32 | sorted local row index [rc] u16 | bins in row order [rc] u8 | bins in
// sorted order [rc + 8] u8 | cand [kCand][dp] f64 | cbin [kCand] i32.
__host__ __device__ inline SmallLayout small_layout(const gbdtmo_problem& p, int64_t rcap) {
  SmallLayout L;
  const int rc = (int)((rcap + 7) / 8 * 8);
  L.dp = p.d | 1;
  L.o_qs = 4 * rc;
  L.o_warps = L.o_qs + 4 * channels(p) * rc;
  L.o_sidx = 1024;
  L.o_bk = L.o_sidx + 2 * rc;
  L.o_sb = L.o_bk + rc;
  L.o_cand = L.o_sb + rc + 8;
  L.o_cbin = L.o_cand + 8 * kCand * L.dp;
  L.warp_bytes = L.o_cbin + 4 * kCand;
  L.bytes = L.o_warps + kSortWarps * L.warp_bytes;
  return L;
}

__host__ __device__ inline int64_t small_cap(const gbdtmo_problem& p) {
  const SmallLayout L0 = small_layout(p, 0);
  int64_t r = (kHistSmemBudget - L0.bytes) / (4 + 4 * channels(p) + kSortWarps * 4) - 8;
  if (r > 65535) r = 65535;                                    // 16-bit local row indices
  return r < 0 ? 0 : r;
}

__device__ __forceinline__ double warp_sum_d(double x) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
  return x;
}

template <bool SOFTMAX>
__global__ void __launch_bounds__(kSortWarps * 32)
k_sort_search(gbdtmo_problem p, int level, int rcap, const uint8_t* __restrict__ bins,
              const int32_t* __restrict__ q, const int32_t* __restrict__ rows, int use_rows,
              const int32_t* __restrict__ nbins, const float* __restrict__ scales, State s,
              uint64_t* __restrict__ keys) {
  extern __shared__ __align__(16) unsigned char smraw[];
  __shared__ unsigned long long sh_best[kSortWarps];
  if ((int)blockIdx.y >= s.misc[MISC_SNODE_COUNT]) return;
  const int4 nd = s.snodes[blockIdx.y];
  const int64_t h = (int64_t(1) << level) - 1 + nd.x;
  const int r = nd.z - nd.y;
  const int V = channels(p), B = p.B, m = p.m, d = p.d;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const SmallLayout L = small_layout(p, rcap);
  int32_t* rid = reinterpret_cast<int32_t*>(smraw);
  int32_t* qs = reinterpret_cast<int32_t*>(smraw + L.o_qs);
  unsigned char* wb = smraw + L.o_warps + warp * L.warp_bytes;
  uint32_t* cnt = reinterpret_cast<uint32_t*>(wb);
  uint16_t* sidx = reinterpret_cast<uint16_t*>(wb + L.o_sidx);
  unsigned char* bk = wb + L.o_bk;
  unsigned char* sb = wb + L.o_sb;
  double* cand = reinterpret_cast<double*>(wb + L.o_cand);
  int32_t* cbin = reinterpret_cast<int32_t*>(wb + L.o_cbin);
  // stage the node's row ids and q rows (shared by every feature of this CTA)
  for (int i = threadIdx.x; i < r; i += blockDim.x) rid[i] = use_rows ? rows[nd.y + i] : nd.y + i;
  __syncthreads();
  for (int e = threadIdx.x; e < r * V; e += blockDim.x) {
    const int i = e / V, c = e - i * V;
    qs[e] = __ldg(&q[(int64_t)rid[i] * V + c]);
  }
  __syncthreads();
  // node totals (exact) and the parent term of Eq. (3)
  const int64_t* S = s.node_sum + h * (V + 1);
  const long long C = S[V];
  const double lam = p.lambda;
  const bool kon = lane < d;
  const double sg = kon ? (double)scales[lane] : 0.0;
  const double sh = (SOFTMAX && kon) ? (double)scales[d + lane] : 0.0;
  const long long Gt = kon ? S[lane] : 0, Ht = (SOFTMAX && kon) ? S[d + lane] : 0;
  const double Gd = (double)Gt * sg;
  const double P = SOFTMAX ? warp_sum_d(kon ? Gd * Gd / ((double)Ht * sh + lam) : 0.0)
                           : warp_sum_d(Gd * Gd) / (2.0 * (double)C + lam);
  const int32_t* qg = qs + (kon ? lane : 0);
  const int32_t* qh = qs + (kon ? d + lane : 0);
  uint64_t best = 0;
  int64_t fb0 = 0;
  // reduce the buffered candidates: lanes = candidates, sum of the per-output terms
  auto flush = [&](int nc) {
    __syncwarp();
    if (lane < nc) {
      double t = 0.0;
      for (int k = 0; k < d; ++k) t += cand[lane * L.dp + k];
      const double gain = 0.5 * (t - P);
      if (gain > p.gamma) {
        const uint64_t key = pack_split_key(gain, fb0 + cbin[lane]);
        best = key > best ? key : best;
      }
    }
    __syncwarp();
  };
  for (int f = blockIdx.x * kSortWarps + warp; f < m; f += gridDim.x * kSortWarps) {
    // ---- counting sort of the node's rows by bin
#pragma unroll
    for (int t = 0; t < 8; ++t) cnt[lane * 8 + t] = 0;
    __syncwarp();
    for (int i0 = 0; i0 < r; i0 += 128) {
      int bv[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int i = i0 + u * 32 + lane;
        bv[u] = i < r ? (int)bins[(int64_t)rid[i] * p.ld_bins + f] : -1;
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        if (bv[u] >= 0) {
          bk[i0 + u * 32 + lane] = (unsigned char)bv[u];
          atomicAdd(&cnt[bv[u]], 1u);
        }
      }
    }
    __syncwarp();
    {
      uint32_t v[8], run = 0;
#pragma unroll
      for (int t = 0; t < 8; ++t) { v[t] = run; run += cnt[lane * 8 + t]; }
      uint32_t x = run;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
      }
      const uint32_t ex = x - run;
      __syncwarp();
#pragma unroll
      for (int t = 0; t < 8; ++t) cnt[lane * 8 + t] = ex + v[t];
    }
    __syncwarp();
    for (int i = lane; i < r; i += 32) {
      const int b = bk[i];
      const uint32_t pos = atomicAdd(&cnt[b], 1u);
      sidx[pos] = (uint16_t)i;
      sb[pos] = (unsigned char)b;
    }
    __syncwarp();
    // ---- walk in bin order: after row j, "bin <= sb[j]" is a candidate when sb[j+1] differs
    const int nb = nbins[f];
    fb0 = (int64_t)(p.f_begin + f) * B;
    long long GL = 0, HL = 0;
    int nc = 0;
    for (int j0 = 0; j0 < r - 1; j0 += 4) {
      int ix[4];
      int gv[4], hv[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) ix[u] = (j0 + u < r - 1) ? (int)sidx[j0 + u] : -1;
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        gv[u] = (ix[u] >= 0 && kon) ? qg[ix[u] * V] : 0;
        hv[u] = (SOFTMAX && ix[u] >= 0 && kon) ? qh[ix[u] * V] : 0;
      }
      const uint32_t b4 = *reinterpret_cast<const uint32_t*>(sb + j0);     // sb is 8-aligned, j0 % 4 == 0
      const uint32_t n4 = (uint32_t)sb[j0 + 4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        GL += gv[u];
        if (SOFTMAX) HL += hv[u];
        const int b = (b4 >> (8 * u)) & 0xff;
        const int bn = u < 3 ? (int)((b4 >> (8 * (u + 1))) & 0xff) : (int)n4;
        const long long CL = j0 + u + 1;
        if (ix[u] >= 0 && b != bn && b <= nb - 2 && CL >= p.min_node && C - CL >= p.min_node) {
          const double gl = (double)GL * sg, gr = (double)(Gt - GL) * sg;
          double t;
          if (SOFTMAX) {
            t = gl * gl / ((double)HL * sh + lam) + gr * gr / ((double)(Ht - HL) * sh + lam);
          } else {
            t = gl * gl / (2.0 * (double)CL + lam) + gr * gr / (2.0 * (double)(C - CL) + lam);
          }
          if (kon) cand[nc * L.dp + lane] = t;
          if (lane == 0) cbin[nc] = b;
          if (++nc == kCand) {
            flush(nc);
            nc = 0;
          }
        }
      }
    }
    if (nc) flush(nc);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {                     // lanes hold their candidates' bests
    const unsigned long long y = __shfl_xor_sync(0xffffffffu, (unsigned long long)best, o);
    best = y > best ? y : best;
  }
  if (lane == 0) sh_best[warp] = best;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint64_t bb = 0;
    for (int w = 0; w < kSortWarps; ++w) bb = sh_best[w] > bb ? sh_best[w] : bb;
    if (bb) atomicMax((unsigned long long*)&keys[nd.x], (unsigned long long)bb);
  }
}

bool small_supported(const gbdtmo_problem& p) { return p.d <= 32 && small_cap(p) >= 64; }
int64_t small_rows_cap(const gbdtmo_problem& p) { return small_cap(p); }

}  // namespace gbdtmo

using namespace gbdtmo;

extern "C" gbdtmo_status gbdtmo_search_small(gbdtmo_ctx c, const gbdtmo_problem* p, int32_t level,
                                             const uint8_t* bins, const int32_t* q, const int32_t* nbins,
                                             const float* scales, void* state, uint64_t* keys) {
  Ctx* ctx = (Ctx*)c;
  DeviceGuard device_guard_(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(level >= 0 && level < p->D, "level out of range [0, D)");
  GB_CHECK_ARG(bins && q && nbins && scales && state && keys, "null pointer");
  const int64_t rcap = small_rows(ctx, *p);
  if (rcap <= 0) return GBDTMO_OK;                          // no node is ever marked SMALL
  const SmallLayout L = small_layout(*p, rcap);
  State s = state_view(*p, state);
  const int32_t* rows = (level & 1) ? s.rows1 : s.rows0;
  const int use_rows = level > 0;
  const int64_t LN = int64_t(1) << level;
  // feature blocks per node: enough CTAs for ~3 waves of resident CTAs, at most one warp per feature
  const int fb_max = (p->m + kSortWarps - 1) / kSortWarps;
  const int per_sm = L.bytes > 0 ? (int)((ctx->max_smem_optin - 1024) / (L.bytes + 1024)) : 1;
  int64_t fb = (3LL * ctx->num_sms * (per_sm < 1 ? 1 : per_sm) + LN - 1) / LN;
  if (fb > fb_max) fb = fb_max;
  if (fb < 1) fb = 1;
  auto kern = p->loss == GBDTMO_LOSS_SOFTMAX ? k_sort_search<true> : k_sort_search<false>;
  static unsigned long long attr_mask[2] = {0, 0};
  smem_optin_once(ctx, kern, attr_mask[p->loss == GBDTMO_LOSS_SOFTMAX], ctx->max_smem_optin - 1024);
  GB_LAUNCH(kern, dim3((unsigned)fb, (unsigned)LN), kSortWarps * 32, L.bytes, *p, level, (int)rcap, bins, q, rows,
            use_rows, nbins, scales, s, keys);
  return GBDTMO_OK;
}
