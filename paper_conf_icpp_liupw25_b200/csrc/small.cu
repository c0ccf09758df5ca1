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

// A warp searches G features at once (G = 32 / d rounded down to 1, 2, 3, 4 or 8): lanes are
// (feature group g, output k), so a d = 10 softmax node keeps 30 of 32 lanes busy instead of 10.
constexpr int kSortWarpsMax = 16;

__host__ __device__ inline int small_groups(int d) { return d <= 4 ? 8 : d <= 8 ? 4 : d <= 10 ? 3 : d <= 16 ? 2 : 1; }
__host__ __device__ inline int small_warps(int G) { return G > 1 ? 8 : 16; }
__host__ __device__ inline int small_cpg(int G) { return G > 1 ? 32 / G : 16; }   // buffered candidates per group

struct SmallLayout {
  int G, W, CPG;                   // features per warp, warps per CTA, candidates per group
  int dp;                          // doubles per buffered candidate (d rounded up to odd: conflict-free reads)
  int o_qs, o_warps;               // CTA-shared: row ids [rc] i32 at 0, q rows [rc][V] i32 at o_qs
  int g_bytes;                     // per (warp, group): counts[256] u32 | sidx [rc] u16 | bk [rc] u8 | sb [rc + 8] u8
  int o_sidx, o_bk, o_sb;          // offsets inside a group's region
  int o_cand, o_cbin, warp_bytes;  // per warp: G regions, then cand [G][CPG][dp] f64, cbin [G][CPG] i32
  int bytes;                       // dynamic shared memory of one CTA
};

__host__ __device__ inline SmallLayout small_layout(const gbdtmo_problem& p, int64_t rcap) {
  SmallLayout L;
  const int rc = (int)((rcap + 7) / 8 * 8);
  L.G = small_groups(p.d);
  L.W = small_warps(L.G);
  L.CPG = small_cpg(L.G);
  L.dp = p.d | 1;
  L.o_qs = 4 * rc;
  L.o_warps = L.o_qs + 4 * channels(p) * rc;
  L.o_sidx = 1024;
  L.o_bk = L.o_sidx + 2 * rc;
  L.o_sb = L.o_bk + rc;
  L.g_bytes = (L.o_sb + rc + 8 + 7) / 8 * 8;
  L.o_cand = L.G * L.g_bytes;
  L.o_cbin = L.o_cand + 8 * L.G * L.CPG * L.dp;
  L.warp_bytes = L.o_cbin + 4 * L.G * L.CPG;
  L.bytes = L.o_warps + L.W * L.warp_bytes;
  return L;
}

__host__ __device__ inline int64_t small_cap(const gbdtmo_problem& p) {
  const SmallLayout L0 = small_layout(p, 0);
  int64_t r = (kHistSmemBudget - L0.bytes) / (4 + 4 * channels(p) + L0.W * L0.G * 4) - 8;
  if (r > 65535) r = 65535;                                    // 16-bit local row indices
  return r < 0 ? 0 : r;
}

__device__ __forceinline__ double warp_sum_d(double x) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
  return x;
}

template <bool SOFTMAX, int G>
__global__ void __launch_bounds__(G > 1 ? 256 : 512)
k_sort_search(gbdtmo_problem p, int level, int rcap, const uint8_t* __restrict__ bins,
              const int32_t* __restrict__ q, const int32_t* __restrict__ rows, int use_rows,
              const int32_t* __restrict__ nbins, const float* __restrict__ scales, State s,
              uint64_t* __restrict__ keys) {
  extern __shared__ __align__(16) unsigned char smraw[];
  __shared__ unsigned long long sh_best[kSortWarpsMax];
  if ((int)blockIdx.y >= s.misc[MISC_SNODE_COUNT]) return;
  const int4 nd = s.snodes[blockIdx.y];
  const int64_t h = (int64_t(1) << level) - 1 + nd.x;
  const int r = nd.z - nd.y;
  const int V = channels(p), B = p.B, m = p.m, d = p.d;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const SmallLayout L = small_layout(p, rcap);
  constexpr int CPG = G > 1 ? 32 / G : 16;
  const int W = L.W;
  int32_t* rid = reinterpret_cast<int32_t*>(smraw);
  int32_t* qs = reinterpret_cast<int32_t*>(smraw + L.o_qs);
  unsigned char* wb = smraw + L.o_warps + warp * L.warp_bytes;
  double* cand = reinterpret_cast<double*>(wb + L.o_cand);          // [G][CPG][dp]
  int32_t* cbin = reinterpret_cast<int32_t*>(wb + L.o_cbin);        // [G][CPG]
  // stage the node's row ids and q rows (shared by every feature of this CTA)
  for (int i = threadIdx.x; i < r; i += blockDim.x) rid[i] = use_rows ? rows[nd.y + i] : nd.y + i;
  __syncthreads();
  for (int e = threadIdx.x; e < r * V; e += blockDim.x) {
    const int i = e / V, c = e - i * V;
    qs[e] = __ldg(&q[(int64_t)rid[i] * V + c]);
  }
  __syncthreads();
  // lanes: (group g, output k)
  const int g = G > 1 ? lane / d : 0, k = G > 1 ? lane - g * d : lane;
  const bool lon = g < G && k < d;
  // node totals (exact) and the parent term of Eq. (3): the same for every feature
  const int64_t* S = s.node_sum + h * (V + 1);
  const long long C = S[V];
  const double lam = p.lambda;
  const bool k0 = lane < d;                               // lanes 0..d-1 compute the parent term once
  const double sg = lon ? (double)scales[k] : 0.0;
  const double sh = (SOFTMAX && lon) ? (double)scales[d + k] : 0.0;
  const long long Gt = lon ? S[k] : 0, Ht = (SOFTMAX && lon) ? S[d + k] : 0;
  double P;
  {
    const double sg0 = k0 ? (double)scales[lane] : 0.0, sh0 = (SOFTMAX && k0) ? (double)scales[d + lane] : 0.0;
    const double Gd0 = k0 ? (double)S[lane] * sg0 : 0.0;
    const double Hd0 = (SOFTMAX && k0) ? (double)S[d + lane] * sh0 : 0.0;
    P = SOFTMAX ? warp_sum_d(k0 ? Gd0 * Gd0 / (Hd0 + lam) : 0.0) : warp_sum_d(Gd0 * Gd0) / (2.0 * (double)C + lam);
  }
  const int32_t* qg = qs + (lon ? k : 0);
  const int32_t* qh = qs + (lon ? d + k : 0);
  uint64_t best = 0;
  for (int f0 = (blockIdx.x * W + warp) * G; f0 < m; f0 += gridDim.x * W * G) {
    // ---- counting sort of the node's rows by bin, one feature per group
#pragma unroll 1
    for (int gg = 0; gg < G; ++gg) {
      const int f = f0 + gg;
      if (f >= m) break;
      unsigned char* gr = wb + gg * L.g_bytes;
      uint32_t* cnt = reinterpret_cast<uint32_t*>(gr);
      uint16_t* sidx = reinterpret_cast<uint16_t*>(gr + L.o_sidx);
      unsigned char* bk = gr + L.o_bk;
      unsigned char* sb = gr + L.o_sb;
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
    }
    // ---- walk in bin order, all groups together: after row j of group g's order, "bin <= sb[j]"
    //      is a candidate when sb[j + 1] differs (only bins present in the node, R27)
    const int fg = f0 + g;
    const bool gon = lon && fg < m;
    const unsigned char* gr = wb + (gon ? g : 0) * L.g_bytes;
    const uint16_t* sidx = reinterpret_cast<const uint16_t*>(gr + L.o_sidx);
    const unsigned char* sb = gr + L.o_sb;
    const int nb = gon ? nbins[fg] : 0;
    long long GL = 0, HL = 0;
    int nc = 0;                                           // candidates buffered for this lane's group
    auto flush = [&]() {
      __syncwarp();
      // lanes = (group, candidate): lane L2 = gg * CPG + c
      const int gg = lane / CPG, c = lane - gg * CPG;
      const int ncg = __shfl_sync(0xffffffffu, nc, gg < G ? gg * d : 0);
      if (gg < G && c < ncg) {
        double t = 0.0;
        const double* cd = cand + ((int64_t)gg * CPG + c) * L.dp;
        for (int kk = 0; kk < d; ++kk) t += cd[kk];
        const double gain = 0.5 * (t - P);
        if (gain > p.gamma) {
          const int64_t fbg = (int64_t)(p.f_begin + f0 + gg) * B;
          const uint64_t key = pack_split_key(gain, fbg + cbin[gg * CPG + c]);
          best = key > best ? key : best;
        }
      }
      __syncwarp();
      nc = 0;
    };
    for (int j0 = 0; j0 < r - 1; j0 += 4) {
      int ix[4];
      int gv[4], hv[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) ix[u] = (gon && j0 + u < r - 1) ? (int)sidx[j0 + u] : -1;
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        gv[u] = ix[u] >= 0 ? qg[ix[u] * V] : 0;
        hv[u] = (SOFTMAX && ix[u] >= 0) ? qh[ix[u] * V] : 0;
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
          const double gl = (double)GL * sg, gr_ = (double)(Gt - GL) * sg;
          double t;
          if (SOFTMAX) {
            t = eq3_pair(gl, (double)HL * sh + lam, gr_, (double)(Ht - HL) * sh + lam);
          } else {
            t = gl * gl / (2.0 * (double)CL + lam) + gr_ * gr_ / (2.0 * (double)(C - CL) + lam);
          }
          cand[((int64_t)g * CPG + nc) * L.dp + k] = t;
          if (k == 0) cbin[g * CPG + nc] = b;
          ++nc;
        }
        // a group whose buffer is full makes the whole warp reduce (lanes = (group, candidate))
        if (__any_sync(0xffffffffu, nc == CPG)) flush();
      }
    }
    if (__any_sync(0xffffffffu, nc > 0)) flush();
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
    for (int w = 0; w < W; ++w) bb = sh_best[w] > bb ? sh_best[w] : bb;
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
  GB_ENTRY(ctx);
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
  // feature blocks per node: enough CTAs for ~3 waves of resident CTAs, at most one warp per G features
  const int fb_max = (p->m + L.W * L.G - 1) / (L.W * L.G);
  const int per_sm = L.bytes > 0 ? (int)((ctx->max_smem_optin - 1024) / (L.bytes + 1024)) : 1;
  int64_t fb = (3LL * ctx->num_sms * (per_sm < 1 ? 1 : per_sm) + LN - 1) / LN;
  if (fb > fb_max) fb = fb_max;
  if (fb < 1) fb = 1;
  const bool sm = p->loss == GBDTMO_LOSS_SOFTMAX;
  decltype(&k_sort_search<true, 1>) kern;
  switch (L.G) {
    case 8: kern = sm ? k_sort_search<true, 8> : k_sort_search<false, 8>; break;
    case 4: kern = sm ? k_sort_search<true, 4> : k_sort_search<false, 4>; break;
    case 3: kern = sm ? k_sort_search<true, 3> : k_sort_search<false, 3>; break;
    case 2: kern = sm ? k_sort_search<true, 2> : k_sort_search<false, 2>; break;
    default: kern = sm ? k_sort_search<true, 1> : k_sort_search<false, 1>; break;
  }
  static unsigned long long attr_mask[2][9] = {};
  smem_optin_once(ctx, kern, attr_mask[sm][L.G], ctx->max_smem_optin - 1024);
  GB_LAUNCH(kern, dim3((unsigned)fb, (unsigned)LN), L.W * 32, L.bytes, *p, level, (int)rcap, bins, q, rows,
            use_rows, nbins, scales, s, keys);
  return GBDTMO_OK;
}
