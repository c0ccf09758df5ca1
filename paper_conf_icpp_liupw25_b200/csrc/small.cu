// small.cu — split search for deep, small nodes by sort-and-segment (the paper's "sort-and-
// reduce" approach, redesigned for B200; reading R27).
//
// Deep levels hold many nodes with few rows (C2 at depth 7: ~470 rows per node) against
// histograms of B x V entries per feature (C2: 40 KB per feature, 32 MB per node): building,
// subtracting and re-reading them in HBM costs far more than the rows themselves.  A node marked
// SMALL by the plan (both children of its parent fit GBDTMO_OPT_SMALL_MAX_ROWS) is searched
// directly from its rows instead, and never materialised (k_seg_search below).
#include "common.cuh"

namespace gbdtmo {

// Segmented-scan search (round 2).  It replaces a serial walk (one lane per output stepping through
// the node's rows in bin order: ~470 dependent steps at C2's deepest level, 3 features' buffers per
// warp, one 8-warp CTA per SM: 12.5% occupancy, 38% issue, `profiles/r02_ncu_small_C2.txt`; 3x
// slower per level, `profiles/r02c_ncu_small_seg_C2.txt`).  A warp takes ONE feature at a time and
// its lanes take positions of the node's rows in bin order:
//   - counting sort by bin (shared counters), the sorted row indices stored lane-major
//     (sidxT[i][lane] = row at position lane * PL + i, PL = ceil(R / 32): conflict-free reads);
//   - candidates = positions j < R - 1 ending a bin (sb[j] != sb[j + 1], R27) that are valid
//     (bin <= nb - 2, both sides >= min_node), compacted per warp (cpos, cbin);
//   - per output k: each lane sums q[., k] (and q[., d + k]) over its PL positions, writing the
//     running sum at its candidates; a warp scan of the lane totals turns those into the exact
//     int64 prefix sums G_L (H_L); then lanes take candidates round-robin and add the output's
//     Eq. (3) term in the same fp64 order as k_find_split_h (acc = fma(GL, GL, acc) / eq3_pair),
//     with the parent term P summed the same way, so gains and keys are bit-identical to the
//     histogram path's.
// The CTA stages the node's row ids and q rows once for all the features its warps walk.
#ifndef GBDTMO_BOUNDS_CHECK
#define GBDTMO_BOUNDS_CHECK 0  // (debug builds) trap on any out-of-range shared-memory index below
#endif
#define SEG_CHECK(cond) do { if (GBDTMO_BOUNDS_CHECK && !(cond)) __trap(); } while (0)
constexpr int kSegWarps = 16;
#ifndef GBDTMO_SEG_ILP
#define GBDTMO_SEG_ILP 4
#endif
constexpr int kSegILP = GBDTMO_SEG_ILP;   // row loads in flight per lane in the per-output walk
constexpr int kSegCand = 256;          // candidates per (node, feature) <= distinct bins - 1 <= 255

struct SegLayout {
  int rc, V;
  int o_qs, o_warps, warp_bytes, bytes;
  // per warp: candG[256] i64 (bk[rc] u8 during the sort) | aux[256] (softmax candH i64 / MSE accR f64) |
  //           acc[256] f64 (cnt[256] u32 during the sort) | cpos[256] u16 | cbin[256] u8 | sb[rc + 16] u8 |
  //           sidxT[rc32] u16.  cnt and bk are dead once the rows are scattered in bin order, before
  //           the candidate arrays are written, so they share space with acc and candG.
  int o_cnt, o_candG, o_aux, o_acc, o_cpos, o_cbin, o_bk, o_sb, o_sidx;
};

__host__ __device__ inline SegLayout seg_layout(const gbdtmo_problem& p, int64_t rcap) {
  SegLayout L;
  L.rc = (int)((rcap + 31) / 32 * 32);
  L.V = channels(p);
  L.o_qs = 4 * L.rc;
  L.o_warps = (L.o_qs + 4 * L.V * L.rc + 15) / 16 * 16;
  L.o_candG = 0;
  L.o_bk = L.o_candG;                                // (rc <= 1024 <= 8 kSegCand bytes)
  L.o_aux = L.o_candG + 8 * kSegCand;
  L.o_acc = L.o_aux + 8 * kSegCand;
  L.o_cnt = L.o_acc;                                 // 4 x 256 <= 8 kSegCand bytes
  L.o_cpos = L.o_acc + 8 * kSegCand;
  L.o_cbin = L.o_cpos + 2 * kSegCand;
  L.o_sb = L.o_cbin + kSegCand;
  L.o_sidx = L.o_sb + L.rc + 16;
  L.warp_bytes = (L.o_sidx + 2 * L.rc + 15) / 16 * 16;
  L.bytes = L.o_warps + kSegWarps * L.warp_bytes;
  return L;
}

__host__ __device__ inline int64_t seg_cap(const gbdtmo_problem& p) {
  const int V = channels(p);
  // bytes(rc) = 4 rc (1 + V) + W (6912 + 3 rc + 16) (+ alignment)
  const int64_t fixed = (int64_t)kSegWarps * (3 * 8 * kSegCand + 2 * kSegCand + kSegCand + 16 + 16) + 64;
  int64_t r = (kHistSmemBudget - fixed) / (4 * (1 + V) + 3 * kSegWarps);
  r = r / 32 * 32;
  if (r > 1024) r = 1024;                          // <= 32 positions per lane (one candidate bit each)
  return r < 0 ? 0 : r;
}

template <bool SOFTMAX>
__global__ void __launch_bounds__(kSegWarps * 32)
k_seg_search(gbdtmo_problem p, int level, int rcap, const uint8_t* __restrict__ bins,
             const int32_t* __restrict__ q, const int32_t* __restrict__ rows, int use_rows,
             const int32_t* __restrict__ nbins, const float* __restrict__ scales, State s,
             uint64_t* __restrict__ keys) {
  extern __shared__ __align__(16) unsigned char smraw[];
  __shared__ unsigned long long sh_best[kSegWarps];
  if ((int)blockIdx.y >= s.misc[MISC_SNODE_COUNT]) return;
  const int4 nd = s.snodes[blockIdx.y];
  const int64_t h = (int64_t(1) << level) - 1 + nd.x;
  const int R = nd.z - nd.y;
  const int V = channels(p), B = p.B, m = p.m, d = p.d;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const SegLayout L = seg_layout(p, rcap);
  SEG_CHECK(R >= 0 && R <= rcap && (R + 31) / 32 <= 32);
  int32_t* rid = reinterpret_cast<int32_t*>(smraw);
  int32_t* qs = reinterpret_cast<int32_t*>(smraw + L.o_qs);
  unsigned char* wb = smraw + L.o_warps + warp * L.warp_bytes;
  uint32_t* cnt = reinterpret_cast<uint32_t*>(wb + L.o_cnt);
  long long* candG = reinterpret_cast<long long*>(wb + L.o_candG);
  long long* candH = reinterpret_cast<long long*>(wb + L.o_aux);      // softmax
  double* accR = reinterpret_cast<double*>(wb + L.o_aux);             // MSE
  double* acc = reinterpret_cast<double*>(wb + L.o_acc);
  uint16_t* cpos = reinterpret_cast<uint16_t*>(wb + L.o_cpos);
  unsigned char* cbin = wb + L.o_cbin;
  unsigned char* bk = wb + L.o_bk;
  unsigned char* sb = wb + L.o_sb;
  uint16_t* sidxT = reinterpret_cast<uint16_t*>(wb + L.o_sidx);
  for (int i = threadIdx.x; i < R; i += blockDim.x) rid[i] = use_rows ? rows[nd.y + i] : nd.y + i;
  __syncthreads();
  // q rows of the node: 8 independent loads in flight per thread (the CTA waits on this once)
  for (int e0 = threadIdx.x; e0 < R * V; e0 += 8 * blockDim.x) {
    int v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int e = e0 + u * blockDim.x;
      if (e < R * V) {
        const int i = e / V, c = e - i * V;
        v[u] = __ldg(&q[(int64_t)rid[i] * V + c]);
      }
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int e = e0 + u * blockDim.x;
      if (e < R * V) {
        // softmax: (g_k, h_k) interleaved, one 8-byte load per (row, output) in the walk
        const int i = e / V, c = e - i * V;
        qs[SOFTMAX ? i * V + 2 * (c < d ? c : c - d) + (c < d ? 0 : 1) : e] = v[u];
      }
    }
  }
  __syncthreads();
  const int64_t* S = s.node_sum + h * (V + 1);
  const long long C = S[V];
  const double lam = p.lambda;
  // parent term, summed over outputs in k_find_split_h's order
  double P = 0.0;
  for (int k = 0; k < d; ++k) {
    const double Gd = (double)S[k] * (double)scales[k];
    if (SOFTMAX) {
      const double Hd = (double)S[d + k] * (double)scales[d + k];
      P += Gd * Gd / (Hd + lam);
    } else {
      P = fma(Gd, Gd, P);
    }
  }
  const int PL = (R + 31) >> 5;                    // positions per lane
  uint64_t best = 0;
  for (int f = blockIdx.x * kSegWarps + warp; f < m; f += gridDim.x * kSegWarps) {
    // ---- counting sort of the node's rows by bin
#pragma unroll
    for (int t = 0; t < 8; ++t) cnt[lane * 8 + t] = 0;
    __syncwarp();
    for (int i0 = 0; i0 < R; i0 += 128) {
      int bv[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int i = i0 + u * 32 + lane;
        bv[u] = i < R ? (int)__ldg(&bins[(int64_t)rid[i] * p.ld_bins + f]) : -1;
      }
#pragma unroll
      for (int u = 0; u < 4; ++u)
        if (bv[u] >= 0) {
          SEG_CHECK(i0 + u * 32 + lane < L.rc && bv[u] < 256);
          bk[i0 + u * 32 + lane] = (unsigned char)bv[u];
          atomicAdd(&cnt[bv[u]], 1u);
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
    for (int i = lane; i < R; i += 32) {
      const int b = bk[i];
      const uint32_t pos = atomicAdd(&cnt[b], 1u);
      sb[pos] = (unsigned char)b;
      const uint32_t ow = pos / PL, oi = pos - ow * PL;
      SEG_CHECK(pos < (uint32_t)R && ow < 32 && oi * 32 + ow < (uint32_t)L.rc);
      sidxT[oi * 32 + ow] = (uint16_t)i;
    }
    __syncwarp();
    // ---- candidates of this lane's positions [lane PL, lane PL + PL), compacted per warp
    const int nb = nbins[f];
    const int p0 = lane * PL;
    uint32_t cm = 0;                               // bit i: position p0 + i is a candidate
    for (int i = 0; i < PL; ++i) {
      const int j = p0 + i;
      if (j < R - 1) {
        const int b = sb[j];
        const long long CL = j + 1;
        if (b != (int)sb[j + 1] && b <= nb - 2 && CL >= p.min_node && C - CL >= p.min_node) cm |= 1u << i;
      }
    }
    int cb = __popc(cm), ctot;
    {
      int x = cb;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
      }
      ctot = __shfl_sync(0xffffffffu, x, 31);
      cb = x - cb;                                 // this lane's first candidate index
    }
    if (ctot == 0) continue;                       // (warp-uniform)
    {
      int ci = cb;
      for (uint32_t mm = cm; mm; mm &= mm - 1) {
        const int i = __ffs(mm) - 1;
        SEG_CHECK(ci < kSegCand && p0 + i < R - 1);
        cpos[ci] = (uint16_t)(p0 + i);
        cbin[ci] = sb[p0 + i];
        ++ci;
      }
    }
    for (int c = lane; c < ctot; c += 32) { acc[c] = 0.0; if (!SOFTMAX) accR[c] = 0.0; }
    __syncwarp();
    // ---- per output: exact prefix sums at the candidates, then the Eq. (3) terms
    for (int k = 0; k < d; ++k) {
      long long g = 0, hh = 0;
      int ci = cb;
      const int pe = min(PL, R - p0);              // this lane's positions
      for (int i0 = 0; i0 < pe; i0 += kSegILP) {   // kSegILP independent row loads in flight
        int qg[kSegILP], qh[kSegILP];
#pragma unroll
        for (int u = 0; u < kSegILP; ++u) {
          const int r = i0 + u < pe ? (int)sidxT[(i0 + u) * 32 + lane] : -1;
          SEG_CHECK(r < R);
          if (SOFTMAX) {
            const int2 gh = r >= 0 ? *reinterpret_cast<const int2*>(qs + r * V + 2 * k) : make_int2(0, 0);
            qg[u] = gh.x;
            qh[u] = gh.y;
          } else {
            qg[u] = r >= 0 ? qs[r * V + k] : 0;
            qh[u] = 0;
          }
        }
#pragma unroll
        for (int u = 0; u < kSegILP; ++u) {
          g += qg[u];
          if (SOFTMAX) hh += qh[u];
          if ((cm >> (i0 + u)) & 1u) {
            candG[ci] = g;
            if (SOFTMAX) candH[ci] = hh;
            ++ci;
          }
        }
      }
      // exclusive offsets of the lane totals
      long long og = g, oh = hh;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const long long yg = __shfl_up_sync(0xffffffffu, og, o);
        const long long yh = SOFTMAX ? __shfl_up_sync(0xffffffffu, oh, o) : 0;
        if (lane >= o) { og += yg; if (SOFTMAX) oh += yh; }
      }
      og -= g;
      oh -= hh;
      for (int c = cb; c < ci; ++c) { candG[c] += og; if (SOFTMAX) candH[c] += oh; }
      __syncwarp();
      const long long G = S[k];
      const double sg = (double)scales[k];
      if (SOFTMAX) {
        const long long H = S[d + k];
        const double sh = (double)scales[d + k];
        for (int c = lane; c < ctot; c += 32) {
          const long long gl = candG[c], hl = candH[c];
          const double GL = (double)gl * sg, GR = (double)(G - gl) * sg;
          const double HL = (double)hl * sh, HR = (double)(H - hl) * sh;
          acc[c] += eq3_pair(GL, HL + lam, GR, HR + lam);
        }
      } else {
        for (int c = lane; c < ctot; c += 32) {
          const long long gl = candG[c];
          const double GL = (double)gl * sg, GR = (double)(G - gl) * sg;
          acc[c] = fma(GL, GL, acc[c]);
          accR[c] = fma(GR, GR, accR[c]);
        }
      }
      __syncwarp();
    }
    // ---- gains and keys (k_find_split_h's formulas)
    const int64_t fbg = (int64_t)(p.f_begin + f) * B;
    for (int c = lane; c < ctot; c += 32) {
      const long long CL = (long long)cpos[c] + 1;
      double gain;
      if (SOFTMAX)
        gain = 0.5 * (acc[c] - P);
      else
        gain = 0.5 * (acc[c] / (2.0 * (double)CL + lam) + accR[c] / (2.0 * (double)(C - CL) + lam) -
                      P / (2.0 * (double)C + lam));
      if (gain > p.gamma) {
        const uint64_t key = pack_split_key(gain, fbg + cbin[c]);
        best = key > best ? key : best;
      }
    }
    __syncwarp();
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const unsigned long long y = __shfl_xor_sync(0xffffffffu, (unsigned long long)best, o);
    best = y > best ? y : best;
  }
  if (lane == 0) sh_best[warp] = best;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint64_t bb = 0;
    for (int w = 0; w < kSegWarps; ++w) bb = sh_best[w] > bb ? sh_best[w] : bb;
    if (bb) atomicMax((unsigned long long*)&keys[nd.x], (unsigned long long)bb);
  }
}

// (k_split_record's row pass for SMALL nodes covers at most 64 channels: d <= 32 softmax / 64 MSE)
bool small_supported(const gbdtmo_problem& p) { return p.B <= 256 && channels(p) <= 64 && seg_cap(p) >= 64; }
int64_t small_rows_cap(const gbdtmo_problem& p) { return seg_cap(p); }

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
  State s = state_view(*p, state);
  const int32_t* rows = (level & 1) ? s.rows1 : s.rows0;
  const int use_rows = level > 0;
  const int64_t LN = int64_t(1) << level;
  const bool sm = p->loss == GBDTMO_LOSS_SOFTMAX;
  const SegLayout L = seg_layout(*p, rcap);
  // feature blocks per node: GBDTMO_SEG_WAVES waves of resident CTAs over the level's (at most LN) small nodes,
  // so nodes of different sizes balance (ncu at 2.6 waves: 46% issue, idle SMs in the tail)
  const int per_sm = (int)((ctx->max_smem_optin) / (L.bytes + 1024));
#ifndef GBDTMO_SEG_WAVES
#define GBDTMO_SEG_WAVES 32   // waves of (node, feature block) CTAs: C2 4.28 / 4.23 / 4.20 / 4.20 ms per tree at 8 / 16 / 32 / 64
#endif
  int64_t fb = ((int64_t)GBDTMO_SEG_WAVES * ctx->num_sms * (per_sm < 1 ? 1 : per_sm) + LN - 1) / LN;
  const int64_t fb_max = (p->m + kSegWarps - 1) / kSegWarps;
  if (fb > fb_max) fb = fb_max;
  if (fb < 1) fb = 1;
  auto kern = sm ? k_seg_search<true> : k_seg_search<false>;
  static unsigned long long seg_mask[2] = {};
  smem_optin_once(ctx, kern, seg_mask[sm], ctx->max_smem_optin - 1024);
  GB_LAUNCH(kern, dim3((unsigned)fb, (unsigned)LN), kSegWarps * 32, L.bytes, *p, level, (int)rcap, bins, q, rows,
            use_rows, nbins, scales, s, keys);
  return GBDTMO_OK;
}
