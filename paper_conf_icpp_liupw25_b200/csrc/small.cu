// small.cu — fused histogram build + split search for small nodes (reading R27).
//
// Deep levels hold many nodes with few rows (C2 at depth 7: ~470 rows per node against a
// 32 MB histogram per node), where materialising, subtracting and re-reading histograms in HBM
// costs far more than the updates themselves.  A node marked SMALL by the plan (both children of
// its parent fit the threshold GBDTMO_OPT_SMALL_MAX_ROWS) is instead built from its own rows in
// shared memory (same two-limb fixed-point accumulation as k_hist_smem, all channels of a
// feature tile in one work item) and searched in place (Eq. 3): the histogram
// never reaches HBM and no sibling is derived.  Each work item max-reduces its best packed key
// into keys[slot] exactly like k_find_split, so the result is identical.
#include "common.cuh"
#include "hist_common.cuh"

namespace gbdtmo {

constexpr int kSmallSeg = 32;                     // bins per scan segment (one per lane)

struct SmallCfg {
  int K, n_ct, kf, n_ft, smem;
  bool ok;
};

__host__ __device__ inline SmallCfg small_config(const gbdtmo_problem& p) {
  SmallCfg c;
  const int V = channels(p);
  c.K = V <= 4 ? 4 : V <= 8 ? 8 : 16;
  c.n_ct = (V + c.K - 1) / c.K;
  const int nseg = (p.B + kSmallSeg - 1) / kSmallSeg;
  const int per_feature = c.n_ct * p.B * 2 * c.K * 4 + p.B * 4 + nseg * (V + 1) * 8;
  const int allowed[9] = {24, 16, 12, 8, 6, 4, 3, 2, 1};
  c.kf = 0;
  for (int i = 0; i < 9; ++i) {
    const int k = allowed[i];
    const int need = k * per_feature + kHistWarps * 32 * 8 * ((k + 7) / 8) + 64;
    if (k <= p.m && need <= kHistSmemBudget) { c.kf = k; break; }
  }
  c.ok = c.kf > 0 && p.d <= 32;
  if (!c.ok) c.kf = 1;
  c.n_ft = (p.m + c.kf - 1) / c.kf;
  c.smem = c.kf * per_feature + kHistWarps * 32 * 8 * ((c.kf + 7) / 8) + 64;
  return c;
}

__device__ __forceinline__ double warp_sum_d(double x) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
  return x;
}

template <int K, int KF, bool SOFTMAX>
__global__ void __launch_bounds__(kHistThreads, 1)
k_search_small(gbdtmo_problem p, int level, SmallCfg sc, const uint8_t* __restrict__ bins,
               const int32_t* __restrict__ q, const int32_t* __restrict__ rows, int use_rows,
               const int32_t* __restrict__ nbins, const float* __restrict__ scales, State s,
               uint64_t* __restrict__ keys) {
  extern __shared__ __align__(16) uint32_t sm[];
  __shared__ int sh_item;
  __shared__ unsigned long long sh_best[kHistWarps];
  constexpr int RPI = 32 / K, G = K, SB = G < 8 ? G : 8;
  constexpr int RS = KF * 2 * K;                         // limb words per bin per channel tile
  constexpr int NW = HistRow<KF>::NW, SW = HistRow<KF>::SW;
  const int V = channels(p), B = p.B, m = p.m, d = p.d;
  const int nseg = (B + kSmallSeg - 1) / kSmallSeg;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
  const int ri = lane / K, c = lane % K;
  const int n_ct = sc.n_ct;
  const int region = B * RS;                             // words per channel tile
  const int limb_words = n_ct * region;
  uint32_t* cnts = sm + limb_words;                      // [KF][B]
  long long* segtot = reinterpret_cast<long long*>(sm + ((limb_words + KF * B + 1) & ~1));   // [KF][nseg][V+1]
  uint64_t* scratch = reinterpret_cast<uint64_t*>(segtot + KF * nseg * (V + 1)) + (size_t)warp * 32 * SW;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(sm);
  const int slotA = c + ((ri & 1) ? K : 0), slotB = slotA ^ K;
  const int64_t ld = p.ld_bins;
  const int nsmall = s.misc[MISC_SNODE_COUNT];
  const int nitems = nsmall * sc.n_ft;
  const double lam = p.lambda;

  for (;;) {
    if (threadIdx.x == 0) sh_item = atomicAdd(&s.misc[MISC_SWORK_COUNTER], 1);
    __syncthreads();
    const int item = sh_item;
    if (item >= nitems) break;
    const int sn = item / sc.n_ft, ft = item - sn * sc.n_ft;
    const int4 nd = s.snodes[sn];
    const int f0 = ft * KF;
    const int kk = min(KF, m - f0);
    const int words = limb_words + KF * B;
    for (int i = threadIdx.x * 4; i < limb_words; i += blockDim.x * 4)
      *reinterpret_cast<uint4*>(&sm[i]) = make_uint4(0, 0, 0, 0);
    for (int i = limb_words + threadIdx.x; i < words; i += blockDim.x) sm[i] = 0;
    __syncthreads();

    // ---------------- accumulate the node's rows (all channel tiles of the feature tile)
    const int beg = nd.y, end = nd.z;
    const int o = f0 & 7;
    const uint8_t* bbase = bins + (f0 & ~7);
    for (int b0 = beg + warp * 32; b0 < end; b0 += nwarps * 32) {
      const int pos = b0 + lane;
      const int r = pos < end ? (use_rows ? __ldg(&rows[pos]) : pos) : -1;
      uint64_t sw[SW];
#pragma unroll
      for (int i = 0; i < SW; ++i) sw[i] = 0;
      if (r >= 0) {
        uint64_t w[NW];
        const uint64_t* wp = reinterpret_cast<const uint64_t*>(bbase + (int64_t)r * ld);
#pragma unroll
        for (int i = 0; i < NW; ++i) w[i] = __ldg(wp + i);
        shift_window<NW, SW>(w, o, sw);
#pragma unroll
        for (int j = 0; j < KF; ++j)
          if (j < kk) red_shared_add(sbase + 4u * (limb_words + j * B + byte_of<SW>(sw, j)), 1u);
      }
#pragma unroll
      for (int i = 0; i < SW; ++i) scratch[lane * SW + i] = sw[i];
      __syncwarp();
      for (int ct = 0; ct < n_ct; ++ct) {
        const int c0 = ct * K;
        const bool chan_on = (c0 + c) < V;
        const uint32_t aA = sbase + 4u * (ct * region + slotA), aB = sbase + 4u * (ct * region + slotB);
#pragma unroll
        for (int t0 = 0; t0 < G; t0 += SB) {
          int qv[SB];
#pragma unroll
          for (int t = 0; t < SB; ++t) {
            const int rr = __shfl_sync(0xffffffffu, r, (t0 + t) * RPI + ri);
            qv[t] = (rr >= 0 && chan_on) ? __ldg(&q[(int64_t)rr * V + c0 + c]) : 0;
          }
#pragma unroll
          for (int t = 0; t < SB; ++t) {
            const int i = (t0 + t) * RPI + ri;
            if (b0 + i < end) {
              uint64_t bw[SW];
#pragma unroll
              for (int u = 0; u < SW; ++u) bw[u] = scratch[i * SW + u];
              const uint32_t lo = (uint32_t)qv[t] & 0xFFFFu, hi = (uint32_t)(qv[t] >> 16);
              const uint32_t va = (ri & 1) ? hi : lo, vb = (ri & 1) ? lo : hi;
#pragma unroll
              for (int j = 0; j < KF; ++j) {
                if (j < kk) {
                  const uint32_t bin = byte_of<SW>(bw, j);
                  red_shared_add(aA + bin * (4u * RS) + 8u * K * j, va);
                  red_shared_add(aB + bin * (4u * RS) + 8u * K * j, vb);
                }
              }
            }
          }
        }
      }
      __syncwarp();
    }
    __syncthreads();

    // ---------------- search in place.  value(ch, j, b) = lo + hi * 2^16 (lo in half 0, hi in half 1)
    auto val = [&](int ch, int j, int b) -> long long {
      const int ct = ch / K, cc = ch - ct * K;
      const uint32_t* r0 = sm + ct * region + b * RS + j * 2 * K;
      return (long long)(int32_t)r0[K + cc] * 65536LL + (long long)r0[cc];
    };
    // pass 1: per (feature, segment) totals of every channel and of the counts
    for (int pr = warp; pr < kk * nseg; pr += nwarps) {
      const int j = pr / nseg, seg = pr - j * nseg;
      long long tg = 0, th = 0, tc = 0;
      for (int bi = 0; bi < kSmallSeg; ++bi) {
        const int b = seg * kSmallSeg + bi;
        if (b >= B) break;
        if (lane < d) {
          tg += val(lane, j, b);
          if (SOFTMAX) th += val(d + lane, j, b);
        }
        tc += cnts[j * B + b];
      }
      long long* st = segtot + ((size_t)j * nseg + seg) * (V + 1);
      if (lane < d) {
        st[lane] = tg;
        if (SOFTMAX) st[d + lane] = th;
      }
      if (lane == 0) st[V] = tc;
    }
    __syncthreads();
    // pass 2: prefix with the segment carries, Eq. (3) per bin, best key
    uint64_t best = 0;
    for (int pr = warp; pr < kk * nseg; pr += nwarps) {
      const int j = pr / nseg, seg = pr - j * nseg;
      const int f = f0 + j;
      long long GL = 0, HL = 0, CL = 0, Gt = 0, Ht = 0, Ct = 0;
      for (int s2 = 0; s2 < nseg; ++s2) {
        const long long* st = segtot + ((size_t)j * nseg + s2) * (V + 1);
        const long long g = lane < d ? st[lane] : 0;
        const long long hh = (SOFTMAX && lane < d) ? st[d + lane] : 0;
        const long long cc = st[V];
        if (s2 < seg) { GL += g; HL += hh; CL += cc; }
        Gt += g; Ht += hh; Ct += cc;
      }
      const double sg = lane < d ? (double)scales[lane] : 0.0;
      const double sh = (SOFTMAX && lane < d) ? (double)scales[d + lane] : 0.0;
      const double Gd = (double)Gt * sg;
      const double P = SOFTMAX ? warp_sum_d(lane < d ? Gd * Gd / ((double)Ht * sh + lam) : 0.0)
                               : warp_sum_d(Gd * Gd) / (2.0 * (double)Ct + lam);
      const int nb = nbins[f];
      for (int bi = 0; bi < kSmallSeg; ++bi) {
        const int b = seg * kSmallSeg + bi;
        if (b >= B) break;
        if (lane < d) {
          GL += val(lane, j, b);
          if (SOFTMAX) HL += val(d + lane, j, b);
        }
        CL += cnts[j * B + b];
        if (b > nb - 2) continue;                        // (uniform across the warp)
        if (CL < p.min_node || Ct - CL < p.min_node) continue;
        const double gl = (double)GL * sg, gr = (double)(Gt - GL) * sg;
        double gain;
        if (!SOFTMAX) {
          const double sl = warp_sum_d(gl * gl), sr = warp_sum_d(gr * gr);
          gain = 0.5 * (sl / (2.0 * (double)CL + lam) + sr / (2.0 * (double)(Ct - CL) + lam) - P);
        } else {
          const double hl = (double)HL * sh, hr = (double)(Ht - HL) * sh;
          const double t = lane < d ? gl * gl / (hl + lam) + gr * gr / (hr + lam) : 0.0;
          gain = 0.5 * (warp_sum_d(t) - P);
        }
        if (gain > p.gamma) {
          const uint64_t key = pack_split_key(gain, (int64_t)(p.f_begin + f) * B + b);
          best = key > best ? key : best;
        }
      }
    }
    if (lane == 0) sh_best[warp] = best;
    __syncthreads();
    if (threadIdx.x == 0) {
      uint64_t bb = 0;
      for (int w = 0; w < nwarps; ++w) bb = sh_best[w] > bb ? sh_best[w] : bb;
      if (bb) atomicMax((unsigned long long*)&keys[nd.x], (unsigned long long)bb);
    }
    __syncthreads();
  }
}

template <int K, int KF>
static gbdtmo_status launch_small_kf(Ctx* ctx, const gbdtmo_problem& p, int level, const SmallCfg& sc,
                                     const uint8_t* bins, const int32_t* q, const int32_t* rows, int use_rows,
                                     const int32_t* nbins, const float* scales, const State& s, uint64_t* keys) {
  const bool softmax = p.loss == GBDTMO_LOSS_SOFTMAX;
  auto kern = softmax ? k_search_small<K, KF, true> : k_search_small<K, KF, false>;
  static bool attr_done[2] = {false, false};
  if (!attr_done[softmax]) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, ctx->max_smem_optin - 1024);
    attr_done[softmax] = true;
  }
  GB_LAUNCH(kern, ctx->num_sms, kHistThreads, sc.smem, p, level, sc, bins, q, rows, use_rows, nbins, scales, s, keys);
  return GBDTMO_OK;
}

template <int K>
static gbdtmo_status launch_small(Ctx* ctx, const gbdtmo_problem& p, int level, const SmallCfg& sc,
                                  const uint8_t* bins, const int32_t* q, const int32_t* rows, int use_rows,
                                  const int32_t* nbins, const float* scales, const State& s, uint64_t* keys) {
  switch (sc.kf) {
    case 24: return launch_small_kf<K, 24>(ctx, p, level, sc, bins, q, rows, use_rows, nbins, scales, s, keys);
    case 16: return launch_small_kf<K, 16>(ctx, p, level, sc, bins, q, rows, use_rows, nbins, scales, s, keys);
    case 12: return launch_small_kf<K, 12>(ctx, p, level, sc, bins, q, rows, use_rows, nbins, scales, s, keys);
    case 8: return launch_small_kf<K, 8>(ctx, p, level, sc, bins, q, rows, use_rows, nbins, scales, s, keys);
    case 6: return launch_small_kf<K, 6>(ctx, p, level, sc, bins, q, rows, use_rows, nbins, scales, s, keys);
    case 4: return launch_small_kf<K, 4>(ctx, p, level, sc, bins, q, rows, use_rows, nbins, scales, s, keys);
    case 3: return launch_small_kf<K, 3>(ctx, p, level, sc, bins, q, rows, use_rows, nbins, scales, s, keys);
    case 2: return launch_small_kf<K, 2>(ctx, p, level, sc, bins, q, rows, use_rows, nbins, scales, s, keys);
    default: return launch_small_kf<K, 1>(ctx, p, level, sc, bins, q, rows, use_rows, nbins, scales, s, keys);
  }
}

bool small_supported(const gbdtmo_problem& p) { return small_config(p).ok; }

}  // namespace gbdtmo

using namespace gbdtmo;

extern "C" gbdtmo_status gbdtmo_search_small(gbdtmo_ctx c, const gbdtmo_problem* p, int32_t level,
                                             const uint8_t* bins, const int32_t* q, const int32_t* nbins,
                                             const float* scales, void* state, uint64_t* keys) {
  Ctx* ctx = (Ctx*)c;
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(level >= 0 && level < p->D, "level out of range [0, D)");
  GB_CHECK_ARG(bins && q && nbins && scales && state && keys, "null pointer");
  if (ctx->small_max_rows <= 0) return GBDTMO_OK;             // no node is ever marked SMALL
  const SmallCfg sc = small_config(*p);
  if (!sc.ok) return GBDTMO_OK;
  State s = state_view(*p, state);
  const int32_t* rows = (level & 1) ? s.rows1 : s.rows0;
  const int use_rows = level > 0;
  switch (sc.K) {
    case 4: return launch_small<4>(ctx, *p, level, sc, bins, q, rows, use_rows, nbins, scales, s, keys);
    case 8: return launch_small<8>(ctx, *p, level, sc, bins, q, rows, use_rows, nbins, scales, s, keys);
    default: return launch_small<16>(ctx, *p, level, sc, bins, q, rows, use_rows, nbins, scales, s, keys);
  }
}
