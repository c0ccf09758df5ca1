// split.cu — (a)4 sibling histogram by subtraction, (a)5 multi-output split search, and the
// (a)6 exchange payload (split records + row-direction bitmap).
//
// Split search: for node N, feature f, bin b (left = bins <= b):
//   G_L^k, H_L^k, C_L = prefix sums over bins (exact int64 fixed point, MSE: H = 2 C),
//   gain = 1/2 sum_k [G_L^2/(H_L+l) + G_R^2/(H_R+l) - G^2/(H+l)]   (Eq. 3, fp64),
// valid iff C_L, C_R >= min_node; best per node by an atomicMax on a packed 64-bit key.
#include <string.h>

#include "common.cuh"
#include "peer.cuh"

namespace gbdtmo {

constexpr int kFsWarps = 8;      // warps per block = features of one node per block
#ifndef GBDTMO_FS_PF
#define GBDTMO_FS_PF 2           // channels of L2 prefetch ahead in the split search
#endif
#ifndef GBDTMO_FS_SOFTMAX_MINB
#define GBDTMO_FS_SOFTMAX_MINB 4  // resident blocks per SM of the softmax half-row search: 4 (64 registers, 24 B spilled): C2 find_split 1.80 -> 1.70 ms (profiles/r02_ab_fs_softmax_minb4.jsonl)
#endif
#ifndef GBDTMO_REC_TRANSPOSE
#define GBDTMO_REC_TRANSPOSE 1   // SMALL nodes' split records: rows' q through a shared tile (0: serial per left row)
#endif
#ifndef GBDTMO_FS_CG_OFF
#define GBDTMO_FS_CG_OFF 0       // (A/B) 1: no channel-split search (k_find_split_c)
#endif
#ifndef GBDTMO_FS_HALF
#define GBDTMO_FS_HALF 1         // 1: half-row split search (k_find_split_h) where it applies
#endif


constexpr int kFsBins = 8;       // bins per lane (32 x 8 = 256 = max B)
constexpr int kRecChannels = 64; // record channels per k_split_record block


// Exclusive prefix (over lanes) and total of a per-lane int64.
__device__ __forceinline__ long long warp_excl(long long x, long long* total) {
  const int lane = threadIdx.x & 31;
  long long v = x;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const long long y = __shfl_up_sync(0xffffffffu, v, o);
    if (lane >= o) v += y;
  }
  *total = __shfl_sync(0xffffffffu, v, 31);
  return v - x;
}

// 8 consecutive int64 bins [8 lane, 8 lane + 8) of one channel row (raw values; for a derived
// node parent - sibling, written back when `store`).
__device__ __forceinline__ void load_row8(long long (&v)[kFsBins], const int64_t* cur, const int64_t* par,
                                          const int64_t* sib, bool derive, bool store, int B) {
  const int lane = threadIdx.x & 31;
  const int b0 = lane * kFsBins;
  if (b0 + kFsBins <= B) {
    const longlong2* pc = reinterpret_cast<const longlong2*>(cur + b0);
    if (derive) {
      const longlong2* pp = reinterpret_cast<const longlong2*>(par + b0);
      const longlong2* ps = reinterpret_cast<const longlong2*>(sib + b0);
#pragma unroll
      for (int i = 0; i < kFsBins / 2; ++i) {
        const longlong2 a = pp[i], c = ps[i];
        const longlong2 x = make_longlong2(a.x - c.x, a.y - c.y);
        if (store) const_cast<longlong2*>(pc)[i] = x;
        v[2 * i] = x.x; v[2 * i + 1] = x.y;
      }
    } else {
#pragma unroll
      for (int i = 0; i < kFsBins / 2; ++i) { const longlong2 x = pc[i]; v[2 * i] = x.x; v[2 * i + 1] = x.y; }
    }
  } else {
#pragma unroll
    for (int i = 0; i < kFsBins; ++i) {
      const int b = b0 + i;
      long long x = 0;
      if (b < B) {
        if (derive) { x = par[b] - sib[b]; if (store) const_cast<int64_t*>(cur)[b] = x; }
        else x = cur[b];
      }
      v[i] = x;
    }
  }
}

// Inclusive prefix over bins of one row held 8 bins per lane.  The default bin `db` (sparsity-
// aware skip; -1: none) is not trusted: its value is recovered as node total - sum of the other
// bins, written back through `wb` when non-null.  Returns the node total.
__device__ __forceinline__ long long row_prefix(long long (&v)[kFsBins], int db, long long node_total,
                                                int64_t* wb, long long* delta_out = nullptr) {
  const int lane = threadIdx.x & 31;
  const int b0 = lane * kFsBins;
  const bool mine = db >= b0 && db < b0 + kFsBins;
#pragma unroll
  for (int i = 0; i < kFsBins; ++i) if (mine && db == b0 + i) v[i] = 0;
#pragma unroll
  for (int i = 1; i < kFsBins; ++i) v[i] += v[i - 1];
  long long others;
  const long long ex = warp_excl(v[kFsBins - 1], &others);
  if (db < 0) {
#pragma unroll
    for (int i = 0; i < kFsBins; ++i) v[i] += ex;
    return others;
  }
  const long long delta = node_total - others;
#pragma unroll
  for (int i = 0; i < kFsBins; ++i) v[i] += ex + ((b0 + i >= db) ? delta : 0);
  if (mine && wb) wb[db] = delta;
  if (delta_out) *delta_out = delta;
  return node_total;
}

// One warp per (node, feature); lane l owns bins [8l, 8l + 8).  Per channel the warp reads the
// contiguous row of B int64 bins (channel-major histogram: coalesced 16-byte loads), prefix-sums
// it (in-lane + warp scan; the feature's default bin recovered from the exact node totals), and
// accumulates per bin: MSE sum_k G_L^2 and sum_k G_R^2 (H = 2 C is shared by all outputs: two
// divisions per bin), softmax the Eq. (3) terms.
template <bool SOFTMAX>
__global__ void __launch_bounds__(kFsWarps * 32)
k_find_split(gbdtmo_problem p, int level, const int32_t* __restrict__ nbins, const int32_t* __restrict__ dflt,
             const float* __restrict__ scales, State s, int64_t* __restrict__ hist, int32_t* __restrict__ cnt,
             const int64_t* __restrict__ phist, const int32_t* __restrict__ pcnt,
             uint64_t* __restrict__ keys, int write_derived) {
  // level 0: one node, warps = 8 features.  Deeper: a block holds a sibling pair, warps 0-3 the
  // left child and 4-7 the right child over the same 4 features, so the derived child's reads
  // of its built sibling's rows meet them in L2 while the sibling's own search streams them
  // from DRAM (one DRAM pass over the built histogram instead of two).
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const bool paired = level > 0;
  const int slot = paired ? 2 * blockIdx.y + (warp >> 2) : 0;
  const int f = paired ? blockIdx.x * (kFsWarps / 2) + (warp & 3) : blockIdx.x * kFsWarps + warp;
  const int64_t h = (int64_t(1) << level) - 1 + slot;
  const bool searched = s.node_state[h] == GBDTMO_NODE_ACTIVE && s.node_mode[h] != MODE_SMALL;  // SMALL: small.cu
  const bool derive = s.node_mode[h] == MODE_DERIVE;
  const bool store = derive && write_derived;
  const bool own = !derive || store;                  // this node's histogram may be written
  const int V = channels(p), B = p.B, m = p.m, d = p.d;
  const int sib = slot ^ 1, par = slot >> 1;
  const double lam = p.lambda;
  const int64_t* S = s.node_sum + h * (V + 1);         // exact node totals (channels, count)
  __shared__ unsigned long long wbest[kFsWarps];
  uint64_t best = 0;
  if (searched && f < m) {
    const int db = dflt ? dflt[f] : -1;
    const int b0 = lane * kFsBins;
    // counts
    long long cl[kFsBins];
    long long ctot;
    {
      const int64_t oc = (hist_index(p, level, slot) * m + f) * B, os = (hist_index(p, level, sib) * m + f) * B, op = ((int64_t)par * m + f) * B;
#pragma unroll
      for (int i = 0; i < kFsBins; ++i) {
        const int b = b0 + i;
        long long x = 0;
        if (b < B) {
          if (derive) { x = pcnt[op + b] - cnt[os + b]; if (store) cnt[oc + b] = (int32_t)x; }
          else x = cnt[oc + b];
        }
        cl[i] = x;
      }
      long long dc = 0;
      ctot = row_prefix(cl, db, S[V], nullptr, &dc);
      if (own && db >= b0 && db < b0 + kFsBins) cnt[oc + db] = (int32_t)dc;   // recovered default-bin count
    }
    // ---- channels
    const int64_t rowc = (hist_index(p, level, slot) * m + f) * V * B, rows_ = (hist_index(p, level, sib) * m + f) * V * B,
                  rowp = ((int64_t)par * m + f) * V * B;
    double accL[kFsBins], accR[kFsBins];
#pragma unroll
    for (int i = 0; i < kFsBins; ++i) { accL[i] = 0.0; accR[i] = 0.0; }
    double P = 0.0;
    // L2 prefetch of the channel rows GBDTMO_FS_PF channels ahead (softmax: g and h rows): the
    // warp's loads are one dependent chain per channel, so without it ~55% of DRAM bandwidth
    // is reached at this kernel's register-limited occupancy (ncu, profiles/r01f_ncu_fs_c5.txt)
    auto prefetch = [&](int k) {
      if (k >= V) return;
      const int64_t o = (int64_t)k * B + lane * kFsBins;
      if (derive) {
        asm volatile("prefetch.global.L2 [%0];" ::"l"(phist + rowp + o));
        asm volatile("prefetch.global.L2 [%0];" ::"l"(hist + rows_ + o));
      } else {
        asm volatile("prefetch.global.L2 [%0];" ::"l"(hist + rowc + o));
      }
    };
    constexpr int PF = GBDTMO_FS_PF;
#pragma unroll
    for (int k = 0; k < PF; ++k) {
      prefetch(k);
      if (SOFTMAX) prefetch(d + k);
    }
    for (int k = 0; k < d; ++k) {
      if (PF > 0) {
        prefetch(k + PF);
        if (SOFTMAX && k + PF < d) prefetch(d + k + PF);
      }
      long long gv[kFsBins];
      int64_t* rg = hist + rowc + (int64_t)k * B;
      load_row8(gv, rg, phist + rowp + (int64_t)k * B, hist + rows_ + (int64_t)k * B, derive, store, B);
      const long long G = row_prefix(gv, db, S[k], own ? rg : nullptr);
      const double sg = (double)scales[k];
      if (!SOFTMAX) {
#pragma unroll
        for (int i = 0; i < kFsBins; ++i) {
          const double GL = (double)gv[i] * sg, GR = (double)(G - gv[i]) * sg;
          accL[i] = fma(GL, GL, accL[i]);
          accR[i] = fma(GR, GR, accR[i]);
        }
        const double Gd = (double)G * sg;
        P = fma(Gd, Gd, P);
      } else {
        long long hv[kFsBins];
        int64_t* rh = hist + rowc + (int64_t)(d + k) * B;
        load_row8(hv, rh, phist + rowp + (int64_t)(d + k) * B, hist + rows_ + (int64_t)(d + k) * B, derive, store, B);
        const long long H = row_prefix(hv, db, S[d + k], own ? rh : nullptr);
        const double sh = (double)scales[d + k];
#pragma unroll
        for (int i = 0; i < kFsBins; ++i) {
          const double GL = (double)gv[i] * sg, GR = (double)(G - gv[i]) * sg;
          const double HL = (double)hv[i] * sh, HR = (double)(H - hv[i]) * sh;
          accL[i] += eq3_pair(GL, HL + lam, GR, HR + lam);
        }
        const double Gd = (double)G * sg, Hd = (double)H * sh;
        P += Gd * Gd / (Hd + lam);
      }
    }
    // ---- gains and the lane's best candidate
    const int nb = nbins[f];
    const int64_t fb0 = (int64_t)(p.f_begin + f) * B;
#pragma unroll
    for (int i = 0; i < kFsBins; ++i) {
      const int b = b0 + i;
      const long long c = cl[i];
      if (b < B && b <= nb - 2 && c >= p.min_node && ctot - c >= p.min_node) {
        double gain;
        if (!SOFTMAX)
          gain = 0.5 * (accL[i] / (2.0 * (double)c + lam) + accR[i] / (2.0 * (double)(ctot - c) + lam) -
                        P / (2.0 * (double)ctot + lam));
        else
          gain = 0.5 * (accL[i] - P);
        if (gain > p.gamma) {
          const uint64_t key = pack_split_key(gain, fb0 + b);
          best = key > best ? key : best;
        }
      }
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const uint64_t y = __shfl_xor_sync(0xffffffffu, best, o);
    best = y > best ? y : best;
  }
  if (lane == 0) wbest[warp] = best;
  __syncthreads();
  if (lane == 0 && (paired ? (warp & 3) == 0 : warp == 0)) {   // one reducer per slot in the block
    const int w0 = paired ? warp : 0, nw = paired ? kFsWarps / 2 : kFsWarps;
    uint64_t bb = 0;
    for (int w = w0; w < w0 + nw; ++w) bb = wbest[w] > bb ? wbest[w] : bb;
    if (bb) atomicMax((unsigned long long*)&keys[slot], (unsigned long long)bb);
  }
}

// Half-row variant (no default bins, 128 < B <= 256): two warps per (node, feature), lane l of
// half h owns bins [128 h + 4 l, +4), so a lane holds half the row state of k_find_split and
// the kernel runs at twice the occupancy (the 8-bin kernel is latency-bound at 128 registers:
// ncu, profiles/r02_ncu_fs_C2.txt).  The halves need no exchange: half 0 prefix-sums its
// bins (left sums), half 1 suffix-sums its bins (right sums, bins > b) and both complete the
// other side from the exact node totals (node_sum = the sum of the node's histogram row in
// int64), so every G_L, G_R, C_L is the same integer as in k_find_split and the gains and
// keys are bit-identical.
constexpr int kFsHBins = 4;

// half 0: inclusive prefix of 4 bins per lane over the warp; half 1: exclusive suffix (bins > b).
__device__ __forceinline__ void half_scan(long long (&v)[kFsHBins], bool suffix) {
  const int lane = threadIdx.x & 31;
  if (!suffix) {
#pragma unroll
    for (int i = 1; i < kFsHBins; ++i) v[i] += v[i - 1];
    long long tot;
    const long long ex = warp_excl(v[kFsHBins - 1], &tot);
#pragma unroll
    for (int i = 0; i < kFsHBins; ++i) v[i] += ex;
  } else {
    long long run = 0;
#pragma unroll
    for (int i = kFsHBins - 1; i >= 0; --i) { const long long x = v[i]; v[i] = run; run += x; }
    long long sfx = run;                                    // inclusive suffix over lanes
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const long long y = __shfl_down_sync(0xffffffffu, sfx, o);
      if (lane + o < 32) sfx += y;
    }
    const long long ex = sfx - run;                         // lanes above this one
#pragma unroll
    for (int i = 0; i < kFsHBins; ++i) v[i] += ex;
  }
}

// 4 consecutive bins [b0, b0 + 4) of one row (derived: parent - sibling, written back if store)
__device__ __forceinline__ void load_row4(long long (&v)[kFsHBins], int b0, const int64_t* cur, const int64_t* par,
                                          const int64_t* sib, bool derive, bool store, int B) {
  if (b0 + kFsHBins <= B) {
    if (derive) {
      const longlong2* pp = reinterpret_cast<const longlong2*>(par + b0);
      const longlong2* ps = reinterpret_cast<const longlong2*>(sib + b0);
      const longlong2 a0 = pp[0], a1 = pp[1], c0 = ps[0], c1 = ps[1];
      const longlong2 x0 = make_longlong2(a0.x - c0.x, a0.y - c0.y), x1 = make_longlong2(a1.x - c1.x, a1.y - c1.y);
      if (store) {
        longlong2* pc = reinterpret_cast<longlong2*>(const_cast<int64_t*>(cur) + b0);
        pc[0] = x0; pc[1] = x1;
      }
      v[0] = x0.x; v[1] = x0.y; v[2] = x1.x; v[3] = x1.y;
    } else {
      const longlong2* pc = reinterpret_cast<const longlong2*>(cur + b0);
      const longlong2 x0 = pc[0], x1 = pc[1];
      v[0] = x0.x; v[1] = x0.y; v[2] = x1.x; v[3] = x1.y;
    }
  } else {
#pragma unroll
    for (int i = 0; i < kFsHBins; ++i) {
      const int b = b0 + i;
      long long x = 0;
      if (b < B) {
        if (derive) { x = par[b] - sib[b]; if (store) const_cast<int64_t*>(cur)[b] = x; }
        else x = cur[b];
      }
      v[i] = x;
    }
  }
}

// MINB = resident blocks per SM the kernel is compiled for: 3 (80 registers); MSE problems with at
// most 16 channels take 4 (64 registers, 8 bytes spilled): C5 9.60 -> 9.27 ms per tree, while C3 / C4
// lose 3-6% with it (profiles/r02_ab_find_split_minb4.jsonl).  Softmax takes 4 as well (GBDTMO_FS_SOFTMAX_MINB; 2: C2 2.40 -> 2.99 ms, 4: 1.80 -> 1.70).
template <bool SOFTMAX, int MINB>
__global__ void __launch_bounds__(kFsWarps * 32, MINB)
k_find_split_h(gbdtmo_problem p, int level, const int32_t* __restrict__ nbins, const float* __restrict__ scales,
               State s, int64_t* __restrict__ hist, int32_t* __restrict__ cnt, const int64_t* __restrict__ phist,
               const int32_t* __restrict__ pcnt, uint64_t* __restrict__ keys, int write_derived) {
  // warps: [sibling (paired levels: warp >> 2)][feature][half]; level 0: [feature (4)][half]
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int half = warp & 1;
  const bool paired = level > 0;
  const int slot = paired ? 2 * blockIdx.y + (warp >> 2) : 0;
  const int f = paired ? blockIdx.x * 2 + ((warp >> 1) & 1) : blockIdx.x * 4 + (warp >> 1);
  const int64_t h = (int64_t(1) << level) - 1 + slot;
  const bool searched = s.node_state[h] == GBDTMO_NODE_ACTIVE && s.node_mode[h] != MODE_SMALL;
  const bool derive = s.node_mode[h] == MODE_DERIVE;
  const bool store = derive && write_derived;
  const int V = channels(p), B = p.B, m = p.m, d = p.d;
  const int sib = slot ^ 1, par = slot >> 1;
  const double lam = p.lambda;
  const int64_t* S = s.node_sum + h * (V + 1);
  __shared__ unsigned long long wbest[kFsWarps];
  uint64_t best = 0;
  const int b0 = half * (32 * kFsHBins) + lane * kFsHBins;
  if (searched && f < m && half * (32 * kFsHBins) < B) {
    // counts -> C_L per bin (kept as int32 through the channel loop: C_L < n < 2^31; this keeps
    // the softmax instantiation inside its 80-register budget without spilling)
    int cl[kFsHBins];
    const int ctot = (int)S[V];
    {
      long long cw[kFsHBins];
      const int64_t oc = (hist_index(p, level, slot) * m + f) * B, os = (hist_index(p, level, sib) * m + f) * B, op = ((int64_t)par * m + f) * B;
#pragma unroll
      for (int i = 0; i < kFsHBins; ++i) {
        const int b = b0 + i;
        long long x = 0;
        if (b < B) {
          if (derive) { x = pcnt[op + b] - cnt[os + b]; if (store) cnt[oc + b] = (int32_t)x; }
          else x = cnt[oc + b];
        }
        cw[i] = x;
      }
      half_scan(cw, half);
#pragma unroll
      for (int i = 0; i < kFsHBins; ++i) cl[i] = (int)(half ? (long long)ctot - cw[i] : cw[i]);
    }
    const int64_t rowc = (hist_index(p, level, slot) * m + f) * V * B, rows_ = (hist_index(p, level, sib) * m + f) * V * B,
                  rowp = ((int64_t)par * m + f) * V * B;
    double accL[kFsHBins], accR[kFsHBins];
#pragma unroll
    for (int i = 0; i < kFsHBins; ++i) { accL[i] = 0.0; accR[i] = 0.0; }
    double P = 0.0;
    auto prefetch = [&](int k) {
      if (k >= V) return;
      const int64_t o = (int64_t)k * B + b0;
      if (derive) {
        asm volatile("prefetch.global.L2 [%0];" ::"l"(phist + rowp + o));
        asm volatile("prefetch.global.L2 [%0];" ::"l"(hist + rows_ + o));
      } else {
        asm volatile("prefetch.global.L2 [%0];" ::"l"(hist + rowc + o));
      }
    };
    constexpr int PF = GBDTMO_FS_PF;
#pragma unroll
    for (int k = 0; k < PF; ++k) {
      prefetch(k);
      if (SOFTMAX) prefetch(d + k);
    }
    auto mse_acc = [&](long long (&gl)[kFsHBins], int k) {
      half_scan(gl, half);
      const long long G = S[k];
      if (half) {
#pragma unroll
        for (int i = 0; i < kFsHBins; ++i) gl[i] = G - gl[i];
      }
      const double sg = (double)scales[k];
#pragma unroll
      for (int i = 0; i < kFsHBins; ++i) {
        const double GL = (double)gl[i] * sg, GR = (double)(G - gl[i]) * sg;
        accL[i] = fma(GL, GL, accL[i]);
        accR[i] = fma(GR, GR, accR[i]);
      }
      const double Gd = (double)G * sg;
      P = fma(Gd, Gd, P);
    };
    for (int k = 0; k < d; ++k) {
      if (PF > 0) {
        prefetch(k + PF);
        if (SOFTMAX && k + PF < d) prefetch(d + k + PF);
      }
      // left sums GL[i] and right sums G - GL[i] as exact integers
      long long gl[kFsHBins];
      load_row4(gl, b0, hist + rowc + (int64_t)k * B, phist + rowp + (int64_t)k * B, hist + rows_ + (int64_t)k * B,
                derive, store, B);
      if (!SOFTMAX) {
        mse_acc(gl, k);
      } else {
        half_scan(gl, half);
        const long long G = S[k];
        if (half) {
#pragma unroll
          for (int i = 0; i < kFsHBins; ++i) gl[i] = G - gl[i];
        }
        const double sg = (double)scales[k];
        long long hl[kFsHBins];
        load_row4(hl, b0, hist + rowc + (int64_t)(d + k) * B, phist + rowp + (int64_t)(d + k) * B,
                  hist + rows_ + (int64_t)(d + k) * B, derive, store, B);
        half_scan(hl, half);
        const long long H = S[d + k];
        if (half) {
#pragma unroll
          for (int i = 0; i < kFsHBins; ++i) hl[i] = H - hl[i];
        }
        const double sh = (double)scales[d + k];
#pragma unroll
        for (int i = 0; i < kFsHBins; ++i) {
          const double GL = (double)gl[i] * sg, GR = (double)(G - gl[i]) * sg;
          const double HL = (double)hl[i] * sh, HR = (double)(H - hl[i]) * sh;
          accL[i] += eq3_pair(GL, HL + lam, GR, HR + lam);
        }
        const double Gd = (double)G * sg, Hd = (double)H * sh;
        P += Gd * Gd / (Hd + lam);
      }
    }
    const int nb = nbins[f];
    const int64_t fb0 = (int64_t)(p.f_begin + f) * B;
#pragma unroll
    for (int i = 0; i < kFsHBins; ++i) {
      const int b = b0 + i;
      const long long c = cl[i];
      if (b < B && b <= nb - 2 && c >= p.min_node && ctot - c >= p.min_node) {
        double gain;
        if (!SOFTMAX)
          gain = 0.5 * (accL[i] / (2.0 * (double)c + lam) + accR[i] / (2.0 * (double)(ctot - c) + lam) -
                        P / (2.0 * (double)ctot + lam));
        else
          gain = 0.5 * (accL[i] - P);
        if (gain > p.gamma) {
          const uint64_t key = pack_split_key(gain, fb0 + b);
          best = key > best ? key : best;
        }
      }
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const uint64_t y = __shfl_xor_sync(0xffffffffu, best, o);
    best = y > best ? y : best;
  }
  if (lane == 0) wbest[warp] = best;
  __syncthreads();
  if (lane == 0 && (paired ? (warp & 3) == 0 : warp == 0)) {
    const int w0 = paired ? warp : 0, nw = paired ? kFsWarps / 2 : kFsWarps;
    uint64_t bb = 0;
    for (int w = w0; w < w0 + nw; ++w) bb = wbest[w] > bb ? wbest[w] : bb;
    if (bb) atomicMax((unsigned long long*)&keys[slot], (unsigned long long)bb);
  }
}

// Channel-split search for shallow levels of wide problems: the half-row kernel
// gives every (node, feature) two warps that each walk all V channel rows, so a level with few
// nodes x features leaves most SMs idle (C4 root: 125 blocks for 148 SMs, 12% occupancy, 22% of
// HBM; C3 root: 25 blocks).  Eq. (3) is a sum over outputs, so the channel loop splits: one block
// per (node, feature), warps = [channel group cg < CG][half]; warp (cg, half) takes outputs
// k = cg, cg + CG, ... of its half's bins, and the per-bin partial sums (sum_k G_L^2, sum_k G_R^2,
// sum_k G^2 for MSE; the Eq. (3) terms for softmax) are added in shared memory in cg order (a fixed
// order: deterministic; the sums differ from the sequential kernel's by fp64 rounding only).
// Integer work (prefix sums, derived rows, validity) is exactly k_find_split_h's.
// Blocks are (slot, feature) with the slot fastest, so the two children of a split run side by
// side and the derived child's reads of its built sibling hit L2.
template <bool SOFTMAX, int CGMAX>
__global__ void __launch_bounds__(2 * 32 * CGMAX, CGMAX <= 4 ? 3 : 1)
k_find_split_c(gbdtmo_problem p, int level, const int32_t* __restrict__ nbins, const float* __restrict__ scales,
               State s, int64_t* __restrict__ hist, int32_t* __restrict__ cnt, const int64_t* __restrict__ phist,
               const int32_t* __restrict__ pcnt, uint64_t* __restrict__ keys, int write_derived) {
  constexpr int kFsCgMax = CGMAX;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int half = warp & 1, cg = warp >> 1, CG = blockDim.x >> 6;
  const int slot = blockIdx.x, f = blockIdx.y;
  const int64_t h = (int64_t(1) << level) - 1 + slot;
  // block-uniform exits (before any barrier)
  if (!(s.node_state[h] == GBDTMO_NODE_ACTIVE && s.node_mode[h] != MODE_SMALL) || f >= p.m) return;
  const bool derive = level > 0 && s.node_mode[h] == MODE_DERIVE;
  const bool store = derive && write_derived;
  const int V = channels(p), B = p.B, m = p.m, d = p.d;
  const int sib = slot ^ 1, par = slot >> 1;
  const double lam = p.lambda;
  const int64_t* S = s.node_sum + h * (V + 1);
  constexpr int NP = 2 * kFsHBins + 1;                    // accL[4], accR[4], P
  __shared__ double part[2 * kFsCgMax][NP][32];
  __shared__ unsigned long long hbest[2];
  const int b0 = half * (32 * kFsHBins) + lane * kFsHBins;
  int cl[kFsHBins];
  const int ctot = (int)S[V];
  {
    long long cw[kFsHBins];
    const int64_t oc = (hist_index(p, level, slot) * m + f) * B, os = (hist_index(p, level, sib) * m + f) * B,
                  op = ((int64_t)par * m + f) * B;
#pragma unroll
    for (int i = 0; i < kFsHBins; ++i) {
      const int b = b0 + i;
      long long x = 0;
      if (b < B) {
        if (derive) { x = pcnt[op + b] - cnt[os + b]; if (store && cg == 0) cnt[oc + b] = (int32_t)x; }
        else x = cnt[oc + b];
      }
      cw[i] = x;
    }
    half_scan(cw, half);
#pragma unroll
    for (int i = 0; i < kFsHBins; ++i) cl[i] = (int)(half ? (long long)ctot - cw[i] : cw[i]);
  }
  const int64_t rowc = (hist_index(p, level, slot) * m + f) * V * B, rows_ = (hist_index(p, level, sib) * m + f) * V * B,
                rowp = ((int64_t)par * m + f) * V * B;
  double accL[kFsHBins], accR[kFsHBins];
#pragma unroll
  for (int i = 0; i < kFsHBins; ++i) { accL[i] = 0.0; accR[i] = 0.0; }
  double P = 0.0;
  auto prefetch = [&](int k) {                           // channel rows two of this warp's iterations ahead
    if (k >= d) return;
    const int64_t o = (int64_t)k * B + b0;
    if (derive) {
      asm volatile("prefetch.global.L2 [%0];" ::"l"(phist + rowp + o));
      asm volatile("prefetch.global.L2 [%0];" ::"l"(hist + rows_ + o));
    } else {
      asm volatile("prefetch.global.L2 [%0];" ::"l"(hist + rowc + o));
    }
    if (SOFTMAX) {
      const int64_t oh = (int64_t)(d + k) * B + b0;
      if (derive) {
        asm volatile("prefetch.global.L2 [%0];" ::"l"(phist + rowp + oh));
        asm volatile("prefetch.global.L2 [%0];" ::"l"(hist + rows_ + oh));
      } else {
        asm volatile("prefetch.global.L2 [%0];" ::"l"(hist + rowc + oh));
      }
    }
  };
  prefetch(cg);
  prefetch(cg + CG);
  for (int k = cg; k < d; k += CG) {
    prefetch(k + 2 * CG);
    long long gl[kFsHBins];
    load_row4(gl, b0, hist + rowc + (int64_t)k * B, phist + rowp + (int64_t)k * B, hist + rows_ + (int64_t)k * B,
              derive, store, B);
    half_scan(gl, half);
    const long long G = S[k];
    if (half) {
#pragma unroll
      for (int i = 0; i < kFsHBins; ++i) gl[i] = G - gl[i];
    }
    const double sg = (double)scales[k];
    if (!SOFTMAX) {
#pragma unroll
      for (int i = 0; i < kFsHBins; ++i) {
        const double GL = (double)gl[i] * sg, GR = (double)(G - gl[i]) * sg;
        accL[i] = fma(GL, GL, accL[i]);
        accR[i] = fma(GR, GR, accR[i]);
      }
      const double Gd = (double)G * sg;
      P = fma(Gd, Gd, P);
    } else {
      long long hl[kFsHBins];
      load_row4(hl, b0, hist + rowc + (int64_t)(d + k) * B, phist + rowp + (int64_t)(d + k) * B,
                hist + rows_ + (int64_t)(d + k) * B, derive, store, B);
      half_scan(hl, half);
      const long long H = S[d + k];
      if (half) {
#pragma unroll
        for (int i = 0; i < kFsHBins; ++i) hl[i] = H - hl[i];
      }
      const double sh = (double)scales[d + k];
#pragma unroll
      for (int i = 0; i < kFsHBins; ++i) {
        const double GL = (double)gl[i] * sg, GR = (double)(G - gl[i]) * sg;
        const double HL = (double)hl[i] * sh, HR = (double)(H - hl[i]) * sh;
        accL[i] += eq3_pair(GL, HL + lam, GR, HR + lam);
      }
      const double Gd = (double)G * sg, Hd = (double)H * sh;
      P += Gd * Gd / (Hd + lam);
    }
  }
#pragma unroll
  for (int i = 0; i < kFsHBins; ++i) { part[warp][i][lane] = accL[i]; part[warp][kFsHBins + i][lane] = accR[i]; }
  part[warp][2 * kFsHBins][lane] = P;
  __syncthreads();
  if (cg == 0) {
    for (int g = 1; g < CG; ++g) {                     // fixed order: cg 0, 1, ..., CG-1
      const int w = 2 * g + half;
#pragma unroll
      for (int i = 0; i < kFsHBins; ++i) { accL[i] += part[w][i][lane]; accR[i] += part[w][kFsHBins + i][lane]; }
      P += part[w][2 * kFsHBins][lane];
    }
    uint64_t best = 0;
    if (half * (32 * kFsHBins) < B) {
      const int nb = nbins[f];
      const int64_t fb0 = (int64_t)(p.f_begin + f) * B;
#pragma unroll
      for (int i = 0; i < kFsHBins; ++i) {
        const int b = b0 + i;
        const long long c = cl[i];
        if (b < B && b <= nb - 2 && c >= p.min_node && ctot - c >= p.min_node) {
          double gain;
          if (!SOFTMAX)
            gain = 0.5 * (accL[i] / (2.0 * (double)c + lam) + accR[i] / (2.0 * (double)(ctot - c) + lam) -
                          P / (2.0 * (double)ctot + lam));
          else
            gain = 0.5 * (accL[i] - P);
          if (gain > p.gamma) {
            const uint64_t key = pack_split_key(gain, fb0 + b);
            best = key > best ? key : best;
          }
        }
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      const uint64_t y = __shfl_xor_sync(0xffffffffu, best, o);
      best = y > best ? y : best;
    }
    if (lane == 0) hbest[half] = best;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    const uint64_t bb = hbest[0] > hbest[1] ? hbest[0] : hbest[1];
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
__global__ void k_split_record(gbdtmo_problem p, int level, const int32_t* __restrict__ dflt,
                               const uint8_t* __restrict__ bins, const int32_t* __restrict__ q, State s,
                               const int64_t* __restrict__ hist,
                               const int32_t* __restrict__ cnt, const int64_t* __restrict__ phist,
                               const int32_t* __restrict__ pcnt, const uint64_t* __restrict__ keys,
                               const float* __restrict__ scales, int64_t* __restrict__ xchg, PeerView pv,
                               uint64_t* __restrict__ keys_merged) {
  const int slot = blockIdx.x;
  const int64_t h = (int64_t(1) << level) - 1 + slot;
  const int V = channels(p), B = p.B, m = p.m;
  const int64_t RW = rec_words(p);
  int64_t* rec = xchg + slot * RW;
  // blockIdx.y: block of kRecChannels channels of the record (c = V is the count)
  const int c0 = blockIdx.y * kRecChannels, c1 = min(V + 1, c0 + kRecChannels);
  uint64_t key;
  if (pv.world > 0) {
    // fused key exchange (peer.cuh): block 0 publishes this rank's keys, every block waits for the
    // peers and takes the max of its slot's key over the N windows (= the MAX all-reduce)
    __shared__ unsigned long long sk;
    if (threadIdx.x == 0) {
      const uint64_t E = peer_next_epoch(pv);
      peer_publish_wait(pv, PEER_FLAG_KEYS, E, slot == 0 && blockIdx.y == 0);
      const int64_t ko = peer_keys_off(p, level) / 8 + slot;
      uint64_t k = 0;
      for (int r = 0; r < pv.world; ++r) {
        const uint64_t x = peer_load(reinterpret_cast<const uint64_t*>(pv.win[r]) + ko);
        k = x > k ? x : k;
      }
      if (blockIdx.y == 0) keys_merged[slot] = k;
      sk = k;
    }
    __syncthreads();
    key = sk;
  } else {
    key = keys[slot];
  }
  int fl = 0, b = 0, fg = 0;
  const bool own = s.node_state[h] == GBDTMO_NODE_ACTIVE && decode_local(p, key, &fl, &b, &fg);
  if (!own) {
    for (int i = c0 + threadIdx.x; i < c1; i += blockDim.x) rec[i] = 0;
    if (blockIdx.y == 0 && threadIdx.x < 3) rec[V + 1 + threadIdx.x] = 0;
    return;
  }
  const bool derive = s.node_mode[h] == MODE_DERIVE;
  const int sib = slot ^ 1, par = slot >> 1;
  const int64_t rc = (hist_index(p, level, slot) * m + fl) * B, rs = (hist_index(p, level, sib) * m + fl) * B, rp = ((int64_t)par * m + fl) * B;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const int db = dflt ? dflt[fl] : -1;            // default bin: recovered from the node totals
  const int64_t* S = s.node_sum + h * (V + 1);
  if (s.node_mode[h] == MODE_SMALL) {             // not materialised: left sums straight from the rows
    if (blockIdx.y != 0) return;                  // (d <= 32: one block covers every channel)
    // one pass: warps take 32 rows at a time, lanes = channels sum the rows that go left
    __shared__ long long acc[2 * 32 + 1];
    __shared__ int32_t tq[GBDTMO_REC_TRANSPOSE ? 8 : 1][32][33];
    for (int c = threadIdx.x; c <= V; c += blockDim.x) acc[c] = 0;
    __syncthreads();
    const int32_t* rl = (level & 1) ? s.rows1 : s.rows0;
    const int nb0 = s.node_begin[h], nb1 = s.node_end[h];
    long long a0 = 0, a1 = 0, nleft = 0;
    for (int pos0 = nb0 + warp * 32; pos0 < nb1; pos0 += nw * 32) {
      const int pos = pos0 + lane;
      const int r = pos < nb1 ? (level > 0 ? rl[pos] : pos) : -1;
      const bool left = r >= 0 && bins[(int64_t)r * p.ld_bins + fl] <= b;
      const unsigned msk = __ballot_sync(0xffffffffu, left);
      nleft += __popc(msk);
      if (GBDTMO_REC_TRANSPOSE) {
        // lanes = rows: each left row's q values go through a [32][33] shared tile (independent
        // loads, no per-row serial chain), then lanes = channels add the 32 rows
        for (int cc = 0; cc < V; cc += 32) {
#pragma unroll 8
          for (int c = 0; c < 32; ++c)
            tq[warp][lane][c] = (left && cc + c < V) ? q[(int64_t)r * V + cc + c] : 0;
          __syncwarp();
          long long sacc = 0;
#pragma unroll 8
          for (int i = 0; i < 32; ++i) sacc += tq[warp][i][lane];
          if (cc == 0) a0 += sacc; else a1 += sacc;
          __syncwarp();
        }
      } else {
        unsigned mm = msk;
        while (mm) {
          const int src = __ffs(mm) - 1;
          mm &= mm - 1;
          const int64_t rr = (int64_t)__shfl_sync(0xffffffffu, r, src) * V;
          if (lane < V) a0 += q[rr + lane];
          if (lane + 32 < V) a1 += q[rr + lane + 32];
        }
      }
    }
    if (lane < V) atomicAdd((unsigned long long*)&acc[lane], (unsigned long long)a0);
    if (lane + 32 < V) atomicAdd((unsigned long long*)&acc[lane + 32], (unsigned long long)a1);
    if (lane == 0) atomicAdd((unsigned long long*)&acc[V], (unsigned long long)nleft);
    __syncthreads();
    for (int c = threadIdx.x; c <= V; c += blockDim.x) rec[c] = acc[c];
  } else
  for (int c = c0 + warp; c < c1; c += nw) {      // c == V: the counts
    long long le = 0, all = 0;
    for (int bb = lane; bb < B; bb += 32) {
      if (bb == db) continue;
      long long x;
      if (c < V) x = derive ? (phist[(rp * V) + (int64_t)c * B + bb] - hist[(rs * V) + (int64_t)c * B + bb])
                            : hist[(rc * V) + (int64_t)c * B + bb];
      else x = derive ? (long long)(pcnt[rp + bb] - cnt[rs + bb]) : (long long)cnt[rc + bb];
      all += x;
      if (bb <= b) le += x;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      le += __shfl_xor_sync(0xffffffffu, le, o);
      all += __shfl_xor_sync(0xffffffffu, all, o);
    }
    if (db >= 0 && db <= b) le += S[c] - all;      // (S[V] = the node's row count)
    if (lane == 0) rec[c] = le;
  }
  if (blockIdx.y == 0 && threadIdx.x == 0) {
    rec[V + 1] = fg + 1;
    rec[V + 2] = b;
  }
}

// Exact Eq. (3) at each owned winner from the record's exact left sums (informational: the tree
// record's gain; the choice was made on the keys).  One warp per slot, lanes over outputs.
__global__ void k_record_gain(gbdtmo_problem p, int level, State s, const float* __restrict__ scales,
                              int64_t* __restrict__ xchg) {
  const int lane = threadIdx.x & 31;
  const int64_t slot = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t LN = int64_t(1) << level;
  if (slot >= LN) return;
  const int V = channels(p), d = p.d;
  const int64_t RW = rec_words(p);
  int64_t* rec = xchg + slot * RW;
  if (rec[V + 1] == 0) return;                   // not split here / not owned by this rank
  const int64_t h = LN - 1 + slot;
  const int64_t* S = s.node_sum + h * (V + 1);
  const bool softmax = p.loss == GBDTMO_LOSS_SOFTMAX;
  const long long ctot = S[V], cl = rec[V];
  double g = 0.0;
  for (int k = lane; k < d; k += 32) {
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
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) g += __shfl_xor_sync(0xffffffffu, g, o);
  if (lane == 0) rec[V + 3] = __double_as_longlong(0.5 * g);
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
                                           const int32_t* nbins, const int32_t* dflt, const float* scales, void* state,
                                           int64_t* hist, int32_t* cnt, const int64_t* parent_hist,
                                           const int32_t* parent_cnt, uint64_t* keys) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(level >= 0 && level < p->D, "level out of range [0, D)");
  GB_CHECK_ARG(nbins && scales && state && hist && cnt && keys, "null pointer");
  GB_CHECK_ARG(level == 0 || (parent_hist && parent_cnt), "parent histogram required for level > 0");
  State s = state_view(*p, state);
  const int64_t LN = int64_t(1) << level;
  GB_LAUNCH(k_zero_u64, 1, 256, 0, keys, LN);
  const bool softmax = p->loss == GBDTMO_LOSS_SOFTMAX;
  if (GBDTMO_FS_HALF && !dflt && p->B > 128) {
    // two warps per (node, feature): 2 features x 2 siblings per block, level 0: 4 features
    dim3 grid(level > 0 ? (p->m + 1) / 2 : (p->m + 3) / 4, (unsigned)(level > 0 ? LN / 2 : 1));
    // few (node, feature) warps for the machine: split the channel loop over CG warp pairs
    int CG = (int)ctx->fs_channel_groups;               // 0: automatic, 1: off, 2 / 4 / 8: forced
    if (CG == 0) {
      const int64_t warps = (int64_t)grid.x * grid.y * kFsWarps, want = (int64_t)ctx->num_sms * 32;
      CG = warps * 8 <= want ? 8 : warps * 4 <= want ? 4 : warps * 2 <= want ? 2 : 1;
    }
    while (CG > 1 && CG > p->d) CG >>= 1;
    if (GBDTMO_FS_CG_OFF) CG = 1;                        // (A/B builds)
    if (CG > 1) {
      auto kc = CG > 4 ? (softmax ? k_find_split_c<true, 8> : k_find_split_c<false, 8>)
                       : (softmax ? k_find_split_c<true, 4> : k_find_split_c<false, 4>);
      GB_LAUNCH(kc, dim3((unsigned)LN, (unsigned)p->m), 64 * CG, 0, *p, level, nbins, scales, s, hist, cnt,
                level > 0 ? parent_hist : hist, level > 0 ? parent_cnt : cnt, keys, level < p->D - 1 ? 1 : 0);
      return GBDTMO_OK;
    }
    auto kern = softmax ? k_find_split_h<true, GBDTMO_FS_SOFTMAX_MINB> : channels(*p) <= 16 ? k_find_split_h<false, 4>
                                                                        : k_find_split_h<false, 3>;
    GB_LAUNCH(kern, grid, kFsWarps * 32, 0, *p, level, nbins, scales, s, hist, cnt, level > 0 ? parent_hist : hist,
              level > 0 ? parent_cnt : cnt, keys, level < p->D - 1 ? 1 : 0);
    return GBDTMO_OK;
  }
  dim3 grid(level > 0 ? (p->m + kFsWarps / 2 - 1) / (kFsWarps / 2) : (p->m + kFsWarps - 1) / kFsWarps,
            (unsigned)(level > 0 ? LN / 2 : 1));             // level > 0: sibling pairs (k_find_split)
  auto kern = softmax ? k_find_split<true> : k_find_split<false>;
  GB_LAUNCH(kern, grid, kFsWarps * 32, 0, *p, level, nbins, dflt, scales, s, hist, cnt,
            level > 0 ? parent_hist : hist, level > 0 ? parent_cnt : cnt, keys, level < p->D - 1 ? 1 : 0);
  return GBDTMO_OK;
}

static gbdtmo_status split_record_impl(Ctx* ctx, const gbdtmo_problem* p, int32_t level, const uint8_t* bins,
                                       const int32_t* dflt, const int32_t* q, const float* scales, void* state,
                                       const int64_t* hist, const int32_t* cnt, const int64_t* parent_hist,
                                       const int32_t* parent_cnt, const uint64_t* keys, int64_t* xchg,
                                       const PeerView& pv, uint64_t* keys_merged) {
  State s = state_view(*p, state);
  const int64_t LN = int64_t(1) << level;
  const unsigned cb = (unsigned)((channels(*p) + 1 + kRecChannels - 1) / kRecChannels);
  GB_LAUNCH(k_split_record, dim3((unsigned)LN, cb), 256, 0, *p, level, dflt, bins, q, s, hist, cnt,
            level > 0 ? parent_hist : hist, level > 0 ? parent_cnt : cnt, keys, scales, xchg, pv, keys_merged);
  GB_LAUNCH(k_record_gain, (unsigned)((LN + 7) / 8), 256, 0, *p, level, s, scales, xchg);
  // zero the record words of the unused slots of this buffer (levels < D-1) so SUM-merging is clean
  const int64_t used = LN * rec_words(*p), cap = bitmap_offset(*p);
  if (cap > used) GB_LAUNCH(k_zero_u64, 64, 256, 0, reinterpret_cast<uint64_t*>(xchg + used), cap - used);
  GB_LAUNCH(k_bitmap, ctx->num_sms * 4, 256, (size_t)(2 * LN * sizeof(int)), *p, level, bins, s,
            pv.world > 0 ? keys_merged : keys, xchg);
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_split_record(gbdtmo_ctx c, const gbdtmo_problem* p, int32_t level,
                                             const uint8_t* bins, const int32_t* dflt, const int32_t* q,
                                             const float* scales, void* state,
                                             const int64_t* hist, const int32_t* cnt,
                                             const int64_t* parent_hist, const int32_t* parent_cnt,
                                             const uint64_t* keys, int64_t* xchg) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(level >= 0 && level < p->D, "level out of range [0, D)");
  GB_CHECK_ARG(bins && state && hist && cnt && keys && xchg && scales, "null pointer");
  GB_CHECK_ARG(level == 0 || (parent_hist && parent_cnt), "parent histogram required for level > 0");
  PeerView none;
  memset(&none, 0, sizeof(none));
  return split_record_impl(ctx, p, level, bins, dflt, q, scales, state, hist, cnt, parent_hist, parent_cnt, keys, xchg,
                           none, nullptr);
}

extern "C" gbdtmo_status gbdtmo_split_record_peer(gbdtmo_ctx c, const gbdtmo_problem* p, int32_t level,
                                                  const uint8_t* bins, const int32_t* dflt, const int32_t* q,
                                                  const float* scales, void* state,
                                                  const int64_t* hist, const int32_t* cnt,
                                                  const int64_t* parent_hist, const int32_t* parent_cnt,
                                                  uint64_t* keys_merged) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(level >= 0 && level < p->D, "level out of range [0, D)");
  GB_CHECK_ARG(bins && state && hist && cnt && keys_merged && scales, "null pointer");
  GB_CHECK_ARG(level == 0 || (parent_hist && parent_cnt), "parent histogram required for level > 0");
  GB_CHECK_ARG(peer_ready(ctx, *p), "peer group not connected for this problem shape (gbdtmo_peer_open/_connect)");
  char* w = peer_own_window(ctx);
  const uint64_t* keys = reinterpret_cast<const uint64_t*>(w + peer_keys_off(*p, level));
  int64_t* xchg = reinterpret_cast<int64_t*>(w + peer_xchg_off(*p, level));
  return split_record_impl(ctx, p, level, bins, dflt, q, scales, state, hist, cnt, parent_hist, parent_cnt, keys, xchg,
                           peer_view(ctx), keys_merged);
}
