// hist.cu — (a)3: per-node histogram build (§3.3; Alg. 2's body is missing,
// PAPER.md:216-218, so the kernel is designed for sm_100a from the definition):
//
//   hist[slot][f][c][b] = sum_{i in node, bin(i,f) = b} q[i][c],   cnt[slot][f][b] = #{...}
//
// B200 design:
//  - persistent CTAs (1 per SM, ~200 KB shared memory) pull work items (row chunk x feature
//    tile x channel tile) from a device counter; the items of one chunk are adjacent so the
//    chunk's bin rows and q rows are read from HBM once and served from L2 to every tile;
//  - accumulators are two 16-bit limbs of the 31-bit fixed-point q, accumulated with native
//    32-bit shared atomics (ATOMS.ADD; float/64-bit shared atomics are CAS loops on sm_100a,
//    profiles/r01_microbench_atomics_*.txt), flushed exactly into the int64 global histogram;
//  - lanes = (row-in-group, channel): one warp instruction updates K channels of 32/K rows of
//    one feature, all on distinct banks (lo/hi limbs of alternating rows are swapped);
//  - each lane loads its row's q once and an 8-byte-aligned window (<= 32 bytes) of the row's
//    bins once, then walks the tile's k features (the paper's "bin packing", PAPER.md:239,
//    becomes one vector load of up to 32 bin ids);
//  - with tile-packed bins (gbdtmo_pack_bins: [tile][row][8 bytes]) that window is one aligned
//    8-byte load from a plane holding only this tile's bins: consecutive rows are adjacent, so
//    a warp's 32 rows touch 2-32 cache lines instead of 32-64 (ncu: the gathered window loads
//    were ~18% of the L1 data-pipe wavefronts, the pipe this kernel saturated);
//  - the inner loop is kept to PRMT + 2 IMAD + 2 ATOMS per (row pair, feature): rows past the
//    end of the item carry q = 0 and features past m sit in shared-memory slots that are never
//    flushed, so neither needs a test; the two limbs come from one PRMT each with per-lane
//    selectors; q is loaded one sub-batch ahead of use.
#include "common.cuh"
#include "hist_common.cuh"

namespace gbdtmo {

// K channels per lane group, KF features per tile (both compile-time).
// Shared layout, bin-major: limbs[b][j][2K] (two halves of K words: the lo and hi limbs),
// counts[KF][b], then a per-warp scratch of 32 rows x SW bin words.  Even rows of a warp
// instruction put lo in half 0 and hi in half 1, odd rows the other way round, so one
// instruction's 32 lanes always hit 32 distinct banks.
//
// A warp consumes its rows in batches of 32: lane l loads row l's id and bin window once,
// shifts it, counts it (CNT) and parks the bins in the scratch; then the K groups of
// 32/K rows are accumulated, lanes (row, channel) reading their bins back with one LDS and
// their q value from a batch-wide prefetch.
template <int KF>
__device__ __forceinline__ int dfl_of(const int (&dfl)[KF], int j) {   // dfl[j], j runtime
  int v = -1;
#pragma unroll
  for (int u = 0; u < KF; ++u) v = (u == j) ? dfl[u] : v;
  return v;
}

template <int K, int KF, bool SKIP, bool PACKED>
__global__ void __launch_bounds__(kHistThreads, kHistCtas)
k_hist_smem(gbdtmo_problem p, HistCfg hc, const uint8_t* __restrict__ bins, const uint8_t* __restrict__ packed,
            const int32_t* __restrict__ dflt, const int32_t* __restrict__ q,
            const int32_t* __restrict__ rows, int use_rows, State s,
            int64_t* __restrict__ hist, int32_t* __restrict__ cnt) {
  extern __shared__ __align__(16) uint32_t sm[];
  __shared__ int sh_item;
  constexpr int RPI = 32 / K;                  // rows per warp instruction
  constexpr int G = K;                         // groups per 32-row batch
#ifndef GBDTMO_HIST_NOCOUNT
#define GBDTMO_HIST_NOCOUNT 0      // (experiment only: drops the counts; results invalid)
#endif
#ifndef GBDTMO_HIST_SB
#define GBDTMO_HIST_SB 2          // q-prefetch groups: 2 keeps the batch loop spill-free at 64 registers (8 spilled: C5 -10%)
#endif
#ifndef GBDTMO_HIST_MATCHCNT
#define GBDTMO_HIST_MATCHCNT 0     // (A/B) 1: counts combined across lanes with MATCH.ANY
#endif
#ifndef GBDTMO_HIST_WDEPTH
#define GBDTMO_HIST_WDEPTH 1       // batches of bin-window prefetch (2: A/B for gathered levels)
#endif
#ifndef GBDTMO_HIST_SHFL
#define GBDTMO_HIST_SHFL 0         // (A/B) 1: phase 2 takes the bins by SHFL, no scratch round trip
#endif
  constexpr int SB = G < GBDTMO_HIST_SB ? G : GBDTMO_HIST_SB;   // groups per q-prefetch sub-batch
  constexpr int RS = KF * 2 * K;               // limb words per bin
  constexpr int NW = PACKED ? 1 : HistRow<KF>::NW, SW = PACKED ? 1 : HistRow<KF>::SW;
  static_assert(!PACKED || KF <= 8, "packed tiles hold <= 8 features");
  const int V = channels(p), B = p.B, m = p.m;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
  const int ri = lane / K, c = lane % K;
  const int tiles = hc.n_ft * hc.n_ct;
  const int nitems = s.misc[MISC_CHUNK_COUNT] * tiles;
  const int limb_words = B * RS;
  constexpr bool LCNT = GBDTMO_HIST_LCNT && K == 16 && KF <= 8;
  const int cnt_words = LCNT ? ((B + 1) >> 1) * 32 : B * KF;
  uint64_t* scratch = reinterpret_cast<uint64_t*>(sm + limb_words + cnt_words + ((limb_words + cnt_words) & 1)) +
                      (size_t)warp * 32 * SW;
  const int slotA = c + ((ri & 1) ? K : 0), slotB = slotA ^ K;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(sm);
  const uint32_t aA = sbase + 4u * slotA, aB = sbase + 4u * slotB;
  const uint32_t acnt = sbase + 4u * limb_words;
  const int64_t ld = p.ld_bins;
  // limb selectors for PRMT(q, sel, 0): lo = bytes 0-1 zero-extended (0x4410), hi = bytes 2-3
  // sign-extended (0xBB32); even rows add (lo, hi) at (slotA, slotB), odd rows (hi, lo)
  const uint32_t selA = (ri & 1) ? 0xBB32u : 0x4410u, selB = (ri & 1) ? 0x4410u : 0xBB32u;
  // lane counts (LCNT): lane (ri, c < 2 KF) counts feature cj of the earlier (c < KF) or later
  // row pair of every two, into column 16 ri + c of the [bin/2][32] table (bank = column)
  const int cj = c < KF ? c : c - KF;
  const uint32_t acol = sbase + 4u * (limb_words + 16 * ri + c);
  const uint32_t cshift = 8u * cj;

  for (;;) {
    if (threadIdx.x == 0) sh_item = atomicAdd(&s.misc[MISC_WORK_COUNTER], 1);
    __syncthreads();
    const int item = sh_item;
    if (item >= nitems) break;
    const int chunk = item / tiles, tile = item - chunk * tiles;
    const int ft = tile / hc.n_ct, ct = tile - ft * hc.n_ct;
    const int4 ch = s.chunks[chunk];
    const int f0 = ft * KF;
    const int kk = min(KF, m - f0);
    const int c0 = ct * K;
    const bool do_cnt = (ct == 0) && !hc.no_cnt;
    int dfl[KF];                                   // default (skipped) bin per feature, -1: none
#pragma unroll
    for (int j = 0; j < KF; ++j) dfl[j] = (SKIP && j < kk) ? __ldg(&dflt[f0 + j]) : -1;

    const int words = limb_words + cnt_words;
    for (int i = threadIdx.x * 4; i < limb_words; i += blockDim.x * 4)
      *reinterpret_cast<uint4*>(&sm[i]) = make_uint4(0, 0, 0, 0);
    for (int i = limb_words + threadIdx.x; i < words; i += blockDim.x) sm[i] = 0;
    __syncthreads();

    const int beg = ch.y, end = ch.z;
    const int o = PACKED ? 0 : f0 & 7;
    const uint8_t* bbase = PACKED ? packed + ((int64_t)(ft / kPackGroup) * p.n * kPackGroup + ft % kPackGroup) * 8
                                  : bins + (f0 & ~7);
    const int64_t rstride = PACKED ? 8 * kPackGroup : ld;
    const bool chan_on = (c0 + c) < V;
    const int32_t* qc = q + c0 + c;
    // cross-batch pipeline: row ids two batches ahead, bin windows one batch ahead, q one
    // sub-batch ahead
    const int bstep = nwarps * 32;
    auto load_rid = [&](int pos) -> int { return pos < end ? (use_rows ? __ldg(&rows[pos]) : pos) : -1; };
    auto load_win = [&](int rr, uint64_t (&w)[NW]) {
      if (rr >= 0) {
        const uint64_t* wp = reinterpret_cast<const uint64_t*>(bbase + (int64_t)rr * rstride);
#pragma unroll
        for (int i = 0; i < NW; ++i) w[i] = __ldg(wp + i);
      } else {
#pragma unroll
        for (int i = 0; i < NW; ++i) w[i] = 0;
      }
    };
    auto load_q = [&](int rid, int t0, int (&qv)[SB]) {
#pragma unroll
      for (int t = 0; t < SB; ++t) {
        const int rr = __shfl_sync(0xffffffffu, rid, (t0 + t) * RPI + ri);
        qv[t] = (rr >= 0 && chan_on) ? __ldg(qc + (int64_t)rr * V) : 0;
      }
    };
    int r_cur = load_rid(beg + warp * 32 + lane);
    int r_nxt = load_rid(beg + warp * 32 + bstep + lane);
#if GBDTMO_HIST_WDEPTH == 2
    int r_n2 = load_rid(beg + warp * 32 + 2 * bstep + lane);
    uint64_t w_n1[NW];
    load_win(r_nxt, w_n1);
#endif
    uint64_t w_cur[NW];
    load_win(r_cur, w_cur);
    int qv[SB];
    load_q(r_cur, 0, qv);
    for (int b0 = beg + warp * 32; b0 < end; b0 += bstep) {
#if GBDTMO_HIST_WDEPTH == 2
      // (gathered deep levels) bin windows two batches ahead, row ids three
      const int r_n3 = load_rid(b0 + 3 * bstep + lane);
      uint64_t w_n2[NW];
      load_win(r_n2, w_n2);
#else
      const int r_nn = load_rid(b0 + 2 * bstep + lane);
      uint64_t w_nxt[NW];
      load_win(r_nxt, w_nxt);
#endif
      // ---- phase 1: lane l owns row b0 + l (invalid rows: window 0, q 0, not counted)
      const int r = r_cur;
      uint64_t sw[SW];
#pragma unroll
      for (int i = 0; i < SW; ++i) sw[i] = 0;
      if (r >= 0) {
        shift_window<NW, SW>(w_cur, o, sw);
        if (!PACKED && kk < KF) {                // last tile: bytes past feature m-1 -> bin 0
#pragma unroll
          for (int i = 0; i < SW; ++i) {
            const int keep = kk - 8 * i;           // bytes of word i that hold features < m
            sw[i] = keep >= 8 ? sw[i] : keep <= 0 ? 0ull : (sw[i] & ((1ull << (8 * keep)) - 1));
          }
        }
        if (!LCNT && do_cnt && !GBDTMO_HIST_NOCOUNT && !GBDTMO_HIST_MATCHCNT) {
#pragma unroll
          for (int j = 0; j < KF; ++j) {         // features j >= kk land in slots never flushed
            const uint32_t bin = byte_of<SW>(sw, j);
            if (!SKIP || (int)bin != dfl[j]) red_shared_add(acnt + 4u * (j * B + bin), 1u);  // counts[j][b]
          }
        }
      }
      if (GBDTMO_HIST_MATCHCNT && !LCNT && do_cnt && !GBDTMO_HIST_NOCOUNT) {
        // (A/B) lanes with equal bins combine first: one atomic per distinct bin (MATCH.ANY)
#pragma unroll
        for (int j = 0; j < KF; ++j) {
          const uint32_t bin = byte_of<SW>(sw, j);
          const bool on = r >= 0 && (!SKIP || (int)bin != dfl[j]);
          const unsigned peers = __match_any_sync(0xffffffffu, on ? bin : 0x100u + lane);
          if (on && lane == __ffs(peers) - 1) red_shared_add(acnt + 4u * (j * B + bin), (uint32_t)__popc(peers));
        }
      }
#pragma unroll
      for (int i = 0; i < SW; ++i) scratch[lane * SW + i] = sw[i];
      __syncwarp();
      // ---- phase 2: groups of RPI rows x K channels
      const bool cnt_on = LCNT && do_cnt && c < 2 * KF && cj < kk;
      uint64_t bprev = 0;
#pragma unroll
      for (int t0 = 0; t0 < G; t0 += SB) {
        int qn[SB];
        if (t0 + SB < G) load_q(r, t0 + SB, qn);
        else load_q(r_nxt, 0, qn);
#pragma unroll
        for (int t = 0; t < SB; ++t) {
          const int i = (t0 + t) * RPI + ri;
          uint64_t bw[SW];
          if (GBDTMO_HIST_SHFL && SW == 1) {       // (A/B) bins by shuffle instead of the scratch
            const uint32_t w0 = __shfl_sync(0xffffffffu, (uint32_t)sw[0], i);
            const uint32_t w1 = KF > 4 ? __shfl_sync(0xffffffffu, (uint32_t)(sw[0] >> 32), i) : 0u;
            bw[0] = ((uint64_t)w1 << 32) | w0;
          } else {
#pragma unroll
            for (int u = 0; u < SW; ++u) bw[u] = scratch[i * SW + u];
          }
          if (LCNT) {
            if ((t0 + t) & 1) {
              const uint64_t w = c < KF ? bprev : bw[0];
              const int row = c < KF ? i - 2 : i;
              const uint32_t bin = (uint32_t)(w >> cshift) & 0xFFu;
              if (cnt_on && b0 + row < end && (!SKIP || (int)bin != dfl_of(dfl, cj)))
                red_shared_add(acol + (bin >> 1) * 128u, 1u << ((bin & 1) << 4));
            }
            bprev = bw[0];
          }
          const uint32_t va = prmt_sx((uint32_t)qv[t], selA);
          const uint32_t vb = prmt_sx((uint32_t)qv[t], selB);
#pragma unroll
          for (int j = 0; j < KF; ++j) {
            const uint32_t bin = byte_of<SW>(bw, j);
            if (!SKIP || (int)bin != dfl[j]) {
              red_shared_add(aA + bin * (4u * RS) + 8u * K * j, va);
              red_shared_add(aB + bin * (4u * RS) + 8u * K * j, vb);
            }
          }
        }
#pragma unroll
        for (int t = 0; t < SB; ++t) qv[t] = qn[t];
      }
      __syncwarp();
#if GBDTMO_HIST_WDEPTH == 2
      r_cur = r_nxt;
      r_nxt = r_n2;
      r_n2 = r_n3;
#pragma unroll
      for (int i = 0; i < NW; ++i) { w_cur[i] = w_n1[i]; w_n1[i] = w_n2[i]; }
#else
      r_cur = r_nxt;
      r_nxt = r_nn;
#pragma unroll
      for (int i = 0; i < NW; ++i) w_cur[i] = w_nxt[i];
#endif
    }
    __syncthreads();

    // flush: exact int64 = hi * 2^16 + lo into the node histogram (global REDG.ADD.64, or plain
    // stores of every entry when this item is the node's only writer: no zeroing, no read-back)
    const int64_t slot = ch.x;
    const bool sole = ch.w != 0;
    const int64_t gbase = (slot * m + f0) * (int64_t)B;        // (slot, f0, bin 0)
    if (K == 16) {
      // Warp-transposed flush: the limb records are bin-major with bank = slot, the global
      // histogram is bin-minor.  A warp takes (feature j, 32 bins): reads them with lanes = slots
      // (conflict-free), writes each bin's 32 slots back XOR-swizzled by the bin, reads them again
      // with lanes = bins (conflict-free), and stores 32 consecutive bins per channel (2 lines per
      // instruction instead of 32).
      const int nblk = (B + 31) >> 5;
      for (int task = warp; task < kk * nblk; task += nwarps) {
        const int j = task / nblk, bb = (task - j * nblk) << 5;
        uint32_t* rec = sm + j * 2 * K;                        // + b * RS + slot
#pragma unroll
        for (int h = 0; h < 32; h += 16) {
          uint32_t v[16];
#pragma unroll
          for (int u = 0; u < 16; ++u) v[u] = (bb + h + u < B) ? rec[(bb + h + u) * RS + lane] : 0u;
          __syncwarp();
#pragma unroll
          for (int u = 0; u < 16; ++u)
            if (bb + h + u < B) rec[(bb + h + u) * RS + (lane ^ (h + u))] = v[u];
        }
        __syncwarp();
        const int b = bb + lane;
        if (b < B) {
          const uint32_t* rb = rec + b * RS;
          int64_t* dst = &hist[((slot * m + f0 + j) * V + c0) * (int64_t)B + b];
#pragma unroll 4
          for (int cc = 0; cc < K; ++cc) {
            if (c0 + cc >= V) break;
            const uint32_t los = rb[cc ^ lane], his = rb[(K + cc) ^ lane];
            const long long v = (long long)(int32_t)his * 65536LL + (long long)los;
            if (sole) dst[(int64_t)cc * B] = v;
            else if (v != 0) atomicAdd(reinterpret_cast<unsigned long long*>(dst + (int64_t)cc * B), (unsigned long long)v);
          }
        }
        __syncwarp();
      }
    } else {
    const int total = kk * B * K;
    for (int e = threadIdx.x; e < total; e += blockDim.x) {
      const int cc = e % K, jb = e / K;                        // jb = j * B + b
      if (c0 + cc >= V) continue;
      const int j = jb / B, b = jb - j * B;
      const uint32_t* rowp = sm + b * RS + j * 2 * K;
      const uint32_t los = rowp[cc], his = rowp[K + cc];
      const long long v = (long long)(int32_t)his * 65536LL + (long long)los;
      int64_t* dst = &hist[((slot * m + f0 + j) * V + c0 + cc) * B + b];   // channel-major [f][c][b]
      if (sole) *dst = v;
      else if (v != 0) atomicAdd(reinterpret_cast<unsigned long long*>(dst), (unsigned long long)v);
    }
    }
    if (do_cnt) {
      for (int e = threadIdx.x; e < kk * B; e += blockDim.x) {
        uint32_t nv;                                               // count of (feature j, bin b), e = j * B + b
        if (LCNT) {
          const int j = e / B, b = e - j * B;
          const uint32_t* cw = sm + limb_words + (b >> 1) * 32;
          const int sh = 16 * (b & 1);
          nv = ((cw[j] >> sh) & 0xFFFFu) + ((cw[j + KF] >> sh) & 0xFFFFu) + ((cw[16 + j] >> sh) & 0xFFFFu) +
               ((cw[16 + j + KF] >> sh) & 0xFFFFu);
        } else {
          nv = sm[limb_words + e];                                 // counts[j][b]
        }
        if (sole) cnt[gbase + e] = (int32_t)nv;
        else if (nv) atomicAdd(&cnt[gbase + e], (int32_t)nv);
      }
    }
    __syncthreads();
  }
}

// Global-atomic variant (the paper's "global memory approach"; for small nodes,
// where the shared-memory variant's per-item zero/flush of ~200 KB tiles dominates): one warp
// per row of the level's small BUILD nodes, lanes over features, one REDG.ADD.64 per
// (row, feature, channel) straight into the node's (zeroed) int64 histogram.
template <bool SKIP>
__global__ void __launch_bounds__(256)
k_hist_gmem(gbdtmo_problem p, const uint8_t* __restrict__ bins, const int32_t* __restrict__ dflt,
            const int32_t* __restrict__ q, const int32_t* __restrict__ rows, int use_rows, State s,
            int64_t* __restrict__ hist, int32_t* __restrict__ cnt) {
  __shared__ int4 gn[512];
  const int ng = s.misc[MISC_GNODE_COUNT];
  const int total = s.misc[MISC_GNODE_ROWS];
  if (ng == 0) return;
  const int V = channels(p), B = p.B, m = p.m;
  const int lane = threadIdx.x & 31;
  const int64_t wid = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int base = 0; base < ng; base += 512) {        // node lists longer than 512: in slices
    const int cnt_here = min(512, ng - base);
    __syncthreads();
    for (int i = threadIdx.x; i < cnt_here; i += blockDim.x) gn[i] = s.gnodes[base + i];
    __syncthreads();
    const int r_lo = gn[0].w, r_hi = (base + cnt_here < ng) ? s.gnodes[base + cnt_here].w : total;
    for (int64_t ri = r_lo + wid; ri < r_hi; ri += nwarps) {
      int lo = 0, hi = cnt_here - 1;                  // last node with prefix <= ri
      while (lo < hi) { const int mid = (lo + hi + 1) >> 1; if (gn[mid].w <= ri) lo = mid; else hi = mid - 1; }
      const int4 nd = gn[lo];
      const int pos = nd.y + (int)(ri - nd.w);
      const int r = use_rows ? __ldg(&rows[pos]) : pos;
      const uint8_t* br = bins + (int64_t)r * p.ld_bins;
      const int32_t* qr = q + (int64_t)r * V;
      const int64_t sbase = (int64_t)nd.x * m;
      for (int f = lane; f < m; f += 32) {
        const int b = br[f];
        if (SKIP && b == __ldg(&dflt[f])) continue;
        atomicAdd(&cnt[(sbase + f) * B + b], 1);
        int64_t* hb = hist + (sbase + f) * V * B + b;
        for (int c = 0; c < V; ++c) {
          const int v = __ldg(&qr[c]);
          if (v) atomicAdd(reinterpret_cast<unsigned long long*>(hb + (int64_t)c * B), (unsigned long long)(long long)v);
        }
      }
    }
  }
}

// Zero the histogram slots of the level's BUILD nodes (the flush accumulates atomically).  With
// cached root counts (level 0), the root's count slot is filled from the cache instead (the
// histogram kernels then skip the count atomics), whatever the root's build mode.
__global__ void k_zero_build(gbdtmo_problem p, int level, State s, int64_t* __restrict__ hist,
                             int32_t* __restrict__ cnt, const int32_t* __restrict__ root_cnt) {
  const int64_t slot = blockIdx.y;
  const int64_t h = (int64_t(1) << level) - 1 + slot;
  if (root_cnt) {
    const int64_t cw = (int64_t)p.m * p.B;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cw; i += (int64_t)gridDim.x * blockDim.x)
      cnt[i] = root_cnt[i];
  }
  if (s.node_mode[h] != MODE_BUILD) return;
  const int64_t V = channels(p);
  const int64_t hw = (int64_t)p.m * p.B * V;           // int64 words per slot
  const int64_t cw = (int64_t)p.m * p.B;               // int32 words per slot
  int64_t* hb = hist + hist_index(p, level, slot) * hw;
  int32_t* cb = cnt + hist_index(p, level, slot) * cw;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  // hw is even when V is even; handle generally with a scalar tail
  const int64_t hv = hw / 2;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < hv; i += stride)
    reinterpret_cast<longlong2*>(hb)[i] = make_longlong2(0, 0);
  for (int64_t i = 2 * hv + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < hw; i += stride) hb[i] = 0;
  if (!root_cnt)
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cw; i += stride) cb[i] = 0;
}

template <int K, int KF, bool SKIP, bool PACKED>
static gbdtmo_status launch_hist_kfs(Ctx* ctx, const gbdtmo_problem& p, const HistCfg& hc, const uint8_t* bins,
                                     const uint8_t* packed, const int32_t* dflt, const int32_t* q,
                                     const int32_t* rows, int use_rows, const State& s, int64_t* hist, int32_t* cnt) {
  static unsigned long long attr_mask = 0;
  smem_optin_once(ctx, k_hist_smem<K, KF, SKIP, PACKED>, attr_mask, ctx->max_smem_optin - 1024);
  GB_LAUNCH((k_hist_smem<K, KF, SKIP, PACKED>), ctx->num_sms * kHistCtas, kHistThreads, hc.smem, p, hc, bins, packed, dflt, q,
            rows, use_rows, s, hist, cnt);
  return GBDTMO_OK;
}

template <int K, int KF>
static gbdtmo_status launch_hist_kf(Ctx* ctx, const gbdtmo_problem& p, const HistCfg& hc, const uint8_t* bins,
                                    const uint8_t* packed, const int32_t* dflt, const int32_t* q,
                                    const int32_t* rows, int use_rows, const State& s, int64_t* hist, int32_t* cnt) {
  if constexpr (KF <= 8) {
    if (packed) {
      if (dflt) return launch_hist_kfs<K, KF, true, true>(ctx, p, hc, bins, packed, dflt, q, rows, use_rows, s, hist, cnt);
      return launch_hist_kfs<K, KF, false, true>(ctx, p, hc, bins, packed, dflt, q, rows, use_rows, s, hist, cnt);
    }
  }
  if (dflt) return launch_hist_kfs<K, KF, true, false>(ctx, p, hc, bins, nullptr, dflt, q, rows, use_rows, s, hist, cnt);
  return launch_hist_kfs<K, KF, false, false>(ctx, p, hc, bins, nullptr, dflt, q, rows, use_rows, s, hist, cnt);
}

template <int K>
static gbdtmo_status launch_hist(Ctx* ctx, const gbdtmo_problem& p, const HistCfg& hc, const uint8_t* bins,
                                 const uint8_t* packed, const int32_t* dflt, const int32_t* q, const int32_t* rows,
                                 int use_rows, const State& s, int64_t* hist, int32_t* cnt) {
  switch (hc.k) {
    case 24: return launch_hist_kf<K, 24>(ctx, p, hc, bins, packed, dflt, q, rows, use_rows, s, hist, cnt);
    case 16: return launch_hist_kf<K, 16>(ctx, p, hc, bins, packed, dflt, q, rows, use_rows, s, hist, cnt);
    case 12: return launch_hist_kf<K, 12>(ctx, p, hc, bins, packed, dflt, q, rows, use_rows, s, hist, cnt);
    case 8: return launch_hist_kf<K, 8>(ctx, p, hc, bins, packed, dflt, q, rows, use_rows, s, hist, cnt);
    case 6: return launch_hist_kf<K, 6>(ctx, p, hc, bins, packed, dflt, q, rows, use_rows, s, hist, cnt);
    case 4: return launch_hist_kf<K, 4>(ctx, p, hc, bins, packed, dflt, q, rows, use_rows, s, hist, cnt);
    case 3: return launch_hist_kf<K, 3>(ctx, p, hc, bins, packed, dflt, q, rows, use_rows, s, hist, cnt);
    case 2: return launch_hist_kf<K, 2>(ctx, p, hc, bins, packed, dflt, q, rows, use_rows, s, hist, cnt);
    default: return launch_hist_kf<K, 1>(ctx, p, hc, bins, packed, dflt, q, rows, use_rows, s, hist, cnt);
  }
}

// Tile-packed copy of the bins, groups of kPackGroup tiles per row:
//   packed[((t / G) * n + i) * G + t % G] (8-byte words) = bins of features [k t, k t + k) of row i
// Threads walk (row, tile) with the tile fastest: a warp reads one row's bins contiguously and
// writes its 32-byte groups contiguously.  Once per dataset (like gbdtmo_bin).
__global__ void k_pack_bins(gbdtmo_problem p, int k, int n_ft, const uint8_t* __restrict__ bins,
                            uint64_t* __restrict__ packed) {
  const int n_g = (n_ft + kPackGroup - 1) / kPackGroup;
  const int64_t total = p.n * (int64_t)n_g * kPackGroup;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += stride) {
    const int64_t i = e / (n_g * kPackGroup);
    const int t = (int)(e - i * n_g * kPackGroup);
    const uint8_t* src = bins + i * p.ld_bins + (int64_t)t * k;
    const int kk = min(k, p.m - t * k);
    uint64_t v = 0;
    for (int j = 0; j < kk; ++j) v |= (uint64_t)__ldg(src + j) << (8 * j);
    packed[((int64_t)(t / kPackGroup) * p.n + i) * kPackGroup + t % kPackGroup] = v;
  }
}

gbdtmo_status build_hist_impl(Ctx* ctx, const gbdtmo_problem* p, int32_t level, const uint8_t* bins,
                              const uint8_t* packed, const int32_t* dflt, const int32_t* q, void* state,
                              int64_t* hist, int32_t* cnt) {
  State s = state_view(*p, state);
  HistCfg hc = hist_config(*p);
  const int64_t LN = int64_t(1) << level;
  // cached root counts: level 0, a variant that can skip its counts, and no global-atomic root
  const bool tma = ctx->hist_kernel == 2 && !dflt && hist_tma_supported(*p, bins);
  const int32_t* root_cnt = (level == 0 && ctx->root_cnt && !tma && ctx->gmem_max_rows < p->n) ? ctx->root_cnt : nullptr;
  hc.no_cnt = root_cnt ? 1 : 0;
  int gx = (int)(2 * ctx->num_sms / (LN > 1 ? LN / 2 : 1));
  if (gx < 8) gx = 8;
  GB_LAUNCH(k_zero_build, dim3(gx, (unsigned)LN), 256, 0, *p, level, s, hist, cnt, root_cnt);
  const int32_t* rows = (level & 1) ? s.rows1 : s.rows0;
  const int use_rows = level > 0;
  gbdtmo_status st;
  if (ctx->hist_kernel == 1 && !dflt) {
    st = launch_hist_diag(ctx, *p, bins, q, rows, use_rows, s, hist, cnt, root_cnt != nullptr);
  } else if (tma) {
    st = launch_hist_tma(ctx, *p, bins, q, rows, use_rows, s, hist, cnt);
  } else switch (hc.K) {
    case 4: st = launch_hist<4>(ctx, *p, hc, bins, packed, dflt, q, rows, use_rows, s, hist, cnt); break;
    case 8: st = launch_hist<8>(ctx, *p, hc, bins, packed, dflt, q, rows, use_rows, s, hist, cnt); break;
    default: st = launch_hist<16>(ctx, *p, hc, bins, packed, dflt, q, rows, use_rows, s, hist, cnt); break;
  }
  if (st != GBDTMO_OK || ctx->gmem_max_rows <= 0) return st;
  if (dflt) GB_LAUNCH(k_hist_gmem<true>, ctx->num_sms * 8, 256, 0, *p, bins, dflt, q, rows, use_rows, s, hist, cnt);
  else GB_LAUNCH(k_hist_gmem<false>, ctx->num_sms * 8, 256, 0, *p, bins, dflt, q, rows, use_rows, s, hist, cnt);
  return GBDTMO_OK;
}

}  // namespace gbdtmo

using namespace gbdtmo;

extern "C" gbdtmo_status gbdtmo_build_hist(gbdtmo_ctx c, const gbdtmo_problem* p, int32_t level,
                                           const uint8_t* bins, const int32_t* dflt, const int32_t* q, void* state,
                                           int64_t* hist, int32_t* cnt) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(level >= 0 && level < p->D, "level out of range [0, D)");
  GB_CHECK_ARG(bins && q && state && hist && cnt, "null pointer");
  GB_CHECK_ARG(((uintptr_t)bins & 7) == 0, "bins must be 8-byte aligned");
  return build_hist_impl(ctx, p, level, bins, nullptr, dflt, q, state, hist, cnt);
}

extern "C" gbdtmo_status gbdtmo_build_hist_packed(gbdtmo_ctx c, const gbdtmo_problem* p, int32_t level,
                                                  const uint8_t* bins, const uint8_t* packed, const int32_t* dflt,
                                                  const int32_t* q, void* state, int64_t* hist, int32_t* cnt) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(level >= 0 && level < p->D, "level out of range [0, D)");
  GB_CHECK_ARG(bins && packed && q && state && hist && cnt, "null pointer");
  GB_CHECK_ARG(((uintptr_t)bins & 7) == 0 && ((uintptr_t)packed & 7) == 0, "bins / packed must be 8-byte aligned");
  GB_CHECK_ARG(hist_packable(*p), "feature tiles wider than 8 features: no packed layout (gbdtmo_packed_bins_bytes = 0)");
  return build_hist_impl(ctx, p, level, bins, packed, dflt, q, state, hist, cnt);
}

extern "C" size_t gbdtmo_packed_bins_bytes(const gbdtmo_problem* p) {
  if (check_problem(p) || !hist_packable(*p)) return 0;
  const size_t groups = (size_t)(hist_config(*p).n_ft + kPackGroup - 1) / kPackGroup;
  return groups * (size_t)p->n * 8 * kPackGroup;
}

extern "C" gbdtmo_status gbdtmo_pack_bins(gbdtmo_ctx c, const gbdtmo_problem* p, const uint8_t* bins,
                                          uint8_t* packed) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(bins && packed, "null pointer");
  GB_CHECK_ARG(((uintptr_t)packed & 7) == 0, "packed must be 8-byte aligned");
  GB_CHECK_ARG(hist_packable(*p), "feature tiles wider than 8 features: no packed layout (gbdtmo_packed_bins_bytes = 0)");
  const HistCfg hc = hist_config(*p);
  GB_LAUNCH(k_pack_bins, ctx->num_sms * 8, 256, 0, *p, hc.k, hc.n_ft, bins, reinterpret_cast<uint64_t*>(packed));
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_set_root_counts(gbdtmo_ctx c, const int32_t* root_cnt) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  ctx->root_cnt = root_cnt;
  return GBDTMO_OK;
}
