// hist_diag.cu — (a)3 histogram build, "diagonal" shared-memory variant.
//
// Same definition, accumulator and work items as k_hist_smem (hist.cu); what differs is the
// lane mapping, chosen so that channel counts that are not a multiple of 16 (C2: V = 20, S5:
// V = 10) waste no lanes and no instruction ever has a bank conflict, whatever the bins:
//  - channel tiles of K = 4, eight rows per warp instruction (lanes = (row slot ri, channel c));
//  - shared layout limbs[b][s][4] with s = 2j + limb ("slots": lo and hi limb of feature j),
//    KF a multiple of 4 so a bin record is a multiple of 32 words: the bank of (b, s, c) is
//    (4s + c) mod 32, independent of the bin;
//  - instruction t makes row slot ri add to slot (t + ri) mod 2KF, so the eight rows of one
//    instruction always address eight different 4-bank groups (a diagonal through the slots);
//  - each row's KF bins are rotated in registers once per group (a ring of KF bytes with its
//    first word duplicated), so every instruction extracts its bin at a compile-time byte.
#include "common.cuh"
#include "hist_common.cuh"

namespace gbdtmo {

constexpr int kDiagK = 4;

HistCfg hist_config_diag(const gbdtmo_problem& p) {
  HistCfg c;
  const int V = channels(p);
  c.K = kDiagK;
  c.n_ct = (V + kDiagK - 1) / kDiagK;
  const int per_feature = p.B * (2 * kDiagK + 1) * 4;
  const int allowed[5] = {20, 16, 12, 8, 4};
  int k = 4;
  for (int i = 0; i < 5; ++i) {
    const int kk = allowed[i];
    const int need = kk * per_feature + kHistWarps * 32 * 4 * (kk / 4 + 1);
    if ((kk <= p.m || kk == 4) && need <= kHistTileBudget) { k = kk; break; }
  }
  c.k = k;
  c.n_ft = (p.m + k - 1) / k;
  c.smem = k * per_feature + kHistWarps * 32 * 4 * (k / 4 + 1);
  c.no_cnt = 0;
  return c;
}

// Instruction t of a group, unrolled by recursion so the slot offset 16 t is an immediate of the
// atomic (per instruction: one PRMT for the bin, one IMAD for the address, the ATOMS).
template <int T, int S, int R, int RS, int WD>
struct DiagStep {
  static __device__ __forceinline__ void run(const uint32_t (&we)[WD], const uint32_t (&wo)[WD], uint32_t lane_addr,
                                             int ri, uint32_t va, uint32_t vb) {
    constexpr int k = T >> 1;
    const uint32_t word = (T & 1) ? wo[k >> 2] : we[k >> 2];
    const uint32_t bin = __byte_perm(word, 0u, 0x4440u | (uint32_t)(k & 3));
    uint32_t a = bin * (4u * RS) + lane_addr;
    if (T >= S - (R - 1) && T + ri >= S) a -= 16u * S;     // slot wraps to the ring's start
    asm volatile("red.shared.add.u32 [%0+%2], %1;" ::"r"(a), "r"((T & 1) ? vb : va), "n"(16 * T) : "memory");
    DiagStep<T + 1, S, R, RS, WD>::run(we, wo, lane_addr, ri, va, vb);
  }
};
template <int S, int R, int RS, int WD>
struct DiagStep<S, S, R, RS, WD> {
  static __device__ __forceinline__ void run(const uint32_t (&)[WD], const uint32_t (&)[WD], uint32_t, int, uint32_t,
                                             uint32_t) {}
};

template <int KF>
__global__ void __launch_bounds__(kHistThreads, kHistCtas)
k_hist_diag(gbdtmo_problem p, HistCfg hc, const uint8_t* __restrict__ bins, const int32_t* __restrict__ q,
            const int32_t* __restrict__ rows, int use_rows, State s, int64_t* __restrict__ hist,
            int32_t* __restrict__ cnt) {
  extern __shared__ __align__(16) uint32_t sm[];
  __shared__ int sh_item;
  constexpr int K = kDiagK;
  constexpr int R = 32 / K;                    // rows per warp instruction
  constexpr int S = 2 * KF;                    // slots per row (lo, hi per feature)
  constexpr int RS = KF * 2 * K;               // limb words per bin (a multiple of 32)
  constexpr int WD = KF / 4;                   // u32 words of a row's KF bins
  constexpr int SWD = WD + 1;                  // + the first word again (ring)
  constexpr int NW = HistRow<KF>::NW, SW = HistRow<KF>::SW;
  static_assert(KF % 4 == 0 && RS % 32 == 0, "diagonal layout needs KF % 4 == 0");
  const int V = channels(p), B = p.B, m = p.m;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
  const int ri = lane / K, c = lane % K;
  const int tiles = hc.n_ft * hc.n_ct;
  const int nitems = s.misc[MISC_CHUNK_COUNT] * tiles;
  const int limb_words = B * RS;
  const int cnt_words = B * KF;
  uint32_t* scratch = sm + limb_words + cnt_words + (size_t)warp * 32 * SWD;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(sm);
  const uint32_t lane_addr = (uint32_t)__cvta_generic_to_shared(sm) + 4u * (uint32_t)(ri * K + c);
  const uint32_t acnt = sbase + 4u * limb_words;
  const int64_t ld = p.ld_bins;
  const int re = ri >> 1, ro = (ri >> 1) + (ri & 1);   // ring rotations for even / odd instructions

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
    for (int i = threadIdx.x * 4; i < limb_words; i += blockDim.x * 4)
      *reinterpret_cast<uint4*>(&sm[i]) = make_uint4(0, 0, 0, 0);
    for (int i = limb_words + threadIdx.x; i < limb_words + cnt_words; i += blockDim.x) sm[i] = 0;
    __syncthreads();

    const int beg = ch.y, end = ch.z;
    const int o = f0 & 7;
    const uint8_t* bbase = bins + (f0 & ~7);
    const bool chan_on = (c0 + c) < V;
    const int32_t* qc = q + c0 + c;
    // bytes of the window past the tile's last feature are zeroed (they then only touch
    // accumulators the flush ignores, and never index past the bins)
    uint32_t kmask[WD];
#pragma unroll
    for (int w = 0; w < WD; ++w)
      kmask[w] = kk >= 4 * w + 4 ? 0xFFFFFFFFu : (kk <= 4 * w ? 0u : ((1u << (8 * (kk - 4 * w))) - 1u));
    const int bstep = nwarps * 32;
    auto load_rid = [&](int pos) -> int { return pos < end ? (use_rows ? __ldg(&rows[pos]) : pos) : -1; };
    auto load_win = [&](int rr, uint64_t (&w)[NW]) {
      if (rr >= 0) {
        const uint64_t* wp = reinterpret_cast<const uint64_t*>(bbase + (int64_t)rr * ld);
#pragma unroll
        for (int i = 0; i < NW; ++i) w[i] = __ldg(wp + i);
      } else {
#pragma unroll
        for (int i = 0; i < NW; ++i) w[i] = 0;
      }
    };
    int r_cur = load_rid(beg + warp * 32 + lane);
    int r_nxt = load_rid(beg + warp * 32 + bstep + lane);
    uint64_t w_cur[NW];
    load_win(r_cur, w_cur);
    for (int b0 = beg + warp * 32; b0 < end; b0 += bstep) {
      const int r_nn = load_rid(b0 + 2 * bstep + lane);
      uint64_t w_nxt[NW];
      load_win(r_nxt, w_nxt);
      // ---- phase 1: lane l owns row b0 + l: counts, and its bins as a KF-byte ring in scratch
      const int r = r_cur;
      uint64_t sw[SW];
#pragma unroll
      for (int i = 0; i < SW; ++i) sw[i] = 0;
      if (r >= 0) {
        shift_window<NW, SW>(w_cur, o, sw);
        if (do_cnt) {
#pragma unroll
          for (int j = 0; j < KF; ++j)
            if (j < kk) red_shared_add(acnt + 4u * (j * B + byte_of<SW>(sw, j)), 1u);
        }
      }
      {
        uint32_t w32[SWD];
#pragma unroll
        for (int w = 0; w < WD; ++w)
          w32[w] = ((w & 1) ? (uint32_t)(sw[w >> 1] >> 32) : (uint32_t)sw[w >> 1]) & kmask[w];
        w32[WD] = w32[0];
#pragma unroll
        for (int w = 0; w < SWD; ++w) scratch[lane * SWD + w] = w32[w];
      }
      // q of the batch's rows for this lane's channel, one load per group, issued together
      constexpr int G = 32 / R;
      int qv[G];
#pragma unroll
      for (int g = 0; g < G; ++g) {
        const int rr = __shfl_sync(0xffffffffu, r, g * R + ri);
        qv[g] = (rr >= 0 && chan_on) ? __ldg(qc + (int64_t)rr * V) : 0;
      }
      __syncwarp();
      // ---- phase 2: group g = rows g*R .. g*R+R-1; instruction t: row slot ri -> slot (t+ri) mod S
#pragma unroll
      for (int g = 0; g < G; ++g) {
        const int i = g * R + ri;
        if (b0 + i < end) {
          uint32_t w32[SWD + 1];
#pragma unroll
          for (int w = 0; w < SWD; ++w) w32[w] = scratch[i * SWD + w];
          w32[SWD] = w32[1 < WD ? 1 : 0];
          uint32_t we[WD], wo[WD];                       // ring rotated by re / ro bytes
#pragma unroll
          for (int w = 0; w < WD; ++w) {
            we[w] = __funnelshift_r(w32[w], w32[w + 1], 8 * re);
            const uint32_t a = (ro >> 2) ? w32[w + 1] : w32[w];
            const uint32_t b = (ro >> 2) ? w32[w + 2] : w32[w + 1];
            wo[w] = __funnelshift_r(a, b, 8 * (ro & 3));
          }
          const uint32_t lo = (uint32_t)qv[g] & 0xFFFFu;
          const uint32_t hi = (uint32_t)(qv[g] >> 16);   // arithmetic shift, two's complement
          const uint32_t va = (ri & 1) ? hi : lo, vb = (ri & 1) ? lo : hi;
          DiagStep<0, S, R, RS, WD>::run(we, wo, lane_addr, ri, va, vb);
        }
      }
      __syncwarp();
      r_cur = r_nxt;
      r_nxt = r_nn;
#pragma unroll
      for (int i = 0; i < NW; ++i) w_cur[i] = w_nxt[i];
    }
    __syncthreads();

    // flush (as k_hist_smem): lo = slot 2j, hi = slot 2j + 1
    const int64_t slot = ch.x;
    const bool sole = ch.w != 0;
    const int64_t gbase = (slot * m + f0) * (int64_t)B;
    const int total = kk * B * K;
    for (int e = threadIdx.x; e < total; e += blockDim.x) {
      const int cc = e % K, jb = e / K;
      if (c0 + cc >= V) continue;
      const int j = jb / B, b = jb - j * B;
      const uint32_t* rowp = sm + b * RS + j * 2 * K;
      const uint32_t los = rowp[cc], his = rowp[K + cc];
      const long long v = (long long)(int32_t)his * 65536LL + (long long)los;
      int64_t* dst = &hist[((slot * m + f0 + j) * V + c0 + cc) * B + b];
      if (sole) *dst = v;
      else if (v != 0) atomicAdd(reinterpret_cast<unsigned long long*>(dst), (unsigned long long)v);
    }
    if (do_cnt) {
      for (int e = threadIdx.x; e < kk * B; e += blockDim.x) {
        const uint32_t nv = sm[limb_words + e];
        if (sole) cnt[gbase + e] = (int32_t)nv;
        else if (nv) atomicAdd(&cnt[gbase + e], (int32_t)nv);
      }
    }
    __syncthreads();
  }
}

template <int KF>
static gbdtmo_status launch_diag_kf(Ctx* ctx, const gbdtmo_problem& p, const HistCfg& hc, const uint8_t* bins,
                                    const int32_t* q, const int32_t* rows, int use_rows, const State& s, int64_t* hist,
                                    int32_t* cnt) {
  static unsigned long long attr_mask = 0;
  smem_optin_once(ctx, k_hist_diag<KF>, attr_mask, ctx->max_smem_optin - 1024);
  GB_LAUNCH(k_hist_diag<KF>, ctx->num_sms * kHistCtas, kHistThreads, hc.smem, p, hc, bins, q, rows, use_rows, s, hist, cnt);
  return GBDTMO_OK;
}

gbdtmo_status launch_hist_diag(Ctx* ctx, const gbdtmo_problem& p, const uint8_t* bins, const int32_t* q,
                               const int32_t* rows, int use_rows, const State& s, int64_t* hist, int32_t* cnt,
                               bool no_cnt) {
  HistCfg hc = hist_config_diag(p);
  hc.no_cnt = no_cnt ? 1 : 0;
  switch (hc.k) {
    case 20: return launch_diag_kf<20>(ctx, p, hc, bins, q, rows, use_rows, s, hist, cnt);
    case 16: return launch_diag_kf<16>(ctx, p, hc, bins, q, rows, use_rows, s, hist, cnt);
    case 12: return launch_diag_kf<12>(ctx, p, hc, bins, q, rows, use_rows, s, hist, cnt);
    case 8: return launch_diag_kf<8>(ctx, p, hc, bins, q, rows, use_rows, s, hist, cnt);
    default: return launch_diag_kf<4>(ctx, p, hc, bins, q, rows, use_rows, s, hist, cnt);
  }
}

}  // namespace gbdtmo
