// hist_tma.cu — (a)3 histogram build, TMA-staged variant (GBDTMO_OPT_HIST_KERNEL = 2).
//
// Same definition, accumulator, work items and flush as k_hist_smem (hist.cu):
//   hist[slot][f][c][b] = sum_{i in node, bin(i,f) = b} q[i][c],   cnt[slot][f][b] = #{...}
// (§3.3).  What differs is how a row's bins reach the accumulating lanes.
//
// ncu on k_hist_smem (profiles/r01h_ncu_hist_c5.txt) shows the L1 data pipe (1 wavefront / clk / SM)
// as the limiter at 94%, and only ~60% of its wavefronts are the limb atomics that do the work:
// each warp-wide load of 32 gathered rows' bin windows costs ~32 tag wavefronts (one per row),
// two such loads per 32 rows, and the per-row count atomics are ~3-way bank-conflicted.  Here:
//  - a warp's rows reach shared memory by TMA: `cp.async.bulk.tensor ... tile::gather4` copies
//    the 32-byte bin window of four gathered rows per instruction (8 per 32-row batch) into a
//    2-stage per-warp ring, completed on an mbarrier — no LSU wavefronts for the gather.
//    Measured on B200 (tools/microbench/tma_probe.cu): gather4 needs a 16-byte aligned column
//    coordinate and a 128-byte aligned destination, so the window starts at f0 & ~15 and the
//    tile's KF bins sit at byte o = f0 & 15 of it;
//  - lanes (row-of-pair ri, channel c) read their row's window back with one LDS.128 per pair
//    of rows (2 distinct addresses: 1 wavefront; a second LDS.64 only when o + KF > 16), shift
//    it to byte o, and add the limbs exactly as k_hist_smem;
//  - counts are taken in the accumulation loop, once per two row pairs: lane (ri, c < 2 KF)
//    counts (row, feature) pair number c of its row slot into its own column `16 ri + c` of a
//    [bin / 2][32] table of 16-bit counter pairs, so the 32 lanes always hit 32 different banks
//    (bank = column) whatever the bins; the flush sums the 4 columns of each feature.
#include <cuda.h>

#include "common.cuh"
#include "hist_common.cuh"
#include "tma.cuh"

namespace gbdtmo {

constexpr int kTmaWarps = 8;
constexpr int kTmaThreads = kTmaWarps * 32;
constexpr int kTmaStages = 2;
constexpr int kTmaRowBytes = 32;                        // TMA box: 32 bytes x 1 row, 4 rows per gather4
constexpr int kTmaStageBytes = 32 * kTmaRowBytes;       // one 32-row batch
constexpr int kTmaK = 16;                               // channels per tile

static int tma_cnt_words(int B) { return ((B + 1) / 2) * 32; }
static int tma_fixed_bytes(int B) {
  return 4 * tma_cnt_words(B) + 128 /* stage alignment */ + kTmaWarps * kTmaStages * (kTmaStageBytes + 8);
}

bool hist_tma_supported(const gbdtmo_problem& p, const uint8_t* bins) {
  return channels(p) > 8 && p.ld_bins % 16 == 0 && ((uintptr_t)bins & 15) == 0;  // bins == nullptr: shape only
}

HistCfg hist_config_tma(const gbdtmo_problem& p, int max_smem) {
  HistCfg c;
  const int V = channels(p);
  c.K = kTmaK;
  c.n_ct = (V + kTmaK - 1) / kTmaK;
  const int per_feature = p.B * 2 * kTmaK * 4;
  const int budget = max_smem - 1024;
  const int allowed[6] = {8, 6, 4, 3, 2, 1};            // 2 KF count columns per row slot <= 16
  int k = 1;
  for (int i = 0; i < 6; ++i) {
    const int kk = allowed[i];
    if (kk <= p.m && kk * per_feature + tma_fixed_bytes(p.B) <= budget) { k = kk; break; }
  }
  c.k = k;
  c.n_ft = (p.m + k - 1) / k;
  c.smem = k * per_feature + tma_fixed_bytes(p.B);
  c.no_cnt = 0;
  return c;
}

// ------------------------------------------------------------------ PTX helpers

__device__ __forceinline__ void tma_gather4(uint32_t dst, uint64_t tmap, int col, int r0, int r1, int r2, int r3,
                                            uint32_t mbar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(dst),
      "l"(tmap), "r"(col), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(mbar)
      : "memory");
}
__device__ __forceinline__ uint64_t lds64(uint32_t addr) {
  uint64_t v;
  asm volatile("ld.shared.u64 %0, [%1];" : "=l"(v) : "r"(addr) : "memory");
  return v;
}
__device__ __forceinline__ void lds128(uint32_t addr, uint64_t& a, uint64_t& b) {
  asm volatile("ld.shared.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "r"(addr) : "memory");
}

// ------------------------------------------------------------------ kernel

template <int KF>
__global__ void __launch_bounds__(kTmaThreads, 1)
k_hist_tma(gbdtmo_problem p, HistCfg hc, const __grid_constant__ CUtensorMap tmap, const int32_t* __restrict__ q,
           const int32_t* __restrict__ rows, int use_rows, State s, int64_t* __restrict__ hist,
           int32_t* __restrict__ cnt) {
  extern __shared__ __align__(16) uint32_t sm[];
  __shared__ int sh_item;
  constexpr int K = kTmaK;
  constexpr int RS = KF * 2 * K;                 // limb words per bin
  constexpr int G = 16;                          // row pairs per 32-row batch
  const int V = channels(p), B = p.B, m = p.m;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int ri = lane >> 4, c = lane & 15;
  const int tiles = hc.n_ft * hc.n_ct;
  const int nitems = s.misc[MISC_CHUNK_COUNT] * tiles;
  const int limb_words = B * RS;
  const int cnt_words = ((B + 1) >> 1) * 32;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(sm);
  const uint32_t acnt = sbase + 4u * limb_words;
  const uint32_t stg = (sbase + 4u * (limb_words + cnt_words) + 127u) & ~127u;
  const uint32_t mybuf = stg + warp * kTmaStages * kTmaStageBytes;
  const uint32_t mbar = stg + kTmaWarps * kTmaStages * kTmaStageBytes + warp * 8 * kTmaStages;
  const int slotA = c + (ri ? K : 0), slotB = slotA ^ K;
  const uint32_t aA = sbase + 4u * slotA, aB = sbase + 4u * slotB;
  const uint64_t tmap_addr = reinterpret_cast<uint64_t>(&tmap);
  // count job of this lane: column 16 ri + c; c < KF -> feature c of the earlier row pair,
  // KF <= c < 2 KF -> feature c - KF of the later one
  const bool cnt_lane = c < 2 * KF;
  const int cj = c < KF ? c : c - KF;
  const uint32_t acol = acnt + 4u * (16 * ri + c);

  if (lane == 0) {
#pragma unroll
    for (int st = 0; st < kTmaStages; ++st) mbar_init(mbar + 8 * st, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  uint32_t phase = 0;                            // bit st: parity of the next completion of stage st

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
    const bool do_cnt = (ct == 0);

    const int words = limb_words + cnt_words;
    for (int i = threadIdx.x * 4; i < words; i += blockDim.x * 4)
      *reinterpret_cast<uint4*>(&sm[i]) = make_uint4(0, 0, 0, 0);
    __syncthreads();

    const int beg = ch.y, end = ch.z;
    const int ow = (f0 >> 3) & 1, ob = f0 & 7;             // window byte o = f0 & 15 = 8 ow + ob
    const bool third = ow && ob + KF > 8;                 // bins reach past byte 16 of the window
    const bool chan_on = (c0 + c) < V;
    const int32_t* qc = q + c0 + c;
    constexpr int bstep = kTmaWarps * 32;
    auto load_rid = [&](int pos) -> int { return pos < end ? (use_rows ? __ldg(&rows[pos]) : pos) : -1; };
    // stage `st` <- bin windows of the 32 rows whose ids the lanes hold (invalid rows: row 0, masked later)
    auto issue = [&](int rid, int st) {
      const int rr = rid < 0 ? 0 : rid;
      const int g = 4 * (lane & 7);
      const int x0 = __shfl_sync(0xffffffffu, rr, g), x1 = __shfl_sync(0xffffffffu, rr, g + 1);
      const int x2 = __shfl_sync(0xffffffffu, rr, g + 2), x3 = __shfl_sync(0xffffffffu, rr, g + 3);
      if (lane == 0) mbar_arrive_expect_tx(mbar + 8 * st, kTmaStageBytes);
      __syncwarp();
      if (lane < 8)
        tma_gather4(mybuf + st * kTmaStageBytes + lane * 4 * kTmaRowBytes, tmap_addr, f0 & ~15, x0, x1, x2, x3,
                    mbar + 8 * st);
    };
    auto load_q = [&](int rid, int (&qv)[G]) {
#pragma unroll
      for (int t = 0; t < G; ++t) {
        const int rr = __shfl_sync(0xffffffffu, rid, 2 * t + ri);
        qv[t] = (rr >= 0 && chan_on) ? __ldg(qc + (int64_t)rr * V) : 0;
      }
    };

    int b0 = beg + warp * 32;
    int r_cur = load_rid(b0 + lane);
    int r_nxt = load_rid(b0 + bstep + lane);
    if (b0 < end) issue(r_cur, 0);
    if (b0 + bstep < end) issue(r_nxt, 1);
    int qcur[G];
    load_q(r_cur, qcur);
    int st = 0;
    for (; b0 < end; b0 += bstep) {
      const int r_nn = load_rid(b0 + 2 * bstep + lane);
      int qnxt[G];
      load_q(r_nxt, qnxt);
      mbar_wait(mbar + 8 * st, (phase >> st) & 1u);
      phase ^= 1u << st;
      const uint32_t buf = mybuf + st * kTmaStageBytes;
      uint64_t bprev = 0;
#pragma unroll
      for (int t = 0; t < G; ++t) {
        const int i = 2 * t + ri;
        uint64_t a0, a1, a2 = 0;
        lds128(buf + i * kTmaRowBytes, a0, a1);
        if (third) a2 = lds64(buf + i * kTmaRowBytes + 16);
        const uint64_t wl = ow ? a1 : a0, wh = ow ? a2 : a1;
        const uint64_t bw = ob ? (wl >> (8 * ob)) | (wh << (64 - 8 * ob)) : wl;
        const uint32_t lo = (uint32_t)qcur[t] & 0xFFFFu;
        const uint32_t hi = (uint32_t)(qcur[t] >> 16);       // arithmetic shift, two's complement
        const uint32_t va = ri ? hi : lo, vb = ri ? lo : hi;
        if (b0 + i < end) {
          if (kk == KF) {
#pragma unroll
            for (int j = 0; j < KF; ++j) {
              const uint32_t bin = (uint32_t)(bw >> (8 * j)) & 0xFFu;
              red_shared_add(aA + bin * (4u * RS) + 8u * K * j, va);
              red_shared_add(aB + bin * (4u * RS) + 8u * K * j, vb);
            }
          } else {
#pragma unroll
            for (int j = 0; j < KF; ++j) {
              const uint32_t bin = (uint32_t)(bw >> (8 * j)) & 0xFFu;
              if (j < kk) {
                red_shared_add(aA + bin * (4u * RS) + 8u * K * j, va);
                red_shared_add(aB + bin * (4u * RS) + 8u * K * j, vb);
              }
            }
          }
        }
        if ((t & 1) && do_cnt) {
          // rows 2(t-1)+ri (window bprev) and 2t+ri (window bw)
          const uint64_t w = c < KF ? bprev : bw;
          const int row = c < KF ? i - 2 : i;
          if (cnt_lane && cj < kk && b0 + row < end) {
            const uint32_t bin = (uint32_t)(w >> (8 * cj)) & 0xFFu;
            red_shared_add(acol + (bin >> 1) * 128u, 1u << (16 * (bin & 1)));
          }
        }
        bprev = bw;
      }
      __syncwarp();
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      if (b0 + 2 * bstep < end) issue(r_nn, st);
      r_cur = r_nxt;
      r_nxt = r_nn;
#pragma unroll
      for (int t = 0; t < G; ++t) qcur[t] = qnxt[t];
      st ^= 1;
    }
    __syncthreads();

    // flush (as k_hist_smem): exact int64 = hi * 2^16 + lo; sole writer stores, else REDG.ADD.64
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
        const int j = e / B, b = e - j * B;
        const uint32_t* cw = sm + limb_words + (b >> 1) * 32;
        const int sh = 16 * (b & 1);
        const uint32_t nv = ((cw[j] >> sh) & 0xFFFFu) + ((cw[j + KF] >> sh) & 0xFFFFu) +
                            ((cw[16 + j] >> sh) & 0xFFFFu) + ((cw[16 + j + KF] >> sh) & 0xFFFFu);
        if (sole) cnt[gbase + e] = (int32_t)nv;
        else if (nv) atomicAdd(&cnt[gbase + e], (int32_t)nv);
      }
    }
    __syncthreads();
  }
}

// ------------------------------------------------------------------ host

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult qr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &qr) == cudaSuccess &&
        qr == cudaDriverEntryPointSuccess)
      fn = (EncodeTiledFn)f;
    cudaGetLastError();
  }
  return fn;
}

template <int KF>
static gbdtmo_status launch_tma_kf(Ctx* ctx, const gbdtmo_problem& p, const HistCfg& hc, const CUtensorMap& tm,
                                   const int32_t* q, const int32_t* rows, int use_rows, const State& s, int64_t* hist,
                                   int32_t* cnt) {
  static unsigned long long attr_mask = 0;
  smem_optin_once(ctx, k_hist_tma<KF>, attr_mask, ctx->max_smem_optin - 1024);
  GB_LAUNCH(k_hist_tma<KF>, ctx->num_sms, kTmaThreads, hc.smem, p, hc, tm, q, rows, use_rows, s, hist, cnt);
  return GBDTMO_OK;
}

gbdtmo_status launch_hist_tma(Ctx* ctx, const gbdtmo_problem& p, const uint8_t* bins, const int32_t* q,
                              const int32_t* rows, int use_rows, const State& s, int64_t* hist, int32_t* cnt) {
  EncodeTiledFn enc = encode_fn();
  if (!enc) {
    ctx->err = "gbdtmo_build_hist: cuTensorMapEncodeTiled unavailable";
    return GBDTMO_ECUDA;
  }
  CUtensorMap tm;
  const cuuint64_t gdim[2] = {(cuuint64_t)p.ld_bins, (cuuint64_t)p.n};
  const cuuint64_t gstride[1] = {(cuuint64_t)p.ld_bins};
  const cuuint32_t box[2] = {(cuuint32_t)kTmaRowBytes, 1};
  const cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, (void*)bins, gdim, gstride, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    ctx->err = "gbdtmo_build_hist: cuTensorMapEncodeTiled failed (" + std::to_string((int)r) + ")";
    return GBDTMO_ECUDA;
  }
  const HistCfg hc = hist_config_tma(p, ctx->max_smem_optin);
  switch (hc.k) {
    case 8: return launch_tma_kf<8>(ctx, p, hc, tm, q, rows, use_rows, s, hist, cnt);
    case 6: return launch_tma_kf<6>(ctx, p, hc, tm, q, rows, use_rows, s, hist, cnt);
    case 4: return launch_tma_kf<4>(ctx, p, hc, tm, q, rows, use_rows, s, hist, cnt);
    case 3: return launch_tma_kf<3>(ctx, p, hc, tm, q, rows, use_rows, s, hist, cnt);
    case 2: return launch_tma_kf<2>(ctx, p, hc, tm, q, rows, use_rows, s, hist, cnt);
    default: return launch_tma_kf<1>(ctx, p, hc, tm, q, rows, use_rows, s, hist, cnt);
  }
}

}  // namespace gbdtmo
