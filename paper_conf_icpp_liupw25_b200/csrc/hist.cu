// hist.cu — (a)3: per-node histogram build (§3.3; Alg. 2's body is missing,
// PAPER.md:216-218, so the kernel is designed for sm_100a from the definition):
//
//   hist[slot][f][b][c] = sum_{i in node, bin(i,f) = b} q[i][c],   cnt[slot][f][b] = #{...}
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
//    becomes one vector load of up to 32 bin ids).
#include "common.cuh"

namespace gbdtmo {

__device__ __forceinline__ int byte_at(uint64_t w0, uint64_t w1, uint64_t w2, uint64_t w3, int idx) {
  uint64_t w = (idx < 8) ? w0 : (idx < 16) ? w1 : (idx < 24) ? w2 : w3;
  return (int)((w >> ((idx & 7) * 8)) & 0xFFu);
}

template <int K>
__global__ void __launch_bounds__(kHistThreads, 1)
k_hist_smem(gbdtmo_problem p, HistCfg hc, const uint8_t* __restrict__ bins, const int32_t* __restrict__ q,
            const int32_t* __restrict__ rows, int use_rows, State s,
            int64_t* __restrict__ hist, int32_t* __restrict__ cnt) {
  extern __shared__ __align__(16) uint32_t sm[];
  __shared__ int sh_item;
  constexpr int RPI = 32 / K;                 // rows per warp instruction
  const int V = channels(p), B = p.B, m = p.m;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
  const int ri = lane / K, c = lane % K;
  const int tiles = hc.n_ft * hc.n_ct;
  const int nitems = s.misc[MISC_CHUNK_COUNT] * tiles;
  const int limb_words = hc.k * B * 2 * K;
  uint32_t* limbs = sm;
  uint32_t* cnts = sm + limb_words;
  const int oa = (ri & 1) ? K : 0, ob = K - oa;   // alternate rows swap limb halves (banks)

  for (;;) {
    if (threadIdx.x == 0) sh_item = atomicAdd(&s.misc[MISC_WORK_COUNTER], 1);
    __syncthreads();
    const int item = sh_item;
    if (item >= nitems) break;
    const int chunk = item / tiles, tile = item - chunk * tiles;
    const int ft = tile / hc.n_ct, ct = tile - ft * hc.n_ct;
    const int4 ch = s.chunks[chunk];
    const int f0 = ft * hc.k;
    const int kk = min(hc.k, m - f0);
    const int c0 = ct * K;
    const bool do_cnt = (ct == 0);

    // zero the tile's accumulators
    const int words = limb_words + hc.k * B;
    for (int i = threadIdx.x * 4; i < limb_words; i += blockDim.x * 4)
      *reinterpret_cast<uint4*>(&sm[i]) = make_uint4(0, 0, 0, 0);
    for (int i = limb_words + threadIdx.x; i < words; i += blockDim.x) sm[i] = 0;
    __syncthreads();

    const int beg = ch.y, end = ch.z;
    const int o = f0 & 7;
    const int nwin = (o + kk + 7) >> 3;
    const uint8_t* bbase = bins + (f0 & ~7);
    const bool chan_on = (c0 + c) < V;
    for (int g = beg + warp * RPI; g < end; g += nwarps * RPI) {
      const int pos = g + ri;
      if (pos < end) {
        const int r = use_rows ? __ldg(&rows[pos]) : pos;
        const int qv = chan_on ? __ldg(&q[(int64_t)r * V + c0 + c]) : 0;
        const uint64_t* wp = reinterpret_cast<const uint64_t*>(bbase + (int64_t)r * p.ld_bins);
        uint64_t w0 = __ldg(wp), w1 = 0, w2 = 0, w3 = 0;
        if (nwin > 1) w1 = __ldg(wp + 1);
        if (nwin > 2) w2 = __ldg(wp + 2);
        if (nwin > 3) w3 = __ldg(wp + 3);
        const uint32_t lo = (uint32_t)qv & 0xFFFFu;
        const uint32_t hi = (uint32_t)(qv >> 16);          // arithmetic shift, two's complement
        const uint32_t va = (ri & 1) ? hi : lo, vb = (ri & 1) ? lo : hi;
        uint32_t* lb = limbs + c;
#pragma unroll 4
        for (int j = 0; j < kk; ++j) {
          const int bin = byte_at(w0, w1, w2, w3, o + j);
          uint32_t* a = lb + (j * B + bin) * (2 * K);
          atomicAdd(a + oa, va);
          atomicAdd(a + ob, vb);
        }
        if (do_cnt) {
          for (int j = c; j < kk; j += K) {
            const int bin = byte_at(w0, w1, w2, w3, o + j);
            atomicAdd(&cnts[j * B + bin], 1u);
          }
        }
      }
    }
    __syncthreads();

    // flush: exact int64 = hi * 2^16 + lo into the node histogram (global REDG.ADD.64)
    const int64_t slot = ch.x;
    const int64_t gbase = (slot * m + f0) * (int64_t)B;        // (slot, f0, bin 0)
    const int total = kk * B * K;
    for (int e = threadIdx.x; e < total; e += blockDim.x) {
      const int cc = e % K, jb = e / K;                        // jb = j * B + b
      if (c0 + cc >= V) continue;
      const uint32_t los = limbs[jb * 2 * K + cc], his = limbs[jb * 2 * K + K + cc];
      const long long v = (long long)(int32_t)his * 65536LL + (long long)los;
      if (v != 0)
        atomicAdd(reinterpret_cast<unsigned long long*>(&hist[(gbase + jb) * V + c0 + cc]), (unsigned long long)v);
    }
    if (do_cnt) {
      for (int e = threadIdx.x; e < kk * B; e += blockDim.x) {
        const uint32_t nv = cnts[e];
        if (nv) atomicAdd(&cnt[gbase + e], (int32_t)nv);
      }
    }
    __syncthreads();
  }
}

// Zero the histogram slots of the level's BUILD nodes (the flush accumulates atomically).
__global__ void k_zero_build(gbdtmo_problem p, int level, State s, int64_t* __restrict__ hist,
                             int32_t* __restrict__ cnt) {
  const int64_t slot = blockIdx.y;
  const int64_t h = (int64_t(1) << level) - 1 + slot;
  if (s.node_mode[h] != MODE_BUILD) return;
  const int64_t V = channels(p);
  const int64_t hw = (int64_t)p.m * p.B * V;           // int64 words per slot
  const int64_t cw = (int64_t)p.m * p.B;               // int32 words per slot
  int64_t* hb = hist + slot * hw;
  int32_t* cb = cnt + slot * cw;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  // hw is even when V is even; handle generally with a scalar tail
  const int64_t hv = hw / 2;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < hv; i += stride)
    reinterpret_cast<longlong2*>(hb)[i] = make_longlong2(0, 0);
  for (int64_t i = 2 * hv + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < hw; i += stride) hb[i] = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cw; i += stride) cb[i] = 0;
}

template <int K>
static gbdtmo_status launch_hist(Ctx* ctx, const gbdtmo_problem& p, const HistCfg& hc, const uint8_t* bins,
                                 const int32_t* q, const int32_t* rows, int use_rows, const State& s,
                                 int64_t* hist, int32_t* cnt) {
  static bool attr_done = false;
  if (!attr_done) {
    cudaFuncSetAttribute(k_hist_smem<K>, cudaFuncAttributeMaxDynamicSharedMemorySize, kHistSmemBudget + 4096);
    attr_done = true;
  }
  GB_LAUNCH(k_hist_smem<K>, ctx->num_sms, kHistThreads, hc.smem, p, hc, bins, q, rows, use_rows, s, hist, cnt);
  return GBDTMO_OK;
}

}  // namespace gbdtmo

using namespace gbdtmo;

extern "C" gbdtmo_status gbdtmo_build_hist(gbdtmo_ctx c, const gbdtmo_problem* p, int32_t level,
                                           const uint8_t* bins, const int32_t* q, void* state,
                                           int64_t* hist, int32_t* cnt) {
  Ctx* ctx = (Ctx*)c;
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(level >= 0 && level < p->D, "level out of range [0, D)");
  GB_CHECK_ARG(bins && q && state && hist && cnt, "null pointer");
  GB_CHECK_ARG(((uintptr_t)bins & 7) == 0, "bins must be 8-byte aligned");
  State s = state_view(*p, state);
  HistCfg hc = hist_config(*p);
  const int64_t LN = int64_t(1) << level;
  int gx = (int)(2 * ctx->num_sms / (LN > 1 ? LN / 2 : 1));
  if (gx < 8) gx = 8;
  GB_LAUNCH(k_zero_build, dim3(gx, (unsigned)LN), 256, 0, *p, level, s, hist, cnt);
  const int32_t* rows = (level & 1) ? s.rows1 : s.rows0;
  const int use_rows = level > 0;
  switch (hc.K) {
    case 4: return launch_hist<4>(ctx, *p, hc, bins, q, rows, use_rows, s, hist, cnt);
    case 8: return launch_hist<8>(ctx, *p, hc, bins, q, rows, use_rows, s, hist, cnt);
    case 16: return launch_hist<16>(ctx, *p, hc, bins, q, rows, use_rows, s, hist, cnt);
    default: return launch_hist<32>(ctx, *p, hc, bins, q, rows, use_rows, s, hist, cnt);
  }
}
