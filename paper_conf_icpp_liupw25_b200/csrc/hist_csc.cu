// hist_csc.cu — (a)3 on the paper's sparse storage (§3.2 "Sparsity-aware data
// storage"; NEXT-1): histograms built from the CSC non-zeros only.  The paper gives each thread
// block one or more attribute columns; here the column-major entries are spread
// evenly instead (one thread per stored entry, its column by a binary search of col_ptr), since
// column lengths vary by orders of magnitude in sparse data (a block-per-column variant was
// latency-bound and slower: DESIGN.md §7, "CSC-driven histograms").
//
//   hist[slot][f][c][b] = sum_{i in node, x_if != 0, bin(i,f) = b, b != z_f} q[i][c]   (exact int64)
//   cnt [slot][f][b]    = #{...}
//
// The implicit zeros never appear: z_f = bin(0) of feature f is filled in last as the node total
// minus the other bins (exact, as the default-bin recovery of reading R25), which also covers
// explicit entries binned with zero (they are skipped), so the histograms equal the dense path's.
// Work is proportional to the non-zeros: one thread per non-zero (grid-stride), its column found by
// a binary search of col_ptr, its node from the per-row node ids; only the level's BUILD nodes
// accumulate (global REDG.ADD.64 into slots zeroed first), derived siblings still come from
// subtraction in gbdtmo_find_split.
#include "common.cuh"

namespace gbdtmo {

// Zero the histogram and count slots of every BUILD / BUILD1 node of the level (all accumulate).
__global__ void k_zero_build_csc(gbdtmo_problem p, int level, State s, int64_t* __restrict__ hist,
                                 int32_t* __restrict__ cnt) {
  const int64_t slot = blockIdx.y;
  const int64_t h = (int64_t(1) << level) - 1 + slot;
  const int md = s.node_mode[h];
  if (md != MODE_BUILD && md != MODE_BUILD1) return;
  const int64_t V = channels(p);
  const int64_t hw = (int64_t)p.m * p.B * V, cw = (int64_t)p.m * p.B;
  int64_t* hb = hist + hist_index(p, level, slot) * hw;
  int32_t* cb = cnt + hist_index(p, level, slot) * cw;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < hw; i += stride) hb[i] = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cw; i += stride) cb[i] = 0;
}

__global__ void __launch_bounds__(256)
k_hist_csc(gbdtmo_problem p, int level, const int64_t* __restrict__ col_ptr, const int32_t* __restrict__ row_idx,
           const uint8_t* __restrict__ nz_bins, const int32_t* __restrict__ zbin, const int32_t* __restrict__ q,
           State s, int64_t* __restrict__ hist, int32_t* __restrict__ cnt) {
  const int m = p.m, B = p.B, V = channels(p);
  const int64_t nnz = col_ptr[m];
  const int64_t LN = int64_t(1) << level, first = LN - 1;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x) {
    int lo = 0, hi = m - 1;                                   // column: last f with col_ptr[f] <= e
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (__ldg(&col_ptr[mid]) <= e) lo = mid; else hi = mid - 1;
    }
    const int f = lo;
    const int b = nz_bins[e];
    if (b == __ldg(&zbin[f])) continue;                      // recovered from the node totals
    const int32_t r = row_idx[e];
    const int64_t h = s.nid[r];
    if (h < first || h >= first + LN) continue;
    const int md = s.node_mode[h];
    if (md != MODE_BUILD && md != MODE_BUILD1) continue;
    const int64_t slot = hist_index(p, level, h - first);
    atomicAdd(&cnt[(slot * m + f) * B + b], 1);
    int64_t* hb = hist + (slot * m + f) * (int64_t)V * B + b;
    const int32_t* qr = q + (int64_t)r * V;
    for (int c = 0; c < V; ++c) {
      const int v = __ldg(&qr[c]);
      if (v) atomicAdd(reinterpret_cast<unsigned long long*>(hb + (int64_t)c * B), (unsigned long long)(long long)v);
    }
  }
}

// Completes every BUILD node's histogram: bin zbin[f] = node total - sum of the other bins, per
// channel and for the counts (exact int64), so the histograms leaving gbdtmo_build_hist_csc are the
// dense path's and the split search needs no default-bin recovery.  One block per (feature, slot),
// one warp per channel row (+ the count row).
__global__ void __launch_bounds__(256)
k_csc_fill_zero_bin(gbdtmo_problem p, int level, const int32_t* __restrict__ zbin, State s, int64_t* __restrict__ hist,
                    int32_t* __restrict__ cnt) {
  const int f = blockIdx.x;
  const int64_t slot = blockIdx.y;
  const int64_t h = (int64_t(1) << level) - 1 + slot;
  const int md = s.node_mode[h];
  if (f >= p.m || (md != MODE_BUILD && md != MODE_BUILD1)) return;
  const int V = channels(p), B = p.B;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const int z = zbin[f];
  const int64_t* S = s.node_sum + h * (V + 1);
  const int64_t hs = hist_index(p, level, slot);
  for (int c = warp; c <= V; c += nw) {
    long long acc = 0;
    if (c < V) {
      const int64_t* row = hist + ((hs * p.m + f) * V + c) * (int64_t)B;
      for (int b = lane; b < B; b += 32) acc += b == z ? 0 : row[b];
    } else {
      const int32_t* row = cnt + (hs * p.m + f) * (int64_t)B;
      for (int b = lane; b < B; b += 32) acc += b == z ? 0 : row[b];
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0) {
      if (c < V) hist[((hs * p.m + f) * V + c) * (int64_t)B + z] = S[c] - acc;
      else cnt[(hs * p.m + f) * (int64_t)B + z] = (int32_t)(S[V] - acc);
    }
  }
}

// Bins of the stored values (gathered from the binned matrix, one block per column) and the bin of
// an implicit zero per feature (#{cuts <= 0}, R14).
__global__ void k_csc_nz_bins(int32_t m, int32_t B, const int64_t* __restrict__ col_ptr,
                              const int32_t* __restrict__ row_idx, const uint8_t* __restrict__ bins, int64_t ld_bins,
                              const float* __restrict__ cuts, uint8_t* __restrict__ nz_bins,
                              int32_t* __restrict__ zbin) {
  const int f = blockIdx.x;
  if (f >= m) return;
  for (int64_t e = col_ptr[f] + threadIdx.x; e < col_ptr[f + 1]; e += blockDim.x)
    nz_bins[e] = bins[(int64_t)row_idx[e] * ld_bins + f];
  if (threadIdx.x == 0) {
    int z = 0;
    const float* cf = cuts + (int64_t)f * (B - 1);
    while (z < B - 1 && cf[z] <= 0.0f) ++z;                // cuts ascending, +inf padded
    zbin[f] = z;
  }
}

}  // namespace gbdtmo

using namespace gbdtmo;

extern "C" gbdtmo_status gbdtmo_csc_nz_bins(gbdtmo_ctx c, int32_t m, int32_t B, const int64_t* col_ptr,
                                            const int32_t* row_idx, const uint8_t* bins, int64_t ld_bins,
                                            const float* cuts, uint8_t* nz_bins, int32_t* zbin) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  GB_CHECK_ARG(m >= 1 && B >= 2 && B <= 256 && ld_bins >= m, "bad shape");
  GB_CHECK_ARG(col_ptr && bins && cuts && zbin, "null pointer");
  GB_LAUNCH(k_csc_nz_bins, (unsigned)m, 256, 0, m, B, col_ptr, row_idx, bins, ld_bins, cuts, nz_bins, zbin);
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_build_hist_csc(gbdtmo_ctx c, const gbdtmo_problem* p, int32_t level,
                                               const int64_t* col_ptr, const int32_t* row_idx, const uint8_t* nz_bins,
                                               int64_t nnz_host, const int32_t* zbin, const int32_t* q, void* state,
                                               int64_t* hist, int32_t* cnt) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(level >= 0 && level < p->D, "level out of range [0, D)");
  GB_CHECK_ARG(col_ptr && zbin && q && state && hist && cnt, "null pointer");
  GB_CHECK_ARG(nnz_host >= 0, "nnz < 0");
  State s = state_view(*p, state);
  const int64_t LN = int64_t(1) << level;
  const int64_t hw = (int64_t)p->m * p->B * channels(*p);
  const unsigned gx = (unsigned)std::min<int64_t>((hw + 255) / 256, 4 * (int64_t)ctx->num_sms);
  GB_LAUNCH(k_zero_build_csc, dim3(gx, (unsigned)LN), 256, 0, *p, level, s, hist, cnt);
  if (nnz_host > 0) {
    const unsigned g = (unsigned)std::min<int64_t>((nnz_host + 255) / 256, 32 * (int64_t)ctx->num_sms);
    GB_LAUNCH(k_hist_csc, g, 256, 0, *p, level, col_ptr, row_idx, nz_bins, zbin, q, s, hist, cnt);
  }
  GB_LAUNCH(k_csc_fill_zero_bin, dim3((unsigned)p->m, (unsigned)LN), 256, 0, *p, level, zbin, s, hist, cnt);
  return GBDTMO_OK;
}
