// common.cuh — context, state layout and launch configuration shared by the kernels
// of libgbdtmo.so (the product path).  Nothing here is shared with oracle/.
#pragma once

#include <nvtx3/nvToolsExt.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

#include <string>

#include "gbdtmo.h"

namespace gbdtmo {

// ------------------------------------------------------------------ context

struct Peer;                   // peer-memory exchange group (peer.cu)

struct Ctx {
  int device = 0;
  cudaStream_t stream = 0;
  int num_sms = 148;
  int max_smem_optin = 227 * 1024;
  int64_t launches = 0;
  int64_t gmem_max_rows = 0;   // GBDTMO_OPT_GMEM_MAX_ROWS: BUILD nodes with <= rows use the global-atomic variant
  int64_t small_max_rows = 0;  // GBDTMO_OPT_SMALL_MAX_ROWS: nodes whose parent's children both fit -> fused path
  int64_t hist_kernel = 0;     // GBDTMO_OPT_HIST_KERNEL: 0 row-pair (K <= 16), 1 diagonal (K = 4), 2 TMA-staged row-pair
  int64_t peer_timeout_ms = 30000;   // GBDTMO_OPT_PEER_TIMEOUT_MS: bound of every peer-flag wait
  int64_t fs_channel_groups = 0;     // GBDTMO_OPT_FS_CHANNEL_GROUPS: 0 automatic, 1 off, 2 / 4 forced
  int64_t hist_waves = 0;            // GBDTMO_OPT_HIST_WAVES: histogram work items per level in SM multiples (0: default)
  Peer* peer = nullptr;        // gbdtmo_peer_open / _connect (peer.cu)
  const int32_t* root_cnt = nullptr;   // gbdtmo_set_root_counts: cached root counts [m][B] (or null)
  cudaStream_t copy_stream = nullptr;  // gbdtmo_bin_host: host -> device strip copies (created on first use)
  cudaEvent_t strip_ready[2] = {nullptr, nullptr}, strip_free[2] = {nullptr, nullptr};
  std::string err;
};
void ctx_release_streams(Ctx* ctx);   // bin.cu

// Every entry point runs its CUDA calls on ctx->device and restores the caller's current device
// on return (the library must not depend on, or change, the caller's current device).
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(const Ctx* ctx) {
    int cur = -1;
    if (ctx && cudaGetDevice(&cur) == cudaSuccess && cur != ctx->device) {
      prev = cur;
      cudaSetDevice(ctx->device);
    }
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

// NVTX range over one C-ABI call (tracing): shows every entry point by name in Nsight
// Systems and `ncu --nvtx` filters; a no-op branch unless a tool is attached (header-only NVTX3).
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};
// Every extern "C" entry point opens with GB_ENTRY(ctx): the context's device made current (the
// caller's restored on return) and an NVTX range named after the call.
#define GB_ENTRY(ctx)               \
  DeviceGuard device_guard_(ctx);   \
  NvtxRange nvtx_range_(__func__)

// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) applies per device: one bit per device per
// kernel instantiation (the caller keeps a static mask), set with the context's device current.
template <typename F>
inline void smem_optin_once(const Ctx* ctx, F* kernel, unsigned long long& mask, int bytes) {
  const unsigned long long bit = 1ull << (ctx->device & 63);
  if (!(__atomic_load_n(&mask, __ATOMIC_ACQUIRE) & bit)) {
    cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    __atomic_fetch_or(&mask, bit, __ATOMIC_RELEASE);
  }
}

#define GB_CHECK_ARG(cond, msg)                  \
  do {                                           \
    if (!(cond)) {                               \
      ctx->err = std::string(__func__) + ": " + (msg); \
      return GBDTMO_EINVAL;                      \
    }                                            \
  } while (0)

#define GB_CHECK_LAUNCH()                                                        \
  do {                                                                           \
    cudaError_t e_ = cudaGetLastError();                                         \
    if (e_ != cudaSuccess) {                                                     \
      ctx->err = std::string(__func__) + ": " + cudaGetErrorString(e_);          \
      return GBDTMO_ECUDA;                                                       \
    }                                                                            \
  } while (0)

// ----------------------------------------------------------------- constants

constexpr int kQShift = 30;            // q = rint(g * 2^30 / P), |q| <= 2^30
#ifndef GBDTMO_CHUNK_MAX
#define GBDTMO_CHUNK_MAX 65536
#endif
constexpr int kChunkMax = GBDTMO_CHUNK_MAX;   // rows per histogram work item: lo-limb sums < 2^32 (<= 65536)
constexpr int kChunkMin = 512;
constexpr int kPartTile = 2048;        // positions per partition block
#ifndef GBDTMO_HIST_THREADS
#define GBDTMO_HIST_THREADS 1024
#endif
constexpr int kHistThreads = GBDTMO_HIST_THREADS;   // histogram CTA (1 CTA / SM, ~200 KB smem)
constexpr int kHistSmemBudget = 218 * 1024;   // limbs + counts + per-warp row scratch
#ifndef GBDTMO_HIST_CTAS
#define GBDTMO_HIST_CTAS 1        // (A/B) resident histogram CTAs per SM: 2 -> half tiles, overlapping fixed costs
#endif
constexpr int kHistCtas = GBDTMO_HIST_CTAS;
constexpr int kHistTileBudget = kHistCtas == 1 ? kHistSmemBudget : (226 * 1024) / kHistCtas - 2 * 1024;
constexpr int kHistWarps = kHistThreads / 32;
constexpr int kMaxTileFeatures = 24;   // features per histogram tile (32-byte bin window)

// MODE_BUILD1: built by exactly one work item per tile -> the flush stores instead of adding, and
// the slot needs no zeroing (saves 2 passes over the node's histogram in HBM).
// MODE_SMALL: built from its rows and searched in shared memory (small.cu), never materialised.
enum : int32_t { MODE_NONE = 0, MODE_BUILD = 1, MODE_DERIVE = 2, MODE_BUILD1 = 3, MODE_SMALL = 4 };

// The two child terms of Eq. (3) for one output, G_L^2/(H_L + l) + G_R^2/(H_R + l), with one fp64
// division instead of two (the softmax split search is division-bound: ncu, profiles/r02_ncu_fs_C2.txt).
// Differs from the two-division form by a few ulp, far below the fixed-point sums' own error.
#ifndef GBDTMO_EQ3_TWO_DIV
#define GBDTMO_EQ3_TWO_DIV 0      // (A/B) 1: the literal two-division form
#endif
__device__ __forceinline__ double eq3_pair(double GL, double HLl, double GR, double HRl) {   // HLl = H_L + l, HRl = H_R + l
  if (GBDTMO_EQ3_TWO_DIV) return GL * GL / HLl + GR * GR / HRl;
  return fma(GL * GL, HRl, GR * GR * HLl) / (HLl * HRl);
}

// Packed split key: larger gain wins, ties -> smallest (f_global * B + b).
__device__ __forceinline__ uint64_t pack_split_key(double gain, int64_t fb) {
  return ((uint64_t)__double_as_longlong(gain) & ~0xFFFFFFull) | (uint64_t)(0xFFFFFF - fb);
}

__host__ __device__ inline int channels(const gbdtmo_problem& p) {
  return p.loss == GBDTMO_LOSS_SOFTMAX ? 2 * p.d : p.d;
}
__host__ __device__ inline int64_t heap_nodes(const gbdtmo_problem& p) { return (int64_t(1) << (p.D + 1)) - 1; }
__host__ __device__ inline int64_t max_level_nodes(const gbdtmo_problem& p) { return int64_t(1) << (p.D > 0 ? p.D - 1 : 0); }
__host__ __device__ inline int64_t max_chunks(const gbdtmo_problem& p) {
  return p.n / kChunkMin + (int64_t(1) << p.D) + 2;
}
__host__ __device__ inline int64_t part_tiles(const gbdtmo_problem& p) { return (p.n + kPartTile - 1) / kPartTile; }
constexpr int kLeafRows = 1024;        // rows per leaf-sum chunk (gbdtmo_leaf_values with fp64 g/h)
__host__ __device__ inline int64_t leaf_chunks_max(const gbdtmo_problem& p) {
  return p.n / kLeafRows + heap_nodes(p) + 1;
}
// Histogram slot of node `slot` (index within its level) in that level's buffer.  At the last
// level (D-1 > 0) only the BUILT child of each sibling pair is ever materialised (the derived
// one is searched as parent - built and never written), so the pair shares slot >> 1: the last
// level's buffer holds 2^(D-2) nodes instead of 2^(D-1) (C5 at D = 11 and a
// Delicious-shaped d = 983 problem at depth 8 fit in HBM).
__host__ __device__ inline int64_t hist_index(const gbdtmo_problem& p, int level, int64_t slot) {
  return (level == p.D - 1 && level > 0) ? (slot >> 1) : slot;
}
__host__ __device__ inline int64_t hist_slots(const gbdtmo_problem& p, int level) {
  return (level == p.D - 1 && level > 0) ? (int64_t(1) << (level - 1)) : (int64_t(1) << level);
}
__host__ __device__ inline int64_t rec_words(const gbdtmo_problem& p) { return channels(p) + 4; }
__host__ __device__ inline int64_t bitmap_offset(const gbdtmo_problem& p) { return max_level_nodes(p) * rec_words(p); }

// Histogram tiling: a work item is (row chunk, feature tile of
// k features, channel tile of K channels).  Lanes map to (row-in-group, channel) with
// K channels per row and 32/K rows per warp instruction.
struct HistCfg {
  int K;      // channels per tile (4, 8, 16 or 32)
  int k;      // features per tile
  int n_ct;   // channel tiles
  int n_ft;   // feature tiles
  int smem;   // bytes of dynamic shared memory
  int no_cnt; // 1: counts come from the cached root counts (gbdtmo_set_root_counts), not accumulated
};

#ifndef GBDTMO_HIST_LCNT
#define GBDTMO_HIST_LCNT 0   // (A/B) 1: K = 16 tiles count in the accumulation loop, bank-per-lane table
#endif
__host__ __device__ inline bool hist_lane_counts(int K, int k) { return GBDTMO_HIST_LCNT && K == 16 && k <= 8; }
// counts[k][B] int32, or with lane counts a [ceil(B/2)][32] table of 16-bit counter pairs
__host__ __device__ inline int hist_cnt_words(int K, int k, int B) {
  return hist_lane_counts(K, k) ? ((B + 1) / 2) * 32 : k * B;
}

__host__ __device__ inline HistCfg hist_config(const gbdtmo_problem& p) {
  HistCfg c;
  int V = channels(p);
  c.K = V <= 4 ? 4 : V <= 8 ? 8 : 16;   // K = 32 halves the atomics per loaded row (measured slower)
  c.n_ct = (V + c.K - 1) / c.K;
  const int limbs_per_feature = p.B * 2 * c.K * 4;
  // compile-time tile widths the kernel is instantiated for; each needs a per-warp scratch of
  // 32 rows x ceil(k/8) 8-byte bin words
  const int allowed[9] = {24, 16, 12, 8, 6, 4, 3, 2, 1};
  int k = 1;
  for (int i = 0; i < 9; ++i) {
    const int kk = allowed[i];
    const int need = kk * limbs_per_feature + 4 * hist_cnt_words(c.K, kk, p.B) + kHistWarps * 32 * 8 * ((kk + 7) / 8);
    if (kk <= p.m && need <= kHistTileBudget) { k = kk; break; }
  }
  c.k = k;
  c.n_ft = (p.m + k - 1) / k;
  c.smem = k * limbs_per_feature + 4 * hist_cnt_words(c.K, k, p.B) + kHistWarps * 32 * 8 * ((k + 7) / 8);
  c.no_cnt = 0;
  return c;
}

// Tile-packed bins (gbdtmo_pack_bins): uint8 [ceil(n_ft/G)][n][G][8], G = kPackGroup tiles per
// row group; word (t, i) = bins of features [k t, k t + k) of row i, zero padded; only for tiles
// of <= 8 features.  G = 4: a 32-byte sector holds one row's bins for 4 consecutive tiles, which
// the work order runs concurrently, so gathered rows at deep levels fetch each sector once (with
// G = 1 every (row, tile) was its own sector: 79 GB of DRAM reads in one C5 level-7 launch).
#ifndef GBDTMO_PACK_GROUP
#define GBDTMO_PACK_GROUP 4
#endif
constexpr int kPackGroup = GBDTMO_PACK_GROUP;
__host__ __device__ inline bool hist_packable(const gbdtmo_problem& p) { return hist_config(p).k <= 8; }

// ------------------------------------------------------------- state layout

struct StateLayout {
  size_t rows0, rows1, nid;
  size_t node_begin, node_end, node_state, node_mode, node_feat, node_bin, node_gain, node_nleft, node_sum;
  size_t chunks, gnodes, snodes, misc, scale_max, tile_cnt, lpart;
  size_t leaf_chunk, leaf_c0, leaf_part;
  size_t total;
};

__host__ __device__ inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

__host__ __device__ inline StateLayout state_layout(const gbdtmo_problem& p) {
  StateLayout L;
  size_t o = 0;
  const size_t n = (size_t)p.n, NH = (size_t)heap_nodes(p), V = (size_t)channels(p);
  auto take = [&](size_t bytes) { size_t r = o; o = align_up(o + bytes, 256); return r; };
  L.rows0 = take(4 * n);
  L.rows1 = take(4 * n);
  L.nid = take(4 * n);
  L.node_begin = take(4 * NH);
  L.node_end = take(4 * NH);
  L.node_state = take(4 * NH);
  L.node_mode = take(4 * NH);
  L.node_feat = take(4 * NH);
  L.node_bin = take(4 * NH);
  L.node_gain = take(8 * NH);
  L.node_nleft = take(8 * NH);
  L.node_sum = take(8 * NH * (V + 1));
  L.chunks = take(16 * (size_t)max_chunks(p));
  L.gnodes = take(16 * (size_t)(max_level_nodes(p) + 1));
  L.snodes = take(16 * (size_t)(max_level_nodes(p) + 1));
  L.misc = take(64);
  L.scale_max = take(8 * V);
  L.tile_cnt = take(4 * ((size_t)part_tiles(p) + 1));
  L.lpart = take(4 * NH);
  L.leaf_chunk = take(16 * (size_t)leaf_chunks_max(p));
  L.leaf_c0 = take(4 * (NH + 1));
  L.leaf_part = take(8 * V * (size_t)leaf_chunks_max(p));
  L.total = o;
  return L;
}

// misc words
enum { MISC_CHUNK_COUNT = 0, MISC_WORK_COUNTER = 1, MISC_CHUNK_ROWS = 2, MISC_GNODE_COUNT = 3, MISC_GNODE_ROWS = 4,
       MISC_SNODE_COUNT = 5, MISC_SWORK_COUNTER = 6 };

struct State {
  int32_t *rows0, *rows1, *nid;
  int32_t *node_begin, *node_end, *node_state, *node_mode, *node_feat, *node_bin;
  double* node_gain;
  int64_t* node_nleft;
  int64_t* node_sum;  // [NH][V+1]: V channel sums of q, then the row count
  int4* chunks;       // (slot, begin, end, unused)
  int4* gnodes;       // global-atomic variant nodes: (slot, begin, end, row prefix)
  int4* snodes;       // fused small-node path: (slot, begin, end, unused)
  int32_t* misc;
  unsigned long long* scale_max;   // bits of max_i |g_ic| (fp64, non-negative)
  int32_t* tile_cnt;
  int32_t* lpart;
  int4* leaf_chunk;   // fp64 leaf sums: (leaf, begin, end, unused) chunks of <= kLeafRows rows of the final list
  int32_t* leaf_c0;   // [NH + 1]: first chunk of every heap node (exclusive prefix; non-leaves own none)
  double* leaf_part;  // [chunk][V] fp64 partial sums
};

__host__ __device__ inline State state_view(const gbdtmo_problem& p, void* base) {
  StateLayout L = state_layout(p);
  char* b = (char*)base;
  State s;
  s.rows0 = (int32_t*)(b + L.rows0);
  s.rows1 = (int32_t*)(b + L.rows1);
  s.nid = (int32_t*)(b + L.nid);
  s.node_begin = (int32_t*)(b + L.node_begin);
  s.node_end = (int32_t*)(b + L.node_end);
  s.node_state = (int32_t*)(b + L.node_state);
  s.node_mode = (int32_t*)(b + L.node_mode);
  s.node_feat = (int32_t*)(b + L.node_feat);
  s.node_bin = (int32_t*)(b + L.node_bin);
  s.node_gain = (double*)(b + L.node_gain);
  s.node_nleft = (int64_t*)(b + L.node_nleft);
  s.node_sum = (int64_t*)(b + L.node_sum);
  s.chunks = (int4*)(b + L.chunks);
  s.gnodes = (int4*)(b + L.gnodes);
  s.snodes = (int4*)(b + L.snodes);
  s.misc = (int32_t*)(b + L.misc);
  s.scale_max = (unsigned long long*)(b + L.scale_max);
  s.tile_cnt = (int32_t*)(b + L.tile_cnt);
  s.lpart = (int32_t*)(b + L.lpart);
  s.leaf_chunk = (int4*)(b + L.leaf_chunk);
  s.leaf_c0 = (int32_t*)(b + L.leaf_c0);
  s.leaf_part = (double*)(b + L.leaf_part);
  return s;
}

// ------------------------------------------------------------ validation

inline const char* check_problem(const gbdtmo_problem* p) {
  if (!p) return "problem is NULL";
  if (p->n < 1 || p->n >= (int64_t(1) << 31)) return "n out of range [1, 2^31)";
  if (p->m < 1) return "m < 1";
  if (p->m_global < p->m || p->f_begin < 0 || p->f_begin + p->m > p->m_global) return "bad feature shard";
  if (p->d < 1 || p->d > 1024) return "d out of range [1, 1024]";
  if (p->B < 2 || p->B > 256) return "B out of range [2, 256]";
  if ((int64_t)p->m_global * p->B >= (int64_t(1) << 24)) return "m_global * B must be < 2^24";
  if (p->D < 1 || p->D > 12) return "D out of range [1, 12]";
  if (p->loss != GBDTMO_LOSS_MSE && p->loss != GBDTMO_LOSS_SOFTMAX) return "unknown loss";
  if (p->min_node < 1) return "min_node < 1";
  if (!(p->lambda >= 0.0)) return "lambda < 0";
  if (!(p->gamma >= 0.0)) return "gamma < 0";
  if (p->ld_bins < p->m || p->ld_bins % 8 != 0) return "ld_bins must be >= m and a multiple of 8";
  return nullptr;
}

// The diagonal shared-memory histogram variant (hist_diag.cu).
HistCfg hist_config_diag(const gbdtmo_problem& p);
gbdtmo_status launch_hist_diag(Ctx* ctx, const gbdtmo_problem& p, const uint8_t* bins, const int32_t* q,
                               const int32_t* rows, int use_rows, const State& s, int64_t* hist, int32_t* cnt,
                               bool no_cnt);
// The TMA-staged shared-memory histogram variant (hist_tma.cu).
bool hist_tma_supported(const gbdtmo_problem& p, const uint8_t* bins);
HistCfg hist_config_tma(const gbdtmo_problem& p, int max_smem);
gbdtmo_status launch_hist_tma(Ctx* ctx, const gbdtmo_problem& p, const uint8_t* bins, const int32_t* q,
                              const int32_t* rows, int use_rows, const State& s, int64_t* hist, int32_t* cnt);

// Histogram work items wanted per level -> chunks per build level (grad.cu).
int target_chunks_for(const Ctx* ctx, const gbdtmo_problem& p);
// Whether the sort-and-segment small-node search fits this problem (small.cu), the largest node
// its shared-memory staging holds, and the effective threshold min(option, cap).
bool small_supported(const gbdtmo_problem& p);
int64_t small_rows_cap(const gbdtmo_problem& p);
inline int64_t small_rows(const Ctx* ctx, const gbdtmo_problem& p) {
  if (ctx->small_max_rows <= 0 || !small_supported(p)) return 0;
  const int64_t cap = small_rows_cap(p);
  return ctx->small_max_rows < cap ? ctx->small_max_rows : cap;
}

// Launch helpers: count kernels and check errors.
#define GB_LAUNCH(kernel, grid, block, smem, ...)                 \
  do {                                                            \
    kernel<<<(grid), (block), (smem), ctx->stream>>>(__VA_ARGS__); \
    ctx->launches++;                                              \
    GB_CHECK_LAUNCH();                                            \
  } while (0)

}  // namespace gbdtmo
