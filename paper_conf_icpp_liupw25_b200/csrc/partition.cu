// partition.cu — (a)7: split decisions, stable partition of the row-index list, per-row node
// ids, and the next level's plan (Alg. 1 lines 14-17; reading R3, R4, R19).
//
// The row list is segmented by node.  A splitting node's rows move to [begin, begin + n_left)
// (bit = 1, left) and [begin + n_left, end) (right), both in their previous order, using a
// global left-count prefix over positions (3 passes: tile counts, tile scan, scatter).
#include "common.cuh"
#include "peer.cuh"
#include "plan.cuh"

namespace gbdtmo {

// Apply the merged records: decisions for the level's nodes, child nodes, next-level plan.
__global__ void __launch_bounds__(kPlanThreads)
k_apply_records(gbdtmo_problem p, int level, State s, const int64_t* __restrict__ xchg, int target_chunks,
                int64_t gmem_max_rows, int64_t small_max_rows, uint64_t* __restrict__ peer_hdr) {
  // peer exchange: both phases of this level are complete on this rank -> next epoch (peer.cuh).
  // After an expired wait the merged records may be partial: no node splits (the tree ends in
  // leaves, nothing is partitioned from inconsistent counts); the error stays recorded.
  const bool peer_failed = peer_hdr && *reinterpret_cast<volatile uint64_t*>(peer_hdr + PEER_ERROR) != 0;
  __syncthreads();
  if (peer_hdr && threadIdx.x == 0) peer_hdr[PEER_EPOCH] += 1;
  const int64_t LN = int64_t(1) << level, first = LN - 1;
  const int V = channels(p);
  const int64_t RW = rec_words(p);
  for (int64_t i = threadIdx.x; i < LN; i += blockDim.x) {
    const int64_t h = first + i;
    if (s.node_state[h] != GBDTMO_NODE_ACTIVE) continue;
    const int64_t* rec = xchg + i * RW;
    if (rec[V + 1] == 0 || peer_failed) {       // no valid split with gain > gamma: leaf
      s.node_state[h] = GBDTMO_NODE_LEAF;
      continue;
    }
    s.node_state[h] = GBDTMO_NODE_SPLIT;
    s.node_feat[h] = (int32_t)(rec[V + 1] - 1);
    s.node_bin[h] = (int32_t)rec[V + 2];
    s.node_gain[h] = __longlong_as_double(rec[V + 3]);
    const int64_t nl = rec[V];
    s.node_nleft[h] = nl;
    const int64_t hl = 2 * h + 1, hr = 2 * h + 2;
    const int32_t b = s.node_begin[h], e = s.node_end[h];
    s.node_begin[hl] = b; s.node_end[hl] = b + (int32_t)nl;
    s.node_begin[hr] = b + (int32_t)nl; s.node_end[hr] = e;
    const int64_t* S = s.node_sum + h * (V + 1);
    int64_t* SL = s.node_sum + hl * (V + 1);
    int64_t* SR = s.node_sum + hr * (V + 1);
    SL[V] = nl; SR[V] = S[V] - nl;                  // (the V channel sums: block-wide loop below)
    const bool deeper = level + 1 < p.D;
    const int64_t nr = (e - b) - nl;
    const bool al = deeper && nl >= 2 * (int64_t)p.min_node;
    const bool ar = deeper && nr >= 2 * (int64_t)p.min_node;
    s.node_state[hl] = al ? GBDTMO_NODE_ACTIVE : GBDTMO_NODE_LEAF;
    s.node_state[hr] = ar ? GBDTMO_NODE_ACTIVE : GBDTMO_NODE_LEAF;
    const bool left_small = nl <= nr;
    const int64_t hs = left_small ? hl : hr, hg = left_small ? hr : hl;
    const bool as = left_small ? al : ar, ag = left_small ? ar : al;
    int32_t ms = MODE_NONE, mg = MODE_NONE;
    if ((int64_t)(nl > nr ? nl : nr) <= small_max_rows) {   // both small: fused build + search, no subtraction
      ms = as ? MODE_SMALL : MODE_NONE;
      mg = ag ? MODE_SMALL : MODE_NONE;
    } else if (ag) { ms = MODE_BUILD; mg = MODE_DERIVE; }      // build the smaller, derive the larger
    else if (as) { ms = MODE_BUILD; }
    s.node_mode[hs] = ms;
    s.node_mode[hg] = mg;
  }
  __syncthreads();
  // children's exact channel sums, spread over the block (one thread per node and channel: with
  // V = 2 x 983 channels a per-node loop was ~0.2 ms per level)
  for (int64_t e = threadIdx.x; e < LN * V; e += blockDim.x) {
    const int64_t i = e / V;
    const int c = (int)(e - i * V);
    const int64_t h = first + i;
    if (s.node_state[h] != GBDTMO_NODE_SPLIT) continue;
    const int64_t* rec = xchg + i * RW;
    const int64_t S = s.node_sum[h * (V + 1) + c];
    s.node_sum[(2 * h + 1) * (V + 1) + c] = rec[c];
    s.node_sum[(2 * h + 2) * (V + 1) + c] = S - rec[c];
  }
  __syncthreads();
  plan_level_chunks(p, s, level + 1, target_chunks, gmem_max_rows);
}

__device__ __forceinline__ bool bitmap_bit(const int64_t* __restrict__ bm, int32_t r) {
  return (bm[r >> 6] >> (r & 63)) & 1;
}

// Block-wide exclusive scan for kPartThreads threads of int.
constexpr int kPartThreads = 256;
constexpr int kPartPer = kPartTile / kPartThreads;   // 8 positions per thread

__device__ __forceinline__ int part_block_scan(int v, int* total) {
  __shared__ int ws[kPartThreads / 32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) ws[w] = x;
  __syncthreads();
  if (w == 0) {
    int t = lane < kPartThreads / 32 ? ws[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int y = __shfl_up_sync(0xffffffffu, t, o);
      if (lane >= o) t += y;
    }
    if (lane < kPartThreads / 32) ws[lane] = t;
  }
  __syncthreads();
  const int base = w ? ws[w - 1] : 0;
  *total = ws[kPartThreads / 32 - 1];
  __syncthreads();
  return base + x - v;
}

// Flag of a position: 1 iff its row sits in a node of `level` that splits and goes left.
struct PosInfo { int32_t r; int32_t h; bool split; bool left; };

__device__ __forceinline__ PosInfo pos_info(const gbdtmo_problem& p, int level, const State& s,
                                            const int32_t* __restrict__ rows_in, const int64_t* __restrict__ bm,
                                            int64_t pos) {
  PosInfo pi;
  pi.r = rows_in[pos];
  pi.h = s.nid[pi.r];
  const int64_t first = (int64_t(1) << level) - 1;
  pi.split = pi.h >= first && pi.h < 2 * first + 1 && s.node_state[pi.h] == GBDTMO_NODE_SPLIT;
  pi.left = pi.split && bitmap_bit(bm, pi.r);
  return pi;
}

// Pass 1: per-tile left counts; lpart[h] = lefts in [tile start, begin_h) for node starts in the tile.
__global__ void __launch_bounds__(kPartThreads)
k_part_count(gbdtmo_problem p, int level, State s, const int32_t* __restrict__ rows_in, const int64_t* __restrict__ bm) {
  const int64_t t0 = (int64_t)blockIdx.x * kPartTile;
  const int64_t p0 = t0 + (int64_t)threadIdx.x * kPartPer;
  int flags[kPartPer];
  int local = 0;
#pragma unroll
  for (int i = 0; i < kPartPer; ++i) {
    flags[i] = 0;
    if (p0 + i < p.n) flags[i] = pos_info(p, level, s, rows_in, bm, p0 + i).left;
    local += flags[i];
  }
  int total;
  int excl = part_block_scan(local, &total);
#pragma unroll
  for (int i = 0; i < kPartPer; ++i) {
    const int64_t pos = p0 + i;
    if (pos < p.n) {
      PosInfo pi = pos_info(p, level, s, rows_in, bm, pos);
      if (pi.split && s.node_begin[pi.h] == pos) s.lpart[pi.h] = excl;
    }
    excl += flags[i];
  }
  if (threadIdx.x == 0) s.tile_cnt[blockIdx.x] = total;
}

// Pass 2: exclusive scan of the tile counts (single block).
__global__ void __launch_bounds__(kPartThreads) k_part_scan(int64_t ntiles, State s) {
  __shared__ int carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (int64_t b0 = 0; b0 < ntiles; b0 += kPartThreads) {
    const int64_t i = b0 + threadIdx.x;
    const int v = i < ntiles ? s.tile_cnt[i] : 0;
    int total;
    const int ex = part_block_scan(v, &total);
    if (i < ntiles) s.tile_cnt[i] = carry + ex;
    __syncthreads();
    if (threadIdx.x == 0) carry += total;
    __syncthreads();
  }
}

// Pass 3: scatter rows to their new positions, move node ids to the children.
__global__ void __launch_bounds__(kPartThreads)
k_part_scatter(gbdtmo_problem p, int level, State s, const int32_t* __restrict__ rows_in,
               int32_t* __restrict__ rows_out, const int64_t* __restrict__ bm) {
  const int64_t t0 = (int64_t)blockIdx.x * kPartTile;
  const int64_t p0 = t0 + (int64_t)threadIdx.x * kPartPer;
  PosInfo pi[kPartPer];
  int local = 0;
#pragma unroll
  for (int i = 0; i < kPartPer; ++i) {
    if (p0 + i < p.n) pi[i] = pos_info(p, level, s, rows_in, bm, p0 + i);
    else { pi[i].split = false; pi[i].left = false; pi[i].r = 0; pi[i].h = 0; }
    local += pi[i].left;
  }
  int total;
  int excl = part_block_scan(local, &total) + s.tile_cnt[blockIdx.x];
#pragma unroll
  for (int i = 0; i < kPartPer; ++i) {
    const int64_t pos = p0 + i;
    if (pos >= p.n) break;
    if (!pi[i].split) {
      rows_out[pos] = pi[i].r;
    } else {
      const int32_t h = pi[i].h;
      const int32_t b = s.node_begin[h];
      const int64_t lseg = (int64_t)s.tile_cnt[b / kPartTile] + s.lpart[h];
      const int64_t lrank = excl - lseg;                 // lefts of this node before pos
      int64_t dst;
      if (pi[i].left) {
        dst = b + lrank;
        s.nid[pi[i].r] = 2 * h + 1;
      } else {
        dst = b + s.node_nleft[h] + (pos - b - lrank);
        s.nid[pi[i].r] = 2 * h + 2;
      }
      if (dst >= 0 && dst < p.n) rows_out[dst] = pi[i].r;   // (always true for consistent records)
    }
    excl += pi[i].left;
  }
}

}  // namespace gbdtmo

using namespace gbdtmo;

static gbdtmo_status partition_impl(Ctx* ctx, const gbdtmo_problem* p, int32_t level, void* state,
                                    const int64_t* xchg, uint64_t* peer_hdr) {
  State s = state_view(*p, state);
  const int64_t* bm = xchg + bitmap_offset(*p);
  const int32_t* rows_in = (level & 1) ? s.rows1 : s.rows0;
  int32_t* rows_out = (level & 1) ? s.rows0 : s.rows1;
  const int64_t ntiles = part_tiles(*p);
  GB_LAUNCH(k_apply_records, 1, kPlanThreads, 0, *p, level, s, xchg, target_chunks_for(ctx, *p),
            ctx->gmem_max_rows, small_rows(ctx, *p), peer_hdr);
  GB_LAUNCH(k_part_count, (unsigned)ntiles, kPartThreads, 0, *p, level, s, rows_in, bm);
  GB_LAUNCH(k_part_scan, 1, kPartThreads, 0, ntiles, s);
  GB_LAUNCH(k_part_scatter, (unsigned)ntiles, kPartThreads, 0, *p, level, s, rows_in, rows_out, bm);
  return GBDTMO_OK;
}

extern "C" gbdtmo_status gbdtmo_partition(gbdtmo_ctx c, const gbdtmo_problem* p, int32_t level, void* state,
                                          const int64_t* xchg) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(level >= 0 && level < p->D, "level out of range [0, D)");
  GB_CHECK_ARG(state && xchg, "null pointer");
  return partition_impl(ctx, p, level, state, xchg, nullptr);
}

extern "C" gbdtmo_status gbdtmo_partition_peer(gbdtmo_ctx c, const gbdtmo_problem* p, int32_t level, void* state,
                                               int64_t* xchg_merged) {
  Ctx* ctx = (Ctx*)c;
  GB_ENTRY(ctx);
  if (!ctx) return GBDTMO_EINVAL;
  const char* bad = check_problem(p);
  GB_CHECK_ARG(!bad, bad ? bad : "");
  GB_CHECK_ARG(level >= 0 && level < p->D, "level out of range [0, D)");
  GB_CHECK_ARG(state && xchg_merged, "null pointer");
  GB_CHECK_ARG(peer_ready(ctx, *p), "peer group not connected for this problem shape (gbdtmo_peer_open/_connect)");
  const gbdtmo_status st = peer_gather(ctx, *p, level, xchg_merged);
  if (st != GBDTMO_OK) return st;
  return partition_impl(ctx, p, level, state, xchg_merged, reinterpret_cast<uint64_t*>(peer_own_window(ctx)));
}
