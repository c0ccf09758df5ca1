/*
 * gbdtmo.h — C ABI of the B200-native GBDT-MO hot path (libgbdtmo.so, sm_100a).
 *
 * Method: Liu, Peng, Wen, "Accelerating Multi-Output GBDTs with GPUs", ICPP'25
 * (/root/reference/PAPER.md, cited as PAPER.md:<line>).  Notation follows the paper:
 * n instances, m features, d outputs, B bins, maximum depth
 * D (Alg. 1's "d", renamed to avoid the clash with #outputs; reading R5),
 * lambda (l2 on leaves), gamma (split threshold, Alg. 1 input).
 *
 * One training tree (Algorithm 1, level-wise reading R6) is driven as
 *
 *     gbdtmo_grad                                   (g, h for every instance; tree init)
 *     for level = 0 .. D-1:
 *         gbdtmo_build_hist      (level)            (histograms of the nodes marked "build")
 *         gbdtmo_find_split      (level)            (sibling by subtraction + Eq. (3) + argmax)
 *         [N > 1: all-reduce MAX of `keys`, or fused: gbdtmo_split_record_peer below]
 *         gbdtmo_split_record    (level)            (owner: left sums + row-direction bitmap)
 *         [N > 1: all-reduce SUM of `xchg`]
 *         gbdtmo_partition       (level)            (decisions, stable partition, next level plan)
 *     gbdtmo_leaf_values
 *     gbdtmo_update_pred
 *
 * Every step is a hand-written CUDA kernel; there is no host fallback.  Nothing in a tree
 * synchronises with the host: every grid is sized from upper bounds and the per-level node
 * tables live in device memory (`state`), so a whole tree can be captured in a CUDA graph.
 *
 * Conventions
 *  - Pointers are DEVICE pointers unless marked (host).  The caller owns every buffer; the
 *    library never allocates device memory except inside gbdtmo_create (nothing) — sizes
 *    of caller-provided scratch come from the *_bytes queries below.
 *  - All calls are asynchronous on the context's stream (gbdtmo_set_stream; default: the
 *    legacy stream 0).  They validate arguments first (GBDTMO_EINVAL, nothing launched),
 *    then launch and check cudaGetLastError (GBDTMO_ECUDA).  gbdtmo_last_error() returns a
 *    context-owned message valid until the next call on that context.  No exceptions cross
 *    the ABI and nothing calls exit/abort.  Outputs of a failed call are unspecified;
 *    inputs are never written.
 *  - One context per host thread per device.
 *  - Fixed point: per tree and per channel c the gradient is stored
 *    as q = rint(g * 2^30 / P_c), P_c = 2^ceil(log2 max_i |g_ic|) (a power of two, so the
 *    dequantisation q * scale_c with scale_c = P_c * 2^-30 is exact in fp64).  Histograms
 *    are exact int64 sums of q; parent = left + right holds exactly and results do not
 *    depend on the GPU count or the summation order.
 */
#ifndef GBDTMO_H
#define GBDTMO_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GBDTMO_ABI_VERSION 2   /* 2: gbdtmo_predict takes m; gbdtmo_peer_status_async */

typedef enum {
  GBDTMO_OK = 0,
  GBDTMO_EINVAL = 1,       /* bad argument; nothing launched                              */
  GBDTMO_ECUDA = 2,        /* CUDA launch / runtime error (message in gbdtmo_last_error)  */
  GBDTMO_ENOMEM = 3,       /* caller-provided scratch too small                           */
  GBDTMO_EUNSUPPORTED = 5  /* shape outside the supported envelope (see each call)        */
} gbdtmo_status;

typedef enum {
  GBDTMO_LOSS_MSE = 0,     /* l = sum_k (yhat_k - y_k)^2: g = 2(yhat - y), h = 2        */
  GBDTMO_LOSS_SOFTMAX = 1  /* softmax cross-entropy (reading R12): g = p - y, h = p(1-p) */
} gbdtmo_loss;

/* Node state in the heap-indexed tree record (root 0, children 2i+1, 2i+2). */
enum { GBDTMO_NODE_NONE = 0, GBDTMO_NODE_SPLIT = 1, GBDTMO_NODE_LEAF = 2, GBDTMO_NODE_ACTIVE = 3 };

typedef struct gbdtmo_ctx_s* gbdtmo_ctx;

/* Problem description, passed by (host) pointer to every tree call.
 *   channels V = d (MSE: g only; h = 2 is implicit, H = 2 * count) or 2d (softmax: g then h). */
typedef struct {
  int64_t n;          /* instances (rows), 1 <= n < 2^31                                     */
  int32_t m;          /* features held by this process (its shard), 1 <= m                  */
  int32_t f_begin;    /* global id of local feature 0 (feature partitioning)   */
  int32_t m_global;   /* total features over all processes; m_global * B < 2^24             */
  int32_t d;          /* outputs, 1 <= d <= 1024                                             */
  int32_t B;          /* maximum bins per feature, 2 <= B <= 256 (bins are uint8)            */
  int32_t D;          /* maximum depth, 1 <= D <= 12                                         */
  int32_t loss;       /* gbdtmo_loss                                                         */
  int32_t min_node;   /* minimum instances per node (reading R4), >= 1         */
  double lambda;      /* > 0; 0 allowed for tests (H > 0 required then)       */
  double gamma;       /* >= 0; a node splits iff its best gain > gamma (reading R2, R3)      */
  double lr;          /* learning rate applied to leaf values (reading R9)     */
  int64_t ld_bins;    /* row stride of the bins matrix in bytes, multiple of 8, >= m         */
} gbdtmo_problem;

/* ------------------------------------------------------------------ lifecycle */

int           gbdtmo_abi_version(void);
gbdtmo_status gbdtmo_create(int device, gbdtmo_ctx* out /* host */);
gbdtmo_status gbdtmo_destroy(gbdtmo_ctx ctx);
gbdtmo_status gbdtmo_set_stream(gbdtmo_ctx ctx, void* cuda_stream /* cudaStream_t */);
const char*   gbdtmo_last_error(gbdtmo_ctx ctx);
/* Context options (apply to subsequent calls on the context):
 *   GBDTMO_OPT_GMEM_MAX_ROWS: histogram variant selection — BUILD nodes with at most this many
 *     rows use the global-atomic variant (one REDG per (row, feature, channel) into the node's
 *     histogram) instead of the shared-memory privatised variant;
 *     0 (default) = shared memory for every node.  The threshold comes from measurement
 *     (tools/calibrate_hist.py).
 *   GBDTMO_OPT_SMALL_MAX_ROWS: fused small-node path — when both children of a split have at most
 *     this many rows they are marked SMALL: built from their rows and searched in shared memory by
 *     gbdtmo_search_small, never materialised and not derived by subtraction (reading R27);
 *     0 (default) = off.  Requires d <= 32 and a feature tile that fits shared memory.
 *   GBDTMO_OPT_HIST_KERNEL: shared-memory histogram lane mapping — 0 (default): channel tiles of
 *     K = 4/8/16 with 32/K rows per instruction; 1: "diagonal" channel tiles of 4, eight rows per
 *     instruction each adding to a different slot, conflict-free for any channel count (DESIGN.md
 *     §7); 2: row-pair tiles whose bin windows are staged in shared memory by TMA gather4
 *     (measured slower, kept as the recorded alternative).  Same results; chosen per workload
 *     shape by measurement.  1 and 2 are not used with default bins.
 *   GBDTMO_OPT_FS_CHANNEL_GROUPS: split search parallelism (gbdtmo_find_split, B > 128, no default
 *     bins) — 0 (default): automatic: a level whose (node, feature) warps would not fill the GPU
 *     (fewer than 32 / CG warps per SM) splits every (node, feature)'s channel loop over CG = 2, 4
 *     or 8 warp pairs whose Eq. (3) partial sums are added in shared memory in a fixed order; 1:
 *     never; 2 / 4 / 8: always, with that CG (at most d).  Same (f, b) decisions up to near-ties;
 *     gains differ by fp64 summation order.
 *   GBDTMO_OPT_HIST_WAVES: histogram work items wanted per level, in multiples of the SM count
 *     (a level's BUILD rows are cut into chunks so that chunks x tiles reaches it); 0 (default) = 2.
 *     Fewer waves leave more nodes to a single chunk (sole-writer flushes, no zeroing); chosen per
 *     shape by measurement (tools/calibrate_hist.py).  Same results. */
enum { GBDTMO_OPT_GMEM_MAX_ROWS = 1, GBDTMO_OPT_SMALL_MAX_ROWS = 2, GBDTMO_OPT_HIST_KERNEL = 3,
       GBDTMO_OPT_PEER_TIMEOUT_MS = 4 /* bound of every peer-flag wait (gbdtmo_peer_*), default 30000 */,
       GBDTMO_OPT_FS_CHANNEL_GROUPS = 5, GBDTMO_OPT_HIST_WAVES = 6 };
gbdtmo_status gbdtmo_set_option(gbdtmo_ctx ctx, int32_t option, int64_t value);
/* Cached root counts.  The root holds all n rows in every tree, so its count histogram
 * cnt[0][f][b] = #{i : bin(i, f) = b} (PAPER.md:214's histogram, count channel) is the same for
 * every tree of a dataset.  root_cnt: int32 [m][B] device, e.g. a copy of the level-0 `cnt` of
 * the first tree (after gbdtmo_find_split, which completes default-bin counts); owned by the
 * caller, must stay valid while set; NULL (default) disables.  While set, gbdtmo_build_hist at
 * level 0 copies it into `cnt` and skips the count accumulation (not with histogram kernel 2 or
 * when the root would use the global-atomic variant).  Results are identical. */
gbdtmo_status gbdtmo_set_root_counts(gbdtmo_ctx ctx, const int32_t* root_cnt);
/* Number of kernels this context has launched so far (for launch accounting). */
int64_t       gbdtmo_launch_count(gbdtmo_ctx ctx);

/* ------------------------------------------------------------- size queries (host) */

/* Bytes of the bins buffer: n rows of ld_bins bytes plus 32 bytes of read slack
 * (the histogram kernel loads 8-byte-aligned windows of up to 32 bytes per row).  Bytes past column
 * m of a row and the slack are read but never used; zero them (once) for sanitizer-clean runs. */
size_t gbdtmo_bins_bytes(int64_t n, int64_t ld_bins);
/* Scratch needed by gbdtmo_bin for n rows and m columns. */
size_t gbdtmo_bin_workspace_bytes(int64_t n, int32_t m, int32_t B);
/* Opaque per-tree state (row lists, per-row node ids, heap node tables, launch plans). */
gbdtmo_status gbdtmo_state_bytes(const gbdtmo_problem* p, size_t* bytes /* host */);
/* Histogram buffers of one level: hist int64 [S][m][V][B] (channel-major: bins contiguous),
 * cnt int32 [S][m][B], S = 2^level slots, except at the last level (level = D-1 > 0), where only
 * the built child of each sibling pair is materialised and S = 2^(D-2): node `slot` of that level
 * lives in slot >> 1. */
gbdtmo_status gbdtmo_hist_bytes(const gbdtmo_problem* p, int32_t level, size_t* hist_bytes, size_t* cnt_bytes);
/* Exchange buffer (int64 elements): 2^(D-1) split records of V+4 words, then ceil(n/64) bitmap words. */
gbdtmo_status gbdtmo_xchg_count(const gbdtmo_problem* p, int64_t* count /* host */);

/* --------------------------------------------------------------- (a)1 binning */

/* Per-feature quantile binning ("feature-value bin mapping", "cut points"
 * PAPER.md:166, at most B bins PAPER.md:237, 255; exact rule = reading R14):
 *   s = sorted column; if it has <= B distinct values the cuts are every distinct value but
 *   the smallest, else c_j = s[floor(j n / B)], j = 1..B-1, deduplicated, those <= s[0] dropped;
 *   bin(x) = #{cuts <= x}.
 * X       float32 row-major, element (i, f) at X[i*ld_x + f]; finite values (-0.0 == +0.0).
 * bins    uint8, element (i, f) at bins[i*ld_bins + f]; only columns [0, m) are written.
 * cuts    float32 [m][B-1], ascending, +inf padded.      nbins int32 [m] = #cuts + 1.
 * ws      scratch of gbdtmo_bin_workspace_bytes(n, m, B) bytes.
 * Columns are independent: a column slice of a larger matrix may be binned by offsetting
 * X, bins, cuts and nbins.  EUNSUPPORTED if B > 256. */
gbdtmo_status gbdtmo_bin(gbdtmo_ctx ctx, const float* X, int64_t n, int32_t m, int64_t ld_x, int32_t B,
                         uint8_t* bins, int64_t ld_bins, float* cuts, int32_t* nbins,
                         void* ws, size_t ws_bytes);

/* The same binning from a HOST matrix (the e2e entry point: the caller's data never needs to fit the
 * device): X_host float32 row-major [n][ld_x] in host memory (pinned for asynchronous copies; pageable
 * works, synchronously); the columns are uploaded in strips of `strip` columns on a copy stream owned
 * by the context while the previous strip is binned on the context's stream (two staging buffers in
 * ws).  bins, cuts, nbins: device, as for gbdtmo_bin.  ws: device, 256-byte aligned,
 * gbdtmo_bin_host_workspace_bytes(n, m, B, strip) bytes.  Returns when everything is enqueued; the
 * host matrix must stay valid until the context's stream has passed this call. */
size_t gbdtmo_bin_host_workspace_bytes(int64_t n, int32_t m, int32_t B, int32_t strip);
gbdtmo_status gbdtmo_bin_host(gbdtmo_ctx ctx, const float* X_host, int64_t n, int32_t m, int64_t ld_x, int32_t B,
                              uint8_t* bins, int64_t ld_bins, float* cuts, int32_t* nbins, void* ws, size_t ws_bytes,
                              int32_t strip);

/* The same binning from the paper's sparse storage (Compressed Sparse Column:
 * "values", "row_indices", "col_pointers"; entries not stored are 0).  Result identical to
 * gbdtmo_bin on the dense matrix.  The implicit zeros are never materialised: they join the
 * selection counts per column and fill the bins before the stored values are scattered.
 * values       float32 [nnz] (device), column by column; explicit zeros allowed
 * row_idx      int32 [nnz] (device), row of each value; at most one entry per (row, column)
 *              (duplicates: undefined result)
 * col_ptr      int64 [m+1] (device), column j holds entries [col_ptr[j], col_ptr[j+1])
 * col_ptr_host the same array in host memory (validated; sizes the launches)
 * bins, cuts, nbins, ws as for gbdtmo_bin (ws of gbdtmo_bin_workspace_bytes(n, m, B) bytes).
 * EINVAL if col_ptr[0] != 0, it decreases, or a column holds more than n entries. */
gbdtmo_status gbdtmo_bin_csc(gbdtmo_ctx ctx, const float* values, const int32_t* row_idx, const int64_t* col_ptr,
                             const int64_t* col_ptr_host, int64_t n, int32_t m, int32_t B, uint8_t* bins,
                             int64_t ld_bins, float* cuts, int32_t* nbins, void* ws, size_t ws_bytes);

/* Sparsity-aware default bins (zeros are implicit in the paper's CSC
 * storage; here every feature's most frequent bin plays that role): dflt[f] = the bin of feature
 * f holding the most of the n rows (ties: smallest bin), or -1 when that bin holds fewer than
 * min_count rows.  The histogram calls skip rows whose bin is the default and recover that bin
 * exactly as node total - sum of the other bins.
 * bins as produced by gbdtmo_bin; dflt int32 [m] (out). */
gbdtmo_status gbdtmo_default_bins(gbdtmo_ctx ctx, const uint8_t* bins, int64_t n, int32_t m, int64_t ld_bins,
                                  int32_t B, int64_t min_count, int32_t* dflt);

/* ------------------------------------------------------------ (a)2 gradients */

/* First/second derivatives per output (softmax reading R12, diagonal
 * Hessian PAPER.md:96), quantised to fixed point, plus initialisation of the tree state:
 *   y      float32 [n][d]   targets (softmax: one-hot or any row summing to 1)
 *   pred   float64 [n][d]   current prediction yhat (sum of previous trees)
 *   q      int32   [n][V]   out: q[i][c] (MSE: g; softmax: g for c < d, h for c >= d)
 *   scales float32 [V]      out: dequantisation factor P_c * 2^-30 (a power of two)
 *   gh     float64 [n][V]   out, may be NULL: the fp64 g (and softmax h) before quantisation, for
 *                           gbdtmo_leaf_values' fp64 leaf sums
 *   state  gbdtmo_state_bytes(p) bytes, out: root node = all rows (sums of q = exact int64),
 *          per-row node ids = root, level-0 build plan. */
gbdtmo_status gbdtmo_grad(gbdtmo_ctx ctx, const gbdtmo_problem* p, const float* y, const double* pred,
                          int32_t* q, float* scales, void* state, double* gh /* may be NULL */);

/* ------------------------------------------------------ (a)3 histogram build */

/* For every node of `level` marked "build" by the plan in `state` (the root at level 0, the
 * smaller child of each split afterwards, reading R19), for every local feature f, bin b and
 * channel c:   hist[slot][f][c][b] = sum_{i in node, bin(i,f) = b} q[i][c]   (exact int64),
 *              cnt [slot][f][b]    = #{i in node : bin(i,f) = b}.
 * (§3.3; the paper's Alg. 2 body is missing.)
 * bins uint8 with ld = p->ld_bins and gbdtmo_bins_bytes() of storage; q from gbdtmo_grad;
 * hist / cnt: this level's buffers (gbdtmo_hist_bytes(level)); slot = node index within the
 * level (heap id - (2^level - 1)), stored at slot >> 1 on the last level.  Slots not built are
 * left untouched.
 * dflt (may be NULL): per-feature default bins (gbdtmo_default_bins); rows in a feature's
 * default bin are not accumulated and that bin's entries are left undefined until
 * gbdtmo_find_split recovers them from the node totals. */
gbdtmo_status gbdtmo_build_hist(gbdtmo_ctx ctx, const gbdtmo_problem* p, int32_t level,
                                const uint8_t* bins, const int32_t* dflt, const int32_t* q, void* state,
                                int64_t* hist, int32_t* cnt);

/* Tile-packed bins for the histogram kernel (DESIGN.md §7 "Packed bins"; the B200 form of the
 * paper's "bin packing").  The shared-memory histogram kernel works on tiles of k
 * features (k from the problem's shape, at most 8 for a packed layout); with the row-major
 * matrix every row of a tile is its own cache line, so a warp's 32 gathered rows cost 32-64 L1
 * wavefronts per load.  The packed copy stores each tile's bins contiguously per row:
 *   packed uint8 [ceil(n_tiles/4)][n][4][8]:
 *     packed[(((t / 4) * n + i) * 4 + t % 4) * 8 + j] = bins[i * ld + k t + j]  (j < k),
 *     0 for j >= k or k t + j >= m,
 * so one row's bins for 4 consecutive tiles are one 32-byte sector and adjacent rows are adjacent
 * sectors.  gbdtmo_packed_bins_bytes: bytes of `packed`, 0 when
 * the problem's tiles are wider than 8 features (then use gbdtmo_build_hist).  The caller owns
 * `packed`; gbdtmo_pack_bins fills it from `bins` (once per dataset and problem shape).
 * gbdtmo_build_hist_packed = gbdtmo_build_hist reading the tile bins from `packed` (and `bins`
 * for the global-atomic small-node variant); identical results. */
size_t gbdtmo_packed_bins_bytes(const gbdtmo_problem* p);
gbdtmo_status gbdtmo_pack_bins(gbdtmo_ctx ctx, const gbdtmo_problem* p, const uint8_t* bins, uint8_t* packed);
gbdtmo_status gbdtmo_build_hist_packed(gbdtmo_ctx ctx, const gbdtmo_problem* p, int32_t level,
                                       const uint8_t* bins, const uint8_t* packed, const int32_t* dflt,
                                       const int32_t* q, void* state, int64_t* hist, int32_t* cnt);

/* Histograms from the paper's sparse storage (§3.2; NEXT-1), column-wise as the
 * paper distributes the work: the same hist / cnt result as gbdtmo_build_hist
 * (no default bins), built from the stored (non-zero) entries only:
 *   hist[slot][f][c][b] = sum_{i in node, x_if stored, bin(i,f) = b != zbin[f]} q[i][c],  cnt likewise,
 * then the zero bin of every feature (the implicit zeros and stored values binned with them) is
 * filled in as node total - other bins (exact).  Work is proportional to nnz plus one pass over the
 * built histograms.  All BUILD nodes of the level are zeroed and accumulated with global atomics
 * (no shared-memory tiles, no root-count cache).
 * col_ptr  int64 [m+1] (device), row_idx int32 [nnz] (device), nz_bins uint8 [nnz] (device: the bin
 *          of each stored value, gbdtmo_csc_nz_bins), nnz = col_ptr[m] (host copy, sizes the grid)
 * zbin     int32 [m] (device): bin of the value 0 per feature (gbdtmo_csc_nz_bins). */
gbdtmo_status gbdtmo_build_hist_csc(gbdtmo_ctx ctx, const gbdtmo_problem* p, int32_t level, const int64_t* col_ptr,
                                    const int32_t* row_idx, const uint8_t* nz_bins, int64_t nnz, const int32_t* zbin,
                                    const int32_t* q, void* state, int64_t* hist, int32_t* cnt);
/* Bins of the stored CSC values, gathered from the matrix gbdtmo_bin_csc wrote (nz_bins[e] =
 * bins[row_idx[e] * ld_bins + f] for e in column f), and zbin[f] = bin(0) = #{cuts[f] <= 0} (R14).
 * All pointers device; nz_bins uint8 [nnz] out, zbin int32 [m] out. */
gbdtmo_status gbdtmo_csc_nz_bins(gbdtmo_ctx ctx, int32_t m, int32_t B, const int64_t* col_ptr, const int32_t* row_idx,
                                 const uint8_t* bins, int64_t ld_bins, const float* cuts, uint8_t* nz_bins,
                                 int32_t* zbin);

/* ------------------------------------- (a)4 subtraction + (a)5 split search */

/* For every active node of `level`:
 *   - if marked "derive": hist = parent_hist[parent] - hist[sibling] (and cnt likewise),
 *     written to its slot when level < D-1 (it is a parent at the next level);
 *   - for every local feature f and candidate bin b in [0, nbins[f]-2] (left = bins <= b,
 *     reading R15): G_L, H_L, C_L by prefix sums over bins, valid iff
 *     C_L >= min_node and C_R >= min_node (R4), gain by Eq. (3) in fp64;
 *   - keys[slot] = max over candidates with gain > gamma of
 *       (bits(gain) & ~0xFFFFFF) | (0xFFFFFF - (f_global * B + b))
 *     (0 if none): larger gain wins, ties -> smallest (f, b) (reading R16); the same key is
 *     max-reduced across GPUs.
 * nbins int32 [m] (local features); scales from gbdtmo_grad; keys uint64 [2^level] (out,
 * every slot written).  parent_hist / parent_cnt: level-1 buffers (ignored at level 0).
 * dflt (may be NULL, must match gbdtmo_build_hist's): the default bin of every feature is
 * recomputed as node total - sum of the other bins and written back to the node's histogram. */
gbdtmo_status gbdtmo_find_split(gbdtmo_ctx ctx, const gbdtmo_problem* p, int32_t level,
                                const int32_t* nbins, const int32_t* dflt, const float* scales, void* state,
                                int64_t* hist, int32_t* cnt,
                                const int64_t* parent_hist, const int32_t* parent_cnt,
                                uint64_t* keys);

/* (a)3 + (a)5 fused for small nodes: for every node of `level` marked SMALL (see
 * GBDTMO_OPT_SMALL_MAX_ROWS) build its histograms from its rows in shared memory and evaluate
 * Eq. (3) in place, max-reducing the packed keys into keys[slot] (same key and tie rule as
 * gbdtmo_find_split); nothing is written to the global histograms.  Call after
 * gbdtmo_find_split (which zeroes keys) and before the key exchange.  No-op when the option is 0. */
gbdtmo_status gbdtmo_search_small(gbdtmo_ctx ctx, const gbdtmo_problem* p, int32_t level,
                                  const uint8_t* bins, const int32_t* q, const int32_t* nbins,
                                  const float* scales, void* state, uint64_t* keys);

/* ------------------------------------------------------------ (a)6 exchange */

/* Split records of `level`, written by the process that owns each winning feature
 * (all-zero elsewhere, so a SUM all-reduce across processes merges them):
 *   xchg[slot*(V+4) + c]   = G_L sums (int64 fixed point) at the winner, c < V
 *   xchg[slot*(V+4) + V]   = C_L
 *   xchg[slot*(V+4) + V+1] = winning global feature + 1 (0: node does not split)
 *   xchg[slot*(V+4) + V+2] = winning bin
 *   xchg[slot*(V+4) + V+3] = bits of the fp64 gain
 *   xchg[2^(D-1)*(V+4) + w] bitmap: bit (i & 63) of word (i >> 6) = 1 iff instance i sits in a
 *                            splitting node of this level and goes left (bin <= b).
 * keys: this level's keys after the (optional) MAX all-reduce; scales from gbdtmo_grad;
 * hist / cnt / parent_hist / parent_cnt as for gbdtmo_find_split (a derived winner's sums are
 * parent - sibling); q from gbdtmo_grad (the left sums of a SMALL winner are summed from its
 * rows).  Every xchg word is written. */
gbdtmo_status gbdtmo_split_record(gbdtmo_ctx ctx, const gbdtmo_problem* p, int32_t level,
                                  const uint8_t* bins, const int32_t* dflt, const int32_t* q,
                                  const float* scales, void* state,
                                  const int64_t* hist, const int32_t* cnt,
                                  const int64_t* parent_hist, const int32_t* parent_cnt,
                                  const uint64_t* keys, int64_t* xchg);

/* ------------------------------------------------------------ (a)7 partition */

/* Applies the (merged) split records of `level` (Alg. 1 lines 14-17):
 * nodes with a record split, the others become leaves; the rows of each splitting node are
 * stably partitioned into left (bit = 1) then right, preserving their order; per-row node ids
 * move to the children; children get exact sums (left = record, right = parent - left), the
 * state ACTIVE if level+1 < D and they hold >= 2*min_node rows (else LEAF); the smaller child
 * (ties: left) is marked "build", the larger "derive" (reading R19); the next level's build
 * plan is written.  Identical on every process given identical xchg. */
gbdtmo_status gbdtmo_partition(gbdtmo_ctx ctx, const gbdtmo_problem* p, int32_t level, void* state,
                               const int64_t* xchg);

/* ------------------------------------------------------------ (a)8, (a)9 */

/* Leaf values: for every heap node in state LEAF,
 *   leaf[h][k] = -lr * G_k / (H_k + lambda)         (MSE: H = 2 * count);
 * other heap nodes get 0.  leaf float64 [2^(D+1)-1][d].
 * With gh (gbdtmo_grad's fp64 g / h of this tree): G, H are fp64 sums over the leaf's rows (reading
 * R17) in a fixed order (deterministic, identical on every rank) -- the oracle's definition up to
 * summation order.  With gh = NULL: G, H from the exact fixed-point node sums (scales from
 * gbdtmo_grad), whose absolute resolution is n_leaf P 2^-31 (R29). */
gbdtmo_status gbdtmo_leaf_values(gbdtmo_ctx ctx, const gbdtmo_problem* p, const float* scales, void* state,
                                 const double* gh /* may be NULL */, double* leaf);

/* Incremental prediction (rows read their leaf directly, no traversal):
 *   pred[i][k] += leaf[node_of(i)][k]   for every instance i.   pred float64 [n][d] in/out
 * (fp64 so that the prediction does not drift from the fp64 definition over many trees). */
gbdtmo_status gbdtmo_update_pred(gbdtmo_ctx ctx, const gbdtmo_problem* p, const void* state,
                                 const double* leaf, double* pred);

/* Copy of the tree record (heap-indexed, 2^(D+1)-1 entries each) out of `state`:
 * node_state (GBDTMO_NODE_*), feature (global id, -1 if none), bin, gain (fp64),
 * n_rows, n_left, and threshold = cuts[f][bin] (float32, x < threshold goes left, reading R15)
 * for split features held by this process (0 elsewhere: a SUM across processes merges them).
 * cuts: gbdtmo_bin's [m][B-1] of the local features (may be NULL when threshold is NULL).
 * Any output pointer may be NULL. */
gbdtmo_status gbdtmo_tree_export(gbdtmo_ctx ctx, const gbdtmo_problem* p, const void* state,
                                 int32_t* node_state, int32_t* feature, int32_t* bin, double* gain,
                                 int64_t* n_rows, int64_t* n_left, const float* cuts, float* threshold);

/* Inference for unseen instances ("instance-level and tree-level parallelism";
 * SURVEY NEXT-3): for every row i and tree t = 0..T-1 in order, walk from the root: at a SPLIT node
 * go left iff X[i][feature] < threshold (reading R15), at a LEAF add its value:
 *   pred[i][k] += leaf[t][h][k]      (fp64, trees added in order t = 0, 1, ..., so the predictions of
 *                                     training rows equal the training path's pred bit for bit).
 * X float32 row-major [n][ld_x] over ALL (global) features 0..m-1 (m <= ld_x); node_state / feature
 * int32 [T][NH], threshold float32 [T][NH], leaf float64 [T][NH][d] as exported per tree
 * (gbdtmo_tree_export; NH = 2^(D+1)-1, 1 <= D <= 12); pred float64 [n][d] in/out (start from zeros
 * for a fresh prediction).  Rows are staged in shared memory in tiles (m <= ~40k features; wider
 * rows are read from global memory); (row, tree) pairs walk concurrently.  A split on a feature
 * >= m ends that walk without adding (malformed model). */
gbdtmo_status gbdtmo_predict(gbdtmo_ctx ctx, const float* X, int64_t n, int32_t m, int64_t ld_x, int32_t T,
                             int32_t D, int32_t d, const int32_t* node_state, const int32_t* feature,
                             const float* threshold, const double* leaf, double* pred);

/* Copy of the row bookkeeping out of `state` (tests, debugging): the row-index list as seen by
 * `level` (level = D: after the last partition), int32 [n]; the heap node of every instance,
 * int32 [n]; and the [begin, end) positions of every heap node in that list, int32 [2^(D+1)-1]
 * each.  Any output pointer may be NULL. */
gbdtmo_status gbdtmo_rows_export(gbdtmo_ctx ctx, const gbdtmo_problem* p, const void* state, int32_t level,
                                 int32_t* rows, int32_t* node_of_row, int32_t* node_begin, int32_t* node_end);

/* ------------------------------------- (e) / NEXT-4: fused peer-memory exchange (multi-GPU)
 *
 * The feature-partitioned scheme (each GPU owns a feature shard, finds its best
 * split, the global best is agreed across GPUs) without host-issued collectives.  Every rank
 * owns one "window" of device memory, allocated by the library and mapped by all ranks through
 * CUDA IPC (NVLink / NVSwitch peer loads on a multi-GPU box).  Per level:
 *   gbdtmo_find_split / gbdtmo_search_small   with keys = this level's window keys
 *                                              (gbdtmo_peer_buffers): written in place;
 *   gbdtmo_split_record_peer                   its kernel publishes a flag, waits for every
 *                                              peer's, and takes each node's key as the max over
 *                                              the N windows (= MAX all-reduce), then writes the
 *                                              owner's records + bitmap into the own window;
 *   gbdtmo_partition_peer                      its first kernel publishes / waits likewise and
 *                                              sums the N windows' records + bitmaps (= SUM
 *                                              all-reduce) into xchg_merged, then partitions.
 * Results are identical to the all-reduce path (same keys, same sums).  Flags are epoch counters
 * kept in device memory, so trees captured in CUDA graphs replay correctly.  Waits are bounded
 * (GBDTMO_OPT_PEER_TIMEOUT_MS); an expired wait records an error and the kernel continues (its
 * outputs are then invalid) — check gbdtmo_peer_status after a run.  Windows are per level:
 * peer_window_bytes = 512 + 8 D 2^(D-1) + 8 D xchg_count (rounded).
 *
 * gbdtmo_peer_open: allocates and zeroes this rank's window for problems of p's shape (n, D,
 *   channels), returns its IPC handle (host, GBDTMO_PEER_HANDLE_BYTES bytes).  Collective in
 *   the sense that every rank must open before any rank connects.  1 <= world <= 8.
 * gbdtmo_peer_connect: handles = the world handles in rank order (host, world * 64 bytes;
 *   the caller exchanges them, e.g. with torch.distributed all_gather); maps the peers' windows.
 * gbdtmo_peer_buffers: this rank's keys [2^(D-1)] / xchg [xchg_count] of `level` in its window
 *   (host out: device pointers, owned by the context; either pointer may be NULL).
 * gbdtmo_peer_status: synchronous read of the window's epoch (exchanges completed) and error
 *   word (0 = none; else (epoch << 8) | phase, phase 1 = keys, 2 = records).
 * gbdtmo_peer_close: unmaps and frees (also done by gbdtmo_destroy).  Synchronises the device. */
#define GBDTMO_PEER_HANDLE_BYTES 64
size_t        gbdtmo_peer_window_bytes(const gbdtmo_problem* p);
gbdtmo_status gbdtmo_peer_open(gbdtmo_ctx ctx, const gbdtmo_problem* p, int32_t rank, int32_t world,
                               uint8_t* handle /* host out, 64 bytes */);
gbdtmo_status gbdtmo_peer_connect(gbdtmo_ctx ctx, const uint8_t* handles /* host, world * 64 bytes */);
gbdtmo_status gbdtmo_peer_buffers(gbdtmo_ctx ctx, const gbdtmo_problem* p, int32_t level,
                                  uint64_t** keys /* host out */, int64_t** xchg /* host out */);
gbdtmo_status gbdtmo_peer_status(gbdtmo_ctx ctx, int64_t* epoch /* host */, int64_t* error /* host */);
/* gbdtmo_peer_status_async: the same two words (epoch, error) copied asynchronously on the
 *   context's stream into out[0], out[1] (int64; pinned host or device memory, caller-owned), so
 *   a driver can check the error word once per tree without a device synchronisation. */
gbdtmo_status gbdtmo_peer_status_async(gbdtmo_ctx ctx, int64_t* out /* 2 words */);
gbdtmo_status gbdtmo_peer_close(gbdtmo_ctx ctx);
/* gbdtmo_split_record with the key exchange fused in: keys are read from every window (no
 * `keys` argument), records and bitmap go to the own window (no `xchg` argument); keys_merged
 * uint64 [2^level] (out) receives the agreed keys. */
gbdtmo_status gbdtmo_split_record_peer(gbdtmo_ctx ctx, const gbdtmo_problem* p, int32_t level,
                                       const uint8_t* bins, const int32_t* dflt, const int32_t* q,
                                       const float* scales, void* state,
                                       const int64_t* hist, const int32_t* cnt,
                                       const int64_t* parent_hist, const int32_t* parent_cnt,
                                       uint64_t* keys_merged);
/* gbdtmo_partition with the record exchange fused in: xchg_merged int64 [xchg_count] (out)
 * receives the sum over the windows, then the level is partitioned from it. */
gbdtmo_status gbdtmo_partition_peer(gbdtmo_ctx ctx, const gbdtmo_problem* p, int32_t level, void* state,
                                    int64_t* xchg_merged);

#ifdef __cplusplus
}
#endif
#endif /* GBDTMO_H */
