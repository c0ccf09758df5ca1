/*
 * oracle.h — plain, slow, obviously-correct CPU oracle for the GBDT-MO hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_icpp_liupw25_b200/, include/gbdtmo.h) never includes, links or
 * calls anything under oracle/, and this file shares no code, header, table or
 * constant with the CUDA path.
 *
 * Everything is fp64, in the paper's notation (Liu, Peng, Wen, "Accelerating
 * Multi-Output GBDTs with GPUs", ICPP'25 = /root/reference/PAPER.md):
 *   n instances, m features, d outputs (§2.2), B bins,
 *   depth D (Alg. 1 "d: the maximum depth"; renamed D, R5).
 * Readings of passages the paper leaves silent/garbled are DESIGN.md "Readings" R1..R24.
 *
 * Layouts: bins are COLUMN-major uint16 [m][n] (feature f at bins + f*n), g/h/y/pred
 * row-major [n][d], histograms [m][B][d] (HG, HH) and [m][B] (CNT).
 *
 * Parity status per function:
 *   oracle_bin            pinned  (closed form on permutations; distinct-value rank)
 *   oracle_csc_from_dense pinned  (the paper's worked example, tests/golden/)
 *   oracle_dense_from_csc pinned  (same example; round trip)
 *   oracle_grad           pinned  (finite differences of the loss; softmax invariants)
 *   oracle_build_hist     pinned  (row-sum invariants, exact dyadic parent = L + R, brute force)
 *   oracle_find_split     pinned  (exhaustive raw-threshold enumeration; sklearn CART, MSE λ=0)
 *   oracle_partition      pinned  (Python stable sort)
 *   oracle_leaf_value     pinned  (MSE λ=0 → sklearn leaf means)
 *   oracle_update_pred    pinned  (sklearn boosting on residuals)
 *   oracle_train (MSE)    pinned  (sklearn residual-tree boosting, λ=0)
 *   oracle_train (softmax) pinned  (d = 2: sklearn HistGradientBoostingClassifier, binary log loss;
 *                                   d > 2: per-step pins only)
 *   oracle_predict        pinned  (on the training rows = oracle_train's incremental prediction,
 *                                   a different computation; sklearn tree.predict on unseen rows)
 */
#ifndef GBDTMO_ORACLE_H
#define GBDTMO_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum { ORACLE_LOSS_MSE = 0, ORACLE_LOSS_SOFTMAX = 1 };

/* Per-feature quantile binning (R14).
 * X row-major, element (i, f) at X[i*ld_x + f].  Outputs cuts[f*(B-1) + j] (ascending,
 * +inf padded), nbins[f] = #cuts + 1, bins_cm[f*n + i] = #{cuts of f <= X(i,f)}. */
void oracle_bin(const float* X, int64_t n, int32_t m, int64_t ld_x, int32_t B,
                float* cuts, int32_t* nbins, uint16_t* bins_cm);

/* Compressed Sparse Column storage (§3.2): traverse the matrix column-wise;
 * values = the non-zero entries, row_idx = their rows, col_ptr[j] = index in values where column
 * j starts, col_ptr[m] = number of non-zeros.  X row-major, element (i, f) at X[i*ld_x + f].
 * Pass values = row_idx = NULL to obtain col_ptr only (the sizes). */
void oracle_csc_from_dense(const float* X, int64_t n, int32_t m, int64_t ld_x,
                           float* values, int32_t* row_idx, int64_t* col_ptr);
/* The inverse: X (row-major, ld_x) = 0 everywhere, then X(row_idx[p], j) = values[p]. */
void oracle_dense_from_csc(const float* values, const int32_t* row_idx, const int64_t* col_ptr,
                           int64_t n, int32_t m, int64_t ld_x, float* X);

/* Per-output first/second derivatives (PAPER.md:164 MSE; R12 softmax-CE; R13 diagonal H). */
void oracle_grad(int32_t loss, const double* y, const double* pred, int64_t n, int32_t d,
                 double* g, double* h);

/* Histogram of one node (§3.3): for every f, b, k
 *   HG[f][b][k] = sum_{r in rows, bin(r,f)=b} g[r][k];  HH likewise with h;
 *   CNT[f][b] = #{r in rows : bin(r,f)=b}.   Row order = order of `rows`. */
void oracle_build_hist(const uint16_t* bins_cm, int64_t n, int32_t m, int32_t B,
                       const double* g, const double* h, int32_t d,
                       const int32_t* rows, int64_t nrows,
                       double* HG, double* HH, int64_t* CNT);

typedef struct {
  int32_t valid;    /* 1 iff some candidate has C_L, C_R >= min_node                */
  int32_t feature;  /* argmax feature (ties -> smallest f, then smallest b; R16)      */
  int32_t bin;      /* left = {bin <= b} (R15)                                        */
  int32_t pad;
  double  gain;     /* Eq. (3) at (feature, bin)                                      */
  int64_t n_left;   /* C_L at the winner                                              */
} oracle_split;

/* Eq. (3) for one candidate given left sums and node totals. */
double oracle_gain(const double* GL, const double* HL, const double* G, const double* H,
                   int32_t d, double lambda);

/* Best split of one node from its histogram (Alg. 1 lines 5-13).
 * G[d], H[d] are the node totals (summed from the node's rows, R17), cnt = |rows|.
 * Candidates b in [0, nbins_f - 2]; valid iff C_L >= min_node and C_R >= min_node (R4).
 * all_gains (may be NULL): [m][B] gain of every candidate, -inf where not a candidate. */
void oracle_find_split(const double* HG, const double* HH, const int64_t* CNT,
                       int32_t m, const int32_t* nbins, int32_t B, int32_t d,
                       const double* G, const double* H, int64_t cnt,
                       double lambda, int64_t min_node,
                       oracle_split* out, double* all_gains);

/* Stable partition of rows by bin(r, f) <= b (Alg. 1 line 16 SplitNode; R15). */
void oracle_partition(const uint16_t* bins_cm, int64_t n, const int32_t* rows, int64_t nrows,
                      int32_t f, int32_t b, int32_t* left, int32_t* right, int64_t* n_left);

/* Diagonal-Hessian optimal leaf: v_k = -lr * G_k / (H_k + lambda) (R9). */
void oracle_leaf_value(const double* G, const double* H, int32_t d, double lambda, double lr,
                       double* v);

/* Incremental prediction: pred[r] += v for every r in rows. */
void oracle_update_pred(double* pred, int32_t d, const int32_t* rows, int64_t nrows,
                        const double* v);

typedef struct {
  int32_t loss, T, D;
  int32_t min_node;
  double  lambda, gamma, lr;
} oracle_params;

/* Whole Algorithm 1, level-wise reading R6, heap node ids
 * (root 0, children 2i+1, 2i+2).  Per tree t the arrays hold (2^(D+1)-1) slots:
 *   state[t][i]  0 = no node, 1 = split, 2 = leaf
 *   feat/bin/gain/n_left of split nodes, nrows of every node, leaf[t][i][d] of leaves.
 * pred [n][d] in/out (starts at base score 0, R10).  Any output pointer may be NULL. */
void oracle_train(const uint16_t* bins_cm, int64_t n, int32_t m, const int32_t* nbins, int32_t B,
                  const double* y, int32_t d, const oracle_params* p,
                  double* pred,
                  int32_t* state, int32_t* feat, int32_t* bin, double* gain, int64_t* n_left,
                  int64_t* nrows, double* leaf);

/* Inference for (unseen) instances ("predictions" for new data; the traversal the
 * training path avoids).  For every row i and tree t = 0..T-1 in order: start at the
 * root (heap id 0); at a split node (state 1) go to child 2h+1 iff bin(X[i][feat], cuts of feat)
 * <= bin (the split's own definition, R14 + R15: left = {bin <= b}), else 2h+2; at a leaf
 * (state 2) add leaf[t][h][0..d) to pred[i].  X row-major [n][ld_x] (raw features), cuts
 * [m][B-1] from oracle_bin, state/feat/bin int32 [T][NH], leaf fp64 [T][NH][d] as written by
 * oracle_train (NH = 2^(D+1) - 1); pred [n][d] in/out. */
void oracle_predict(const float* X, int64_t n, int64_t ld_x, const float* cuts, const int32_t* nbins,
                    int32_t B, int32_t T, int32_t D, int32_t d, const int32_t* state,
                    const int32_t* feat, const int32_t* bin, const double* leaf, double* pred);

/* Number of worker threads the oracle uses (OpenMP), for reporting. */
int32_t oracle_num_threads(void);

#ifdef __cplusplus
}
#endif
#endif
