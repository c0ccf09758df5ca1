/*
 * oracle.c — plain fp64 CPU oracle for the GBDT-MO hot path.
 *
 * TEST INFRASTRUCTURE ONLY (see oracle.h).  Written from /root/reference/PAPER.md;
 * each function states the passage it follows.  No blocking, fusion, subtraction
 * trick, fixed point or reordering: every quantity is computed from its definition
 * in the order the paper (or the DESIGN.md reading) gives.  OpenMP is used only
 * over independent features/columns; each feature's sums have exactly one owner
 * thread and run in row order, so results do not depend on the thread count.
 */
#include "oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

int32_t oracle_num_threads(void) {
#ifdef _OPENMP
  return (int32_t)omp_get_max_threads();
#else
  return 1;
#endif
}

/* ---------------------------------------------------------------- binning */

static int cmp_float(const void* a, const void* b) {
  float x = *(const float*)a, y = *(const float*)b;
  return (x < y) ? -1 : (x > y) ? 1 : 0;
}

/* bin(x) = #{c in cuts : c <= x}  (R14; "feature-value bin mapping").
 * Written as the count it defines; cuts are ascending so the count is the first
 * index whose cut exceeds x (found by bisection). */
static int32_t count_cuts_le(const float* cuts, int32_t ncuts, float x) {
  int32_t lo = 0, hi = ncuts;           /* invariant: cuts[<lo] <= x, cuts[>=hi] > x */
  while (lo < hi) {
    int32_t mid = lo + (hi - lo) / 2;
    if (cuts[mid] <= x) lo = mid + 1; else hi = mid;
  }
  return lo;
}

/* Quantile binning, reading R14 (paper: "cut points", max 256 bins):
 *   s = sorted column.
 *   (i)  <= B distinct values: cuts = every distinct value except the smallest.
 *   (ii) otherwise: c_j = s[floor(j*n/B)], j = 1..B-1, duplicates dropped, and every c <= s[0] dropped.
 *   nbins = #cuts + 1. */
/* "For non-zero values, we traverse the matrix column-wise", "For row indices,
 * we store the row number of each non-zero value", "The column pointer array has an additional
 * element indicating the end of the last column". */
void oracle_csc_from_dense(const float* X, int64_t n, int32_t m, int64_t ld_x,
                           float* values, int32_t* row_idx, int64_t* col_ptr) {
  int64_t p = 0;
  for (int32_t j = 0; j < m; ++j) {
    col_ptr[j] = p;
    for (int64_t i = 0; i < n; ++i) {
      const float x = X[i * ld_x + j];
      if (x != 0.0f) {
        if (values) values[p] = x;
        if (row_idx) row_idx[p] = (int32_t)i;
        ++p;
      }
    }
  }
  col_ptr[m] = p;
}

void oracle_dense_from_csc(const float* values, const int32_t* row_idx, const int64_t* col_ptr,
                           int64_t n, int32_t m, int64_t ld_x, float* X) {
  for (int64_t i = 0; i < n; ++i)
    for (int32_t j = 0; j < m; ++j) X[i * ld_x + j] = 0.0f;
  for (int32_t j = 0; j < m; ++j)
    for (int64_t p = col_ptr[j]; p < col_ptr[j + 1]; ++p) X[(int64_t)row_idx[p] * ld_x + j] = values[p];
}

void oracle_bin(const float* X, int64_t n, int32_t m, int64_t ld_x, int32_t B,
                float* cuts, int32_t* nbins, uint16_t* bins_cm) {
#pragma omp parallel for schedule(dynamic, 1)
  for (int32_t f = 0; f < m; ++f) {
    float* s = (float*)malloc(sizeof(float) * (size_t)(n > 0 ? n : 1));
    for (int64_t i = 0; i < n; ++i) s[i] = X[i * ld_x + f];
    qsort(s, (size_t)n, sizeof(float), cmp_float);
    float* c = cuts + (int64_t)f * (B - 1);
    for (int32_t j = 0; j < B - 1; ++j) c[j] = INFINITY;
    int64_t distinct = (n > 0) ? 1 : 0;
    for (int64_t i = 1; i < n; ++i) if (s[i] != s[i - 1]) ++distinct;
    int32_t k = 0;
    if (distinct <= B) {                                   /* rule (i) */
      for (int64_t i = 1; i < n; ++i) if (s[i] != s[i - 1]) c[k++] = s[i];
    } else {                                               /* rule (ii) */
      for (int32_t j = 1; j <= B - 1; ++j) {
        float v = s[((int64_t)j * n) / B];
        if (v <= s[0]) continue;
        if (k > 0 && v == c[k - 1]) continue;
        c[k++] = v;
      }
    }
    nbins[f] = k + 1;
    for (int64_t i = 0; i < n; ++i)
      bins_cm[(int64_t)f * n + i] = (uint16_t)count_cuts_le(c, k, X[i * ld_x + f]);
    free(s);
  }
}

/* ------------------------------------------------------------- gradients */

/* MSE: l = sum_k (yhat_k - y_k)^2, g = 2(yhat - y), h = 2 (R11).
 * Softmax cross-entropy (named at PAPER.md:156; formula = reading R12):
 *   p = softmax(yhat) (max-subtracted), l = -sum_k y_k log p_k,
 *   g_k = p_k - y_k (for one-hot / sum-to-one y), h_k = p_k (1 - p_k) (diagonal). */
void oracle_grad(int32_t loss, const double* y, const double* pred, int64_t n, int32_t d,
                 double* g, double* h) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    const double* yi = y + i * d;
    const double* pi = pred + i * d;
    double* gi = g + i * d;
    double* hi = h + i * d;
    if (loss == ORACLE_LOSS_MSE) {
      for (int32_t k = 0; k < d; ++k) { gi[k] = 2.0 * (pi[k] - yi[k]); hi[k] = 2.0; }
    } else {
      double mx = pi[0];
      for (int32_t k = 1; k < d; ++k) if (pi[k] > mx) mx = pi[k];
      double z = 0.0;
      for (int32_t k = 0; k < d; ++k) z += exp(pi[k] - mx);
      for (int32_t k = 0; k < d; ++k) {
        double p = exp(pi[k] - mx) / z;
        gi[k] = p - yi[k];
        hi[k] = p * (1.0 - p);
      }
    }
  }
}

/* ------------------------------------------------------------ histograms */

/* HG[f][b][k] = sum over the node's rows with bin(r,f) = b of g[r][k], likewise HH, CNT
 * ("aggregate gradient statistics ... into discrete bins for each feature"). */
void oracle_build_hist(const uint16_t* bins_cm, int64_t n, int32_t m, int32_t B,
                       const double* g, const double* h, int32_t d,
                       const int32_t* rows, int64_t nrows,
                       double* HG, double* HH, int64_t* CNT) {
#pragma omp parallel for schedule(dynamic, 1)
  for (int32_t f = 0; f < m; ++f) {
    double* hg = HG + (int64_t)f * B * d;
    double* hh = HH + (int64_t)f * B * d;
    int64_t* cnt = CNT + (int64_t)f * B;
    memset(hg, 0, sizeof(double) * (size_t)B * d);
    memset(hh, 0, sizeof(double) * (size_t)B * d);
    memset(cnt, 0, sizeof(int64_t) * (size_t)B);
    const uint16_t* col = bins_cm + (int64_t)f * n;
    for (int64_t t = 0; t < nrows; ++t) {
      int32_t r = rows[t];
      int32_t b = col[r];
      for (int32_t k = 0; k < d; ++k) {
        hg[(int64_t)b * d + k] += g[(int64_t)r * d + k];
        hh[(int64_t)b * d + k] += h[(int64_t)r * d + k];
      }
      cnt[b] += 1;
    }
  }
}

/* ----------------------------------------------------------- split search */

/* Eq. (3), PAPER.md:110:
 *   gain = 1/2 sum_{k=1..d} [ GL^2/(HL+l) + GR^2/(HR+l) - (GL+GR)^2/(HL+HR+l) ],
 * with GR = G - GL, HR = H - HL (G, H = node totals).  k ascending (R7). */
double oracle_gain(const double* GL, const double* HL, const double* G, const double* H,
                   int32_t d, double lambda) {
  double s = 0.0;
  for (int32_t k = 0; k < d; ++k) {
    double gl = GL[k], hl = HL[k];
    double gr = G[k] - gl, hr = H[k] - hl;
    s += gl * gl / (hl + lambda) + gr * gr / (hr + lambda) - (gl + gr) * (gl + gr) / (hl + hr + lambda);
  }
  return 0.5 * s;
}

/* G_L, H_L by a prefix sum over bins (ascending b), the gain of every
 * candidate, best per feature, best over features.  Ties: scan f ascending, b ascending,
 * replace only on a strictly greater gain (R16). */
void oracle_find_split(const double* HG, const double* HH, const int64_t* CNT,
                       int32_t m, const int32_t* nbins, int32_t B, int32_t d,
                       const double* G, const double* H, int64_t cnt,
                       double lambda, int64_t min_node,
                       oracle_split* out, double* all_gains) {
  double* GL = (double*)malloc(sizeof(double) * (size_t)d);
  double* HL = (double*)malloc(sizeof(double) * (size_t)d);
  out->valid = 0; out->feature = -1; out->bin = -1; out->pad = 0; out->gain = -INFINITY; out->n_left = 0;
  for (int32_t f = 0; f < m; ++f) {
    const double* hg = HG + (int64_t)f * B * d;
    const double* hh = HH + (int64_t)f * B * d;
    const int64_t* c = CNT + (int64_t)f * B;
    for (int32_t k = 0; k < d; ++k) { GL[k] = 0.0; HL[k] = 0.0; }
    int64_t CL = 0;
    if (all_gains) for (int32_t b = 0; b < B; ++b) all_gains[(int64_t)f * B + b] = -INFINITY;
    for (int32_t b = 0; b + 1 < nbins[f]; ++b) {
      for (int32_t k = 0; k < d; ++k) { GL[k] += hg[(int64_t)b * d + k]; HL[k] += hh[(int64_t)b * d + k]; }
      CL += c[b];
      int64_t CR = cnt - CL;
      if (CL < min_node || CR < min_node) continue;
      double gn = oracle_gain(GL, HL, G, H, d, lambda);
      if (all_gains) all_gains[(int64_t)f * B + b] = gn;
      if (!out->valid || gn > out->gain) {
        out->valid = 1; out->feature = f; out->bin = b; out->gain = gn; out->n_left = CL;
      }
    }
  }
  free(GL); free(HL);
}

/* ------------------------------------------------------------- partition */

/* Alg. 1 line 16 SplitNode: left = {bin <= b} in input order, then the rest. */
void oracle_partition(const uint16_t* bins_cm, int64_t n, const int32_t* rows, int64_t nrows,
                      int32_t f, int32_t b, int32_t* left, int32_t* right, int64_t* n_left) {
  const uint16_t* col = bins_cm + (int64_t)f * n;
  int64_t nl = 0, nr = 0;
  for (int64_t t = 0; t < nrows; ++t) {
    int32_t r = rows[t];
    if (col[r] <= b) left[nl++] = r; else right[nr++] = r;
  }
  *n_left = nl;
}

/* --------------------------------------------------------- leaves, update */

/* [v*]_k = -sum g_k / (sum h_k + lambda), scaled by the learning rate (R9). */
void oracle_leaf_value(const double* G, const double* H, int32_t d, double lambda, double lr,
                       double* v) {
  for (int32_t k = 0; k < d; ++k) v[k] = -lr * G[k] / (H[k] + lambda);
}

/* the prediction is updated incrementally from the leaf the row sits in. */
void oracle_update_pred(double* pred, int32_t d, const int32_t* rows, int64_t nrows,
                        const double* v) {
  for (int64_t t = 0; t < nrows; ++t)
    for (int32_t k = 0; k < d; ++k) pred[(int64_t)rows[t] * d + k] += v[k];
}

/* ------------------------------------------------------------- inference */

/* Tree walk for unseen rows (see oracle.h).  The split test is bin(x) <= b with
 * bin(x) = #{cuts <= x} (R14, R15), evaluated from the raw feature value. */
void oracle_predict(const float* X, int64_t n, int64_t ld_x, const float* cuts, const int32_t* nbins,
                    int32_t B, int32_t T, int32_t D, int32_t d, const int32_t* state,
                    const int32_t* feat, const int32_t* bin, const double* leaf, double* pred) {
  const int64_t slots = ((int64_t)1 << (D + 1)) - 1;
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    for (int32_t t = 0; t < T; ++t) {
      const int32_t* st = state + (int64_t)t * slots;
      int64_t h = 0;
      while (h < slots && st[h] == 1) {
        const int32_t f = feat[(int64_t)t * slots + h];
        const int32_t b = count_cuts_le(cuts + (int64_t)f * (B - 1), nbins[f] - 1, X[i * ld_x + f]);
        h = (b <= bin[(int64_t)t * slots + h]) ? 2 * h + 1 : 2 * h + 2;
      }
      if (h < slots && st[h] == 2)
        for (int32_t k = 0; k < d; ++k) pred[i * d + k] += leaf[((int64_t)t * slots + h) * d + k];
    }
  }
}

/* ----------------------------------------------------------- Algorithm 1 */

static void node_totals(const double* g, const double* h, int32_t d, const int32_t* rows,
                        int64_t nrows, double* G, double* H) {
  for (int32_t k = 0; k < d; ++k) { G[k] = 0.0; H[k] = 0.0; }
  for (int64_t t = 0; t < nrows; ++t)
    for (int32_t k = 0; k < d; ++k) {
      G[k] += g[(int64_t)rows[t] * d + k];
      H[k] += h[(int64_t)rows[t] * d + k];
    }
}

/* Algorithm 1, readings R1-R10, R16, R17:
 *   repeat T times: compute g, h (line "3.1.1"); grow one tree level by
 *   level from the root (depth 0); a node of depth < D with >= 2*min_node rows gets its
 *   histogram and best split (lines 5-13); if no valid candidate or best gain <= gamma
 *   it becomes a leaf, else its rows are split (lines 14-17); nodes of depth D are leaves;
 *   every leaf gets v = -lr G/(H+lambda) and pred += v for its rows. */
void oracle_train(const uint16_t* bins_cm, int64_t n, int32_t m, const int32_t* nbins, int32_t B,
                  const double* y, int32_t d, const oracle_params* p,
                  double* pred,
                  int32_t* state, int32_t* feat, int32_t* bin, double* gain, int64_t* n_left,
                  int64_t* nrows_out, double* leaf) {
  const int64_t slots = ((int64_t)1 << (p->D + 1)) - 1;
  double* g = (double*)malloc(sizeof(double) * (size_t)(n * d));
  double* h = (double*)malloc(sizeof(double) * (size_t)(n * d));
  double* HG = (double*)malloc(sizeof(double) * (size_t)((int64_t)m * B * d));
  double* HH = (double*)malloc(sizeof(double) * (size_t)((int64_t)m * B * d));
  int64_t* CNT = (int64_t*)malloc(sizeof(int64_t) * (size_t)((int64_t)m * B));
  double* G = (double*)malloc(sizeof(double) * (size_t)d);
  double* H = (double*)malloc(sizeof(double) * (size_t)d);
  double* v = (double*)malloc(sizeof(double) * (size_t)d);
  /* rows of every heap slot of the current and next level, as (offset, count) into a list */
  int32_t* cur = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  int32_t* nxt = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  int32_t* tmp = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  int64_t* off = (int64_t*)malloc(sizeof(int64_t) * (size_t)slots);
  int64_t* cnt = (int64_t*)malloc(sizeof(int64_t) * (size_t)slots);

  for (int32_t t = 0; t < p->T; ++t) {
    int32_t* st = state ? state + (int64_t)t * slots : NULL;
    if (st) for (int64_t i = 0; i < slots; ++i) st[i] = 0;
    oracle_grad(p->loss, y, pred, n, d, g, h);
    for (int64_t i = 0; i < slots; ++i) { off[i] = 0; cnt[i] = -1; }
    for (int64_t i = 0; i < n; ++i) cur[i] = (int32_t)i;
    off[0] = 0; cnt[0] = n;
    for (int32_t lvl = 0; lvl <= p->D; ++lvl) {
      int64_t first = ((int64_t)1 << lvl) - 1, last = ((int64_t)1 << (lvl + 1)) - 1;
      int64_t pos = 0;                                   /* write cursor into nxt */
      for (int64_t id = first; id < last; ++id) {
        if (cnt[id] < 0) continue;                       /* no node in this slot */
        const int32_t* rows = cur + off[id];
        int64_t nr = cnt[id];
        if (nrows_out) nrows_out[(int64_t)t * slots + id] = nr;
        node_totals(g, h, d, rows, nr, G, H);
        int is_split = 0;
        oracle_split sp;
        if (lvl < p->D && nr >= 2 * (int64_t)p->min_node) {
          oracle_build_hist(bins_cm, n, m, B, g, h, d, rows, nr, HG, HH, CNT);
          oracle_find_split(HG, HH, CNT, m, nbins, B, d, G, H, nr, p->lambda, p->min_node, &sp, NULL);
          is_split = sp.valid && sp.gain > p->gamma;
        }
        if (is_split) {
          int64_t nl = 0;
          oracle_partition(bins_cm, n, rows, nr, sp.feature, sp.bin, nxt + pos, tmp, &nl);
          memcpy(nxt + pos + nl, tmp, sizeof(int32_t) * (size_t)(nr - nl));   /* right part behind the left */
          int64_t lc = 2 * id + 1, rc = 2 * id + 2;
          off[lc] = pos; cnt[lc] = nl;
          off[rc] = pos + nl; cnt[rc] = nr - nl;
          pos += nr;
          if (st) st[id] = 1;
          if (feat) feat[(int64_t)t * slots + id] = sp.feature;
          if (bin) bin[(int64_t)t * slots + id] = sp.bin;
          if (gain) gain[(int64_t)t * slots + id] = sp.gain;
          if (n_left) n_left[(int64_t)t * slots + id] = nl;
        } else {
          oracle_leaf_value(G, H, d, p->lambda, p->lr, v);
          oracle_update_pred(pred, d, rows, nr, v);
          if (st) st[id] = 2;
          if (leaf) for (int32_t k = 0; k < d; ++k) leaf[((int64_t)t * slots + id) * d + k] = v[k];
        }
      }
      int32_t* tmp = cur; cur = nxt; nxt = tmp;
      /* the children's offsets refer to the list just written (now `cur`) */
    }
  }
  free(g); free(h); free(HG); free(HH); free(CNT); free(G); free(H); free(v);
  free(cur); free(nxt); free(tmp); free(off); free(cnt);
}
