/*
 * oracle/gbdt_oracle.c -- TEST INFRASTRUCTURE ONLY (never on the product path).
 *
 * A plain, slow, obviously-correct, single-threaded CPU implementation of exact-greedy GBDT
 * training as GPU-GBDT computes it (Wen et al., IPDPS 2018; /root/reference/PAPER.md, cited
 * below as P:<line>).  It shares no code, header, table or helper with the CUDA path under
 * paper_conf_ipps_wenhkls18_b200/ and includes nothing from it.  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may load it.
 *
 * Where the paper is silent or garbled, the readings R1..R24 of SURVEY.md §8(c) are used and
 * are listed again in DESIGN.md ("Readings").  Key ones:
 *   R1  Eq. 2 parent denominator is H_L + H_R + lambda (P:128 prints "- lambda": garble).
 *   R2  split iff best gain > max(gamma, 0), strictly (Alg. 1 l.15-17).
 *   R3  leaf weight w = -G / (H + lambda) (never printed; "weight of the leaf node").
 *   R5  logistic (cross-entropy; Eq. 1): p = 1/(1+exp(-yhat)), g = p - y,
 *       h = max(p(1-p), 1e-16), both derivatives taken at p itself.
 *   R6  squared: g = 2(yhat - y), h = 2.
 *   R8  attribute lists sorted descending; high/left = prefix side.
 *   R9  equal values ordered by ascending instance id.
 *   R10 one candidate per distinct value, at the END of its run.
 *   R11 split_value = smallest value on the high side; present x >= v -> high.
 *   R12 total order: gain desc, attr asc, value desc, dir (missing->low first).
 *   R13 the boundary after the last run (all present high, missing low) is a candidate.
 *   R14 children must be non-empty by INTEGER count.
 *   R15 root depth 0; nodes with depth < d may split.
 *   R17 values fp32; g, h, yhat, sums, gains, weights fp64.
 *
 * Parity pins for every exported function live in tests/test_oracle_pins.py.
 */
#define _POSIX_C_SOURCE 199309L
#include <math.h>
#include <stdint.h>
#include <time.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------ public structs */
typedef struct {
  int32_t max_depth;
  int32_t n_trees;
  double lambda;
  double gamma;
  double eta;
  double base_margin;
  int32_t loss; /* 0 squared, 1 logistic */
} orc_params;

typedef struct {
  int32_t heap_id;      /* -1: slot unused */
  int32_t is_leaf;
  int32_t attr;         /* -1 for leaves */
  int32_t default_left; /* 1: missing goes to the high/left child */
  float split_value;    /* smallest value on the high side */
  int32_t follow_status;/* -1 n/a, 0 exact, 1 near-tie accepted, 2 mismatch */
  double gain;
  double G, H, weight;
  int64_t count;
} orc_node;

typedef struct {
  int64_t nodes_exact;
  int64_t nodes_near_tie;
  int64_t nodes_mismatch;
} orc_stats;

/* ------------------------------------------------------------------ helpers */
static float canon(float v) { return v == 0.0f ? 0.0f : v; } /* -0.0 -> +0.0 */

typedef struct { float v; int32_t i; } orc_entry;

static int cmp_entry(const void* pa, const void* pb) {
  const orc_entry* a = (const orc_entry*)pa;
  const orc_entry* b = (const orc_entry*)pb;
  if (a->v > b->v) return -1; /* descending value */
  if (a->v < b->v) return 1;
  return (a->i > b->i) - (a->i < b->i); /* ascending instance id (R9) */
}

/* Transposed, per-attribute sorted lists. NaN = missing, dropped.
 * col_ptr[m+1]; val/ins have capacity nnz. Returns the number of stored entries. */
int64_t orc_presort(int64_t n, int64_t m, const int64_t* indptr, const int32_t* indices,
                    const float* values, int64_t* col_ptr, float* val, int32_t* ins) {
  int64_t nnz = indptr[n];
  for (int64_t a = 0; a <= m; ++a) col_ptr[a] = 0;
  for (int64_t p = 0; p < nnz; ++p)
    if (!isnan(values[p])) col_ptr[indices[p] + 1]++;
  for (int64_t a = 0; a < m; ++a) col_ptr[a + 1] += col_ptr[a];
  int64_t* fill = (int64_t*)malloc(sizeof(int64_t) * (size_t)(m > 0 ? m : 1));
  orc_entry* tmp = (orc_entry*)malloc(sizeof(orc_entry) * (size_t)(nnz > 0 ? nnz : 1));
  for (int64_t a = 0; a < m; ++a) fill[a] = col_ptr[a];
  for (int64_t i = 0; i < n; ++i)
    for (int64_t p = indptr[i]; p < indptr[i + 1]; ++p) {
      if (isnan(values[p])) continue;
      int64_t q = fill[indices[p]]++;
      tmp[q].v = canon(values[p]);
      tmp[q].i = (int32_t)i;
    }
  for (int64_t a = 0; a < m; ++a)
    qsort(tmp + col_ptr[a], (size_t)(col_ptr[a + 1] - col_ptr[a]), sizeof(orc_entry), cmp_entry);
  for (int64_t q = 0; q < col_ptr[m]; ++q) { val[q] = tmp[q].v; ins[q] = tmp[q].i; }
  free(tmp);
  free(fill);
  return col_ptr[m];
}

/* Run-length encoding of a sorted value sequence (1.2,1.2,1.2,3.4,... -> (1.2,3),(3.4,4)). */
int64_t orc_rle_encode(int64_t len, const float* vals, float* run_val, int32_t* run_len) {
  int64_t r = -1;
  for (int64_t p = 0; p < len; ++p) {
    if (r < 0 || vals[p] != run_val[r]) { ++r; run_val[r] = vals[p]; run_len[r] = 0; }
    run_len[r]++;
  }
  return r + 1;
}

/* Segmented inclusive prefix sum (Fig. 1): out[i] = x[i] + out[i-1] unless head[i]. */
void orc_seg_scan(int64_t len, const double* x, const uint8_t* head, double* out) {
  double run = 0.0;
  for (int64_t p = 0; p < len; ++p) {
    run = (p == 0 || head[p]) ? x[p] : run + x[p];
    out[p] = run;
  }
}

/* First/second derivatives (Eq. 1). squared: P:193 (R6); logistic: R5. */
void orc_gradients(int32_t loss, int64_t n, const double* yhat, const float* y, double* g, double* h) {
  for (int64_t i = 0; i < n; ++i) {
    if (loss == 0) {
      g[i] = 2.0 * (yhat[i] - (double)y[i]);
      h[i] = 2.0;
    } else {
      double p = 1.0 / (1.0 + exp(-yhat[i]));
      g[i] = p - (double)y[i];
      double hh = p * (1.0 - p);  /* second derivative of the cross-entropy at p (Eq. 1) */
      h[i] = hh > 1e-16 ? hh : 1e-16;
    }
  }
}

/* Eq. 2 with the +lambda reading (R1): 1/2 [GL^2/(HL+l) + GR^2/(HR+l) - G^2/(H+l)]. */
static double eq2_gain(double GL, double HL, double G, double H, double lam, double* S) {
  double GR = G - GL, HR = H - HL;
  double t1 = (GL * GL) / (HL + lam);
  double t2 = (GR * GR) / (HR + lam);
  double t0 = (G * G) / (H + lam);
  double s = t1 + t2;
  if (S) *S = s;
  return 0.5 * (s - t0);
}

double orc_gain(double GL, double HL, double G, double H, double lam) {
  return eq2_gain(GL, HL, G, H, lam, NULL);
}

/* ------------------------------------------------------------------ timing (bench / tests only) */
/* Wall-clock seconds of the last orc_train on this thread: [0] presort, [1 + t] tree t.  No part
 * of the method; lets the cpu_baseline report per-tree time with the presort excluded. */
#define ORC_MAX_TIMED 4096
static _Thread_local double orc_times[ORC_MAX_TIMED + 1];
static _Thread_local int orc_n_times;

static double now_s(void) {
  struct timespec ts;
  clock_gettime(CLOCK_MONOTONIC, &ts);
  return (double)ts.tv_sec + 1e-9 * (double)ts.tv_nsec;
}

int orc_last_timings(double* out, int cap) {
  int k = orc_n_times < cap ? orc_n_times : cap;
  for (int i = 0; i < k; ++i) out[i] = orc_times[i];
  return orc_n_times;
}

/* ------------------------------------------------------------------ training */
typedef struct {
  int valid;
  double gain, S;
  double GL, HL; /* high/left side including missing when dir == 1 */
  int64_t cntL;
  int32_t attr;
  float value;
  int32_t dir;   /* 0: missing -> low/right; 1: missing -> high/left */
} cand;

static int cand_better(const cand* a, const cand* b) { /* R12 total order */
  if (!a->valid) return 0;
  if (!b->valid) return 1;
  if (a->gain != b->gain) return a->gain > b->gain;
  if (a->attr != b->attr) return a->attr < b->attr;
  if (a->value != b->value) return a->value > b->value;
  return a->dir < b->dir;
}

typedef struct {
  int64_t n, m;
  const int64_t* indptr;
  const int32_t* indices;
  const float* values;
  orc_params P;
  const double* g;
  const double* h;
  const int32_t* node_of;
} ctx_t;

/* x_i[a] by binary search in CSR row i; returns 0 if missing (absent or NaN). */
static int lookup(const ctx_t* c, int64_t i, int32_t a, float* out) {
  int64_t lo = c->indptr[i], hi = c->indptr[i + 1];
  while (lo < hi) {
    int64_t mid = lo + (hi - lo) / 2;
    if (c->indices[mid] < a) lo = mid + 1; else hi = mid;
  }
  if (lo < c->indptr[i + 1] && c->indices[lo] == a && !isnan(c->values[lo])) {
    *out = canon(c->values[lo]);
    return 1;
  }
  return 0;
}

/* Direct evaluation of one split of node k (plain definition, instances in ascending id).
 * Used by follow mode to price the GPU's choice independently of the scan. */
static cand eval_direct(const ctx_t* c, int32_t k, double G, double H, int64_t cnt,
                        int32_t a, float v, int32_t dir) {
  cand r; memset(&r, 0, sizeof r);
  double GL = 0, HL = 0; int64_t nL = 0, nPresent = 0; float x; int found_v = 0;
  for (int64_t i = 0; i < c->n; ++i) {
    if (c->node_of[i] != k) continue;
    int pres = lookup(c, i, a, &x);
    if (pres) { nPresent++; if (x == v) found_v = 1; }
    int high = pres ? (x >= v) : (dir == 1);
    if (high) { GL += c->g[i]; HL += c->h[i]; nL++; }
  }
  int64_t cntM = cnt - nPresent;
  r.attr = a; r.value = v; r.dir = dir;
  r.GL = GL; r.HL = HL; r.cntL = nL;
  r.valid = found_v && nL >= 1 && (cnt - nL) >= 1 && (dir == 0 || cntM > 0);
  r.gain = eq2_gain(GL, HL, G, H, c->P.lambda, &r.S);
  if (r.gain == 0.0) r.gain = 0.0;
  return r;
}

int orc_train(int64_t n, int64_t m, const int64_t* indptr, const int32_t* indices,
              const float* values, const float* labels, const orc_params* P,
              const orc_node* follow, orc_node* out_nodes, double* out_margin,
              orc_stats* stats) {
  if (n < 1 || m < 1 || P->max_depth < 1 || P->max_depth > 20 || P->n_trees < 1) return 1;
  const int d = P->max_depth;
  const int64_t NH = ((int64_t)1 << (d + 1)) - 1; /* heap slots per tree */
  const double lam = P->lambda;
  const double thr = P->gamma > 0.0 ? P->gamma : 0.0;
  int64_t nnz = indptr[n];

  double t_start = now_s();
  orc_n_times = 0;
  int64_t* col_ptr = (int64_t*)malloc(sizeof(int64_t) * (size_t)(m + 1));
  float* cval = (float*)malloc(sizeof(float) * (size_t)(nnz > 0 ? nnz : 1));
  int32_t* cins = (int32_t*)malloc(sizeof(int32_t) * (size_t)(nnz > 0 ? nnz : 1));
  orc_presort(n, m, indptr, indices, values, col_ptr, cval, cins);
  double t_prev = now_s();
  orc_times[orc_n_times++] = t_prev - t_start;

  double* yhat = (double*)malloc(sizeof(double) * (size_t)n);
  double* g = (double*)malloc(sizeof(double) * (size_t)n);
  double* h = (double*)malloc(sizeof(double) * (size_t)n);
  int32_t* node_of = (int32_t*)malloc(sizeof(int32_t) * (size_t)n);
  /* per heap-node state */
  double* nG = (double*)malloc(sizeof(double) * (size_t)NH);
  double* nH = (double*)malloc(sizeof(double) * (size_t)NH);
  int64_t* nC = (int64_t*)malloc(sizeof(int64_t) * (size_t)NH);
  int8_t* open = (int8_t*)malloc((size_t)NH);
  cand* best = (cand*)malloc(sizeof(cand) * (size_t)NH);
  double* GP = (double*)malloc(sizeof(double) * (size_t)NH);
  double* HP = (double*)malloc(sizeof(double) * (size_t)NH);
  int64_t* CP = (int64_t*)malloc(sizeof(int64_t) * (size_t)NH);
  double* GLr = (double*)malloc(sizeof(double) * (size_t)NH);
  double* HLr = (double*)malloc(sizeof(double) * (size_t)NH);
  int64_t* CLr = (int64_t*)malloc(sizeof(int64_t) * (size_t)NH);
  float* lastv = (float*)malloc(sizeof(float) * (size_t)NH);
  int8_t* has_last = (int8_t*)malloc((size_t)NH);
  double* wleaf = (double*)malloc(sizeof(double) * (size_t)NH);

  ctx_t C = {n, m, indptr, indices, values, *P, g, h, node_of};
  if (stats) memset(stats, 0, sizeof *stats);
  for (int64_t i = 0; i < n; ++i) yhat[i] = P->base_margin; /* R7 */

  for (int t = 0; t < P->n_trees; ++t) {
    orc_node* T = out_nodes + (int64_t)t * NH;
    const orc_node* F = follow ? follow + (int64_t)t * NH : NULL;
    for (int64_t k = 0; k < NH; ++k) {
      memset(&T[k], 0, sizeof(orc_node));
      T[k].heap_id = -1; T[k].attr = -1; T[k].follow_status = -1;
      open[k] = 0;
    }
    orc_gradients(P->loss, n, yhat, labels, g, h);           /* Eq. 1 */
    double G0 = 0, H0 = 0;
    for (int64_t i = 0; i < n; ++i) { node_of[i] = 0; G0 += g[i]; H0 += h[i]; }
    nG[0] = G0; nH[0] = H0; nC[0] = n; open[0] = 1;
    T[0].heap_id = 0; T[0].G = G0; T[0].H = H0; T[0].count = n;

    for (int lvl = 0; lvl < d; ++lvl) {                      /* depth(n) < d */
      int64_t k0 = ((int64_t)1 << lvl) - 1, k1 = ((int64_t)1 << (lvl + 1)) - 1;
      int any = 0;
      for (int64_t k = k0; k < k1; ++k) { memset(&best[k], 0, sizeof(cand)); any |= open[k]; }
      if (!any) break;
      /* Alg. 1 l.7-13: every attribute, every split point */
      for (int64_t a = 0; a < m; ++a) {
        for (int64_t k = k0; k < k1; ++k) {
          GP[k] = HP[k] = 0; CP[k] = 0; GLr[k] = HLr[k] = 0; CLr[k] = 0; has_last[k] = 0;
        }
        /* pass 1: present totals per node */
        for (int64_t q = col_ptr[a]; q < col_ptr[a + 1]; ++q) {
          int32_t i = cins[q]; int32_t k = node_of[i];
          if (k < k0 || !open[k]) continue;
          GP[k] += g[i]; HP[k] += h[i]; CP[k]++;
        }
        /* pass 2: running sums; a candidate at the end of each run of equal values (R10) */
        for (int64_t q = col_ptr[a]; q <= col_ptr[a + 1]; ++q) {
          int final = (q == col_ptr[a + 1]);
          int32_t i = final ? -1 : cins[q];
          int32_t kq = final ? -1 : node_of[i];
          if (!final && (kq < k0 || !open[kq])) continue;
          for (int64_t k = (final ? k0 : kq); k < (final ? k1 : kq + 1); ++k) {
            if (!has_last[k]) continue;
            if (!final && cval[q] == lastv[k]) continue;
            /* candidate "x >= lastv -> high" with sums over values >= lastv */
            int64_t cntM = nC[k] - CP[k];
            double GM = nG[k] - GP[k], HM = nH[k] - HP[k];
            for (int dir = 0; dir < 2; ++dir) {
              if (dir == 1 && cntM <= 0) break;            /* both directions only with missing */
              cand c; memset(&c, 0, sizeof c);
              c.GL = GLr[k] + (dir ? GM : 0.0);
              c.HL = HLr[k] + (dir ? HM : 0.0);
              c.cntL = CLr[k] + (dir ? cntM : 0);
              c.attr = (int32_t)a; c.value = lastv[k]; c.dir = dir;
              c.valid = c.cntL >= 1 && (nC[k] - c.cntL) >= 1;  /* R14 */
              if (!c.valid) continue;
              c.gain = eq2_gain(c.GL, c.HL, nG[k], nH[k], lam, &c.S);
              if (c.gain == 0.0) c.gain = 0.0;
              if (cand_better(&c, &best[k])) best[k] = c;
            }
          }
          if (final) break;
          GLr[kq] += g[i]; HLr[kq] += h[i]; CLr[kq]++;
          lastv[kq] = cval[q]; has_last[kq] = 1;
        }
      }
      /* Alg. 1 l.14-21: decide, then split */
      for (int64_t k = k0; k < k1; ++k) {
        if (!open[k]) continue;
        cand* b = &best[k];
        int split = b->valid && b->gain > thr;                    /* R2 */
        cand use = *b;
        if (F) {
          const orc_node* f = &F[k];
          int fsplit = (f->heap_id == k) && !f->is_leaf;
          int status = 0;
          if (fsplit) {
            cand fc = eval_direct(&C, (int32_t)k, nG[k], nH[k], nC[k], f->attr, f->split_value,
                                  f->default_left ? 1 : 0);
            if (split && fc.attr == b->attr && fc.value == b->value && fc.dir == b->dir) {
              status = fc.valid ? 0 : 2;
            } else if (!fc.valid) {
              status = 2;
            } else if (split) {
              status = fabs(fc.gain - b->gain) <= 1e-6 * fabs(b->gain) ? 1 : 2;
            } else {
              double tol = fmax(1e-6 * fabs(fc.gain), 1e-12 * fc.S);
              status = (b->valid && fabs(b->gain - thr) <= tol) || fabs(fc.gain - thr) <= tol ? 1 : 2;
            }
            if (status == 0) { split = 1; }               /* identical choice: keep scan result */
            else if (fc.valid) { use = fc; split = 1; } else { split = 0; }
          } else {
            if (split) {
              double tol = fmax(1e-6 * fabs(b->gain), 1e-12 * b->S);
              status = fabs(b->gain - thr) <= tol ? 1 : 2;
            }
            split = 0;
          }
          T[k].follow_status = status;
          if (stats) {
            if (status == 0) stats->nodes_exact++;
            else if (status == 1) stats->nodes_near_tie++;
            else stats->nodes_mismatch++;
          }
        }
        if (!split) { open[k] = 0; T[k].is_leaf = 1; T[k].gain = 0; continue; }
        T[k].is_leaf = 0; T[k].attr = use.attr; T[k].split_value = use.value;
        T[k].default_left = use.dir; T[k].gain = use.gain;
        int64_t hi = 2 * k + 1, lo = 2 * k + 2;
        nG[hi] = nH[hi] = nG[lo] = nH[lo] = 0; nC[hi] = nC[lo] = 0;
        /* route by x >= v* (R11); missing -> dir* */
        for (int64_t i = 0; i < n; ++i) {
          if (node_of[i] != k) continue;
          float x;
          int high = lookup(&C, i, use.attr, &x) ? (x >= use.value) : (use.dir == 1);
          node_of[i] = (int32_t)(high ? hi : lo);
        }
        /* child totals by plain summation over members in ascending id */
        for (int64_t i = 0; i < n; ++i) {
          int32_t c2 = node_of[i];
          if (c2 == hi || c2 == lo) { nG[c2] += g[i]; nH[c2] += h[i]; nC[c2]++; }
        }
        for (int64_t c2 = hi; c2 <= lo; ++c2) {
          T[c2].heap_id = (int32_t)c2; T[c2].G = nG[c2]; T[c2].H = nH[c2]; T[c2].count = nC[c2];
          T[c2].attr = -1; T[c2].follow_status = -1;
          open[c2] = (lvl + 1 < d);
          if (!open[c2]) T[c2].is_leaf = 1;
        }
        open[k] = 0;
      }
    }
    /* leaves: w = -G/(H+lambda) (R3); SmartGD: yhat += eta * w[leaf(i)] */
    for (int64_t k = 0; k < NH; ++k) {
      wleaf[k] = 0.0;
      if (T[k].heap_id == k && T[k].is_leaf) {
        T[k].weight = -T[k].G / (T[k].H + lam);
        wleaf[k] = T[k].weight;
      }
    }
    for (int64_t i = 0; i < n; ++i) yhat[i] = yhat[i] + P->eta * wleaf[node_of[i]];
    double t_now = now_s();
    if (orc_n_times <= ORC_MAX_TIMED) orc_times[orc_n_times++] = t_now - t_prev;
    t_prev = t_now;
  }
  if (out_margin) memcpy(out_margin, yhat, sizeof(double) * (size_t)n);

  free(col_ptr); free(cval); free(cins); free(yhat); free(g); free(h); free(node_of);
  free(nG); free(nH); free(nC); free(open); free(best); free(GP); free(HP); free(CP);
  free(GLr); free(HLr); free(CLr); free(lastv); free(has_last); free(wleaf);
  return 0;
}

/* Prediction by tree traversal (P:252-254, P:279 reading R11): one instance at a time, trees in
 * order, yhat = base + sum_t eta * w_t(leaf). */
void orc_predict(int64_t n, const int64_t* indptr, const int32_t* indices, const float* values,
                 const orc_node* nodes, int32_t n_trees, int32_t max_depth, double eta,
                 double base_margin, double* out) {
  const int64_t NH = ((int64_t)1 << (max_depth + 1)) - 1;
  ctx_t C; memset(&C, 0, sizeof C);
  C.n = n; C.indptr = indptr; C.indices = indices; C.values = values;
  for (int64_t i = 0; i < n; ++i) {
    double y = base_margin;
    for (int t = 0; t < n_trees; ++t) {
      const orc_node* T = nodes + (int64_t)t * NH;
      int64_t k = 0;
      while (!T[k].is_leaf) {
        float x;
        int high = lookup(&C, i, T[k].attr, &x) ? (x >= T[k].split_value) : T[k].default_left;
        k = high ? 2 * k + 1 : 2 * k + 2;
      }
      y = y + eta * T[k].weight;
    }
    out[i] = y;
  }
}
