/* TEST INFRASTRUCTURE ONLY: a standalone driver that runs the CPU oracle (gbdt_oracle.c) under
 * AddressSanitizer / UndefinedBehaviorSanitizer (tests/test_oracle_sanitizers.py builds it with
 * -fsanitize=address,undefined).  It trains on the Table I example and on seeded
 * random matrices with NaN-missing values, repeated values and follow mode, then predicts. */
#include <math.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

typedef struct { int32_t max_depth, n_trees; double lambda, gamma, eta, base_margin; int32_t loss; } orc_params;
typedef struct {
  int32_t heap_id, is_leaf, attr, default_left;
  float split_value;
  int32_t follow_status;
  double gain, G, H, weight;
  int64_t count;
} orc_node;
typedef struct { int64_t nodes_exact, nodes_near_tie, nodes_mismatch; } orc_stats;
int orc_train(int64_t n, int64_t m, const int64_t* indptr, const int32_t* indices, const float* values,
              const float* labels, const orc_params* P, const orc_node* follow, orc_node* out_nodes,
              double* out_margin, orc_stats* stats);
void orc_predict(int64_t n, const int64_t* indptr, const int32_t* indices, const float* values,
                 const orc_node* nodes, int32_t n_trees, int32_t max_depth, double eta, double base_margin,
                 double* out);

static uint64_t rng_state = 88172645463325252ull;
static uint64_t xs(void) { rng_state ^= rng_state << 13; rng_state ^= rng_state >> 7; rng_state ^= rng_state << 17; return rng_state; }

static int run(int64_t n, int64_t m, double nan_frac, int loss, int d, int T) {
  int64_t* indptr = malloc(sizeof(int64_t) * (n + 1));
  int32_t* idx = malloc(sizeof(int32_t) * n * m);
  float* val = malloc(sizeof(float) * n * m);
  float* y = malloc(sizeof(float) * n);
  int64_t k = 0;
  indptr[0] = 0;
  for (int64_t i = 0; i < n; ++i) {
    for (int64_t a = 0; a < m; ++a) {
      if ((double)(xs() % 1000) / 1000.0 < nan_frac) continue;
      idx[k] = (int32_t)a;
      val[k] = (xs() % 7 == 0) ? NAN : (float)((int)(xs() % 9) - 4) * 0.5f;
      ++k;
    }
    indptr[i + 1] = k;
    y[i] = loss == 0 ? (float)(xs() % 100) / 50.0f : (float)(xs() % 2);
  }
  orc_params P = {d, T, 1.0, 0.0, 0.5, 0.0, loss};
  const int64_t NH = ((int64_t)1 << (d + 1)) - 1;
  orc_node* nodes = calloc((size_t)(T * NH), sizeof(orc_node));
  orc_node* again = calloc((size_t)(T * NH), sizeof(orc_node));
  double* margin = malloc(sizeof(double) * n);
  double* pred = malloc(sizeof(double) * n);
  orc_stats st;
  int rc = orc_train(n, m, indptr, idx, val, y, &P, NULL, nodes, margin, &st);
  rc |= orc_train(n, m, indptr, idx, val, y, &P, nodes, again, margin, &st);  /* follow mode */
  orc_predict(n, indptr, idx, val, nodes, T, d, P.eta, P.base_margin, pred);
  for (int64_t i = 0; i < n; ++i)
    if (pred[i] != margin[i]) rc |= 2;
  if (st.nodes_mismatch) rc |= 4;
  free(indptr); free(idx); free(val); free(y); free(nodes); free(again); free(margin); free(pred);
  return rc;
}

int main(void) {
  int rc = 0;
  /* Table I: x1 = {a3:0.1}, x2 = {a1:1.2, a3:0.1, a4:0.6}, x3 = {a1:0.5, a2:1.0}, x4 = {a1:1.2, a3:2.0} */
  {
    int64_t ip[5] = {0, 1, 4, 6, 8};
    int32_t ix[8] = {2, 0, 2, 3, 0, 1, 0, 2};
    float vv[8] = {0.1f, 1.2f, 0.1f, 0.6f, 0.5f, 1.0f, 1.2f, 2.0f};
    float yy[4] = {1, 0, 1, 0};
    orc_params P = {2, 2, 1.0, 0.0, 1.0, 0.0, 0};
    orc_node nodes[2 * 7];
    double margin[4];
    orc_stats st;
    rc |= orc_train(4, 4, ip, ix, vv, yy, &P, NULL, nodes, margin, &st);
  }
  for (int s = 0; s < 12; ++s) rc |= run(3 + s * 17, 2 + s % 5, 0.25, s % 2, 1 + s % 4, 2);
  rc |= run(400, 6, 0.0, 1, 6, 3);
  printf("rc=%d\n", rc);
  return rc;
}
