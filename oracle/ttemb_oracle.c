/*
 * ttemb_oracle.c -- plain, slow, obviously-correct CPU oracle (fp64).
 *
 * TEST INFRASTRUCTURE ONLY (see ttemb_oracle.h).  Nothing here is blocked,
 * fused or reordered beyond what the paper's definitions state; OpenMP only
 * splits independent loop iterations, and every floating-point sum is taken
 * in a fixed order that does not depend on the thread count.
 *
 * Parity status (pins live in tests/test_oracle_pins.py):
 *   ttref_digits       pinned: Fig. 5(b) worked example, brute force
 *   ttref_row_*        pinned: dense materialisation + torch embedding_bag,
 *                      R=1 Kronecker closed form, identity-core table
 *   ttref_plan         pinned: numpy.unique / stable argsort / unravel_index
 *   ttref_forward      pinned: dense embedding_bag on the materialised table
 *   ttref_backward     pinned: torch.autograd, exact central differences
 *   ttref_update       pinned: torch.optim.SGD / torch.optim.Adagrad
 */
#include "ttemb_oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

int ttref_num_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

/* Eq. 3:  i_k = floor(i_emb / prod_{l>k} m_l) mod m_k. */
void ttref_digits(const int32_t m[3], int64_t i, int64_t d[3]) {
  for (int k = 0; k < 3; ++k) {
    int64_t div = 1;
    for (int l = k + 1; l < 3; ++l) div *= m[l];
    d[k] = (i / div) % m[k];
  }
}

/* Slice pointers of table t for row `row` (Eq. 2: one slice per core). */
static void slices(const ttref_shape* s, int t, const float* C1, const float* C2,
                   const float* C3, int64_t row, const float** a, const float** b,
                   const float** c) {
  const int32_t* m = s->mfac + 3 * t;
  const int n1 = s->n[0], n2 = s->n[1], n3 = s->n[2], R = s->R;
  int64_t d[3];
  ttref_digits(m, row, d);
  *a = C1 + d[0] * (int64_t)n1 * R;            /* C1[i1] : [n1][R]      */
  *b = C2 + d[1] * (int64_t)R * n2 * R;        /* C2[i2] : [R][n2][R]   */
  *c = C3 + d[2] * (int64_t)R * n3;            /* C3[i3] : [R][n3]      */
}

/* Eq. 2 as a chain of two matrix products: L = C1[i1] C2[i2], e = L C3[i3].
 * Column order col = (j1*n2 + j2)*n3 + j3 (R2). */
void ttref_row_chain(const ttref_shape* s, int t, const float* C1, const float* C2,
                     const float* C3, int64_t row, double* e) {
  const int n1 = s->n[0], n2 = s->n[1], n3 = s->n[2], R = s->R;
  const float *a, *b, *c;
  slices(s, t, C1, C2, C3, row, &a, &b, &c);
  double* L = (double*)malloc(sizeof(double) * (size_t)n1 * n2 * R);
  for (int j1 = 0; j1 < n1; ++j1)
    for (int j2 = 0; j2 < n2; ++j2)
      for (int r2 = 0; r2 < R; ++r2) {
        double acc = 0.0;
        for (int r1 = 0; r1 < R; ++r1)
          acc += (double)a[j1 * R + r1] * (double)b[(r1 * n2 + j2) * R + r2];
        L[(j1 * n2 + j2) * R + r2] = acc;
      }
  for (int j1 = 0; j1 < n1; ++j1)
    for (int j2 = 0; j2 < n2; ++j2)
      for (int j3 = 0; j3 < n3; ++j3) {
        double acc = 0.0;
        for (int r2 = 0; r2 < R; ++r2)
          acc += L[(j1 * n2 + j2) * R + r2] * (double)c[r2 * n3 + j3];
        e[(j1 * n2 + j2) * n3 + j3] = acc;
      }
  free(L);
}

/* Eq. 1 literally: T(i,j) = sum_{r1,r2} C1(i1j1, r1) C2(r1, i2j2, r2) C3(r2, i3j3). */
void ttref_row_literal(const ttref_shape* s, int t, const float* C1, const float* C2,
                       const float* C3, int64_t row, double* e) {
  const int n1 = s->n[0], n2 = s->n[1], n3 = s->n[2], R = s->R;
  const float *a, *b, *c;
  slices(s, t, C1, C2, C3, row, &a, &b, &c);
  for (int j1 = 0; j1 < n1; ++j1)
    for (int j2 = 0; j2 < n2; ++j2)
      for (int j3 = 0; j3 < n3; ++j3) {
        double acc = 0.0;
        for (int r1 = 0; r1 < R; ++r1)
          for (int r2 = 0; r2 < R; ++r2)
            acc += (double)a[j1 * R + r1] * (double)b[(r1 * n2 + j2) * R + r2] *
                   (double)c[r2 * n3 + j3];
        e[(j1 * n2 + j2) * n3 + j3] = acc;
      }
}

/* ------------------------------------------------------------------------ */
/* Input validation and keys                                                 */
/* ------------------------------------------------------------------------ */
static int is_dense(const ttref_shape* s, int t) { return s->dense && s->dense[t]; }

static int check_shape(const ttref_shape* s) {
  if (!s || s->T < 1 || !s->rows || !s->mfac || s->R < 1) return -1;
  for (int k = 0; k < 3; ++k) if (s->n[k] < 1) return -1;
  uint64_t tot = 0;
  for (int t = 0; t < s->T; ++t) {
    const int32_t* m = s->mfac + 3 * t;
    if (s->rows[t] < 1) return -1;
    if (!is_dense(s, t)) {
      if (m[0] < 1 || m[1] < 1 || m[2] < 1) return -1;
      if ((int64_t)m[0] * m[1] * m[2] < s->rows[t]) return -1;
    }
    tot += (uint64_t)s->rows[t];
  }
  if (tot > 0xFFFFFFFFull) return -1;
  return 0;
}

static int check_offsets(const int64_t* offsets, int64_t nbags, int64_t nnz) {
  if (offsets[0] != 0 || offsets[nbags] != nnz) return -1;
  for (int64_t b = 0; b < nbags; ++b)
    if (offsets[b + 1] < offsets[b]) return -1;
  return 0;
}

/* key_j = rowbase_t + idx_j (rowbase = exclusive prefix sum of M_t), plus the
 * output row b*T + t of the bag holding position j. */
static int build_keys(const ttref_shape* s, const int64_t* indices, const int64_t* offsets,
                      int64_t nnz, int32_t B, uint32_t* key, uint32_t* bag_of) {
  const int T = s->T;
  if (check_offsets(offsets, (int64_t)T * B, nnz)) return -1;
  uint64_t base = 0;
  int bad = 0;
  for (int t = 0; t < T; ++t) {
    for (int32_t b = 0; b < B; ++b) {
      const int64_t bag = (int64_t)t * B + b;
      for (int64_t j = offsets[bag]; j < offsets[bag + 1]; ++j) {
        const int64_t id = indices[j];
        if (id < 0 || id >= s->rows[t]) { bad = 1; key[j] = (uint32_t)base; }
        else key[j] = (uint32_t)(base + (uint64_t)id);
        if (bag_of) bag_of[j] = (uint32_t)((int64_t)b * T + t);
      }
    }
    base += (uint64_t)s->rows[t];
  }
  return bad ? -3 : 0;
}

/* Weight of position j in its bag (nn.EmbeddingBag semantics, P:48 / P:306 drop-in):
 * mode 0 (sum): psw[j] if per-sample weights are given, else 1; mode 1 (mean): 1 / |bag|
 * (PyTorch allows per-sample weights only with sum).  NULL result = all ones. */
static double* position_weights(const ttref_shape* s, const int64_t* offsets, int64_t nnz, int32_t B,
                                const float* psw, int mode) {
  if (!psw && mode == 0) return NULL;
  double* w = (double*)malloc(sizeof(double) * (size_t)(nnz ? nnz : 1));
  for (int64_t bag = 0; bag < (int64_t)s->T * B; ++bag) {
    const int64_t a = offsets[bag], e = offsets[bag + 1];
    for (int64_t j = a; j < e; ++j) w[j] = mode == 1 ? 1.0 / (double)(e - a) : (double)psw[j];
  }
  return w;
}

static int table_of_key(const ttref_shape* s, uint32_t key, uint64_t* rowbase) {
  uint64_t base = 0;
  for (int t = 0; t < s->T; ++t) {
    if ((uint64_t)key < base + (uint64_t)s->rows[t]) { *rowbase = base; return t; }
    base += (uint64_t)s->rows[t];
  }
  *rowbase = base;
  return s->T - 1;
}

typedef struct { uint32_t key, pos; } kp_t;
static int cmp_kp(const void* x, const void* y) {
  const kp_t* a = (const kp_t*)x; const kp_t* b = (const kp_t*)y;
  if (a->key != b->key) return a->key < b->key ? -1 : 1;
  return a->pos < b->pos ? -1 : (a->pos > b->pos);   /* stable: ties by position */
}

/* Sorted distinct keys of the batch; returns U. */
static int64_t unique_keys(const uint32_t* key, int64_t nnz, uint32_t* ukey) {
  kp_t* v = (kp_t*)malloc(sizeof(kp_t) * (size_t)(nnz ? nnz : 1));
  for (int64_t j = 0; j < nnz; ++j) { v[j].key = key[j]; v[j].pos = (uint32_t)j; }
  qsort(v, (size_t)nnz, sizeof(kp_t), cmp_kp);
  int64_t U = 0;
  for (int64_t k = 0; k < nnz; ++k)
    if (k == 0 || v[k].key != v[k - 1].key) ukey[U++] = v[k].key;
  free(v);
  return U;
}

static int64_t find_key(const uint32_t* ukey, int64_t U, uint32_t key) {
  int64_t lo = 0, hi = U - 1;
  while (lo <= hi) {
    int64_t mid = (lo + hi) / 2;
    if (ukey[mid] == key) return mid;
    if (ukey[mid] < key) lo = mid + 1; else hi = mid - 1;
  }
  return -1;
}

/* ------------------------------------------------------------------------ */
/* Plan                                                                      */
/* ------------------------------------------------------------------------ */
/* The plan orders distinct rows "group-major": by table t, then the C2 digit i2, then the C1
 * digit i1, then i3 (R29), i.e. by the plan key
 *     K(t, i) = gbase_t + (i2 * m1 + i1) * m3 + i3,   gbase_t = sum_{t' < t} m1 m2 m3,
 * with (i1, i2, i3) the digits of Eq. 3.  Rows sharing a prefix (i1, i2) (Alg. 1's
 * Buf_idx = idx / length_3) are then consecutive, and prefixes sharing a C2 slice
 * (the i2-groups) are consecutive too. */
static int plan_keys(const ttref_shape* s, const int64_t* indices, const int64_t* offsets,
                     int64_t nnz, int32_t B, uint32_t* key, uint32_t* bag_of) {
  const int T = s->T;
  if (check_offsets(offsets, (int64_t)T * B, nnz)) return -1;
  uint64_t gbase = 0;
  int bad = 0;
  for (int pass = 0; pass < 2; ++pass)       /* TT tables first, then the dense ones */
    for (int t = 0; t < T; ++t) {
      if (is_dense(s, t) != pass) continue;
      const int32_t* m = s->mfac + 3 * t;
      for (int32_t b = 0; b < B; ++b) {
        const int64_t bag = (int64_t)t * B + b;
        for (int64_t j = offsets[bag]; j < offsets[bag + 1]; ++j) {
          const int64_t id = indices[j];
          if (id < 0 || id >= s->rows[t]) { bad = 1; key[j] = (uint32_t)gbase; }
          else if (pass) key[j] = (uint32_t)(gbase + (uint64_t)id);
          else {
            int64_t d[3];
            ttref_digits(m, id, d);
            key[j] = (uint32_t)(gbase + (uint64_t)((d[1] * m[0] + d[0]) * m[2] + d[2]));
          }
          bag_of[j] = (uint32_t)((int64_t)b * T + t);
        }
      }
      gbase += pass ? (uint64_t)s->rows[t] : (uint64_t)m[0] * m[1] * m[2];
    }
  return bad ? -3 : 0;
}

int ttref_plan(const ttref_shape* s, const int64_t* indices, const int64_t* offsets,
               int64_t nnz, int32_t B,
               uint32_t* skey, uint32_t* spos, uint32_t* bag_of,
               uint32_t* ukey, uint32_t* seg_off, uint32_t* inverse,
               uint32_t* row_pfx, uint32_t* row_i3,
               uint32_t* pfx_t, uint32_t* pfx_i1, uint32_t* pfx_i2, uint32_t* row_seg,
               uint32_t* grp_pfx, uint32_t* grp_off, uint32_t* grp_t, uint32_t* grp_i2,
               int64_t counts[3]) {
  if (check_shape(s) || B < 0 || nnz < 0) return -1;
  uint32_t* key = (uint32_t*)malloc(sizeof(uint32_t) * (size_t)(nnz ? nnz : 1));
  int rc = plan_keys(s, indices, offsets, nnz, B, key, bag_of);
  if (rc) { free(key); return rc; }

  /* stable sort of (key, position) */
  kp_t* v = (kp_t*)malloc(sizeof(kp_t) * (size_t)(nnz ? nnz : 1));
  for (int64_t j = 0; j < nnz; ++j) { v[j].key = key[j]; v[j].pos = (uint32_t)j; }
  qsort(v, (size_t)nnz, sizeof(kp_t), cmp_kp);
  int64_t U = 0;
  for (int64_t k = 0; k < nnz; ++k) {
    skey[k] = v[k].key; spos[k] = v[k].pos;
    if (k == 0 || v[k].key != v[k - 1].key) { ukey[U] = v[k].key; seg_off[U] = (uint32_t)k; ++U; }
    inverse[v[k].pos] = (uint32_t)(U - 1);
  }
  seg_off[U] = (uint32_t)nnz;

  /* digits back from the plan key; unique prefixes (t, i2, i1) and i2-groups (t, i2) are runs */
  int64_t P = 0, NG = 0, Utt = U;
  uint64_t ttkeys = 0;
  for (int t = 0; t < s->T; ++t)
    if (!is_dense(s, t)) ttkeys += (uint64_t)s->mfac[3 * t] * s->mfac[3 * t + 1] * s->mfac[3 * t + 2];
  for (int64_t u = 0; u < U; ++u) {
    if ((uint64_t)ukey[u] >= ttkeys) {          /* a dense-table row: no TT digits, no prefix */
      if (Utt == U) Utt = u;
      row_pfx[u] = 0xFFFFFFFFu;
      row_i3[u] = 0;
      continue;
    }
    uint64_t gbase = 0;
    int t = 0;
    for (; t < s->T - 1; ++t) {
      if (is_dense(s, t)) continue;
      const int32_t* m = s->mfac + 3 * t;
      const uint64_t span = (uint64_t)m[0] * m[1] * m[2];
      if ((uint64_t)ukey[u] < gbase + span) break;
      gbase += span;
    }
    const int32_t* m = s->mfac + 3 * t;
    const uint64_t local = (uint64_t)ukey[u] - gbase;
    const uint32_t i3 = (uint32_t)(local % (uint64_t)m[2]);
    const uint64_t pq = local / (uint64_t)m[2];           /* i2 * m1 + i1 */
    const uint32_t i1 = (uint32_t)(pq % (uint64_t)m[0]), i2 = (uint32_t)(pq / (uint64_t)m[0]);
    if (P == 0 || pfx_t[P - 1] != (uint32_t)t || pfx_i2[P - 1] != i2 || pfx_i1[P - 1] != i1) {
      if (P == 0 || pfx_t[P - 1] != (uint32_t)t || pfx_i2[P - 1] != i2) {
        grp_off[NG] = (uint32_t)P; grp_t[NG] = (uint32_t)t; grp_i2[NG] = i2; ++NG;
      }
      pfx_t[P] = (uint32_t)t; pfx_i1[P] = i1; pfx_i2[P] = i2; row_seg[P] = (uint32_t)u;
      grp_pfx[P] = (uint32_t)P;
      ++P;
    }
    row_pfx[u] = (uint32_t)(P - 1);
    row_i3[u] = i3;
  }
  row_seg[P] = (uint32_t)Utt;
  grp_off[NG] = (uint32_t)P;
  counts[0] = U; counts[1] = P; counts[2] = NG;
  free(v); free(key);
  return 0;
}

/* ------------------------------------------------------------------------ */
/* Forward (Eq. 2-4)                                                         */
/* ------------------------------------------------------------------------ */
/* the lookup uses New_Batch = { index(i_j) } instead of the raw ids. */
int ttref_apply_bijection(const ttref_shape* s, const int64_t* const* bij, const int64_t* indices,
                          const int64_t* offsets, int64_t nnz, int32_t B, int64_t* out_ids) {
  if (check_shape(s) || B < 0 || nnz < 0) return -1;
  const int T = s->T;
  if (offsets[0] != 0 || offsets[(int64_t)T * B] != nnz) return -1;
  for (int t = 0; t < T; ++t) {
    const int64_t M = s->rows[t];
    for (int32_t b = 0; b < B; ++b) {
      const int64_t bag = (int64_t)t * B + b;
      if (offsets[bag + 1] < offsets[bag]) return -1;
      for (int64_t j = offsets[bag]; j < offsets[bag + 1]; ++j) {
        const int64_t i = indices[j];
        if (i < 0 || i >= M) return -3;
        const int64_t k = bij[t][i];
        if (k < 0 || k >= M) return -3;
        out_ids[j] = k;
      }
    }
  }
  return 0;
}

int ttref_forward(const ttref_shape* s, const float* const* C1, const float* const* C2,
                  const float* const* C3, const int64_t* indices, const int64_t* offsets,
                  int64_t nnz, int32_t B, int literal, double* out) {
  return ttref_forward_ex(s, C1, C2, C3, indices, offsets, nnz, B, NULL, 0, literal, out);
}

int ttref_forward_ex(const ttref_shape* s, const float* const* C1, const float* const* C2,
                     const float* const* C3, const int64_t* indices, const int64_t* offsets,
                     int64_t nnz, int32_t B, const float* psw, int mode, int literal, double* out) {
  if (check_shape(s) || B < 0 || nnz < 0 || mode < 0 || mode > 1 || (psw && mode != 0)) return -1;
  const int T = s->T;
  const int N = s->n[0] * s->n[1] * s->n[2];
  uint32_t* key = (uint32_t*)malloc(sizeof(uint32_t) * (size_t)(nnz ? nnz : 1));
  int rc = build_keys(s, indices, offsets, nnz, B, key, NULL);
  if (rc) { free(key); return rc; }
  uint32_t* ukey = (uint32_t*)malloc(sizeof(uint32_t) * (size_t)(nnz ? nnz : 1));
  const int64_t U = unique_keys(key, nnz, ukey);

  /* every distinct row evaluated once on its own (memoised Eq. 2) */
  double* rows = (double*)malloc(sizeof(double) * (size_t)(U ? U : 1) * N);
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t u = 0; u < U; ++u) {
    uint64_t rb; int t = table_of_key(s, ukey[u], &rb);
    int64_t row = (int64_t)ukey[u] - (int64_t)rb;
    if (is_dense(s, t)) {                       /* uncompressed table: W[row] */
      for (int c = 0; c < N; ++c) rows[u * N + c] = (double)C1[t][row * N + c];
    } else if (literal) ttref_row_literal(s, t, C1[t], C2[t], C3[t], row, rows + u * N);
    else ttref_row_chain(s, t, C1[t], C2[t], C3[t], row, rows + u * N);
  }

  /* Eq. 4: out[b][t] = sum of the rows of bag (t, b), in index order; empty -> 0.
   * Weighted / mean bags (nn.EmbeddingBag): out = sum_j w_j row_j */
  double* w = position_weights(s, offsets, nnz, B, psw, mode);
  memset(out, 0, sizeof(double) * (size_t)B * T * N);
  for (int t = 0; t < T; ++t)
    for (int32_t b = 0; b < B; ++b) {
      const int64_t bag = (int64_t)t * B + b;
      double* o = out + ((int64_t)b * T + t) * N;
      for (int64_t j = offsets[bag]; j < offsets[bag + 1]; ++j) {
        const double* e = rows + find_key(ukey, U, key[j]) * N;
        const double wj = w ? w[j] : 1.0;
        for (int c = 0; c < N; ++c) o[c] += wj * e[c];
      }
    }
  free(w); free(rows); free(ukey); free(key);
  return 0;
}

/* ------------------------------------------------------------------------ */
/* Backward (Eq. 6 read as left^T . G . right^T)          */
/* ------------------------------------------------------------------------ */

/* Per-row core gradients from the aggregated row gradient G[N] (textbook chain
 * rule with explicit partial products):
 *   dC1[j1][r1]     = sum_{j2,j3} G[j1,j2,j3] Rt[r1,j2,j3],  Rt = C2[i2] C3[i3]
 *   dC2[r1][j2][r2] = sum_{j1,j3} C1[j1,r1] G[j1,j2,j3] C3[r2,j3]
 *   dC3[r2][j3]     = sum_{j1,j2} Lf[j1,j2,r2] G[j1,j2,j3],  Lf = C1[i1] C2[i2] */
static void row_grads(const ttref_shape* s, const float* a, const float* b, const float* c,
                      const double* G, double* g1, double* g2, double* g3, double* tmp) {
  const int n1 = s->n[0], n2 = s->n[1], n3 = s->n[2], R = s->R;
  /* right partial product Rt[r1][j2][j3] */
  double* Rt = tmp;
  for (int r1 = 0; r1 < R; ++r1)
    for (int j2 = 0; j2 < n2; ++j2)
      for (int j3 = 0; j3 < n3; ++j3) {
        double acc = 0.0;
        for (int r2 = 0; r2 < R; ++r2) acc += (double)b[(r1 * n2 + j2) * R + r2] * (double)c[r2 * n3 + j3];
        Rt[(r1 * n2 + j2) * n3 + j3] = acc;
      }
  for (int j1 = 0; j1 < n1; ++j1)
    for (int r1 = 0; r1 < R; ++r1) {
      double acc = 0.0;
      for (int j2 = 0; j2 < n2; ++j2)
        for (int j3 = 0; j3 < n3; ++j3)
          acc += G[(j1 * n2 + j2) * n3 + j3] * Rt[(r1 * n2 + j2) * n3 + j3];
      g1[j1 * R + r1] = acc;
    }
  /* middle core: left = C1[i1], right = C3[i3] */
  double* H = tmp;   /* H[j1][j2][r2] = sum_j3 G[j1,j2,j3] C3[r2,j3] */
  for (int j1 = 0; j1 < n1; ++j1)
    for (int j2 = 0; j2 < n2; ++j2)
      for (int r2 = 0; r2 < R; ++r2) {
        double acc = 0.0;
        for (int j3 = 0; j3 < n3; ++j3) acc += G[(j1 * n2 + j2) * n3 + j3] * (double)c[r2 * n3 + j3];
        H[(j1 * n2 + j2) * R + r2] = acc;
      }
  for (int r1 = 0; r1 < R; ++r1)
    for (int j2 = 0; j2 < n2; ++j2)
      for (int r2 = 0; r2 < R; ++r2) {
        double acc = 0.0;
        for (int j1 = 0; j1 < n1; ++j1) acc += (double)a[j1 * R + r1] * H[(j1 * n2 + j2) * R + r2];
        g2[(r1 * n2 + j2) * R + r2] = acc;
      }
  /* left partial product Lf[j1][j2][r2] */
  double* Lf = tmp;
  for (int j1 = 0; j1 < n1; ++j1)
    for (int j2 = 0; j2 < n2; ++j2)
      for (int r2 = 0; r2 < R; ++r2) {
        double acc = 0.0;
        for (int r1 = 0; r1 < R; ++r1) acc += (double)a[j1 * R + r1] * (double)b[(r1 * n2 + j2) * R + r2];
        Lf[(j1 * n2 + j2) * R + r2] = acc;
      }
  for (int r2 = 0; r2 < R; ++r2)
    for (int j3 = 0; j3 < n3; ++j3) {
      double acc = 0.0;
      for (int j1 = 0; j1 < n1; ++j1)
        for (int j2 = 0; j2 < n2; ++j2)
          acc += Lf[(j1 * n2 + j2) * R + r2] * G[(j1 * n2 + j2) * n3 + j3];
      g3[r2 * n3 + j3] = acc;
    }
}

/* The same three gradients as literal sums over all free indices (tiny sizes). */
static void row_grads_literal(const ttref_shape* s, const float* a, const float* b,
                              const float* c, const double* G, double* g1, double* g2,
                              double* g3) {
  const int n1 = s->n[0], n2 = s->n[1], n3 = s->n[2], R = s->R;
  for (int j1 = 0; j1 < n1; ++j1)
    for (int r1 = 0; r1 < R; ++r1) {
      double acc = 0.0;
      for (int j2 = 0; j2 < n2; ++j2) for (int j3 = 0; j3 < n3; ++j3) for (int r2 = 0; r2 < R; ++r2)
        acc += G[(j1 * n2 + j2) * n3 + j3] * (double)b[(r1 * n2 + j2) * R + r2] * (double)c[r2 * n3 + j3];
      g1[j1 * R + r1] = acc;
    }
  for (int r1 = 0; r1 < R; ++r1)
    for (int j2 = 0; j2 < n2; ++j2)
      for (int r2 = 0; r2 < R; ++r2) {
        double acc = 0.0;
        for (int j1 = 0; j1 < n1; ++j1) for (int j3 = 0; j3 < n3; ++j3)
          acc += (double)a[j1 * R + r1] * G[(j1 * n2 + j2) * n3 + j3] * (double)c[r2 * n3 + j3];
        g2[(r1 * n2 + j2) * R + r2] = acc;
      }
  for (int r2 = 0; r2 < R; ++r2)
    for (int j3 = 0; j3 < n3; ++j3) {
      double acc = 0.0;
      for (int j1 = 0; j1 < n1; ++j1) for (int j2 = 0; j2 < n2; ++j2) for (int r1 = 0; r1 < R; ++r1)
        acc += (double)a[j1 * R + r1] * (double)b[(r1 * n2 + j2) * R + r2] * G[(j1 * n2 + j2) * n3 + j3];
      g3[r2 * n3 + j3] = acc;
    }
}

int ttref_backward(const ttref_shape* s, const float* const* C1, const float* const* C2,
                   const float* const* C3, const int64_t* indices, const int64_t* offsets,
                   int64_t nnz, int32_t B, const float* grad_out, int literal,
                   double* const* dC1, double* const* dC2, double* const* dC3) {
  return ttref_backward_ex(s, C1, C2, C3, indices, offsets, nnz, B, NULL, 0, grad_out, literal,
                           dC1, dC2, dC3);
}

int ttref_backward_ex(const ttref_shape* s, const float* const* C1, const float* const* C2,
                      const float* const* C3, const int64_t* indices, const int64_t* offsets,
                      int64_t nnz, int32_t B, const float* psw, int mode, const float* grad_out,
                      int literal, double* const* dC1, double* const* dC2, double* const* dC3) {
  if (check_shape(s) || B < 0 || nnz < 0 || mode < 0 || mode > 1 || (psw && mode != 0)) return -1;
  const int T = s->T;
  const int n1 = s->n[0], n2 = s->n[1], n3 = s->n[2], R = s->R;
  const int N = n1 * n2 * n3;
  const int64_t s1 = (int64_t)n1 * R, s2 = (int64_t)R * n2 * R, s3 = (int64_t)R * n3;

  for (int t = 0; t < T; ++t) {
    const int32_t* m = s->mfac + 3 * t;
    if (is_dense(s, t)) {                       /* dW of an uncompressed table */
      memset(dC1[t], 0, sizeof(double) * (size_t)s->rows[t] * N);
      continue;
    }
    memset(dC1[t], 0, sizeof(double) * (size_t)m[0] * s1);
    memset(dC2[t], 0, sizeof(double) * (size_t)m[1] * s2);
    memset(dC3[t], 0, sizeof(double) * (size_t)m[2] * s3);
  }
  uint32_t* key = (uint32_t*)malloc(sizeof(uint32_t) * (size_t)(nnz ? nnz : 1));
  uint32_t* bag = (uint32_t*)malloc(sizeof(uint32_t) * (size_t)(nnz ? nnz : 1));
  int rc = build_keys(s, indices, offsets, nnz, B, key, bag);
  if (rc) { free(key); free(bag); return rc; }
  uint32_t* ukey = (uint32_t*)malloc(sizeof(uint32_t) * (size_t)(nnz ? nnz : 1));
  const int64_t U = unique_keys(key, nnz, ukey);

  /* in-advance aggregation: G[u] = sum over the positions holding row u,
   * ascending position order */
  double* G = (double*)calloc((size_t)(U ? U : 1) * N, sizeof(double));
  double* w = position_weights(s, offsets, nnz, B, psw, mode);   /* dout/drow_j = w_j */
  for (int64_t j = 0; j < nnz; ++j) {
    double* g = G + find_key(ukey, U, key[j]) * N;
    const float* go = grad_out + (int64_t)bag[j] * N;
    const double wj = w ? w[j] : 1.0;
    for (int c = 0; c < N; ++c) g[c] += wj * (double)go[c];
  }
  free(w);

  /* uncompressed tables: dW[row] = G_u */
  for (int64_t u = 0; u < U; ++u) {
    uint64_t rb; int t = table_of_key(s, ukey[u], &rb);
    if (!is_dense(s, t)) continue;
    const int64_t row = (int64_t)ukey[u] - (int64_t)rb;
    for (int c = 0; c < N; ++c) dC1[t][row * N + c] += G[u * N + c];
  }

  /* chunks of unique rows: per-row contributions in parallel, then summed into
   * the core gradients in ascending row order (parallel over slice elements) */
  int64_t per_row = s1 + s2 + s3;
  int64_t CH = (int64_t)((256ull << 20) / (sizeof(double) * (size_t)per_row));
  if (CH < 1) CH = 1;
  double* contrib = (double*)malloc(sizeof(double) * (size_t)CH * per_row);
  int64_t* dig = (int64_t*)malloc(sizeof(int64_t) * 4 * (size_t)CH);
  const int64_t tmpn = (int64_t)n1 * n2 * R > (int64_t)R * n2 * n3 ? (int64_t)n1 * n2 * R : (int64_t)R * n2 * n3;
  for (int64_t u0 = 0; u0 < U; u0 += CH) {
    const int64_t u1 = (u0 + CH < U) ? u0 + CH : U;
#pragma omp parallel
    {
      double* tmp = (double*)malloc(sizeof(double) * (size_t)tmpn);
#pragma omp for schedule(dynamic, 16)
      for (int64_t u = u0; u < u1; ++u) {
        uint64_t rb; int t = table_of_key(s, ukey[u], &rb);
        int64_t row = (int64_t)ukey[u] - (int64_t)rb;
        if (is_dense(s, t)) { dig[4 * (u - u0)] = -1; continue; }
        int64_t d[3];
        ttref_digits(s->mfac + 3 * t, row, d);
        int64_t* dg = dig + 4 * (u - u0);
        dg[0] = t; dg[1] = d[0]; dg[2] = d[1]; dg[3] = d[2];
        const float* a = C1[t] + d[0] * s1;
        const float* b = C2[t] + d[1] * s2;
        const float* c = C3[t] + d[2] * s3;
        double* cr = contrib + (u - u0) * per_row;
        if (literal) row_grads_literal(s, a, b, c, G + u * N, cr, cr + s1, cr + s1 + s2);
        else row_grads(s, a, b, c, G + u * N, cr, cr + s1, cr + s1 + s2, tmp);
      }
      free(tmp);
    }
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < per_row; ++e) {
      for (int64_t u = u0; u < u1; ++u) {
        const int64_t* dg = dig + 4 * (u - u0);
        if (dg[0] < 0) continue;                  /* dense-table row (done above) */
        const double v = contrib[(u - u0) * per_row + e];
        if (e < s1) dC1[dg[0]][dg[1] * s1 + e] += v;
        else if (e < s1 + s2) dC2[dg[0]][dg[2] * s2 + (e - s1)] += v;
        else dC3[dg[0]][dg[3] * s3 + (e - s1 - s2)] += v;
      }
    }
  }
  free(dig); free(contrib); free(G); free(ukey); free(bag); free(key);
  return 0;
}

/* ------------------------------------------------------------------------ */
/* Update (a12; R15)                                     */
/* ------------------------------------------------------------------------ */
int ttref_update(int opt, double lr, double eps, int64_t n, float* param, float* state,
                 const double* grad) {
  if (n < 0 || (opt != 0 && opt != 1) || (opt == 1 && !state)) return -1;
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    double p = (double)param[i];
    const double g = grad[i];
    if (opt == 0) {
      p -= lr * g;
    } else {
      const double sum = (double)state[i] + g * g;
      p -= lr * g / (sqrt(sum) + eps);
      state[i] = (float)sum;
    }
    param[i] = (float)p;
  }
  return 0;
}
