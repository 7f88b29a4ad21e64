/*
 * ttemb_oracle.h -- CPU oracle for the TT-EmbeddingBag hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load or call this.
 * It shares no code, header, table or constant with the CUDA path
 * (paper_conf_sc_wangwfmmd22_b200/csrc) and neither side includes the other.
 *
 * Plain, slow, fp64 loops written from PAPER.md (cited P:<line>):
 *   Eq. 1-2  TT table element = product of core slices
 *   Eq. 3    TT index conversion, big-endian digits
 *   Eq. 4    bag = sum of rows
 *   Eq. 6    core gradient = left^T . dL/de . right^T
 *   P:193    gradients aggregated per unique row            (exact algebra)
 *   P:195-6  core update (SGD / Adagrad; R15)
 * The oracle evaluates every unique row on its own (no prefix reuse).
 *
 * Layouts (R4): per table t with row factors (m1,m2,m3),
 *   C1[m1][n1][R], C2[m2][R][n2][R], C3[m3][R][n3]   (float32 inputs)
 * indices int64 [nnz]; offsets int64 [T*B+1], table-major: bag (t,b) is
 * indices[offsets[t*B+b] .. offsets[t*B+b+1]); out [B][T][N].
 *
 * Status codes: 0 ok, -1 invalid argument / offsets, -3 index out of range.
 */
#ifndef TTEMB_ORACLE_H
#define TTEMB_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  int32_t T;              /* number of tables */
  const int64_t* rows;    /* [T] M_t */
  const int32_t* mfac;    /* [T][3] row factors, prod >= M_t */
  int32_t n[3];           /* column factors, N = n1*n2*n3 */
  int32_t R;              /* TT rank, R1 = R2 = R, R0 = R3 = 1 */
  const int32_t* dense;   /* [T] or NULL: dense[t] != 0 = table t kept uncompressed (hybrid
                             placement): its "C1" is the plain table W[M][N], C2 / C3 are
                             absent (NULL), row factors ignored */
} ttref_shape;

/* Eq. 3 digits of row id i of a table with factors m[3]. */
void ttref_digits(const int32_t m[3], int64_t i, int64_t d[3]);

/* One row of W_t (Eq. 2) as the matrix chain (C1[i1] C2[i2]) C3[i3]; e[N]. */
void ttref_row_chain(const ttref_shape* s, int t, const float* C1, const float* C2,
                     const float* C3, int64_t row, double* e);
/* The same row as the literal sum over (r1, r2) for every element (Eq. 1). */
void ttref_row_literal(const ttref_shape* s, int t, const float* C1, const float* C2,
                       const float* C3, int64_t row, double* e);

/* Integer plan: arrays sized nnz (U, P, NG <= nnz), the
 * *_off / row_seg arrays one more.  counts = {U, P, NG}.  Plan keys number the TT tables first
 * (user order), then the dense tables; dense rows have row_pfx = 0xFFFFFFFF, row_i3 = 0 and no
 * prefix, so row_seg[P] = number of TT rows. */
int ttref_plan(const ttref_shape* s, const int64_t* indices, const int64_t* offsets,
               int64_t nnz, int32_t B,
               uint32_t* skey, uint32_t* spos, uint32_t* bag_of,
               uint32_t* ukey, uint32_t* seg_off, uint32_t* inverse,
               uint32_t* row_pfx, uint32_t* row_i3,
               uint32_t* pfx_t, uint32_t* pfx_i1, uint32_t* pfx_i2, uint32_t* row_seg,
               uint32_t* grp_pfx, uint32_t* grp_off, uint32_t* grp_t, uint32_t* grp_i2,
               int64_t counts[3]);

/* Forward: out[B][T][N] (fp64).  literal != 0 uses ttref_row_literal. */
int ttref_forward(const ttref_shape* s, const float* const* C1, const float* const* C2,
                  const float* const* C3, const int64_t* indices, const int64_t* offsets,
                  int64_t nnz, int32_t B, int literal, double* out);

/* nn.EmbeddingBag pooling variants ("drop-in replacement of nn.EmbeddingBag"):
 * mode 0 = sum (psw = per-sample weights [nnz] or NULL), mode 1 = mean (psw must be NULL,
 * empty bag -> 0).  out[b][t] = sum_j w_j W_t[idx_j], w_j = psw[j] or 1 or 1/|bag|. */
int ttref_forward_ex(const ttref_shape* s, const float* const* C1, const float* const* C2,
                     const float* const* C3, const int64_t* indices, const int64_t* offsets,
                     int64_t nnz, int32_t B, const float* psw, int mode, int literal, double* out);

/* Backward: dC_k (fp64, same layouts as the cores, overwritten) of
 * L = sum(out * grad_out), grad_out [B][T][N] float32.  literal != 0 uses the
 * 6-deep loop nest per element instead of explicit partial products. */
int ttref_backward(const ttref_shape* s, const float* const* C1, const float* const* C2,
                   const float* const* C3, const int64_t* indices, const int64_t* offsets,
                   int64_t nnz, int32_t B, const float* grad_out, int literal,
                   double* const* dC1, double* const* dC2, double* const* dC3);

/* Backward of the weighted / mean forward (G_u = sum_j w_j grad_out[bag(j)]). */
int ttref_backward_ex(const ttref_shape* s, const float* const* C1, const float* const* C2,
                      const float* const* C3, const int64_t* indices, const int64_t* offsets,
                      int64_t nnz, int32_t B, const float* psw, int mode, const float* grad_out,
                      int literal, double* const* dC1, double* const* dC2, double* const* dC3);

/* Update (a12): opt 0 = SGD  p -= lr g;  opt 1 = Adagrad (PyTorch semantics):
 * s += g^2; p -= lr g / (sqrt(s) + eps).  fp64 math, rounded to fp32 once. */
int ttref_update(int opt, double lr, double eps, int64_t n, float* param, float* state,
                 const double* grad);

/* Runtime index bijection (Sec. IV-B): New_Batch = { index_t(i_j) }.
 * bij[t] is table t's map [M_t] (new id of old id i); out_ids[j] = bij[t][indices[j]]
 * for every position j of every bag of table t.  -3 if an id or a mapped id is
 * outside [0, M_t), -1 for malformed offsets. */
int ttref_apply_bijection(const ttref_shape* s, const int64_t* const* bij, const int64_t* indices,
                          const int64_t* offsets, int64_t nnz, int32_t B, int64_t* out_ids);

/* Threads the oracle's OpenMP loops use (1 if built without OpenMP). */
int ttref_num_threads(void);

#ifdef __cplusplus
}
#endif
#endif
