/*
 * oracle.c — CPU fp64 ORACLE for column-vector-sparse SpMM / SDDMM.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no code, header,
 * table or helper with the CUDA path (paper_conf_sc_chenqldx21_b200/csrc, include/vs.h).
 *
 * It is the plain definition of what the method computes (Chen et al., SC'21; "P:n" =
 * line n of PAPER.md), written out with no blocking, fusion or reordering:
 *
 *   oracle_encode  §4.2, Fig. 8 P:599-613 — column-vector sparse encoding.
 *   oracle_decode  inverse scatter of the encoding (test helper).
 *   oracle_spmm    §4.1 P:571-588 — C = A*B with A in the encoding, B/C row-major.
 *   oracle_sddmm   §4.1, §6.4 P:1178-1179 — (A*B) sampled at a column-vector
 *                  mask, B passed transposed (Bt[N x K] row-major).
 *   *_sample       the same sums for a caller-chosen list of output elements (used where
 *                  the full problem is too large for the host).
 *   oracle_softmax §7.4 Eq. 1 P:1535-1545 (NEXT item) — row softmax over the
 *                  stored entries of the column-vector matrix (the masked attention scores;
 *                  entries outside the mask are -inf in the dense view).
 *
 * Inputs are fp16 bit patterns (uint16_t); each is widened to double exactly by
 * half_to_double() and every product and sum is formed in double.  Alongside each result
 * the oracle returns the error scale S = sum |a*b| of the same terms, which the acceptance
 * rule |gpu - oracle| <= 2e-3*S + 2^-24 uses (north star).
 *
 * Pins (tests/test_oracle_*.py): Fig. 8 golden encoding; scipy CSR (V=1) and BSR (V x 1)
 * products; numpy fp64 brute force on tiny shapes; identity and integer-exact closed forms;
 * all-ones-mask SDDMM = GEMM; the SpMM/SDDMM adjoint identity.
 */
#define _POSIX_C_SOURCE 199309L
#include <stdint.h>
#include <stddef.h>
#include <stdlib.h>
#include <math.h>
#include <string.h>
#include <time.h>

/* IEEE binary16 -> double, exact.  sign(1) exponent(5, bias 15) mantissa(10). */
static double half_to_double(uint16_t h) {
  int sign = (h >> 15) & 1;
  int e = (h >> 10) & 0x1F;
  int m = h & 0x3FF;
  double v;
  if (e == 0)
    v = ldexp((double)m, -24); /* subnormal (or zero): m * 2^-14 * 2^-10 */
  else if (e == 31)
    v = (m == 0) ? INFINITY : NAN;
  else
    v = ldexp((double)(m + 1024), e - 25); /* (1 + m/1024) * 2^(e-15) */
  return sign ? -v : v;
}

double oracle_half_to_double(uint16_t h) { return half_to_double(h); }

static int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

/*
 * Encoding, Fig. 8 / §4.2: window w = rows [wV, wV+V); for k ascending keep column vector
 * (w, k) if any of its (existing) entries is nonzero — by mask byte when a mask is given,
 * else by fp16 bit pattern.  Kept vectors append k to col_idx and their V values (rows
 * >= M padded with +0.0 = bit pattern 0) to vals.  row_ptr[w+1] = number kept so far.
 * col_idx / vals may be NULL (count only).  Returns nnz_v.
 */
int64_t oracle_encode(int64_t M, int64_t K, int V, const uint16_t* dense, const uint8_t* mask,
                      int32_t* row_ptr, int32_t* col_idx, uint16_t* vals) {
  int64_t W = ceil_div(M, V);
  int64_t nnz = 0;
  row_ptr[0] = 0;
  for (int64_t w = 0; w < W; ++w) {
    for (int64_t k = 0; k < K; ++k) {
      int keep = 0;
      for (int r = 0; r < V; ++r) {
        int64_t i = w * V + r;
        if (i >= M) break;
        if (mask ? (mask[i * K + k] != 0) : (dense[i * K + k] != 0)) keep = 1;
      }
      if (!keep) continue;
      if (col_idx) col_idx[nnz] = (int32_t)k;
      if (vals) {
        for (int r = 0; r < V; ++r) {
          int64_t i = w * V + r;
          vals[nnz * V + r] = (i < M) ? dense[i * K + k] : (uint16_t)0;
        }
      }
      ++nnz;
    }
    row_ptr[w + 1] = (int32_t)nnz;
  }
  return nnz;
}

/* Inverse of the encoding: zero [M x K] then scatter every stored vector (rows < M). */
void oracle_decode(int64_t M, int64_t K, int V, const int32_t* row_ptr, const int32_t* col_idx,
                   const uint16_t* vals, uint16_t* dense_out) {
  int64_t W = ceil_div(M, V);
  memset(dense_out, 0, (size_t)(M * K) * sizeof(uint16_t));
  for (int64_t w = 0; w < W; ++w)
    for (int64_t p = row_ptr[w]; p < row_ptr[w + 1]; ++p)
      for (int r = 0; r < V; ++r) {
        int64_t i = w * V + r;
        if (i < M) dense_out[i * K + col_idx[p]] = vals[p * V + r];
      }
}

/*
 * SpMM, §4.1: C[i][j] = sum over the vectors p of window w = i / V of
 *   vals[p*V + r] * B[col_idx[p]][j],  r = i - wV.
 * C64 [M x N] and S64 [M x N] (S64 may be NULL) are written in full.
 */
void oracle_spmm(int64_t M, int64_t K, int64_t N, int V, const int32_t* row_ptr,
                 const int32_t* col_idx, const uint16_t* vals, const uint16_t* B,
                 double* C64, double* S64) {
  (void)K;
  int64_t W = ceil_div(M, V);
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t w = 0; w < W; ++w) {
    for (int r = 0; r < V; ++r) {
      int64_t i = w * V + r;
      if (i >= M) break;
      for (int64_t j = 0; j < N; ++j) {
        double acc = 0.0, sc = 0.0;
        for (int64_t p = row_ptr[w]; p < row_ptr[w + 1]; ++p) {
          double t = half_to_double(vals[p * V + r]) * half_to_double(B[(int64_t)col_idx[p] * N + j]);
          acc += t;
          sc += fabs(t);
        }
        C64[i * N + j] = acc;
        if (S64) S64[i * N + j] = sc;
      }
    }
  }
}

/*
 * SDDMM, §4.1 / §6.4: for every stored mask vector p of window w and r < V,
 *   out[p*V + r] = sum_{k<K} A[wV+r][k] * Bt[col_idx[p]][k]   (0 when wV+r >= M).
 * out64 / S64 (S64 may be NULL) have nnz_v*V entries.
 */
void oracle_sddmm(int64_t M, int64_t N, int64_t K, int V, const int32_t* row_ptr,
                  const int32_t* col_idx, const uint16_t* A, const uint16_t* Bt,
                  double* out64, double* S64) {
  (void)N;
  int64_t W = ceil_div(M, V);
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t w = 0; w < W; ++w) {
    for (int64_t p = row_ptr[w]; p < row_ptr[w + 1]; ++p) {
      for (int r = 0; r < V; ++r) {
        int64_t i = w * V + r;
        double acc = 0.0, sc = 0.0;
        if (i < M) {
          for (int64_t k = 0; k < K; ++k) {
            double t = half_to_double(A[i * K + k]) * half_to_double(Bt[(int64_t)col_idx[p] * K + k]);
            acc += t;
            sc += fabs(t);
          }
        }
        out64[p * V + r] = acc;
        if (S64) S64[p * V + r] = sc;
      }
    }
  }
}

/* SpMM for a list of output elements (rows[s], cols[s]); same sum as oracle_spmm. */
void oracle_spmm_sample(int64_t M, int64_t K, int64_t N, int V, const int32_t* row_ptr,
                        const int32_t* col_idx, const uint16_t* vals, const uint16_t* B,
                        int64_t nsamp, const int64_t* rows, const int64_t* cols,
                        double* out64, double* S64) {
  (void)M; (void)K;
#pragma omp parallel for schedule(static)
  for (int64_t s = 0; s < nsamp; ++s) {
    int64_t i = rows[s], j = cols[s];
    int64_t w = i / V;
    int r = (int)(i - w * V);
    double acc = 0.0, sc = 0.0;
    for (int64_t p = row_ptr[w]; p < row_ptr[w + 1]; ++p) {
      double t = half_to_double(vals[p * V + r]) * half_to_double(B[(int64_t)col_idx[p] * N + j]);
      acc += t;
      sc += fabs(t);
    }
    out64[s] = acc;
    if (S64) S64[s] = sc;
  }
}

/* SDDMM for a list of stored vectors: vec_p[s] is the vector index, vec_w[s] its window;
   writes V values per sample (out64[s*V + r]). */
void oracle_sddmm_sample(int64_t M, int64_t N, int64_t K, int V, const int32_t* col_idx,
                         const uint16_t* A, const uint16_t* Bt, int64_t nsamp,
                         const int64_t* vec_p, const int64_t* vec_w, double* out64,
                         double* S64) {
  (void)N;
#pragma omp parallel for schedule(static)
  for (int64_t s = 0; s < nsamp; ++s) {
    int64_t p = vec_p[s], w = vec_w[s];
    for (int r = 0; r < V; ++r) {
      int64_t i = w * V + r;
      double acc = 0.0, sc = 0.0;
      if (i < M) {
        for (int64_t k = 0; k < K; ++k) {
          double t = half_to_double(A[i * K + k]) * half_to_double(Bt[(int64_t)col_idx[p] * K + k]);
          acc += t;
          sc += fabs(t);
        }
      }
      out64[s * V + r] = acc;
      if (S64) S64[s * V + r] = sc;
    }
  }
}

/*
 * Row softmax (Eq. 1): for every row i = wV + r < M, over the stored vectors p of
 * window w: out[p*V + r] = exp(scale*x_p - m) / sum_q exp(scale*x_q - m), x_p = vals[p*V + r],
 * m = max_q scale*x_q.  Rows >= M get 0.
 */
void oracle_softmax(int64_t M, int V, const int32_t* row_ptr, const uint16_t* vals, double scale,
                    double* out64) {
  int64_t W = ceil_div(M, V);
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t w = 0; w < W; ++w) {
    for (int r = 0; r < V; ++r) {
      int64_t i = w * V + r;
      int64_t p;
      if (i >= M) {
        for (p = row_ptr[w]; p < row_ptr[w + 1]; ++p) out64[p * V + r] = 0.0;
        continue;
      }
      double m = -INFINITY, sum = 0.0;
      for (p = row_ptr[w]; p < row_ptr[w + 1]; ++p) {
        double x = scale * half_to_double(vals[p * V + r]);
        if (x > m) m = x;
      }
      if (m == -INFINITY) { /* every stored score is -inf: the row attends to nothing, 0
                               (reading R23; the plain formula gives 0/0) */
        for (p = row_ptr[w]; p < row_ptr[w + 1]; ++p) out64[p * V + r] = 0.0;
        continue;
      }
      for (p = row_ptr[w]; p < row_ptr[w + 1]; ++p)
        sum += exp(scale * half_to_double(vals[p * V + r]) - m);
      for (p = row_ptr[w]; p < row_ptr[w + 1]; ++p)
        out64[p * V + r] = exp(scale * half_to_double(vals[p * V + r]) - m) / sum;
    }
  }
}

/* Threads of the OpenMP team (the CPU baseline uses every core of the host even when a
   launcher exported OMP_NUM_THREADS=1); n <= 0 leaves it unchanged.  Returns the team size. */
int oracle_set_num_threads(int n) {
#ifdef _OPENMP
  extern void omp_set_num_threads(int);
  extern int omp_get_max_threads(void);
  if (n > 0) omp_set_num_threads(n);
  return omp_get_max_threads();
#else
  (void)n;
  return 1;
#endif
}

int oracle_num_threads(void) {
#ifdef _OPENMP
  extern int omp_get_max_threads(void);
  return omp_get_max_threads();
#else
  return 1;
#endif
}

/*
 * CPU-baseline timing: one layer step of the bench -- encode W, C = W X
 * (SpMM), dW = (G X^T) o pattern(W) (SDDMM, inner dimension N) -- run `reps` times with
 * `threads` OpenMP threads (0 = the default team), each rep timed with the monotonic clock
 * (clock_gettime(CLOCK_MONOTONIC), the C counterpart of steady_clock).  Writes the seconds of
 * each rep to secs[reps]; returns nnz_v (or -1 if a buffer cannot be allocated).  The timed
 * work is exactly the functions above: nothing is tuned for the benchmark.
 */
static double mono_seconds(void) {
  struct timespec ts;
  clock_gettime(CLOCK_MONOTONIC, &ts);
  return (double)ts.tv_sec + 1e-9 * (double)ts.tv_nsec;
}

int64_t oracle_time_layer(int64_t M, int64_t K, int64_t N, int V, const uint16_t* dense,
                          const uint16_t* X, const uint16_t* G, int threads, int reps,
                          double* secs) {
#ifdef _OPENMP
  extern void omp_set_num_threads(int);
  extern int omp_get_max_threads(void);
  int saved = omp_get_max_threads();
  if (threads > 0) omp_set_num_threads(threads);
#endif
  int64_t W = ceil_div(M, V), nnz = 0, r;
  int32_t* row_ptr = (int32_t*)malloc(sizeof(int32_t) * (size_t)(W + 1));
  double* C = (double*)malloc(sizeof(double) * (size_t)(M * N));
  double* S = (double*)malloc(sizeof(double) * (size_t)(M * N));
  int32_t* col_idx = NULL;
  uint16_t* vals = NULL;
  double *o = NULL, *so = NULL;
  for (r = 0; r < reps; ++r) {
    double t0 = mono_seconds();
    nnz = oracle_encode(M, K, V, dense, NULL, row_ptr, NULL, NULL);
    if (r == 0) {
      col_idx = (int32_t*)malloc(sizeof(int32_t) * (size_t)(nnz + 1));
      vals = (uint16_t*)malloc(sizeof(uint16_t) * (size_t)(nnz * V + 1));
      o = (double*)malloc(sizeof(double) * (size_t)(nnz * V + 1));
      so = (double*)malloc(sizeof(double) * (size_t)(nnz * V + 1));
    }
    if (!row_ptr || !C || !S || !col_idx || !vals || !o || !so) { nnz = -1; break; }
    oracle_encode(M, K, V, dense, NULL, row_ptr, col_idx, vals);
    oracle_spmm(M, K, N, V, row_ptr, col_idx, vals, X, C, S);
    oracle_sddmm(M, K, N, V, row_ptr, col_idx, G, X, o, so);
    secs[r] = mono_seconds() - t0;
  }
  free(row_ptr); free(C); free(S); free(col_idx); free(vals); free(o); free(so);
#ifdef _OPENMP
  omp_set_num_threads(saved);
#endif
  return nnz;
}
