/*
 * memxct_oracle.h -- plain, slow fp64 CPU oracle for the MemXCT hot path (single-threaded
 * arithmetic; the sampled-row helpers and the CPU-baseline SpMV spread independent rays / rows over
 * host threads without changing any operation).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  The product (paper_conf_sc_hidayetoglubgrg19_b200/,
 * include/memxct.h) shares no code, header, table or helper with it.
 *
 * Paper: M. Hidayetoglu et al., "MemXCT: Memory-Centric X-ray CT Reconstruction with Massive
 * Parallelization", SC'19.  Citations "P:n" are lines of the paper text.
 * Readings R1..R17 are listed in DESIGN.md section 3 (they follow SURVEY.md section 8(c)).
 *
 * Every function states which passage (or reading) it follows and which test pins it.
 */
#ifndef MEMXCT_ORACLE_H
#define MEMXCT_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- geometry + Siddon tracing (sec. 2.3, readings R1-R5) ------------------------- */

/* Trace ray `ray` (natural index m*C + k).  Writes up to `cap` (pixel natural index i*N+j,
 * fp64 length) pairs in trace order (ascending ray parameter).  Returns the number of entries,
 * or -1 if cap is too small.  Pinned by: closed-form chord, brute-force clipping, Table 3. */
int64_t orc_trace_ray(int32_t n, int32_t m_proj, int32_t c_chan, int64_t ray,
                      int32_t* pix, double* len, int64_t cap);

/* Number of nonzeros of A for the whole geometry (count only).  Pinned by Table 3. */
int64_t orc_count_nnz(int32_t n, int32_t m_proj, int32_t c_chan);

/* Row lengths of A (per natural ray).  row_len has m_proj*c_chan entries. */
void orc_row_lengths(int32_t n, int32_t m_proj, int32_t c_chan, int32_t* row_len);

/* Whole A as COO in ray-major trace order.  Arrays must hold orc_count_nnz entries.
 * Returns nnz written. */
int64_t orc_trace_all(int32_t n, int32_t m_proj, int32_t c_chan,
                      int32_t* rows, int32_t* cols, double* vals, int64_t cap);

/* ---- two-level pseudo-Hilbert ordering (sec. 3.2, readings R6-R9) ----------------- */

/* gilbert2d over a w x h grid: writes the visiting order as (x, y) pairs (x = column, y = row).
 * Returns w*h.  Pinned by Fig. 4(a) fragments and the textbook 2^k special case. */
int64_t orc_gilbert2d(int32_t w, int32_t h, int32_t* xs, int32_t* ys);

/* Textbook Hilbert d -> (x, y) on an n x n grid (n power of two), start (0,0), end (n-1,0). */
void orc_d2xy(int32_t n, int64_t d, int32_t* x, int32_t* y);

/* Two-level ordering of an H x W domain (rows x cols) with tile side T (power of two).
 * rank[i*W + j] = position of cell (row i, col j) along the curve.  Returns 0 on success. */
int orc_hilbert_rank(int32_t h, int32_t w, int32_t t, int64_t* rank);

/* ---- SpMV (Listing 2; semantics of Listing 3) ---------------------------- */

/* y = A x over COO (y zeroed first, entries accumulated in the given order). */
void orc_spmv_coo(int64_t nnz, const int32_t* rows, const int32_t* cols, const double* vals,
                  const double* x, int64_t nrows, double* y);

/* Canonical row sums (reading R16): for each output row, entries sorted by key[col] ascending,
 * acc = fma(val, x[col], acc) from acc = 0.  CSR input (row_ptr over nrows). */
void orc_spmv_canonical(int64_t nrows, const int64_t* row_ptr, const int32_t* cols,
                        const double* vals, const int64_t* col_key, const double* x, double* y);

/* ---- CGLS (sec. 3.5.2, readings R13-R16) ------------------------------------------ */

/* Plain CGLS on A (nrows x ncols, COO), x0 = 0, exactly `iters` iterations.
 * canonical = 0: plain sums (COO order), dots as sequential fp64 sums in natural order.
 * canonical = 1: row sums per orc_spmv_canonical with keys row_key/col_key (Hilbert ranks);
 *   dots as fma chains over chunks of `chunk_rows` (resp. `chunk_cols`) consecutive
 *   Hilbert-ordered elements, chunk partials added sequentially in chunk order.
 * Outputs x (ncols), res[k] = ||r_k|| (iters+1 entries, nullable), true_res[k] = ||y - A x_k||
 * (nullable).  Returns the number of iterations performed. */
int orc_cgls(int64_t nrows, int64_t ncols, int64_t nnz, const int32_t* rows, const int32_t* cols,
             const double* vals, const double* y, int32_t iters, int32_t canonical,
             const int64_t* row_key, const int64_t* col_key, int64_t chunk_rows, int64_t chunk_cols,
             double* x, double* res, double* true_res);

/* SIRT: x_0 = 0, x_{k+1} = x_k + C A^T R (y - A x_k), R = 1/row
 * sums, C = 1/column sums (0 for empty rows/columns).  res[k] = ||y - A x_k||, k = 0..iters
 * (nullable).  Pinned by the weighted least-squares fixed point and the closed-form x_1. */
int orc_sirt(int64_t nrows, int64_t ncols, int64_t nnz, const int32_t* rows, const int32_t* cols,
             const double* vals, const double* y, int32_t iters, double* x, double* res);

/* Canonical dot (reading R16): elements visited in ascending key order, fma chains over chunks
 * of `chunk` elements, chunk partials summed sequentially. */
double orc_dot_canonical(int64_t n, const double* a, const double* b, const int64_t* key,
                         int64_t chunk);


/* ---- closed-form chord and sampled rows / columns ------------------------- */

/* Closed-form length of ray `ray` inside the grid square [-L, L]^2 (C.4): with
 * c' = max(|cos|, |sin|), s' = min(...), tau = |t|: 2L/c' if tau <= L(c'-s'); (L(c'+s') - tau) /
 * (c' s') if tau < L(c'+s'); else 0 (s' < 1e-15: 2L if tau < L).  Equals the row sum of A.
 * Pinned by: Liang-Barsky clipping of the line against the square, and the tracer's row sums. */
double orc_chord(int32_t n, int32_t m_proj, int32_t c_chan, int64_t ray);
void orc_chords(int32_t n, int32_t m_proj, int32_t c_chan, double* out /* m_proj*c_chan */);

/* CSR result of the sampled functions (library-allocated; free with orc_csr_free). */
typedef struct { int64_t nrows, nnz; int64_t* ptr; int32_t* idx; double* len; } orc_csr_t;
orc_csr_t* orc_csr_alloc(int64_t nrows, int64_t nnz);
void orc_csr_free(orc_csr_t* s);

/* Rows of A for `nrays` natural ray indices: row i = (pixel, length) pairs of rays[i] in trace
 * order, exactly orc_trace_ray's.  Rays are spread over `nthreads` host threads (0 = all online
 * cores); no arithmetic changes.  Pinned by: equality with orc_trace_all's rows. */
orc_csr_t* orc_sample_rows(int32_t n, int32_t m_proj, int32_t c_chan, int64_t nrays,
                           const int64_t* rays, int32_t nthreads);

/* Columns of A (rows of A^T) for `npix` distinct natural pixel indices: row q = (ray, length)
 * pairs of every ray crossing pixels[q], rays ascending.  Per projection, candidate channels are
 * those whose line can meet the pixel square (|t_k - tc| <= (|cos| + |sin|)/2, +-1 channel), each
 * traced in full by the tracer.  NULL if pixels repeat.  Pinned by: equality with the columns of
 * the full transpose of orc_trace_all (tests/test_oracle_sampled.py). */
orc_csr_t* orc_sample_columns(int32_t n, int32_t m_proj, int32_t c_chan, int64_t npix,
                              const int64_t* pixels, int32_t nthreads);

/* Stable transpose of a CSR (nrows x ncols): output row c lists the input rows holding column c
 * in ascending input-row order.  Pinned by: equality with the sort-based coo_to_csr. */
orc_csr_t* orc_csr_transpose(int64_t nrows, const int64_t* ptr, const int32_t* idx, const double* len,
                             int64_t ncols);

/* y = A x over CSR with rows split over host threads (the threaded CPU
 * baseline).  Each row is summed sequentially in entry order, bit-identical to orc_spmv_coo on
 * row-major COO.  Returns the number of threads used. */
int32_t orc_spmv_csr_threaded(int64_t nrows, const int64_t* ptr, const int32_t* cols,
                              const double* vals, const double* x, double* y, int32_t nthreads);

#ifdef __cplusplus
}
#endif
#endif
