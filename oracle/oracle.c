/*
 * oracle.c -- plain, slow, obviously-correct CPU definitions of what the
 * libctaclust hot path computes.  fp64 accumulation throughout.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or constant with the CUDA path
 * (paper_conf_asplos_lis0l0c17_b200/csrc); neither side includes the other.
 *
 * Why these definitions are the oracle: CTA clustering is a schedule
 * transformation.  The paper's "orderless" property (§2
 * "Execution Model": "a kernel should always obtain correct result in
 * arbitrary dispatching/execution order of CTAs") means every clustered
 * execution must reach exactly the result of the unclustered kernel, which
 * in turn is the plain mathematical definition written out below.  So each
 * function is that definition, evaluated directly, with no tiling, blocking
 * or reordering.
 *
 * OpenMP: built plainly (gcc -O2, liboracle.so) the `#pragma omp` lines are
 * ignored and every loop runs serially.  The same file built with -fopenmp
 * (liboracle_omp.so) is only used to time the oracle on all host cores
 * (bench.py cpu_baseline); the pragmas split independent outputs across
 * threads (rows, or the columns of a transposed product inside each row
 * step), so every output keeps its summation order and value.
 *
 * Parity status (see DESIGN.md §Oracle pins): every function here is pinned
 * by tests/test_oracle_kernels.py against closed forms, special cases and
 * independent library routines (numpy / scipy).
 */
#include <stddef.h>
#include <stdint.h>

/* ------------------------------------------------------------------------
 * a7.1  Matrix-vector multiply  C[i] += sum_j A[i][j] * B[j]
 * PAPER.md Listing 1 ("Loop1: Matrix-Vector-Multiply") and
 * Listing 2 (the MVM kernel).  Row-major A with leading dim lda.
 * y_out[i] = sum_{j<n} A[i*lda+j] * x[j]   (y starts at 0)
 * ---------------------------------------------------------------------- */
void oracle_matvec(int64_t m, int64_t n, const float* A, int64_t lda,
                   const float* x, double* y_out)
{
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < m; ++i) {
        double acc = 0.0;
        for (int64_t j = 0; j < n; ++j)
            acc += (double)A[i * lda + j] * (double)x[j];
        y_out[i] = acc;
    }
}

/* Transposed product  y[j] = sum_i A[i][j] * x[i]  (j < n, i < m). */
static void matvec_t(int64_t m, int64_t n, const float* A, int64_t lda,
                     const double* x, double* y_out)
{
    for (int64_t j = 0; j < n; ++j) y_out[j] = 0.0;
    #pragma omp parallel
    for (int64_t i = 0; i < m; ++i) {
        #pragma omp for schedule(static)
        for (int64_t j = 0; j < n; ++j)
            y_out[j] += (double)A[i * lda + j] * x[i];
    }
}

/* ------------------------------------------------------------------------
 * a7.2  PolyBench/GPU kernels named in PAPER.md Table 2:
 *   atax "Matrix transpose and vector multiply", mvt "Matrix vector product
 *   and transpose", bicg "BiCGStab linear solver" sub-kernel.  The paper only
 *   names them; the definitions are the PolyBench ones (reading R13).
 * ---------------------------------------------------------------------- */

/* ATAX: tmp = A x ; y = A^T tmp.  A is m x n. tmp_out has m, y_out has n. */
void oracle_atax(int64_t m, int64_t n, const float* A, int64_t lda,
                 const float* x, double* tmp_out, double* y_out)
{
    oracle_matvec(m, n, A, lda, x, tmp_out);
    matvec_t(m, n, A, lda, tmp_out, y_out);
}

/* ATAX second pass given an fp32 tmp (what the GPU stores between passes):
 * y = A^T tmp.  Lets tests separate pass-1 and pass-2 error. */
void oracle_atax_pass2(int64_t m, int64_t n, const float* A, int64_t lda,
                       const float* tmp, double* y_out)
{
    for (int64_t j = 0; j < n; ++j) y_out[j] = 0.0;
    #pragma omp parallel
    for (int64_t i = 0; i < m; ++i) {
        #pragma omp for schedule(static)
        for (int64_t j = 0; j < n; ++j)
            y_out[j] += (double)A[i * lda + j] * (double)tmp[i];
    }
}

/* BICG: q = A p ; s = A^T r.  A is m x n; p has n, r has m; q has m, s has n. */
void oracle_bicg(int64_t m, int64_t n, const float* A, int64_t lda,
                 const float* p, const float* r, double* q_out, double* s_out)
{
    oracle_matvec(m, n, A, lda, p, q_out);
    for (int64_t j = 0; j < n; ++j) s_out[j] = 0.0;
    #pragma omp parallel
    for (int64_t i = 0; i < m; ++i) {
        #pragma omp for schedule(static)
        for (int64_t j = 0; j < n; ++j)
            s_out[j] += (double)A[i * lda + j] * (double)r[i];
    }
}

/* MVT: x1 += A y1 ; x2 += A^T y2.  A is n x n (PolyBench), here m x n:
 * x1, y2 have m entries; y1, x2 have n entries. */
void oracle_mvt(int64_t m, int64_t n, const float* A, int64_t lda,
                const float* x1_in, const float* x2_in,
                const float* y1, const float* y2,
                double* x1_out, double* x2_out)
{
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < m; ++i) {
        double acc = (double)x1_in[i];
        for (int64_t j = 0; j < n; ++j)
            acc += (double)A[i * lda + j] * (double)y1[j];
        x1_out[i] = acc;
    }
    for (int64_t j = 0; j < n; ++j) x2_out[j] = (double)x2_in[j];
    #pragma omp parallel
    for (int64_t i = 0; i < m; ++i) {
        #pragma omp for schedule(static)
        for (int64_t j = 0; j < n; ++j)
            x2_out[j] += (double)A[i * lda + j] * (double)y2[i];
    }
}

/* ------------------------------------------------------------------------
 * a7.3  2D 5-point Jacobi (PolyBench jacobi-2d form; reading R14):
 *   B[i][j] = 0.2 * (A[i][j] + A[i][j-1] + A[i][j+1] + A[i-1][j] + A[i+1][j])
 * on the interior 1 <= i < rows-1, 1 <= j < cols-1; boundary cells keep their
 * initial values (Dirichlet).  One iteration = one sweep A->B then swap.
 * out receives the field written by the last sweep (iters >= 1), or the
 * input when iters == 0.  work must hold 2*rows*cols doubles.
 * ---------------------------------------------------------------------- */
void oracle_jacobi5(int64_t rows, int64_t cols, const float* u0, int iters,
                    double* out, double* work)
{
    double* a = work;
    double* b = work + rows * cols;
    for (int64_t k = 0; k < rows * cols; ++k) { a[k] = (double)u0[k]; b[k] = a[k]; }
    for (int t = 0; t < iters; ++t) {
        #pragma omp parallel for schedule(static)
        for (int64_t i = 1; i < rows - 1; ++i)
            for (int64_t j = 1; j + 1 < cols; ++j)
                b[i * cols + j] = 0.2 * (a[i * cols + j] + a[i * cols + j - 1] + a[i * cols + j + 1]
                                         + a[(i - 1) * cols + j] + a[(i + 1) * cols + j]);
        double* s = a; a = b; b = s;
    }
    for (int64_t k = 0; k < rows * cols; ++k) out[k] = a[k];
}

/* fp32 variant: the PolyBench jacobi-2d statement (reading R14) evaluated in
 * fp32 exactly as C evaluates it, left to right with no contraction:
 *     B[i][j] = 0.2f * (A[i][j] + A[i][j-1] + A[i][1+j] + A[1+i][j] + A[i-1][j])
 * i.e. centre, west, east, south (row i+1), north (row i-1).  This is the
 * sum order the GPU sweep reproduces bit for bit; pinned by the fp64 oracle
 * and by an order-sensitive by-hand case (tests/test_oracle_kernels.py). */
void oracle_jacobi5_f32(int64_t rows, int64_t cols, const float* u0, int iters,
                        float* out, float* work)
{
    float* a = work;
    float* b = work + rows * cols;
    for (int64_t k = 0; k < rows * cols; ++k) { a[k] = u0[k]; b[k] = u0[k]; }
    for (int t = 0; t < iters; ++t) {
        for (int64_t i = 1; i + 1 < rows; ++i)
            for (int64_t j = 1; j + 1 < cols; ++j) {
                float c = a[i * cols + j], w = a[i * cols + j - 1], e = a[i * cols + j + 1];
                float s = a[(i + 1) * cols + j], n = a[(i - 1) * cols + j];
                b[i * cols + j] = 0.2f * ((((c + w) + e) + s) + n);
            }
        float* sw = a; a = b; b = sw;
    }
    for (int64_t k = 0; k < rows * cols; ++k) out[k] = a[k];
}

/* ------------------------------------------------------------------------
 * a7.4  2D convolution as cross-correlation (reading R15):
 *   out[i][j] = sum_{a,b in [-R,R]} w[(a+R)*(2R+1) + (b+R)] * in[i+a][j+b]
 * for interior i in [R, rows-R), j in [R, cols-R); other outputs are 0.
 * ---------------------------------------------------------------------- */
void oracle_conv2d(int64_t rows, int64_t cols, const float* in, int R,
                   const float* w, double* out)
{
    const int K = 2 * R + 1;
    for (int64_t k = 0; k < rows * cols; ++k) out[k] = 0.0;
    #pragma omp parallel for schedule(static)
    for (int64_t i = R; i < rows - R; ++i)
        for (int64_t j = R; j + R < cols; ++j) {
            double acc = 0.0;
            for (int a = -R; a <= R; ++a)
                for (int b = -R; b <= R; ++b)
                    acc += (double)w[(a + R) * K + (b + R)] * (double)in[(i + a) * cols + (j + b)];
            out[i * cols + j] = acc;
        }
}

/* ------------------------------------------------------------------------
 * a7.5  CSR sparse matrix-vector product (data-related locality class,
 * PAPER.md P:1757-1761):  y[i] = sum_{k in [rp[i], rp[i+1])} val[k]*x[col[k]]
 * ---------------------------------------------------------------------- */
void oracle_spmv_csr(int64_t rows, const int32_t* row_ptr, const int32_t* col,
                     const float* val, const float* x, double* y_out)
{
    #pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t i = 0; i < rows; ++i) {
        double acc = 0.0;
        for (int64_t k = row_ptr[i]; k < row_ptr[i + 1]; ++k)
            acc += (double)val[k] * (double)x[col[k]];
        y_out[i] = acc;
    }
}

/* ------------------------------------------------------------------------
 * S§8(f)3  64-bin histogram (HST): PAPER.md Table 2 ("histogram
 * 64-bin histogramming", category Data; the data-related class of P:1761,
 * source [40] = the CUDA SDK).  Reading R24: the SDK's histogram64 bins each
 * input byte by its top six bits, so
 *     counts[k] = #{ i < n : data[i] >> 2 == k },   k = 0..63.
 */
void oracle_hist64(int64_t n, const uint8_t* data, uint64_t* counts) {
    for (int k = 0; k < 64; ++k) counts[k] = 0;
    for (int64_t i = 0; i < n; ++i) counts[data[i] >> 2] += 1;
}
