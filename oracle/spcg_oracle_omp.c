/*
 * spcg_oracle_omp.c — the oracle's ITERATIVE PHASE (Algorithm 1, O9/O10) on all
 * host cores with OpenMP: the multicore CPU baseline of BASELINE.md §3 / SURVEY
 * §8(d) ("an OpenMP build of the oracle's solve phase: level-scheduled SpTRSV with
 * a barrier per level, plus parallel SpMV, dots and axpys").
 *
 * TEST / BENCH INFRASTRUCTURE ONLY (bench.py's cpu_baseline leg).  Not a parity
 * reference: OpenMP reductions sum in a thread-dependent order, so its values
 * differ from spcg_oracle.c by rounding; iteration counts agree to +-1.  The
 * product never links or calls it.  Paper: Algorithm 1; the
 * preconditioner application z = U^-1 L^-1 r by forward and backward substitution
 * over the level sets of Fig. 1.  It is the analogue of
 * the paper's CPU solve-phase run (AMD EPYC).
 *
 * Level sets (level_ptr / level_rows, rows ascending inside a level) come from the
 * oracle's or_levels_lower / or_levels_upper / or_level_sets (setup, not timed).
 * One parallel region spans the whole solve; every level is an `omp for` with its
 * implicit barrier.  Timed with omp_get_wtime from the prologue to loop exit (A19).
 */
#include <math.h>
#include <omp.h>
#include <stdint.h>
#include <stdlib.h>

typedef struct {
    int64_t n, nnz;
    int64_t* rowptr;
    int32_t* col;
    double* val;
} or_csr;

enum { OMP_OK = 0, OMP_NOT_CONVERGED = 1, OMP_BREAKDOWN = -4 };

int or_omp_threads(void) { return omp_get_max_threads(); }

/* Returns status; *k_out iterations, *rnorm_out ||r_k||, *seconds the iterative phase. */
int or_pcg_omp(const or_csr* A, const or_csr* L, const or_csr* U, const int64_t* lpL, const int32_t* lrL, int64_t wL,
               const int64_t* lpU, const int32_t* lrU, int64_t wU, const double* b, double eps, int64_t kmax,
               int threads, double* x, int64_t* k_out, double* rnorm_out, double* seconds) {
    const int64_t n = A->n;
    double* r = (double*)malloc(sizeof(double) * (size_t)(n ? n : 1));
    double* z = (double*)malloc(sizeof(double) * (size_t)(n ? n : 1));
    double* p = (double*)malloc(sizeof(double) * (size_t)(n ? n : 1));
    double* w = (double*)malloc(sizeof(double) * (size_t)(n ? n : 1));
    double* y = (double*)malloc(sizeof(double) * (size_t)(n ? n : 1));
    if (threads > 0) omp_set_num_threads(threads);
    double s_pw = 0.0, s_rz = 0.0, s_rr = 0.0;
    int status = OMP_NOT_CONVERGED;
    int64_t k_final = 0;
    double rn_final = 0.0;
    const double t0 = omp_get_wtime();
#pragma omp parallel
    {
        double rho = 0.0, rr = 0.0;
        int64_t k;
        /* ---- prologue: x0 = 0, r0 = b, z0 = M^-1 r0, p0 = z0 */
#pragma omp for schedule(static)
        for (int64_t i = 0; i < n; ++i) { x[i] = 0.0; r[i] = b[i]; }
        for (int64_t l = 0; l < wL; ++l) {
#pragma omp for schedule(static)
            for (int64_t t = lpL[l]; t < lpL[l + 1]; ++t) {
                const int32_t i = lrL[t];
                double acc = r[i];
                for (int64_t q = L->rowptr[i]; q < L->rowptr[i + 1]; ++q) acc -= L->val[q] * y[L->col[q]];
                y[i] = acc;
            }
        }
        for (int64_t l = 0; l < wU; ++l) {
#pragma omp for schedule(static)
            for (int64_t t = lpU[l]; t < lpU[l + 1]; ++t) {
                const int32_t i = lrU[t];
                const int64_t q0 = U->rowptr[i];
                double acc = y[i];
                for (int64_t q = q0 + 1; q < U->rowptr[i + 1]; ++q) acc -= U->val[q] * z[U->col[q]];
                z[i] = acc / U->val[q0];
            }
        }
#pragma omp single
        { s_rz = 0.0; s_rr = 0.0; }
#pragma omp for schedule(static) reduction(+ : s_rz, s_rr)
        for (int64_t i = 0; i < n; ++i) {
            p[i] = z[i];
            s_rz += r[i] * z[i];
            s_rr += r[i] * r[i];
        }
        rho = s_rz;
        rr = s_rr;
        for (k = 0;; ++k) {
            const double rn = sqrt(rr);
            if (rn < eps || rr == 0.0) {
#pragma omp single
                { status = OMP_OK; k_final = k; rn_final = rn; }
                break;
            }
            if (k == kmax) {
#pragma omp single
                { status = eps > 0.0 ? OMP_NOT_CONVERGED : OMP_OK; k_final = k; rn_final = rn; }
                break;
            }
#pragma omp single
            s_pw = 0.0;
#pragma omp for schedule(static) reduction(+ : s_pw)
            for (int64_t i = 0; i < n; ++i) {
                double acc = 0.0;
                for (int64_t q = A->rowptr[i]; q < A->rowptr[i + 1]; ++q) acc += A->val[q] * p[A->col[q]];
                w[i] = acc;
                s_pw += p[i] * acc;
            }
            const double pw = s_pw;
            if (!(pw > 0.0) || !isfinite(pw) || !isfinite(rho)) {
#pragma omp single
                { status = OMP_BREAKDOWN; k_final = k; rn_final = rn; }
                break;
            }
            const double alpha = rho / pw;
#pragma omp for schedule(static)
            for (int64_t i = 0; i < n; ++i) {
                x[i] += alpha * p[i];
                r[i] -= alpha * w[i];
            }
            for (int64_t l = 0; l < wL; ++l) {
#pragma omp for schedule(static)
                for (int64_t t = lpL[l]; t < lpL[l + 1]; ++t) {
                    const int32_t i = lrL[t];
                    double acc = r[i];
                    for (int64_t q = L->rowptr[i]; q < L->rowptr[i + 1]; ++q) acc -= L->val[q] * y[L->col[q]];
                    y[i] = acc;
                }
            }
            for (int64_t l = 0; l < wU; ++l) {
#pragma omp for schedule(static)
                for (int64_t t = lpU[l]; t < lpU[l + 1]; ++t) {
                    const int32_t i = lrU[t];
                    const int64_t q0 = U->rowptr[i];
                    double acc = y[i];
                    for (int64_t q = q0 + 1; q < U->rowptr[i + 1]; ++q) acc -= U->val[q] * z[U->col[q]];
                    z[i] = acc / U->val[q0];
                }
            }
#pragma omp single
            { s_rz = 0.0; s_rr = 0.0; }
#pragma omp for schedule(static) reduction(+ : s_rz, s_rr)
            for (int64_t i = 0; i < n; ++i) {
                s_rz += r[i] * z[i];
                s_rr += r[i] * r[i];
            }
            const double rho_new = s_rz;
            rr = s_rr;
            const double beta = rho_new / rho;
            rho = rho_new;
#pragma omp for schedule(static)
            for (int64_t i = 0; i < n; ++i) p[i] = z[i] + beta * p[i];
        }
    }
    *seconds = omp_get_wtime() - t0;
    *k_out = k_final;
    *rnorm_out = rn_final;
    free(r); free(z); free(p); free(w); free(y);
    return status;
}
