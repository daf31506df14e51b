/*
 * spcg_gen.c — seeded synthetic SPD workload generators (shared INPUT module).
 *
 * This module produces the test/benchmark inputs (matrix A in full symmetric
 * CSR, right-hand side b, manufactured solution x_true).  It holds none of the
 * SPCG method's arithmetic (no sparsification, no ILU, no triangular solve, no
 * PCG); both the oracle (oracle/) and the CUDA library consume its output.
 *
 * Workload recipe: SURVEY.md §8(d) "Workloads", restated in DESIGN.md §3.
 *   - RNG  u(seed,i) = (splitmix64(seed*0x9E3779B97F4A7C15 + i) >> 11) * 2^-53
 *   - natural x-fastest ordering, homogeneous Dirichlet (boundary nodes eliminated)
 *   - only + - * / and ldexp, so values are reproducible bit for bit.
 * The paper's own workloads are 107 SuiteSparse SPD matrices (PAPER.md L621-628,
 * §4.1); these families stand in for its 2D/3D PDE, thermal/structural FEM and
 * heterogeneous-diffusion classes (Fig. 9 labels).
 *
 * Families (param vector p):
 *   0 poisson2d  p = {nx, ny}            5-point,  a_ii = 4, neighbours -1
 *   1 poisson3d  p = {nx, ny, nz}        7-point,  a_ii = 6, neighbours -1
 *   2 fem_q1     p = {nx, ny, nz, seed}  27-point Q1 FEM of -div(k grad u) + sigma u
 *   3 aniso      p = {nx, ny, seed}      layered anisotropic 5-point diffusion
 *
 * Two-call API: gen_count() gives n and nnz, gen_fill() writes caller buffers.
 */
#include <stdint.h>
#include <math.h>
#include <string.h>

static inline uint64_t splitmix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

double gen_u(uint64_t seed, uint64_t i) {
    uint64_t s = seed * 0x9E3779B97F4A7C15ULL + i;
    return (double)(splitmix64(s) >> 11) * 0x1.0p-53;
}

/* ------------------------------------------------------------------ */
/* Q1 trilinear unit-cube element tables, by pair type                  */
/* type = number of axes on which the two corners differ (0..3)         */
static double q1_K(int type) {
    switch (type) {
        case 0: return 4.0 / 12.0;
        case 1: return 0.0;
        default: return -1.0 / 12.0;   /* face diagonal and body diagonal */
    }
}
static double q1_M(int type) {
    /* prod_d (2 if same coordinate else 1) / 216 */
    switch (type) {
        case 0: return 8.0 / 216.0;
        case 1: return 4.0 / 216.0;
        case 2: return 2.0 / 216.0;
        default: return 1.0 / 216.0;
    }
}

static void fem_elem_coef(uint64_t seed, int64_t e, double* k_e, double* s_e) {
    double u0 = gen_u(seed, (uint64_t)(3 * e));
    double u1 = gen_u(seed, (uint64_t)(3 * e + 1));
    double u2 = gen_u(seed, (uint64_t)(3 * e + 2));
    int ex = (int)floor(4.0 * u1) - 2;
    *k_e = ldexp(1.0 + u0, ex);
    *s_e = ldexp(1.0 + u2, -7);
}

/* value of A(P, P+d) for interior nodes P=(X,Y,Z) (1-based), d in {-1,0,1}^3:
 * sum over the shared elements in ascending element index of k_e*K + s_e*M. */
static double fem_entry(int64_t nx, int64_t ny, uint64_t seed,
                        int64_t X, int64_t Y, int64_t Z, int dx, int dy, int dz) {
    int64_t exs[2], eys[2], ezs[2];
    int nxs, nys, nzs;
    int type = (dx != 0) + (dy != 0) + (dz != 0);
    if (dx == 0) { exs[0] = X - 1; exs[1] = X; nxs = 2; } else { exs[0] = dx > 0 ? X : X - 1; nxs = 1; }
    if (dy == 0) { eys[0] = Y - 1; eys[1] = Y; nys = 2; } else { eys[0] = dy > 0 ? Y : Y - 1; nys = 1; }
    if (dz == 0) { ezs[0] = Z - 1; ezs[1] = Z; nzs = 2; } else { ezs[0] = dz > 0 ? Z : Z - 1; nzs = 1; }
    double Kt = q1_K(type), Mt = q1_M(type);
    double acc = 0.0;
    for (int c = 0; c < nzs; ++c)
        for (int b = 0; b < nys; ++b)
            for (int a = 0; a < nxs; ++a) {
                int64_t e = exs[a] + (nx + 1) * (eys[b] + (ny + 1) * ezs[c]);
                double ke, se;
                fem_elem_coef(seed, e, &ke, &se);
                double contrib = ke * Kt + se * Mt;
                acc = acc + contrib;
            }
    return acc;
}

/* ------------------------------------------------------------------ */
/* layered anisotropic diffusion                                        */
static double aniso_c(uint64_t seed, int64_t nx, int64_t i) {
    int64_t x = i % nx;
    double base = (x % 16 == 15) ? 0x1.0p-10 : 1.0;
    return base * (1.0 + 0.25 * gen_u(seed, (uint64_t)i));
}
static double harm(double ca, double cb) { return (2.0 * ca * cb) / (ca + cb); }
#define ANISO_EPS 0x1.0p-7

/* ------------------------------------------------------------------ */
/* generic row emitter                                                  */
typedef struct {
    int64_t n, nnz;
    int64_t* rowptr; int32_t* col; double* val;  /* NULL during count */
} sink_t;

static inline void emit(sink_t* s, int64_t j, double v) {
    if (s->col) { s->col[s->nnz] = (int32_t)j; s->val[s->nnz] = v; }
    s->nnz++;
}
static inline void end_row(sink_t* s, int64_t i) {
    if (s->rowptr) s->rowptr[i + 1] = s->nnz;
}

static int run(int family, const int64_t* p, sink_t* s) {
    s->nnz = 0;
    if (s->rowptr) s->rowptr[0] = 0;
    if (family == 0) {
        int64_t nx = p[0], ny = p[1];
        s->n = nx * ny;
        for (int64_t y = 0; y < ny; ++y)
            for (int64_t x = 0; x < nx; ++x) {
                int64_t i = x + nx * y;
                if (y > 0) emit(s, i - nx, -1.0);
                if (x > 0) emit(s, i - 1, -1.0);
                emit(s, i, 4.0);
                if (x < nx - 1) emit(s, i + 1, -1.0);
                if (y < ny - 1) emit(s, i + nx, -1.0);
                end_row(s, i);
            }
        return 0;
    }
    if (family == 1) {
        int64_t nx = p[0], ny = p[1], nz = p[2], pl = nx * ny;
        s->n = nx * ny * nz;
        for (int64_t z = 0; z < nz; ++z)
            for (int64_t y = 0; y < ny; ++y)
                for (int64_t x = 0; x < nx; ++x) {
                    int64_t i = x + nx * y + pl * z;
                    if (z > 0) emit(s, i - pl, -1.0);
                    if (y > 0) emit(s, i - nx, -1.0);
                    if (x > 0) emit(s, i - 1, -1.0);
                    emit(s, i, 6.0);
                    if (x < nx - 1) emit(s, i + 1, -1.0);
                    if (y < ny - 1) emit(s, i + nx, -1.0);
                    if (z < nz - 1) emit(s, i + pl, -1.0);
                    end_row(s, i);
                }
        return 0;
    }
    if (family == 2) {
        int64_t nx = p[0], ny = p[1], nz = p[2];
        uint64_t seed = (uint64_t)p[3];
        s->n = nx * ny * nz;
        for (int64_t Z = 1; Z <= nz; ++Z)
            for (int64_t Y = 1; Y <= ny; ++Y)
                for (int64_t X = 1; X <= nx; ++X) {
                    int64_t i = (X - 1) + nx * ((Y - 1) + ny * (Z - 1));
                    /* neighbours in ascending column order: dz, dy, dx each -1..1 */
                    for (int dz = -1; dz <= 1; ++dz)
                        for (int dy = -1; dy <= 1; ++dy)
                            for (int dx = -1; dx <= 1; ++dx) {
                                int64_t Xq = X + dx, Yq = Y + dy, Zq = Z + dz;
                                if (Xq < 1 || Xq > nx || Yq < 1 || Yq > ny || Zq < 1 || Zq > nz) continue;
                                int64_t j = (Xq - 1) + nx * ((Yq - 1) + ny * (Zq - 1));
                                double v = 0.0;
                                if (s->col) {
                                    /* assemble from the lower endpoint's view, then mirror */
                                    if (j <= i) v = fem_entry(nx, ny, seed, X, Y, Z, dx, dy, dz);
                                    else        v = fem_entry(nx, ny, seed, Xq, Yq, Zq, -dx, -dy, -dz);
                                }
                                emit(s, j, v);
                            }
                    end_row(s, i);
                }
        return 0;
    }
    if (family == 3) {
        int64_t nx = p[0], ny = p[1];
        uint64_t seed = (uint64_t)p[2];
        s->n = nx * ny;
        for (int64_t y = 0; y < ny; ++y)
            for (int64_t x = 0; x < nx; ++x) {
                int64_t i = x + nx * y;
                if (!s->col) {
                    if (y > 0) emit(s, i - nx, 0);
                    if (x > 0) emit(s, i - 1, 0);
                    emit(s, i, 0);
                    if (x < nx - 1) emit(s, i + 1, 0);
                    if (y < ny - 1) emit(s, i + nx, 0);
                    end_row(s, i);
                    continue;
                }
                double c = aniso_c(seed, nx, i);
                double fS = (y > 0)      ? harm(c, aniso_c(seed, nx, i - nx)) : c;
                double fW = (x > 0)      ? ANISO_EPS * harm(c, aniso_c(seed, nx, i - 1)) : ANISO_EPS * c;
                double fE = (x < nx - 1) ? ANISO_EPS * harm(c, aniso_c(seed, nx, i + 1)) : ANISO_EPS * c;
                double fN = (y < ny - 1) ? harm(c, aniso_c(seed, nx, i + nx)) : c;
                double d = ((fS + fW) + fE) + fN;
                if (y > 0) emit(s, i - nx, -fS);
                if (x > 0) emit(s, i - 1, -fW);
                emit(s, i, d);
                if (x < nx - 1) emit(s, i + 1, -fE);
                if (y < ny - 1) emit(s, i + nx, -fN);
                end_row(s, i);
            }
        return 0;
    }
    return -1;
}

int gen_count(int family, const int64_t* p, int64_t* n, int64_t* nnz) {
    sink_t s; memset(&s, 0, sizeof s);
    int rc = run(family, p, &s);
    *n = s.n; *nnz = s.nnz;
    return rc;
}

int gen_fill(int family, const int64_t* p, int64_t* rowptr, int32_t* col, double* val) {
    sink_t s; memset(&s, 0, sizeof s);
    s.rowptr = rowptr; s.col = col; s.val = val;
    return run(family, p, &s);
}

/* Right-hand side: x_true_i = 2u(seed,i) - 1, b = A x_true, then both scaled by
 * 1/||b||_2 so that ||b||_2 = 1 (absolute eps == relative eps). */
void gen_rhs(int64_t n, const int64_t* rowptr, const int32_t* col, const double* val,
             uint64_t seed, double* b, double* x_true) {
    for (int64_t i = 0; i < n; ++i) x_true[i] = 2.0 * gen_u(seed, (uint64_t)i) - 1.0;
    double ss = 0.0;
    for (int64_t i = 0; i < n; ++i) {
        double acc = 0.0;
        for (int64_t q = rowptr[i]; q < rowptr[i + 1]; ++q) acc += val[q] * x_true[col[q]];
        b[i] = acc;
        ss += acc * acc;
    }
    double inv = 1.0 / sqrt(ss);
    for (int64_t i = 0; i < n; ++i) { b[i] *= inv; x_true[i] *= inv; }
}
