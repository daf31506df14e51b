// api.cpp — the extern "C" entry points declared in include/spcg.h.
#include <algorithm>
#include <cmath>
#include <cstring>
#include <new>

#include "internal.h"

#ifdef _OPENMP
#include <omp.h>
#endif

namespace spcg {
const char* last_error_cstr();
}

using namespace spcg;

struct spcg_handle_s {
    int64_t n = 0;
    int K = 0;
    bool identity = false;
    Csr A;                      // deep copy of the input (device copy lives in dev)
    SparsifyResult sp;
    Factors F;
    Layouts lay;
    spcg_setup_info_t info{};
    spcg_device_t* dev = nullptr;
    int device = -1;
    std::vector<double> rhist;
};

template <class T, class Al>
static spcg_status_t put(const std::vector<T, Al>& v, void* buf, size_t* bytes) {
    size_t need = v.size() * sizeof(T);
    if (!buf) { *bytes = need; return SPCG_OK; }
    if (*bytes < need) { set_error("export buffer too small"); return SPCG_ERR_INVALID_ARG; }
    if (need) std::memcpy(buf, v.data(), need);
    *bytes = need;
    return SPCG_OK;
}

static void level_sets(const std::vector<int32_t>& lev, int64_t w, std::vector<int64_t>& ptr, std::vector<int32_t>& rows) {
    ptr.assign(w + 1, 0);
    for (int32_t l : lev) ptr[l + 1]++;
    for (int64_t l = 0; l < w; ++l) ptr[l + 1] += ptr[l];
    rows.assign(lev.size(), 0);
    std::vector<int64_t> nx(ptr.begin(), ptr.end() - 1);
    for (size_t i = 0; i < lev.size(); ++i) rows[nx[lev[i]]++] = (int32_t)i;
}

extern "C" {

int32_t spcg_abi_version(void) { return SPCG_ABI_VERSION; }

const char* spcg_status_string(spcg_status_t s) {
    switch (s) {
        case SPCG_OK: return "ok";
        case SPCG_NOT_CONVERGED: return "not converged (x holds x_kmax)";
        case SPCG_ERR_INVALID_ARG: return "invalid argument";
        case SPCG_ERR_BAD_MATRIX: return "bad matrix (not square/sorted/symmetric/positive-diagonal/finite)";
        case SPCG_ERR_ZERO_PIVOT: return "zero or non-finite pivot in ILU";
        case SPCG_ERR_BREAKDOWN: return "PCG breakdown ((p,w) <= 0 or non-finite scalar)";
        case SPCG_ERR_OOM: return "out of memory";
        case SPCG_ERR_CUDA: return "CUDA error";
        case SPCG_ERR_INTERNAL: return "internal error";
        case SPCG_ERR_NO_DEVICE: return "handle has no device (host-only setup)";
        default: return "unknown status";
    }
}

const char* spcg_last_error(void) { return last_error_cstr(); }

void spcg_drop_params_default(spcg_drop_params_t* p) {
    if (!p) return;
    std::memset(p, 0, sizeof *p);
    p->mode = SPCG_DROP_WAVEFRONT_AWARE;
    p->n_ratios = 3;
    p->ratios_pct[0] = 10.0; p->ratios_pct[1] = 5.0; p->ratios_pct[2] = 1.0;
    p->tau = 1.0;
    p->omega_pct = 10.0;
    p->norm_reading = SPCG_NORM_FRO;
    p->reduction_denominator = SPCG_DENOM_WA;
}

void spcg_options_default(spcg_options_t* o) {
    if (!o) return;
    std::memset(o, 0, sizeof *o);
    o->device = 0;
    o->stream = nullptr;
    o->sptrsv = SPCG_SPTRSV_AUTO;
    o->parts = 0;
    o->host_threads = 0;
    o->exec = SPCG_EXEC_AUTO;
    o->dev_alloc = nullptr;
    o->dev_free = nullptr;
    o->alloc_ctx = nullptr;
    o->wide_min = 0.0;
    o->chunk_partition = -1;
}

int spcg_dev_sm_count(int device);   // kernels.cu

spcg_status_t spcg_setup(const spcg_csr_t* Ain, const spcg_drop_params_t* drop_in, int32_t K,
                         const spcg_options_t* opt_in, spcg_handle_t* out) {
    if (!out) { set_error("out is NULL"); return SPCG_ERR_INVALID_ARG; }
    *out = nullptr;
    if (!Ain || !Ain->row_ptr || (Ain->nnz > 0 && (!Ain->col_idx || !Ain->val))) {
        set_error("A or its arrays are NULL");
        return SPCG_ERR_INVALID_ARG;
    }
    if (K < -1) { set_error("K must be >= -1"); return SPCG_ERR_INVALID_ARG; }
    spcg_drop_params_t drop;
    if (drop_in) drop = *drop_in; else spcg_drop_params_default(&drop);
    if (drop.mode < 0 || drop.mode > 2) { set_error("bad drop mode"); return SPCG_ERR_INVALID_ARG; }
    if (drop.norm_reading < 0 || drop.norm_reading > SPCG_NORM_SPECTRAL) {
        set_error("bad norm_reading");
        return SPCG_ERR_INVALID_ARG;
    }
    spcg_options_t opt;
    if (opt_in) opt = *opt_in; else spcg_options_default(&opt);
    if (opt.exec == SPCG_EXEC_GRAPH_WHILE) {
        set_error("exec GRAPH_WHILE is not built: the iterative phase runs as one persistent kernel");
        return SPCG_ERR_INVALID_ARG;
    }
    if (opt.exec < 0 || opt.exec > SPCG_EXEC_GRAPH_WHILE) { set_error("bad exec"); return SPCG_ERR_INVALID_ARG; }
    if ((opt.dev_alloc == nullptr) != (opt.dev_free == nullptr)) {
        set_error("dev_alloc and dev_free must be given together");
        return SPCG_ERR_INVALID_ARG;
    }
#ifdef _OPENMP
    if (opt.host_threads > 0) omp_set_num_threads(opt.host_threads);
#endif
    spcg_handle_s* h = new (std::nothrow) spcg_handle_s();
    if (!h) return SPCG_ERR_OOM;
    try {
        double t0 = now_ms();
        h->n = Ain->n;
        h->K = K;
        h->identity = (K < 0);
        h->device = opt.device;
        if (Ain->n <= 0) { delete h; set_error("n must be >= 1"); return SPCG_ERR_INVALID_ARG; }
        if (Ain->row_ptr[Ain->n] != Ain->nnz) { delete h; set_error("row_ptr[n] != nnz"); return SPCG_ERR_BAD_MATRIX; }
        h->A.n = Ain->n;
        h->A.rp.assign(Ain->row_ptr, Ain->row_ptr + Ain->n + 1);
        h->A.col.assign(Ain->col_idx, Ain->col_idx + Ain->nnz);
        h->A.val.assign(Ain->val, Ain->val + Ain->nnz);
        if (opt.setup_device < 0 || opt.setup_device > SPCG_SETUP_GPU) {
            delete h;
            set_error("bad setup_device");
            return SPCG_ERR_INVALID_ARG;
        }
        // the GPU setup covers ILU(0) with the FRO / INF readings; SPECTRAL runs on the host
        const bool on_gpu = opt.setup_device == SPCG_SETUP_GPU && K == 0 && opt.device >= 0 &&
                            (drop.mode != SPCG_DROP_WAVEFRONT_AWARE || drop.norm_reading != SPCG_NORM_SPECTRAL);
        double t1, t2, t3, t4;
        spcg_status_t st;
        if (on_gpu) {
            // NEXT-1: validation, Algorithm 2, ILU(0) and the level sets on the GPU
            DevAllocator alc;
            alc.alloc = opt.dev_alloc;
            alc.free = opt.dev_free;
            alc.ctx = opt.alloc_ctx;
            double ph[5] = {0, 0, 0, 0, 0};
            st = gpu_setup_k0(h->A, drop, opt.device, opt.stream, alc, h->sp, h->F, ph);
            h->info.zero_pivot_row = h->F.zero_pivot_row;
            if (st != SPCG_OK) { delete h; return st; }
            t1 = t0 + ph[0];
            t2 = t1 + ph[1];
            t3 = t2 + ph[2];
            t4 = now_ms();               // ILU(0), factor levels, download of Ahat / L / U
        } else {
            std::vector<int64_t> pos_t;
            st = validate_and_mirror(h->A, pos_t);
            if (st != SPCG_OK) { delete h; return st; }
            t1 = now_ms();
            st = sparsify_select(h->A, pos_t, drop, h->sp);
            if (st != SPCG_OK) { delete h; return st; }
            t2 = now_ms();
            st = iluk_symbolic(h->sp.Ahat, K < 0 ? 0 : K, h->F);
            if (st != SPCG_OK) { delete h; return st; }
            t3 = now_ms();
            st = ilu_numeric(h->sp.Ahat, h->F);
            h->info.zero_pivot_row = h->F.zero_pivot_row;
            if (st != SPCG_OK) { delete h; return st; }
            t4 = now_ms();
        }
        const Csr& Ah = h->sp.Ahat;
        // NEXT-2: fp32 factors: round every stored L / U value to fp32 (IEEE
        // round to nearest even); the operator is M = fl32(L) fl32(U), applied in fp64
        if (opt.factor_precision < 0 || opt.factor_precision > SPCG_FACTORS_F32) {
            delete h;
            set_error("bad factor_precision");
            return SPCG_ERR_INVALID_ARG;
        }
        if (opt.factor_precision == SPCG_FACTORS_F32 && !h->identity) {
            for (double& v : h->F.L.val) v = (double)(float)v;
            for (double& v : h->F.U.val) v = (double)(float)v;
            for (int64_t i = 0; i < h->n; ++i) {
                const double d = h->F.U.val[h->F.U.rp[i]];
                if (d == 0.0 || !std::isfinite(d)) {
                    h->info.zero_pivot_row = i;
                    delete h;
                    set_error("pivot u_ii rounds to 0 or overflows in fp32 at row " + std::to_string(i));
                    return SPCG_ERR_ZERO_PIVOT;
                }
            }
            for (double v : h->F.L.val)
                if (!std::isfinite(v)) {
                    delete h;
                    set_error("a factor value overflows fp32");
                    return SPCG_ERR_INVALID_ARG;
                }
        }
        const bool f32 = opt.factor_precision == SPCG_FACTORS_F32 && !h->identity;

        // executor and grid
        int sms = 148;
        if (opt.device >= 0) {
            sms = spcg_dev_sm_count(opt.device);
            if (sms <= 0) { delete h; return SPCG_ERR_CUDA; }
        }
        // AUTO: the chunked executor streams thread-per-row records of <= SPCG_WCAP entry
        // columns; rows wider than that (ILU(K) fill of 3-D stencils: ~57 entries per L row
        // for 27-point ILU(2)) need continuation records on the serial chain.  For those the
        // sync-free executor with one warp per row is fastest (measured, FEM 48^3 ILU(2), per
        // iteration: chunked 31.5 ms, level warp-per-row 6.3 ms, sync-free warp-per-row
        // 2.2 ms).
        int strategy = opt.sptrsv;
        // AUTO: the warp-chain executor whenever it applies (narrow rows, a chain
        // partition exists): every wavefront handoff inside a chain is a register
        // shuffle; otherwise the round-1 choice below.
        std::string chain_why;
        bool chain_built = false;
        const int slots = sms * spcg_dev_ctas_per_sm();        // co-resident persistent CTAs
        int chain_ctas = 0;
        if ((strategy == SPCG_SPTRSV_AUTO || strategy == SPCG_SPTRSV_WCHAIN) && !h->identity) {
            // components are packed onto as many chains as there are SMs (or the CTAs asked for)
            const int target = opt.parts > 0 ? opt.parts : sms;
            chain_built = build_chain_layout(h->A, h->F, std::max(1, target), f32, h->lay.C, &chain_why);
            if (chain_built) {
                // CTAs: one per chain up to the SM count (more chains share CTAs, one solver
                // warp each); large systems take every SM so the SpMV and vector phases use
                // them all.  The chains of a CTA must fit its shared memory.
                const int nch = h->lay.C.nchains;
                const int64_t npos = 32 * h->lay.C.nsteps;
                int p = opt.parts > 0 ? opt.parts : ((nch >= slots || npos >= (1 << 17)) ? slots : nch);
                p = std::max(1, std::min<int>(p, slots));
                if ((nch + p - 1) / p > 8) p = std::min(slots, (nch + 7) / 8);
                ChainSmemCfg cfg;
                if ((nch + p - 1) / p > 8 || !chain_smem_config(h->lay.C, (nch + p - 1) / p, cfg)) {
                    chain_built = false;
                    chain_why = "the chains per CTA do not fit shared memory";
                    h->lay.C = ChainLayout();
                } else {
                    chain_ctas = p;
                }
            }
            // AUTO keeps the chain executor where it measured fastest (profiles/r02/exec_cmp):
            // 2-D chains (components, grid2d; 1024^2 Poisson 2.94 vs 3.17 ms/it chunked); not
            // 3-D grids, whose z-couplings cross chains through flags (64^3 Poisson 1.06 vs
            // 0.43 ms/it chunked tiles); and small systems only when every dependency is a
            // shuffle (else the one-CTA resident executor: 64^2 Poisson 0.089 vs 0.142 ms/it)
            if (chain_built && strategy == SPCG_SPTRSV_AUTO) {
                const ChainLayout& CL = h->lay.C;
                const bool pure = CL.hist_entries + CL.glob_entries + CL.ext_entries == 0;
                if (CL.partition == "grid3d" || (h->n <= SPCG_RESIDENT_MAX_N && !pure)) {
                    chain_built = false;
                    h->lay.C = ChainLayout();
                }
            }
            if (chain_built) strategy = SPCG_SPTRSV_WCHAIN;
            else if (strategy == SPCG_SPTRSV_WCHAIN) {
                delete h;
                set_error("warp-chain executor does not apply: " + chain_why);
                return SPCG_ERR_INVALID_ARG;
            }
        }
        if (strategy == SPCG_SPTRSV_AUTO) {
            const double wl = h->n > 0 ? (double)h->F.L.nnz() / (double)h->n : 0.0;
            strategy = (h->identity || wl <= (double)SPCG_WCAP) ? SPCG_SPTRSV_CHUNKED : SPCG_SPTRSV_SYNCFREE;
            // Small systems: the one-CTA resident executor (vectors in shared memory, CTA
            // barriers) beats the chunked pipeline on every narrow case measured (per
            // iteration: 32^2 Poisson 53 -> 46 us, 64^2 Poisson 133 -> 90, 16^3 Poisson
            // 129 -> 49, layered 64x48 93 -> 54); wide ILU(K) rows stay sync-free
            // (DESIGN.md §5.3).
            if (!h->identity && wl <= (double)SPCG_WCAP && h->n <= SPCG_RESIDENT_MAX_N)
                strategy = SPCG_SPTRSV_RESIDENT;
        }
        if (strategy < 1 || strategy > 5) { delete h; set_error("bad sptrsv executor"); return SPCG_ERR_INVALID_ARG; }
        if (strategy == SPCG_SPTRSV_RESIDENT && h->n > SPCG_RESIDENT_MAX_N) {
            delete h;
            set_error("the resident executor holds every vector in one CTA's shared memory: n <= SPCG_RESIDENT_MAX_N");
            return SPCG_ERR_INVALID_ARG;
        }
        int parts = opt.parts;
        // small systems: one CTA, except sync-free (wide ILU(K) rows), whose rows of a
        // wavefront spread over every warp of the grid (FEM 20^3 ILU(2), per iteration:
        // 1 CTA 2.38 ms, 37 CTAs 0.81 ms; profiles/r01_final/fem_parts.jsonl)
        // Mid-size narrow systems (4096 < n <= 16384) take 16 CTAs: one CTA walks every
        // wavefront alone, 16 let the inspector split the chains (components / strided /
        // tiles); per iteration, layered 90x91 231 -> 84 us, 25^3 Poisson 487 -> 169 us,
        // 128^2 Poisson 449 -> 298 us (profiles/r01_final/mid_parts.jsonl; 16 has the
        // smallest sum over the four cases of 1..37).
        if (parts <= 0) {
            if (strategy == SPCG_SPTRSV_SYNCFREE || h->n > 16384) parts = slots;
            else parts = (h->n <= 4096 || h->identity) ? 1 : std::min(16, slots);
        }
        if (strategy == SPCG_SPTRSV_RESIDENT) parts = 1;
        if (strategy == SPCG_SPTRSV_WCHAIN) {
            parts = chain_ctas;
        } else {
            parts = std::max(1, std::min<int>(parts, slots));
            if ((int64_t)parts > h->n) parts = (int)h->n;
        }
        if (strategy != SPCG_SPTRSV_WCHAIN) {
            h->lay.C = ChainLayout();
            build_spmv_layout(h->A, h->lay.A);
        }
        if (strategy == SPCG_SPTRSV_WCHAIN) {
            // the warp-chain kernel reads only lay.C (its own SpMV layout and records)
            h->lay.strategy = strategy;
            h->lay.parts = parts;
            h->lay.ring = 0;
            h->lay.part_begin.assign({0, h->n});
        } else {
            build_tri_layouts(h->F, strategy, parts, spcg_dev_ring_max(), opt.wide_min, opt.chunk_partition, h->lay);
        }
        double t5 = now_ms();
        int64_t bytes = 0;
        if (opt.device >= 0) {
            DevAllocator alc;
            alc.alloc = opt.dev_alloc;
            alc.free = opt.dev_free;
            alc.ctx = opt.alloc_ctx;
            st = spcg_dev_create(opt.device, opt.stream, h->lay, h->n, h->identity, alc, &h->dev, &bytes);
            if (st != SPCG_OK) { delete h; return st; }
        }
        double t6 = now_ms();

        spcg_setup_info_t& I = h->info;
        I.chosen_pct = h->sp.chosen_pct;
        I.m_t = h->sp.m_t;
        I.w_A = h->sp.w_A;
        I.w_Ahat = h->sp.w_Ahat;
        I.n_tried = h->sp.n_tried;
        for (int r = 0; r < 8; ++r) {
            I.tried_pct[r] = h->sp.tried_pct[r];
            I.indicator[r] = h->sp.indicator[r];
            I.tried_w[r] = h->sp.tried_w[r];
            I.tried_reduction_pct[r] = h->sp.reduction[r];
        }
        I.n = h->n;
        I.nnz_A = h->A.nnz();
        I.nnz_Ahat = Ah.nnz();
        I.nnz_L = h->F.L.nnz();
        I.nnz_U = h->F.U.nnz();
        I.levels_L = h->F.wL;
        I.levels_U = h->F.wU;
        I.zero_pivot_row = -1;
        I.setup_ms_validate = t1 - t0;
        I.setup_ms_sparsify = t2 - t1;
        I.setup_ms_symbolic = t3 - t2;
        I.setup_ms_numeric = t4 - t3;
        I.setup_ms_layout = t5 - t4;
        I.setup_ms_upload = t6 - t5;
        I.sptrsv = strategy;
        I.parts = parts;
        I.device_bytes = bytes;
        I.setup_device = on_gpu ? SPCG_SETUP_GPU : SPCG_SETUP_HOST;
        I.factor_precision = f32 ? SPCG_FACTORS_F32 : SPCG_FACTORS_F64;
        I.record_value_bytes = strategy == SPCG_SPTRSV_WCHAIN ? h->lay.C.vb : 8;
        {
            static const char* kinds[] = {"contiguous", "strided", "affinity", "components", "tiles"};
            I.partition = -1;
            if (strategy == SPCG_SPTRSV_CHUNKED)
                for (int k = 0; k < 5; ++k) if (h->lay.partition == kinds[k]) I.partition = k;
            if (strategy == SPCG_SPTRSV_WCHAIN) {
                static const char* ck[] = {"components", "grid3d", "grid2d"};
                for (int k = 0; k < 3; ++k) if (h->lay.C.partition == ck[k]) I.partition = 5 + k;
                I.chains = h->lay.C.nchains;
                I.positions = 32 * h->lay.C.nsteps;
                I.chain_entries[0] = h->lay.C.prev_entries;
                I.chain_entries[1] = h->lay.C.hist_entries;
                I.chain_entries[2] = h->lay.C.glob_entries;
                I.chain_entries[3] = h->lay.C.ext_entries;
            }
        }
        // B_iter: 12 B per stored entry of A, L_s, U_s; 1/u_ii; three row
        // pointers; two level_rows arrays; 120 B of vector traffic per row.
        const double n = (double)h->n;
        const double nU_s = (double)(I.nnz_U - h->n);
        if (h->identity) {
            I.algo_bytes_per_iter = 12.0 * I.nnz_A + 4.0 * (n + 1) + 96.0 * n;
            I.algo_flops_per_iter = 2.0 * I.nnz_A + 10.0 * n;
        } else {
            // NEXT-2: 4-byte factor values where the records carry them (8 B per entry)
            const double fb = I.record_value_bytes == 4 ? 8.0 : 12.0;
            I.algo_bytes_per_iter = 12.0 * I.nnz_A + fb * (I.nnz_L + nU_s) + 8.0 * n + 12.0 * (n + 1) + 8.0 * n +
                                    120.0 * n;
            I.algo_flops_per_iter = 2.0 * (I.nnz_A + I.nnz_L + nU_s) + n + 12.0 * n;
        }
        I.setup_ms_total = now_ms() - t0;
        *out = h;
        return SPCG_OK;
    } catch (const std::bad_alloc&) {
        delete h;
        set_error("host allocation failed");
        return SPCG_ERR_OOM;
    } catch (...) {
        delete h;
        set_error("unexpected exception in setup");
        return SPCG_ERR_INTERNAL;
    }
}

spcg_status_t spcg_get_setup_info(spcg_handle_t h, spcg_setup_info_t* info) {
    if (!h || !info) return SPCG_ERR_INVALID_ARG;
    *info = h->info;
    return SPCG_OK;
}

// NEXT-4: several right-hand sides of one system together
spcg_status_t spcg_solve_multi(spcg_handle_t h, const double* B, double* X, int32_t nrhs, double eps, int64_t kmax,
                               uint32_t flags, spcg_solve_info_t* info) {
    if (!h || !B || !X || nrhs < 1 || kmax < 0 || !(eps >= 0.0)) {
        set_error("bad solve_multi arguments");
        return SPCG_ERR_INVALID_ARG;
    }
    if (flags != 0) { set_error("solve_multi: flags must be 0 (device pointers, x0 = 0)"); return SPCG_ERR_INVALID_ARG; }
    if (kmax > SPCG_KMAX_LIMIT) { set_error("kmax > SPCG_KMAX_LIMIT"); return SPCG_ERR_INVALID_ARG; }
    if (!h->dev) { set_error("host-only handle"); return SPCG_ERR_NO_DEVICE; }
    try {
        spcg_status_t worst = SPCG_OK;
        for (int32_t g0 = 0; g0 < nrhs; g0 += 4) {            // groups of at most 4
            const int m = std::min<int32_t>(4, nrhs - g0);
            double out[16], ms = 0.0;
            const double t0 = now_ms();
            spcg_status_t st = spcg_dev_solve_multi(h->dev, B + (size_t)g0 * h->n, X + (size_t)g0 * h->n, m, eps, kmax,
                                                    out, &ms);
            if (st != SPCG_OK) return st;
            for (int j = 0; j < m; ++j) {
                if (!info) continue;
                spcg_solve_info_t& I = info[g0 + j];
                std::memset(&I, 0, sizeof I);
                I.iterations = (int64_t)out[4 * j];
                I.rnorm = std::sqrt(out[4 * j + 1]);
                I.status = (spcg_status_t)out[4 * j + 2];
                I.converged = I.status == SPCG_OK && eps > 0.0;
                I.iter_phase_ms = ms;                         // one launch for the whole group
                I.total_ms = now_ms() - t0;
            }
            for (int j = 0; j < m; ++j) {
                const spcg_status_t sj = (spcg_status_t)out[4 * j + 2];
                if (sj < 0 && (worst >= 0 || sj < worst)) worst = sj;
                else if (sj == SPCG_NOT_CONVERGED && worst == SPCG_OK) worst = sj;
            }
        }
        return worst;
    } catch (...) {
        set_error("unexpected exception in solve_multi");
        return SPCG_ERR_INTERNAL;
    }
}

spcg_status_t spcg_solve(spcg_handle_t h, const double* b, double* x, double eps, int64_t kmax,
                         uint32_t flags, spcg_solve_info_t* info) {
    if (!h || !b || !x || kmax < 0 || !(eps >= 0.0)) { set_error("bad solve arguments"); return SPCG_ERR_INVALID_ARG; }
    if (kmax > SPCG_KMAX_LIMIT) { set_error("kmax > SPCG_KMAX_LIMIT"); return SPCG_ERR_INVALID_ARG; }
    if (!h->dev) { set_error("host-only handle"); return SPCG_ERR_NO_DEVICE; }
    spcg_solve_info_t tmp{};
    spcg_solve_info_t* I = info ? info : &tmp;
    std::memset(I, 0, sizeof *I);
    try {
        double t0 = now_ms();
        spcg_status_t st;
        if (flags & SPCG_HOST_PTRS) {
            // host buffers: H2D of b (and x0), solve, D2H of x — all inside the call
            double* db = nullptr;
            st = spcg_dev_copy(h->dev, &db, nullptr, 0, -1);    // the handle's staging buffer (b | x)
            if (st != SPCG_OK) return st;
            double* dx = db + h->n;
            st = spcg_dev_copy(h->dev, db, b, (size_t)h->n * 8, 1);
            if (st != SPCG_OK) return st;
            if (flags & SPCG_USE_X0) {
                st = spcg_dev_copy(h->dev, dx, x, (size_t)h->n * 8, 1);
                if (st != SPCG_OK) return st;
            }
            st = spcg_dev_solve(h->dev, db, dx, eps, kmax, (flags & SPCG_USE_X0) != 0, I, &h->rhist);
            // x is written back only when the kernel ran (it then holds x_k, Alg. 1 line 17);
            // on a launch/argument error the caller's x stays untouched
            if (st == SPCG_OK || st == SPCG_NOT_CONVERGED || st == SPCG_ERR_BREAKDOWN) {
                spcg_status_t cs = spcg_dev_copy(h->dev, x, dx, (size_t)h->n * 8, 2);
                if (cs != SPCG_OK) return cs;
            }
        } else {
            st = spcg_dev_solve(h->dev, b, x, eps, kmax, (flags & SPCG_USE_X0) != 0, I, &h->rhist);
        }
        I->total_ms = now_ms() - t0;
        return st;
    } catch (...) {
        set_error("unexpected exception in solve");
        return SPCG_ERR_INTERNAL;
    }
}

spcg_status_t spcg_solve_async(spcg_handle_t h, const double* b, double* x, double eps, int64_t kmax,
                               uint32_t flags) {
    if (!h || !b || !x || kmax < 0 || !(eps >= 0.0)) { set_error("bad solve arguments"); return SPCG_ERR_INVALID_ARG; }
    if (flags & SPCG_HOST_PTRS) { set_error("spcg_solve_async takes device pointers only"); return SPCG_ERR_INVALID_ARG; }
    if (kmax > SPCG_KMAX_LIMIT) { set_error("kmax > SPCG_KMAX_LIMIT"); return SPCG_ERR_INVALID_ARG; }
    if (!h->dev) { set_error("host-only handle"); return SPCG_ERR_NO_DEVICE; }
    try {
        return spcg_dev_solve_begin(h->dev, b, x, eps, kmax, (flags & SPCG_USE_X0) != 0);
    } catch (...) {
        set_error("unexpected exception in solve");
        return SPCG_ERR_INTERNAL;
    }
}

spcg_status_t spcg_set_stream(spcg_handle_t h, void* stream) {
    if (!h) return SPCG_ERR_INVALID_ARG;
    if (!h->dev) { set_error("host-only handle"); return SPCG_ERR_NO_DEVICE; }
    return spcg_dev_set_stream(h->dev, stream);
}

spcg_status_t spcg_solve_wait(spcg_handle_t h, spcg_solve_info_t* info) {
    if (!h) return SPCG_ERR_INVALID_ARG;
    if (!h->dev) { set_error("host-only handle"); return SPCG_ERR_NO_DEVICE; }
    spcg_solve_info_t tmp{};
    spcg_solve_info_t* I = info ? info : &tmp;
    std::memset(I, 0, sizeof *I);
    try {
        return spcg_dev_solve_end(h->dev, I, &h->rhist);
    } catch (...) {
        set_error("unexpected exception in solve");
        return SPCG_ERR_INTERNAL;
    }
}

spcg_status_t spcg_apply_spmv(spcg_handle_t h, const double* p, double* w, double* pw) {
    if (!h || !p || !w) return SPCG_ERR_INVALID_ARG;
    if (!h->dev) return SPCG_ERR_NO_DEVICE;
    return spcg_dev_apply(h->dev, 1, p, w, nullptr, pw);
}
spcg_status_t spcg_apply_lower(spcg_handle_t h, const double* r, double* y) {
    if (!h || !r || !y) return SPCG_ERR_INVALID_ARG;
    if (!h->dev) return SPCG_ERR_NO_DEVICE;
    return spcg_dev_apply(h->dev, 2, r, y, nullptr, nullptr);
}
spcg_status_t spcg_apply_upper(spcg_handle_t h, const double* y, double* z, const double* r, double* rz) {
    if (!h || !y || !z) return SPCG_ERR_INVALID_ARG;
    if (!h->dev) return SPCG_ERR_NO_DEVICE;
    return spcg_dev_apply(h->dev, 3, y, z, r, rz);
}
spcg_status_t spcg_apply_precond(spcg_handle_t h, const double* r, double* z, double* rz) {
    if (!h || !r || !z) return SPCG_ERR_INVALID_ARG;
    if (!h->dev) return SPCG_ERR_NO_DEVICE;
    return spcg_dev_apply(h->dev, 4, r, z, r, rz);
}

spcg_status_t spcg_export(spcg_handle_t h, int32_t what, void* buf, size_t* bytes) {
    if (!h || !bytes) return SPCG_ERR_INVALID_ARG;
    const Csr& Ah = h->sp.Ahat;
    std::vector<int64_t> p64;
    std::vector<int32_t> r32;
    switch (what) {
        case SPCG_EXPORT_AHAT_ROWPTR: return put(Ah.rp, buf, bytes);
        case SPCG_EXPORT_AHAT_COL: return put(Ah.col, buf, bytes);
        case SPCG_EXPORT_AHAT_VAL: return put(Ah.val, buf, bytes);
        case SPCG_EXPORT_L_ROWPTR: return put(h->F.L.rp, buf, bytes);
        case SPCG_EXPORT_L_COL: return put(h->F.L.col, buf, bytes);
        case SPCG_EXPORT_L_VAL: return put(h->F.L.val, buf, bytes);
        case SPCG_EXPORT_U_ROWPTR: return put(h->F.U.rp, buf, bytes);
        case SPCG_EXPORT_U_COL: return put(h->F.U.col, buf, bytes);
        case SPCG_EXPORT_U_VAL: return put(h->F.U.val, buf, bytes);
        case SPCG_EXPORT_FILL_LEVEL: return put(h->F.fill_level, buf, bytes);
        case SPCG_EXPORT_LEVEL_L: return put(h->F.levL, buf, bytes);
        case SPCG_EXPORT_LEVEL_U: return put(h->F.levU, buf, bytes);
        case SPCG_EXPORT_LEVELPTR_L: level_sets(h->F.levL, h->F.wL, p64, r32); return put(p64, buf, bytes);
        case SPCG_EXPORT_LEVELROWS_L: level_sets(h->F.levL, h->F.wL, p64, r32); return put(r32, buf, bytes);
        case SPCG_EXPORT_LEVELPTR_U: level_sets(h->F.levU, h->F.wU, p64, r32); return put(p64, buf, bytes);
        case SPCG_EXPORT_LEVELROWS_U: level_sets(h->F.levU, h->F.wU, p64, r32); return put(r32, buf, bytes);
        case SPCG_EXPORT_RHIST: return put(h->rhist, buf, bytes);
        case 100: return put(h->lay.S.bytes, buf, bytes);          // debug: chunked record stream
        case 101: return put(h->lay.S.part_chunk, buf, bytes);
        case 102: return put(h->lay.S.part_uchunk, buf, bytes);
        case 103: return put(h->lay.part_begin, buf, bytes);
        case 104: return put(h->lay.C.recL, buf, bytes);           // debug: warp-chain records
        case 105: return put(h->lay.C.recU, buf, bytes);
        case 106: return put(h->lay.C.perm, buf, bytes);
        case 107: return put(h->lay.C.chain_step, buf, bytes);
        case 108: return put(h->lay.C.chain_flags, buf, bytes);
        case 109: return put(h->lay.C.A.eoff, buf, bytes);
        case 110: return put(h->lay.C.A.col, buf, bytes);
        case 111: return put(h->lay.C.A.val, buf, bytes);
        default: set_error("unknown export item"); return SPCG_ERR_INVALID_ARG;
    }
}

// debug only (not in spcg.h): heartbeat snapshot of a possibly running solve
int spcg_dbg_heartbeats(void* dev, unsigned long long* out, int n);
int spcg_dbg_handle_heartbeats(spcg_handle_t h, unsigned long long* out, int n) {
    if (!h || !h->dev) return -1;
    return spcg_dbg_heartbeats((void*)h->dev, out, n);
}

void spcg_destroy(spcg_handle_t h) {
    if (!h) return;
    if (h->dev) spcg_dev_destroy(h->dev);
    delete h;
}

}  // extern "C"
