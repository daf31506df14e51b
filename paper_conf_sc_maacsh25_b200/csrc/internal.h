// internal.h — host-side structures shared by the library's translation units.
// Not part of the ABI (include/spcg.h is).  No oracle code or header is used here.
#pragma once
#include <cstdint>
#include <memory>
#include <utility>
#include <string>
#include <vector>

#include "../../include/spcg.h"

struct DevAllocator;               // spcg_options_t allocator hooks (defined below)

namespace spcg {

// Allocator whose value-construction is a no-op: the large layout arrays are filled in
// parallel (first touch by the filling threads) instead of zeroed by one thread first.
template <class T>
struct NoInit : std::allocator<T> {
    template <class U>
    struct rebind { using other = NoInit<U>; };
    NoInit() = default;
    template <class U>
    NoInit(const NoInit<U>&) {}
    template <class U>
    void construct(U* p) { ::new ((void*)p) U; }
    template <class U, class... A>
    void construct(U* p, A&&... a) { ::new ((void*)p) U(std::forward<A>(a)...); }
};
template <class T>
using fast_vector = std::vector<T, NoInit<T>>;

struct Csr {                       // host CSR, int64 row pointers
    int64_t n = 0;
    std::vector<int64_t> rp;
    fast_vector<int32_t> col;      // resize() leaves entries uninitialised: every builder writes them all
    fast_vector<double> val;
    int64_t nnz() const { return rp.empty() ? 0 : rp.back(); }
};

void set_error(const std::string& s);
double now_ms();

// ---- setup.cpp -------------------------------------------------------------
// Validation (O1 contract) and the transpose map pos_t[q] = position of the
// mirror entry (j,i) of entry q = (i,j).
spcg_status_t validate_and_mirror(const Csr& A, std::vector<int64_t>& pos_t);

// Longest-path wavefront levels by Kahn frontier peeling (independent of the
// oracle's dynamic programme).  lower = true: i depends on j < i in row i;
// lower = false: i depends on j > i.  Returns number of levels.
int64_t kahn_levels(const Csr& M, bool lower, std::vector<int32_t>& lev);

struct SparsifyResult {
    Csr Ahat;
    double chosen_pct = 0.0;
    int64_t m_t = 0, w_A = 0, w_Ahat = 0;
    int n_tried = 0;
    double tried_pct[8] = {0}, indicator[8] = {0}, reduction[8] = {0};
    int64_t tried_w[8] = {0};
};
spcg_status_t sparsify_select(const Csr& A, const std::vector<int64_t>& pos_t,
                              const spcg_drop_params_t& p, SparsifyResult& out);

// ILU(K) symbolic by the fill-path characterisation (BFS through lower-numbered
// vertices), numeric IKJ factorisation (level-parallel over rows).
struct Factors {
    Csr L;                         // strictly lower, unit diagonal implicit
    Csr U;                         // upper incl. diagonal (first in each row)
    std::vector<int32_t> fill_level;   // per entry of the merged row (L then U), row-major
    std::vector<int32_t> levL, levU;   // per-row wavefront level of the L / U solve
    int64_t wL = 0, wU = 0;
    int64_t zero_pivot_row = -1;
};
spcg_status_t iluk_symbolic(const Csr& Ahat, int K, Factors& F);
spcg_status_t ilu_numeric(const Csr& Ahat, Factors& F);

// ---- gsetup.cu (NEXT-1) ------------------------------------------------------
// Validation, Algorithm 2, ILU(0) and the factor level sets on the GPU; fills sp and F
// exactly as validate_and_mirror + sparsify_select + iluk_symbolic(K = 0) + ilu_numeric
// do (bit-exact; the Frobenius indicator values up to summation order).  phase_ms[5]:
// upload + validation, Algorithm 2, L/U split, ILU(0) + levels, download.
spcg_status_t gpu_setup_k0(const Csr& A, const spcg_drop_params_t& p, int device, void* stream,
                           const ::DevAllocator& alc, SparsifyResult& sp, Factors& F, double* phase_ms);

// ---- layout.cpp ------------------------------------------------------------
// Sliced-ELL (slice height 32, column-major inside a slice) triangular-solve
// schedule for one factor.  Entries of slice s occupy [eoff[s]*32, eoff[s+1]*32).
struct TriLayout {
    int32_t nslices = 0;
    std::vector<int64_t> eoff;     // [nslices+1] in units of 32-entry columns
    std::vector<int32_t> rows;     // [nslices*32], -1 = padding lane
    std::vector<uint8_t> publish;  // [nslices*32] 1 if the row's value is read through its flag slot
    std::vector<int32_t> rlen;     // [nslices*32] dependencies of the row (entries beyond are padding)
    std::vector<int32_t> src;      // [entries*32] >= 0: smem ring slot; < 0: -(j+1) global/flagged
    std::vector<double> val;       // [entries*32]
    std::vector<double> dinv;      // [nslices*32] 1/u_ii (upper only)
    std::vector<int32_t> gptr;     // [ngroups+1] slice ranges of the wavefront groups
    std::vector<int32_t> part_gptr;// [parts+1]  group ranges per part (chunked); levels: [0, ngroups]
    int32_t ngroups = 0;
    int64_t total_cols = 0;        // sum of slice widths
    // LEVEL with wide rows (mean dependencies per row > SPCG_WCAP, e.g. ILU(K) fill):
    // warp-per-row CSR in execution order (level, ascending row), read coalesced by
    // the 32 lanes of a warp and reduced with shuffles.
    bool wide = false;
    std::vector<int32_t> wrow;     // [n] row at each position
    std::vector<int64_t> wptr;     // [n+1] dependency range of each position
    std::vector<int32_t> wcol;     // dependencies (U: diagonal excluded)
    std::vector<double> wval;
    std::vector<double> wdinv;     // [n] 1/u_ii per position (upper only)
    std::vector<int32_t> wgptr;    // [ngroups+1] position range of each level
    // RESIDENT: one fixed 64-byte record per slice slot (slice s, lane l at s*32+l), so
    // the kernel can stage a slice with four 16-byte cp.async per lane, addressed by the
    // slot alone: {int32 (row+1) | level<<16, int32 len | next<<16, double 1/u_ii,
    // int32 col[4], double val[4]} (the vector fields 16-byte aligned); next = level of
    // slice s + SPCG_RES_WARPS (the same warp's next slice; 0xffff: none).  Entries k >= 4 stay in src/val above (read through eoff).
    std::vector<uint8_t> rrec;
};
constexpr int SPCG_RREC_BYTES = 64;
constexpr int SPCG_RREC_PF = 4;
constexpr int SPCG_RES_WARPS = 8;      // warps of the resident CTA (slice s -> warp s % 8)

struct SpmvLayout {                // SELL-32 of the original A, natural row order
    int32_t nslices = 0;
    std::vector<int64_t> eoff;
    fast_vector<int32_t> col;      // every element written by the builder (no zero pass)
    fast_vector<double> val;
};

// Chunked executor stream.  Per part (CTA) one byte stream of
// slice records, L section then U section, cut into CHUNK-byte chunks that the
// kernel copies into a shared-memory ring with cp.async.bulk.
#ifndef SPCG_CHUNK_KB
#define SPCG_CHUNK_KB 8      // 8 KB: ~7 records of a 2-D stencil per chunk (4 KB: 3; measured -24 % per iteration)
#endif
constexpr int SPCG_CHUNK_BYTES = SPCG_CHUNK_KB * 1024;   // record-stream chunk (one TMA bulk copy)
#ifndef SPCG_NCHUNK_SLOTS
#define SPCG_NCHUNK_SLOTS 8
#endif
constexpr int SPCG_NCHUNK = SPCG_NCHUNK_SLOTS;   // chunk ring slots in shared memory (kernel side)
constexpr int SPCG_MAXREC = 8;          // records per chunk (side-data slots)
constexpr int SPCG_WCAP = 8;            // entry columns per record
#ifndef SPCG_NSOLVER_WARPS
#define SPCG_NSOLVER_WARPS 1
#endif
// solver warps per CTA: the slices of a part's stream are dealt round-robin to them
// and a shared-memory chain counter orders their ring accesses
constexpr int SPCG_NSOLVER = SPCG_NSOLVER_WARPS;
constexpr int SPCG_REC_HDR = 272;       // 16 B header + 32 x {int32 row, uint32 meta}
constexpr int SPCG_CHUNK_HDR = 32;      // u16 nrec, u16 -, u32 used, u16 rec_off[8], pad
enum { REC_FIRST = 1, REC_LAST = 2, REC_SYNC = 4, REC_UPPER = 8, REC_EXT = 16, REC_WIDE = 32 };
constexpr int SPCG_WP = 4;              // entry columns the pipelined solver keeps in registers

struct ChunkStream {
    std::vector<uint8_t> bytes;          // nchunks * CHUNK_BYTES
    std::vector<int32_t> part_chunk;     // [parts+1] first chunk of each part
    std::vector<int32_t> part_uchunk;    // [parts]   first U chunk of each part
    std::vector<uint32_t> chunk_bytes;   // [nchunks]  used bytes (what the bulk copy moves)
    int64_t used_bytes = 0;
    int64_t records = 0;
};

// Warp-chain executor.  Rows are split into chains; a chain is
// walked by one warp in steps of <= 32 rows (one per lane) of one wavefront level,
// levels ascending (L) and the same steps in reverse (U: the reverse of a topological
// order of L is one of U, the ILU(K) pattern being symmetric).  All vectors of
// Algorithm 1 live in execution ("position") order pos = 32 * global_step + lane for
// the whole solve; b and x are permuted on entry and exit.  A record per step holds,
// lane-major, W (a power of two) dependency tags + values (and 1/u_ii for U):
//   tag u32 [32][W] at 0, value f64 [32][W] (f32 with vb = 4) at 128 W, (U) 1/u_ii f64
//   [32] at (128 + 32 vb) W, trailer {u32 publish mask (lanes whose value another chain
//   reads), u32 flags}.
//   tag = kind << 29 | payload:
//     PREV (0): payload = the lane whose previous-step value is the dependency (a warp
//               shuffle, no memory access); padding entries are PREV lane 0, value 0
//     HIST (1): lane payload & 31, `(payload >> 5) & 255` steps back (shared-memory ring)
//     GLOB (2): own chain, older than the ring: position payload, read from global
//     EXT  (3): another chain: position payload & (2^28-1), ordinal (payload >> 28) & 1
//               of the lane's prefetched flags (ready flag prefetched one chunk ahead)
//     EXTS (4): another chain, beyond two per lane and step: polled at use
enum { CT_PREV = 0, CT_HIST = 1, CT_GLOB = 2, CT_EXT = 3, CT_EXTS = 4 };
enum { CS_SLOW = 1, CS_EXT = 2 };                 // record trailer flags
// per-chain flags: which kinds a pass of the chain uses (the kernel picks the plain
// shuffle-only step body when none is set)
enum { CC_LHIST = 1, CC_LEXT = 2, CC_UHIST = 4, CC_UEXT = 8, CC_LGLOB = 16, CC_UGLOB = 32, CC_LPUB = 64,
       CC_UPUB = 128 };
constexpr int SPCG_CHAIN_WMAX = 16;              // dependency columns per record (wider: other executors)
constexpr int SPCG_CHAIN_HIST = 32;              // steps kept in the per-warp history ring

struct ChainLayout {
    int32_t nchains = 0;
    int32_t W_L = 0, W_U = 0;
    int32_t rec_L = 0, rec_U = 0;         // bytes per record
    int32_t vb = 8;                       // bytes per factor value in the records (8, or 4 with fp32 factors)
    int64_t nsteps = 0;                   // global steps; positions = 32 * nsteps
    std::vector<int64_t> chain_step;      // [nchains+1] first global step of each chain
    std::vector<uint32_t> chain_flags;    // [nchains] CC_*
    std::vector<int32_t> perm;            // [npos] row at each position (-1 padding)
    std::vector<int32_t> iperm;           // [n] position of each row
    fast_vector<uint8_t> recL, recU;      // nsteps records each (zeroed in parallel by the builder)
    SpmvLayout A;                         // SELL-32 of A over positions (slice = step), uniform width WA
    int32_t WA = 0;
    std::string partition;                // components / grid2d / grid3d
    int64_t ext_entries = 0, hist_entries = 0, glob_entries = 0, prev_entries = 0;
};
// Builds the chain layout when the factors suit it (dependency columns <= WMAX, a
// partition into chains found); returns false (why set) otherwise.
// f32: the factor values are fp32-representable (NEXT-2) -> 4-byte record values when
// the records are narrow (W <= 4; wider records keep 8-byte values).
bool build_chain_layout(const Csr& A, const Factors& F, int target_chains, bool f32, ChainLayout& out,
                        std::string* why);

// Shared memory of the warp-chain kernel per solver warp: mbarriers (128 B), NST stages
// of SPCG_CHAIN_C steps (records + the pass's operand slices), the prefetched-flag queue,
// the history ring.  The most stages (2..16) whose per-CTA total fits; false if none.
#ifndef SPCG_CHAIN_STEPS
#define SPCG_CHAIN_STEPS 8
#endif
constexpr int SPCG_CHAIN_C = SPCG_CHAIN_STEPS;   // steps per stage (compile-time in the kernel)
struct ChainSmemCfg {
    int32_t nst = 0;
    uint32_t stage_bytes = 0, warp_bytes = 0, ext_off = 0, hist_off = 0;
    int32_t sp_nst = 0;                   // SpMV: stages per warp (0: register path), SPCG_SPMV_G slices each
    uint32_t sp_stage_bytes = 0;
    size_t cta_bytes = 0;                 // max of the triangular-solve and SpMV needs
};
constexpr int SPCG_SPMV_G = 4;           // SpMV slices per TMA stage
// dynamic shared memory of the warp-chain kernel: 227 KB per CTA minus its static blocks
constexpr size_t SPCG_CHAIN_SMEM_LIMIT = 227 * 1024 - 4096;
bool chain_smem_config(const ChainLayout& CL, int per_cta, ChainSmemCfg& out);

struct Layouts {
    int32_t strategy = SPCG_SPTRSV_LEVEL;
    int32_t parts = 1;
    int32_t ring = 0;              // entries of the shared-memory ring (chunked)
    std::vector<int64_t> part_begin; // [parts+1] prefix of part sizes (chunked)
    std::string partition;           // partition the inspector chose (chunked)
    SpmvLayout A;
    TriLayout L, U;
    ChunkStream S;                 // chunked executor only
    ChainLayout C;                 // warp-chain executor only
};

void build_spmv_layout(const Csr& A, SpmvLayout& out);
void build_tri_layouts(const Factors& F, int strategy, int parts, int ring_max, double wide_min, int force_part,
                       Layouts& out);

}  // namespace spcg

// ---- device side (kernels.cu), plain C++ interface -------------------------
struct spcg_device_s;
typedef struct spcg_device_s spcg_device_t;

struct DevAllocator {         // spcg_options_t allocator hooks (NULL: cudaMalloc / cudaFree)
    spcg_dev_alloc_fn alloc = nullptr;
    spcg_dev_free_fn free = nullptr;
    void* ctx = nullptr;
};
spcg_status_t spcg_dev_create(int device, void* stream, const spcg::Layouts& lay, int64_t n,
                              bool identity_precond, const DevAllocator& alloc, spcg_device_t** out,
                              int64_t* bytes);
void spcg_dev_destroy(spcg_device_t* d);
spcg_status_t spcg_dev_solve(spcg_device_t* d, const double* b, double* x, double eps, int64_t kmax,
                             bool use_x0, spcg_solve_info_t* info, std::vector<double>* rhist);
spcg_status_t spcg_dev_solve_begin(spcg_device_t* d, const double* b, double* x, double eps, int64_t kmax,
                                   bool use_x0);
int spcg_dev_ctas_per_sm();
int spcg_dev_ring_max();
spcg_status_t spcg_dev_set_stream(spcg_device_t* d, void* stream);
spcg_status_t spcg_dev_solve_end(spcg_device_t* d, spcg_solve_info_t* info, std::vector<double>* rhist);
spcg_status_t spcg_dev_apply(spcg_device_t* d, int op, const double* in, double* out,
                             const double* aux, double* scalar_out);
spcg_status_t spcg_dev_copy(spcg_device_t* d, void* dst, const void* src, size_t bytes, int kind);
spcg_status_t spcg_dev_solve_multi(spcg_device_t* d, const double* B, double* X, int nrhs, double eps, int64_t kmax,
                                   double* out_host, double* ms);
