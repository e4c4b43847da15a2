// efit_api.cu -- C ABI (include/efit.h): validation, tiling plan, workspace carve, CUDA-graph
// capture of the fit step.  Host code only; kernels live in efit_kernels.cu.
#include <dlfcn.h>
#include <nccl.h>  // types only: the functions are resolved at run time (see nccl_api)

#include <cmath>
#include <cstdarg>
#include <mutex>
#include <cstdio>
#include <cstring>
#include <new>
#include <vector>

#include "efit_internal.h"

using efit::Ctx;

struct efit_ctx {
    Ctx c;
};

namespace efit {
cudaError_t prepare_kernels(Ctx& c);
cudaError_t launch_make_pair(Ctx& c, const double* pcurr, cudaStream_t s);
}  // namespace efit

static thread_local char g_err[256] = "";

static int fail(Ctx* c, int code, const char* fmt, ...) {
    char* dst = c ? c->err : g_err;
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(dst, 256, fmt, ap);
    va_end(ap);
    if (c) std::snprintf(g_err, sizeof(g_err), "%s", c->err);
    return code;
}

// ------------------------------------------------------------------ NCCL, loaded at run time
// The library does not link libnccl: a Python host process already holds torch's libnccl.so.2
// (and a second copy of NCCL in one process is a hazard), so the functions are resolved from the
// copy already loaded (RTLD_NOLOAD), else from the system library; EFIT_NCCL_LIB names another file.
struct NcclApi {
    bool ok = false;
    char why[200] = "";
    ncclResult_t (*get_unique_id)(ncclUniqueId*) = nullptr;
    ncclResult_t (*comm_init_rank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*all_reduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                               cudaStream_t) = nullptr;
    ncclResult_t (*comm_destroy)(ncclComm_t) = nullptr;
    const char* (*error_string)(ncclResult_t) = nullptr;
};

static NcclApi& nccl_api() {
    static NcclApi api;
    static std::once_flag once;
    std::call_once(once, [] {
        const char* env = getenv("EFIT_NCCL_LIB");
        void* h = nullptr;
        if (env) h = dlopen(env, RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
        if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
        if (!h) {
            std::snprintf(api.why, sizeof(api.why), "cannot load NCCL: %s", dlerror());
            return;
        }
        api.get_unique_id = (decltype(api.get_unique_id))dlsym(h, "ncclGetUniqueId");
        api.comm_init_rank = (decltype(api.comm_init_rank))dlsym(h, "ncclCommInitRank");
        api.all_reduce = (decltype(api.all_reduce))dlsym(h, "ncclAllReduce");
        api.comm_destroy = (decltype(api.comm_destroy))dlsym(h, "ncclCommDestroy");
        api.error_string = (decltype(api.error_string))dlsym(h, "ncclGetErrorString");
        api.ok = api.get_unique_id && api.comm_init_rank && api.all_reduce && api.comm_destroy && api.error_string;
        if (!api.ok) std::snprintf(api.why, sizeof(api.why), "NCCL library lacks a required symbol");
    });
    return api;
}

static int cuda_fail(Ctx* c, cudaError_t e, const char* where) {
    if (c && c->nccl_err) {
        const int r = c->nccl_err;
        c->nccl_err = 0;
        return fail(c, EFIT_E_NCCL, "%s: NCCL: %s", where, nccl_api().error_string((ncclResult_t)r));
    }
    return fail(c, EFIT_E_CUDA, "%s: %s", where, cudaGetErrorString(e));
}

namespace efit {
cudaError_t xch_allreduce(Ctx& c, double* buf, size_t n, cudaStream_t s) {
    if (!c.comm) return cudaErrorInvalidValue;
    const ncclResult_t r = nccl_api().all_reduce(buf, buf, n, ncclFloat64, ncclSum, (ncclComm_t)c.comm, s);
    if (r != ncclSuccess) {
        c.nccl_err = (int)r;
        return cudaErrorUnknown;
    }
    return cudaSuccess;
}
}  // namespace efit

extern "C" int efit_nccl_unique_id(void* id_out) {
    if (!id_out) return fail(nullptr, EFIT_E_INVAL, "id_out is null");
    NcclApi& api = nccl_api();
    if (!api.ok) return fail(nullptr, EFIT_E_NCCL, "%s", api.why);
    ncclUniqueId id;
    const ncclResult_t r = api.get_unique_id(&id);
    if (r != ncclSuccess) return fail(nullptr, EFIT_E_NCCL, "ncclGetUniqueId: %s", api.error_string(r));
    std::memcpy(id_out, &id, sizeof(id));
    return EFIT_OK;
}

static inline long long round_up(long long x, long long m) { return (x + m - 1) / m * m; }

extern "C" void efit_shard(int32_t n, int32_t rank, int32_t world, int32_t* lo, int32_t* hi) {
    if (world < 1) world = 1;
    int32_t base = n / world, rem = n % world;
    int32_t l = rank * base + (rank < rem ? rank : rem);
    *lo = l;
    *hi = l + base + (rank < rem ? 1 : 0);
}

static bool finite_arr(const double* p, int n) {
    for (int i = 0; i < n; ++i)
        if (!std::isfinite(p[i])) return false;
    return true;
}

static int validate(const efit_grid* g, const efit_basis* b, const efit_geometry* geo, const efit_dist* d, int mode) {
    if (!g || !b || !geo) return fail(nullptr, EFIT_E_INVAL, "null grid/basis/geometry");
    if (g->nw < 3 || g->nh < 3 || g->nw > efit::kMaxN || g->nh > efit::kMaxN)
        return fail(nullptr, EFIT_E_INVAL, "grid size %dx%d outside [3, %d]", g->nw, g->nh, efit::kMaxN);
    int nm = g->nh - 1;
    if ((nm & (nm - 1)) != 0)
        return fail(nullptr, EFIT_E_INVAL, "nh-1 = %d must be a power of two (FFT-based interior solve)", nm);
    if (!(g->rmin > 0.0) || !(g->rmax > g->rmin) || !(g->zmax > g->zmin) || !std::isfinite(g->rmax) ||
        !std::isfinite(g->zmin) || !std::isfinite(g->zmax))
        return fail(nullptr, EFIT_E_INVAL, "need 0 < rmin < rmax and zmin < zmax (finite)");
    if (b->kind != 0 && b->kind != 1) return fail(nullptr, EFIT_E_INVAL, "basis kind %d", b->kind);
    if (b->n_pp < 0 || b->n_ff < 0 || b->n_pp + b->n_ff < 1 || b->n_pp + b->n_ff > efit::kMaxBasis)
        return fail(nullptr, EFIT_E_INVAL, "need 1 <= n_pp + n_ff <= %d", efit::kMaxBasis);
    if (b->kind == 1) {
        if (b->n_knots < 0 || b->n_knots > efit::kMaxKnots || (b->n_knots > 0 && !b->knots))
            return fail(nullptr, EFIT_E_INVAL, "spline: 0 <= n_knots <= %d", efit::kMaxKnots);
        if (b->n_pp != b->n_knots + 4 || b->n_ff != b->n_knots + 4)
            return fail(nullptr, EFIT_E_INVAL, "spline: n_pp = n_ff = n_knots + 4 required");
        for (int k = 0; k < b->n_knots; ++k) {
            double lo = k ? b->knots[k - 1] : 0.0;
            if (!(b->knots[k] > lo) || !(b->knots[k] < 1.0))
                return fail(nullptr, EFIT_E_INVAL, "spline knots must increase strictly inside (0,1)");
        }
    }
    if (geo->n_fl < 0 || geo->n_mp < 0 || geo->n_int < 0 || geo->n_fl + geo->n_mp + geo->n_int < 1)
        return fail(nullptr, EFIT_E_INVAL, "need at least one diagnostic");
    if (geo->n_fl + geo->n_mp + geo->n_int > efit::kLsqMaxRowsHost)
        return fail(nullptr, EFIT_E_INVAL, "at most %d diagnostics", efit::kLsqMaxRowsHost);
    if (geo->n_fl + geo->n_mp + geo->n_int < b->n_pp + b->n_ff)
        return fail(nullptr, EFIT_E_INVAL, "fewer diagnostics than basis functions");
    if ((geo->n_fl && (!geo->fl_r || !geo->fl_z)) || (geo->n_mp && (!geo->mp_r || !geo->mp_z || !geo->mp_ang)) ||
        (geo->n_int && (!geo->int_r || !geo->int_z)))
        return fail(nullptr, EFIT_E_INVAL, "null diagnostic array");
    if (geo->n_lim < 3 || !geo->lim_r || !geo->lim_z) return fail(nullptr, EFIT_E_INVAL, "limiter needs >= 3 vertices");
    if (!finite_arr(geo->fl_r, geo->n_fl) || !finite_arr(geo->fl_z, geo->n_fl) || !finite_arr(geo->mp_r, geo->n_mp) ||
        !finite_arr(geo->mp_z, geo->n_mp) || !finite_arr(geo->mp_ang, geo->n_mp) ||
        !finite_arr(geo->int_r, geo->n_int) || !finite_arr(geo->int_z, geo->n_int) ||
        !finite_arr(geo->lim_r, geo->n_lim) || !finite_arr(geo->lim_z, geo->n_lim))
        return fail(nullptr, EFIT_E_INVAL, "non-finite geometry");
    for (int m = 0; m < geo->n_fl; ++m) if (!(geo->fl_r[m] > 0)) return fail(nullptr, EFIT_E_INVAL, "flux loop R <= 0");
    for (int m = 0; m < geo->n_mp; ++m) if (!(geo->mp_r[m] > 0)) return fail(nullptr, EFIT_E_INVAL, "probe R <= 0");
    for (int m = 0; m < geo->n_int; ++m) if (!(geo->int_r[m] > 0)) return fail(nullptr, EFIT_E_INVAL, "internal point R <= 0");
    if (geo->ip_sign != 1 && geo->ip_sign != -1) return fail(nullptr, EFIT_E_INVAL, "ip_sign must be +1 or -1");
    if (mode != EFIT_GREEN_TABLE && mode != EFIT_GREEN_ONTHEFLY && mode != EFIT_GREEN_TABLE_SYM &&
        mode != EFIT_GREEN_ONTHEFLY_SYM && mode != EFIT_GREEN_VONHAGENOW)
        return fail(nullptr, EFIT_E_INVAL, "mode %d", mode);
    if (mode == EFIT_GREEN_VONHAGENOW && d && d->world > 1)
        return fail(nullptr, EFIT_E_INVAL, "EFIT_GREEN_VONHAGENOW runs on one GPU (world == 1)");
    if (mode == EFIT_GREEN_VONHAGENOW && (g->nw < 4 || g->nh < 4))
        return fail(nullptr, EFIT_E_INVAL, "EFIT_GREEN_VONHAGENOW needs nw, nh >= 4");
    if (d && (d->world < 1 || d->rank < 0 || d->rank >= d->world))
        return fail(nullptr, EFIT_E_INVAL, "rank %d / world %d", d->rank, d->world);
    return EFIT_OK;
}

// Tiling + sharding plan (host logic; DESIGN.md §"Tiling").
static void plan(Ctx& c, const efit_grid* g, const efit_basis* b, const efit_geometry* geo, const efit_dist* d,
                 int mode) {
    c.nw = g->nw; c.nh = g->nh;
    c.rmin = g->rmin; c.rmax = g->rmax; c.zmin = g->zmin; c.zmax = g->zmax;
    c.dr = (g->rmax - g->rmin) / (double)(g->nw - 1);
    c.dz = (g->zmax - g->zmin) / (double)(g->nh - 1);
    c.kind = b->kind; c.n_pp = b->n_pp; c.n_ff = b->n_ff; c.nb = b->n_pp + b->n_ff;
    c.n_knots = b->kind == 1 ? b->n_knots : 0;
    for (int k = 0; k < efit::kMaxKnots; ++k) c.knots[k] = k < c.n_knots ? b->knots[k] : 1.0;
    c.n_fl = geo->n_fl; c.n_mp = geo->n_mp; c.n_int = geo->n_int;
    c.ndiag = geo->n_fl + geo->n_mp + geo->n_int;
    c.n_lim = geo->n_lim; c.ip_sign = geo->ip_sign;
    c.mode = mode;
    c.sym = mode == EFIT_GREEN_TABLE_SYM || mode == EFIT_GREEN_ONTHEFLY_SYM;
    c.otf = mode == EFIT_GREEN_ONTHEFLY || mode == EFIT_GREEN_ONTHEFLY_SYM;
    c.vh = mode == EFIT_GREEN_VONHAGENOW;
    c.rank = d ? d->rank : 0;
    c.world = d ? d->world : 1;
    c.n_edge = 2 * c.nh + 2 * (c.nw - 2);
    c.ni = c.nw - 2;
    c.ni_pad = 32 * ((c.ni + 31) / 32);  // segment-interleaved factor layout: 32 lanes x L rows
    c.fhat_ld = (c.ni + 3) / 4 * 4;
    c.nmode = c.nh - 2;
    c.fft_m = 2 * (c.nh - 1);
    c.fft_log2 = 0;
    while ((1 << c.fft_log2) < c.fft_m) ++c.fft_log2;
    const long long n = (long long)c.nw * c.nh;
    c.S = round_up(n, 64);
    efit::Tiling& t = c.t;
    {
        // response chunk: a multiple of 128 nodes (the permuted shared layout), at most the size
        // whose NB x gc basis slice keeps 2 CTAs per SM, chosen to minimise the busiest CTA slot's
        // nodes (ceil(chunks / 296 slots) x gc): one CTA wave without a partial tail where possible
        const int gc_max = c.nb <= 8 ? 1152 : (c.nb <= 16 ? 768 : 512);
        const long long slots = 2LL * efit::kNumSMs;
        long long best = -1;
        for (int gc = 256; gc <= gc_max; gc += 128) {
            const long long nch = (n + gc - 1) / gc;
            const long long cost = (nch + slots - 1) / slots * gc;
            if (best < 0 || cost <= best) { best = cost; t.resp_gc = gc; }  // ties -> larger chunks
        }
    }
    if (const char* ev = getenv("EFIT_RESP_GC")) {  // tuning override (multiple of 128)
        const int g = atoi(ev);
        if (g >= 128 && g % 128 == 0 && g <= 1152) t.resp_gc = g;
    }
    t.resp_nchunk = (int)((n + t.resp_gc - 1) / t.resp_gc);
    c.tbb_nchunk = (int)((n + efit::kBatchCh - 1) / efit::kBatchCh);
    c.respb_nchunk = (int)((n + efit::kRespBatchGc - 1) / efit::kRespBatchGc);
    c.respb = false;
    // single-slice response on the DMMA kernel: for wide bases (nb >= 8: the scalar kernel's nb
    // accumulators per row limit its loads in flight; measured 117 -> 48 us at C3, nb = 20) and
    // ~129^2 grids (C2: 18.0 -> 15.5 us); the scalar stream stays at 65^2 (C1: 13.1 vs 14.7 us) and at
    // 257^2+ with narrow bases (C4: 58 vs 66 us).  EFIT_RESP_MMA=1 / =0 forces either.
    {
        const char* ev = getenv("EFIT_RESP_MMA");
        const long long nn = (long long)c.nw * c.nh;
        const bool want = ev ? ev[0] != '0' : (c.nb >= 8 || (nn > 96LL * 96LL && nn <= 160LL * 160LL));
        c.resp_mma = c.nb <= 8 * efit::kRespBatchMaxBlk && want;
    }
    c.resp_fuse = getenv("EFIT_RESP_NOFUSE") == nullptr;
    t.tb_ch = 2048;
    t.tb_nchunk = (int)((n + t.tb_ch - 1) / t.tb_ch);
    t.tb_gi = 8;
    t.lr_jt = c.nh <= 96 ? 3 : (c.nh <= 160 ? 5 : (c.nh <= 288 ? 9 : 17));
    // left/right nest: the direct Toeplitz kernel on small grids (one launch; measured +10 % it/s at
    // 65^2), the FFT chain from nh > 96 (EFIT_LR_DIRECT=1 / EFIT_LR_FFT=1 force either)
    c.lr_direct = getenv("EFIT_LR_DIRECT") != nullptr || (c.nh <= 96 && getenv("EFIT_LR_FFT") == nullptr);
    c.lr_ldi = (c.nw + 3) / 4 * 4;
    // the FFT path computes all left/right targets at once: a single "tile"
    t.lr_njt = c.lr_direct ? (c.nh + 32 * t.lr_jt - 1) / (32 * t.lr_jt) : 1;
    t.lr_iib = 2;
    t.lr_nblk = (c.nw + t.lr_iib - 1) / t.lr_iib;
    {
        const int q = (c.nh + 3) / 4;  // sources per warp (one quarter), multiple of lr_jt
        t.lr_jj = (q + t.lr_jt - 1) / t.lr_jt * t.lr_jt;
    }
    t.red_blocks = 592;  // 4 per SM: enough loads in flight for the psi scans
    // shards: response rows and top/bottom target rows (full table) or row-pair tiles (SYM); every
    // exchanged slot has exactly one writer => bitwise identical results for any world size
    int lo, hi;
    efit_shard(c.ndiag, c.rank, c.world, &lo, &hi);
    c.m_lo = lo; c.m_hi = hi;
    efit_shard(c.nw - 2, c.rank, c.world, &lo, &hi);
    c.i_lo = 1 + lo; c.i_hi = 1 + hi;
    // left/right targets: replicated on every rank (an FP64-bound chain under the table stream; the
    // interior solve's overlapped forward DST needs them locally)
    c.jt_lo = 0; c.jt_hi = t.lr_njt;
    // SYM modes: row-pair tiles of 8 x 8 interior rows; the tiles (not the targets) are sharded
    c.sym_nblk = (c.ni + 7) / 8;
    c.sym_ntile = (long long)c.sym_nblk * (c.sym_nblk + 1) / 2;
    {
        const long long base = c.sym_ntile / c.world, rem = c.sym_ntile % c.world;
        c.sym_tile_lo = c.rank * base + (c.rank < rem ? c.rank : rem);
        c.sym_tile_hi = c.sym_tile_lo + base + (c.rank < rem ? 1 : 0);
    }
    // one chunk (F read mirrored from the staged I: 128 nh B of staging) up to nh = 576, else
    // chunks of <= 440 values with I and F staged (256 mc B): 3 CTAs per SM either way
    t.sym_nmc = c.nh <= 576 ? 1 : (c.nh + 439) / 440;
    t.sym_mc = ((c.nh + t.sym_nmc - 1) / t.sym_nmc + 1) / 2 * 2;  // even: 16-byte chunk starts
    c.nhp = (c.nh + 1) / 2 * 2;
    t.tb_ngroup = (c.i_hi - c.i_lo + t.tb_gi - 1) / t.tb_gi;
    if (t.tb_ngroup < 1) t.tb_ngroup = 1;
    // response rows per warp block: fewest rows on the busiest warp, registers MB*NB <= 40
    const int nrows = c.m_hi - c.m_lo;
    // a CTA covers 8*MB rows (one MB-row block per warp); pick MB (<= 5, MB*NB <= 40 registers'
    // worth of accumulators) minimising padded rows, then preferring more rows per warp
    int best_mb = 1, best_cost = 1 << 30;
    for (int mb = 4; mb >= 1; --mb) {  // ties -> more rows per warp (more reuse of each basis value)
        const int np = efit::resp_np(c.nb, mb);                // register-ring depth (k_response)
        if (4 * np * mb + mb * c.nb > 56 && mb > 1) continue;  // ring + accumulators (no spills)
        const int nmb = (nrows + mb - 1) / mb;        // row blocks, dealt round-robin to 8 warps
        int cost = ((nmb + 7) / 8) * mb;               // rows on the busiest warp
        if (cost < best_cost) { best_cost = cost; best_mb = mb; }
    }
    t.resp_mb = best_mb;
    if (const char* ev = getenv("EFIT_RESP_MB")) {  // tuning override (1..4)
        const int mb = atoi(ev);
        if (mb >= 1 && mb <= 4) t.resp_mb = mb;
    }
}

// Per-iteration scratch (also the whole of a batch slice context).  batch: tb_part sized for the
// k_bnd_tb_mma chunks.
template <typename Take>
static size_t carve_scratch(Ctx& c, Take& take, size_t& off, bool batch) {
    const long long n = (long long)c.nw * c.nh;
    const int nrows = c.m_hi - c.m_lo;
    c.axbd = (double*)take(sizeof(double) * 2);
    c.status = (int*)take(sizeof(int) * 4);
    c.tickets = (unsigned*)take(sizeof(unsigned) * 8);
    c.norm_part = (double*)take(sizeof(double) * 2 * (size_t)(c.t.red_blocks > c.ni + 2 ? c.t.red_blocks : c.ni + 2));
    const int rchunk = (batch || c.resp_mma) && c.respb_nchunk > c.t.resp_nchunk ? c.respb_nchunk : c.t.resp_nchunk;
    c.resp_part = (double*)take(sizeof(double) * (size_t)rchunk * (nrows > 0 ? nrows : 1) * c.nb);
    c.resp_cnt = (double*)take(sizeof(double) * c.t.resp_nchunk);
    c.bmat = (double*)take(sizeof(double) * (size_t)c.nb * c.t.resp_nchunk * c.t.resp_gc);
    c.resp = (double*)take(sizeof(double) * (size_t)c.ndiag * c.nb);
    c.coef = (double*)take(sizeof(double) * 32);
    c.chi2 = (double*)take(sizeof(double) * 4);
    c.pcurr = (double*)take(sizeof(double) * (size_t)round_up(n, c.t.tb_ch));
    c.pflip = (double*)take(sizeof(double) * (size_t)round_up(n, c.t.tb_ch));
    c.tb_part = (double*)take(sizeof(double) * (size_t)(batch ? c.tbb_nchunk : c.t.tb_nchunk) * c.nw * 2);
    c.lr_part = (double*)take(sizeof(double) * (size_t)c.t.lr_nblk * 2 * c.nh);
    c.lr_xh = (double2*)take(sizeof(double2) * (size_t)c.nh * c.lr_ldi);
    c.lr_y = (double2*)take(sizeof(double2) * 2 * (size_t)c.nh);
    c.psib = (double*)take(sizeof(double) * c.n_edge);
    c.fhat = (double*)take(sizeof(double) * (size_t)c.fhat_ld * c.nmode);
    c.psip = (double*)take(sizeof(double) * (size_t)n);
    c.eps_part = (double*)take(sizeof(double) * ((c.ni + 1) / 2 + 2));
    c.sym_edge = c.sym ? (double*)take(sizeof(double) * 2 * (size_t)(c.nw > 2 ? c.nw - 2 : 1)) : nullptr;
    c.vh_psi0 = c.vh ? (double*)take(sizeof(double) * (size_t)n) : nullptr;
    c.vh_src = c.vh ? (double*)take(sizeof(double) * ((c.n_edge + 3) / 4 * 4)) : nullptr;
    c.zero_edge = c.vh ? (double*)take(sizeof(double) * ((c.n_edge + 3) / 4 * 4)) : nullptr;
    // full steps_ (f3): always carved (efit_set_steps switches without a new workspace)
    c.pmask = (uint8_t*)take((size_t)n);
    c.st_info = (double*)take(sizeof(double) * 16);
    c.st_cnt = (unsigned*)take(sizeof(unsigned) * 4);
    c.st_cand = (double2*)take(sizeof(double2) * (size_t)efit::steps_cand_cap(c.nw, c.nh));
    c.st_bits = (uint64_t*)take(sizeof(uint64_t) * (size_t)c.nw * efit::steps_words(c.nh));
    return (size_t)round_up((long long)off, 256);
}

// Carve the workspace (base == nullptr: sizing only).  Returns total bytes.
static size_t carve(Ctx& c, char* base) {
    size_t off = 0;
    auto take = [&](size_t bytes) -> char* {
        off = (size_t)round_up((long long)off, 256);
        char* p = base ? base + off : nullptr;
        off += bytes;
        return p;
    };
    const long long n = (long long)c.nw * c.nh;
    const int nrows = c.m_hi - c.m_lo;
    const int nslab = c.i_hi - c.i_lo;
    c.T = (c.mode == EFIT_GREEN_TABLE && nslab > 0) ? (double*)take(sizeof(double) * (size_t)nslab * c.S) : nullptr;
    const long long ntile_rank = c.sym_tile_hi - c.sym_tile_lo;
    c.U = (c.mode == EFIT_GREEN_TABLE_SYM && ntile_rank > 0)
              ? (double*)take(sizeof(double) * 64 * (size_t)c.nh * (size_t)ntile_rank) : nullptr;
    c.symq = c.sym ? (double*)take(sizeof(double) * 16 * (size_t)c.sym_nblk * c.nh) : nullptr;
    c.symp = c.sym ? (double*)take(sizeof(double) * 16 * (size_t)c.sym_nblk * c.nhp) : nullptr;
    c.sym_part = c.sym ? (double*)take(sizeof(double) * 2 * (size_t)(c.ni > 0 ? c.ni : 1) * c.sym_nblk * c.t.sym_nmc)
                       : nullptr;
    c.Tedge = (double*)take(sizeof(double) * 2 * (size_t)c.S);
    c.Kvh = c.vh ? (double*)take(sizeof(double) * (size_t)c.n_edge * ((c.n_edge + 3) / 4 * 4)) : nullptr;
    c.Gd = (double*)take(sizeof(double) * (size_t)(nrows > 0 ? nrows : 1) * c.S);
    c.inlim = (uint8_t*)take((size_t)n);
    c.dgeo = (double*)take(sizeof(double) * 4 * c.ndiag);
    c.dkind = (int*)take(sizeof(int) * c.ndiag);
    c.lim = (double*)take(sizeof(double) * 2 * c.n_lim);
    c.tri_a = (double*)take(sizeof(double) * c.ni);
    c.tri_cp = (double*)take(sizeof(double) * (size_t)c.ni_pad * c.nmode);
    c.tri_inv = (double*)take(sizeof(double) * (size_t)c.ni_pad * c.nmode);
    c.tri_alpha = (double*)take(sizeof(double) * (size_t)c.ni_pad * c.nmode);
    c.twiddle = (double2*)take(sizeof(double2) * (size_t)(c.fft_m / 2));
    c.sin_tab = (double*)take(sizeof(double) * (size_t)c.nmode);
    c.lr_spec = (double*)take(sizeof(double) * 2 * (size_t)c.nh * c.lr_ldi);
    for (int b = 0; b < 2; ++b) {  // efit_fit_host staging slots
        c.hslot[b].psi = (double*)take(sizeof(double) * (size_t)n);
        c.hslot[b].meas = (double*)take(sizeof(double) * c.ndiag);
        c.hslot[b].sigma = (double*)take(sizeof(double) * c.ndiag);
        c.hslot[b].coef = (double*)take(sizeof(double) * 32);
        c.hslot[b].chi2 = (double*)take(sizeof(double) * 2);
        c.hslot[b].eps = (double*)take(sizeof(double) * 2);
    }
    return carve_scratch(c, take, off, false);
}

// Captured graphs keep the priorities of the streams their kernels were enqueued on: the left/right
// chain and the forward DST run on the high-priority side stream so that their CTAs are placed
// between the waves of the table stream (without this flag every node takes the launch stream's
// priority and the side chain is starved: 196 instead of 179 us per C4 iteration).
static constexpr unsigned long long kGraphFlags = cudaGraphInstantiateFlagUseNodePriority;

static bool aligned16(const void* p) { return ((uintptr_t)p & 15u) == 0; }

extern "C" int efit_workspace_bytes(const efit_grid* grid, const efit_basis* basis, const efit_geometry* geom,
                                    const efit_dist* dist, int mode, size_t* bytes_out) {
    int st = validate(grid, basis, geom, dist, mode);
    if (st) return st;
    if (!bytes_out) return fail(nullptr, EFIT_E_INVAL, "bytes_out is null");
    Ctx* c = new (std::nothrow) Ctx();
    if (!c) return fail(nullptr, EFIT_E_NOMEM, "host allocation");
    plan(*c, grid, basis, geom, dist, mode);
    *bytes_out = carve(*c, nullptr);
    delete c;
    return EFIT_OK;
}

extern "C" int efit_green_init(efit_ctx** out, const efit_grid* grid, const efit_basis* basis,
                               const efit_geometry* geom, const efit_dist* dist, int mode, void* d_workspace,
                               size_t ws_bytes, efit_stream_t stream) {
    if (!out) return fail(nullptr, EFIT_E_INVAL, "out is null");
    *out = nullptr;
    int st = validate(grid, basis, geom, dist, mode);
    if (st) return st;
    if (!d_workspace || ((uintptr_t)d_workspace & 255u))
        return fail(nullptr, EFIT_E_INVAL, "workspace must be non-null and 256-byte aligned");
    efit_ctx* h = new (std::nothrow) efit_ctx();
    if (!h) return fail(nullptr, EFIT_E_NOMEM, "host allocation");
    Ctx& c = h->c;
    plan(c, grid, basis, geom, dist, mode);
    size_t need = carve(c, nullptr);
    if (ws_bytes < need) {
        delete h;
        return fail(nullptr, EFIT_E_NOMEM, "workspace %zu bytes < required %zu", ws_bytes, need);
    }
    c.ws_bytes = carve(c, (char*)d_workspace);
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e = cudaGetDevice(&c.device);
    if (e) { delete h; return cuda_fail(nullptr, e, "cudaGetDevice"); }
    cudaPointerAttributes pa;
    e = cudaPointerGetAttributes(&pa, d_workspace);
    if (e || pa.type != cudaMemoryTypeDevice) {
        cudaGetLastError();
        delete h;
        return fail(nullptr, EFIT_E_INVAL, "workspace is not device memory");
    }
    // geometry to the device
    std::vector<double> dgeo(4 * (size_t)c.ndiag);
    std::vector<int> dkind(c.ndiag);
    int m = 0;
    for (int k = 0; k < geom->n_fl; ++k, ++m) {
        dgeo[4 * m] = geom->fl_r[k]; dgeo[4 * m + 1] = geom->fl_z[k]; dgeo[4 * m + 2] = 0; dgeo[4 * m + 3] = 0; dkind[m] = 0;
    }
    for (int k = 0; k < geom->n_mp; ++k, ++m) {
        dgeo[4 * m] = geom->mp_r[k]; dgeo[4 * m + 1] = geom->mp_z[k];
        dgeo[4 * m + 2] = std::cos(geom->mp_ang[k]); dgeo[4 * m + 3] = std::sin(geom->mp_ang[k]); dkind[m] = 1;
    }
    for (int k = 0; k < geom->n_int; ++k, ++m) {
        dgeo[4 * m] = geom->int_r[k]; dgeo[4 * m + 1] = geom->int_z[k]; dgeo[4 * m + 2] = 0; dgeo[4 * m + 3] = 0; dkind[m] = 2;
    }
    std::vector<double> lim(2 * (size_t)c.n_lim);
    for (int k = 0; k < c.n_lim; ++k) { lim[k] = geom->lim_r[k]; lim[c.n_lim + k] = geom->lim_z[k]; }
    if ((e = cudaMemcpyAsync(c.dgeo, dgeo.data(), sizeof(double) * dgeo.size(), cudaMemcpyHostToDevice, s)) ||
        (e = cudaMemcpyAsync(c.dkind, dkind.data(), sizeof(int) * dkind.size(), cudaMemcpyHostToDevice, s)) ||
        (e = cudaMemcpyAsync(c.lim, lim.data(), sizeof(double) * lim.size(), cudaMemcpyHostToDevice, s))) {
        delete h;
        return cuda_fail(nullptr, e, "geometry upload");
    }
    if ((e = efit::prepare_kernels(c)) || (e = efit::launch_init_tables(c, s)) || (e = cudaStreamSynchronize(s))) {
        delete h;
        return cuda_fail(nullptr, e, "table build");
    }
    c.side = nullptr; c.ev_fork = nullptr; c.ev_join = nullptr;
    int prio_lo = 0, prio_hi = 0;
    cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
    if ((e = cudaStreamCreateWithPriority(&c.side, cudaStreamNonBlocking, getenv("EFIT_SIDE_LOPRIO") ? prio_lo : prio_hi)) ||
        (e = cudaEventCreateWithFlags(&c.ev_fork, cudaEventDisableTiming)) ||
        (e = cudaEventCreateWithFlags(&c.ev_join, cudaEventDisableTiming))) {
        if (c.side) cudaStreamDestroy(c.side);
        if (c.ev_fork) cudaEventDestroy(c.ev_fork);
        delete h;
        return cuda_fail(nullptr, e, "side stream");
    }
    for (int k = 0; k < Ctx::kGraphCache; ++k) c.gexec[k] = nullptr;
    c.gnext = 0;
    c.hs = c.ds = nullptr;
    c.hstart = nullptr;
    for (int b = 0; b < 2; ++b) c.hin[b] = c.hdone[b] = c.hfree[b] = nullptr;
    c.hgexec[0] = c.hgexec[1] = nullptr;
    c.hgraph[0] = c.hgraph[1] = nullptr;
    c.hkey[0] = c.hkey[1] = nullptr;
    c.prof_on = false;
    c.prof_rec = false;
    c.prof_every = 1;
    c.prof_calls = 0;
    c.prof_capture = false;
    c.prof_ev = nullptr;
    c.prof_slots = c.prof_next = 0;
    c.pgraph = nullptr;
    c.pexec = nullptr;
    for (int id = 0; id < 16; ++id) c.prof_place[id] = nullptr;
    for (int id = 0; id < efit::kNumMarks; ++id) {
        if ((e = cudaEventCreate(&c.prof_place[id]))) {
            for (int q = 0; q < id; ++q) cudaEventDestroy(c.prof_place[q]);
            cudaStreamDestroy(c.side); cudaEventDestroy(c.ev_fork); cudaEventDestroy(c.ev_join);
            delete h;
            return cuda_fail(nullptr, e, "profile events");
        }
    }
    c.comm = nullptr;
    c.nccl_err = 0;
    if (dist && dist->nccl_id) {  // collective: every rank of the world calls efit_green_init
        NcclApi& api = nccl_api();
        if (!api.ok) {
            for (int id = 0; id < efit::kNumMarks; ++id) cudaEventDestroy(c.prof_place[id]);
            cudaStreamDestroy(c.side); cudaEventDestroy(c.ev_fork); cudaEventDestroy(c.ev_join);
            delete h;
            return fail(nullptr, EFIT_E_NCCL, "%s", api.why);
        }
        ncclUniqueId id;
        std::memcpy(&id, dist->nccl_id, sizeof(id));
        ncclComm_t comm = nullptr;
        const ncclResult_t r = api.comm_init_rank(&comm, c.world, id, c.rank);
        if (r != ncclSuccess) {
            for (int k = 0; k < efit::kNumMarks; ++k) cudaEventDestroy(c.prof_place[k]);
            cudaStreamDestroy(c.side); cudaEventDestroy(c.ev_fork); cudaEventDestroy(c.ev_join);
            delete h;
            return fail(nullptr, EFIT_E_NCCL, "ncclCommInitRank(world %d, rank %d): %s", c.world, c.rank,
                        api.error_string(r));
        }
        c.comm = comm;
    }
    c.use_graph = getenv("EFIT_NO_GRAPH") == nullptr;
    c.nslice = 0;
    for (int k = 0; k < efit::kMaxSlices; ++k) c.slice[k] = nullptr;
    c.shadow = false;
    c.bev_fork = c.bev_tb = c.bev_resp = nullptr;
    c.bexec = nullptr;
    c.err[0] = 0;
    *out = h;
    return EFIT_OK;
}

static void fill_info(const Ctx& c, efit_info_t* info) {
    info->nw = c.nw; info->nh = c.nh; info->ndiag = c.ndiag; info->nbasis = c.nb; info->n_edge = c.n_edge;
    info->mode = c.mode; info->rank = c.rank; info->world = c.world;
    info->resp_row_lo = c.m_lo; info->resp_row_hi = c.m_hi;
    info->bnd_row_lo = c.i_lo; info->bnd_row_hi = c.i_hi;
    info->lr_blk_lo = c.jt_lo; info->lr_blk_hi = c.jt_hi;
    const int tile = c.lr_direct ? 32 * c.t.lr_jt : c.nh;  // FFT mode: one tile holds every j
    info->lr_j_lo = c.jt_lo * tile < c.nh ? c.jt_lo * tile : c.nh;
    info->lr_j_hi = c.jt_hi * tile < c.nh ? c.jt_hi * tile : c.nh;
    info->slab_stride = c.S;
    info->sym_nblk = c.sym_nblk;
    info->sym_tile_lo = (int32_t)c.sym_tile_lo;
    info->sym_tile_hi = (int32_t)c.sym_tile_hi;
    info->xbuf_len = c.sym ? 2LL * c.ni * c.sym_nblk * c.t.sym_nmc : 2LL * (c.nw - 2);
    info->exchange = c.comm ? 1 : 0;
    info->workspace_bytes = c.ws_bytes;
}

extern "C" int efit_plan_info(const efit_grid* grid, const efit_basis* basis, const efit_geometry* geom,
                              const efit_dist* dist, int mode, efit_info_t* info) {
    int st = validate(grid, basis, geom, dist, mode);
    if (st) return st;
    if (!info) return fail(nullptr, EFIT_E_INVAL, "info is null");
    Ctx* c = new (std::nothrow) Ctx();
    if (!c) return fail(nullptr, EFIT_E_NOMEM, "host allocation");
    plan(*c, grid, basis, geom, dist, mode);
    c->ws_bytes = carve(*c, nullptr);
    fill_info(*c, info);
    delete c;
    return EFIT_OK;
}

extern "C" int efit_info(const efit_ctx* h, efit_info_t* info) {
    if (!h || !info) return fail(nullptr, EFIT_E_INVAL, "null argument");
    fill_info(h->c, info);
    return EFIT_OK;
}

#define EFIT_CHECK_PTR(c, p, name)                                                                  \
    do {                                                                                            \
        if (!(p)) return fail(&(c), EFIT_E_INVAL, "%s is null", name);                              \
        if (!aligned16(p)) return fail(&(c), EFIT_E_INVAL, "%s is not 16-byte aligned", name);      \
    } while (0)

extern "C" int efit_response(efit_ctx* h, const double* d_psi, double* d_resp, double* d_axbd,
                             efit_stream_t stream) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    EFIT_CHECK_PTR(c, d_psi, "d_psi");
    EFIT_CHECK_PTR(c, d_resp, "d_resp");
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e;
    if ((e = efit::launch_normalize(c, d_psi, s))) return cuda_fail(&c, e, "normalize");
    const size_t nresp = (size_t)c.ndiag * c.nb;
    if (c.comm && c.world > 1 && (e = cudaMemsetAsync(d_resp, 0, sizeof(double) * nresp, s)))
        return cuda_fail(&c, e, "response clear");
    if ((e = efit::launch_response(c, d_psi, d_resp + (size_t)c.m_lo * c.nb, s))) return cuda_fail(&c, e, "response");
    if (c.comm && (e = efit::xch_allreduce(c, d_resp, nresp, s))) return cuda_fail(&c, e, "response exchange");
    if (d_axbd && (e = cudaMemcpyAsync(d_axbd, c.axbd, 2 * sizeof(double), cudaMemcpyDeviceToDevice, s)))
        return cuda_fail(&c, e, "axbd copy");
    return EFIT_OK;
}

// cached fit-step graphs were captured for one normalisation rule: drop them when it changes
static void drop_fit_graphs(Ctx& c) {
    for (int k = 0; k < Ctx::kGraphCache; ++k)
        if (c.gexec[k]) { cudaGraphExecDestroy(c.gexec[k]); c.gexec[k] = nullptr; }
    for (int b = 0; b < 2; ++b) {
        if (c.hgexec[b]) { cudaGraphExecDestroy(c.hgexec[b]); c.hgexec[b] = nullptr; }
        if (c.hgraph[b]) { cudaGraphDestroy(c.hgraph[b]); c.hgraph[b] = nullptr; }
    }
    c.hkey[0] = c.hkey[1] = nullptr;
}

extern "C" int efit_set_steps(efit_ctx* h, int32_t steps_mode) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    if (steps_mode != EFIT_STEPS_LIMITER && steps_mode != EFIT_STEPS_FULL)
        return fail(&c, EFIT_E_INVAL, "steps_mode must be EFIT_STEPS_LIMITER or EFIT_STEPS_FULL");
    if (steps_mode == EFIT_STEPS_FULL) {
        int optin = 0;
        cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, c.device);
        if (c.nw < 6 || c.nh < 6 || efit::steps_words(c.nh) > 32 || efit::steps_fill_smem(c.nw, c.nh, nullptr) > (size_t)optin)
            return fail(&c, EFIT_E_INVAL, "EFIT_STEPS_FULL needs 6 <= nw, nh and a plasma bitmap in shared memory (nw*nh <= ~1025^2)");
    }
    if (c.steps != steps_mode) {
        drop_fit_graphs(c);
        if (c.bexec) { cudaGraphExecDestroy(c.bexec); c.bexec = nullptr; }
    }
    c.steps = steps_mode;
    for (int k = 0; k < c.nslice; ++k) c.slice[k]->steps = steps_mode;  // batch slices normalise alike
    return EFIT_OK;
}

extern "C" int efit_normalize(efit_ctx* h, const double* d_psi, double* d_info, uint8_t* d_mask, efit_stream_t stream) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    EFIT_CHECK_PTR(c, d_psi, "d_psi");
    EFIT_CHECK_PTR(c, d_info, "d_info");
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e;
    if ((e = efit::launch_normalize(c, d_psi, s))) return cuda_fail(&c, e, "normalize");
    if (c.steps) {
        if ((e = cudaMemcpyAsync(d_info, c.st_info, 16 * sizeof(double), cudaMemcpyDeviceToDevice, s)))
            return cuda_fail(&c, e, "info copy");
        if (d_mask && (e = cudaMemcpyAsync(d_mask, c.pmask, (size_t)c.nw * c.nh, cudaMemcpyDeviceToDevice, s)))
            return cuda_fail(&c, e, "mask copy");
        return EFIT_OK;
    }
    // limiter rule: {psi_axis, psi_bdry}, kind 0, the rest NaN
    const double nan = __builtin_nan("");
    double hinfo[16];
    for (int k = 0; k < 16; ++k) hinfo[k] = nan;
    hinfo[12] = 0.0;
    if ((e = cudaMemcpyAsync(c.st_info, hinfo, sizeof(hinfo), cudaMemcpyHostToDevice, s)) ||
        (e = cudaMemcpyAsync(c.st_info, c.axbd, 2 * sizeof(double), cudaMemcpyDeviceToDevice, s)) ||
        (e = cudaMemcpyAsync(d_info, c.st_info, 16 * sizeof(double), cudaMemcpyDeviceToDevice, s)))
        return cuda_fail(&c, e, "info copy");
    if (d_mask && (e = efit::launch_mask_o8(c, d_psi, d_mask, s))) return cuda_fail(&c, e, "mask");
    return EFIT_OK;
}

extern "C" int efit_current(efit_ctx* h, const double* d_psi, const double* d_coef, double* d_pcurr,
                            efit_stream_t stream) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    EFIT_CHECK_PTR(c, d_psi, "d_psi");
    EFIT_CHECK_PTR(c, d_coef, "d_coef");
    EFIT_CHECK_PTR(c, d_pcurr, "d_pcurr");
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e;
    if ((e = efit::launch_normalize(c, d_psi, s))) return cuda_fail(&c, e, "normalize");
    if ((e = efit::launch_current(c, d_psi, d_coef, d_pcurr, false, s))) return cuda_fail(&c, e, "current");
    return EFIT_OK;
}

extern "C" int efit_boundary_flux(efit_ctx* h, const double* d_pcurr, double* d_psib, efit_stream_t stream) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    EFIT_CHECK_PTR(c, d_pcurr, "d_pcurr");
    EFIT_CHECK_PTR(c, d_psib, "d_psib");
    if (c.world > 1 && !c.comm)
        return fail(&c, EFIT_E_STATE, "world > 1 without NCCL exchange: use efit_boundary_partials/finish");
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e;
    if (c.vh) {  // the caller's current into the internal buffer, then the von Hagenow construction
        if ((e = cudaMemcpyAsync(c.pcurr, d_pcurr, sizeof(double) * (size_t)c.nw * c.nh, cudaMemcpyDeviceToDevice, s)) ||
            (e = efit::launch_boundary(c, c.pcurr, d_psib, s)))
            return cuda_fail(&c, e, "boundary (von Hagenow)");
        return EFIT_OK;
    }
    if ((e = efit::launch_make_pair(c, d_pcurr, s))) return cuda_fail(&c, e, "pair");
    if ((e = efit::launch_boundary(c, d_pcurr, d_psib, s, false, false, c.comm ? efit::XCH_NCCL : efit::XCH_NONE)))
        return cuda_fail(&c, e, "boundary");
    return EFIT_OK;
}

extern "C" int efit_boundary_partials(efit_ctx* h, const double* d_pcurr, double* d_xbuf, efit_stream_t stream) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    if (c.vh) return fail(&c, EFIT_E_STATE, "no exchange slices in EFIT_GREEN_VONHAGENOW mode");
    EFIT_CHECK_PTR(c, d_pcurr, "d_pcurr");
    EFIT_CHECK_PTR(c, d_xbuf, "d_xbuf");
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e;
    if ((e = efit::launch_make_pair(c, d_pcurr, s))) return cuda_fail(&c, e, "pair");
    if ((e = efit::launch_boundary(c, d_pcurr, nullptr, s, false, false, efit::XCH_PARTIALS, d_xbuf)))
        return cuda_fail(&c, e, "boundary partials");
    return EFIT_OK;
}

extern "C" int efit_boundary_finish(efit_ctx* h, const double* d_pcurr, const double* d_xbuf, double* d_psib,
                                    efit_stream_t stream) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    if (c.vh) return fail(&c, EFIT_E_STATE, "no exchange slices in EFIT_GREEN_VONHAGENOW mode");
    EFIT_CHECK_PTR(c, d_pcurr, "d_pcurr");
    EFIT_CHECK_PTR(c, d_xbuf, "d_xbuf");
    EFIT_CHECK_PTR(c, d_psib, "d_psib");
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e;
    if ((e = efit::launch_make_pair(c, d_pcurr, s))) return cuda_fail(&c, e, "pair");
    if ((e = efit::launch_boundary(c, d_pcurr, d_psib, s, false, false, efit::XCH_FINISH, const_cast<double*>(d_xbuf))))
        return cuda_fail(&c, e, "boundary finish");
    return EFIT_OK;
}

extern "C" int efit_interior_solve(efit_ctx* h, const double* d_pcurr, const double* d_psib, double* d_psi_p,
                                   efit_stream_t stream) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    EFIT_CHECK_PTR(c, d_pcurr, "d_pcurr");
    EFIT_CHECK_PTR(c, d_psib, "d_psib");
    EFIT_CHECK_PTR(c, d_psi_p, "d_psi_p");
    cudaError_t e = efit::launch_solve(c, d_pcurr, d_psib, d_psi_p, nullptr, nullptr, nullptr, (cudaStream_t)stream);
    if (e) return cuda_fail(&c, e, "interior solve");
    return EFIT_OK;
}

extern "C" int efit_lsq(efit_ctx* h, const double* d_resp, const double* d_meas, const double* d_sigma,
                        double* d_coef, double* d_chi2, efit_stream_t stream) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    EFIT_CHECK_PTR(c, d_resp, "d_resp");
    EFIT_CHECK_PTR(c, d_meas, "d_meas");
    EFIT_CHECK_PTR(c, d_sigma, "d_sigma");
    EFIT_CHECK_PTR(c, d_coef, "d_coef");
    EFIT_CHECK_PTR(c, d_chi2, "d_chi2");
    cudaError_t e = efit::launch_lsq(c, d_resp, d_meas, d_sigma, d_coef, d_chi2, (cudaStream_t)stream);
    if (e) return cuda_fail(&c, e, "lsq");
    return EFIT_OK;
}

namespace efit {
void mark(Ctx& c, cudaStream_t s, int id) {
    if (c.prof_capture) {  // building the profiled graph: external event-record node
        cudaEventRecordWithFlags(c.prof_place[id], s, cudaEventRecordExternal);
        return;
    }
    if (!c.prof_on || !c.prof_rec || c.prof_next >= c.prof_slots) return;
    cudaEvent_t ev = c.prof_ev[(size_t)c.prof_next * kNumMarks + id];
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    cudaStreamIsCapturing(s, &cs);
    if (cs == cudaStreamCaptureStatusActive) cudaEventRecordWithFlags(ev, s, cudaEventRecordExternal);
    else cudaEventRecord(ev, s);
}
}  // namespace efit

// One Picard iteration.  `normalize`: compute psi_axis/psi_bdry of psi first; otherwise they were
// produced by the previous chained iteration's k_dst_inv.  Every iteration's k_dst_inv produces the
// next axis/boundary (cheap: a per-block argmax over the nodes it writes + the last block).
static cudaError_t enqueue_fit_step(Ctx& c, double* psi, const double* psi_ext, const double* meas,
                                    const double* sigma, double* coef, double* chi2, double* eps, cudaStream_t s,
                                    bool normalize = true) {
    using namespace efit;
    cudaError_t e;
    c.prof_rec = c.prof_on && (c.prof_calls++ % c.prof_every == 0);
    mark(c, s, M_BEGIN);
    if ((normalize || c.steps) && (e = launch_normalize(c, psi, s))) return e;  // f3: steps_ every iteration
    mark(c, s, M_NORM);
    const size_t nresp = (size_t)c.ndiag * c.nb;
    if (c.comm && c.world > 1 && (e = cudaMemsetAsync(c.resp, 0, sizeof(double) * nresp, s))) return e;
    if ((e = launch_response(c, psi, c.resp + (size_t)c.m_lo * c.nb, s))) return e;
    if (c.comm && (e = xch_allreduce(c, c.resp, nresp, s))) return e;  // replicated response (exact sum)
    mark(c, s, M_RESP);
    if ((e = launch_lsq(c, c.resp, meas, sigma, coef, chi2, s))) return e;
    if ((e = launch_current(c, psi, coef, c.pcurr, !c.vh, s))) return e;  // + mirrored pair (table modes)
    mark(c, s, M_CUR);
    if (c.vh) {  // von Hagenow: zero-Dirichlet solve -> boundary operator -> the Dirichlet solve + update
        if ((e = launch_boundary(c, c.pcurr, c.psib, s))) return e;
        mark(c, s, M_LR);
        if ((e = launch_solve(c, c.pcurr, c.psib, nullptr, psi, psi_ext, eps, s, true))) return e;
        mark(c, s, M_SOLVE);
        if (c.prof_on && c.prof_rec && !c.prof_capture && c.prof_next < c.prof_slots) ++c.prof_next;
        c.prof_rec = false;
        return cudaSuccess;
    }
    // boundary flux (marks M_TB, M_LR inside); in FFT mode the forward DST (without the bottom/top
    // edge terms) runs on the side stream under k_bnd_tb and the tridiagonal solve adds those terms
    const bool overlap = !c.lr_direct;
    if ((e = launch_boundary(c, c.pcurr, c.psib, s, overlap, c.sym, c.comm ? XCH_NCCL : XCH_NONE))) return e;
    if (!overlap && (e = launch_solve_fwd(c, c.pcurr, c.psib, s, 1))) return e;
    if ((e = launch_solve_rest(c, c.psib, nullptr, psi, psi_ext, eps, s, true, overlap))) return e;
    mark(c, s, M_SOLVE);
    if (c.prof_on && c.prof_rec && !c.prof_capture && c.prof_next < c.prof_slots) ++c.prof_next;
    c.prof_rec = false;
    return cudaSuccess;
}

static int fit_steps_impl(efit_ctx* h, int32_t nsteps, double* d_psi, const double* d_psi_ext, const double* d_meas,
                          const double* d_sigma, double* d_coef, double* d_chi2, double* d_eps, efit_stream_t stream) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    if (c.world != 1 && !c.comm)
        return fail(&c, EFIT_E_STATE, "efit_fit_step(s) with world > 1 needs the NCCL exchange (efit_dist.nccl_id)");
    if (nsteps < 1) return fail(&c, EFIT_E_INVAL, "nsteps < 1");
    EFIT_CHECK_PTR(c, d_psi, "d_psi");
    EFIT_CHECK_PTR(c, d_psi_ext, "d_psi_ext");
    EFIT_CHECK_PTR(c, d_meas, "d_meas");
    EFIT_CHECK_PTR(c, d_sigma, "d_sigma");
    EFIT_CHECK_PTR(c, d_coef, "d_coef");
    EFIT_CHECK_PTR(c, d_chi2, "d_chi2");
    EFIT_CHECK_PTR(c, d_eps, "d_eps");
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e;
    auto enqueue = [&]() -> cudaError_t {
        for (int k = 0; k < nsteps; ++k) {
            cudaError_t e1 = enqueue_fit_step(c, d_psi, d_psi_ext, d_meas, d_sigma, d_coef, d_chi2, d_eps, s, k == 0);
            if (e1) return e1;
        }
        return cudaSuccess;
    };
    const void* key[9] = {d_psi, d_psi_ext, d_meas, d_sigma, d_coef, d_chi2, d_eps, (const void*)s,
                          (const void*)(intptr_t)nsteps};
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if (s != nullptr && (e = cudaStreamIsCapturing(s, &cs))) return cuda_fail(&c, e, "capture query");
    // eager enqueue when the caller is capturing the stream itself (the kernels then become nodes
    // of the caller's graph), when profiling, when graphs are disabled, or on the legacy stream
    if (!c.use_graph || s == nullptr || c.prof_on || cs == cudaStreamCaptureStatusActive) {
        if ((e = enqueue())) return cuda_fail(&c, e, "fit step");
        return EFIT_OK;
    }
    int slot = -1;
    for (int k = 0; k < Ctx::kGraphCache; ++k)
        if (c.gexec[k] && std::memcmp(key, c.gkey[k], sizeof(key)) == 0) slot = k;
    if (slot < 0) {
        slot = c.gnext;
        c.gnext = (c.gnext + 1) % Ctx::kGraphCache;
        if (c.gexec[slot]) { cudaGraphExecDestroy(c.gexec[slot]); c.gexec[slot] = nullptr; }
        cudaGraph_t graph = nullptr;
        if ((e = cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal))) return cuda_fail(&c, e, "begin capture");
        cudaError_t e2 = enqueue();
        e = cudaStreamEndCapture(s, &graph);
        if (e2) { if (graph) cudaGraphDestroy(graph); return cuda_fail(&c, e2, "fit step capture"); }
        if (e) return cuda_fail(&c, e, "end capture");
        e = cudaGraphInstantiateWithFlags(&c.gexec[slot], graph, kGraphFlags);
        cudaGraphDestroy(graph);
        if (e) { c.gexec[slot] = nullptr; return cuda_fail(&c, e, "graph instantiate"); }
        std::memcpy(c.gkey[slot], key, sizeof(key));
    }
    if ((e = cudaGraphLaunch(c.gexec[slot], s))) return cuda_fail(&c, e, "graph launch");
    return EFIT_OK;
}

extern "C" int efit_fit_step(efit_ctx* h, double* d_psi, const double* d_psi_ext, const double* d_meas,
                             const double* d_sigma, double* d_coef, double* d_chi2, double* d_eps,
                             efit_stream_t stream) {
    return fit_steps_impl(h, 1, d_psi, d_psi_ext, d_meas, d_sigma, d_coef, d_chi2, d_eps, stream);
}

extern "C" int efit_fit_steps(efit_ctx* h, int32_t nsteps, double* d_psi, const double* d_psi_ext,
                              const double* d_meas, const double* d_sigma, double* d_coef, double* d_chi2,
                              double* d_eps, efit_stream_t stream) {
    return fit_steps_impl(h, nsteps, d_psi, d_psi_ext, d_meas, d_sigma, d_coef, d_chi2, d_eps, stream);
}

// Pipelined host path (efit_fit_host): one graph launch per slice.  Graph b (slot b) = the chained
// fit of slot b's staging buffers, plus a parallel branch that downloads the previous slice's results
// from slot b^1 and then uploads the next slice's inputs into it; the branch's 7 copy nodes are
// re-pointed at the neighbouring slices' host arrays before every launch (and disabled at the ends).
// Returns EFIT_OK, 1 if the graphs cannot be built for these buffers (caller falls back to the stream
// pipeline), or an error code.
static int fit_host_graphs(efit_ctx* h, int32_t nslice, int32_t iters, const double* h_psi0, const double* h_meas,
                           const double* h_sigma, const double* d_psi_ext, double* h_psi, double* h_coef,
                           double* h_chi2, double* h_eps, cudaStream_t s) {
    Ctx& c = h->c;
    const size_t n = (size_t)c.nw * c.nh, nd = (size_t)c.ndiag, nb = (size_t)c.nb;
    cudaError_t e;
    const void* key0 = (const void*)(intptr_t)iters;
    if (!c.hgexec[0] || c.hkey[0] != key0 || c.hkey[1] != (const void*)d_psi_ext) {
        auto drop = [&c]() {
            for (int b = 0; b < 2; ++b) {
                if (c.hgexec[b]) { cudaGraphExecDestroy(c.hgexec[b]); c.hgexec[b] = nullptr; }
                if (c.hgraph[b]) { cudaGraphDestroy(c.hgraph[b]); c.hgraph[b] = nullptr; }
            }
        };
        drop();
        for (int b = 0; b < 2; ++b) {
            Ctx::HostSlot& q = c.hslot[b];
            Ctx::HostSlot& o = c.hslot[b ^ 1];
            cudaGraph_t g = nullptr;
            if ((e = cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal))) return cuda_fail(&c, e, "begin capture");
            cudaError_t e2 = cudaSuccess;
            for (int k = 0; k < iters && !e2; ++k)
                e2 = enqueue_fit_step(c, q.psi, d_psi_ext, q.meas, q.sigma, q.coef, q.chi2, q.eps, s, k == 0);
            e = cudaStreamEndCapture(s, &g);
            if (e2 || e) { if (g) cudaGraphDestroy(g); return cuda_fail(&c, e2 ? e2 : e, "host graph capture"); }
            // the copy branch: D2H of slot b^1 (roots), then H2D into it
            cudaGraphNode_t* nd7 = c.hnode[b];
            const bool ok =
                cudaGraphAddMemcpyNode1D(&nd7[0], g, nullptr, 0, h_psi, o.psi, sizeof(double) * n, cudaMemcpyDeviceToHost) == cudaSuccess &&
                cudaGraphAddMemcpyNode1D(&nd7[1], g, nullptr, 0, h_coef, o.coef, sizeof(double) * nb, cudaMemcpyDeviceToHost) == cudaSuccess &&
                cudaGraphAddMemcpyNode1D(&nd7[2], g, nullptr, 0, h_chi2, o.chi2, sizeof(double), cudaMemcpyDeviceToHost) == cudaSuccess &&
                cudaGraphAddMemcpyNode1D(&nd7[3], g, nullptr, 0, h_eps, o.eps, sizeof(double), cudaMemcpyDeviceToHost) == cudaSuccess &&
                cudaGraphAddMemcpyNode1D(&nd7[4], g, nd7, 4, o.psi, h_psi0, sizeof(double) * n, cudaMemcpyHostToDevice) == cudaSuccess &&
                cudaGraphAddMemcpyNode1D(&nd7[5], g, nd7, 4, o.meas, h_meas, sizeof(double) * nd, cudaMemcpyHostToDevice) == cudaSuccess &&
                cudaGraphAddMemcpyNode1D(&nd7[6], g, nd7, 4, o.sigma, h_sigma, sizeof(double) * nd, cudaMemcpyHostToDevice) == cudaSuccess &&
                cudaGraphInstantiateWithFlags(&c.hgexec[b], g, kGraphFlags) == cudaSuccess;
            c.hgraph[b] = g;
            if (!ok) {
                cudaGetLastError();
                drop();
                return 1;
            }
        }
        c.hkey[0] = key0;
        c.hkey[1] = (const void*)d_psi_ext;
    }
    // slice 0's inputs into slot 0
    Ctx::HostSlot& q0 = c.hslot[0];
    if ((e = cudaMemcpyAsync(q0.psi, h_psi0, sizeof(double) * n, cudaMemcpyHostToDevice, s)) ||
        (e = cudaMemcpyAsync(q0.meas, h_meas, sizeof(double) * nd, cudaMemcpyHostToDevice, s)) ||
        (e = cudaMemcpyAsync(q0.sigma, h_sigma, sizeof(double) * nd, cudaMemcpyHostToDevice, s)))
        return cuda_fail(&c, e, "H2D");
    for (int k = 0; k < nslice; ++k) {
        const int b = k & 1;
        Ctx::HostSlot& o = c.hslot[b ^ 1];
        cudaGraphExec_t x = c.hgexec[b];
        cudaGraphNode_t* nd7 = c.hnode[b];
        const bool dn = k >= 1, up = k + 1 < nslice;
        const size_t kp = dn ? (size_t)(k - 1) : 0, kn = up ? (size_t)(k + 1) : 0;
        struct { void* dst; const void* src; size_t bytes; cudaMemcpyKind kind; } cp[7] = {
            {h_psi + kp * n, o.psi, sizeof(double) * n, cudaMemcpyDeviceToHost},
            {h_coef + kp * nb, o.coef, sizeof(double) * nb, cudaMemcpyDeviceToHost},
            {h_chi2 + kp, o.chi2, sizeof(double), cudaMemcpyDeviceToHost},
            {h_eps + kp, o.eps, sizeof(double), cudaMemcpyDeviceToHost},
            {o.psi, h_psi0 + kn * n, sizeof(double) * n, cudaMemcpyHostToDevice},
            {o.meas, h_meas + kn * nd, sizeof(double) * nd, cudaMemcpyHostToDevice},
            {o.sigma, h_sigma + kn * nd, sizeof(double) * nd, cudaMemcpyHostToDevice}};
        for (int q = 0; q < 7; ++q)
            if ((e = cudaGraphExecMemcpyNodeSetParams1D(x, nd7[q], cp[q].dst, cp[q].src, cp[q].bytes, cp[q].kind)))
                return fail(&c, EFIT_E_CUDA, "host graph update: copy node %d of slice %d: %s", q, k, cudaGetErrorString(e));
        for (int q = 0; q < 7; ++q)
            if ((e = cudaGraphNodeSetEnabled(x, nd7[q], q < 4 ? dn : up)))
                return fail(&c, EFIT_E_CUDA, "host graph enable: node %d of slice %d: %s", q, k, cudaGetErrorString(e));
        if ((e = cudaGraphLaunch(x, s))) return cuda_fail(&c, e, "host graph launch");
    }
    // the last slice's results
    const size_t kl = (size_t)(nslice - 1);
    Ctx::HostSlot& ql = c.hslot[(nslice - 1) & 1];
    if ((e = cudaMemcpyAsync(h_psi + kl * n, ql.psi, sizeof(double) * n, cudaMemcpyDeviceToHost, s)) ||
        (e = cudaMemcpyAsync(h_coef + kl * nb, ql.coef, sizeof(double) * nb, cudaMemcpyDeviceToHost, s)) ||
        (e = cudaMemcpyAsync(h_chi2 + kl, ql.chi2, sizeof(double), cudaMemcpyDeviceToHost, s)) ||
        (e = cudaMemcpyAsync(h_eps + kl, ql.eps, sizeof(double), cudaMemcpyDeviceToHost, s)))
        return cuda_fail(&c, e, "D2H");
    return EFIT_OK;
}

// The host-buffer stream pipeline of one efit_fit_host call (fallback of the per-slice graphs).
// Staging slot k & 1: H2D of slice k on the copy stream hs (after slot k-2's results left on ds) ->
// the fit steps on s -> D2H on ds; so the copies of slices k+1 / k-1 overlap slice k's iterations.
static int fit_host_pipeline(efit_ctx* h, int32_t nslice, int32_t iters, const double* h_psi0, const double* h_meas,
                                     const double* h_sigma, const double* d_psi_ext, double* h_psi, double* h_coef,
                                     double* h_chi2, double* h_eps, cudaStream_t s) {
    Ctx& c = h->c;
    const size_t n = (size_t)c.nw * c.nh, nd = (size_t)c.ndiag, nb = (size_t)c.nb;
    cudaError_t e;
    if ((e = cudaEventRecord(c.hstart, s)) || (e = cudaStreamWaitEvent(c.hs, c.hstart, 0)) ||
        (e = cudaStreamWaitEvent(c.ds, c.hstart, 0)))
        return cuda_fail(&c, e, "host pipeline");
    for (int k = 0; k < nslice; ++k) {
        const int b = k & 1;
        Ctx::HostSlot& q = c.hslot[b];
        if (k >= 2 && (e = cudaStreamWaitEvent(c.hs, c.hfree[b], 0))) return cuda_fail(&c, e, "host pipeline");
        if ((e = cudaMemcpyAsync(q.psi, h_psi0 + k * n, sizeof(double) * n, cudaMemcpyHostToDevice, c.hs)) ||
            (e = cudaMemcpyAsync(q.meas, h_meas + k * nd, sizeof(double) * nd, cudaMemcpyHostToDevice, c.hs)) ||
            (e = cudaMemcpyAsync(q.sigma, h_sigma + k * nd, sizeof(double) * nd, cudaMemcpyHostToDevice, c.hs)) ||
            (e = cudaEventRecord(c.hin[b], c.hs)) || (e = cudaStreamWaitEvent(s, c.hin[b], 0)))
            return cuda_fail(&c, e, "host pipeline");
        const int st = fit_steps_impl(h, iters, q.psi, d_psi_ext, q.meas, q.sigma, q.coef, q.chi2, q.eps, s);
        if (st) return st;
        if ((e = cudaEventRecord(c.hdone[b], s)) || (e = cudaStreamWaitEvent(c.ds, c.hdone[b], 0)) ||
            (e = cudaMemcpyAsync(h_psi + k * n, q.psi, sizeof(double) * n, cudaMemcpyDeviceToHost, c.ds)) ||
            (e = cudaMemcpyAsync(h_coef + k * nb, q.coef, sizeof(double) * nb, cudaMemcpyDeviceToHost, c.ds)) ||
            (e = cudaMemcpyAsync(h_chi2 + k, q.chi2, sizeof(double), cudaMemcpyDeviceToHost, c.ds)) ||
            (e = cudaMemcpyAsync(h_eps + k, q.eps, sizeof(double), cudaMemcpyDeviceToHost, c.ds)) ||
            (e = cudaEventRecord(c.hfree[b], c.ds)))
            return cuda_fail(&c, e, "host pipeline");
    }
    for (int b = 0; b < 2 && b < nslice; ++b)
        if ((e = cudaStreamWaitEvent(s, c.hfree[(nslice - 1 - b) & 1], 0))) return cuda_fail(&c, e, "host pipeline");
    return EFIT_OK;
}
// Host-buffer pipeline: nslice successive reconstructions (time slices), each `iters` chained
// fit iterations, with their inputs read from and results written to HOST memory.  Staging slot
// k & 1: H2D of slice k on the copy stream hs (after slot k-2's results left on ds) -> the cached
// fit-step graph on `stream` -> D2H on ds; so the copies of slices k+1 / k-1 overlap slice k's step.
extern "C" int efit_fit_host(efit_ctx* h, int32_t nslice, int32_t iters, const double* h_psi0, const double* h_meas,
                             const double* h_sigma, const double* d_psi_ext, double* h_psi, double* h_coef,
                             double* h_chi2, double* h_eps, efit_stream_t stream) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    if (nslice < 1 || iters < 1) return fail(&c, EFIT_E_INVAL, "nslice and iters must be >= 1");
    if (!h_psi0 || !h_meas || !h_sigma || !h_psi || !h_coef || !h_chi2 || !h_eps)
        return fail(&c, EFIT_E_INVAL, "null host buffer");
    EFIT_CHECK_PTR(c, d_psi_ext, "d_psi_ext");
    if (c.world != 1 && !c.comm) return fail(&c, EFIT_E_STATE, "world > 1 needs the NCCL exchange");
    cudaStream_t s = (cudaStream_t)stream;
    if (s == nullptr) return fail(&c, EFIT_E_INVAL, "efit_fit_host needs a non-default stream");
    cudaError_t e;
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if ((e = cudaStreamIsCapturing(s, &cs))) return cuda_fail(&c, e, "capture query");
    if (cs != cudaStreamCaptureStatusNone) return fail(&c, EFIT_E_STATE, "efit_fit_host cannot be captured");
    if (!c.hs) {
        int lo = 0, hi = 0;
        cudaDeviceGetStreamPriorityRange(&lo, &hi);
        if ((e = cudaStreamCreateWithPriority(&c.hs, cudaStreamNonBlocking, hi)) ||
            (e = cudaStreamCreateWithPriority(&c.ds, cudaStreamNonBlocking, hi)) ||
            (e = cudaEventCreateWithFlags(&c.hstart, cudaEventDisableTiming)))
            return cuda_fail(&c, e, "host pipeline streams");
        for (int b = 0; b < 2; ++b)
            if ((e = cudaEventCreateWithFlags(&c.hin[b], cudaEventDisableTiming)) ||
                (e = cudaEventCreateWithFlags(&c.hdone[b], cudaEventDisableTiming)) ||
                (e = cudaEventCreateWithFlags(&c.hfree[b], cudaEventDisableTiming)))
                return cuda_fail(&c, e, "host pipeline events");
    }
    if (c.use_graph && !c.prof_on && getenv("EFIT_HOST_STREAMS") == nullptr) {
        const int st = fit_host_graphs(h, nslice, iters, h_psi0, h_meas, h_sigma, d_psi_ext, h_psi, h_coef, h_chi2,
                                       h_eps, s);
        if (st != 1) return st;  // 1: graphs not available for these buffers -> stream pipeline below
    }
    return fit_host_pipeline(h, nslice, iters, h_psi0, h_meas, h_sigma, d_psi_ext, h_psi, h_coef, h_chi2, h_eps, s);
}

// ------------------------------------------------------------------ multi-time-slice batch
// (EFIT reconstructs many time slices of a discharge with the same machine, P:L161;
// S slices share one pass over the top/bottom Green's table.)

static void release_slices(Ctx& c);

static size_t slice_bytes(const Ctx& c) {
    Ctx* tmp = new (std::nothrow) Ctx(c);
    if (!tmp) return 0;
    size_t off = 0;
    auto take = [&](size_t bytes) -> char* {
        off = (size_t)round_up((long long)off, 256);
        off += bytes;
        return nullptr;
    };
    size_t b = carve_scratch(*tmp, take, off, true);
    delete tmp;
    return b;
}

static int batch_check(Ctx& c, int32_t nslice) {
    if (c.shadow) return fail(&c, EFIT_E_STATE, "not a primary context");
    if (nslice < 1 || nslice > efit::kMaxSlices)
        return fail(&c, EFIT_E_INVAL, "nslice %d outside [1, %d]", nslice, efit::kMaxSlices);
    if (c.mode != EFIT_GREEN_TABLE) return fail(&c, EFIT_E_STATE, "batching needs mode EFIT_GREEN_TABLE");
    if (c.world != 1) return fail(&c, EFIT_E_STATE, "batching needs world == 1");
    return EFIT_OK;
}

extern "C" int efit_batch_workspace_bytes(const efit_ctx* h, int32_t nslice, size_t* bytes_out) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = const_cast<efit_ctx*>(h)->c;
    int st = batch_check(c, nslice);
    if (st) return st;
    if (!bytes_out) return fail(&c, EFIT_E_INVAL, "bytes_out is null");
    *bytes_out = (size_t)nslice * slice_bytes(c);
    return EFIT_OK;
}

extern "C" int efit_batch_attach(efit_ctx* h, int32_t nslice, void* d_workspace, size_t ws_bytes) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    int st = batch_check(c, nslice);
    if (st) return st;
    const size_t per = slice_bytes(c);
    if (!d_workspace || ((uintptr_t)d_workspace & 255u))
        return fail(&c, EFIT_E_INVAL, "batch workspace must be non-null and 256-byte aligned");
    if (ws_bytes < per * (size_t)nslice)
        return fail(&c, EFIT_E_NOMEM, "batch workspace %zu bytes < required %zu", ws_bytes, per * (size_t)nslice);
    cudaError_t e;
    if ((e = cudaDeviceSynchronize())) return cuda_fail(&c, e, "batch attach sync");
    release_slices(c);
    if ((e = cudaMemset(d_workspace, 0, per * (size_t)nslice))) return cuda_fail(&c, e, "batch workspace clear");
    if (!c.bev_fork && (e = cudaEventCreateWithFlags(&c.bev_fork, cudaEventDisableTiming))) return cuda_fail(&c, e, "event");
    if (!c.bev_tb && (e = cudaEventCreateWithFlags(&c.bev_tb, cudaEventDisableTiming))) return cuda_fail(&c, e, "event");
    if (!c.bev_resp && (e = cudaEventCreateWithFlags(&c.bev_resp, cudaEventDisableTiming))) return cuda_fail(&c, e, "event");
    int prio_lo = 0, prio_hi = 0;
    cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
    for (int k = 0; k < nslice; ++k) {
        Ctx* q = new (std::nothrow) Ctx(c);  // tables, tiling and constants shared with the primary
        if (!q) { release_slices(c); return fail(&c, EFIT_E_NOMEM, "host allocation"); }
        q->shadow = true;
        q->nslice = 0;
        for (int j = 0; j < efit::kMaxSlices; ++j) q->slice[j] = nullptr;
        for (int k = 0; k < Ctx::kGraphCache; ++k) q->gexec[k] = nullptr;
        q->hs = q->ds = nullptr;
        q->hgexec[0] = q->hgexec[1] = nullptr;
        q->hgraph[0] = q->hgraph[1] = nullptr;
        q->bexec = nullptr; q->pexec = nullptr; q->pgraph = nullptr;
        q->prof_on = q->prof_rec = q->prof_capture = false;
        q->prof_ev = nullptr;
        for (int j = 0; j < 16; ++j) q->prof_place[j] = nullptr;
        q->side = nullptr; q->ev_fork = q->ev_join = nullptr;
        q->comm = nullptr;  // slices never exchange (batching needs world == 1)
        c.slice[k] = q;
        char* base = (char*)d_workspace + per * (size_t)k;
        size_t off = 0;
        auto take = [&](size_t bytes) -> char* {
            off = (size_t)round_up((long long)off, 256);
            char* p = base + off;
            off += bytes;
            return p;
        };
        carve_scratch(*q, take, off, true);  // incl. the slice's own status word (a failing slice, e.g. a
                                             // pre-plasma time slice, never poisons the others)
        // slice streams at normal priority: the shared table pass (main stream) keeps its SMs while the
        // slices' latency-bound chains fill in (measured +1.7 % at S = 8 over high priority)
        const int prio = getenv("EFIT_BATCH_HIPRIO") ? prio_hi : prio_lo;
        if ((e = cudaStreamCreateWithPriority(&q->side, cudaStreamNonBlocking, prio)) ||
            (e = cudaEventCreateWithFlags(&q->ev_fork, cudaEventDisableTiming)) ||
            (e = cudaEventCreateWithFlags(&q->ev_join, cudaEventDisableTiming))) {
            release_slices(c);
            return cuda_fail(&c, e, "slice stream");
        }
    }
    c.nslice = nslice;
    c.respb = efit::response_batch_ok(c, nslice) && getenv("EFIT_NO_RESP_BATCH") == nullptr;
    return EFIT_OK;
}

// One Picard iteration of every slice.  Slice k runs its own chain on its stream (normalise,
// response, LSQ, current, left/right FFT chain + forward DST); the shared table pass (k_bnd_tb_mma)
// joins all slices' currents; then each slice reduces its boundary and finishes its solve.
static cudaError_t enqueue_fit_step_batch(Ctx& c, double* psi, const double* psi_ext, const double* meas,
                                          const double* sigma, double* coef, double* chi2, double* eps,
                                          cudaStream_t s, bool normalize) {
    using namespace efit;
    cudaError_t e;
    const size_t n = (size_t)c.nw * c.nh;
    if ((e = cudaEventRecord(c.bev_fork, s))) return e;
    if (c.respb) {  // every slice's basis matrix, then one pass over Gd for all slices
        for (int k = 0; k < c.nslice; ++k) {
            Ctx& q = *c.slice[k];
            cudaStream_t sk = q.side;
            double* pk = psi + k * n;
            if ((e = cudaStreamWaitEvent(sk, c.bev_fork, 0))) return e;
            if ((normalize || q.steps) && (e = launch_normalize(q, pk, sk))) return e;  // f3: every iteration
            if ((e = launch_basis(q, pk, sk))) return e;
            if ((e = cudaEventRecord(q.ev_join, sk))) return e;
        }
        for (int k = 0; k < c.nslice; ++k)
            if ((e = cudaStreamWaitEvent(s, c.slice[k]->ev_join, 0))) return e;
        if ((e = launch_response_batch(c, c.nslice, c.slice, s))) return e;
        if ((e = cudaEventRecord(c.bev_resp, s))) return e;
    }
    for (int k = 0; k < c.nslice; ++k) {
        Ctx& q = *c.slice[k];
        cudaStream_t sk = q.side;
        double* pk = psi + k * n;
        if (c.respb) {
            if ((e = cudaStreamWaitEvent(sk, c.bev_resp, 0))) return e;
            if ((e = launch_resp_reduce_batch(q, c.respb_nchunk, q.resp, sk))) return e;
        } else {
            if ((e = cudaStreamWaitEvent(sk, c.bev_fork, 0))) return e;
            if ((normalize || q.steps) && (e = launch_normalize(q, pk, sk))) return e;
            if ((e = launch_response(q, pk, q.resp, sk))) return e;
        }
        if ((e = launch_lsq(q, q.resp, meas + (size_t)k * c.ndiag, sigma + (size_t)k * c.ndiag, coef + (size_t)k * c.nb,
                            chi2 + k, sk)))
            return e;
        if ((e = launch_current(q, pk, coef + (size_t)k * c.nb, q.pcurr, true, sk))) return e;
        if ((e = cudaEventRecord(q.ev_fork, sk))) return e;  // this slice's current pair is ready
        if ((e = launch_lr_fft(q, q.psib, sk))) return e;
        if ((e = launch_solve_fwd(q, q.pcurr, q.psib, sk, 2))) return e;
    }
    for (int k = 0; k < c.nslice; ++k)
        if ((e = cudaStreamWaitEvent(s, c.slice[k]->ev_fork, 0))) return e;
    if ((e = launch_boundary_batch(c, c.nslice, c.slice, s))) return e;
    if ((e = cudaEventRecord(c.bev_tb, s))) return e;
    for (int k = 0; k < c.nslice; ++k) {
        Ctx& q = *c.slice[k];
        cudaStream_t sk = q.side;
        if ((e = cudaStreamWaitEvent(sk, c.bev_tb, 0))) return e;
        if ((e = launch_bnd_reduce(q, q.tb_part, c.tbb_nchunk, q.psib, sk))) return e;
        if ((e = launch_solve_rest(q, q.psib, nullptr, psi + k * n, psi_ext + k * n, eps + k, sk, true, true))) return e;
        if ((e = cudaEventRecord(q.ev_join, sk))) return e;
    }
    for (int k = 0; k < c.nslice; ++k)
        if ((e = cudaStreamWaitEvent(s, c.slice[k]->ev_join, 0))) return e;
    return cudaSuccess;
}

static int fit_steps_batch_impl(efit_ctx* h, int32_t nsteps, double* d_psi, const double* d_psi_ext,
                                const double* d_meas, const double* d_sigma, double* d_coef, double* d_chi2,
                                double* d_eps, efit_stream_t stream) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    if (c.nslice < 1) return fail(&c, EFIT_E_STATE, "no batch attached (efit_batch_attach)");
    if (nsteps < 1) return fail(&c, EFIT_E_INVAL, "nsteps < 1");
    EFIT_CHECK_PTR(c, d_psi, "d_psi");
    EFIT_CHECK_PTR(c, d_psi_ext, "d_psi_ext");
    EFIT_CHECK_PTR(c, d_meas, "d_meas");
    EFIT_CHECK_PTR(c, d_sigma, "d_sigma");
    EFIT_CHECK_PTR(c, d_coef, "d_coef");
    EFIT_CHECK_PTR(c, d_chi2, "d_chi2");
    EFIT_CHECK_PTR(c, d_eps, "d_eps");
    cudaStream_t s = (cudaStream_t)stream;
    if (s == nullptr) return fail(&c, EFIT_E_INVAL, "batched calls need a non-default stream");
    cudaError_t e;
    auto enqueue = [&]() -> cudaError_t {
        for (int k = 0; k < nsteps; ++k) {
            cudaError_t e1 = enqueue_fit_step_batch(c, d_psi, d_psi_ext, d_meas, d_sigma, d_coef, d_chi2, d_eps, s, k == 0);
            if (e1) return e1;
        }
        return cudaSuccess;
    };
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if ((e = cudaStreamIsCapturing(s, &cs))) return cuda_fail(&c, e, "capture query");
    if (!c.use_graph || cs == cudaStreamCaptureStatusActive) {
        if ((e = enqueue())) return cuda_fail(&c, e, "batched fit step");
        return EFIT_OK;
    }
    const void* key[10] = {d_psi, d_psi_ext, d_meas, d_sigma, d_coef, d_chi2, d_eps, (const void*)s,
                           (const void*)(intptr_t)nsteps, (const void*)(intptr_t)c.nslice};
    if (!c.bexec || std::memcmp(key, c.bkey, sizeof(key)) != 0) {
        if (c.bexec) { cudaGraphExecDestroy(c.bexec); c.bexec = nullptr; }
        cudaGraph_t graph = nullptr;
        if ((e = cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal))) return cuda_fail(&c, e, "begin capture");
        cudaError_t e2 = enqueue();
        e = cudaStreamEndCapture(s, &graph);
        if (e2) { if (graph) cudaGraphDestroy(graph); return cuda_fail(&c, e2, "batched fit step capture"); }
        if (e) return cuda_fail(&c, e, "end capture");
        e = cudaGraphInstantiateWithFlags(&c.bexec, graph, kGraphFlags);
        cudaGraphDestroy(graph);
        if (e) { c.bexec = nullptr; return cuda_fail(&c, e, "graph instantiate"); }
        std::memcpy(c.bkey, key, sizeof(key));
    }
    if ((e = cudaGraphLaunch(c.bexec, s))) return cuda_fail(&c, e, "graph launch");
    return EFIT_OK;
}

extern "C" int efit_fit_step_batch(efit_ctx* h, double* d_psi, const double* d_psi_ext, const double* d_meas,
                                   const double* d_sigma, double* d_coef, double* d_chi2, double* d_eps,
                                   efit_stream_t stream) {
    return fit_steps_batch_impl(h, 1, d_psi, d_psi_ext, d_meas, d_sigma, d_coef, d_chi2, d_eps, stream);
}

extern "C" int efit_fit_steps_batch(efit_ctx* h, int32_t nsteps, double* d_psi, const double* d_psi_ext,
                                    const double* d_meas, const double* d_sigma, double* d_coef, double* d_chi2,
                                    double* d_eps, efit_stream_t stream) {
    return fit_steps_batch_impl(h, nsteps, d_psi, d_psi_ext, d_meas, d_sigma, d_coef, d_chi2, d_eps, stream);
}

// Shared table pass for ns current pairs: slice k's current is src + k * src_ld (n nodes); its
// boundary flux goes to d_psib + k * n_edge.  Slice streams fork from / join into s.
static cudaError_t enqueue_boundary_batch(Ctx& c, int ns, const double* src, size_t src_ld, double* d_psib,
                                          cudaStream_t s) {
    cudaError_t e1;
    if ((e1 = cudaEventRecord(c.bev_fork, s))) return e1;
    for (int k = 0; k < ns; ++k) {
        Ctx& q = *c.slice[k];
        if ((e1 = cudaStreamWaitEvent(q.side, c.bev_fork, 0))) return e1;
        if ((e1 = efit::launch_make_pair(q, src + k * src_ld, q.side))) return e1;
        if ((e1 = cudaEventRecord(q.ev_fork, q.side))) return e1;
        if ((e1 = efit::launch_lr_fft(q, d_psib + (size_t)k * c.n_edge, q.side))) return e1;
    }
    for (int k = 0; k < ns; ++k)
        if ((e1 = cudaStreamWaitEvent(s, c.slice[k]->ev_fork, 0))) return e1;
    if ((e1 = efit::launch_boundary_batch(c, ns, c.slice, s))) return e1;
    if ((e1 = cudaEventRecord(c.bev_tb, s))) return e1;
    for (int k = 0; k < ns; ++k) {
        Ctx& q = *c.slice[k];
        if ((e1 = cudaStreamWaitEvent(q.side, c.bev_tb, 0))) return e1;
        if ((e1 = efit::launch_bnd_reduce(q, q.tb_part, c.tbb_nchunk, d_psib + (size_t)k * c.n_edge, q.side))) return e1;
        if ((e1 = cudaEventRecord(q.ev_join, q.side))) return e1;
    }
    for (int k = 0; k < ns; ++k)
        if ((e1 = cudaStreamWaitEvent(s, c.slice[k]->ev_join, 0))) return e1;
    return cudaSuccess;
}

extern "C" int efit_boundary_flux_batch(efit_ctx* h, const double* d_pcurr, double* d_psib, efit_stream_t stream) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    if (c.nslice < 1) return fail(&c, EFIT_E_STATE, "no batch attached (efit_batch_attach)");
    EFIT_CHECK_PTR(c, d_pcurr, "d_pcurr");
    EFIT_CHECK_PTR(c, d_psib, "d_psib");
    cudaStream_t s = (cudaStream_t)stream;
    if (s == nullptr) return fail(&c, EFIT_E_INVAL, "batched calls need a non-default stream");
    cudaError_t e = enqueue_boundary_batch(c, c.nslice, d_pcurr, (size_t)c.nw * c.nh, d_psib, s);
    if (e) return cuda_fail(&c, e, "batched boundary flux");
    return EFIT_OK;
}

extern "C" int efit_boundary_basis(efit_ctx* h, const double* d_psi, double* d_rb, double* d_axbd,
                                   efit_stream_t stream) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    if (c.nslice < c.nb)
        return fail(&c, EFIT_E_STATE, "efit_boundary_basis needs a batch of >= nbasis (%d) slices", c.nb);
    EFIT_CHECK_PTR(c, d_psi, "d_psi");
    EFIT_CHECK_PTR(c, d_rb, "d_rb");
    cudaStream_t s = (cudaStream_t)stream;
    if (s == nullptr) return fail(&c, EFIT_E_INVAL, "batched calls need a non-default stream");
    cudaError_t e;
    if ((e = efit::launch_normalize(c, d_psi, s))) return cuda_fail(&c, e, "normalize");
    if ((e = efit::launch_basis(c, d_psi, s))) return cuda_fail(&c, e, "basis");
    const size_t ldb = (size_t)c.t.resp_nchunk * c.t.resp_gc;  // basis matrix row stride
    if ((e = enqueue_boundary_batch(c, c.nb, c.bmat, ldb, d_rb, s))) return cuda_fail(&c, e, "boundary basis");
    if (d_axbd && (e = cudaMemcpyAsync(d_axbd, c.axbd, 2 * sizeof(double), cudaMemcpyDeviceToDevice, s)))
        return cuda_fail(&c, e, "axbd copy");
    return EFIT_OK;
}

extern "C" int efit_solve_update(efit_ctx* h, const double* d_pcurr, const double* d_psib, const double* d_psi_ext,
                                 double* d_psi, double* d_eps, efit_stream_t stream) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    EFIT_CHECK_PTR(c, d_pcurr, "d_pcurr");
    EFIT_CHECK_PTR(c, d_psib, "d_psib");
    EFIT_CHECK_PTR(c, d_psi_ext, "d_psi_ext");
    EFIT_CHECK_PTR(c, d_psi, "d_psi");
    EFIT_CHECK_PTR(c, d_eps, "d_eps");
    cudaError_t e = efit::launch_solve(c, d_pcurr, d_psib, nullptr, d_psi, d_psi_ext, d_eps, (cudaStream_t)stream);
    if (e) return cuda_fail(&c, e, "solve update");
    return EFIT_OK;
}

extern "C" int efit_profile_begin(efit_ctx* h, int32_t nsteps, int32_t every) {
    if (!h || nsteps < 1 || every < 1) return fail(nullptr, EFIT_E_INVAL, "profile_begin: bad argument");
    Ctx& c = h->c;
    if (c.prof_ev) return fail(&c, EFIT_E_STATE, "profiling already active");
    size_t n = (size_t)nsteps * efit::kNumMarks;
    c.prof_ev = new (std::nothrow) cudaEvent_t[n];
    if (!c.prof_ev) return fail(&c, EFIT_E_NOMEM, "events");
    for (size_t i = 0; i < n; ++i) {
        cudaError_t e = cudaEventCreate(&c.prof_ev[i]);
        if (e) {
            for (size_t k = 0; k < i; ++k) cudaEventDestroy(c.prof_ev[k]);
            delete[] c.prof_ev;
            c.prof_ev = nullptr;
            return cuda_fail(&c, e, "event create");
        }
    }
    c.prof_slots = nsteps;
    c.prof_next = 0;
    c.prof_every = every;
    c.prof_calls = 0;
    c.prof_on = true;
    return EFIT_OK;
}

extern "C" int efit_profile_end(efit_ctx* h, double* ms_out, int32_t nout, int32_t* nsteps_out) {
    if (!h || !ms_out || nout < efit::kNumProfileFields) return fail(nullptr, EFIT_E_INVAL, "profile_end: bad argument");
    Ctx& c = h->c;
    if (!c.prof_ev) return fail(&c, EFIT_E_STATE, "profiling not active");
    for (int k = 0; k < nout; ++k) ms_out[k] = 0.0;
    int rc = EFIT_OK;
    for (int st = 0; st < c.prof_next && rc == EFIT_OK; ++st) {
        cudaEvent_t* ev = c.prof_ev + (size_t)st * efit::kNumMarks;
        if (cudaEventSynchronize(ev[efit::M_SOLVE])) { rc = cuda_fail(&c, cudaGetLastError(), "event sync"); break; }
        using namespace efit;
        // (from, to) mark pairs of the nine reported intervals; k_bnd_tb and k_bnd_lr both
        // start at the fork after the current kernel and run concurrently
        static const int pairs[kNumProfileFields][2] = {{M_BEGIN, M_SOLVE}, {M_BEGIN, M_NORM}, {M_NORM, M_RESP},
                                                        {M_RESP, M_CUR},    {M_CUR, M_TB},     {M_CUR, M_LR},
                                                        {M_TB, M_SOLVE}};
        float t;
        for (int k = 0; k < kNumProfileFields; ++k)
            if (cudaEventElapsedTime(&t, ev[pairs[k][0]], ev[pairs[k][1]]) == cudaSuccess) ms_out[k] += t;
    }
    if (nsteps_out) *nsteps_out = c.prof_next;
    for (size_t i = 0; i < (size_t)c.prof_slots * efit::kNumMarks; ++i) cudaEventDestroy(c.prof_ev[i]);
    delete[] c.prof_ev;
    c.prof_ev = nullptr;
    c.prof_on = false;
    c.prof_slots = c.prof_next = 0;
    return rc;
}

extern "C" int efit_status(efit_ctx* h, efit_stream_t stream) {
    if (!h) return fail(nullptr, EFIT_E_INVAL, "ctx is null");
    Ctx& c = h->c;
    cudaStream_t s = (cudaStream_t)stream;
    int st[1 + efit::kMaxSlices] = {0};
    cudaError_t e;
    // the context's word and every attached slice's own word (OR-ed; cleared)
    for (int k = 0; k <= c.nslice; ++k) {
        int* w = k == 0 ? c.status : c.slice[k - 1]->status;
        if ((e = cudaMemcpyAsync(&st[k], w, sizeof(int), cudaMemcpyDeviceToHost, s)) ||
            (e = cudaMemsetAsync(w, 0, sizeof(int), s)))
            return cuda_fail(&c, e, "status");
    }
    if ((e = cudaStreamSynchronize(s))) return cuda_fail(&c, e, "status");
    int all = 0, first = -1;
    for (int k = 0; k <= c.nslice; ++k) {
        all |= st[k];
        if (st[k] && first < 0) first = k;
    }
    const char* where = "";
    char buf[32] = "";
    if (first > 0) { std::snprintf(buf, sizeof(buf), " (slice %d)", first - 1); where = buf; }
    if (all & EFIT_ST_NONFINITE) return fail(&c, EFIT_E_NONFINITE, "non-finite psi%s", where);
    if (all & EFIT_ST_NOPLASMA) return fail(&c, EFIT_E_NOPLASMA, "empty plasma mask or psi_axis == psi_bdry%s", where);
    if (all & EFIT_ST_SINGULAR) return fail(&c, EFIT_E_SINGULAR, "singular least-squares matrix%s", where);
    return EFIT_OK;
}

extern "C" int efit_table(const efit_ctx* h, int which, const void** d_ptr) {
    if (!h || !d_ptr) return fail(nullptr, EFIT_E_INVAL, "null argument");
    const Ctx& c = h->c;
    switch (which) {
        case 0: *d_ptr = c.T; break;
        case 1: *d_ptr = c.Gd; break;
        case 2: *d_ptr = c.inlim; break;
        case 3: *d_ptr = c.Tedge; break;
        case 4: *d_ptr = c.U; break;
        default: return fail(nullptr, EFIT_E_INVAL, "which = %d", which);
    }
    if (!*d_ptr) return fail(nullptr, EFIT_E_STATE, "table %d not built in this mode", which);
    return EFIT_OK;
}

static void release_slices(Ctx& c) {
    for (int k = 0; k < efit::kMaxSlices; ++k) {
        Ctx* q = c.slice[k];
        if (!q) continue;
        if (q->side) cudaStreamDestroy(q->side);
        if (q->ev_fork) cudaEventDestroy(q->ev_fork);
        if (q->ev_join) cudaEventDestroy(q->ev_join);
        delete q;
        c.slice[k] = nullptr;
    }
    c.nslice = 0;
    if (c.bexec) { cudaGraphExecDestroy(c.bexec); c.bexec = nullptr; }
}

extern "C" int efit_destroy(efit_ctx* h) {
    if (!h) return EFIT_OK;
    release_slices(h->c);
    if (h->c.bev_fork) cudaEventDestroy(h->c.bev_fork);
    if (h->c.bev_tb) cudaEventDestroy(h->c.bev_tb);
    if (h->c.bev_resp) cudaEventDestroy(h->c.bev_resp);
    for (int k = 0; k < Ctx::kGraphCache; ++k)
        if (h->c.gexec[k]) cudaGraphExecDestroy(h->c.gexec[k]);
    for (int b = 0; b < 2; ++b) {
        if (h->c.hgexec[b]) cudaGraphExecDestroy(h->c.hgexec[b]);
        if (h->c.hgraph[b]) cudaGraphDestroy(h->c.hgraph[b]);
    }
    if (h->c.hs) cudaStreamDestroy(h->c.hs);
    if (h->c.ds) cudaStreamDestroy(h->c.ds);
    if (h->c.hstart) cudaEventDestroy(h->c.hstart);
    for (int b = 0; b < 2; ++b) {
        if (h->c.hin[b]) cudaEventDestroy(h->c.hin[b]);
        if (h->c.hdone[b]) cudaEventDestroy(h->c.hdone[b]);
        if (h->c.hfree[b]) cudaEventDestroy(h->c.hfree[b]);
    }
    if (h->c.pexec) cudaGraphExecDestroy(h->c.pexec);
    if (h->c.pgraph) cudaGraphDestroy(h->c.pgraph);
    for (int id = 0; id < efit::kNumMarks; ++id)
        if (h->c.prof_place[id]) cudaEventDestroy(h->c.prof_place[id]);
    if (h->c.side) cudaStreamDestroy(h->c.side);
    if (h->c.ev_fork) cudaEventDestroy(h->c.ev_fork);
    if (h->c.ev_join) cudaEventDestroy(h->c.ev_join);
    if (h->c.prof_ev) {
        for (size_t i = 0; i < (size_t)h->c.prof_slots * efit::kNumMarks; ++i) cudaEventDestroy(h->c.prof_ev[i]);
        delete[] h->c.prof_ev;
    }
    if (h->c.comm && !h->c.shadow) nccl_api().comm_destroy((ncclComm_t)h->c.comm);
    delete h;
    return EFIT_OK;
}

extern "C" const char* efit_strerror(int status) {
    switch (status) {
        case EFIT_OK: return "ok";
        case EFIT_E_INVAL: return "invalid argument";
        case EFIT_E_NOMEM: return "out of memory / workspace too small";
        case EFIT_E_CUDA: return "CUDA error";
        case EFIT_E_NCCL: return "collective error";
        case EFIT_E_SINGULAR: return "singular least-squares matrix";
        case EFIT_E_NOPLASMA: return "no plasma (empty mask)";
        case EFIT_E_NONFINITE: return "non-finite value";
        case EFIT_E_STATE: return "invalid state for this call";
        default: return "unknown status";
    }
}

extern "C" const char* efit_last_error(const efit_ctx* h) { return h ? h->c.err : g_err; }

extern "C" const char* efit_version(void) { return "efit_b200 0.1 (sm_100a)"; }
