// efit_internal.h -- private state of the B200 EFIT library (not part of the ABI).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <stddef.h>

#include "efit.h"

namespace efit {

constexpr int kMaxBasis = 24;
constexpr int kNumSMs = 148;  // B200 (sm_100a): grid sizing in multiples of the SM count
constexpr int kMaxKnots = 20;
constexpr int kMaxN = 2049;  // FFT working set 2.5*M*16 B of shared memory, M = 2(nh-1)
constexpr int kLsqMaxRowsHost = 960;
constexpr int kMaxSlices = 8;   // multi-time-slice batch (efit_batch_attach): slices per pass
constexpr int kBatchCh = 512;   // k_bnd_tb_mma: table elements per chunk (16 per mma k-step quad)
constexpr int kRespBatchGc = 256;   // k_response_mma: grid nodes per chunk
constexpr int kRespBatchMaxBlk = 5; // k_response_mma: <= 40 basis columns (slices x nbasis) per pass  // k_lsq shared memory: (nb|1 + 2)*nd doubles

// k_response: depth of the register ring of MB-row load steps (4 registers per 256-bit load),
// keeping ring (4 NP MB) + accumulators (MB NB) <= 56 registers (the rest of the 128-register
// budget goes to addressing and the staged basis vector; larger rings spill), 2 <= NP <= 4.
__host__ __device__ constexpr int resp_np(int nb, int mb) {
    return (56 - mb * nb) / (4 * mb) >= 4 ? 4 : ((56 - mb * nb) / (4 * mb) >= 2 ? (56 - mb * nb) / (4 * mb) : 2);
}

// device status-word bits
#define EFIT_ST_NOPLASMA 1
#define EFIT_ST_SINGULAR 2
#define EFIT_ST_NONFINITE 4

// Tiling parameters (chosen on the host from the configuration).
struct Tiling {
    // response: chunks of `resp_gc` grid nodes, partial sums per chunk
    int resp_gc, resp_nchunk, resp_mb;
    // top/bottom boundary: chunks of `tb_ch` doubles of each slab, groups of `tb_gi` slabs
    int tb_ch, tb_nchunk, tb_gi, tb_ngroup;
    // left/right boundary: lr_jt targets per lane (odd), j-tiles of 32*lr_jt targets, 4 source
    // rows per CTA (lr_nblk blocks), source loop padded to lr_jj = roundup(nh, lr_jt)
    int lr_jt, lr_njt, lr_iib, lr_nblk, lr_jj;
    // symmetric (SYM-mode) top/bottom: 8 x 8 row-pair tiles, m split into sym_nmc chunks of
    // <= sym_mc values (the staged source columns and target rows fit 2 CTAs per SM)
    int sym_nmc, sym_mc;
    // normalisation / eps reductions
    int red_blocks;
};

struct Ctx {
    // configuration (host copy)
    int nw, nh;
    double rmin, rmax, zmin, zmax, dr, dz;
    int kind, n_pp, n_ff, nb, n_knots;
    double knots[kMaxKnots];
    int n_fl, n_mp, n_int, ndiag, n_lim, ip_sign;
    int mode, rank, world;
    bool sym, otf;               // SYM modes (half table by reciprocity); on-the-fly Green's
    bool vh;                     // EFIT_GREEN_VONHAGENOW: boundary flux by the von Hagenow construction
    int sym_nblk;                // 8-row blocks of the ni interior rows
    long long sym_ntile;         // sym_nblk (sym_nblk + 1) / 2 row-pair tiles (P <= Q)
    long long sym_tile_lo, sym_tile_hi;  // this rank's tiles
    int n_edge, ni, nmode;       // ni = nw-2 interior rows, nmode = nh-2 sine modes
    int ni_pad;                  // 32 * rows-per-lane: stride of the segment-interleaved Thomas factors
    int fhat_ld;                 // row stride of the mode-major DST coefficients (multiple of 4)
    int fft_m, fft_log2;         // complex FFT length 2(nh-1) and its log2
    int m_lo, m_hi;              // response rows of this rank
    int i_lo, i_hi;              // top/bottom target rows of this rank (within [1, nw-1))
    int jt_lo, jt_hi;            // left/right j-tiles computed here (all of them: replicated on every rank)
    long long S;                 // slab / row stride (doubles), multiple of 32
    Tiling t;
    size_t ws_bytes;
    int device;

    // device pointers carved from the workspace
    double* T;          // [i_hi-i_lo][S]   top/bottom Green's slabs (table mode)
    double* U;          // [sym_tile_hi-sym_tile_lo][8][nh][8]  SYM half table (table mode)
    double* sym_part;   // [ni][2][sym_nblk*sym_nmc]  SYM top/bottom partials (slot = block, chunk)
    double* symq;       // [sym_nblk][2 (I,F)][2 h][nh][2 qh][2]  per-iteration source columns, staged layout
    double* symp;       // [sym_nblk][2 (I,F)][8][nhp]             per-iteration block rows, 16-B aligned rows
    int nhp;            // nh rounded up to even (16-byte rows)
    double* sym_edge;   // [2][nw-2] SYM: edge-row source sums of the top/bottom targets (per iteration)
    double* Tedge;      // [2][S]           slabs i = 0 and i = nw-1 (left/right)
    double* Kvh;        // [n_edge][n_edge] von Hagenow boundary operator (VH mode; see k_vh_table)
    double* Gd;         // [m_hi-m_lo][S]   diagnostic Green's rows
    uint8_t* inlim;     // [nw*nh]
    double* dgeo;       // [ndiag][4]       r, z, cos(ang), sin(ang); kind in dkind
    int* dkind;         // [ndiag]          0 flux loop, 1 probe, 2 internal B_Z
    double* lim;        // [2*n_lim]        r then z
    double* tri_a;      // [ni]             sub-diagonal coefficient a_i
    double* tri_cp;     // [nmode][ld]      Thomas c'_i per mode (mode-major, ld = ni_pad)
    double* tri_inv;    // [nmode][ld]      1/den_i per mode
    double* tri_alpha;  // [nmode][ld]      -a_i/den_i (forward-sweep recurrence coefficient)
    double2* twiddle;   // [fft_m/2]        exp(-2 pi i k/M)
    double* sin_tab;    // [nmode]          sin(pi k/(n+1)), k = 1..n

    // per-iteration scratch
    double* axbd;       // [2] psi_axis, psi_bdry
    int* status;        // [1] sticky data-dependent failure
    unsigned* tickets;  // [8] last-block counters
    double* norm_part;  // [red_blocks][2]  (value, index) partials
    double* resp_part;  // [resp_nchunk][rows][nb]
    double* resp_cnt;   // [resp_nchunk]    masked-node counts
    double* bmat;       // [nb][resp_nchunk*resp_gc]  basis values of this iteration (k-major)
    double* resp;       // [ndiag][nb]      full response (fit step)
    double* coef;       // [nb]
    double* chi2;       // [1]
    double* pcurr;      // [roundup(nw*nh, tb_ch)]  current per cell, zero tail
    double* pflip;      // [roundup(nw*nh, tb_ch)]  I[ii][nh-1-m] (vertically mirrored), zero tail
    double* tb_part;    // [tb_nchunk][nw][2]
    double* lr_part;    // [2][nh][lr_nblk]  (direct left/right path)
    double* lr_spec;    // [2][nh][lr_ldi]   real spectra of the circular left/right kernel rows
    double2* lr_xh;     // [nh][lr_ldi]      half spectra of the source rows (per iteration)
    double2* lr_y;      // [2][nh]           accumulated spectra of both sides
    int lr_ldi;         // row stride of the spectral arrays (multiple of 4)
    bool lr_direct;     // EFIT_LR_DIRECT=1: direct Toeplitz kernel instead of the FFT path
    double* psib;       // [n_edge]
    double* fhat;       // [nmode][fhat_ld]  DST coefficients, mode-major (in place: tridiagonal solution)
    double* psip;       // [nw*nh]
    double* eps_part;   // [red_blocks]

    // multi-GPU exchange (include/efit.h "Multi-GPU"): NCCL communicator owned by the context when
    // efit_dist.nccl_id was given (then every compute call returns replicated outputs)
    double* vh_psi0;    // [nw*nh]  VH: zero-Dirichlet solve of the current
    double* vh_src;     // [n_edge] VH: W_q (1/R_q) dpsi0/dn_q at the edge nodes
    double* zero_edge;  // [n_edge] zeros (the zero-Dirichlet edge values)
    // full steps_ (efit_set_steps): per-iteration plasma mask replacing the limiter flags
    int steps;          // EFIT_STEPS_LIMITER (0) or EFIT_STEPS_FULL (1)
    uint8_t* pmask;     // [nw*nh]  connectivity-filtered plasma mask (steps == 1)
    double* st_info;    // [16]     axis / X-point / boundary record (efit_normalize layout)
    unsigned* st_cnt;   // [4]      candidate count, axis node, non-finite flag
    double2* st_cand;   // [steps_cand_cap] X-point candidates (|grad|^2, g)
    uint64_t* st_bits;  // [nw][steps_words] candidate bitmap, then the plasma component (64-bit words)
    void* comm;         // ncclComm_t or nullptr
    int nccl_err;       // last ncclResult_t != ncclSuccess of xch_allreduce (reported as EFIT_E_NCCL)

    // profiling: CUDA events recorded at marks inside the fit step (efit_profile_begin/end).
    // The profiled step is its own CUDA graph with external event-record nodes at the marks,
    // retargeted to the step's events before every replay.
    bool prof_on, prof_capture;
    int prof_slots, prof_next;
    int prof_every, prof_calls;    // record marks on every prof_every-th fit step only
    bool prof_rec;                 // this fit step records
    cudaEvent_t* prof_ev;          // [prof_slots][kNumMarks]
    cudaEvent_t prof_place[16];    // placeholder events used during capture
    cudaGraph_t pgraph;
    cudaGraphExec_t pexec;
    cudaGraphNode_t pnode[16];
    const void* pkey[8];

    // side stream + events: k_bnd_lr (FP64-bound) runs concurrently with k_bnd_tb (HBM-bound)
    cudaStream_t side;
    cudaEvent_t ev_fork, ev_join;

    // CUDA graph cache for efit_fit_step(s): a few pointer sets (efit_fit_host alternates two
    // staging slots), replaced round-robin
    static constexpr int kGraphCache = 4;
    cudaGraphExec_t gexec[kGraphCache];
    const void* gkey[kGraphCache][9];
    int gnext;
    bool use_graph;

    // host-buffer pipeline (efit_fit_host): two device staging slots, copy streams and events
    struct HostSlot {
        double *psi, *meas, *sigma, *coef, *chi2, *eps;
    } hslot[2];
    cudaStream_t hs, ds;              // H2D / D2H streams (created on first use; fallback pipeline)
    cudaEvent_t hin[2], hdone[2], hfree[2], hstart;
    // pipelined per-slice graphs: graph b = the fit of slot b + (D2H of slot b^1 -> H2D into slot b^1)
    // as a parallel branch; its 7 copy nodes are re-pointed at the neighbouring slices per launch
    cudaGraphExec_t hgexec[2];
    cudaGraph_t hgraph[2];            // kept alive: the copy-node handles below belong to it
    cudaGraphNode_t hnode[2][7];      // D2H psi, coef, chi2, eps | H2D psi, meas, sigma
    const void* hkey[2];              // (iters, d_psi_ext) the graphs were built for

    // multi-time-slice batch: shadow contexts share this context's tables and own
    // their per-iteration scratch (carved from the caller's batch workspace) and a stream each
    int nslice;
    Ctx* slice[kMaxSlices];
    bool shadow;                   // a slice context (tables not owned)
    int tbb_nchunk;                // k_bnd_tb_mma chunks (kBatchCh elements)
    int respb_nchunk;              // k_response_mma chunks (kRespBatchGc nodes)
    bool respb;                    // this batch contracts Gd once for all slices (k_response_mma)
    bool resp_mma;                 // single-slice response on k_response_mma (nb >= 8 or ~129^2; EFIT_RESP_MMA=0/1)
    bool resp_fuse;                // k_response evaluates the basis itself (EFIT_RESP_NOFUSE=1: separate k_basis)
    cudaEvent_t bev_fork, bev_tb;  // batch: fork of the slice streams, end of the shared table pass
    cudaEvent_t bev_resp;          // batch: end of the shared Gd pass
    cudaGraphExec_t bexec;
    const void* bkey[10];

    char err[256];
};

// Marks recorded (as CUDA events) inside a profiled fit step, in stream order.
// Kept minimal: every mark between two kernels on the main stream costs one programmatic
// (PDL) edge.  M_CUR sits where the k_bnd_lr fork already is; M_TB/M_LR precede the join.
enum Mark { M_BEGIN = 0, M_NORM, M_RESP, M_CUR, M_TB, M_LR, M_SOLVE, kNumMarks };
constexpr int kNumProfileFields = 7;  // step, normalize, response, lsq+current, bnd_tb, bnd_lr, tail
void mark(Ctx& c, cudaStream_t s, int id);  // efit_api.cu; no-op unless profiling

// plasma-region flags read by the basis / response / current kernels: the limiter flags (O8 rule,
// psihat tested per node) or the connectivity-filtered mask of the full steps_ (f3)
inline const uint8_t* mask_of(const Ctx& c) { return c.steps ? c.pmask : c.inlim; }

// ---- full steps_ (efit_steps.cu) -------------------------------------------------
int steps_words(int nh);
int steps_cand_cap(int nw, int nh);
size_t steps_fill_smem(int nw, int nh, bool* cand_smem);
cudaError_t prepare_steps(Ctx& c, int smem_optin);
cudaError_t launch_steps(Ctx& c, const double* psi, cudaStream_t s);
cudaError_t launch_mask_o8(Ctx& c, const double* psi, uint8_t* mask, cudaStream_t s);

// ---- launchers (efit_kernels.cu) -------------------------------------------------
cudaError_t launch_init_tables(Ctx& c, cudaStream_t s);
cudaError_t launch_normalize(Ctx& c, const double* psi, cudaStream_t s);
cudaError_t launch_response(Ctx& c, const double* psi, double* resp_rows, cudaStream_t s);
cudaError_t launch_lsq(Ctx& c, const double* resp, const double* meas, const double* sigma,
                       double* coef, double* chi2, cudaStream_t s);
cudaError_t launch_current(Ctx& c, const double* psi, const double* coef, double* pcurr,
                           bool pair, cudaStream_t s);
// Boundary-flux exchange modes (multi-GPU; include/efit.h "Multi-GPU"):
//   XCH_NONE      world 1: the whole psi_b into psib
//   XCH_NCCL      the rank's zero-padded exchange slice, in-place NCCL sum all-reduce, finish into psib
//   XCH_PARTIALS  the rank's zero-padded exchange slice into xbuf only (efit_boundary_partials)
//   XCH_FINISH    psib from the summed exchange slices in xbuf (efit_boundary_finish)
// Exchange slice: SYM modes -> the row-pair-tile partials [ni][2][sym_nblk*sym_nmc]; full table ->
// the top/bottom entries of psi_b [2(nw-2)].  Left/right targets are computed on every rank.
enum { XCH_NONE = 0, XCH_NCCL = 1, XCH_PARTIALS = 2, XCH_FINISH = 3 };
// prepacked: the SYM staged layouts were written by this iteration's current kernel (fit step)
cudaError_t launch_boundary(Ctx& c, const double* pcurr, double* psib, cudaStream_t s,
                            bool overlap_solve = false, bool prepacked = false, int xmode = XCH_NONE,
                            double* xbuf = nullptr);
// in-place NCCL sum all-reduce of n doubles over the context's communicator (efit_api.cu)
cudaError_t xch_allreduce(Ctx& c, double* buf, size_t n, cudaStream_t s);
cudaError_t launch_solve_fwd(Ctx& c, const double* pcurr, const double* psib, cudaStream_t s, int with_bnd);
cudaError_t launch_solve_rest(Ctx& c, const double* psib, double* psi_out, double* psi_inout, const double* psi_ext,
                              double* eps, cudaStream_t s, bool next_norm, bool tb_fix);
cudaError_t launch_basis(Ctx& c, const double* psi, cudaStream_t s);
bool response_batch_ok(const Ctx& c, int nslice);
cudaError_t launch_response_batch(Ctx& c, int nslice, Ctx* const* slices, cudaStream_t s);
cudaError_t launch_resp_reduce_batch(Ctx& q, int nchunk, double* resp_rows, cudaStream_t s);
cudaError_t launch_bnd_reduce(Ctx& c, const double* tb_part, int tb_nchunk, double* psib, cudaStream_t s);
cudaError_t launch_lr_fft(Ctx& c, double* psib, cudaStream_t s);
// multi-slice top/bottom nest: one pass over this rank's slabs for the slices' (pcurr, pflip) pairs
cudaError_t launch_boundary_batch(Ctx& c, int nslice, Ctx* const* slices, cudaStream_t s);
cudaError_t launch_solve(Ctx& c, const double* pcurr, const double* psib, double* psi_out,
                         double* psi_inout, const double* psi_ext, double* eps, cudaStream_t s,
                         bool next_norm = false);

}  // namespace efit
