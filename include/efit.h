/*
 * efit.h -- C ABI of the B200-native EFIT fitting-iteration hot path
 *           (library: paper_conf_sc_anteparawkbml23_b200/libefit_b200.so, sm_100a).
 *
 * The method is the per-iteration Green's-function work of EFIT's fitting call fit_
 * (Antepara et al., SC-W 2023; "P:L<n>" = /root/reference/PAPER.md line n):
 *   green_   diagnostic response of each current basis function
 *   current_ toroidal current on the grid, Eq. (2)
 *   pflux_   computational-boundary flux (the O(N^3) nests of Fig. 2/3,
 *            P:L187, L205-L230, L259-L285) + interior Grad-Shafranov solve, Eq. (1)
 *   steps_   normalised flux and plasma boundary
 *   fit_     one Picard iteration, convergence max|dpsi| < eps
 *
 * Conventions (every call):
 *   - fp64 (IEEE binary64) everywhere; SI units (m, A, Wb/rad, T); mu0 = 4 pi 1e-7.
 *   - Uniform grid R_i = rmin + i dR, Z_j = zmin + j dZ, i < nw, j < nh; node index
 *     g = i*nh + j (Z fastest), the paper's (ii-1)*nh+jj flattening.
 *   - psi is poloidal flux per radian.  pcurr is amperes per grid cell.
 *   - Edge ("computational boundary") order, n_edge = 2*nh + 2*(nw-2):
 *       left i=0, j=0..nh-1 | right i=nw-1, j=0..nh-1 | bottom j=0, i=1..nw-2 | top j=nh-1, i=1..nw-2
 *   - Diagnostic (response row) order: flux loops | magnetic probes | internal B_Z points.
 *   - Basis column order: n_pp P' terms (weight R) | n_ff FF' terms (weight mu0/(4 pi^2 R)).
 *
 * Memory & ownership: every d_* pointer is caller-owned DEVICE memory on the context's
 *   device, 16-byte aligned, never freed by the library.  Host arrays passed to
 *   efit_green_init are copied before it returns.  The workspace (all Green's tables
 *   and scratch) is caller-allocated device memory of efit_workspace_bytes() bytes
 *   that must stay alive until efit_destroy().
 * Asynchrony: compute calls only enqueue work on `stream` (a cudaStream_t; NULL = the
 *   legacy default stream) and never synchronise the host.  Outputs are valid once the
 *   stream reaches the call.  Data-dependent failures (empty plasma mask, singular
 *   least-squares matrix, non-finite input) are recorded in a device status word and
 *   reported by efit_status(); the affected outputs are set to NaN.
 * Errors: arguments are validated on the host before any launch; a failing call returns
 *   a negative EFIT_E_* code, launches nothing and leaves outputs untouched.
 *   efit_last_error() gives a one-line reason.  A context is not thread-safe.
 * Multi-GPU (efit_dist.world > 1; one process per GPU; north_star "grid rows and diagnostic/boundary
 *   points are sharded ... with an NCCL allreduce/allgather"): each rank owns the
 *   response rows [resp_row_lo, resp_row_hi) and its share of the top/bottom boundary stream
 *   (target rows [bnd_row_lo, bnd_row_hi) of the full table, or the row-pair tiles
 *   [sym_tile_lo, sym_tile_hi) of the half table); the left/right targets, the least squares, the
 *   current and the interior solve are computed on every rank.  A rank's exchange slice is
 *   zero-padded and every exchanged entry has exactly one writing rank, so the sum over ranks is
 *   exact and every output is BITWISE identical for any world size (the SYM slots are the per-tile
 *   partial sums, reduced afterwards in the same fixed order as on one GPU).
 *   - efit_dist.nccl_id != NULL: the context owns an NCCL communicator (efit_green_init is then
 *     collective over the ranks) and every compute call returns REPLICATED outputs: the exchange (one
 *     in-place sum all-reduce of the response before the least squares and one of the boundary slice
 *     before the interior solve) is enqueued inside the call on the caller's stream and captured into
 *     the fit step's CUDA graph.  NCCL is loaded at run time (the libnccl.so.2 already in the process,
 *     else the system one; EFIT_NCCL_LIB overrides); EFIT_E_NCCL reports its failures.
 *   - efit_dist.nccl_id == NULL (caller-exchange mode): efit_response writes only the rank's rows of
 *     d_resp (zero the buffer and sum it over ranks); the boundary flux goes through
 *     efit_boundary_partials -> caller's sum over ranks -> efit_boundary_finish; efit_fit_step(s) and
 *     efit_boundary_flux return EFIT_E_STATE.
 */
#ifndef EFIT_H
#define EFIT_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct efit_ctx efit_ctx;
typedef void* efit_stream_t; /* cudaStream_t */

/* Uniform R-Z grid.  Requires 3 <= nw, nh <= 2049, nh - 1 a power of two (FFT-based interior
 * solve), 0 < rmin < rmax, zmin < zmax. */
typedef struct {
    int32_t nw, nh;
    double rmin, rmax, zmin, zmax;
} efit_grid;

/* Current-density basis for P'(psihat) and FF'(psihat), Eq. (2).
 * kind 0: monomials psihat^k, k = 0..n-1.  kind 1: clamped cubic B-splines on the knot
 * vector {0,0,0,0, knots[0..n_knots-1], 1,1,1,1} (knots strictly increasing in (0,1));
 * then n_pp = n_ff = n_knots + 4.  1 <= n_pp + n_ff <= 24.  knots: host array, copied. */
typedef struct {
    int32_t kind;
    int32_t n_pp, n_ff;
    int32_t n_knots;
    const double* knots;
} efit_basis;

/* Machine geometry (host arrays, copied).  Flux loops measure psi; magnetic probes measure
 * B_R cos(ang) + B_Z sin(ang); internal points measure B_Z.  No diagnostic may sit on a
 * grid node.  The limiter is a closed polygon (vertices not repeated), n_lim >= 3.
 * ip_sign = +1 if psi is maximal on the magnetic axis (positive plasma current), -1 otherwise. */
typedef struct {
    int32_t n_fl;  const double *fl_r, *fl_z;
    int32_t n_mp;  const double *mp_r, *mp_z, *mp_ang;
    int32_t n_int; const double *int_r, *int_z;
    int32_t n_lim; const double *lim_r, *lim_z;
    int32_t ip_sign;
} efit_geometry;

/* Sharding across `world` ranks (one process per GPU).  {0, 1, NULL} = single GPU.  nccl_id: a
 * 128-byte ncclUniqueId (efit_nccl_unique_id on one rank, sent to the others by the caller), or NULL
 * for the caller-exchange mode (see "Multi-GPU" above). */
typedef struct {
    int32_t rank, world;
    const void* nccl_id;
} efit_dist;

/* Sizes derived from the configuration (filled by efit_info). */
typedef struct {
    int32_t nw, nh, ndiag, nbasis, n_edge;
    int32_t mode;
    int32_t rank, world;
    int32_t resp_row_lo, resp_row_hi;   /* this rank's response rows [lo, hi)          */
    int32_t bnd_row_lo, bnd_row_hi;     /* this rank's top/bottom target rows i [lo, hi) */
    int32_t lr_blk_lo, lr_blk_hi;       /* left/right target tiles computed (all: replicated) */
    int32_t lr_j_lo, lr_j_hi;           /* left/right targets j [lo, hi) computed (0, nh)    */
    int64_t slab_stride;                /* doubles between Green's-table slabs           */
    int32_t sym_nblk;                   /* SYM modes: 8-row blocks of the nw-2 interior rows */
    int32_t sym_tile_lo, sym_tile_hi;   /* SYM modes: this rank's row-pair tiles [lo, hi)   */
    int64_t xbuf_len;                   /* doubles of a rank's boundary exchange slice       */
    int32_t exchange;                   /* 1 if the context owns an NCCL communicator        */
    size_t workspace_bytes;
} efit_info_t;

/* Green's-function modes of the top/bottom boundary nest (the dominant O(N^3) stream):
 *   EFIT_GREEN_TABLE         full table T[i][ii][m], one slab per target row (the paper's gridpc
 *                            use); targets sharded by row.
 *   EFIT_GREEN_ONTHEFLY      same decomposition, G recomputed from (R_i, R_ii, m dZ); bitwise
 *                            equal to EFIT_GREEN_TABLE.
 *   EFIT_GREEN_TABLE_SYM     half table by reciprocity G(a; b) = G(b; a): only the
 *                            interior row pairs i <= ii are stored, in 8 x 8 row-pair tiles, and each
 *                            stored entry serves both targets i and ii -> half the bytes of TABLE.
 *                            Results equal TABLE to rounding (<= 1e-14 relative), not bit for bit.
 *   EFIT_GREEN_ONTHEFLY_SYM  the SYM decomposition with G recomputed (half the Green's evaluations
 *                            of ONTHEFLY); bitwise equal to EFIT_GREEN_TABLE_SYM.
 *   EFIT_GREEN_VONHAGENOW    no O(N^3) nest at all (the paper's call for "new algorithms that
 *                            are more suitable for GPUs"): psi0 = the interior solve of the current
 *                            with ZERO edge values, then by Green's second identity
 *                            psi_b(p) = -(1/mu0) sum_q G~(x_p; x_q) W_q (1/R_q) dpsi0/dn_q over the edge nodes
 *                            (second-order one-sided normal derivative, trapezoid weights W = dZ or dR, the
 *                            log singularity of G integrated exactly on p's own side; reading R3):
 *                            O(N^2 log N) + an n_edge x n_edge operator table.  Approximates the Green's sum
 *                            to second order in the grid spacing (~1e-5 relative at 513^2), so results are
 *                            NOT those of the table modes; world == 1 only.
 * SYM modes with world > 1: the row-pair tiles are sharded; the exchange slice holds the per-tile
 * partial sums (every slot written by one rank), reduced in a fixed order after the exchange. */
enum { EFIT_GREEN_TABLE = 0, EFIT_GREEN_ONTHEFLY = 1, EFIT_GREEN_TABLE_SYM = 2, EFIT_GREEN_ONTHEFLY_SYM = 3,
       EFIT_GREEN_VONHAGENOW = 4 };

enum {
    EFIT_OK = 0,
    EFIT_E_INVAL = -1,     /* bad argument (host-side validation)                 */
    EFIT_E_NOMEM = -2,     /* workspace too small / host allocation failed        */
    EFIT_E_CUDA = -3,      /* CUDA runtime error (possibly from earlier async work) */
    EFIT_E_NCCL = -4,      /* NCCL not loadable / communicator or collective error */
    EFIT_E_SINGULAR = -5,  /* least-squares: |R_kk| < 1e-13 max|R_jj|              */
    EFIT_E_NOPLASMA = -6,  /* empty plasma mask / psi_axis == psi_bdry             */
    EFIT_E_NONFINITE = -7, /* NaN/Inf met in a reduction                           */
    EFIT_E_STATE = -8      /* call not valid in this context state / mode          */
};

/* Bytes of device workspace efit_green_init needs for this configuration. */
int efit_workspace_bytes(const efit_grid* grid, const efit_basis* basis,
                         const efit_geometry* geom, const efit_dist* dist, int mode,
                         size_t* bytes_out);

/* Validate, carve the workspace and build every Green's table on `stream` (the
 * precomputed gridpc of P:L217-L221 re-laid out as T[i][ii][m] = G(R_i, m dZ; R_ii, 0),
 * m fastest, plus the diagnostic tables Gd[m][g]).  mode = EFIT_GREEN_ONTHEFLY skips T
 * and recomputes G inside efit_boundary_flux.  On success *out owns host state only. */
int efit_green_init(efit_ctx** out, const efit_grid* grid, const efit_basis* basis,
                    const efit_geometry* geom, const efit_dist* dist, int mode,
                    void* d_workspace, size_t ws_bytes, efit_stream_t stream);

int efit_info(const efit_ctx* ctx, efit_info_t* info);

/* Host-only: the same sizes and this rank's shard ranges for a configuration, without a device
 * or a context (validates like efit_workspace_bytes). */
int efit_plan_info(const efit_grid* grid, const efit_basis* basis, const efit_geometry* geom,
                   const efit_dist* dist, int mode, efit_info_t* info);

/* steps_ + green_: psi_axis/psi_bdry from d_psi[nw*nh], then
 * d_resp[m*nbasis + k] = sum_g Gd[m][g] dR dZ mask_g w_k(R_g) phi_k(psihat_g)
 * for every row m (world == 1, or with the NCCL exchange) or for this rank's rows only
 * (caller-exchange mode; the other rows are not written).  d_axbd[2] (may be NULL) receives
 * {psi_axis, psi_bdry}. */
int efit_response(efit_ctx* ctx, const double* d_psi, double* d_resp, double* d_axbd,
                  efit_stream_t stream);

/* current_ (Eq. (2)): d_pcurr[g] = dR dZ mask_g sum_k coef_k w_k(R_g) phi_k(psihat_g)
 * with the mask and psihat of d_psi. */
int efit_current(efit_ctx* ctx, const double* d_psi, const double* d_coef, double* d_pcurr,
                 efit_stream_t stream);

/* pflux_ O(N^3) part (Fig. 2/3): d_psib[p] = sum_g G(x_p; x_g) d_pcurr[g] for the
 * n_edge edge nodes p in the edge order above, physical sign (+; the paper stores the
 * negated sum).  The self term G(x_p; x_p) is the point-to-cell average
 * (reading Q5).  world > 1 needs the NCCL exchange (EFIT_E_STATE otherwise). */
int efit_boundary_flux(efit_ctx* ctx, const double* d_pcurr, double* d_psib,
                       efit_stream_t stream);

/* Caller-exchange form of efit_boundary_flux (any mode, any world size):
 * efit_boundary_partials writes this rank's zero-padded exchange slice d_xbuf[xbuf_len] (efit_info)
 * for the current d_pcurr: SYM modes -> the partial sums of the rank's row-pair tiles, layout
 * [i-1][side][slot] (side 0 = bottom, 1 = top; slot = the tile's other 8-row block x m-chunk);
 * full table -> the rank's top/bottom entries of psi_b (edge order from 2*nh), 0 elsewhere.
 * efit_boundary_finish takes the slices SUMMED over all ranks in d_xbuf and writes all n_edge
 * entries of d_psib (left/right targets computed locally from d_pcurr, the same current).  The
 * result is bitwise that of efit_boundary_flux on one GPU. */
int efit_boundary_partials(efit_ctx* ctx, const double* d_pcurr, double* d_xbuf, efit_stream_t stream);
int efit_boundary_finish(efit_ctx* ctx, const double* d_pcurr, const double* d_xbuf, double* d_psib,
                         efit_stream_t stream);

/* Host: a fresh 128-byte ncclUniqueId into id_out (for efit_dist.nccl_id).  EFIT_E_NCCL if NCCL
 * cannot be loaded. */
int efit_nccl_unique_id(void* id_out);

/* pflux_ O(N^2) part, Eq. (1): solve Delta*_h psi = -mu0 R pcurr/(dR dZ) on the interior
 * nodes (5-point operator, reading Q17) with psi = d_psib on the edge.
 * Writes all nw*nh nodes of d_psi_p. */
int efit_interior_solve(efit_ctx* ctx, const double* d_pcurr, const double* d_psib,
                        double* d_psi_p, efit_stream_t stream);

/* ---- steps_ rule -----------------------------------------------------------------
 * steps_ computes "the dimensionless poloidal fluxes and the location of the plasma boundary";
 * the paper gives no algorithm.  Two rules (readings Q9 and R4):
 *   EFIT_STEPS_LIMITER (default)  axis = in-limiter grid argmax of s psi; boundary = max of s psi
 *                                 (bilinear) over the limiter vertices; mask = in-limiter and
 *                                 0 <= psihat < 1 (a limited plasma).
 *   EFIT_STEPS_FULL               axis refined by Newton's method on the bicubic Hermite interpolant of
 *                                 psi (central-difference nodal derivatives); X-points = Newton-refined
 *                                 saddles from the 8 best discrete candidates (indefinite discrete
 *                                 Hessian, local minimum of |grad psi|^2) inside the limiter; boundary =
 *                                 the largest in s of {limiter value over the vertices between the lower and
 *                                 upper X-point heights, lower X-point, upper X-point}; mask = the
 *                                 4-connected component of the axis node in {in-limiter, 0 <= psihat < 1}
 *                                 (private-flux regions excluded).  Every decision is plain IEEE fp64 in
 *                                 the reading's order (bit-reproducible).  Adds five launches per
 *                                 iteration (the chained fit steps then normalise before every iteration).
 *                                 Needs 6 <= nw, nh <= 2048 and nw * ceil(nh/64) * 8 bytes of component
 *                                 bitmap in shared memory (up to ~1025^2).  Applies to the attached batch slices too
 *                                 (each slice normalises its own psi).
 * efit_set_steps: host-only switch (drops the cached fit-step graphs); EFIT_E_INVAL for a bad mode or
 *   a grid outside the limits above. */
enum { EFIT_STEPS_LIMITER = 0, EFIT_STEPS_FULL = 1 };
int efit_set_steps(efit_ctx* ctx, int32_t steps_mode);

/* The context's steps_ of d_psi[nw*nh] alone.  d_info[16] (device):
 *   [0] psi_axis [1] psi_bdry [2] R_axis [3] Z_axis [4] 1 if the axis was refined off the node
 *   [5] limiter value [6..8] lower X-point (R, Z, psi) [9..11] upper X-point [12] boundary kind
 *   (0 limiter, 1 lower X, 2 upper X) [13] masked nodes [14] X candidates examined [15] axis node g;
 *   NaN where absent (EFIT_STEPS_LIMITER fills [0], [1] and [12] only).
 * d_mask (device uint8[nw*nh], may be NULL) receives the plasma mask.  Not capturable (LIMITER mode
 * uploads a small host record). */
int efit_normalize(efit_ctx* ctx, const double* d_psi, double* d_info, uint8_t* d_mask, efit_stream_t stream);

/* Weighted least squares: minimise sum_m ((meas_m - sum_k resp_mk c_k)/sigma_m)^2
 * over all ndiag rows.  d_coef[nbasis], d_chi2[1]. */
int efit_lsq(efit_ctx* ctx, const double* d_resp, const double* d_meas, const double* d_sigma,
             double* d_coef, double* d_chi2, efit_stream_t stream);

/* fit_: one Picard iteration, entirely on the device (a captured CUDA graph
 * after the first call with the same pointers):
 *   response(psi) -> lsq -> current -> boundary flux -> interior solve ->
 *   psi <- psi_p + d_psi_ext (in place);  d_eps[0] = max|psi_new - psi_old| / |psi_bdry - psi_axis|.
 * d_meas: measurements with the external-coil contribution already removed.
 * world > 1: needs the NCCL exchange (efit_dist.nccl_id), EFIT_E_STATE otherwise; the two
 * exchanges are nodes of the captured graph and every rank ends with the same psi. */
int efit_fit_step(efit_ctx* ctx, double* d_psi, const double* d_psi_ext, const double* d_meas,
                  const double* d_sigma, double* d_coef, double* d_chi2, double* d_eps,
                  efit_stream_t stream);

/* nsteps chained Picard iterations in one call (one CUDA graph): the first normalises d_psi,
 * later ones take psi_axis/psi_bdry from the previous iteration's update kernel (no separate
 * normalisation pass).  d_coef/d_chi2/d_eps hold the last iteration's values; the caller checks
 * eps < 1e-5 every nsteps iterations.  Same arguments and rules as efit_fit_step. */
int efit_fit_steps(efit_ctx* ctx, int32_t nsteps, double* d_psi, const double* d_psi_ext,
                   const double* d_meas, const double* d_sigma, double* d_coef, double* d_chi2,
                   double* d_eps, efit_stream_t stream);

/* End-to-end reconstruction from HOST buffers (the e2e path; EFIT reconstructs many time
 * slices of a discharge).  For each of nslice slices k (one machine: shared d_psi_ext, device):
 *   h_psi0[k][nw*nh], h_meas[k][ndiag], h_sigma[k][ndiag]  (host, pinned for asynchronous copies)
 *   -> copied in, `iters` chained fit iterations (efit_fit_steps semantics), results copied out to
 *   h_psi[k][nw*nh], h_coef[k][nbasis], h_chi2[k], h_eps[k] (host).
 * The copies run on the library's own streams and are double-buffered, so the upload of slice k+1
 * and the download of slice k-1 overlap the fit of slice k.  Enqueue only: the host outputs are
 * valid once `stream` (non-NULL, not capturing) reaches the end of the call.  d_psi_ext must stay
 * constant while the call is in flight. */
int efit_fit_host(efit_ctx* ctx, int32_t nslice, int32_t iters, const double* h_psi0, const double* h_meas,
                  const double* h_sigma, const double* d_psi_ext, double* h_psi, double* h_coef, double* h_chi2,
                  double* h_eps, efit_stream_t stream);

/* Tail of a fit iteration (caller-exchange path), after efit_boundary_finish: interior solve of d_pcurr with edge values d_psib, then
 * psi <- psi_p + d_psi_ext (in place) and d_eps[0] = max|psi_new - psi_old| / |psi_bdry - psi_axis|,
 * with psi_axis/psi_bdry from the most recent efit_response or efit_current call on this ctx. */
int efit_solve_update(efit_ctx* ctx, const double* d_pcurr, const double* d_psib, const double* d_psi_ext,
                      double* d_psi, double* d_eps, efit_stream_t stream);

/* ---- multi-time-slice batch ------------------------------------------------
 * EFIT reconstructs many time slices of one discharge with the same machine and grid (P:L161:
 * slices are independent fits).  A batch of S <= 8 slices shares one pass over the top/bottom
 * Green's table: the O(N^3) nest of P:L187 / Fig. 2-3 becomes a product of the slab matrix with 2S
 * right-hand sides (each slice's current and its mirror), computed on the FP64 tensor cores
 * (mma.sync m8n8k4), while every slice's O(N^2) steps run concurrently on a stream of their own.
 * Each slice's results equal those of efit_fit_step on that slice alone to rounding (the table
 * pass sums in another order; not bit for bit); each slice has its own status word.  Requires mode EFIT_GREEN_TABLE, world == 1.
 *
 * efit_batch_workspace_bytes: device bytes of per-slice scratch for nslice slices.
 * efit_batch_attach: carve that scratch from caller-owned device memory d_workspace (256-byte
 *   aligned, kept alive until efit_destroy or the next attach; cleared here, synchronising the
 *   device) and create one stream per slice.  Re-attaching replaces the previous batch.
 *   EFIT_E_INVAL: nslice outside [1, 8] / bad workspace; EFIT_E_NOMEM: too small;
 *   EFIT_E_STATE: mode != EFIT_GREEN_TABLE or world > 1. */
int efit_batch_workspace_bytes(const efit_ctx* ctx, int32_t nslice, size_t* bytes_out);
int efit_batch_attach(efit_ctx* ctx, int32_t nslice, void* d_workspace, size_t ws_bytes);

/* One fit iteration of every attached slice (efit_fit_step semantics per slice k):
 *   d_psi[S][nw*nh] (in/out), d_psi_ext[S][nw*nh], d_meas[S][ndiag], d_sigma[S][ndiag],
 *   d_coef[S][nbasis], d_chi2[S], d_eps[S]; slices contiguous without padding (base pointers
 *   16-byte aligned; the per-slice sub-arrays need only 8-byte alignment).  stream must not be NULL (the
 *   slice streams fork from and join back into it).  Captured as one CUDA graph per pointer set.
 *   EFIT_E_STATE if no batch is attached. */
int efit_fit_step_batch(efit_ctx* ctx, double* d_psi, const double* d_psi_ext, const double* d_meas,
                        const double* d_sigma, double* d_coef, double* d_chi2, double* d_eps,
                        efit_stream_t stream);
/* nsteps chained iterations per slice (efit_fit_steps semantics). */
int efit_fit_steps_batch(efit_ctx* ctx, int32_t nsteps, double* d_psi, const double* d_psi_ext,
                         const double* d_meas, const double* d_sigma, double* d_coef, double* d_chi2,
                         double* d_eps, efit_stream_t stream);
/* Boundary flux of S currents at once: d_pcurr[S][nw*nh] -> d_psib[S][n_edge] (efit_boundary_flux
 * semantics per slice). */
int efit_boundary_flux_batch(efit_ctx* ctx, const double* d_pcurr, double* d_psib, efit_stream_t stream);

/* Fused single-pass variant: the boundary flux of every basis current instead of
 * the fitted one.  d_rb[k*n_edge + p] = sum_g G(x_p; x_g) I_k[g], with I_k[g] = dR dZ mask_g w_k(R_g)
 * phi_k(psihat_g) the current of basis function k alone (Eq. 2 with c = e_k, mask and psihat of
 * d_psi), edge order as efit_boundary_flux.  By linearity psi_b = sum_k c_k d_rb[k] for any
 * coefficients, so the O(N^3) table pass no longer waits for the least squares (it depends on psi
 * only, like efit_response) at nbasis right-hand-side pairs per table element (the shared
 * tensor-core pass of the batch).  Needs a batch of >= nbasis slices attached (their scratch holds
 * the basis currents); d_axbd[2] (may be NULL) receives {psi_axis, psi_bdry}.  EFIT_E_STATE
 * otherwise. */
int efit_boundary_basis(efit_ctx* ctx, const double* d_psi, double* d_rb, double* d_axbd, efit_stream_t stream);

/* Per-step kernel timing (the measurement hook used by bench.py).  After
 * efit_profile_begin(ctx, n, every), every `every`-th efit_fit_step call (the 1st, (every+1)-th, ...)
 * records CUDA events at seven marks, on the streams the kernels run on, until n steps are recorded.  The calls enqueue eagerly, or -- when the caller is capturing the stream into its own CUDA
 * graph, as bench.py does for its timed region -- as external event-record nodes of that graph;
 * efit_profile_end synchronises and returns, summed over the recorded steps, milliseconds for
 *   ms[0] whole step, ms[1] normalise, ms[2] response (k_basis + k_response + reduce),
 *   ms[3] lsq + current, ms[4] k_bnd_tb (from the fork), ms[5] k_bnd_lr (from the fork, concurrent),
 *   ms[6] boundary reduce + interior solve + update (from the end of k_bnd_tb).
 * nout >= 7.  *nsteps_out = number of steps recorded. */
int efit_profile_begin(efit_ctx* ctx, int32_t nsteps, int32_t every);
int efit_profile_end(efit_ctx* ctx, double* ms_out, int32_t nout, int32_t* nsteps_out);

/* Synchronise `stream` and return the data-dependent failure recorded since the last
 * efit_status() call (EFIT_OK, EFIT_E_NONFINITE, EFIT_E_NOPLASMA, EFIT_E_SINGULAR -- in that
 * priority), or EFIT_E_CUDA.  Every batch slice has its own status word (a failing slice sets only
 * its own outputs to NaN); the words of the context and of all slices are OR-ed, the first failing
 * slice is named in efit_last_error(), and all words are cleared. */
int efit_status(efit_ctx* ctx, efit_stream_t stream);

/* Test/inspection access: device pointers into the workspace.  which = 0: top/bottom Green's
 * slabs (slab of target row i at T + (i - bnd_row_lo)*slab_stride, entry ii*nh + m),
 * 1: Gd (row m at Gd + (m - resp_row_lo)*slab_stride, entry g), 2: in-limiter flags
 * (uint8[nw*nh]), 3: the two edge slabs i = 0 and i = nw-1 (at 0 and slab_stride),
 * 4: the SYM half table: tile t (global index t = Q(Q+1)/2 + P, P <= Q, this rank's tiles
 * [sym_tile_lo, sym_tile_hi) stored contiguously) at (t - sym_tile_lo)*64*nh doubles, entry
 * [p][m][q] (q fastest) = G(R_i, m dZ; R_ii, 0), i = 1 + 8P + p, ii = 1 + 8Q + q (0 if i or ii > nw-2).
 * Returns EFIT_E_STATE if the table is not built in this mode. */
int efit_table(const efit_ctx* ctx, int which, const void** d_ptr);

/* This rank's share of n targets: [lo, hi), contiguous and balanced (host logic, no GPU). */
void efit_shard(int32_t n, int32_t rank, int32_t world, int32_t* lo, int32_t* hi);

int efit_destroy(efit_ctx* ctx);
const char* efit_strerror(int status);
const char* efit_last_error(const efit_ctx* ctx);
const char* efit_version(void);

#ifdef __cplusplus
}
#endif
#endif /* EFIT_H */
