// efit_kernels.cu -- sm_100a kernels of the EFIT fitting-iteration hot path.
//
// Per iteration (DESIGN.md §"Kernels"):
//   k_normalize   psi -> psi_axis, psi_bdry                   (steps_)
//   k_response    Gd x basis(psi) -> per-chunk partials        (green_)   HBM-bound
//   k_resp_reduce fixed-order chunk sum -> R_resp[m][k]
//   k_lsq         column-scaled Householder QR -> c, chi2
//   k_current     I_g and (I, I_flipped) pairs                  (current_, Eq. (2))
//   k_bnd_tb      top/bottom targets, T slabs streamed once     (pflux_ 2nd O(N^3) nest) HBM-bound
//   k_bnd_lr      left/right targets, Toeplitz in registers     (pflux_ Fig. 2 nest)  FP64-bound
//   k_bnd_reduce  fixed-order partial sums -> psi_b (edge order)
//   k_dst_fwd / k_tridiag / k_dst_inv / k_norm_fin   interior GS solve + update + eps (pflux_ O(N^2), Eq. (1))
// Every reduction has a fixed order, so results are bitwise reproducible run to run and
// independent of the number of ranks.
#include <cfloat>
#include <climits>
#include <cstdio>
#include <cstdlib>
#include <utility>

#include "efit_device.cuh"
#include "efit_internal.h"

namespace efit {

static int g_smem_optin = 227 * 1024;  // device opt-in shared memory per block (set in prepare_kernels)

// Programmatic dependent launch: every per-iteration kernel is launched with programmatic stream
// serialisation, so its CTAs are scheduled while the predecessor's last wave drains; the kernel
// itself waits (griddepcontrol.wait) until the predecessor has completed and flushed before it
// touches any of its outputs, then immediately allows its own dependents to launch.
static const bool g_no_pdl = getenv("EFIT_NO_PDL") != nullptr;  // A/B switch for profiling

template <typename... KArgs, typename... Args>
static cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                              Args&&... args) {
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = g_no_pdl ? 0 : 1;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

// Raise (never lower) a kernel's dynamic shared-memory limit to the device maximum minus its
// static shared memory.  The limit is per function and process-wide.
static cudaError_t raise_smem_limit(const void* f, size_t need) {
    cudaFuncAttributes fa;
    cudaError_t e = cudaFuncGetAttributes(&fa, f);
    if (e) return e;
    const int lim = g_smem_optin - (int)fa.sharedSizeBytes;
    if ((long long)need > lim) return cudaErrorInvalidValue;
    if (fa.maxDynamicSharedSizeBytes >= lim) return cudaSuccess;
    return cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, lim);
}


// ------------------------------------------------------------------------------ helpers

__device__ __forceinline__ double2 ldg_stream(const double* p) {
    double2 v;
    asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0, %1}, [%2];"
                 : "=d"(v.x), "=d"(v.y) : "l"(p));
    return v;
}

struct d4 {
    double x, y, z, w;
};

// 256-bit streaming load (LDG.E.NA.EFL2.256): read-only, no L1 allocation, L2 evict-first.
// Used for data read exactly once per iteration (Green's tables).  32-byte aligned.
__device__ __forceinline__ d4 ld256_stream(const double* p) {
    d4 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v4.f64 {%0, %1, %2, %3}, [%4];"
                 : "=d"(v.x), "=d"(v.y), "=d"(v.z), "=d"(v.w) : "l"(p));
    return v;
}

// Asynchronous global -> shared copy of one double (cp.async.ca, 8 bytes); ok == false writes 0.
__device__ __forceinline__ void cp_async8(double* dst, const double* src, bool ok) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" ::"r"(d), "l"(src), "r"(ok ? 8 : 0) : "memory");
}

// mbarrier + bulk (TMA 1-D) copies global -> shared, completing on the barrier's transaction count.
__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(unsigned long long* bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n\tfence.mbarrier_init.release.cluster;" ::"r"(smem_u32(bar)),
                 "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(unsigned long long* bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}

__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, unsigned long long* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void mbar_wait(unsigned long long* bar, unsigned phase) {
    asm volatile("{\n\t.reg .pred p;\n\tWAIT%=:\n\t"
                 "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
                 "@!p bra WAIT%=;\n\t}" ::"r"(smem_u32(bar)), "r"(phase) : "memory");
}

__device__ __forceinline__ void cp_async_wait_all() {
    asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
}

__device__ __forceinline__ d4 lds256(const double* p) {  // two 128-bit shared loads
    const double2 a = reinterpret_cast<const double2*>(p)[0];
    const double2 b = reinterpret_cast<const double2*>(p)[1];
    return d4{a.x, a.y, b.x, b.y};
}

// FP64 tensor-core MMA (DMMA.8x8x4): D[8x8] += A[8x4] B[4x8]; lane (g = lane/4, k4 = lane%4) holds
// A[g][k4], B[k4][g] and D[g][2k4 .. 2k4+1].
__device__ __forceinline__ void dmma884(double& d0, double& d1, double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0, %1}, {%2}, {%3}, {%0, %1};"
                 : "+d"(d0), "+d"(d1) : "d"(a), "d"(b));
}

__device__ __forceinline__ double dot4(const d4& a, const d4& b, double acc) {
    acc = fma(a.x, b.x, acc);
    acc = fma(a.y, b.y, acc);
    acc = fma(a.z, b.z, acc);
    return fma(a.w, b.w, acc);
}

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

__device__ __forceinline__ double warp_max(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = fmax(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}

// (value, index) arg-max with ties to the lowest index (a total order => partition-independent)
__device__ __forceinline__ void argmax_merge(double& v, long long& i, double v2, long long i2) {
    if (v2 > v || (v2 == v && i2 < i)) { v = v2; i = i2; }
}

__device__ __forceinline__ void warp_argmax(double& v, long long& i) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        double v2 = __shfl_xor_sync(0xffffffffu, v, o);
        long long i2 = __shfl_xor_sync(0xffffffffu, i, o);
        argmax_merge(v, i, v2, i2);
    }
}

// Bilinear interpolation of psi at (R, Z); fixed operation order without contraction
// (reading Q9) so the limiter-touch value is reproducible bit for bit.
__device__ double bilinear(const double* psi, int nw, int nh, double rmin, double dr, double zmin,
                           double dz, double R, double Z) {
    double x = __ddiv_rn(__dsub_rn(R, rmin), dr);
    double y = __ddiv_rn(__dsub_rn(Z, zmin), dz);
    int i = (int)floor(x), j = (int)floor(y);
    i = i < 0 ? 0 : (i > nw - 2 ? nw - 2 : i);
    j = j < 0 ? 0 : (j > nh - 2 ? nh - 2 : j);
    double t = __dsub_rn(x, (double)i), u = __dsub_rn(y, (double)j);
    double omt = __dsub_rn(1.0, t), omu = __dsub_rn(1.0, u);
    double w00 = __dmul_rn(omt, omu), w10 = __dmul_rn(t, omu), w01 = __dmul_rn(omt, u), w11 = __dmul_rn(t, u);
    long long g = (long long)i * nh + j;
    // L2 loads: in k_dst_inv's last block psi was just written by other CTAs (an L1 line of this SM
    // may still hold old values of a row it shares with this CTA's rows)
    double s = __dadd_rn(__dmul_rn(w00, __ldcg(psi + g)), __dmul_rn(w10, __ldcg(psi + g + nh)));
    s = __dadd_rn(s, __dmul_rn(w01, __ldcg(psi + g + 1)));
    s = __dadd_rn(s, __dmul_rn(w11, __ldcg(psi + g + nh + 1)));
    return s;
}

cudaError_t launch_lr_spectra(Ctx& c, cudaStream_t s);
cudaError_t launch_lr_fft(Ctx& c, double* psib, cudaStream_t s);
cudaError_t prepare_lr_fft(Ctx& c);

// ================================================================================ init

// Green's slabs: slab r is target row i = row_first + r*row_step;
// T[r][ii*nh + m] = G(R_i, m dZ; R_ii, 0), self term at (i == ii, m == 0).
__global__ void k_green_slabs(double* __restrict__ T, long long S, int nslab, int row_first, int row_step,
                              int nw, int nh, double rmin, double dr, double dz) {
    long long n = (long long)nw * nh;
    long long total = (long long)nslab * n;
    for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < total;
         e += (long long)gridDim.x * blockDim.x) {
        int r = (int)(e / n);
        long long rem = e - (long long)r * n;
        int ii = (int)(rem / nh);
        int m = (int)(rem - (long long)ii * nh);
        int i = row_first + r * row_step;
        double Ri = grid_coord(rmin, i, dr), Rs = grid_coord(rmin, ii, dr);
        double v = (i == ii && m == 0) ? green_self(Ri, dr, dz)
                                       : green_psi(Ri, __dmul_rn((double)m, dz), Rs, 0.0);
        T[(long long)r * S + rem] = v;
    }
}

// Diagnostic rows: Gd[r][g] = response of diagnostic m = m_lo + r to 1 A at node g.
__global__ void k_green_diag(double* __restrict__ Gd, long long S, int nrows, int m_lo,
                             const double* __restrict__ dgeo, const int* __restrict__ dkind,
                             int nw, int nh, double rmin, double dr, double zmin, double dz) {
    long long n = (long long)nw * nh;
    long long total = (long long)nrows * n;
    for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < total;
         e += (long long)gridDim.x * blockDim.x) {
        int r = (int)(e / n);
        long long g = e - (long long)r * n;
        int ii = (int)(g / nh), jj = (int)(g - (long long)ii * nh);
        int m = m_lo + r;
        double Rs = grid_coord(rmin, ii, dr), Zs = grid_coord(zmin, jj, dz);
        double R = dgeo[4 * m], Z = dgeo[4 * m + 1];
        double v;
        int kd = dkind[m];
        if (kd == 0) {
            v = green_psi(R, Z, Rs, Zs);
        } else {
            double BR, BZ;
            green_field(R, Z, Rs, Zs, BR, BZ);
            v = (kd == 1) ? (BR * dgeo[4 * m + 2] + BZ * dgeo[4 * m + 3]) : BZ;
        }
        Gd[(long long)r * S + g] = v;
    }
}

// SYM-mode half table (see the SYM section of the boundary flux below).
__device__ __forceinline__ void sym_tile_pq(long long t, int& P, int& Q) {
    int q = (int)((sqrt(8.0 * (double)t + 1.0) - 1.0) * 0.5);
    while ((long long)(q + 1) * (q + 2) / 2 <= t) ++q;
    while ((long long)q * (q + 1) / 2 > t) --q;
    Q = q;
    P = (int)(t - (long long)q * (q + 1) / 2);
}

// The one expression both the SYM table build and the SYM on-the-fly kernel evaluate (bitwise
// identical modes): same arguments as the full table's k_green_slabs entry for target row i.
__device__ __forceinline__ double sym_entry(int rp, int rq, int m, int ni, double rmin, double dr, double dz) {
    if (rp >= ni || rq >= ni) return 0.0;
    const int i = 1 + rp, ii = 1 + rq;
    const double Ri = grid_coord(rmin, i, dr);
    return (i == ii && m == 0) ? green_self(Ri, dr, dz)
                               : green_psi(Ri, __dmul_rn((double)m, dz), grid_coord(rmin, ii, dr), 0.0);
}

__global__ void k_green_sym(double* __restrict__ U, long long ntile, long long tile_lo, int ni, int nh, double rmin,
                            double dr, double dz) {
    const long long tsz = 64LL * nh;
    const long long total = ntile * tsz;
    for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < total;
         e += (long long)gridDim.x * blockDim.x) {
        const long long tl = e / tsz;
        const long long rem = e - tl * tsz;
        const int p = (int)(rem / (8LL * nh));
        const int rem2 = (int)(rem - (long long)p * 8 * nh);
        const int m = rem2 >> 3, q = rem2 & 7;
        int P, Q;
        sym_tile_pq(tile_lo + tl, P, Q);
        U[e] = sym_entry(8 * P + p, 8 * Q + q, m, ni, rmin, dr, dz);
    }
}

// In-limiter flags: even-odd crossing rule with the fixed formula
// x = ((r1 - r0) * (Z - z0)) / (z1 - z0) + r0 (reading Q9).
__global__ void k_inlim(uint8_t* __restrict__ inlim, const double* __restrict__ lim, int n_lim,
                        int nw, int nh, double rmin, double dr, double zmin, double dz) {
    int n = nw * nh;
    for (int g = blockIdx.x * blockDim.x + threadIdx.x; g < n; g += gridDim.x * blockDim.x) {
        int i = g / nh, j = g - (g / nh) * nh;
        double R = grid_coord(rmin, i, dr), Z = grid_coord(zmin, j, dz);
        int inside = 0;
        for (int k = 0; k < n_lim; ++k) {
            int k1 = (k + 1 == n_lim) ? 0 : k + 1;
            double r0 = lim[k], z0 = lim[n_lim + k], r1 = lim[k1], z1 = lim[n_lim + k1];
            if ((z0 > Z) != (z1 > Z)) {
                double x = __dadd_rn(__ddiv_rn(__dmul_rn(__dsub_rn(r1, r0), __dsub_rn(Z, z0)), __dsub_rn(z1, z0)), r0);
                if (R < x) inside ^= 1;
            }
        }
        inlim[g] = (uint8_t)inside;
    }
}

// Factors of the radial tridiagonal systems, one per sine mode k = 1..nmode:
//   a_i x_{i-1} + (-2/dR^2 + lambda_k) x_i + c_i x_{i+1},  lambda_k = -4 sin^2(pi k/(2(n+1)))/dZ^2
// LU (Thomas) factors den_i = b - a_i c'_{i-1}, c'_i = c_i/den_i, stored mode-major with the
// forward-sweep coefficients  d_i = inv_i f_i + alpha_i d_{i-1},  alpha_i = -a_i/den_i.
__global__ void k_tri_factors(double* __restrict__ tri_a, double* __restrict__ cp, double* __restrict__ inv,
                              double* __restrict__ alpha, int ni, int ld, int nmode, double rmin, double dr,
                              double dz) {
    int k = blockIdx.x * blockDim.x + threadIdx.x;  // mode index 0..nmode-1 (mode k+1)
    double idr2 = 1.0 / (dr * dr);
    if (k == 0) {
        for (int i = 1; i <= ni; ++i) {
            double R = grid_coord(rmin, i, dr);
            tri_a[i - 1] = idr2 + 1.0 / (2.0 * R * dr);
        }
    }
    if (k >= nmode) return;
    double s = sinpi((double)(k + 1) / (2.0 * (double)(nmode + 1)));
    double lam = -4.0 * s * s / (dz * dz);
    double b = -2.0 * idr2 + lam;
    double cprev = 0.0;
    for (int i = 1; i <= ni; ++i) {
        double R = grid_coord(rmin, i, dr);
        double a = idr2 + 1.0 / (2.0 * R * dr);
        double c = idr2 - 1.0 / (2.0 * R * dr);
        double den = (i == 1) ? b : b - a * cprev;
        double cpi = c / den;
        const int r = i - 1, L = ld >> 5;  // segment-interleaved position of row r
        const long long o = (long long)k * ld + (long long)(r % L) * 32 + r / L;
        cp[o] = (i == ni) ? 0.0 : cpi;
        inv[o] = 1.0 / den;
        alpha[o] = (i == 1) ? 0.0 : -a / den;
        cprev = cpi;
    }
}

__global__ void k_sin_table(double* __restrict__ sk, int n) {  // sin(pi k/(n+1)), k = 1..n
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k < n) sk[k] = sinpi((double)(k + 1) / (double)(n + 1));
}

__global__ void k_twiddles(double2* __restrict__ w, int M) {
    int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= M / 2) return;
    double s, c;
    sincospi(2.0 * (double)k / (double)M, &s, &c);
    w[k] = make_double2(c, -s);
}

// ------------------------------------------------------------ von Hagenow boundary (VH mode)
// SURVEY 8(f) f2 / P:L370; include/efit.h EFIT_GREEN_VONHAGENOW.  Green's second identity for
// Delta* = R div(R^-1 grad) with G(x_p, .) (homogeneous inside the box) and psi0 (the interior solve
// with zero edge values) gives psi_b(x_p) = -(1/mu0) \oint G(x_p; x') (1/R') dpsi0/dn' dl'.
// Edge position helpers (edge order of include/efit.h; side 0 left, 1 right, 2 bottom, 3 top).
__device__ __forceinline__ void vh_edge(int p, int nw, int nh, int& i, int& j, int& side) {
    if (p < nh) { i = 0; j = p; side = 0; }
    else if (p < 2 * nh) { i = nw - 1; j = p - nh; side = 1; }
    else if (p < 2 * nh + nw - 2) { i = p - 2 * nh + 1; j = 0; side = 2; }
    else { i = p - 2 * nh - (nw - 2) + 1; j = nh - 1; side = 3; }
}

// K[p][q] = -(1/mu0) G~(x_p; x_q): G itself for q off p's side; on p's side the log singularity's
// point value -ln(rho) replaced by its exact average over q's segment of length W (dZ or dR),
// coefficient (mu0/2pi) sqrt(R_p R_q); q = p: the segment average (mu0/2pi) R (ln(16 R/W) - 1).
// Corner sources are unused (psi0 and its tangential derivatives vanish there): K = 0.
__global__ void k_vh_table(double* __restrict__ K, int nw, int nh, int ldk, double rmin, double dr, double zmin,
                           double dz) {
    const int ne = 2 * nh + 2 * (nw - 2);
    const long long e = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= (long long)ne * ldk) return;
    const int p = (int)(e / ldk), q = (int)(e - (long long)p * ldk);
    if (q >= ne) { K[e] = 0.0; return; }
    int i, j, sp, ii, jj, sq;
    vh_edge(p, nw, nh, i, j, sp);
    vh_edge(q, nw, nh, ii, jj, sq);
    double v = 0.0;
    if (!((ii == 0 || ii == nw - 1) && (jj == 0 || jj == nh - 1))) {
        const double Rp = grid_coord(rmin, i, dr), Zp = grid_coord(zmin, j, dz);
        const double Rq = grid_coord(rmin, ii, dr), Zq = grid_coord(zmin, jj, dz);
        const double w = sq < 2 ? dz : dr;
        double G;
        if (p == q) {
            G = kMu0Over2Pi * Rp * (log(16.0 * Rp / w) - 1.0);
        } else {
            G = green_psi(Rp, Zp, Rq, Zq);
            if (sp == sq) {
                const double d = sq < 2 ? fabs(Zq - Zp) : fabs(Rq - Rp);
                const double a = d - 0.5 * w, b = d + 0.5 * w;
                const double avg = ((b * log(b) - b) - (a * log(a) - a)) / w;
                G += kMu0Over2Pi * sqrt(Rp * Rq) * (log(d) - avg);
            }
        }
        v = -G / kMu0;
    }
    K[e] = v;
}

// s_q = W_q (1/R_q) dpsi0/dn_q at every edge node (outward normal, second-order one-sided
// difference with psi0 = 0 on the edge; 0 at the corners).
__global__ void k_vh_src(const double* __restrict__ psi0, int nw, int nh, double rmin, double dr, double dz,
                         double* __restrict__ src) {
    griddep();
    const int ne = 2 * nh + 2 * (nw - 2);
    const int q = blockIdx.x * blockDim.x + threadIdx.x;
    if (q >= ne) return;
    int i, j, sd;
    vh_edge(q, nw, nh, i, j, sd);
    double v = 0.0;
    if (!((i == 0 || i == nw - 1) && (j == 0 || j == nh - 1))) {
        double dn, w;
        if (sd == 0) { dn = -(4.0 * psi0[(long long)1 * nh + j] - psi0[(long long)2 * nh + j]) / (2.0 * dr); w = dz; }
        else if (sd == 1) { dn = -(4.0 * psi0[(long long)(nw - 2) * nh + j] - psi0[(long long)(nw - 3) * nh + j]) / (2.0 * dr); w = dz; }
        else if (sd == 2) { dn = -(4.0 * psi0[(long long)i * nh + 1] - psi0[(long long)i * nh + 2]) / (2.0 * dz); w = dr; }
        else { dn = -(4.0 * psi0[(long long)i * nh + nh - 2] - psi0[(long long)i * nh + nh - 3]) / (2.0 * dz); w = dr; }
        v = w * dn / grid_coord(rmin, i, dr);
    }
    src[q] = v;
}

// psi_b[p] = sum_q K[p][q] s_q: one warp per target, 256-bit streaming loads of the operator row
// (row stride ldk = n_edge rounded up to 4, zero padded), lane-strided fixed-order partial sums +
// butterfly (deterministic); the operator streams once per iteration (33.5 MB at 513^2).
__global__ void __launch_bounds__(256) k_vh_apply(const double* __restrict__ K, const double* __restrict__ src, int ne,
                                                  int ldk, double* __restrict__ psib) {
    const int p = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
    const double* kr = K + (long long)(p < ne ? p : 0) * ldk;
    constexpr int kU = 4;
    d4 kv[kU];
    const int nv = ldk >> 2;  // 4-double vectors per row
#pragma unroll
    for (int u = 0; u < kU; ++u) {  // the operator is a constant table: first loads before the wait
        const int v = lane + 32 * u;
        kv[u] = v < nv ? ld256_stream(kr + 4 * v) : d4{0.0, 0.0, 0.0, 0.0};
    }
    griddep();
    if (p >= ne) return;
    double s = 0.0;
    for (int v0 = 0; v0 < nv; v0 += 32 * kU) {
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int v = v0 + lane + 32 * u;
            if (v < nv) {
                const double4 x = *reinterpret_cast<const double4*>(src + 4 * v);
                s = dot4(kv[u], d4{x.x, x.y, x.z, x.w}, s);
            }
            const int vn = v + 32 * kU;
            kv[u] = vn < nv ? ld256_stream(kr + 4 * vn) : d4{0.0, 0.0, 0.0, 0.0};
        }
    }
    s = warp_sum(s);
    if (lane == 0) psib[p] = s;
}

cudaError_t launch_init_tables(Ctx& c, cudaStream_t s) {
    const int nw = c.nw, nh = c.nh;
    const long long n = (long long)nw * nh;
    // zero everything first (table padding must read as 0)
    cudaError_t e = cudaMemsetAsync(c.Tedge, 0, sizeof(double) * 2 * c.S, s);
    if (e) return e;
    if (c.T && c.i_hi > c.i_lo) {
        e = cudaMemsetAsync(c.T, 0, sizeof(double) * (size_t)(c.i_hi - c.i_lo) * c.S, s);
        if (e) return e;
    }
    if (c.m_hi > c.m_lo) {
        e = cudaMemsetAsync(c.Gd, 0, sizeof(double) * (size_t)(c.m_hi - c.m_lo) * c.S, s);
        if (e) return e;
    }
    {
        const size_t padn = (size_t)(((n + c.t.tb_ch - 1) / c.t.tb_ch) * c.t.tb_ch);
        if ((e = cudaMemsetAsync(c.pcurr, 0, sizeof(double) * padn, s))) return e;
        if ((e = cudaMemsetAsync(c.pflip, 0, sizeof(double) * padn, s))) return e;
    }
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, c.device);
    const int bs = 256;
    k_green_slabs<<<sms * 8, bs, 0, s>>>(c.Tedge, c.S, 2, 0, nw - 1, nw, nh, c.rmin, c.dr, c.dz);
    if (c.T && c.i_hi > c.i_lo)
        k_green_slabs<<<sms * 16, bs, 0, s>>>(c.T, c.S, c.i_hi - c.i_lo, c.i_lo, 1, nw, nh, c.rmin, c.dr, c.dz);
    if (c.U) {
        const long long ntl = c.sym_tile_hi - c.sym_tile_lo;
        k_green_sym<<<sms * 16, bs, 0, s>>>(c.U, ntl, c.sym_tile_lo, c.ni, nh, c.rmin, c.dr, c.dz);
    }
    if (c.symq && (e = cudaMemsetAsync(c.symq, 0, sizeof(double) * 16 * (size_t)c.sym_nblk * c.nh, s))) return e;
    if (c.symp && (e = cudaMemsetAsync(c.symp, 0, sizeof(double) * 16 * (size_t)c.sym_nblk * c.nhp, s))) return e;
    if (c.sym_part &&
        (e = cudaMemsetAsync(c.sym_part, 0, sizeof(double) * 2 * (size_t)(c.ni > 0 ? c.ni : 1) * c.sym_nblk * c.t.sym_nmc, s)))
        return e;
    if (c.m_hi > c.m_lo)
        k_green_diag<<<sms * 16, bs, 0, s>>>(c.Gd, c.S, c.m_hi - c.m_lo, c.m_lo, c.dgeo, c.dkind, nw, nh,
                                              c.rmin, c.dr, c.zmin, c.dz);
    k_inlim<<<(int)((n + bs - 1) / bs), bs, 0, s>>>(c.inlim, c.lim, c.n_lim, nw, nh, c.rmin, c.dr, c.zmin, c.dz);
    if (c.vh) {
        const int ldk = (c.n_edge + 3) / 4 * 4;
        const long long ne2 = (long long)c.n_edge * ldk;
        k_vh_table<<<(unsigned)((ne2 + bs - 1) / bs), bs, 0, s>>>(c.Kvh, nw, nh, ldk, c.rmin, c.dr, c.zmin, c.dz);
        if ((e = cudaMemsetAsync(c.zero_edge, 0, sizeof(double) * ldk, s))) return e;
        if ((e = cudaMemsetAsync(c.vh_src, 0, sizeof(double) * ldk, s))) return e;
    }
    // the factor arrays are padded to 32-row multiples: zero padding makes the padded rows inert in
    // the warp scans of k_tridiag_reg (compute-sanitizer initcheck, profiles/r02_sanitize_*.txt)
    for (double* f : {c.tri_cp, c.tri_inv, c.tri_alpha})
        if ((e = cudaMemsetAsync(f, 0, sizeof(double) * (size_t)c.ni_pad * c.nmode, s))) return e;
    k_tri_factors<<<(c.nmode + 63) / 64, 64, 0, s>>>(c.tri_a, c.tri_cp, c.tri_inv, c.tri_alpha, c.ni, c.ni_pad,
                                                     c.nmode, c.rmin, c.dr, c.dz);
    k_twiddles<<<(c.fft_m / 2 + 255) / 256, 256, 0, s>>>(c.twiddle, c.fft_m);
    k_sin_table<<<(c.nmode + 255) / 256, 256, 0, s>>>(c.sin_tab, c.nmode);
    {  // needs the edge slabs and the twiddles above (also built in direct mode: the batch uses the FFT chain)
        e = launch_lr_spectra(c, s);
        if (e) return e;
    }
    e = cudaMemsetAsync(c.status, 0, sizeof(int), s);
    if (e) return e;
    e = cudaMemsetAsync(c.tickets, 0, sizeof(unsigned) * 8, s);
    if (e) return e;
    if (c.st_cnt && (e = cudaMemsetAsync(c.st_cnt, 0, sizeof(unsigned) * 4, s))) return e;
    return cudaGetLastError();
}

// ================================================================================ normalize


// psi_axis = s * max_{g in limiter} s psi_g (ties: lowest g);  psi_bdry = s * max over limiter
// vertices of s * bilinear(psi) (ties: lowest vertex).  Per-block (value, index) partials here; the
// one-CTA k_norm_fin behind it merges them and evaluates the limiter vertices.
__global__ void __launch_bounds__(256) k_normalize(const double* __restrict__ psi, const uint8_t* __restrict__ inlim,
                                                   int nw, int nh, double rmin, double dr, double zmin, double dz,
                                                   int sgn, const double* __restrict__ lim, int n_lim,
                                                   double* __restrict__ part, int* status) {
    griddep();
    __shared__ double sv[8];
    __shared__ long long si[8];
    const int n = nw * nh;
    const double s = (double)sgn;
    double best = -DBL_MAX;
    long long bi = LLONG_MAX;
    bool bad = false;
    const int stride = gridDim.x * blockDim.x;
#pragma unroll 4
    for (int g = blockIdx.x * blockDim.x + threadIdx.x; g < n; g += stride) {
        const double p = __ldg(psi + g);
        const uint8_t in = __ldg(inlim + g);
        if (!isfinite(p)) bad = true;
        if (in) argmax_merge(best, bi, s * p, (long long)g);
    }
    if (__syncthreads_or(bad) && threadIdx.x == 0) atomicOr(status, EFIT_ST_NONFINITE);
    warp_argmax(best, bi);
    int w = threadIdx.x >> 5, l = threadIdx.x & 31;
    if (l == 0) { sv[w] = best; si[w] = bi; }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int q = 1; q < (int)(blockDim.x >> 5); ++q) argmax_merge(best, bi, sv[q], si[q]);
        part[2 * blockIdx.x] = best;
        part[2 * blockIdx.x + 1] = (double)bi;
    }
}

static cudaError_t launch_norm_fin(Ctx& c, const double* psi, int nparts, const double* eps_part, double* eps,
                                   cudaStream_t s);  // after k_norm_fin below

cudaError_t launch_normalize(Ctx& c, const double* psi, cudaStream_t s) {
    if (c.steps) return launch_steps(c, psi, s);
    cudaError_t e = launch_pdl(k_normalize, dim3(c.t.red_blocks), dim3(256), 0, s, psi, c.inlim, c.nw, c.nh, c.rmin,
                               c.dr, c.zmin, c.dz, c.ip_sign, c.lim, c.n_lim, c.norm_part, c.status);
    if (e) return e;
    return launch_norm_fin(c, psi, c.t.red_blocks, nullptr, nullptr, s);
}

static BasisParams basis_params(const Ctx& c) {
    BasisParams bp;
    bp.kind = c.kind; bp.n_pp = c.n_pp; bp.n_ff = c.n_ff; bp.n_knots = c.n_knots;
    for (int k = 0; k < 20; ++k) bp.knots[k] = k < c.n_knots ? c.knots[k] : 1.0;
    return bp;
}

// psihat and mask of node g (reading Q9): exact IEEE ops, no contraction possible.
__device__ __forceinline__ bool node_psihat(const double* psi, const uint8_t* inlim, int g, double pa, double pb,
                                            double& h) {
    if (!inlim[g]) return false;
    h = (psi[g] - pa) / (pb - pa);
    return h >= 0.0 && h < 1.0;
}

// ================================================================================ response

// Basis values of every node for this iteration: Bm[k][g] = dR dZ mask_g w_k(R_g) phi_k(psihat_g)
// (k-major, zero-padded to whole chunks), plus the masked-node count per chunk.  ~10 MB at 513^2,
// written once and read by k_response from L2.
template <int NB>
__global__ void __launch_bounds__(1024) k_basis(const double* __restrict__ psi, const uint8_t* __restrict__ inlim,
                                               const double* __restrict__ axbd, int nw, int nh, double rmin,
                                               double dr, double cell, BasisParams bp, int gc, long long ldb,
                                               double* __restrict__ Bm, double* __restrict__ cnt_part) {
    griddep();
    __shared__ int cnt_s[32];
    const int n = nw * nh;
    const int g0 = blockIdx.x * gc;
    const double pa = axbd[0], pb = axbd[1];
    int cnt = 0;
    for (int q = threadIdx.x; q < gc; q += blockDim.x) {
        const int g = g0 + q;
        double f[NB];
#pragma unroll
        for (int k = 0; k < NB; ++k) f[k] = 0.0;
        double h;
        if (g < n && node_psihat(psi, inlim, g, pa, pb, h)) {
            basis_eval<NB>(bp, h, grid_coord(rmin, g / nh, dr), f);
            ++cnt;
        }
#pragma unroll
        for (int k = 0; k < NB; ++k) Bm[k * ldb + g] = cell * f[k];
    }
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int wc = __reduce_add_sync(0xffffffffu, cnt);
    if (lane == 0) cnt_s[warp] = wc;
    __syncthreads();
    if (threadIdx.x == 0) {
        int t = 0;
        for (int q = 0; q < (int)(blockDim.x >> 5); ++q) t += cnt_s[q];
        cnt_part[blockIdx.x] = (double)t;
    }
}

// Grid (chunk of `gc` nodes) x (group of 8*MB diagnostic rows).  The CTA stages the chunk's
// basis values in shared memory, permuted so that the 4 values a lane needs (nodes q..q+3) are
// two 16-byte words at stride 512 B across lanes (conflict-free).  Each warp streams MB Gd rows:
// per step it issues all 2*MB 256-bit loads (2 positions of 128 nodes, 192-256 B per thread in
// flight), then does the 2*MB*NB*4 FMAs; the MB x NB dot products are reduced once per chunk
// with a fixed butterfly.  Every Gd byte is read from HBM exactly once.
__device__ __forceinline__ int bperm(int q) {  // node q of a chunk -> permuted shared offset (per k)
    const int blk = q >> 7, lane = (q >> 2) & 31, h = (q >> 1) & 1, w = q & 1;
    return (blk << 7) + (h << 6) + (lane << 1) + w;
}

// Fused basis (fb.on): instead of staging Bm written by a separate k_basis launch, each CTA evaluates
// the basis of its own chunk from psi (after the wait on the predecessor that produced psi_axis /
// psi_bdry), stores it in the staged layout and writes Bm for the current kernel, plus the chunk's
// masked-node count: one launch less per iteration on the critical path.
struct FusedBasis {
    int on;
    const double* psi;
    const uint8_t* inlim;
    const double* axbd;
    int nh;
    double rmin, dr, cell;
    BasisParams bp;
    double* Bm;        // written: [NB][ldb]
    double* cnt_part;  // written: [nchunk]
};

template <int NB, int MB, int NP>
__global__ void __launch_bounds__(256, 2) k_response(const double* __restrict__ Gd, long long S, int nrows, int n,
                                                     const double* __restrict__ Bm, long long ldb, int gc,
                                                     double* __restrict__ part, FusedBasis fb) {
    // NP = rounds of MB row loads kept in a register ring: the warp's (row block, position) steps
    // form one flat sequence, and step s + NP - 1 is requested before step s is consumed, across
    // row-block boundaries (the first steps before the basis staging and the predecessor wait:
    // Gd is constant).
    extern __shared__ __align__(16) double Bs[];  // [NB][gc] permuted
    const int c = blockIdx.x;
    const int g0 = c * gc;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int qend = min(gc, n - g0);  // valid nodes; a 4-wide load may read up to 3 zero pads
    const int npos = (qend + 127) >> 7;  // 128-node positions of this chunk
    if (gridDim.y > 1) {  // small grids: blockIdx.y splits the rows (whole MB-row blocks) so that enough
        // CTAs stream; every (row, chunk) partial is still written by exactly one CTA.  Folded into
        // the row base once, so the streaming loop is the unsplit one.
        const int rbpc = ((nrows + MB - 1) / MB + gridDim.y - 1) / gridDim.y;
        const int r0 = blockIdx.y * rbpc * MB;
        Gd += (long long)r0 * S;
        part += (long long)r0 * NB * gridDim.x;
        nrows = max(0, min(nrows - r0, rbpc * MB));
    }
    const int nmb = (nrows + MB - 1) / MB;
    const int nwarps = (int)(blockDim.x >> 5);
    const int nmb_w = warp < nmb ? (nmb - warp + nwarps - 1) / nwarps : 0;  // row blocks warp, warp+8, ...
    const int nsteps = nmb_w * npos;
    // the prefetch cursor (row block lj, position lp) runs NP - 1 steps ahead of the consumer
    int lj = 0, lp = 0;
    auto load_step = [&](d4 (&x)[MB]) {
        const int row0 = (warp + lj * nwarps) * MB;
        const int q = lp * 128 + 4 * lane;
        if (++lp == npos) { lp = 0; ++lj; }
        const bool ok = q < qend;
#pragma unroll
        for (int r = 0; r < MB; ++r) {
            const double* rp = Gd + (long long)min(row0 + r, nrows - 1) * S + g0 + q;
            x[r] = ok ? ld256_stream(rp) : d4{0.0, 0.0, 0.0, 0.0};
        }
    };
    d4 ring[NP][MB];
#pragma unroll
    for (int b = 0; b + 1 < NP; ++b)
        if (b < nsteps) load_step(ring[b]);
    griddep();
    if (fb.on) {
        __shared__ int cnt_s;
        if (threadIdx.x == 0) cnt_s = 0;
        __syncthreads();
        const double pa = fb.axbd[0], pb = fb.axbd[1];
        int cnt = 0;
        for (int q = threadIdx.x; q < gc; q += blockDim.x) {
            const int g = g0 + q;
            double f[NB];
#pragma unroll
            for (int k = 0; k < NB; ++k) f[k] = 0.0;
            double h;
            if (g < n && node_psihat(fb.psi, fb.inlim, g, pa, pb, h)) {
                basis_eval<NB>(fb.bp, h, grid_coord(fb.rmin, g / fb.nh, fb.dr), f);
                ++cnt;
            }
#pragma unroll
            for (int k = 0; k < NB; ++k) {
                const double v = fb.cell * f[k];
                Bs[k * gc + bperm(q)] = v;
                if (blockIdx.y == 0) fb.Bm[k * ldb + g] = v;
            }
        }
        cnt = __reduce_add_sync(0xffffffffu, cnt);
        if ((threadIdx.x & 31) == 0) atomicAdd(&cnt_s, cnt);
        __syncthreads();
        if (threadIdx.x == 0 && blockIdx.y == 0) fb.cnt_part[c] = (double)cnt_s;
    } else {
#pragma unroll
        for (int k = 0; k < NB; ++k)
            for (int q = 2 * threadIdx.x; q < gc; q += 2 * blockDim.x) {
                const double2 v = __ldg(reinterpret_cast<const double2*>(Bm + k * ldb + g0 + q));
                *reinterpret_cast<double2*>(Bs + k * gc + bperm(q)) = v;
            }
        __syncthreads();
    }
    double acc[MB][NB];
#pragma unroll
    for (int r = 0; r < MB; ++r)
#pragma unroll
        for (int k = 0; k < NB; ++k) acc[r][k] = 0.0;
    int pos = 0, j = 0;
#pragma unroll 1
    for (int s0 = 0; s0 < nsteps; s0 += NP) {
#pragma unroll
        for (int b = 0; b < NP; ++b) {
            const int st = s0 + b;
            if (st >= nsteps) break;
            if (st + NP - 1 < nsteps) load_step(ring[(b + NP - 1) % NP]);
#pragma unroll
            for (int k = 0; k < NB; ++k) {
                const double* bk = Bs + k * gc + pos * 128 + 2 * lane;
                const double2 b0 = *reinterpret_cast<const double2*>(bk);
                const double2 b1 = *reinterpret_cast<const double2*>(bk + 64);
                const d4 bb{b0.x, b0.y, b1.x, b1.y};
#pragma unroll
                for (int r = 0; r < MB; ++r) acc[r][k] = dot4(ring[b][r], bb, acc[r][k]);
            }
            if (++pos == npos) {  // row block done: reduce and store its MB x NB partials
                const int row0 = (warp + j * nwarps) * MB;
                if constexpr (MB * NB <= 32) {
                    // transpose reduction: V = MB NB sums over the 32 lanes in log2(32) exchange levels
                    // that halve the values per lane (2^L/2 + ... + 1 + 1 shuffles instead of 5 V)
                    constexpr int V = MB * NB;
                    constexpr int P2 = V <= 1 ? 1 : V <= 2 ? 2 : V <= 4 ? 4 : V <= 8 ? 8 : V <= 16 ? 16 : 32;
                    double v[P2];
#pragma unroll
                    for (int i = 0; i < P2; ++i) v[i] = i < V ? acc[i / NB][i % NB] : 0.0;
#pragma unroll
                    for (int h = P2 / 2, o = 16; h >= 1; h >>= 1, o >>= 1) {
                        const bool up = (lane & o) != 0;
#pragma unroll
                        for (int i = 0; i < h; ++i) {
                            const double send = up ? v[i] : v[i + h];
                            const double keep = up ? v[i + h] : v[i];
                            v[i] = keep + __shfl_xor_sync(0xffffffffu, send, o);
                        }
                    }
                    // lane l now holds value index sum_b bit(l, 4 - b) 2^(L-1-b) over the levels done;
                    // finish the sum over the lanes that still share it
                    constexpr int L = P2 == 1 ? 0 : P2 == 2 ? 1 : P2 == 4 ? 2 : P2 == 8 ? 3 : P2 == 16 ? 4 : 5;
#pragma unroll
                    for (int o = 16 >> L; o >= 1; o >>= 1) v[0] += __shfl_xor_sync(0xffffffffu, v[0], o);
                    int idx = 0;
#pragma unroll
                    for (int b = 0; b < L; ++b) idx |= ((lane >> (4 - b)) & 1) << (L - 1 - b);
                    const bool writer = (lane & ((32 >> L) - 1)) == 0;
                    if (writer && idx < V) {
                        const int r = idx / NB, k = idx % NB;
                        if (row0 + r < nrows) part[((long long)(row0 + r) * NB + k) * gridDim.x + c] = v[0];
                    }
#pragma unroll
                    for (int r = 0; r < MB; ++r)
#pragma unroll
                        for (int k = 0; k < NB; ++k) acc[r][k] = 0.0;
                } else {
#pragma unroll
                    for (int r = 0; r < MB; ++r) {
#pragma unroll
                        for (int k = 0; k < NB; ++k) {
                            const double v = warp_sum(acc[r][k]);
                            acc[r][k] = 0.0;
                            if (lane == 0 && row0 + r < nrows) part[((long long)(row0 + r) * NB + k) * gridDim.x + c] = v;
                        }
                    }
                }
                pos = 0;
                ++j;
            }
        }
    }
}

// out[r][k] = sum over chunks (partials stored chunk-fastest): one warp per output, lanes take
// chunks lane, lane+32, ... and a fixed butterfly combines them => deterministic.  The total
// masked-node count decides EFIT_ST_NOPLASMA.
__global__ void k_resp_reduce(const double* __restrict__ part, const double* __restrict__ cnt_part, int nchunk,
                              int ncnt, int total, double* __restrict__ out, int* status) {
    griddep();
    const int w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
    if (w < total) {
        const double* p = part + (long long)w * nchunk;
        double s = 0.0;
        for (int c = lane; c < nchunk; c += 32) s += p[c];
        s = warp_sum(s);
        if (lane == 0) out[w] = s;
    }
    if (blockIdx.x == 0 && threadIdx.x < 32) {
        double cnt = 0.0;
        for (int c = lane; c < ncnt; c += 32) cnt += cnt_part[c];
        cnt = warp_sum(cnt);
        if (lane == 0 && cnt == 0.0) atomicOr(status, EFIT_ST_NOPLASMA);
    }
}

// CTAs per chunk along the row blocks, for small grids only (each split CTA re-evaluates its chunk's
// basis): up to 2 CTAs per SM, >= 8 row blocks (one per warp) per CTA, and no split unless it at
// least triples the CTA count (measured: a 2-way split loses at 257^2 and 513^2, wins at 65^2/129^2)
static unsigned resp_row_split(const Ctx& c, int mb, int nrows) {
    const int nmb = (nrows + mb - 1) / mb;
    int ry = (2 * kNumSMs) / c.t.resp_nchunk;
    const int cap = (nmb + 7) / 8;
    if (ry > cap) ry = cap;
    return (unsigned)(ry < 3 ? 1 : ry);
}

template <int NB>
static void launch_resp_nb(Ctx& c, const double* psi, double* part, cudaStream_t s, int nrows, bool prepare) {
    static_assert(resp_np(NB, 1) >= 1, "positions per step");
    const int gc = c.t.resp_gc;
    const size_t smem = sizeof(double) * NB * gc;
    const long long ldb = (long long)c.t.resp_nchunk * gc;
    FusedBasis fb{c.resp_fuse ? 1 : 0, psi, mask_of(c), c.axbd, c.nh, c.rmin, c.dr, c.dr * c.dz, basis_params(c),
                  c.bmat, c.resp_cnt};
    if (!prepare && !c.resp_fuse) {
        BasisParams bp = basis_params(c);
        launch_pdl(k_basis<NB>, dim3(c.t.resp_nchunk), dim3(gc <= 1024 ? gc : 1024), 0, s, psi, mask_of(c), c.axbd, c.nw, c.nh, c.rmin, c.dr, c.dr * c.dz, bp,
                                                    gc, ldb, c.bmat, c.resp_cnt);
    }
    int mb = c.t.resp_mb;
#define EFIT_RESP_LAUNCH(MBV)                                                                              \
    do {                                                                                                   \
        auto kern = k_response<NB, MBV, resp_np(NB, MBV)>;                                                \
        if (prepare) { raise_smem_limit((const void*)kern, smem); break; }                               \
        dim3 grid(c.t.resp_nchunk, resp_row_split(c, MBV, nrows));                                       \
        launch_pdl(kern, dim3(grid), dim3(256), smem, s, c.Gd, c.S, nrows, c.nw * c.nh, c.bmat, ldb, gc, part, fb);           \
    } while (0)
    if (mb >= 4) EFIT_RESP_LAUNCH(4);
    else if (mb == 3) EFIT_RESP_LAUNCH(3);
    else if (mb == 2) EFIT_RESP_LAUNCH(2);
    else EFIT_RESP_LAUNCH(1);
#undef EFIT_RESP_LAUNCH
}

static cudaError_t response_impl(Ctx& c, const double* psi, double* resp_rows, cudaStream_t s, bool prepare) {
    const int nrows = c.m_hi - c.m_lo;
    if (nrows <= 0) return cudaSuccess;
    if (c.resp_mma && !prepare) {  // the tensor-core contraction with a batch of one slice
        cudaError_t e = launch_basis(c, psi, s);
        if (e) return e;
        Ctx* self = &c;
        if ((e = launch_response_batch(c, 1, &self, s))) return e;
        return launch_resp_reduce_batch(c, c.respb_nchunk, resp_rows, s);
    }
    switch (c.nb) {
#define EFIT_NB_CASE(V) case V: launch_resp_nb<V>(c, psi, c.resp_part, s, nrows, prepare); break;
        EFIT_NB_CASE(1) EFIT_NB_CASE(2) EFIT_NB_CASE(3) EFIT_NB_CASE(4) EFIT_NB_CASE(5) EFIT_NB_CASE(6)
        EFIT_NB_CASE(7) EFIT_NB_CASE(8) EFIT_NB_CASE(9) EFIT_NB_CASE(10) EFIT_NB_CASE(11) EFIT_NB_CASE(12)
        EFIT_NB_CASE(13) EFIT_NB_CASE(14) EFIT_NB_CASE(15) EFIT_NB_CASE(16) EFIT_NB_CASE(17) EFIT_NB_CASE(18)
        EFIT_NB_CASE(19) EFIT_NB_CASE(20) EFIT_NB_CASE(21) EFIT_NB_CASE(22) EFIT_NB_CASE(23) EFIT_NB_CASE(24)
#undef EFIT_NB_CASE
        default: return cudaErrorInvalidValue;
    }
    cudaError_t e = cudaGetLastError();
    if (e || prepare) return e;
    const int total = nrows * c.nb;
    launch_pdl(k_resp_reduce, dim3((total + 7) / 8), dim3(256), 0, s, c.resp_part, c.resp_cnt, c.t.resp_nchunk,
               c.t.resp_nchunk, total, resp_rows,
                                                  c.status);
    return cudaGetLastError();
}

cudaError_t launch_response(Ctx& c, const double* psi, double* resp_rows, cudaStream_t s) {
    return response_impl(c, psi, resp_rows, s, false);
}

// ------------------------------------------------------------ multi-slice response (tensor cores)
//
// S time slices' response matrices in one pass over Gd:
//   R_s[m][k] = sum_g Gd[m][g] B_s[k][g],
// a product of Gd (rows m x N^2 nodes) with the S*NB basis columns of all slices -> DMMA m8n8k4
// exactly as k_bnd_tb_mma: lane (g, k4) streams Gd[8o + g][g0 + 16j + 4k4 .. +3] (one 256-bit
// streaming load; warp octet o = blockIdx.y * 8 + warp) and takes its B values from the staged
// basis columns (column 8bl + g = slice-major s*NB + k, zero past S*NB), 256-bit shared loads with
// rows padded by 2 doubles.  C stays in registers for the whole chunk; lane writes
// (row 8o + g, columns 8bl + 2k4, +1) to the partials of the owning slices.
struct RespBatchIO {
    const double* B[kMaxSlices];  // slice basis matrices [NB][ldb] (k_basis)
    double* part[kMaxSlices];     // slice partials [row][k][chunk]
};

#ifndef EFIT_RESPB_MINB
#define EFIT_RESPB_MINB 2
#endif
template <int NBLK, int NP>
__global__ void __launch_bounds__(256, EFIT_RESPB_MINB) k_response_mma(const double* __restrict__ Gd, long long S, int nrows, int n,
                                                        int nb, int ncol, long long ldb, RespBatchIO io, int nchunk) {
    constexpr int gc = kRespBatchGc, ldx = kRespBatchGc + 2, nstep = kRespBatchGc / 16;
    static_assert(nstep % NP == 0, "ring depth divides the steps");
    extern __shared__ __align__(16) double bsm[];  // [8 NBLK columns][ldx]
    const int c = blockIdx.x;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, k4 = lane & 3;
    const long long g0 = (long long)c * gc;
    const int row = (blockIdx.y * 8 + warp) * 8 + g;
    const bool okr = row < nrows;
    const double* tp = Gd + (long long)min(row, nrows - 1) * S + g0 + 4 * k4;
    auto load = [&](d4& a, int j) {
        const bool ok = okr && g0 + 16 * j + 4 * k4 < n;
        a = ok ? ld256_stream(tp + 16 * j) : d4{0.0, 0.0, 0.0, 0.0};
    };
    d4 ring[NP];
#pragma unroll
    for (int b = 0; b + 1 < NP; ++b) load(ring[b], b);  // Gd is constant: before the wait
    // staging: one bulk (TMA 1-D) copy per basis column, all in flight at once on one mbarrier;
    // padding columns and nodes past ldb (basis matrices are zero-padded to ldb) are zeroed
    __shared__ __align__(8) unsigned long long bar;
    const int nvalid = (int)min((long long)gc, ldb - g0);
    if (threadIdx.x == 0) mbar_init(&bar, 1);
    __syncthreads();
    griddep();
    if (threadIdx.x == 0) {
        mbar_expect_tx(&bar, (unsigned)(sizeof(double) * ncol * nvalid));
        for (int col = 0; col < ncol; ++col) {
            const int sl = col / nb, k = col - sl * nb;
            bulk_g2s(bsm + col * ldx, io.B[sl] + (long long)k * ldb + g0, (unsigned)(sizeof(double) * nvalid), &bar);
        }
    }
    for (int q = threadIdx.x; q < 8 * NBLK * gc; q += blockDim.x) {
        const int col = q / gc, e = q - col * gc;
        if (col >= ncol || e >= nvalid) bsm[col * ldx + e] = 0.0;
    }
    mbar_wait(&bar, 0);
    __syncthreads();
    if ((blockIdx.y * 8 + warp) * 8 >= nrows) return;  // octet past the last row (warp-uniform)
    // two accumulator sets per column block (k-substeps x, y | z, w): twice the independent DMMA
    // chains per warp; summed once at the end
    double acc[NBLK][2][2];
#pragma unroll
    for (int b = 0; b < NBLK; ++b) { acc[b][0][0] = acc[b][0][1] = acc[b][1][0] = acc[b][1][1] = 0.0; }
#pragma unroll 1
    for (int j0 = 0; j0 < nstep; j0 += NP) {
#pragma unroll
        for (int b = 0; b < NP; ++b) {
            const int j = j0 + b;
            if (j + NP - 1 < nstep) load(ring[(b + NP - 1) % NP], j + NP - 1);
#pragma unroll
            for (int bl = 0; bl < NBLK; ++bl) {
                const d4 xb = lds256(bsm + (8 * bl + g) * ldx + 16 * j + 4 * k4);
                dmma884(acc[bl][0][0], acc[bl][0][1], ring[b].x, xb.x);
                dmma884(acc[bl][1][0], acc[bl][1][1], ring[b].z, xb.z);
                dmma884(acc[bl][0][0], acc[bl][0][1], ring[b].y, xb.y);
                dmma884(acc[bl][1][0], acc[bl][1][1], ring[b].w, xb.w);
            }
        }
    }
    if (!okr) return;
#pragma unroll
    for (int bl = 0; bl < NBLK; ++bl)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int col = 8 * bl + 2 * k4 + h;
            if (col < ncol) {
                const int sl = col / nb, k = col - sl * nb;
                io.part[sl][((long long)row * nb + k) * nchunk + c] = acc[bl][0][h] + acc[bl][1][h];
            }
        }
}

// k_basis of one slice (basis matrix + masked-node counts for this iteration's psi)
cudaError_t launch_basis(Ctx& c, const double* psi, cudaStream_t s) {
    const int gc = c.t.resp_gc;
    const long long ldb = (long long)c.t.resp_nchunk * gc;
    BasisParams bp = basis_params(c);
    switch (c.nb) {
#define EFIT_NB_CASE(V)                                                                                              \
    case V:                                                                                                          \
        return launch_pdl(k_basis<V>, dim3(c.t.resp_nchunk), dim3(gc <= 1024 ? gc : 1024), 0, s, psi, mask_of(c), c.axbd, \
                          c.nw, c.nh, c.rmin, c.dr, c.dr * c.dz, bp, gc, ldb, c.bmat, c.resp_cnt);
        EFIT_NB_CASE(1) EFIT_NB_CASE(2) EFIT_NB_CASE(3) EFIT_NB_CASE(4) EFIT_NB_CASE(5) EFIT_NB_CASE(6)
        EFIT_NB_CASE(7) EFIT_NB_CASE(8) EFIT_NB_CASE(9) EFIT_NB_CASE(10) EFIT_NB_CASE(11) EFIT_NB_CASE(12)
        EFIT_NB_CASE(13) EFIT_NB_CASE(14) EFIT_NB_CASE(15) EFIT_NB_CASE(16) EFIT_NB_CASE(17) EFIT_NB_CASE(18)
        EFIT_NB_CASE(19) EFIT_NB_CASE(20) EFIT_NB_CASE(21) EFIT_NB_CASE(22) EFIT_NB_CASE(23) EFIT_NB_CASE(24)
#undef EFIT_NB_CASE
        default: return cudaErrorInvalidValue;
    }
}

bool response_batch_ok(const Ctx& c, int nslice) { return nslice * c.nb <= 8 * kRespBatchMaxBlk; }

#ifndef EFIT_RESPB_NP
#define EFIT_RESPB_NP 8
#endif
constexpr int kRespMmaNP = EFIT_RESPB_NP;
// ring depth: the accumulators of 5 column blocks (20 doubles) leave room for 4 steps in flight
constexpr int resp_mma_np(int nblk) { return nblk >= 5 ? 4 : kRespMmaNP; }

// one pass over Gd for all slices (after every slice's k_basis)
cudaError_t launch_response_batch(Ctx& c, int nslice, Ctx* const* slices, cudaStream_t s) {
    const int nrows = c.m_hi - c.m_lo;
    if (nrows <= 0) return cudaSuccess;
    RespBatchIO io;
    for (int k = 0; k < kMaxSlices; ++k) { io.B[k] = nullptr; io.part[k] = nullptr; }
    for (int k = 0; k < nslice; ++k) { io.B[k] = slices[k]->bmat; io.part[k] = slices[k]->resp_part; }
    const int ncol = nslice * c.nb;
    const long long ldb = (long long)c.t.resp_nchunk * c.t.resp_gc;
    const dim3 grid((unsigned)c.respb_nchunk, (unsigned)((nrows + 63) / 64));
    const int n = c.nw * c.nh;
    const int nblk = (ncol + 7) / 8;
    switch (nblk) {
#define EFIT_RB(V)                                                                                                 \
    case V:                                                                                                        \
        return launch_pdl(k_response_mma<V, resp_mma_np(V)>, grid, dim3(256), sizeof(double) * 8 * V * (kRespBatchGc + 2), s, \
                          (const double*)c.Gd, c.S, nrows, n, c.nb, ncol, ldb, io, c.respb_nchunk);
        EFIT_RB(1) EFIT_RB(2) EFIT_RB(3) EFIT_RB(4) EFIT_RB(5)
#undef EFIT_RB
        default: return cudaErrorInvalidValue;
    }
}

// per-slice chunk sums of the batched partials -> the slice's response rows (+ its NOPLASMA check)
cudaError_t launch_resp_reduce_batch(Ctx& q, int nchunk, double* resp_rows, cudaStream_t s) {
    const int total = (q.m_hi - q.m_lo) * q.nb;
    if (total <= 0) return cudaSuccess;
    return launch_pdl(k_resp_reduce, dim3((total + 7) / 8), dim3(256), 0, s, q.resp_part, q.resp_cnt, nchunk,
                      q.t.resp_nchunk, total, resp_rows, q.status);
}

// ================================================================================ least squares

// Weighted least squares by CholeskyQR2 (Yamamoto, Nakatsukasa, Yanagisawa & Fukaya,
// ETNA 2015): rows scaled by 1/sigma, columns to unit 2-norm (A), then
//   G1 = A^T A = R1^T R1,  Q1 = A R1^-1,  G2 = Q1^T Q1 = R2^T R2  (so A = (Q1 R2^-1)(R2 R1)),
//   c_hat = R1^-1 R2^-1 R2^-T (Q1^T b),  c = c_hat / column scale,
// chi2 = sum((meas - resp c)/sigma)^2 from the unscaled system.  Backward stable for
// cond(A) << eps^-1/2 ~ 1e8 (the synthetic bases: 3.6e3 .. 1.4e7).  Beyond that the first Cholesky
// breaks down; the kernels then fall back to shifted CholeskyQR3 (Fukaya, Kannan, Nakatsukasa,
// Yamamoto & Yanagisawa, SISC 2020): R0 = chol(A^T A + s I), s = 11 (nd nb + nb(nb+1)) u ||A||^2
// (||A||_2^2 <= nb for unit columns), A <- A R0^-1 (now cond ~ u^-1/2), then CholeskyQR2 on it and
// c_hat = R0^-1 (...) -- stable up to cond(A) ~ u^-1, the range of the oracle's Householder QR.
// Unlike Householder's chain of
// nb reflections, both Gram matrices are formed with all entries in parallel and the Q1 rows are
// independent; only the two nb x nb Cholesky factorisations and the triangular solves are serial
// (one warp).  Fixed summation orders => deterministic.  Singular if a Cholesky pivot is not
// positive or |R_kk| < 1e-13 max |R_jj|.
__device__ __forceinline__ void lsq_gram(const double* __restrict__ A, int ld, int nd, int nb, double* G) {
    // G[i*nb + j] for i <= j, one thread per entry, rows in order
    const int ne = nb * (nb + 1) / 2;
    for (int e = threadIdx.x; e < ne; e += blockDim.x) {
        int i = 0, rem = e;
        while (rem >= nb - i) { rem -= nb - i; ++i; }
        const int j = i + rem;
        double s = 0.0;
        for (int m = 0; m < nd; ++m) s = fma(A[m * ld + i], A[m * ld + j], s);
        G[i * nb + j] = s;
        G[j * nb + i] = s;
    }
}

// Upper Cholesky factor R (row-major, R[k*nb + j], j >= k) of G (overwritten), one warp.
// Returns false on a non-positive pivot.  Also stores 1/R_kk in rinv[k].
__device__ __forceinline__ bool lsq_chol(double* G, double* R, double* rinv, int nb) {
    const int lane = threadIdx.x & 31;
    for (int k = 0; k < nb; ++k) {
        const double d = G[k * nb + k];
        if (!(d > 0.0)) return false;
        const double r = sqrt(d), ir = 1.0 / r;
        for (int j = k + lane; j < nb; j += 32) R[k * nb + j] = (j == k) ? r : G[k * nb + j] * ir;
        if (lane == 0) rinv[k] = ir;
        __syncwarp();
        // trailing update, one lane per row i (its upper entries j >= i are independent updates;
        // no integer division per entry): same expression per entry as the textbook loop
        for (int i = k + 1 + lane; i < nb; i += 32) {
            const double rki = R[k * nb + i];
            for (int j = i; j < nb; ++j) {
                const double v = G[i * nb + j] - rki * R[k * nb + j];
                G[i * nb + j] = v;
                G[j * nb + i] = v;
            }
        }
        __syncwarp();
    }
    return true;
}

// Same factorisation for a compile-time NB <= 32, held in registers: lane i keeps row i of G
// (= column i, G stays symmetric), the pivot and the R row are shuffled, so the trailing update is
// NB independent shuffle + FMA pairs per step instead of shared-memory round trips.  Per entry the
// same expressions as lsq_chol (G[i][j] - R[k][i] R[k][j]), hence the same bits.
template <int NB>
__device__ __forceinline__ bool lsq_chol_warp(const double* G, double* R, double* rinv) {
    static_assert(NB <= 32, "one lane per row");
    const int lane = threadIdx.x & 31;
    double g[NB];
#pragma unroll
    for (int j = 0; j < NB; ++j) g[j] = lane < NB ? G[lane * NB + j] : 0.0;
    // the pivot loop is not unrolled: one copy of the step's code, reused NB times (an unrolled NB = 20
    // factorisation is ~2.5k instructions executed once per iteration, fetched cold: ~100k cycles);
    // g[k] (runtime k) is selected from the register array, the update predicated on j > k
#pragma unroll 1
    for (int k = 0; k < NB; ++k) {
        double gk = 0.0;
#pragma unroll
        for (int j = 0; j < NB; ++j) gk = (j == k) ? g[j] : gk;
        const double d = __shfl_sync(0xffffffffu, gk, k);
        if (!(d > 0.0)) return false;
        const double r = sqrt(d), ir = 1.0 / r;
        const double rki = gk * ir;  // R[k][lane] for lane > k
        if (lane == k) {
            R[k * NB + k] = r;
            rinv[k] = ir;
        } else if (lane > k && lane < NB) {
            R[k * NB + lane] = rki;
        }
#pragma unroll
        for (int j = 0; j < NB; ++j) {
            const double rkj = __shfl_sync(0xffffffffu, rki, j);
            if (j > k) g[j] = g[j] - rki * rkj;
        }
    }
    __syncwarp();
    return true;
}

// row m of A (in place): a <- a R^-1  (forward substitution with the upper factor)
__device__ __forceinline__ void lsq_rsolve_rows(double* A, int ld, int nd, int nb, const double* R, const double* rinv) {
    for (int m = threadIdx.x; m < nd; m += blockDim.x) {
        double* a = A + m * ld;
        for (int j = 0; j < nb; ++j) {
            double s = a[j];
            for (int i = 0; i < j; ++i) s = fma(-a[i], R[i * nb + j], s);
            a[j] = s * rinv[j];
        }
    }
}

// NBT > 0: the basis count as a compile-time constant (loops over it unroll, the final triangular
// solves run one lane per unknown and add the back-substitution terms from the last unknown down);
// NBT = 0: runtime nb, serial solves adding them in ascending order.  The two paths therefore agree
// to rounding, not bit for bit (each is deterministic; both are parity-tested against the oracle).
template <int NBT>
__global__ void __launch_bounds__(256) k_lsq(const double* __restrict__ resp, const double* __restrict__ meas,
                                             const double* __restrict__ sigma, int nd, int nb_arg,
                                             double* __restrict__ coef, double* __restrict__ chi2, int* status) {
    const int nb = NBT > 0 ? NBT : nb_arg;
    extern __shared__ __align__(16) double sm[];
    const int ld = nb | 1;                         // odd row stride: conflict-free column walks
    double* A = sm;                                // [nd][ld] scaled rows
    double* b = A + (size_t)nd * ld;               // [nd]
    double* isg = b + nd;                          // [nd] 1/sigma
    double* G = isg + nd;                          // [nb][nb]
    double* R1 = G + nb * nb;                      // [nb][nb]
    double* R2 = R1 + nb * nb;                     // [nb][nb]
    double* r1i = R2 + nb * nb;                    // [32]
    double* r2i = r1i + 32;                        // [32]
    double* sc = r2i + 32;                         // [32] column scales
    double* z = sc + 32;                           // [32]
    double* red = z + 32;                          // [16] chi2 partials
    double* R0 = red + 32;                         // [nb][nb] shifted pass (fallback)
    double* r0i = R0 + nb * nb;                    // [32]
    __shared__ int s_sing, s_shift;
    griddep();
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nwarp = blockDim.x >> 5;
    if (tid == 0) { s_sing = 0; s_shift = 0; }
    for (int m = tid; m < nd; m += blockDim.x) {
        const double is = 1.0 / sigma[m];
        isg[m] = is;
        for (int k = 0; k < nb; ++k) A[m * ld + k] = resp[(size_t)m * nb + k] * is;
        b[m] = meas[m] * is;
    }
    __syncthreads();
    for (int k = warp; k < nb; k += nwarp) {  // column 2-norms
        double s = 0.0;
        for (int m = lane; m < nd; m += 32) s = fma(A[m * ld + k], A[m * ld + k], s);
        s = sqrt(warp_sum(s));
        if (lane == 0) sc[k] = s;
    }
    __syncthreads();
    for (int e = tid; e < nd * nb; e += blockDim.x) {
        const int m = e / nb, k = e - (e / nb) * nb;
        const double s = sc[k];
        A[m * ld + k] = s > 0.0 ? A[m * ld + k] / s : 0.0;
    }
    __syncthreads();
    // pass 1: G1 = A^T A, R1, Q1 = A R1^-1
    lsq_gram(A, ld, nd, nb, G);
    __syncthreads();
    if (warp == 0) {
        bool ok;
        if constexpr (NBT > 0) ok = lsq_chol_warp<NBT>(G, R1, r1i);
        else ok = lsq_chol(G, R1, r1i, nb);
        if (!ok && lane == 0) s_shift = 1;
    }
    __syncthreads();
    if (s_shift) {  // cond(A) beyond ~1e8: shifted CholeskyQR3 (see above)
        if (NBT == 0) {  // lsq_chol factorised G in place: form it again (lsq_chol_warp only read it)
            lsq_gram(A, ld, nd, nb, G);
            __syncthreads();
        }
        if (warp == 0) {
            const double shift = 11.0 * ((double)nd * nb + (double)nb * (nb + 1)) * 0x1p-53 * nb;
            for (int k = lane; k < nb; k += 32) G[k * nb + k] += shift;
            __syncwarp();
            bool ok;
            if constexpr (NBT > 0) ok = lsq_chol_warp<NBT>(G, R0, r0i);
            else ok = lsq_chol(G, R0, r0i, nb);
            if (!ok && lane == 0) s_sing = 1;
        }
        __syncthreads();
        if (!s_sing) lsq_rsolve_rows(A, ld, nd, nb, R0, r0i);
        __syncthreads();
        if (!s_sing) lsq_gram(A, ld, nd, nb, G);
        __syncthreads();
        if (warp == 0 && !s_sing) {
            bool ok;
            if constexpr (NBT > 0) ok = lsq_chol_warp<NBT>(G, R1, r1i);
            else ok = lsq_chol(G, R1, r1i, nb);
            if (!ok && lane == 0) s_sing = 1;
        }
        __syncthreads();
    }
    if (!s_sing) lsq_rsolve_rows(A, ld, nd, nb, R1, r1i);
    __syncthreads();
    // pass 2: G2 = Q1^T Q1, R2, z = Q1^T b
    if (!s_sing) lsq_gram(A, ld, nd, nb, G);
    for (int k = warp; k < nb; k += nwarp) {
        double s = 0.0;
        for (int m = lane; m < nd; m += 32) s = fma(A[m * ld + k], b[m], s);
        s = warp_sum(s);
        if (lane == 0) z[k] = s;
    }
    __syncthreads();
    if (warp == 0 && !s_sing) {
        bool ok;
        if constexpr (NBT > 0) ok = lsq_chol_warp<NBT>(G, R2, r2i);
        else ok = lsq_chol(G, R2, r2i, nb);
        if (!ok && lane == 0) s_sing = 1;
    }
    __syncthreads();
    if (NBT > 0 && warp == 0 && !s_sing) {
        // as below, one lane per unknown: lane j keeps z_j; each step shuffles the finished unknown
        // and the other lanes apply its term.  The forward solve adds the terms in the serial order;
        // the back solves add them from the last unknown down (fixed order => deterministic).
        constexpr int NBC = NBT > 0 ? NBT : 1;
        const int j = lane;
        const bool act = j < NBC;
        double zj = act ? z[j] : 0.0;
        // step loops not unrolled (code reuse; see lsq_chol_warp)
#pragma unroll 1
        for (int i = 0; i < NBC; ++i) {  // z <- R2^-T z
            const double zi = __shfl_sync(0xffffffffu, zj, i) * r2i[i];
            if (j == i) zj = zi;
            else if (act && j > i) zj = fma(-R2[i * NBC + j], zi, zj);
        }
#pragma unroll 1
        for (int k = NBC - 1; k >= 0; --k) {  // z <- R2^-1 z
            const double zk = __shfl_sync(0xffffffffu, zj, k) * r2i[k];
            if (j == k) zj = zk;
            else if (j < k) zj = fma(-R2[j * NBC + k], zk, zj);
        }
#pragma unroll 1
        for (int k = NBC - 1; k >= 0; --k) {  // z <- R1^-1 z
            const double zk = __shfl_sync(0xffffffffu, zj, k) * r1i[k];
            if (j == k) zj = zk;
            else if (j < k) zj = fma(-R1[j * NBC + k], zk, zj);
        }
        if (s_shift) {
#pragma unroll 1
            for (int k = NBC - 1; k >= 0; --k) {  // z <- R0^-1 z
                const double zk = __shfl_sync(0xffffffffu, zj, k) * r0i[k];
                if (j == k) zj = zk;
                else if (j < k) zj = fma(-R0[j * NBC + k], zk, zj);
            }
        }
        if (lane == 0) {
            double rmax = 0.0, rmin = DBL_MAX;
#pragma unroll
            for (int k = 0; k < NBC; ++k) {
                const double d = fabs(R1[k * NBC + k] * R2[k * NBC + k] * (s_shift ? R0[k * NBC + k] : 1.0));
                rmax = fmax(rmax, d);
                rmin = fmin(rmin, d);
                if (!(sc[k] > 0.0)) s_sing = 1;
            }
            if (!(rmin >= 1e-13 * rmax)) s_sing = 1;
        }
        if (act) z[j] = zj / sc[j];
    } else if (tid == 0 && !s_sing) {
        // z <- R2^-T z (forward), z <- R2^-1 z (back), z <- R1^-1 z (back), c = z / scale
        for (int j = 0; j < nb; ++j) {
            double s = z[j];
            for (int i = 0; i < j; ++i) s = fma(-R2[i * nb + j], z[i], s);
            z[j] = s * r2i[j];
        }
        const double* Rs[3] = {R2, R1, R0};
        const double* Ri[3] = {r2i, r1i, r0i};
        for (int t = 0; t < (s_shift ? 3 : 2); ++t)
            for (int k = nb - 1; k >= 0; --k) {
                double s = z[k];
                for (int j = k + 1; j < nb; ++j) s = fma(-Rs[t][k * nb + j], z[j], s);
                z[k] = s * Ri[t][k];
            }
        double rmax = 0.0, rmin = DBL_MAX;
        for (int k = 0; k < nb; ++k) {
            const double d = fabs(R1[k * nb + k] * R2[k * nb + k] * (s_shift ? R0[k * nb + k] : 1.0));
            rmax = fmax(rmax, d);
            rmin = fmin(rmin, d);
            if (!(sc[k] > 0.0)) s_sing = 1;
        }
        if (!(rmin >= 1e-13 * rmax)) s_sing = 1;
        for (int k = 0; k < nb; ++k) z[k] = z[k] / sc[k];
    }
    __syncthreads();
    double s = 0.0;
    for (int m = tid; m < nd; m += blockDim.x) {
        double r = meas[m];
        for (int k = 0; k < nb; ++k) r = fma(-resp[(size_t)m * nb + k], z[k], r);
        r *= isg[m];
        s = fma(r, r, s);
    }
    s = warp_sum(s);
    if (lane == 0) red[warp] = s;
    __syncthreads();
    if (tid == 0) {
        double t = 0.0;
        for (int q = 0; q < nwarp; ++q) t += red[q];
        if (s_sing) atomicOr(status, EFIT_ST_SINGULAR);
        const bool bad = (*status & (EFIT_ST_NOPLASMA | EFIT_ST_NONFINITE)) != 0 || s_sing;
        const double nanv = __longlong_as_double(0x7ff8000000000000ULL);
        *chi2 = bad ? nanv : t;
        for (int k = 0; k < nb; ++k) coef[k] = bad ? nanv : z[k];
    }
}

// Single-warp CholeskyQR2 for small bases (NB <= 8, nd <= 32*RPL): each lane keeps its RPL rows
// in registers, the NB(NB+1)/2 Gram entries are independent warp butterflies (interleaved), and the
// tiny Cholesky factorisations and triangular solves run redundantly in every lane (registers, no
// barriers).  Same arithmetic definition as k_lsq.
template <int NB>
__device__ __forceinline__ void lsq_chol_reg(const double (&G)[NB][NB], double (&R)[NB][NB], double (&ri)[NB],
                                             bool& ok) {
#pragma unroll
    for (int i = 0; i < NB; ++i)
#pragma unroll
        for (int j = 0; j < NB; ++j) R[i][j] = (j >= i) ? G[i][j] : 0.0;
#pragma unroll
    for (int k = 0; k < NB; ++k) {
        const double d = R[k][k];
        ok = ok && (d > 0.0);
        const double r = sqrt(d), ir = 1.0 / r;
        ri[k] = ir;
        R[k][k] = r;
#pragma unroll
        for (int j = k + 1; j < NB; ++j) R[k][j] *= ir;
#pragma unroll
        for (int i = k + 1; i < NB; ++i)
#pragma unroll
            for (int j = i; j < NB; ++j) R[i][j] = fma(-R[k][i], R[k][j], R[i][j]);
    }
}

template <int NB, int RPL>
__device__ __forceinline__ void lsq_gram_reg(const double (&a)[RPL][NB], double (&G)[NB][NB]) {
#pragma unroll
    for (int i = 0; i < NB; ++i)
#pragma unroll
        for (int j = i; j < NB; ++j) {
            double s = 0.0;
#pragma unroll
            for (int r = 0; r < RPL; ++r) s = fma(a[r][i], a[r][j], s);
            G[i][j] = s;
        }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1)
#pragma unroll
        for (int i = 0; i < NB; ++i)
#pragma unroll
            for (int j = i; j < NB; ++j) G[i][j] += __shfl_xor_sync(0xffffffffu, G[i][j], o);
#pragma unroll
    for (int i = 0; i < NB; ++i)
#pragma unroll
        for (int j = 0; j < i; ++j) G[i][j] = G[j][i];
}

template <int NB, int RPL>
__global__ void __launch_bounds__(32) k_lsq_warp(const double* __restrict__ resp, const double* __restrict__ meas,
                                                 const double* __restrict__ sigma, int nd,
                                                 double* __restrict__ coef, double* __restrict__ chi2, int* status) {
    const int lane = threadIdx.x;
    double a[RPL][NB], bb[RPL], is[RPL];
    // sigma and the measurements are inputs of the step (not produced by a predecessor kernel):
    // their loads and the reciprocal overlap the wait on the response reduction
#pragma unroll
    for (int r = 0; r < RPL; ++r) {
        const int m = lane + 32 * r;
        const bool ok = m < nd;
        is[r] = ok ? 1.0 / sigma[m] : 0.0;
        bb[r] = ok ? meas[m] * is[r] : 0.0;
    }
    griddep();
#pragma unroll
    for (int r = 0; r < RPL; ++r) {
        const int m = lane + 32 * r;
        const bool ok = m < nd;
#pragma unroll
        for (int k = 0; k < NB; ++k) a[r][k] = ok ? resp[(size_t)m * NB + k] * is[r] : 0.0;
    }
    double sc[NB];
#pragma unroll
    for (int k = 0; k < NB; ++k) {
        double s = 0.0;
#pragma unroll
        for (int r = 0; r < RPL; ++r) s = fma(a[r][k], a[r][k], s);
        sc[k] = s;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1)
#pragma unroll
        for (int k = 0; k < NB; ++k) sc[k] += __shfl_xor_sync(0xffffffffu, sc[k], o);
    bool ok = true;
#pragma unroll
    for (int k = 0; k < NB; ++k) {
        sc[k] = sqrt(sc[k]);
        ok = ok && (sc[k] > 0.0);
        const double isc = sc[k] > 0.0 ? 1.0 / sc[k] : 0.0;
#pragma unroll
        for (int r = 0; r < RPL; ++r) a[r][k] *= isc;
    }
    double G[NB][NB], R0[NB][NB], R1[NB][NB], R2[NB][NB], r0i[NB], r1i[NB], r2i[NB];
    lsq_gram_reg<NB, RPL>(a, G);
    bool ok1 = true;
    lsq_chol_reg<NB>(G, R1, r1i, ok1);
    const bool shifted = !ok1 && ok;  // warp-uniform: cond(A) beyond ~1e8 -> shifted CholeskyQR3
    if (shifted) {
        const double shift = 11.0 * ((double)nd * NB + (double)NB * (NB + 1)) * 0x1p-53 * NB;
#pragma unroll
        for (int k = 0; k < NB; ++k) G[k][k] += shift;
        lsq_chol_reg<NB>(G, R0, r0i, ok);
#pragma unroll
        for (int r = 0; r < RPL; ++r)  // rows <- rows R0^-1
#pragma unroll
            for (int j = 0; j < NB; ++j) {
                double s = a[r][j];
#pragma unroll
                for (int i = 0; i < j; ++i) s = fma(-a[r][i], R0[i][j], s);
                a[r][j] = s * r0i[j];
            }
        lsq_gram_reg<NB, RPL>(a, G);
        ok1 = true;
        lsq_chol_reg<NB>(G, R1, r1i, ok1);
    }
    ok = ok && ok1;
#pragma unroll
    for (int r = 0; r < RPL; ++r)  // rows <- rows R1^-1
#pragma unroll
        for (int j = 0; j < NB; ++j) {
            double s = a[r][j];
#pragma unroll
            for (int i = 0; i < j; ++i) s = fma(-a[r][i], R1[i][j], s);
            a[r][j] = s * r1i[j];
        }
    lsq_gram_reg<NB, RPL>(a, G);
    lsq_chol_reg<NB>(G, R2, r2i, ok);
    double z[NB];
#pragma unroll
    for (int k = 0; k < NB; ++k) {
        double s = 0.0;
#pragma unroll
        for (int r = 0; r < RPL; ++r) s = fma(a[r][k], bb[r], s);
        z[k] = s;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1)
#pragma unroll
        for (int k = 0; k < NB; ++k) z[k] += __shfl_xor_sync(0xffffffffu, z[k], o);
#pragma unroll
    for (int j = 0; j < NB; ++j) {  // R2^-T
        double s = z[j];
#pragma unroll
        for (int i = 0; i < j; ++i) s = fma(-R2[i][j], z[i], s);
        z[j] = s * r2i[j];
    }
#pragma unroll
    for (int k = NB - 1; k >= 0; --k) {  // R2^-1
        double s = z[k];
#pragma unroll
        for (int j = k + 1; j < NB; ++j) s = fma(-R2[k][j], z[j], s);
        z[k] = s * r2i[k];
    }
#pragma unroll
    for (int k = NB - 1; k >= 0; --k) {  // R1^-1
        double s = z[k];
#pragma unroll
        for (int j = k + 1; j < NB; ++j) s = fma(-R1[k][j], z[j], s);
        z[k] = s * r1i[k];
    }
    if (shifted) {
#pragma unroll
        for (int k = NB - 1; k >= 0; --k) {  // R0^-1
            double s = z[k];
#pragma unroll
            for (int j = k + 1; j < NB; ++j) s = fma(-R0[k][j], z[j], s);
            z[k] = s * r0i[k];
        }
    }
    double rmax = 0.0, rmin = DBL_MAX;
#pragma unroll
    for (int k = 0; k < NB; ++k) {
        const double d = fabs(R1[k][k] * R2[k][k] * (shifted ? R0[k][k] : 1.0));
        rmax = fmax(rmax, d);
        rmin = fmin(rmin, d);
        z[k] = z[k] / sc[k];
    }
    ok = ok && (rmin >= 1e-13 * rmax);
    double cs = 0.0;
#pragma unroll
    for (int r = 0; r < RPL; ++r) {
        const int m = lane + 32 * r;
        if (m < nd) {
            double res = meas[m];
#pragma unroll
            for (int k = 0; k < NB; ++k) res = fma(-resp[(size_t)m * NB + k], z[k], res);
            res *= is[r];
            cs = fma(res, res, cs);
        }
    }
    cs = warp_sum(cs);
    if (lane == 0) {
        if (!ok) atomicOr(status, EFIT_ST_SINGULAR);
        const bool bad = (*status & (EFIT_ST_NOPLASMA | EFIT_ST_NONFINITE)) != 0 || !ok;
        const double nanv = __longlong_as_double(0x7ff8000000000000ULL);
        *chi2 = bad ? nanv : cs;
#pragma unroll
        for (int k = 0; k < NB; ++k) coef[k] = bad ? nanv : z[k];
    }
}

template <int NB>
static bool launch_lsq_warp(int nd, const double* resp, const double* meas, const double* sigma, double* coef,
                            double* chi2, int* status, cudaStream_t s) {
    if (nd <= 64) launch_pdl(k_lsq_warp<NB, 2>, dim3(1), dim3(32), 0, s, resp, meas, sigma, nd, coef, chi2, status);
    else if (nd <= 128) launch_pdl(k_lsq_warp<NB, 4>, dim3(1), dim3(32), 0, s, resp, meas, sigma, nd, coef, chi2, status);
    else if (nd <= 192) launch_pdl(k_lsq_warp<NB, 6>, dim3(1), dim3(32), 0, s, resp, meas, sigma, nd, coef, chi2, status);
    else return false;
    return true;
}

static size_t lsq_smem(const Ctx& c) {
    return sizeof(double) * ((size_t)((c.nb | 1) + 2) * c.ndiag + 4 * (size_t)c.nb * c.nb + 7 * 32);
}

cudaError_t launch_lsq(Ctx& c, const double* resp, const double* meas, const double* sigma, double* coef,
                       double* chi2, cudaStream_t s) {
    size_t smem = lsq_smem(c);
    bool done = false;
    switch (c.nb) {
        case 1: done = launch_lsq_warp<1>(c.ndiag, resp, meas, sigma, coef, chi2, c.status, s); break;
        case 2: done = launch_lsq_warp<2>(c.ndiag, resp, meas, sigma, coef, chi2, c.status, s); break;
        case 3: done = launch_lsq_warp<3>(c.ndiag, resp, meas, sigma, coef, chi2, c.status, s); break;
        case 4: done = launch_lsq_warp<4>(c.ndiag, resp, meas, sigma, coef, chi2, c.status, s); break;
        case 5: done = launch_lsq_warp<5>(c.ndiag, resp, meas, sigma, coef, chi2, c.status, s); break;
        case 6: done = launch_lsq_warp<6>(c.ndiag, resp, meas, sigma, coef, chi2, c.status, s); break;
        default: break;
    }
    if (done) return cudaGetLastError();
    switch (c.nb) {
#define EFIT_LSQ_CASE(V) \
    case V: launch_pdl(k_lsq<V>, dim3(1), dim3(256), smem, s, resp, meas, sigma, c.ndiag, c.nb, coef, chi2, c.status); break;
        EFIT_LSQ_CASE(7) EFIT_LSQ_CASE(8) EFIT_LSQ_CASE(9) EFIT_LSQ_CASE(10) EFIT_LSQ_CASE(11) EFIT_LSQ_CASE(12)
        EFIT_LSQ_CASE(13) EFIT_LSQ_CASE(14) EFIT_LSQ_CASE(15) EFIT_LSQ_CASE(16) EFIT_LSQ_CASE(17) EFIT_LSQ_CASE(18)
        EFIT_LSQ_CASE(19) EFIT_LSQ_CASE(20) EFIT_LSQ_CASE(21) EFIT_LSQ_CASE(22) EFIT_LSQ_CASE(23) EFIT_LSQ_CASE(24)
#undef EFIT_LSQ_CASE
        default:
            launch_pdl(k_lsq<0>, dim3(1), dim3(256), smem, s, resp, meas, sigma, c.ndiag, c.nb, coef, chi2, c.status);
    }
    return cudaGetLastError();
}

// ================================================================================ current

template <int NB>
__device__ __forceinline__ double current_at(const double* psi, const uint8_t* inlim, int g, int nh, double pa,
                                             double pb, double rmin, double dr, double cell, const BasisParams& bp,
                                             const double* cf) {
    double h;
    if (!node_psihat(psi, inlim, g, pa, pb, h)) return 0.0;
    double f[NB];
    basis_eval<NB>(bp, h, grid_coord(rmin, g / nh, dr), f);
    double s = 0.0;
#pragma unroll
    for (int k = 0; k < NB; ++k) s = fma(cf[k], f[k], s);
    return cell * s;
}

template <int NB>
__global__ void k_current(const double* __restrict__ psi, const uint8_t* __restrict__ inlim,
                          const double* __restrict__ axbd, const double* __restrict__ coef, int nw, int nh,
                          double rmin, double dr, double cell, BasisParams bp, double* __restrict__ pcurr,
                          double* __restrict__ pflip) {
    griddep();
    const int n = nw * nh;
    const double pa = axbd[0], pb = axbd[1];
    double cf[NB];
#pragma unroll
    for (int k = 0; k < NB; ++k) cf[k] = coef[k];
    for (int g = blockIdx.x * blockDim.x + threadIdx.x; g < n; g += gridDim.x * blockDim.x) {
        const double I = current_at<NB>(psi, inlim, g, nh, pa, pb, rmin, dr, cell, bp, cf);
        pcurr[g] = I;
        if (pflip) {  // I at the vertically mirrored node, for the top-target dot products
            const int ii = g / nh, m = g - (g / nh) * nh;
            pflip[ii * nh + (nh - 1 - m)] = I;
        }
    }
}

// Fit-step current from this iteration's basis matrix (already masked and scaled by dR dZ):
// I_g = sum_k c_k Bm[k][g]  -- no second basis evaluation.
// SYM modes: the current kernel also writes the staged layouts of k_sym_pack (interior rows only;
// the zero padding of the last 8-row block is set once at init), so the fit step needs no pack launch.
struct SymPackOut {
    double* q;  // symq (nullptr: no packing)
    double* p;  // symp
    int narr, nhp, ni;
};

template <int NB>
__global__ void k_current_from_basis(const double* __restrict__ Bm, long long ldb, const double* __restrict__ coef,
                                     int nw, int nh, double* __restrict__ pcurr, double* __restrict__ pflip,
                                     SymPackOut sp) {
    const int n = nw * nh;
    const int g = blockIdx.x * blockDim.x + threadIdx.x;  // one node per thread (grid covers n)
    // the basis values were written by k_response, three kernels back (complete before the
    // predecessor started), so they are loaded before the wait on the predecessor (the LSQ)
    double b[NB];
#pragma unroll
    for (int k = 0; k < NB; ++k) b[k] = g < n ? Bm[k * ldb + g] : 0.0;
    griddep();
    if (g >= n) return;
    double I = 0.0;
#pragma unroll
    for (int k = 0; k < NB; ++k) I = fma(coef[k], b[k], I);
    pcurr[g] = I;
    const int ii = g / nh, m = g - (g / nh) * nh;
    pflip[ii * nh + (nh - 1 - m)] = I;
    const int r = ii - 1;
    if (sp.q && r >= 0 && r < sp.ni) {  // symq[B][arr][h][m][qh][w], symp[B][arr][p][m] (k_sym_pack)
        const int B = r >> 3, q = r & 7, qh = q >> 2, h = (q >> 1) & 1, w = q & 1;
        const long long qb = (long long)B * 16 * nh + (long long)h * 4 * nh + 2 * qh + w;
        const long long pb = (long long)B * 16 * sp.nhp + (long long)q * sp.nhp;
        sp.q[qb + 4LL * m] = I;
        sp.p[pb + m] = I;
        if (sp.narr == 2) {  // F[ii][nh-1-m] = I
            const int mf = nh - 1 - m;
            sp.q[qb + 8LL * nh + 4LL * mf] = I;
            sp.p[pb + 8LL * sp.nhp + mf] = I;
        }
    }
}

cudaError_t launch_current(Ctx& c, const double* psi, const double* coef, double* pcurr, bool pair,
                           cudaStream_t s) {
    BasisParams bp = basis_params(c);
    if (pair) {  // fit step: the basis matrix of this iteration is in c.bmat (k_basis ran in response)
        const int n = c.nw * c.nh;
        SymPackOut sp{nullptr, nullptr, 0, c.nhp, c.ni};
        if (c.sym && c.sym_tile_hi > c.sym_tile_lo && c.ni > 0) {
            sp.q = c.symq;
            sp.p = c.symp;
            sp.narr = c.t.sym_nmc == 1 ? 1 : 2;
        }
        const long long ldb = (long long)c.t.resp_nchunk * c.t.resp_gc;
        switch (c.nb) {
#define EFIT_NB_CASE(V) \
    case V: launch_pdl(k_current_from_basis<V>, dim3((n + 255) / 256), dim3(256), 0, s, c.bmat, ldb, coef, c.nw, c.nh, pcurr, c.pflip, sp); break;
            EFIT_NB_CASE(1) EFIT_NB_CASE(2) EFIT_NB_CASE(3) EFIT_NB_CASE(4) EFIT_NB_CASE(5) EFIT_NB_CASE(6)
            EFIT_NB_CASE(7) EFIT_NB_CASE(8) EFIT_NB_CASE(9) EFIT_NB_CASE(10) EFIT_NB_CASE(11) EFIT_NB_CASE(12)
            EFIT_NB_CASE(13) EFIT_NB_CASE(14) EFIT_NB_CASE(15) EFIT_NB_CASE(16) EFIT_NB_CASE(17) EFIT_NB_CASE(18)
            EFIT_NB_CASE(19) EFIT_NB_CASE(20) EFIT_NB_CASE(21) EFIT_NB_CASE(22) EFIT_NB_CASE(23) EFIT_NB_CASE(24)
#undef EFIT_NB_CASE
            default: return cudaErrorInvalidValue;
        }
        return cudaGetLastError();
    }
    const int n = c.nw * c.nh;
    const int blocks = (n + 255) / 256;
    double* fl = pair ? c.pflip : nullptr;
    switch (c.nb) {
#define EFIT_NB_CASE(V) \
    case V: launch_pdl(k_current<V>, dim3(blocks), dim3(256), 0, s, psi, mask_of(c), c.axbd, coef, c.nw, c.nh, c.rmin, c.dr, c.dr * c.dz, bp, pcurr, fl); break;
        EFIT_NB_CASE(1) EFIT_NB_CASE(2) EFIT_NB_CASE(3) EFIT_NB_CASE(4) EFIT_NB_CASE(5) EFIT_NB_CASE(6)
        EFIT_NB_CASE(7) EFIT_NB_CASE(8) EFIT_NB_CASE(9) EFIT_NB_CASE(10) EFIT_NB_CASE(11) EFIT_NB_CASE(12)
        EFIT_NB_CASE(13) EFIT_NB_CASE(14) EFIT_NB_CASE(15) EFIT_NB_CASE(16) EFIT_NB_CASE(17) EFIT_NB_CASE(18)
        EFIT_NB_CASE(19) EFIT_NB_CASE(20) EFIT_NB_CASE(21) EFIT_NB_CASE(22) EFIT_NB_CASE(23) EFIT_NB_CASE(24)
#undef EFIT_NB_CASE
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

// ================================================================================ boundary flux

// Top/bottom targets (the second O(N^3) nest, reading Q2): for target row i,
//   psi_b(i, 0)    = sum_{ii,m} T[i][ii][m] I[ii][m]
//   psi_b(i, nh-1) = sum_{ii,m} T[i][ii][m] I[ii][nh-1-m]
// i.e. two dot products of slab T[i] with I and with the vertically mirrored I (F).  A CTA owns
// a chunk of `ch` slab entries (its I and F values staged once in shared memory, consecutive
// lanes -> consecutive 32-byte words, conflict-free) and GI slabs; every T byte is read from HBM
// exactly once with 256-bit streaming loads, UNR slabs x 2 positions (256 B per thread) in flight.
template <int GI, int UNR>
__global__ void __launch_bounds__(256, 2) k_bnd_tb(const double* __restrict__ T, long long S, int nslab,
                                                   int row_lo, int n, const double* __restrict__ Ib,
                                                   const double* __restrict__ Fb, int ch,
                                                   double* __restrict__ part) {
    griddep();
    extern __shared__ __align__(16) double sm_tb[];
    double* sI = sm_tb;        // [ch]
    double* sF = sm_tb + ch;   // [ch]
    __shared__ double red[8][2 * GI];
    const int c = blockIdx.x, grp = blockIdx.y;
    const long long e0 = (long long)c * ch;
    const int len = (int)min((long long)ch, (long long)n - e0);
    for (int q = 4 * threadIdx.x; q < ch; q += 4 * blockDim.x) {
        *reinterpret_cast<double2*>(sI + q) = __ldg(reinterpret_cast<const double2*>(Ib + e0 + q));
        *reinterpret_cast<double2*>(sI + q + 2) = __ldg(reinterpret_cast<const double2*>(Ib + e0 + q + 2));
        *reinterpret_cast<double2*>(sF + q) = __ldg(reinterpret_cast<const double2*>(Fb + e0 + q));
        *reinterpret_cast<double2*>(sF + q + 2) = __ldg(reinterpret_cast<const double2*>(Fb + e0 + q + 2));
    }
    __syncthreads();
    double a0[GI], a1[GI];
#pragma unroll
    for (int t = 0; t < GI; ++t) { a0[t] = 0.0; a1[t] = 0.0; }
    const int s0 = grp * GI;
    const int q0 = 4 * threadIdx.x, q1 = q0 + 4 * blockDim.x;  // two 4-wide positions per slab (ch = 2048)
    const bool v0 = q0 < len, v1 = q1 < len;
#pragma unroll
    for (int t = 0; t < GI; t += UNR) {
        d4 tv[UNR][2];
#pragma unroll
        for (int u = 0; u < UNR; ++u) {
            const int sl = s0 + t + u;
            const double* base = T + (long long)min(sl, nslab - 1) * S + e0;
            const bool ok = sl < nslab;
            tv[u][0] = (ok && v0) ? ld256_stream(base + q0) : d4{0.0, 0.0, 0.0, 0.0};
            tv[u][1] = (ok && v1) ? ld256_stream(base + q1) : d4{0.0, 0.0, 0.0, 0.0};
        }
        const d4 i0 = lds256(sI + q0), i1 = lds256(sI + q1);
        const d4 f0 = lds256(sF + q0), f1 = lds256(sF + q1);
#pragma unroll
        for (int u = 0; u < UNR; ++u) {
            a0[t + u] = dot4(tv[u][0], i0, a0[t + u]);
            a1[t + u] = dot4(tv[u][0], f0, a1[t + u]);
            a0[t + u] = dot4(tv[u][1], i1, a0[t + u]);
            a1[t + u] = dot4(tv[u][1], f1, a1[t + u]);
        }
    }
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
#pragma unroll
    for (int t = 0; t < GI; ++t) {
        double x = warp_sum(a0[t]);
        double y = warp_sum(a1[t]);
        if (lane == 0) { red[warp][2 * t] = x; red[warp][2 * t + 1] = y; }
    }
    __syncthreads();
    if (threadIdx.x < 2 * GI) {
        const int t = threadIdx.x >> 1, side = threadIdx.x & 1;
        const int sl = s0 + t;
        if (sl < nslab) {
            double sum = 0.0;
            for (int w = 0; w < (int)(blockDim.x >> 5); ++w) sum += red[w][threadIdx.x];
            part[((long long)(row_lo + sl) * 2 + side) * gridDim.x + c] = sum;
        }
    }
}

// Left/right targets (the printed Fig. 2 nest): for side s (slab i = 0 or nw-1),
//   psi_b(s, j) = sum_ii sum_jj T[s][ii][|j - jj|] I[ii][jj]
// (a symmetric Toeplitz product per source row ii).  A warp owns one source row ii and one
// quarter of its sources jj; lane l owns JT consecutive targets j = jt0 + JT l + a (JT odd => the
// lane stride is conflict-free in shared memory) and the whole warp steps through jj together
// (x[jj] is a broadcast).  The kernel row is staged mirrored and zero-padded, so target a at step u
// needs tx[JT l + a - u + JQ - 1]: a register window sliding by one per step with one new shared
// load, slot (a - u) mod JT resolved at compile time by unrolling by JT, and no bounds checks
// (sources zero-padded to 4*JQ).  17 FMA per 2 shared loads.  CTA = 2 rows x 4 quarters; the 8
// warps are summed in fixed order, the per-row-pair partials in pair order by k_bnd_reduce.
template <int JT>
__global__ void __launch_bounds__(256) k_bnd_lr(const double* __restrict__ Tedge, long long S,
                                                const double* __restrict__ I, int nw, int nh, int JQ,
                                                int jt_lo, double* __restrict__ part) {
    griddep();
    extern __shared__ __align__(16) double sm_lr[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int TL = 32 * JT + JQ + 1;  // mirrored row window incl. one front pad
    double* tx = sm_lr + (size_t)warp * (TL + JQ);
    double* xs = tx + TL;
    const int side = blockIdx.z, blk = blockIdx.y;
    const int ii = blk * 2 + (warp >> 2);
    const int jb0 = (warp & 3) * JQ;
    const int jt0 = (jt_lo + blockIdx.x) * 32 * JT;
    const bool live = ii < nw;
    const double* t = Tedge + (long long)side * S + (long long)(live ? ii : 0) * nh;
    const double* x = I + (long long)(live ? ii : 0) * nh;
    for (int k = lane; k < TL; k += 32) {
        double v = 0.0;
        if (live && k >= 1) {
            int d = jt0 - jb0 + (k - 1) - (JQ - 1);
            d = d < 0 ? -d : d;
            if (d < nh) v = t[d];
        }
        tx[k] = v;
    }
    for (int k = lane; k < JQ; k += 32) xs[k] = (live && jb0 + k < nh) ? x[jb0 + k] : 0.0;
    __syncwarp();
    const double* tl = tx + 1 + JT * lane + (JQ - 1);
    double w[JT], acc[JT];
#pragma unroll
    for (int a = 0; a < JT; ++a) { w[a] = tl[a]; acc[a] = 0.0; }
    for (int ub = 0; ub < JQ; ub += JT) {
#pragma unroll
        for (int u = 0; u < JT; ++u) {
            const int uu = ub + u;
            const double xv = xs[uu];
#pragma unroll
            for (int a = 0; a < JT; ++a) acc[a] = fma(w[(a - u + JT) % JT], xv, acc[a]);
            w[(2 * JT - 1 - u) % JT] = tl[-uu - 1];  // target a = 0 at step uu + 1
        }
    }
    __syncthreads();
    double* red = sm_lr;  // [8][32 JT]
#pragma unroll
    for (int a = 0; a < JT; ++a) red[warp * 32 * JT + JT * lane + a] = acc[a];
    __syncthreads();
    for (int q = threadIdx.x; q < 32 * JT; q += blockDim.x) {
        const int j = jt0 + q;
        if (j < nh) {
            double v = 0.0;
#pragma unroll
            for (int w8 = 0; w8 < 8; ++w8) v += red[w8 * 32 * JT + q];
            part[((long long)side * nh + j) * gridDim.y + blk] = v;
        }
    }
}

// psi_b in edge order from the partials: one warp per edge target, chunk-fastest partials,
// fixed lane assignment + butterfly => deterministic and independent of the rank count.
// SYM mode: top/bottom partials per (target, side, slot) from k_bnd_sym, plus the edge-row sources
// ii = 0, nw-1 through the edge slabs (reciprocity: T[i][0][m] = Tedge[0][i][m]).
// Multi-GPU (include/efit.h, "Multi-GPU"): every slot of the SYM partials is written by exactly
// one row-pair tile, i.e. by one rank, so the zero-padded partials summed over ranks are the
// world-1 partials exactly and this fixed-order reduction gives world-independent psi_b.
struct SymReduce {
    const double* part;   // nullptr: full-table mode
    int nslot;
    const double* Tedge;
    long long S;
    const double* pc;     // I  (zero-padded pcurr)
    const double* pf;     // F  (vertically mirrored)
    const double* edge;   // SYM: edge-row source sums per top/bottom target (k_sym_edge_src), or nullptr
};

// Destinations of k_bnd_reduce: left/right entries (psi_b[0, 2 nh)) to `lr` (nullptr: not
// written), top/bottom entries (psi_b[2 nh, n_edge)) to `tb` (indexed from 0; nullptr: not
// written) for target rows i in [tb_lo, tb_hi); zero_unowned writes 0 to the other rows' entries
// (the zero padding of a rank's exchange slice).
struct BndOut {
    double* lr;
    double* tb;
    int tb_lo, tb_hi, zero_unowned;
};

// SYM modes: the top/bottom targets' sums over the edge-row sources ii = 0, nw-1 (not in the half
// table), from the replicated edge slabs: out[side*(nw-2) + i-1] = sum_m T0[i][m] X[0][m] + T1[i][m] X[nw-1][m],
// X = I (bottom) or F (top).  One warp per target, every target on every rank (replicated, cheap);
// runs on the side stream under the table stream.
__global__ void k_sym_edge_src(const double* __restrict__ Tedge, long long S, const double* __restrict__ pc,
                               const double* __restrict__ pf, int nw, int nh, double* __restrict__ out) {
    griddep();
    const int w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
    const int q = w;  // 0 .. 2(nw-2)-1
    if (q >= 2 * (nw - 2)) return;
    const int side = q < nw - 2 ? 0 : 1;
    const int i = q - side * (nw - 2) + 1;
    double s = 0.0;
    const double* x0 = (side ? pf : pc);
    const double* x1 = x0 + (long long)(nw - 1) * nh;
    const double* t0 = Tedge + (long long)i * nh;
    const double* t1 = t0 + S;
    for (int m = lane; m < nh; m += 32) s = fma(t0[m], x0[m], fma(t1[m], x1[m], s));
    s = warp_sum(s);
    if (lane == 0) out[q] = s;
}

__global__ void k_bnd_reduce(const double* __restrict__ tb_part, int tb_nchunk, const double* __restrict__ lr_part,
                             int lr_nblk, int nw, int nh, int jlo, int jhi, BndOut o, SymReduce sy) {
    griddep();
    const int n_edge = 2 * nh + 2 * (nw - 2);
    const int p = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
    if (p >= n_edge) return;
    const double* src;
    int cnt;
    double s = 0.0;
    double* dst;
    if (p < 2 * nh) {
        const int side = p < nh ? 0 : 1;
        const int j = p - side * nh;
        if (!o.lr || j < jlo || j >= jhi) return;
        src = lr_part + ((long long)side * nh + j) * lr_nblk;
        cnt = lr_nblk;
        dst = o.lr + p;
    } else {
        const int q = p - 2 * nh;
        const int side = q < nw - 2 ? 0 : 1;
        const int i = q - side * (nw - 2) + 1;
        if (!o.tb) return;
        dst = o.tb + q;
        if (i < o.tb_lo || i >= o.tb_hi) {
            if (o.zero_unowned && lane == 0) *dst = 0.0;
            return;
        }
        if (sy.part) {
            src = sy.part + ((long long)(i - 1) * 2 + side) * sy.nslot;
            cnt = sy.nslot;
            if (sy.edge) {
                if (lane == 0) s = sy.edge[q];
            } else {
                const double* x0 = (side ? sy.pf : sy.pc);
                const double* x1 = x0 + (long long)(nw - 1) * nh;
                const double* t0 = sy.Tedge + (long long)i * nh;
                const double* t1 = t0 + sy.S;
                for (int m = lane; m < nh; m += 32) s = fma(t0[m], x0[m], fma(t1[m], x1[m], s));
            }
        } else {
            src = tb_part + ((long long)i * 2 + side) * tb_nchunk;
            cnt = tb_nchunk;
        }
    }
    for (int c = lane; c < cnt; c += 32) s += src[c];
    s = warp_sum(s);
    if (lane == 0) *dst = s;
}

// On-the-fly variant of k_bnd_tb: G recomputed from (R_i, R_ii, m dZ) with the same device
// function as the table build, same decomposition and summation order => bitwise equal to the
// table mode.  FP64-bound (AGM: 10 square roots per entry).
template <int GI>
__global__ void __launch_bounds__(256) k_bnd_tb_otf(int row_lo, int nslab, int nw, int nh, double rmin, double dr,
                                                    double dz, const double* __restrict__ Ib,
                                                    const double* __restrict__ Fb, int ch,
                                                    double* __restrict__ part) {
    griddep();
    extern __shared__ __align__(16) double sm_tb[];
    double* sI = sm_tb;
    double* sF = sm_tb + ch;
    __shared__ double red[8][2 * GI];
    const int n = nw * nh;
    const int c = blockIdx.x, grp = blockIdx.y;
    const long long e0 = (long long)c * ch;
    const int len = (int)min((long long)ch, (long long)n - e0);
    for (int q = threadIdx.x; q < ch; q += blockDim.x) { sI[q] = Ib[e0 + q]; sF[q] = Fb[e0 + q]; }
    __syncthreads();
    double a0[GI], a1[GI];
#pragma unroll
    for (int t = 0; t < GI; ++t) { a0[t] = 0.0; a1[t] = 0.0; }
    const int s0 = grp * GI;
    const int qs[2] = {4 * (int)threadIdx.x, 4 * (int)threadIdx.x + 4 * (int)blockDim.x};
    for (int t = 0; t < GI; ++t) {
        const int sl = s0 + t;
        if (sl >= nslab) break;
        const int i = row_lo + sl;
        const double Ri = grid_coord(rmin, i, dr);
#pragma unroll
        for (int p = 0; p < 2; ++p) {
            const int q = qs[p];
            if (q >= len) continue;
            double tv[4];
#pragma unroll
            for (int h = 0; h < 4; ++h) {
                const long long e = e0 + q + h;
                if (e < n) {
                    const int ii = (int)(e / nh), m = (int)(e - (long long)ii * nh);
                    const double Rs = grid_coord(rmin, ii, dr);
                    tv[h] = (i == ii && m == 0) ? green_self(Ri, dr, dz)
                                                : green_psi(Ri, __dmul_rn((double)m, dz), Rs, 0.0);
                } else {
                    tv[h] = 0.0;
                }
            }
            const d4 tt{tv[0], tv[1], tv[2], tv[3]};
            a0[t] = dot4(tt, lds256(sI + q), a0[t]);
            a1[t] = dot4(tt, lds256(sF + q), a1[t]);
        }
    }
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
#pragma unroll
    for (int t = 0; t < GI; ++t) {
        double x = warp_sum(a0[t]);
        double y = warp_sum(a1[t]);
        if (lane == 0) { red[warp][2 * t] = x; red[warp][2 * t + 1] = y; }
    }
    __syncthreads();
    if (threadIdx.x < 2 * GI) {
        const int t = threadIdx.x >> 1, side = threadIdx.x & 1;
        const int sl = s0 + t;
        if (sl < nslab) {
            double sum = 0.0;
            for (int w = 0; w < (int)(blockDim.x >> 5); ++w) sum += red[w][threadIdx.x];
            part[((long long)(row_lo + sl) * 2 + side) * gridDim.x + c] = sum;
        }
    }
}

// ------------------------------------------------------------ symmetric (SYM-mode) top/bottom
//
// Reciprocity G(R_i, z; R_ii, 0) = G(R_ii, z; R_i, 0) (pinned in the oracle tests)
// makes the top/bottom table symmetric in the row pair: T[i][ii][m] = T[ii][i][m].  Only the
// interior pairs with i <= ii are stored, blocked into 8 x 8 row-pair tiles (P <= Q of the 8-row
// blocks of the interior index r = i - 1), tile t = Q(Q+1)/2 + P, entry [p][m][q] (q fastest):
//   U_t[p][m][q] = G(R_i, m dZ; R_ii, 0),  i = 1 + 8P + p,  ii = 1 + 8Q + q  (0 outside).
// One streamed entry serves both directions of the pair:
//   row   target i  (bottom, top) += U I[ii][m],  U F[ii][m]     (sources ii of block Q)
//   col   target ii (bottom, top) += U I[i][m],   U F[i][m]      (sources i of block P; P < Q only)
// so every top/bottom Green's byte crosses HBM half as often as in the full-table nest.  The
// edge-row sources ii = 0, nw-1 come from the (replicated) edge slabs in the reduce kernel.

// CTA = one tile x one m-chunk, WG groups of 4 warps.  Warp w of a group streams rows p = w and
// w + 4 of the tile ([m][q], 2 x 32-byte vectors per m: lane l takes vector v = l + 32k of each row,
// i.e. m = m0 + (v >> 1) and q = 4 (l & 1) .. +3, fixed per lane), so every staged source-column
// value it reads serves two table rows; the WG groups split each row's vector range (WG = 2: 16
// warps per SM at the 128-register budget -- measured best on B200; more loads in flight per warp
// spill).  Shared memory holds the chunk's source columns I^T (and F^T) of block Q as two planes
// of 16-byte pairs (q = 4qh + {0,1} | 4qh + {2,3}; a warp's 128-bit reads are contiguous and
// conflict-free) and the tile's own rows I[i][m] (and F[i][m]) of block P (col direction; lane
// pairs read the same word), both bulk-copied (TMA 1-D, one mbarrier) from the per-iteration
// packed arrays of k_sym_pack.  MIRROR (one chunk = the whole column): F[ii][m] = I[ii][nh-1-m] is
// read from the staged I at the mirrored m, halving the staging (65.7 KB at nh = 513).  The table
// stream runs through a register ring of NBUF rounds of UNR vectors per row and lane: round r+NBUF-1
// is requested before round r is consumed, the first rounds before the staging (the table is
// constant, so also before the wait on the predecessor kernel).  Reductions: row direction = warp
// butterfly + fixed-order group sum; col direction = 16-lane butterfly (lanes with the same q set)
// + fixed-order sum over the warps.  Partials go to slot (block, chunk) of each target: row
// direction slot Q, col direction slot P, so every slot of every target is written by exactly one CTA.
#ifndef EFIT_SYM_MINB
#define EFIT_SYM_MINB 0
#endif
template <bool OTF, bool MIRROR, int UNR, int NBUF, int WG>
__global__ void __launch_bounds__(128 * WG, EFIT_SYM_MINB ? EFIT_SYM_MINB : (WG == 1 ? 3 : (WG == 2 ? 2 : 1)))
    k_bnd_sym(const double* __restrict__ U, long long tile_lo, int ni, int nh, int nmc, int mc,
              const double* __restrict__ symq, const double* __restrict__ symp, int nhp, int nslot,
              double* __restrict__ part, double rmin, double dr, double dz) {
    extern __shared__ __align__(16) double xs[];
    __shared__ double red[4 * WG][16];
    __shared__ double rrow[4 * WG][4];
    __shared__ __align__(8) unsigned long long bar;
    if (threadIdx.x == 0) mbar_init(&bar, 1);
    __syncthreads();
    const int tl = blockIdx.x / nmc, mch = blockIdx.x - tl * nmc;
    int P, Q;
    sym_tile_pq(tile_lo + tl, P, Q);
    const bool diag = P == Q;  // diagonal tile: stored in full, row direction only
    const int m0 = mch * mc, mlen = min(mc, nh - m0);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, qh = lane & 1;
    const int wr = warp & 3, grp = warp >> 2;
    const int rp0 = 8 * P + wr, rp1 = rp0 + 4;
    const int nvec = 2 * mlen;
    const int seg = WG == 1 ? nvec : (nvec / (32 * WG)) * 32;  // group g: [g seg, (g+1) seg), last to nvec
    const int vb = grp * seg, ve = grp == WG - 1 ? nvec : vb + seg;
    const double* tp0 = OTF ? nullptr : U + ((long long)tl * 64 + (long long)wr * 8) * nh + 8LL * m0;
    const double* tp1 = OTF ? nullptr : tp0 + 32LL * nh;
    // Lane addressing: vector v = k0 + 32u + lane of a row sits at tp + 4v; its staged plane
    // pair index is v itself (m = v >> 1, qh = v & 1); the mirrored plane index is
    // 2 (nh - 1 - m) + qh = 2 (nh - 1) + 2 qh - v.  Full rounds run without bounds checks.
    auto load = [&](d4 (&x0)[UNR], d4 (&x1)[UNR], int k0, bool tail) {
#pragma unroll
        for (int u = 0; u < UNR; ++u) {
            const int v = k0 + 32 * u + lane;
            const bool ok = !tail || v < ve;
            if (OTF) {
                double a4[4], b4[4];
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const int rq = 8 * Q + 4 * qh + j, m = m0 + (v >> 1);
                    a4[j] = ok ? sym_entry(rp0, rq, m, ni, rmin, dr, dz) : 0.0;
                    b4[j] = ok ? sym_entry(rp1, rq, m, ni, rmin, dr, dz) : 0.0;
                }
                x0[u] = d4{a4[0], a4[1], a4[2], a4[3]};
                x1[u] = d4{b4[0], b4[1], b4[2], b4[3]};
            } else if (!tail) {
                x0[u] = ld256_stream(tp0 + 4 * (k0 + lane) + 128 * u);
                x1[u] = ld256_stream(tp1 + 4 * (k0 + lane) + 128 * u);
            } else {
                x0[u] = ok ? ld256_stream(tp0 + 4 * v) : d4{0.0, 0.0, 0.0, 0.0};
                x1[u] = ok ? ld256_stream(tp1 + 4 * v) : d4{0.0, 0.0, 0.0, 0.0};
            }
        }
    };
    constexpr int kStep = 32 * UNR;
    const int nfull = (ve - vb) / kStep;          // rounds without a bounds check
    const int nround = (ve - vb + kStep - 1) / kStep;
    d4 tv[NBUF][2][UNR];  // ring of NBUF rounds: NBUF - 1 rounds stay in flight while one is consumed
#pragma unroll
    for (int b = 0; b + 1 < NBUF; ++b)
        if (b < nround) load(tv[b][0], tv[b][1], vb + b * kStep, b >= nfull);
    griddep();
    // staged layout: xqi planes [2][mc][2][2] | (xqf planes) | xpi rows [8][ms] | (xpf rows [8][ms]),
    // copied from the per-iteration packed arrays (k_sym_pack) by bulk (TMA 1-D) copies issued by
    // one thread and completing on an mbarrier: no per-element staging instructions
    const int ms = MIRROR ? nhp : mc;  // staged row stride of the block-P rows
    const int ps = MIRROR ? nh : mc;   // staged plane length (m values)
    double* xqi = xs;
    double* xqf = MIRROR ? xs : xs + 8 * mc;
    double* xpi = xs + 8 * ps * (MIRROR ? 1 : 2);
    double* xpf = MIRROR ? xpi : xpi + 8 * ms;
    if (threadIdx.x == 0) {
        const double* q0 = symq + (size_t)Q * 16 * nh;   // [arr][h][nh][2][2]
        const double* p0 = symp + (size_t)P * 16 * nhp;  // [arr][8][nhp]
        if (MIRROR) {
            mbar_expect_tx(&bar, (unsigned)(sizeof(double) * (8 * nh + 8 * nhp)));
            bulk_g2s(xqi, q0, (unsigned)(sizeof(double) * 8 * nh), &bar);
            bulk_g2s(xpi, p0, (unsigned)(sizeof(double) * 8 * nhp), &bar);
        } else {
            const int ml2 = (mlen + 1) & ~1;  // rows are zero-padded to nhp
            mbar_expect_tx(&bar, (unsigned)(sizeof(double) * (2 * 2 * 4 * mlen + 2 * 8 * ml2)));
#pragma unroll 1
            for (int arr = 0; arr < 2; ++arr) {
                double* dq = arr ? xqf : xqi;
                double* dp = arr ? xpf : xpi;
                for (int h = 0; h < 2; ++h)
                    bulk_g2s(dq + h * 4 * mc, q0 + (size_t)arr * 8 * nh + (size_t)h * 4 * nh + 4 * m0,
                             (unsigned)(sizeof(double) * 4 * mlen), &bar);
                for (int r8 = 0; r8 < 8; ++r8)
                    bulk_g2s(dp + r8 * ms, p0 + (size_t)arr * 8 * nhp + (size_t)r8 * nhp + m0,
                             (unsigned)(sizeof(double) * ml2), &bar);
            }
        }
    }
    mbar_wait(&bar, 0);
    const double* xpi0 = xpi + wr * ms;
    const double* xpf0 = xpf + wr * ms;
    const double* xpi1 = xpi0 + 4 * ms;
    const double* xpf1 = xpf0 + 4 * ms;
    const double2* pi0 = reinterpret_cast<const double2*>(xqi);           // q pairs 4qh + {0,1}
    const double2* pi1 = reinterpret_cast<const double2*>(xqi + 4 * ps);  // q pairs 4qh + {2,3}
    const double2* pf0 = reinterpret_cast<const double2*>(xqf);
    const double2* pf1 = reinterpret_cast<const double2*>(xqf + 4 * ps);
    const int wfb = MIRROR ? 2 * (nh - 1) + 2 * qh : 0;   // mirrored plane index = wfb - v
    double arI0 = 0.0, arF0 = 0.0, arI1 = 0.0, arF1 = 0.0, acI[4], acF[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) { acI[j] = 0.0; acF[j] = 0.0; }
    auto compute = [&](const d4 (&x0)[UNR], const d4 (&x1)[UNR], int k0, bool tail) {
        // round base pointers; the u-th vector is at a compile-time offset from them
        const int kl = k0 + lane;
        const double2* ai = pi0 + kl;
        const double2* bi = pi1 + kl;
        const double2* cf = pf0 + (MIRROR ? wfb - kl : kl);
        const double2* df = pf1 + (MIRROR ? wfb - kl : kl);
        const int ml = kl >> 1;
        const double* pI0 = xpi0 + ml;
        const double* pI1 = xpi1 + ml;
        const double* pF0 = xpf0 + (MIRROR ? nh - 1 - ml : ml);
        const double* pF1 = xpf1 + (MIRROR ? nh - 1 - ml : ml);
        constexpr int sgn = MIRROR ? -1 : 1;
#pragma unroll
        for (int u = 0; u < UNR; ++u) {
            double2 a, b, c, d;
            double i0, i1, f0, f1;
            if (!tail) {
                a = ai[32 * u]; b = bi[32 * u]; c = cf[sgn * 32 * u]; d = df[sgn * 32 * u];
                i0 = pI0[16 * u]; i1 = pI1[16 * u]; f0 = pF0[sgn * 16 * u]; f1 = pF1[sgn * 16 * u];
            } else {  // x = 0 past the end: read any valid slot
                const int v = min(k0 + 32 * u + lane, ve - 2 + qh);  // keeps the parity (= qh)
                const int mm = v >> 1, wf = MIRROR ? wfb - v : v, mf = MIRROR ? nh - 1 - mm : mm;
                a = pi0[v]; b = pi1[v]; c = pf0[wf]; d = pf1[wf];
                i0 = xpi0[mm]; i1 = xpi1[mm]; f0 = xpf0[mf]; f1 = xpf1[mf];
            }
            const d4 xi{a.x, a.y, b.x, b.y}, xf{c.x, c.y, d.x, d.y};
            arI0 = dot4(x0[u], xi, arI0);
            arF0 = dot4(x0[u], xf, arF0);
            arI1 = dot4(x1[u], xi, arI1);
            arF1 = dot4(x1[u], xf, arF1);
            acI[0] = fma(x1[u].x, i1, fma(x0[u].x, i0, acI[0]));
            acI[1] = fma(x1[u].y, i1, fma(x0[u].y, i0, acI[1]));
            acI[2] = fma(x1[u].z, i1, fma(x0[u].z, i0, acI[2]));
            acI[3] = fma(x1[u].w, i1, fma(x0[u].w, i0, acI[3]));
            acF[0] = fma(x1[u].x, f1, fma(x0[u].x, f0, acF[0]));
            acF[1] = fma(x1[u].y, f1, fma(x0[u].y, f0, acF[1]));
            acF[2] = fma(x1[u].z, f1, fma(x0[u].z, f0, acF[2]));
            acF[3] = fma(x1[u].w, f1, fma(x0[u].w, f0, acF[3]));
        }
    };
    // round r is consumed from buffer r % NBUF after round r + NBUF - 1 has been requested into the
    // buffer freed by round r - 1
#pragma unroll 1
    for (int r0 = 0; r0 < nround; r0 += NBUF) {
#pragma unroll
        for (int b = 0; b < NBUF; ++b) {
            const int r = r0 + b;
            if (r >= nround) break;
            const int rn = r + NBUF - 1;
            if (rn < nround)
                load(tv[(b + NBUF - 1) % NBUF][0], tv[(b + NBUF - 1) % NBUF][1], vb + rn * kStep, rn >= nfull);
            compute(tv[b][0], tv[b][1], vb + r * kStep, r >= nfull);
        }
    }
    arI0 = warp_sum(arI0);
    arF0 = warp_sum(arF0);
    arI1 = warp_sum(arI1);
    arF1 = warp_sum(arF1);
    if (lane == 0) {
        rrow[warp][0] = arI0; rrow[warp][1] = arF0; rrow[warp][2] = arI1; rrow[warp][3] = arF1;
    }
    if (!diag) {  // CTA-uniform
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            double a = acI[j], b = acF[j];
#pragma unroll
            for (int o = 2; o < 32; o <<= 1) {
                a += __shfl_xor_sync(0xffffffffu, a, o);
                b += __shfl_xor_sync(0xffffffffu, b, o);
            }
            if (lane < 2) {
                const int q = 4 * lane + j;
                red[warp][2 * q] = a;
                red[warp][2 * q + 1] = b;
            }
        }
    }
    __syncthreads();
    const int t = threadIdx.x;
    if (t < 16) {  // row direction: targets 8P + wr (+4), slot Q; groups summed in order
        const int w4 = t >> 2, k = t & 3, rp = 8 * P + w4 + (k >> 1) * 4, side = k & 1;
        double v = 0.0;
#pragma unroll
        for (int g = 0; g < WG; ++g) v += rrow[4 * g + w4][k];
        if (rp < ni) part[((long long)rp * 2 + side) * nslot + Q * nmc + mch] = v;
    } else if (t < 32 && !diag) {  // col direction: targets 8Q + q, slot P
        const int i = t - 16, q = i >> 1, side = i & 1, rq = 8 * Q + q;
        double v = 0.0;
#pragma unroll
        for (int w = 0; w < 4 * WG; ++w) v += red[w][i];
        if (rq < ni) part[((long long)rq * 2 + side) * nslot + P * nmc + mch] = v;
    }
}

static size_t sym_smem(const Ctx& c) {
    return sizeof(double) * (c.t.sym_nmc == 1 ? 8 * (size_t)c.nh + 8 * (size_t)c.nhp : 32 * (size_t)c.t.sym_mc);
}

// Per-iteration packing of the current pair into the layouts k_bnd_sym stages with bulk copies:
//   symq[B][arr][h][m][qh][w] = X_arr[1 + 8B + q][m],  q = 4 qh + 2 h + w  (0 past the interior)
//   symp[B][arr][p][m]        = X_arr[1 + 8B + p][m]   (rows padded to nhp, 0 past the interior)
// X_0 = I (pcurr), X_1 = F (pflip); narr = 1 when F is read mirrored from I.
__global__ void k_sym_pack(const double* __restrict__ I, const double* __restrict__ F, int nh, int nhp, int ni,
                           int nblk, int narr, double* __restrict__ symq, double* __restrict__ symp) {
    griddep();
    const long long nq = 16LL * nh, np = 16LL * nhp;  // per block, both arrays
    const long long total = (long long)nblk * (nq + np);
    for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < total;
         e += (long long)gridDim.x * blockDim.x) {
        if (e < (long long)nblk * nq) {
            const int B = (int)(e / nq);
            const int rem = (int)(e - (long long)B * nq);
            const int arr = rem / (8 * nh);
            if (arr >= narr) continue;
            const int r2 = rem - arr * 8 * nh, h = r2 / (4 * nh), r3 = r2 - h * 4 * nh;
            const int m = r3 >> 2, qh = (r3 >> 1) & 1, w = r3 & 1, q = 4 * qh + 2 * h + w, r = 8 * B + q;
            symq[e] = r < ni ? (arr ? F : I)[(long long)(1 + r) * nh + m] : 0.0;
        } else {
            const long long e2 = e - (long long)nblk * nq;
            const int B = (int)(e2 / np);
            const int rem = (int)(e2 - (long long)B * np);
            const int arr = rem / (8 * nhp);
            if (arr >= narr) continue;
            const int r2 = rem - arr * 8 * nhp, p = r2 / nhp, m = r2 - p * nhp, r = 8 * B + p;
            symp[e2] = (r < ni && m < nh) ? (arr ? F : I)[(long long)(1 + r) * nh + m] : 0.0;
        }
    }
}

// table vectors per row and lane per round, rounds in the register ring (EFIT_SYM_UNR/BUF
// override at build time for tuning)
// u1b4 (one 32-byte vector per row and ring round, four rounds: three in flight while one is
// consumed) -- measured 100.8 vs 109.8 us per boundary call at 513^2 against u2b2 (same 64 ring
// registers, finer rounds: the next loads issue after a quarter of the compute); u1b5 / u2b3 spill
#ifndef EFIT_SYM_UNR
#define EFIT_SYM_UNR 1
#endif
#ifndef EFIT_SYM_BUF
#define EFIT_SYM_BUF 4
#endif
#ifndef EFIT_SYM_WG
#define EFIT_SYM_WG 2
#endif
constexpr int kSymUnr = EFIT_SYM_UNR, kSymBuf = EFIT_SYM_BUF, kSymWg = EFIT_SYM_WG;
// the m-chunked (non-mirrored, nh > 576) variant keeps u2b2: u1b4 measured 932 vs 837 us at 1025^2
constexpr int kSymUnrC = 2, kSymBufC = 2;

constexpr int kTbGI = 8;
constexpr int kTbUnroll = 4;

static size_t lr_smem(const Ctx& c) {
    const int JT = c.t.lr_jt, JQ = c.t.lr_jj;
    return sizeof(double) * 8 * (size_t)(32 * JT + JQ + 1 + JQ);
}

static cudaError_t launch_lr(Ctx& c, cudaStream_t s, bool prepare) {
    const int ntile = c.jt_hi - c.jt_lo;
    const size_t smem = lr_smem(c);
    const void* f = nullptr;
    switch (c.t.lr_jt) {
        case 3: f = (const void*)k_bnd_lr<3>; break;
        case 5: f = (const void*)k_bnd_lr<5>; break;
        case 9: f = (const void*)k_bnd_lr<9>; break;
        case 17: f = (const void*)k_bnd_lr<17>; break;
        default: return cudaErrorInvalidValue;
    }
    if (prepare) return raise_smem_limit(f, smem);
    if (ntile <= 0) return cudaSuccess;
    dim3 grid(ntile, c.t.lr_nblk, 2);
    switch (c.t.lr_jt) {
#define EFIT_LR_CASE(V) \
    case V: launch_pdl(k_bnd_lr<V>, dim3(grid), dim3(256), smem, s, c.Tedge, c.S, c.pcurr, c.nw, c.nh, c.t.lr_jj, c.jt_lo, c.lr_part); break;
        EFIT_LR_CASE(3) EFIT_LR_CASE(5) EFIT_LR_CASE(9) EFIT_LR_CASE(17)
#undef EFIT_LR_CASE
    }
    return cudaGetLastError();
}

cudaError_t launch_solve_fwd(Ctx& c, const double* pcurr, const double* psib, cudaStream_t s, int with_bnd);

cudaError_t launch_boundary(Ctx& c, const double* pcurr, double* psib, cudaStream_t s, bool overlap_solve,
                            bool prepacked, int xmode, double* xbuf) {
    cudaError_t e;
    if (c.vh) {  // von Hagenow: zero-Dirichlet solve, normal derivatives, boundary operator
        if ((e = launch_solve(c, pcurr, c.zero_edge, c.vh_psi0, nullptr, nullptr, nullptr, s))) return e;
        if ((e = launch_pdl(k_vh_src, dim3((c.n_edge + 255) / 256), dim3(256), 0, s, (const double*)c.vh_psi0, c.nw,
                            c.nh, c.rmin, c.dr, c.dz, c.vh_src)))
            return e;
        mark(c, s, M_TB);
        return launch_pdl(k_vh_apply, dim3((c.n_edge + 7) / 8), dim3(256), 0, s, (const double*)c.Kvh,
                          (const double*)c.vh_src, c.n_edge, (c.n_edge + 3) / 4 * 4, psib);
    }
    const bool side_work = xmode != XCH_PARTIALS;  // left/right targets + SYM edge-row sources (replicated)
    const bool tile_work = xmode != XCH_FINISH;    // the rank's share of the top/bottom stream
    if (side_work) {
        // fork: the FP64-bound left/right chain runs on the side stream, concurrently with the
        // HBM-bound top/bottom stream (both only read pcurr / ipair); join before the reduce.
        if ((e = cudaEventRecord(c.ev_fork, s)) || (e = cudaStreamWaitEvent(c.side, c.ev_fork, 0))) return e;
        if (c.lr_direct) {
            if ((e = launch_lr(c, c.side, false))) return e;
        } else {
            if ((e = launch_lr_fft(c, psib, c.side))) return e;
        }
        // superposition: apart from the bottom/top edge terms the GS right-hand side is known once the
        // left/right FFT chain has written psi_b(left/right), so its forward DST also runs under the
        // HBM-bound stream; k_tridiag adds the bottom/top terms in the sine domain afterwards
        if (overlap_solve && (e = launch_solve_fwd(c, pcurr, psib, c.side, 2))) return e;
        if (c.sym && c.sym_edge &&
            (e = launch_pdl(k_sym_edge_src, dim3((2 * (c.nw - 2) + 7) / 8), dim3(256), 0, c.side, (const double*)c.Tedge,
                            c.S, (const double*)c.pcurr, (const double*)c.pflip, c.nw, c.nh, c.sym_edge)))
            return e;
        mark(c, c.side, M_LR);
        if ((e = cudaEventRecord(c.ev_join, c.side))) return e;
    }
    const int nslab = c.i_hi - c.i_lo;
    const size_t smem_tb = 2 * sizeof(double) * c.t.tb_ch;
    const long long sym_len = 2LL * c.ni * c.sym_nblk * c.t.sym_nmc;  // SYM exchange slice (doubles)
    double* sym_out = xmode == XCH_PARTIALS ? xbuf : c.sym_part;
    SymReduce sy{nullptr, 0, c.Tedge, c.S, c.pcurr, c.pflip, nullptr};
    if (tile_work) {
        if (c.sym) {
            // other ranks' slots must read 0 in a zero-padded exchange slice
            if ((xmode == XCH_PARTIALS || (xmode == XCH_NCCL && c.world > 1)) &&
                (e = cudaMemsetAsync(sym_out, 0, sizeof(double) * (size_t)sym_len, s)))
                return e;
            const long long ntl = c.sym_tile_hi - c.sym_tile_lo;
            if (ntl > 0) {
                const int narr = c.t.sym_nmc == 1 ? 1 : 2;
                if (!prepacked)
                    launch_pdl(k_sym_pack, dim3(4 * kNumSMs), dim3(256), 0, s, (const double*)c.pcurr, (const double*)c.pflip,
                               c.nh, c.nhp, c.ni, c.sym_nblk, narr, c.symq, c.symp);
                if ((e = cudaGetLastError())) return e;
                const size_t smem = sym_smem(c);
                const bool mir = c.t.sym_nmc == 1;
                const dim3 grid((unsigned)(ntl * c.t.sym_nmc));
                const int nslot = c.sym_nblk * c.t.sym_nmc;
#define EFIT_SYM_LAUNCH(OTFV, MIRV, UNRV, NBV, WGV)                                                                      \
    launch_pdl(k_bnd_sym<OTFV, MIRV, UNRV, NBV, WGV>, grid, dim3(128 * WGV), smem, s, (const double*)c.U, c.sym_tile_lo,  \
               c.ni, c.nh, c.t.sym_nmc, c.t.sym_mc, (const double*)c.symq, (const double*)c.symp, c.nhp, nslot,       \
               sym_out, c.rmin, c.dr, c.dz)
                if (c.otf) {  // FP64-bound: a short unroll keeps the inlined AGM in registers
                    if (mir) EFIT_SYM_LAUNCH(true, true, 1, 2, kSymWg); else EFIT_SYM_LAUNCH(true, false, 1, 2, kSymWg);
                } else if (mir) {
                    EFIT_SYM_LAUNCH(false, true, kSymUnr, kSymBuf, kSymWg);
                } else {
                    EFIT_SYM_LAUNCH(false, false, kSymUnrC, kSymBufC, kSymWg);
                }
#undef EFIT_SYM_LAUNCH
                if ((e = cudaGetLastError())) return e;
            }
        } else if (nslab > 0) {
            dim3 grid(c.t.tb_nchunk, c.t.tb_ngroup);
            if (!c.otf) {
                launch_pdl(k_bnd_tb<kTbGI, kTbUnroll>, dim3(grid), dim3(256), smem_tb, s, c.T, c.S, nslab, c.i_lo, c.nw * c.nh,
                           c.pcurr, c.pflip, c.t.tb_ch, c.tb_part);
            } else {
                launch_pdl(k_bnd_tb_otf<kTbGI>, dim3(grid), dim3(256), smem_tb, s, c.i_lo, nslab, c.nw, c.nh, c.rmin, c.dr,
                           c.dz, c.pcurr, c.pflip, c.t.tb_ch, c.tb_part);
            }
            if ((e = cudaGetLastError())) return e;
        }
        if (!c.sym && xmode != XCH_NONE) {
            // full table: the rank's own top/bottom rows, zero-padded, are its exchange slice
            BndOut o{nullptr, xmode == XCH_PARTIALS ? xbuf : psib + 2 * c.nh, c.i_lo, c.i_hi, 1};
            if ((e = launch_pdl(k_bnd_reduce, dim3((c.n_edge + 7) / 8), dim3(256), 0, s, (const double*)c.tb_part,
                                c.t.tb_nchunk, (const double*)c.lr_part, c.t.lr_nblk, c.nw, c.nh, 0, 0, o, sy)))
                return e;
        }
    }
    mark(c, s, M_TB);
    if (xmode == XCH_PARTIALS) return cudaSuccess;
    if (xmode == XCH_NCCL) {  // zero-padded slices summed over ranks: exact (one non-zero term each)
        if (c.sym) e = xch_allreduce(c, c.sym_part, (size_t)sym_len, s);
        else e = xch_allreduce(c, psib + 2 * c.nh, (size_t)(2 * (c.nw - 2)), s);
        if (e) return e;
    }
    if ((e = cudaStreamWaitEvent(s, c.ev_join, 0))) return e;
    // finish: left/right entries come from the partials (direct path) or were written by k_lr_ifft;
    // top/bottom from the (exchanged) SYM slots + edge-row sources, or the table chunk partials
    BndOut o{c.lr_direct ? psib : nullptr, nullptr, 1, c.nw - 1, 0};
    if (c.sym) {
        sy.part = xmode == XCH_FINISH ? xbuf : c.sym_part;
        sy.edge = c.sym_edge;
        sy.nslot = c.sym_nblk * c.t.sym_nmc;
        o.tb = psib + 2 * c.nh;
    } else if (xmode == XCH_NONE) {
        o.tb = psib + 2 * c.nh;
        o.tb_lo = c.i_lo;
        o.tb_hi = c.i_hi;
    } else if (xmode == XCH_FINISH) {
        if ((e = cudaMemcpyAsync(psib + 2 * c.nh, xbuf, sizeof(double) * 2 * (size_t)(c.nw - 2), cudaMemcpyDeviceToDevice, s)))
            return e;
    }
    if (!o.lr && !o.tb) return cudaSuccess;
    const int jhi = c.lr_direct ? c.nh : 0;
    launch_pdl(k_bnd_reduce, dim3((c.n_edge + 7) / 8), dim3(256), 0, s, (const double*)c.tb_part, c.t.tb_nchunk,
               (const double*)c.lr_part, c.t.lr_nblk, c.nw, c.nh, 0, jhi, o, sy);
    return cudaGetLastError();
}

// ------------------------------------------------------------ multi-slice top/bottom (tensor cores)
//
// S time slices share one pass over the top/bottom slabs: the nest becomes the
// product  Psi[i][c] = sum_e T[i][e] X_c[e]  of the slab matrix (target rows i x N^2 sources) with
// 2S right-hand sides X_{2s} = I_s, X_{2s+1} = F_s (F = vertically mirrored I), i.e. a dense
// contraction with 2S-fold reuse of every table element -> DMMA (mma.sync m8n8k4 fp64): A = 8 slabs
// x 4 sources, B = 4 sources x 8 columns (NBLK blocks of 8 columns), C = 8 x 8 accumulators in 2
// registers per lane.  Lane (g = lane/4, k4 = lane%4) loads T[slab 8o + g][e0 + 16j + 4k4 .. +3]
// with one 256-bit streaming load (4 lanes = 128 contiguous bytes of a slab) and uses its 4 values
// in 4 consecutive mma k-steps; its B values are X_{8b+g}[same 4 sources], one 256-bit shared load
// (columns padded by 2 doubles: conflict-free).  C needs no cross-lane reduction: lane holds
// (I, F) of slice 4b + k4 for slab 8o + g.  A CTA = one chunk of kBatchCh sources x 8 warps x NOCT
// octets of slabs; a ring of NP steps keeps NP*NOCT*32 B per lane of table loads in flight.
struct BatchIO {
    const double* X[2 * kMaxSlices];  // column c: I_{c/2} (even c) or F_{c/2} (odd), zero past nw*nh
    double* part[kMaxSlices];         // slice partials [row i][side][chunk]
};

template <int NBLK, int NOCT, int NP>
__global__ void __launch_bounds__(256, 2) k_bnd_tb_mma(const double* __restrict__ T, long long S, int nslab,
                                                      int row_lo, int n, int ncol, BatchIO io, int nchunk) {
    constexpr int ch = kBatchCh, ldx = kBatchCh + 2, nstep = kBatchCh / 16;
    static_assert(nstep % NP == 0, "ring depth divides the steps");
    extern __shared__ __align__(16) double xsm[];  // [8 NBLK columns][ldx]
    const int c = blockIdx.x;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, k4 = lane & 3;
    const long long e0 = (long long)c * ch;
    const int s0 = (blockIdx.y * 8 + warp) * 8 * NOCT;  // first slab of this warp
    const double* tp[NOCT];
    bool okr[NOCT];
#pragma unroll
    for (int o = 0; o < NOCT; ++o) {
        const int sl = s0 + 8 * o + g;
        okr[o] = sl < nslab;
        tp[o] = T + (long long)min(sl, nslab - 1) * S + e0 + 4 * k4;
    }
    auto load = [&](d4 (&a)[NOCT], int j) {
        const bool ok = e0 + 16 * j + 4 * k4 < n;
#pragma unroll
        for (int o = 0; o < NOCT; ++o) a[o] = (ok && okr[o]) ? ld256_stream(tp[o] + 16 * j) : d4{0.0, 0.0, 0.0, 0.0};
    };
    d4 ring[NP][NOCT];
#pragma unroll
    for (int b = 0; b + 1 < NP; ++b) load(ring[b], b);  // the table is constant: before the wait
    // staging: one bulk (TMA 1-D) copy per column (the pairs are zero-padded to whole chunks),
    // all in flight at once on one mbarrier; padding columns are zeroed
    __shared__ __align__(8) unsigned long long bar;
    if (threadIdx.x == 0) mbar_init(&bar, 1);
    __syncthreads();
    griddep();
    if (threadIdx.x == 0) {
        mbar_expect_tx(&bar, (unsigned)(sizeof(double) * ncol * ch));
        for (int col = 0; col < ncol; ++col)
            bulk_g2s(xsm + col * ldx, io.X[col] + e0, (unsigned)(sizeof(double) * ch), &bar);
    }
    for (int q = ncol * ch + threadIdx.x; q < 8 * NBLK * ch; q += blockDim.x) {
        const int col = q / ch, e = q - col * ch;
        xsm[col * ldx + e] = 0.0;
    }
    mbar_wait(&bar, 0);
    __syncthreads();
    double acc[NOCT][NBLK][2];
#pragma unroll
    for (int o = 0; o < NOCT; ++o)
#pragma unroll
        for (int b = 0; b < NBLK; ++b) { acc[o][b][0] = 0.0; acc[o][b][1] = 0.0; }
#pragma unroll 1
    for (int j0 = 0; j0 < nstep; j0 += NP) {
#pragma unroll
        for (int b = 0; b < NP; ++b) {
            const int j = j0 + b;
            if (j + NP - 1 < nstep) load(ring[(b + NP - 1) % NP], j + NP - 1);
            d4 xb[NBLK];
#pragma unroll
            for (int bl = 0; bl < NBLK; ++bl) xb[bl] = lds256(xsm + (8 * bl + g) * ldx + 16 * j + 4 * k4);
#pragma unroll
            for (int o = 0; o < NOCT; ++o)
#pragma unroll
                for (int bl = 0; bl < NBLK; ++bl) {
                    dmma884(acc[o][bl][0], acc[o][bl][1], ring[b][o].x, xb[bl].x);
                    dmma884(acc[o][bl][0], acc[o][bl][1], ring[b][o].y, xb[bl].y);
                    dmma884(acc[o][bl][0], acc[o][bl][1], ring[b][o].z, xb[bl].z);
                    dmma884(acc[o][bl][0], acc[o][bl][1], ring[b][o].w, xb[bl].w);
                }
        }
    }
    // lane holds C[slab 8o + g][columns 8bl + 2k4, +1] = (I, F) sums of slice 4bl + k4
#pragma unroll
    for (int o = 0; o < NOCT; ++o) {
        if (!okr[o]) continue;
        const int row = row_lo + s0 + 8 * o + g;
#pragma unroll
        for (int bl = 0; bl < NBLK; ++bl) {
            const int sl = 4 * bl + k4;
            if (2 * sl < ncol) {
                double* pp = io.part[sl];
                pp[((long long)row * 2 + 0) * nchunk + c] = acc[o][bl][0];
                pp[((long long)row * 2 + 1) * nchunk + c] = acc[o][bl][1];
            }
        }
    }
}

constexpr int kMmaOct = 2, kMmaNP = 4;

cudaError_t launch_boundary_batch(Ctx& c, int nslice, Ctx* const* slices, cudaStream_t s) {
    const int nslab = c.i_hi - c.i_lo;
    if (nslab <= 0) return cudaSuccess;
    BatchIO io;
    for (int k = 0; k < 2 * kMaxSlices; ++k) io.X[k] = nullptr;
    for (int k = 0; k < kMaxSlices; ++k) io.part[k] = nullptr;
    for (int k = 0; k < nslice; ++k) {
        io.X[2 * k] = slices[k]->pcurr;
        io.X[2 * k + 1] = slices[k]->pflip;
        io.part[k] = slices[k]->tb_part;
    }
    const int spc = 8 * 8 * kMmaOct;  // slabs per CTA
    const dim3 grid((unsigned)c.tbb_nchunk, (unsigned)((nslab + spc - 1) / spc));
    const int n = c.nw * c.nh;
    if (nslice <= 4)
        return launch_pdl(k_bnd_tb_mma<1, kMmaOct, kMmaNP>, grid, dim3(256), sizeof(double) * 8 * (kBatchCh + 2), s,
                          (const double*)c.T, c.S, nslab, c.i_lo, n, 2 * nslice, io, c.tbb_nchunk);
    return launch_pdl(k_bnd_tb_mma<2, kMmaOct, kMmaNP>, grid, dim3(256), sizeof(double) * 16 * (kBatchCh + 2), s,
                      (const double*)c.T, c.S, nslab, c.i_lo, n, 2 * nslice, io, c.tbb_nchunk);
}

// Top/bottom entries of psib from k_bnd_tb_mma partials (full-table mode, FFT left/right path: the
// left/right entries were written by k_lr_ifft).
cudaError_t launch_bnd_reduce(Ctx& c, const double* tb_part, int tb_nchunk, double* psib, cudaStream_t s) {
    SymReduce sy{nullptr, 0, c.Tedge, c.S, c.pcurr, c.pflip, nullptr};
    BndOut o{nullptr, psib + 2 * c.nh, c.i_lo, c.i_hi, 0};
    return launch_pdl(k_bnd_reduce, dim3((c.n_edge + 7) / 8), dim3(256), 0, s, tb_part, tb_nchunk,
                      (const double*)c.lr_part, c.t.lr_nblk, c.nw, c.nh, 0, 0, o, sy);
}

// ================================================================================ interior solve

// Forward complex FFT (exp(-2 pi i jk/M)) of M = 2^log2m points in shared memory, Stockham
// auto-sort (natural order in and out, ping-pong between x and y), radix 4 while >= 2 bits remain,
// one radix-2 stage otherwise.  At a stage with P sub-problems of length N_s = M/P the layout is
// A[n P + b]; the radix-r DIF butterfly on inputs a_q = A[(n1 + q N_s/r) P + b] gives
// y_k = sum_q a_q w_r^(q k) * w_M^(n1 k P), stored at B[n1 r P + b + k P].  W[e] = exp(-2 pi i e/M)
// for e < M/2 (W[e + M/2] = -W[e]).  Returns the buffer holding the result.
__device__ __forceinline__ double2 cmul(double2 a, double2 b) {
    return make_double2(fma(a.x, b.x, -a.y * b.y), fma(a.x, b.y, a.y * b.x));
}
__device__ __forceinline__ double2 twid(const double2* W, int e, int M) {
    const double2 w = W[e & ((M >> 1) - 1)];
    return (e & (M >> 1)) ? make_double2(-w.x, -w.y) : w;
}

__device__ double2* fft_stockham(double2* x, double2* y, int M, int log2m, const double2* W, int tid, int nthr) {
    double2* a = x;
    double2* b = y;
    int s = 0;  // log2 of the number of sub-problems P
    while (s < log2m) {
        const int P = 1 << s;
        if (log2m - s >= 2) {
            const int q = M >> (s + 2);  // N_s / 4
            for (int t = tid; t < (M >> 2); t += nthr) {
                const int bb = t & (P - 1), n1 = t >> s;
                const double2 a0 = a[n1 * P + bb], a1 = a[(n1 + q) * P + bb];
                const double2 a2 = a[(n1 + 2 * q) * P + bb], a3 = a[(n1 + 3 * q) * P + bb];
                const double2 t0 = make_double2(a0.x + a2.x, a0.y + a2.y), t1 = make_double2(a0.x - a2.x, a0.y - a2.y);
                const double2 t2 = make_double2(a1.x + a3.x, a1.y + a3.y);
                const double2 t3 = make_double2(a1.y - a3.y, a3.x - a1.x);  // -i (a1 - a3)
                const int e1 = (n1 * P) & (M - 1);
                const double2 y1 = cmul(make_double2(t1.x + t3.x, t1.y + t3.y), twid(W, e1, M));
                const double2 y2 = cmul(make_double2(t0.x - t2.x, t0.y - t2.y), twid(W, (2 * e1) & (M - 1), M));
                const double2 y3 = cmul(make_double2(t1.x - t3.x, t1.y - t3.y), twid(W, (3 * e1) & (M - 1), M));
                const int o = n1 * (P << 2) + bb;
                b[o] = make_double2(t0.x + t2.x, t0.y + t2.y);
                b[o + P] = y1;
                b[o + 2 * P] = y2;
                b[o + 3 * P] = y3;
            }
            s += 2;
        } else {
            const int q = M >> (s + 1);  // N_s / 2
            for (int t = tid; t < (M >> 1); t += nthr) {
                const int bb = t & (P - 1), n1 = t >> s;
                const double2 a0 = a[n1 * P + bb], a1 = a[(n1 + q) * P + bb];
                const int o = n1 * (P << 1) + bb;
                b[o] = make_double2(a0.x + a1.x, a0.y + a1.y);
                b[o + P] = cmul(make_double2(a0.x - a1.x, a0.y - a1.y), twid(W, (n1 * P) & (M - 1), M));
            }
            s += 1;
        }
        __syncthreads();
        double2* tmp = a;
        a = b;
        b = tmp;
    }
    return a;
}

// What k_dst_inv needs to produce the next iteration's psi_axis/psi_bdry (chained fit steps).
struct NextNorm {
    int on, sgn, n_lim;
    const uint8_t* inlim;
    const double* lim;
    double rmin, dr, zmin, dz;
    double* part;
    int* status;
};

// Number of Stockham stages for M = 2^log2m (radix 4, plus one radix 2 if log2m is odd): the
// result is in the scratch buffer when it is odd.
__host__ __device__ __forceinline__ int fft_stages(int log2m) { return (log2m >> 1) + (log2m & 1); }

// Forward DST-I along Z of the right-hand side of 2*FPC interior rows per CTA (two rows packed as
// the real and imaginary parts of one complex FFT of the odd extension, length M = 2(n+1); FPC
// FFTs side by side, TPF threads each):
//   f_ij = -mu0 R_i I_ij/(dR dZ) - (Dirichlet terms of the edge values psi_b).
// DST_k(x) = -Im(Z_k)/2 for the real-part row, Re(Z_k)/2 for the imaginary-part row.  Output is
// mode-major, fhat[k-1][r] (r = i-1), the CTA's 2*FPC rows contiguous (16/32-byte stores per mode).
__global__ void __launch_bounds__(512) k_dst_fwd(const double* __restrict__ pcurr, const double* __restrict__ psib,
                                                 const double* __restrict__ tri_a, int nw, int nh, double rmin,
                                                 double dr, double dz, const double2* __restrict__ W, int M,
                                                 int log2m, int FPC, double* __restrict__ fhat, int ld, int with_bnd) {
    extern __shared__ __align__(16) double2 a2[];  // FPC x ([M] data, [M] scratch), then [M/2] twiddles
    double2* Ws = a2 + 2 * FPC * M;
    const int n = nh - 2, ni = nw - 2;
    const int TPF = blockDim.x / FPC;
    const int f = threadIdx.x / TPF, lt = threadIdx.x - f * TPF;
    const int rbase = 2 * FPC * blockIdx.x;  // first 0-based interior row of the CTA
    double2* xf = a2 + 2 * f * M;
    const double idz2 = 1.0 / (dz * dz);
    const double cellinv = 1.0 / (dr * dz);
    for (int k = threadIdx.x; k < M / 2; k += blockDim.x) Ws[k] = __ldg(W + k);  // init-time constants
    griddep();
    for (int j = lt; j < M; j += TPF) {
        double v[2] = {0.0, 0.0};
        int jj = 0;
        double sgn = 0.0;
        if (j >= 1 && j <= n) { jj = j; sgn = 1.0; }
        else if (j >= n + 2) { jj = M - j; sgn = -1.0; }
        if (sgn != 0.0) {
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                const int i = rbase + 2 * f + h + 1;  // grid row
                if (i > ni) continue;
                const double R = grid_coord(rmin, i, dr);
                double fv = -kMu0 * R * pcurr[(long long)i * nh + jj] * cellinv;
                if (with_bnd) {
                    if (i == 1) fv -= tri_a[0] * psib[jj];                                   // left edge
                    if (i == ni) fv -= (2.0 / (dr * dr) - tri_a[ni - 1]) * psib[nh + jj];    // right edge (c_ni)
                }
                if (with_bnd == 1) {  // with_bnd == 2: k_tridiag adds these in the sine domain
                    if (jj == 1) fv -= psib[2 * nh + (i - 1)] * idz2;                        // bottom edge
                    if (jj == n) fv -= psib[2 * nh + (nw - 2) + (i - 1)] * idz2;             // top edge
                }
                v[h] = sgn * fv;
            }
        }
        xf[j] = make_double2(v[0], v[1]);
    }
    __syncthreads();
    fft_stockham(xf, xf + M, M, log2m, Ws, lt, TPF);
    const int ro = (fft_stages(log2m) & 1) ? M : 0;
    for (int k = 1 + threadIdx.x; k <= n; k += blockDim.x) {
        double* dst = fhat + (long long)(k - 1) * ld + rbase;
        for (int g = 0; g < FPC; ++g) {
            const double2 z = a2[2 * g * M + ro + k];
            *reinterpret_cast<double2*>(dst + 2 * g) = make_double2(-0.5 * z.y, 0.5 * z.x);
        }
    }
}

// Bottom/top edge terms of the right-hand side in the sine domain (superposition, see
// launch_boundary): f_{j=1} -= psi_bot/dz^2 and f_{j=n} -= psi_top/dz^2 transform to
//   fhat[k][r] -= (psi_bot(r) + (-1)^(k+1) psi_top(r)) sin(pi k/(n+1)) / dz^2,
// added by the tridiagonal kernel as it loads its mode column (bot == nullptr: nothing to add).
struct TbFix {
    const double* bot;   // psi_b bottom edge, rows i = 1..ni (ABI edge order offset 2 nh)
    const double* top;   // psi_b top edge
    const double* sink;  // sin(pi k/(n+1)), k = 1..n
    double idz2;
};
__device__ __forceinline__ double tb_fix(const TbFix& fx, int mode, int r) {
    const double sgn = (mode & 1) ? -1.0 : 1.0;  // k = mode + 1: (-1)^(k+1)
    return -(fx.bot[r] + sgn * fx.top[r]) * (fx.sink[mode] * fx.idz2);
}

// Radial tridiagonal solve per sine mode, one warp per mode, in place on the mode-major array.
// The warp stages its mode column in shared memory with a skew (row r at r + r/L, L = rows per
// lane) so both the global access and the lane-segment access are conflict-free.  Both Thomas
// sweeps are first-order linear recurrences,  forward d_r = inv_r f_r + alpha_r d_{r-1}
// (d_{-1} = 0),  backward x_r = d_r - c'_r x_{r+1} (x_ni = 0): each lane composes the affine map of
// its segment of L rows, a 5-step shuffle scan composes the maps of the preceding (following)
// lanes, and each lane replays its segment from the exact incoming value.  The factors are stored
// segment-interleaved (row r at (r % L)*32 + r/L) so a lane's factor loads are coalesced across the
// warp.  Padding rows (r >= ni) have alpha = inv = c' = 0 and only follow the real rows.
// |alpha|, |c'| < 1 (diagonal dominance) keeps the reassociation as accurate as the sequential sweep.
__global__ void __launch_bounds__(128) k_tridiag(double* __restrict__ fhat, int ld, const double* __restrict__ alpha,
                                                 const double* __restrict__ inv, const double* __restrict__ cp,
                                                 int ni, int L, int nmode, TbFix fx) {
    extern __shared__ __align__(16) double sm_tri[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int mode = blockIdx.x * 4 + warp;
    double* sf = sm_tri + (size_t)warp * (32 * L + 32);  // skewed: row r at r + r/L < 32L + 32
    griddep();
    if (mode >= nmode) return;
    double* fg = fhat + (long long)mode * ld;
    for (int r = lane; r < 32 * L; r += 32)
        sf[r + r / L] = r < ni ? (fx.bot ? fg[r] + tb_fix(fx, mode, r) : fg[r]) : 0.0;
    __syncwarp();
    const long long fo = (long long)mode * 32 * L + lane;
    const double* al = alpha + fo;
    const double* iv = inv + fo;
    const double* c = cp + fo;
    double* f = sf + lane * (L + 1);  // this lane's segment rows lane*L .. lane*L + L - 1
    double A = 1.0, B = 0.0;
#pragma unroll 4
    for (int e = 0; e < L; ++e) {
        const double a = al[32 * e];
        B = fma(a, B, iv[32 * e] * f[e]);
        A *= a;
    }
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const double Ap = __shfl_up_sync(0xffffffffu, A, off);
        const double Bp = __shfl_up_sync(0xffffffffu, B, off);
        if (lane >= off) { B = fma(A, Bp, B); A *= Ap; }
    }
    double d = __shfl_up_sync(0xffffffffu, B, 1);
    if (lane == 0) d = 0.0;
#pragma unroll 4
    for (int e = 0; e < L; ++e) {
        d = fma(al[32 * e], d, iv[32 * e] * f[e]);
        f[e] = d;
    }
    double C = 1.0, D = 0.0;
#pragma unroll 4
    for (int e = L - 1; e >= 0; --e) {
        const double q = -c[32 * e];
        D = fma(q, D, f[e]);
        C *= q;
    }
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const double Cn = __shfl_down_sync(0xffffffffu, C, off);
        const double Dn = __shfl_down_sync(0xffffffffu, D, off);
        if (lane + off < 32) { D = fma(C, Dn, D); C *= Cn; }
    }
    double x = __shfl_down_sync(0xffffffffu, D, 1);
    if (lane == 31) x = 0.0;
#pragma unroll 4
    for (int e = L - 1; e >= 0; --e) {
        x = fma(-c[32 * e], x, f[e]);
        f[e] = x;
    }
    __syncwarp();
    for (int r = lane; r < ni; r += 32) fg[r] = sf[r + r / L];
}

// Register variant of k_tridiag for L <= 16 rows per lane: every lane loads its whole segment
// (data, alpha, inv, c') with independent loads first, so the two sweeps run from registers after a
// single memory latency.  Same recurrences and scan as k_tridiag (bitwise-identical results).
template <int L>
__global__ void __launch_bounds__(128) k_tridiag_reg(double* __restrict__ fhat, int ld,
                                                     const double* __restrict__ alpha,
                                                     const double* __restrict__ inv, const double* __restrict__ cp,
                                                     int ni, int nmode, TbFix fx) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int mode = blockIdx.x * 4 + warp;
    const bool act = mode < nmode;
    double* fg = fhat + (long long)mode * ld;
    const long long fo = (long long)mode * 32 * L + lane;
    double f[L], al[L], iv[L], c[L];
    // the Thomas factors are constant tables: loaded before the wait on the predecessor
#pragma unroll
    for (int e = 0; e < L; ++e) {
        al[e] = act ? alpha[fo + 32 * e] : 0.0;
        iv[e] = act ? inv[fo + 32 * e] : 0.0;
        c[e] = act ? cp[fo + 32 * e] : 0.0;
    }
    // staging through shared memory: coalesced loads of the mode column (row r at r + r/L: the lane
    // segments r = lane L + e are then conflict-free) and of the bottom/top edge rows (the same for
    // every mode of the CTA), instead of 32-way scattered per-lane segment loads
    __shared__ double sf[4][32 * (L + 1)];
    __shared__ double sbt[2][32 * L];
    griddep();
    if (fx.bot)
        for (int r = threadIdx.x; r < ni; r += blockDim.x) {
            sbt[0][r] = fx.bot[r];
            sbt[1][r] = fx.top[r];
        }
    double* sw = sf[warp];
    if (act) {
#pragma unroll
        for (int e = 0; e < L; ++e) {
            const int r = 32 * e + lane;
            sw[r + r / L] = r < ni ? fg[r] : 0.0;
        }
    }
    __syncthreads();
    if (!act) return;
    const double sgn_fx = (mode & 1) ? -1.0 : 1.0;  // tb_fix's expression, edge rows from shared memory
    const double sk_fx = fx.bot ? fx.sink[mode] * fx.idz2 : 0.0;
#pragma unroll
    for (int e = 0; e < L; ++e) {
        const int r = lane * L + e;
        const double v = sw[r + lane];
        f[e] = r < ni ? (fx.bot ? v + -(sbt[0][r] + sgn_fx * sbt[1][r]) * sk_fx : v) : 0.0;
    }
    double A = 1.0, B = 0.0;
#pragma unroll
    for (int e = 0; e < L; ++e) {
        B = fma(al[e], B, iv[e] * f[e]);
        A *= al[e];
    }
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const double Ap = __shfl_up_sync(0xffffffffu, A, off);
        const double Bp = __shfl_up_sync(0xffffffffu, B, off);
        if (lane >= off) { B = fma(A, Bp, B); A *= Ap; }
    }
    double d = __shfl_up_sync(0xffffffffu, B, 1);
    if (lane == 0) d = 0.0;
#pragma unroll
    for (int e = 0; e < L; ++e) {
        d = fma(al[e], d, iv[e] * f[e]);
        f[e] = d;
    }
    double C = 1.0, D = 0.0;
#pragma unroll
    for (int e = L - 1; e >= 0; --e) {
        D = fma(-c[e], D, f[e]);
        C *= -c[e];
    }
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const double Cn = __shfl_down_sync(0xffffffffu, C, off);
        const double Dn = __shfl_down_sync(0xffffffffu, D, off);
        if (lane + off < 32) { D = fma(C, Dn, D); C *= Cn; }
    }
    double x = __shfl_down_sync(0xffffffffu, D, 1);
    if (lane == 31) x = 0.0;
#pragma unroll
    for (int e = L - 1; e >= 0; --e) {
        x = fma(-c[e], x, f[e]);
        f[e] = x;
    }
    // back through the skewed shared column: coalesced stores
#pragma unroll
    for (int e = 0; e < L; ++e) sw[lane * (L + 1) + e] = f[e];
    __syncwarp();
#pragma unroll
    for (int e = 0; e < L; ++e) {
        const int r = 32 * e + lane;
        if (r < ni) fg[r] = sw[r + r / L];
    }
}

// Inverse DST-I (same transform, scale 2/(n+1)) of 2*FPC rows per CTA, then either
//   psi_out = psi_p                                  (efit_interior_solve), or
//   psi_inout <- psi_p + psi_ext, eps partial max     (efit_fit_step),
// edges (j = 0, nh-1, and rows 0, nw-1 in the extra last block) take psi_b.
__global__ void __launch_bounds__(512) k_dst_inv(const double* __restrict__ fhat, int ld,
                                                 const double* __restrict__ psib,
                                                 int nw, int nh, const double2* __restrict__ W, int M, int log2m,
                                                 int FPC, double* __restrict__ psi_out, double* __restrict__ psi_inout,
                                                 const double* __restrict__ psi_ext, double* __restrict__ eps_part,
                                                 NextNorm nn) {
    extern __shared__ __align__(16) double2 a2[];  // FPC x ([M] data, [M] scratch), then [M/2] twiddles
    double2* Ws = a2 + 2 * FPC * M;
    __shared__ double wmax[16];
    const int n = nh - 2, ni = nw - 2;
    const int nrb = (ni + 2 * FPC - 1) / (2 * FPC);  // row blocks; block nrb does the edge rows
    const int TPF = blockDim.x / FPC;
    const int f = threadIdx.x / TPF, lt = threadIdx.x - f * TPF;
    double dmax = 0.0;
    double best = -DBL_MAX;  // next iteration's axis partial (nn.on)
    long long bi = LLONG_MAX;
    bool bad = false;
    const double sg = (double)nn.sgn;
    auto emit_v = [&](long long g, double pp, double ext, double old) {
        if (psi_out) psi_out[g] = pp;
        if (psi_inout) {
            const double nv = pp + ext;
            dmax = fmax(dmax, fabs(nv - old));
            psi_inout[g] = nv;
            if (nn.on) {
                if (!isfinite(nv)) bad = true;
                if (nn.inlim[g]) argmax_merge(best, bi, sg * nv, g);
            }
        }
    };
    auto emit = [&](long long g, double pp) {
        if (psi_inout) emit_v(g, pp, psi_ext[g], psi_inout[g]);
        else emit_v(g, pp, 0.0, 0.0);
    };
    // one FFT per CTA (FPC = 1): the CTA's two rows of psi_ext (an input) and of the old psi (written
    // by the previous iteration's update, many kernels back) are loaded before the wait on the
    // predecessor, into registers, so the update does not start with a memory round trip
    constexpr int kPre = 8;
    double pe[2][kPre], po[2][kPre];
    const bool pre = psi_inout != nullptr && FPC == 1 && (int)blockIdx.x < nrb &&
                     (nh + (int)blockDim.x - 1) / (int)blockDim.x <= kPre;
    if (pre) {
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int i = 2 * blockIdx.x + h + 1;
#pragma unroll
            for (int q = 0; q < kPre; ++q) {
                const int j = threadIdx.x + q * blockDim.x;
                const bool ok = i <= ni && j < nh;
                pe[h][q] = ok ? psi_ext[(long long)i * nh + j] : 0.0;
                po[h][q] = ok ? psi_inout[(long long)i * nh + j] : 0.0;
            }
        }
    }
    if ((int)blockIdx.x < nrb) {
        const int rbase = 2 * FPC * blockIdx.x;
        for (int k = threadIdx.x; k < M / 2; k += blockDim.x) Ws[k] = __ldg(W + k);
        griddep();
        // stage: for every mode the CTA's rows are contiguous in fhat
        for (int j = threadIdx.x; j < M; j += blockDim.x) {
            int jj = 0;
            double sg = 0.0;
            if (j >= 1 && j <= n) { jj = j; sg = 1.0; }
            else if (j >= n + 2) { jj = M - j; sg = -1.0; }
            const double* src = fhat + (long long)(jj > 0 ? jj - 1 : 0) * ld + rbase;
            for (int g = 0; g < FPC; ++g) {
                double2 v = make_double2(0.0, 0.0);
                if (sg != 0.0) {
                    const double2 w2 = *reinterpret_cast<const double2*>(src + 2 * g);
                    v = make_double2(sg * w2.x, sg * w2.y);
                }
                a2[2 * g * M + j] = v;
            }
        }
        __syncthreads();
        fft_stockham(a2 + 2 * f * M, a2 + 2 * f * M + M, M, log2m, Ws, lt, TPF);
        const int ro = (fft_stages(log2m) & 1) ? M : 0;
        const double sc = 2.0 / (double)(n + 1);
        if (pre) {
            const double2* res = a2 + ro;
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                const int i = rbase + h + 1;
                if (i > ni) break;
#pragma unroll
                for (int q = 0; q < kPre; ++q) {
                    const int j = threadIdx.x + q * blockDim.x;
                    if (j >= nh) break;
                    double pp;
                    if (j == 0) pp = psib[2 * nh + (i - 1)];
                    else if (j == nh - 1) pp = psib[2 * nh + (nw - 2) + (i - 1)];
                    else {
                        const double2 z = res[j];
                        pp = sc * (h == 0 ? -0.5 * z.y : 0.5 * z.x);
                    }
                    emit_v((long long)i * nh + j, pp, pe[h][q], po[h][q]);
                }
            }
        } else {
            for (int g = 0; g < FPC; ++g) {
                const double2* res = a2 + 2 * g * M + ro;
                for (int h = 0; h < 2; ++h) {
                    const int i = rbase + 2 * g + h + 1;
                    if (i > ni) break;
                    for (int j = threadIdx.x; j < nh; j += blockDim.x) {
                        double pp;
                        if (j == 0) pp = psib[2 * nh + (i - 1)];
                        else if (j == nh - 1) pp = psib[2 * nh + (nw - 2) + (i - 1)];
                        else {
                            const double2 z = res[j];
                            pp = sc * (h == 0 ? -0.5 * z.y : 0.5 * z.x);
                        }
                        emit((long long)i * nh + j, pp);
                    }
                }
            }
        }
    } else {
        griddep();
        // rows 0 and nw-1: left/right edge values
        for (int j = threadIdx.x; j < nh; j += blockDim.x) {
            emit((long long)j, psib[j]);
            emit((long long)(nw - 1) * nh + j, psib[nh + j]);
        }
    }
    if (!psi_inout) return;
    dmax = warp_max(dmax);
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
    if (l == 0) wmax[w] = dmax;
    __shared__ double av[16];
    __shared__ long long ai[16];
    if (nn.on) {
        if (__syncthreads_or(bad) && threadIdx.x == 0) atomicOr(nn.status, EFIT_ST_NONFINITE);
        warp_argmax(best, bi);
        if (l == 0) { av[w] = best; ai[w] = bi; }
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        double m = 0.0;
        for (int q = 0; q < (int)(blockDim.x >> 5); ++q) m = fmax(m, wmax[q]);
        eps_part[blockIdx.x] = m;
        if (nn.on) {
            for (int q = 1; q < (int)(blockDim.x >> 5); ++q) argmax_merge(best, bi, av[q], ai[q]);
            nn.part[2 * blockIdx.x] = best;
            nn.part[2 * blockIdx.x + 1] = (double)bi;
        }
    }
}

// Finish of an axis / boundary search (one CTA, launched programmatically behind the partials'
// producer, so the producer's blocks need no fence and no completion ticket):
//   behind k_dst_inv: eps = max over its blocks' partials / |psi_bdry - psi_axis| (the old values),
//     then the new psi's axis / boundary for the next chained iteration;
//   behind k_normalize (eps_part = eps = nullptr): psi_axis / psi_bdry of the given psi.
__global__ void __launch_bounds__(256) k_norm_fin(const double* __restrict__ eps_part, int nparts,
                                                 const double* __restrict__ psi_inout, int nw, int nh,
                                                 double* __restrict__ axbd, double* __restrict__ eps, NextNorm nn) {
    // latency-shaped: the limiter vertices (constant) are read before the wait on k_dst_inv; after it,
    // the eps and argmax partials come in one round trip, the vertex values in a second one
    __shared__ double wv[8], av[8], bv[8];
    __shared__ long long ai[8], bi_s[8];
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31, nwarp = blockDim.x >> 5;
    double lr = 0.0, lz = 0.0;
    const bool hasv = nn.on && (int)threadIdx.x < nn.n_lim;
    if (hasv) { lr = nn.lim[threadIdx.x]; lz = nn.lim[nn.n_lim + threadIdx.x]; }
    griddep();
    const double sg = (double)nn.sgn;
    double m = 0.0, best = -DBL_MAX;
    long long bi = LLONG_MAX;
    for (int b = threadIdx.x; b < nparts; b += blockDim.x) {
        if (eps_part) m = fmax(m, eps_part[b]);
        if (nn.on) argmax_merge(best, bi, nn.part[2 * b], (long long)nn.part[2 * b + 1]);
    }
    // the old axis / boundary (this iteration's eps) before they are replaced below
    const double pa_old = eps ? axbd[0] : 0.0, pb_old = eps ? axbd[1] : 0.0;
    // limiter-vertex values of the new psi (thread v; n_lim <= blockDim handled by the loop below)
    double vb = -DBL_MAX;
    long long vi = LLONG_MAX;
    if (nn.on) {
        if (hasv) argmax_merge(vb, vi, sg * bilinear(psi_inout, nw, nh, nn.rmin, nn.dr, nn.zmin, nn.dz, lr, lz),
                               (long long)threadIdx.x);
        for (int v = threadIdx.x + blockDim.x; v < nn.n_lim; v += blockDim.x)
            argmax_merge(vb, vi, sg * bilinear(psi_inout, nw, nh, nn.rmin, nn.dr, nn.zmin, nn.dz, nn.lim[v],
                                               nn.lim[nn.n_lim + v]), (long long)v);
    }
    m = warp_max(m);
    warp_argmax(best, bi);
    warp_argmax(vb, vi);
    if (l == 0) { wv[w] = m; av[w] = best; ai[w] = bi; bv[w] = vb; bi_s[w] = vi; }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int q = 1; q < nwarp; ++q) {
            m = fmax(m, wv[q]);
            argmax_merge(best, bi, av[q], ai[q]);
            argmax_merge(vb, vi, bv[q], bi_s[q]);
        }
        if (eps) *eps = m / fabs(pb_old - pa_old);
        if (nn.on) {  // psi_axis / psi_bdry: the merged values themselves (s times the value), rule Q9
            const double pa = (bi == LLONG_MAX) ? 0.0 : sg * best;
            const double pb = (vi == LLONG_MAX) ? 0.0 : sg * vb;
            axbd[0] = pa;
            axbd[1] = pb;
            if (bi == LLONG_MAX || !(sg * (pa - pb) > 0.0)) atomicOr(nn.status, EFIT_ST_NOPLASMA);
        }
    }
}

static NextNorm next_norm_args(const Ctx& c, bool on) {
    NextNorm nn;
    nn.on = on ? 1 : 0;
    nn.sgn = c.ip_sign;
    nn.n_lim = c.n_lim;
    nn.inlim = c.inlim;
    nn.lim = c.lim;
    nn.rmin = c.rmin; nn.dr = c.dr; nn.zmin = c.zmin; nn.dz = c.dz;
    nn.part = c.norm_part;
    nn.status = c.status;
    return nn;
}

static cudaError_t launch_norm_fin(Ctx& c, const double* psi, int nparts, const double* eps_part, double* eps,
                                   cudaStream_t s) {
    return launch_pdl(k_norm_fin, dim3(1), dim3(256), 0, s, eps_part, nparts, psi, c.nw, c.nh, c.axbd, eps,
                      next_norm_args(c, true));
}

static void solve_shape(const Ctx& c, int& fpc, int& threads, size_t& smem) {
    const int M = c.fft_m;
    // one FFT (two rows) per CTA: twice the CTAs of the two-FFT shape, so twice the loads in flight
    // and half the rows per CTA on the latency-bound solve (EFIT_SOLVE_FPC=2 restores it)
    static const int want = getenv("EFIT_SOLVE_FPC") ? atoi(getenv("EFIT_SOLVE_FPC")) : 1;
    fpc = (want >= 2 && sizeof(double2) * (size_t)(4 * M + M / 2) <= 160 * 1024) ? 2 : 1;
    int tpf = M / 4;
    if (tpf > 256) tpf = 256;
    if (tpf < 32) tpf = 32;
    threads = fpc * tpf;
    smem = sizeof(double2) * (size_t)(2 * fpc * M + M / 2);
}

// forward DST of the interior right-hand side; with_bnd: 1 = all edge terms, 2 = left/right only
cudaError_t launch_solve_fwd(Ctx& c, const double* pcurr, const double* psib, cudaStream_t s, int with_bnd) {
    int fpc, threads;
    size_t smem;
    solve_shape(c, fpc, threads, smem);
    const int nrb = (c.ni + 2 * fpc - 1) / (2 * fpc);
    return launch_pdl(k_dst_fwd, dim3(nrb), dim3(threads), smem, s, pcurr, psib, c.tri_a, c.nw, c.nh, c.rmin, c.dr,
                      c.dz, c.twiddle, c.fft_m, c.fft_log2, fpc, c.fhat, c.fhat_ld, with_bnd);
}

// tridiagonal solve + inverse DST + update (after the forward coefficients are complete)
// tb_fix: the forward coefficients lack the bottom/top edge terms (superposed fit step)
cudaError_t launch_solve_rest(Ctx& c, const double* psib, double* psi_out, double* psi_inout, const double* psi_ext,
                              double* eps, cudaStream_t s, bool next_norm, bool tb_fix) {
    TbFix fx;
    fx.bot = tb_fix ? psib + 2 * c.nh : nullptr;
    fx.top = psib + 2 * c.nh + (c.nw - 2);
    fx.sink = c.sin_tab;
    fx.idz2 = 1.0 / (c.dz * c.dz);
    int fpc, threads;
    size_t smem;
    solve_shape(c, fpc, threads, smem);
    const int nrb = (c.ni + 2 * fpc - 1) / (2 * fpc);
    cudaError_t e;
    const int L = c.ni_pad / 32;
    const dim3 tg((c.nmode + 3) / 4), tb(128);
    switch (L) {
#define EFIT_TRI(V) case V: e = launch_pdl(k_tridiag_reg<V>, tg, tb, 0, s, c.fhat, c.fhat_ld, c.tri_alpha, c.tri_inv, \
                                           c.tri_cp, c.ni, c.nmode, fx); break;
        EFIT_TRI(1) EFIT_TRI(2) EFIT_TRI(4) EFIT_TRI(8) EFIT_TRI(16)
#undef EFIT_TRI
        default:
            e = launch_pdl(k_tridiag, tg, tb, sizeof(double) * 4 * (32 * (size_t)L + 32), s, c.fhat, c.fhat_ld,
                           c.tri_alpha, c.tri_inv, c.tri_cp, c.ni, L, c.nmode, fx);
    }
    if (e) return e;
    const NextNorm nn = next_norm_args(c, next_norm && psi_inout && !c.steps);  // f3: steps_ before every iteration
    e = launch_pdl(k_dst_inv, dim3(nrb + 1), dim3(threads), smem, s, c.fhat, c.fhat_ld, psib, c.nw, c.nh,
                   c.twiddle, c.fft_m, c.fft_log2, fpc, psi_out, psi_inout, psi_ext, c.eps_part, nn);
    if (e || !psi_inout) return e;
    return launch_pdl(k_norm_fin, dim3(1), dim3(256), 0, s, (const double*)c.eps_part, nrb + 1, (const double*)psi_inout,
                      c.nw, c.nh, c.axbd, eps, nn);
}

cudaError_t launch_solve(Ctx& c, const double* pcurr, const double* psib, double* psi_out, double* psi_inout,
                         const double* psi_ext, double* eps, cudaStream_t s, bool next_norm) {
    cudaError_t e = launch_solve_fwd(c, pcurr, psib, s, 1);
    if (e) return e;
    return launch_solve_rest(c, psib, psi_out, psi_inout, psi_ext, eps, s, next_norm, false);
}

// ================================================================================ left/right via FFT
// The printed Fig. 2 nest is, for each side s, a sum over source rows of symmetric
// Toeplitz products:  psi_b(s, j) = sum_ii sum_jj t_{s,ii}(|j - jj|) x_ii(jj).  With the even
// circular extension c[d] = t(|d|) of length M = 2(nh-1) (d = +-(nh-1) share the same value, so the
// wrap is exact for j, jj in [0, nh)) every row product is a circular convolution, and by linearity
//   psi_b(s, .) = IFFT( sum_ii C_{s,ii} * FFT(x_ii) ),   C_{s,ii} = FFT(c_{s,ii})  (real: c is even).
// C is table data (k_lr_spectra, once at init); per iteration: one FFT per source row pair,
// a frequency-wise multiply-accumulate over rows (fixed order), and one inverse FFT for both sides.
// O(N^2 log N) instead of the nest's 2 N^3 FMAs; same result to rounding (tested against the
// oracle's direct sum at 1e-12).  EFIT_LR_DIRECT=1 selects the direct k_bnd_lr instead.

// Spectra of the circular kernel rows: spec[(s*nh + f)*ldi + ii] = C_{s,ii}[f], f in [0, nh).
__global__ void __launch_bounds__(512) k_lr_spectra(const double* __restrict__ Tedge, long long S, int nw, int nh,
                                                    const double2* __restrict__ W, int M, int log2m, int FPC,
                                                    double* __restrict__ spec, int ldi) {
    extern __shared__ __align__(16) double2 a2[];
    double2* Ws = a2 + 2 * FPC * M;
    const int TPF = blockDim.x / FPC;
    const int f = threadIdx.x / TPF, lt = threadIdx.x - f * TPF;
    const int side = blockIdx.y;
    const int ra = 2 * FPC * blockIdx.x + 2 * f, rb = ra + 1;
    double2* xf = a2 + 2 * f * M;
    for (int k = threadIdx.x; k < M / 2; k += blockDim.x) Ws[k] = W[k];
    const double* ta = Tedge + (long long)side * S + (long long)ra * nh;
    const double* tb = Tedge + (long long)side * S + (long long)rb * nh;
    for (int j = lt; j < M; j += TPF) {
        const int d = j <= nh - 1 ? j : M - j;
        xf[j] = make_double2(ra < nw ? ta[d] : 0.0, rb < nw ? tb[d] : 0.0);
    }
    __syncthreads();
    fft_stockham(xf, xf + M, M, log2m, Ws, lt, TPF);
    const int ro = (fft_stages(log2m) & 1) ? M : 0;
    for (int g = 0; g < FPC; ++g) {
        const int r0 = 2 * FPC * blockIdx.x + 2 * g;
        const double2* res = a2 + 2 * g * M + ro;
        for (int q = threadIdx.x; q < nh; q += blockDim.x) {
            const double2 z = res[q];  // both spectra are real: Re -> row r0, Im -> row r0 + 1
            if (r0 < nw) spec[((long long)side * nh + q) * ldi + r0] = z.x;
            if (r0 + 1 < nw) spec[((long long)side * nh + q) * ldi + r0 + 1] = z.y;
        }
    }
}

// Per iteration: FFT of two source rows x_a + i x_b (zero-padded to M), unpacked to the two
// half spectra X_a[f] = (Z[f] + conj Z[M-f])/2, X_b[f] = (Z[f] - conj Z[M-f])/(2i), f in [0, nh).
__global__ void __launch_bounds__(512) k_lr_fft(const double* __restrict__ pcurr, int nw, int nh,
                                                const double2* __restrict__ W, int M, int log2m, int FPC,
                                                double2* __restrict__ Xh, int ldi) {
    extern __shared__ __align__(16) double2 a2[];
    double2* Ws = a2 + 2 * FPC * M;
    const int TPF = blockDim.x / FPC;
    const int f = threadIdx.x / TPF, lt = threadIdx.x - f * TPF;
    const int ra = 2 * FPC * blockIdx.x + 2 * f, rb = ra + 1;
    double2* xf = a2 + 2 * f * M;
    for (int k = threadIdx.x; k < M / 2; k += blockDim.x) Ws[k] = __ldg(W + k);
    griddep();
    const double* xa = pcurr + (long long)ra * nh;
    const double* xb = pcurr + (long long)rb * nh;
    for (int j = lt; j < M; j += TPF)
        xf[j] = (j < nh) ? make_double2(ra < nw ? xa[j] : 0.0, rb < nw ? xb[j] : 0.0) : make_double2(0.0, 0.0);
    __syncthreads();
    fft_stockham(xf, xf + M, M, log2m, Ws, lt, TPF);
    const int ro = (fft_stages(log2m) & 1) ? M : 0;
    for (int g = 0; g < FPC; ++g) {
        const int r0 = 2 * FPC * blockIdx.x + 2 * g;
        const double2* res = a2 + 2 * g * M + ro;
        for (int q = threadIdx.x; q < nh; q += blockDim.x) {
            const double2 zf = res[q], zm = res[(M - q) & (M - 1)];
            const double2 xa2 = make_double2(0.5 * (zf.x + zm.x), 0.5 * (zf.y - zm.y));
            const double2 xb2 = make_double2(0.5 * (zf.y + zm.y), 0.5 * (zm.x - zf.x));
            double2* dst = Xh + (long long)q * ldi + r0;
            if (r0 + 1 < ldi) {
                dst[0] = xa2;
                dst[1] = xb2;
            } else {
                dst[0] = xa2;
            }
        }
    }
}

// Y_s[f] = sum_ii C_{s,ii}[f] X_ii[f] for both sides; one warp per frequency, lanes over rows,
// fixed butterfly => deterministic.
__global__ void __launch_bounds__(256) k_lr_mac(const double* __restrict__ spec, const double2* __restrict__ Xh,
                                                int nw, int nh, int ldi, double2* __restrict__ Y) {
    griddep();
    const int q = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
    if (q >= nh) return;
    const double* c0 = spec + (long long)q * ldi;
    const double* c1 = spec + ((long long)nh + q) * ldi;
    const double2* x = Xh + (long long)q * ldi;
    double a0r = 0.0, a0i = 0.0, a1r = 0.0, a1i = 0.0;
    for (int ii = lane; ii < nw; ii += 32) {
        const double2 xv = x[ii];
        const double s0 = c0[ii], s1 = c1[ii];
        a0r = fma(s0, xv.x, a0r);
        a0i = fma(s0, xv.y, a0i);
        a1r = fma(s1, xv.x, a1r);
        a1i = fma(s1, xv.y, a1i);
    }
    a0r = warp_sum(a0r);
    a0i = warp_sum(a0i);
    a1r = warp_sum(a1r);
    a1i = warp_sum(a1i);
    if (lane == 0) {
        Y[q] = make_double2(a0r, a0i);
        Y[nh + q] = make_double2(a1r, a1i);
    }
}

// Both real outputs with one inverse FFT: Q = Y_0 + i Y_1 on the full circle (Hermitian
// extension Y_s[M-f] = conj Y_s[f]), q = IFFT(Q) = conj(FFT(conj Q))/M, psi_left = Re q,
// psi_right = Im q.
__global__ void __launch_bounds__(256) k_lr_ifft(const double2* __restrict__ Y, int nh, const double2* __restrict__ W,
                                                 int M, int log2m, double* __restrict__ psib, int jlo, int jhi) {
    extern __shared__ __align__(16) double2 a2[];
    double2* Ws = a2 + 2 * M;
    for (int k = threadIdx.x; k < M / 2; k += blockDim.x) Ws[k] = __ldg(W + k);
    griddep();
    for (int f = threadIdx.x; f < M; f += blockDim.x) {
        double2 y0, y1;
        if (f <= M / 2) {
            y0 = Y[f];
            y1 = Y[nh + f];
        } else {
            const double2 u = Y[M - f], v = Y[nh + M - f];
            y0 = make_double2(u.x, -u.y);
            y1 = make_double2(v.x, -v.y);
        }
        const double2 qv = make_double2(y0.x - y1.y, y0.y + y1.x);  // Y_0 + i Y_1
        a2[f] = make_double2(qv.x, -qv.y);                           // conj
    }
    __syncthreads();
    fft_stockham(a2, a2 + M, M, log2m, Ws, threadIdx.x, blockDim.x);
    const double2* res = a2 + ((fft_stages(log2m) & 1) ? M : 0);
    const double im = 1.0 / (double)M;
    for (int j = jlo + threadIdx.x; j < jhi; j += blockDim.x) {
        const double2 p = res[j];
        psib[j] = p.x * im;
        psib[nh + j] = -p.y * im;
    }
}

static size_t lr_fft_smem(const Ctx& c, int& fpc, int& threads) {
    size_t smem;
    solve_shape(c, fpc, threads, smem);
    return smem;
}

cudaError_t launch_lr_spectra(Ctx& c, cudaStream_t s) {
    int fpc, threads;
    const size_t smem = lr_fft_smem(c, fpc, threads);
    dim3 grid((c.nw + 2 * fpc - 1) / (2 * fpc), 2);
    k_lr_spectra<<<grid, threads, smem, s>>>(c.Tedge, c.S, c.nw, c.nh, c.twiddle, c.fft_m, c.fft_log2, fpc, c.lr_spec,
                                             c.lr_ldi);
    return cudaGetLastError();
}

cudaError_t launch_lr_fft(Ctx& c, double* psib, cudaStream_t s) {
    if (c.jt_hi <= c.jt_lo) return cudaSuccess;  // left/right targets owned by another rank
    int fpc, threads;
    const size_t smem = lr_fft_smem(c, fpc, threads);
    cudaError_t e = launch_pdl(k_lr_fft, dim3((c.nw + 2 * fpc - 1) / (2 * fpc)), dim3(threads), smem, s, c.pcurr,
                               c.nw, c.nh, c.twiddle, c.fft_m, c.fft_log2, fpc, c.lr_xh, c.lr_ldi);
    if (e) return e;
    e = launch_pdl(k_lr_mac, dim3((c.nh + 7) / 8), dim3(256), 0, s, c.lr_spec, c.lr_xh, c.nw, c.nh, c.lr_ldi,
                   c.lr_y);
    if (e) return e;
    return launch_pdl(k_lr_ifft, dim3(1), dim3(256), sizeof(double2) * (size_t)(2 * c.fft_m + c.fft_m / 2), s,
                      c.lr_y, c.nh, c.twiddle, c.fft_m, c.fft_log2, psib, 0, c.nh);
}

cudaError_t prepare_lr_fft(Ctx& c) {
    int fpc, threads;
    const size_t smem = lr_fft_smem(c, fpc, threads);
    cudaError_t e;
    if ((e = raise_smem_limit((const void*)k_lr_spectra, smem))) return e;
    if ((e = raise_smem_limit((const void*)k_lr_fft, smem))) return e;
    return raise_smem_limit((const void*)k_lr_ifft, sizeof(double2) * (size_t)(2 * c.fft_m + c.fft_m / 2));
}

// Caller-supplied current (efit_boundary_flux): copy into the internal zero-padded buffer and
// build the vertically mirrored copy used by the top targets.
__global__ void k_make_pair(const double* __restrict__ I, double* __restrict__ pc, double* __restrict__ pf,
                            int nw, int nh) {
    griddep();
    const int n = nw * nh;
    for (int g = blockIdx.x * blockDim.x + threadIdx.x; g < n; g += gridDim.x * blockDim.x) {
        const int ii = g / nh, m = g - (g / nh) * nh;
        const double v = I[g];
        pc[g] = v;
        pf[ii * nh + (nh - 1 - m)] = v;
    }
}

cudaError_t launch_make_pair(Ctx& c, const double* pcurr, cudaStream_t s) {
    const int n = c.nw * c.nh;
    launch_pdl(k_make_pair, dim3((n + 255) / 256), dim3(256), 0, s, pcurr, c.pcurr, c.pflip, c.nw, c.nh);
    return cudaGetLastError();
}

// One-time kernel attributes: the dynamic shared-memory limit is a per-function, process-wide
// setting, so it is raised to the device opt-in maximum (never lowered by a smaller context).
// Never called during stream capture.
cudaError_t prepare_kernels(Ctx& c) {
    int optin = 0;
    cudaError_t e = cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, c.device);
    if (e) return e;
    g_smem_optin = optin;
    if ((e = response_impl(c, nullptr, nullptr, nullptr, true))) return e;
    auto big = [&](const void* f, size_t need) -> cudaError_t {
        return raise_smem_limit(f, need);
    };
    if ((e = big((const void*)k_lsq<0>, lsq_smem(c)))) return e;
#define EFIT_LSQ_BIG(V) if ((e = big((const void*)k_lsq<V>, lsq_smem(c)))) return e;
    EFIT_LSQ_BIG(7) EFIT_LSQ_BIG(8) EFIT_LSQ_BIG(9) EFIT_LSQ_BIG(10) EFIT_LSQ_BIG(11) EFIT_LSQ_BIG(12)
    EFIT_LSQ_BIG(13) EFIT_LSQ_BIG(14) EFIT_LSQ_BIG(15) EFIT_LSQ_BIG(16) EFIT_LSQ_BIG(17) EFIT_LSQ_BIG(18)
    EFIT_LSQ_BIG(19) EFIT_LSQ_BIG(20) EFIT_LSQ_BIG(21) EFIT_LSQ_BIG(22) EFIT_LSQ_BIG(23) EFIT_LSQ_BIG(24)
#undef EFIT_LSQ_BIG
    if ((e = launch_lr(c, nullptr, true))) return e;
    if ((e = prepare_lr_fft(c))) return e;
    if ((e = big((const void*)k_bnd_tb<kTbGI, kTbUnroll>, 2 * sizeof(double) * c.t.tb_ch))) return e;
    if ((e = big((const void*)k_bnd_tb_otf<kTbGI>, 2 * sizeof(double) * c.t.tb_ch))) return e;
    if ((e = big((const void*)k_bnd_tb_mma<2, kMmaOct, kMmaNP>, sizeof(double) * 16 * (kBatchCh + 2)))) return e;
    if ((e = big((const void*)k_response_mma<3, resp_mma_np(3)>, sizeof(double) * 24 * (kRespBatchGc + 2)))) return e;
    if ((e = big((const void*)k_response_mma<4, resp_mma_np(4)>, sizeof(double) * 32 * (kRespBatchGc + 2)))) return e;
    if ((e = big((const void*)k_response_mma<5, resp_mma_np(5)>, sizeof(double) * 40 * (kRespBatchGc + 2)))) return e;
    {
        const size_t sm = sym_smem(c);
        const void* ks[4] = {(const void*)k_bnd_sym<false, true, kSymUnr, kSymBuf, kSymWg>,
                             (const void*)k_bnd_sym<false, false, kSymUnrC, kSymBufC, kSymWg>,
                             (const void*)k_bnd_sym<true, true, 1, 2, kSymWg>, (const void*)k_bnd_sym<true, false, 1, 2, kSymWg>};
        for (const void* f : ks)
            if ((e = big(f, sm))) return e;
    }
    {
        int fpc, threads;
        size_t smem;
        solve_shape(c, fpc, threads, smem);
        if ((e = big((const void*)k_dst_fwd, smem))) return e;
        if ((e = big((const void*)k_dst_inv, smem))) return e;
        if ((e = big((const void*)k_tridiag, sizeof(double) * 4 * ((size_t)c.ni_pad + 32)))) return e;
    }
    return prepare_steps(c, g_smem_optin);
}

}  // namespace efit
