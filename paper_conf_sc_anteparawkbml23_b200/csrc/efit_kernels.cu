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
//   k_dst_fwd / k_tridiag / k_dst_inv   interior GS solve + update + eps (pflux_ O(N^2), Eq. (1))
// Every reduction has a fixed order, so results are bitwise reproducible run to run and
// independent of the number of ranks.
#include <cfloat>
#include <climits>
#include <cstdio>

#include "efit_device.cuh"
#include "efit_internal.h"

namespace efit {

static int g_smem_optin = 227 * 1024;  // device opt-in shared memory per block (set in prepare_kernels)

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
    double s = __dadd_rn(__dmul_rn(w00, psi[g]), __dmul_rn(w10, psi[g + nh]));
    s = __dadd_rn(s, __dmul_rn(w01, psi[g + 1]));
    s = __dadd_rn(s, __dmul_rn(w11, psi[g + nh + 1]));
    return s;
}

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

// Thomas factors of the radial tridiagonal systems, one per sine mode k = 1..nmode:
//   a_i x_{i-1} + (-2/dR^2 + lambda_k) x_i + c_i x_{i+1},  lambda_k = -4 sin^2(pi k/(2(n+1)))/dZ^2
__global__ void k_tri_factors(double* __restrict__ tri_a, double* __restrict__ cp, double* __restrict__ inv,
                              int ni, int nmode, double rmin, double dr, double dz) {
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
        cp[(long long)(i - 1) * nmode + k] = cpi;
        inv[(long long)(i - 1) * nmode + k] = 1.0 / den;
        cprev = cpi;
    }
}

__global__ void k_twiddles(double2* __restrict__ w, int M) {
    int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= M / 2) return;
    double s, c;
    sincospi(2.0 * (double)k / (double)M, &s, &c);
    w[k] = make_double2(c, -s);
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
    e = cudaMemsetAsync(c.ipair, 0, sizeof(double2) * (size_t)(((n + c.t.tb_ch - 1) / c.t.tb_ch) * c.t.tb_ch), s);
    if (e) return e;
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, c.device);
    const int bs = 256;
    k_green_slabs<<<sms * 8, bs, 0, s>>>(c.Tedge, c.S, 2, 0, nw - 1, nw, nh, c.rmin, c.dr, c.dz);
    if (c.T && c.i_hi > c.i_lo)
        k_green_slabs<<<sms * 16, bs, 0, s>>>(c.T, c.S, c.i_hi - c.i_lo, c.i_lo, 1, nw, nh, c.rmin, c.dr, c.dz);
    if (c.m_hi > c.m_lo)
        k_green_diag<<<sms * 16, bs, 0, s>>>(c.Gd, c.S, c.m_hi - c.m_lo, c.m_lo, c.dgeo, c.dkind, nw, nh,
                                              c.rmin, c.dr, c.zmin, c.dz);
    k_inlim<<<(int)((n + bs - 1) / bs), bs, 0, s>>>(c.inlim, c.lim, c.n_lim, nw, nh, c.rmin, c.dr, c.zmin, c.dz);
    k_tri_factors<<<(c.nmode + 63) / 64, 64, 0, s>>>(c.tri_a, c.tri_cp, c.tri_inv, c.ni, c.nmode, c.rmin, c.dr, c.dz);
    k_twiddles<<<(c.fft_m / 2 + 255) / 256, 256, 0, s>>>(c.twiddle, c.fft_m);
    e = cudaMemsetAsync(c.status, 0, sizeof(int), s);
    if (e) return e;
    e = cudaMemsetAsync(c.tickets, 0, sizeof(unsigned) * 8, s);
    if (e) return e;
    return cudaGetLastError();
}

// ================================================================================ normalize

// psi_axis = s * max_{g in limiter} s psi_g (ties: lowest g);  psi_bdry = s * max over limiter
// vertices of s * bilinear(psi) (ties: lowest vertex).  Last-block pattern: the final block
// combines the per-block partials; `ticket` returns to 0 for the next launch.
__global__ void __launch_bounds__(256) k_normalize(const double* __restrict__ psi, const uint8_t* __restrict__ inlim,
                                                   int nw, int nh, double rmin, double dr, double zmin, double dz,
                                                   int sgn, const double* __restrict__ lim, int n_lim,
                                                   double* __restrict__ part, unsigned* ticket,
                                                   double* __restrict__ axbd, int* status) {
    __shared__ double sv[8];
    __shared__ long long si[8];
    __shared__ bool last;
    const int n = nw * nh;
    const double s = (double)sgn;
    double best = -DBL_MAX;
    long long bi = LLONG_MAX;
    bool bad = false;
    for (int g = blockIdx.x * blockDim.x + threadIdx.x; g < n; g += gridDim.x * blockDim.x) {
        double p = psi[g];
        if (!isfinite(p)) bad = true;
        if (inlim[g]) argmax_merge(best, bi, s * p, (long long)g);
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
        __threadfence();
        unsigned t = atomicAdd(ticket, 1u);
        last = (t == gridDim.x - 1);
    }
    __syncthreads();
    if (!last) return;
    __threadfence();
    best = -DBL_MAX;
    bi = LLONG_MAX;
    for (int b = threadIdx.x; b < (int)gridDim.x; b += blockDim.x) {
        double v = __ldcg(part + 2 * b);
        double ix = __ldcg(part + 2 * b + 1);
        argmax_merge(best, bi, v, (long long)ix);
    }
    warp_argmax(best, bi);
    if (l == 0) { sv[w] = best; si[w] = bi; }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int q = 1; q < (int)(blockDim.x >> 5); ++q) argmax_merge(best, bi, sv[q], si[q]);
        sv[0] = best; si[0] = bi;
    }
    __syncthreads();
    long long gax = si[0];
    __syncthreads();
    // limiter vertices
    double vb = -DBL_MAX;
    long long vi = LLONG_MAX;
    for (int v = threadIdx.x; v < n_lim; v += blockDim.x) {
        double pv = bilinear(psi, nw, nh, rmin, dr, zmin, dz, lim[v], lim[n_lim + v]);
        argmax_merge(vb, vi, s * pv, (long long)v);
    }
    warp_argmax(vb, vi);
    if (l == 0) { sv[w] = vb; si[w] = vi; }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int q = 1; q < (int)(blockDim.x >> 5); ++q) argmax_merge(vb, vi, sv[q], si[q]);
        double pa = (gax == LLONG_MAX) ? 0.0 : psi[gax];
        double pb = (vi == LLONG_MAX) ? 0.0 : bilinear(psi, nw, nh, rmin, dr, zmin, dz, lim[vi], lim[n_lim + vi]);
        axbd[0] = pa;
        axbd[1] = pb;
        if (gax == LLONG_MAX || !(s * (pa - pb) > 0.0)) atomicOr(status, EFIT_ST_NOPLASMA);
        *ticket = 0u;
    }
}

cudaError_t launch_normalize(Ctx& c, const double* psi, cudaStream_t s) {
    k_normalize<<<c.t.red_blocks, 256, 0, s>>>(psi, c.inlim, c.nw, c.nh, c.rmin, c.dr, c.zmin, c.dz,
                                               c.ip_sign, c.lim, c.n_lim, c.norm_part, c.tickets + 0,
                                               c.axbd, c.status);
    return cudaGetLastError();
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

// One CTA per chunk of `gc` nodes: basis values of the chunk (fused basis evaluation, never
// materialised in HBM) into shared memory Bs[k][q], then warps stream the Gd rows of the chunk
// with 128-bit loads, MB rows at a time, accumulating MB x NB dot products in registers.
template <int NB, int MB>
__global__ void __launch_bounds__(256) k_response(const double* __restrict__ Gd, long long S, int nrows,
                                                  const double* __restrict__ psi, const uint8_t* __restrict__ inlim,
                                                  const double* __restrict__ axbd, int nw, int nh,
                                                  double rmin, double dr, double cell, BasisParams bp, int gc,
                                                  double* __restrict__ part, double* __restrict__ cnt_part) {
    extern __shared__ __align__(16) double Bs[];  // [NB][gc]
    __shared__ int cnt_s[8];
    const int n = nw * nh;
    const int c = blockIdx.x;
    const int g0 = c * gc;
    const double pa = axbd[0], pb = axbd[1];
    int cnt = 0;
    for (int q = threadIdx.x; q < gc; q += blockDim.x) {
        int g = g0 + q;
        double f[NB];
#pragma unroll
        for (int k = 0; k < NB; ++k) f[k] = 0.0;
        double h;
        if (g < n && node_psihat(psi, inlim, g, pa, pb, h)) {
            double R = grid_coord(rmin, g / nh, dr);
            basis_eval<NB>(bp, h, R, f);
            ++cnt;
        }
#pragma unroll
        for (int k = 0; k < NB; ++k) Bs[k * gc + q] = cell * f[k];
    }
    int wc = __reduce_add_sync(0xffffffffu, cnt);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (lane == 0) cnt_s[warp] = wc;
    __syncthreads();
    if (threadIdx.x == 0) {
        int t = 0;
        for (int q = 0; q < (int)(blockDim.x >> 5); ++q) t += cnt_s[q];
        cnt_part[c] = (double)t;
    }
    const int nwarps = blockDim.x >> 5;
    const int nmb = (nrows + MB - 1) / MB;
    const int qend = min(gc, n - g0);  // valid nodes in this chunk (pairs may read 1 padding entry)
    for (int mb = warp; mb < nmb; mb += nwarps) {
        double acc[MB][NB];
#pragma unroll
        for (int r = 0; r < MB; ++r)
#pragma unroll
            for (int k = 0; k < NB; ++k) acc[r][k] = 0.0;
        const double* rowp[MB];
#pragma unroll
        for (int r = 0; r < MB; ++r) {
            int row = mb * MB + r;
            rowp[r] = Gd + (long long)(row < nrows ? row : nrows - 1) * S + g0;
        }
#pragma unroll 2
        for (int q = 2 * lane; q < qend; q += 64) {
            double2 gv[MB];
#pragma unroll
            for (int r = 0; r < MB; ++r) gv[r] = ldg_stream(rowp[r] + q);
#pragma unroll
            for (int k = 0; k < NB; ++k) {
                double2 b = *reinterpret_cast<const double2*>(&Bs[k * gc + q]);
#pragma unroll
                for (int r = 0; r < MB; ++r) {
                    acc[r][k] = fma(gv[r].x, b.x, acc[r][k]);
                    acc[r][k] = fma(gv[r].y, b.y, acc[r][k]);
                }
            }
        }
#pragma unroll
        for (int r = 0; r < MB; ++r) {
            int row = mb * MB + r;
#pragma unroll
            for (int k = 0; k < NB; ++k) {
                double v = warp_sum(acc[r][k]);
                if (lane == 0 && row < nrows) part[((long long)c * nrows + row) * NB + k] = v;
            }
        }
    }
}

// out[r][k] = sum over chunks in index order; total masked count -> status.
__global__ void k_resp_reduce(const double* __restrict__ part, const double* __restrict__ cnt_part, int nchunk,
                              int nrows, int nb, double* __restrict__ out, int* status) {
    int t = blockIdx.x * blockDim.x + threadIdx.x;
    int total = nrows * nb;
    if (t < total) {
        double s = 0.0;
        for (int c = 0; c < nchunk; ++c) s += part[(long long)c * total + t];
        out[t] = s;
    }
    if (t == 0) {
        double cnt = 0.0;
        for (int c = 0; c < nchunk; ++c) cnt += cnt_part[c];
        if (cnt == 0.0) atomicOr(status, EFIT_ST_NOPLASMA);
    }
}

template <int NB>
static void launch_resp_nb(Ctx& c, const double* psi, double* part, cudaStream_t s, int nrows, bool prepare) {
    const int gc = c.t.resp_gc;
    const size_t smem = sizeof(double) * NB * gc;
    BasisParams bp = basis_params(c);
    const double* Gd = c.Gd;
    int mb = c.t.resp_mb;
#define EFIT_RESP_LAUNCH(MBV)                                                                              \
    do {                                                                                                   \
        auto kern = k_response<NB, MBV>;                                                                   \
        if (prepare) { raise_smem_limit((const void*)kern, smem); break; } \
        kern<<<c.t.resp_nchunk, 256, smem, s>>>(Gd, c.S, nrows, psi, c.inlim, c.axbd, c.nw, c.nh, c.rmin, c.dr, \
                                                c.dr * c.dz, bp, gc, part, c.resp_cnt);                  \
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
    k_resp_reduce<<<(total + 255) / 256, 256, 0, s>>>(c.resp_part, c.resp_cnt, c.t.resp_nchunk, nrows, c.nb,
                                                      resp_rows, c.status);
    return cudaGetLastError();
}

cudaError_t launch_response(Ctx& c, const double* psi, double* resp_rows, cudaStream_t s) {
    return response_impl(c, psi, resp_rows, s, false);
}

// ================================================================================ least squares

// One CTA: rows scaled by 1/sigma, columns to unit 2-norm, Householder QR (reflectors
// v = x + sign(x_0)|x| e_0), back substitution, unscale; chi2 = sum((meas - A c)/sigma)^2.
// Reductions are fixed-order (warp shuffles + one ordered pass), so the result is deterministic.

__global__ void __launch_bounds__(256) k_lsq(const double* __restrict__ resp, const double* __restrict__ meas,
                                             const double* __restrict__ sigma, int nd, int nb,
                                             double* __restrict__ coef, double* __restrict__ chi2, int* status) {
    extern __shared__ __align__(16) double sm[];
    double* A = sm;                      // [nb][nd] column-major (scaled)
    double* b = A + (size_t)nb * nd;     // [nd]
    double* v = b + nd;                  // [nd]
    double* red = v + nd;                // [32 + 64]
    double* scale = red + 96;            // [nb]
    double* x = scale + 32;              // [nb]
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nwarp = blockDim.x >> 5;
    __shared__ int bad;
    if (tid == 0) bad = (*status & (EFIT_ST_NOPLASMA | EFIT_ST_NONFINITE)) ? 1 : 0;
    for (int e = tid; e < nd * nb; e += blockDim.x) {
        int m = e / nb, k = e - (e / nb) * nb;
        A[(size_t)k * nd + m] = resp[e] / sigma[m];
    }
    for (int m = tid; m < nd; m += blockDim.x) b[m] = meas[m] / sigma[m];
    __syncthreads();
    // column norms: warp per column
    for (int k = warp; k < nb; k += nwarp) {
        double s = 0.0;
        for (int m = lane; m < nd; m += 32) { double a = A[(size_t)k * nd + m]; s += a * a; }
        s = warp_sum(s);
        if (lane == 0) scale[k] = sqrt(s);
    }
    __syncthreads();
    for (int e = tid; e < nd * nb; e += blockDim.x) {
        int k = e / nd;
        double sc = scale[k];
        A[e] = sc > 0.0 ? A[e] / sc : 0.0;
    }
    __syncthreads();
    for (int k = 0; k < nb; ++k) {
        // norm of column k below (and incl.) the diagonal: warp 0
        if (warp == 0) {
            double s = 0.0;
            for (int m = k + lane; m < nd; m += 32) { double a = A[(size_t)k * nd + m]; s += a * a; }
            s = warp_sum(s);
            if (lane == 0) {
                double nx = sqrt(s);
                double x0 = A[(size_t)k * nd + k];
                double alpha = x0 >= 0.0 ? -nx : nx;      // R_kk = alpha
                red[0] = alpha;
                red[1] = nx * (nx + fabs(x0));            // v^T v / 2 with v = x - alpha e_k
            }
        }
        __syncthreads();
        double alpha = red[0], vtv2 = red[1];
        for (int m = tid; m < nd; m += blockDim.x) v[m] = (m < k) ? 0.0 : (m == k ? A[(size_t)k * nd + k] - alpha : A[(size_t)k * nd + m]);
        __syncthreads();
        // apply H = I - v v^T / vtv2 to columns j > k and to b (warp per column)
        for (int j = k + 1 + warp; j <= nb; j += nwarp) {
            double* col = (j < nb) ? A + (size_t)j * nd : b;
            double s = 0.0;
            for (int m = k + lane; m < nd; m += 32) s += v[m] * col[m];
            s = warp_sum(s);
            double f = vtv2 > 0.0 ? s / vtv2 : 0.0;
            for (int m = k + lane; m < nd; m += 32) col[m] -= f * v[m];
        }
        __syncthreads();
        if (tid == 0) {
            A[(size_t)k * nd + k] = alpha;
            for (int m = k + 1; m < nd; ++m) A[(size_t)k * nd + m] = 0.0;
        }
        __syncthreads();
    }
    if (tid == 0) {
        double rmax = 0.0;
        for (int k = 0; k < nb; ++k) rmax = fmax(rmax, fabs(A[(size_t)k * nd + k]));
        bool sing = false;
        for (int k = 0; k < nb; ++k)
            if (!(fabs(A[(size_t)k * nd + k]) >= 1e-13 * rmax) || !(scale[k] > 0.0)) sing = true;
        if (sing) { atomicOr(status, EFIT_ST_SINGULAR); bad = 1; }
        for (int k = nb - 1; k >= 0; --k) {
            double s = b[k];
            for (int j = k + 1; j < nb; ++j) s -= A[(size_t)j * nd + k] * x[j];
            x[k] = s / A[(size_t)k * nd + k];
        }
        for (int k = 0; k < nb; ++k) x[k] = x[k] / scale[k];
    }
    __syncthreads();
    // chi2 with the unscaled matrix
    double s = 0.0;
    for (int m = tid; m < nd; m += blockDim.x) {
        double r = meas[m];
        for (int k = 0; k < nb; ++k) r -= resp[(size_t)m * nb + k] * x[k];
        r /= sigma[m];
        s += r * r;
    }
    s = warp_sum(s);
    if (lane == 0) red[32 + warp] = s;
    __syncthreads();
    if (tid == 0) {
        double t = 0.0;
        for (int q = 0; q < nwarp; ++q) t += red[32 + q];
        const double nanv = __longlong_as_double(0x7ff8000000000000ULL);
        *chi2 = bad ? nanv : t;
        for (int k = 0; k < nb; ++k) coef[k] = bad ? nanv : x[k];
    }
}

static size_t lsq_smem(const Ctx& c) {
    return sizeof(double) * ((size_t)c.nb * c.ndiag + 2 * (size_t)c.ndiag + 96 + 32 + 32);
}

cudaError_t launch_lsq(Ctx& c, const double* resp, const double* meas, const double* sigma, double* coef,
                       double* chi2, cudaStream_t s) {
    size_t smem = lsq_smem(c);
    k_lsq<<<1, 256, smem, s>>>(resp, meas, sigma, c.ndiag, c.nb, coef, chi2, c.status);
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
                          double2* __restrict__ ipair) {
    const int n = nw * nh;
    const double pa = axbd[0], pb = axbd[1];
    double cf[NB];
#pragma unroll
    for (int k = 0; k < NB; ++k) cf[k] = coef[k];
    for (int g = blockIdx.x * blockDim.x + threadIdx.x; g < n; g += gridDim.x * blockDim.x) {
        double I = current_at<NB>(psi, inlim, g, nh, pa, pb, rmin, dr, cell, bp, cf);
        if (pcurr) pcurr[g] = I;
        if (ipair) {
            int ii = g / nh, m = g - (g / nh) * nh;
            int gf = ii * nh + (nh - 1 - m);
            double If = current_at<NB>(psi, inlim, gf, nh, pa, pb, rmin, dr, cell, bp, cf);
            ipair[g] = make_double2(I, If);
        }
    }
}

cudaError_t launch_current(Ctx& c, const double* psi, const double* coef, double* pcurr, bool pair,
                           cudaStream_t s) {
    BasisParams bp = basis_params(c);
    const int n = c.nw * c.nh;
    const int blocks = (n + 255) / 256;
    double2* ip = pair ? c.ipair : nullptr;
    switch (c.nb) {
#define EFIT_NB_CASE(V) \
    case V: k_current<V><<<blocks, 256, 0, s>>>(psi, c.inlim, c.axbd, coef, c.nw, c.nh, c.rmin, c.dr, c.dr * c.dz, bp, pcurr, ip); break;
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
// i.e. two dot products of slab T[i] with the (I, I_flipped) pair array.  A CTA owns a chunk of
// `ch` slab entries (its pair values staged once in shared memory) and GI slabs; every T byte is
// read from HBM exactly once with 128-bit streaming loads.
template <int GI>
__global__ void __launch_bounds__(256) k_bnd_tb(const double* __restrict__ T, long long S, int nslab, int row_lo,
                                                int n, const double2* __restrict__ ipair, int ch,
                                                double* __restrict__ part, int nw) {
    extern __shared__ __align__(16) double2 ips[];  // [ch]
    __shared__ double red[8][2 * GI];
    const int c = blockIdx.x, grp = blockIdx.y;
    const long long e0 = (long long)c * ch;
    const int len = (int)min((long long)ch, (long long)n - e0);  // valid entries in this chunk
    for (int q = threadIdx.x; q < ch; q += blockDim.x) ips[q] = ipair[e0 + q];
    __syncthreads();
    double a0[GI], a1[GI];
#pragma unroll
    for (int t = 0; t < GI; ++t) { a0[t] = 0.0; a1[t] = 0.0; }
    const int s0 = grp * GI;
#pragma unroll
    for (int t = 0; t < GI; ++t) {
        const int sl = s0 + t;
        if (sl < nslab) {
            const double* base = T + (long long)sl * S + e0;
#pragma unroll 4
            for (int q = 2 * threadIdx.x; q < len; q += 2 * blockDim.x) {
                double2 tv = ldg_stream(base + q);
                double2 p0 = ips[q], p1 = ips[q + 1];
                a0[t] = fma(tv.x, p0.x, a0[t]);
                a1[t] = fma(tv.x, p0.y, a1[t]);
                a0[t] = fma(tv.y, p1.x, a0[t]);
                a1[t] = fma(tv.y, p1.y, a1[t]);
            }
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
            double s = 0.0;
            for (int w = 0; w < (int)(blockDim.x >> 5); ++w) s += red[w][threadIdx.x];
            part[((long long)c * nw + row_lo + sl) * 2 + side] = s;
        }
    }
}

// Left/right targets (the printed Fig. 2 nest): for side s (slab i = 0 or nw-1),
//   psi_b(s, j) = sum_ii sum_jj T[s][ii][|j - jj|] I[ii][jj].
// Each row ii is a symmetric Toeplitz product.  A warp owns JT consecutive targets j0..j0+JT-1,
// lanes own contiguous jj ranges and keep the JT kernel values t[|j - jj|] in a register
// window that slides by one per jj step (one new shared-memory load per step, slot index
// (a - u) mod JT resolved at compile time by unrolling).  CTA = 8 warps x JT targets, one block
// of `iib` source rows; partial sums per block are reduced in block order by k_bnd_reduce.
template <int JT>
__global__ void __launch_bounds__(256) k_bnd_lr(const double* __restrict__ Tedge, long long S,
                                                const double* __restrict__ I, int nw, int nh, int iib,
                                                int jt_lo, double* __restrict__ part) {
    extern __shared__ __align__(16) double sm[];
    double* ts = sm;                    // [iib][nh] kernel rows
    double* xs = sm + (size_t)iib * nh; // [iib][nh] current rows
    const int tile = jt_lo + blockIdx.x;
    const int blk = blockIdx.y;
    const int side = blockIdx.z;
    const int ii0 = blk * iib;
    const int nrow = min(iib, nw - ii0);
    const double* tsrc = Tedge + (long long)side * S + (long long)ii0 * nh;
    const double* xsrc = I + (long long)ii0 * nh;
    for (int e = threadIdx.x; e < nrow * nh; e += blockDim.x) {
        ts[e] = tsrc[e];
        xs[e] = xsrc[e];
    }
    __syncthreads();
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int j0 = (tile * 8 + warp) * JT;
    if (j0 >= nh) return;
    const int L = (nh + 31) / 32;
    const int jb = lane * L;
    const int je = min(nh, jb + L);
    double acc[JT];
#pragma unroll
    for (int a = 0; a < JT; ++a) acc[a] = 0.0;
    if (jb < je) {
        for (int r = 0; r < nrow; ++r) {
            const double* t = ts + (size_t)r * nh;
            const double* x = xs + (size_t)r * nh;
            double w[JT];
            // slot (a - u) mod JT holds t[|j0 + a - jj|] at step u (jj = jb + u)
#pragma unroll
            for (int a = 0; a < JT; ++a) {
                int d = j0 + a - jb;
                d = d < 0 ? -d : d;
                w[a] = d < nh ? t[d] : 0.0;
            }
            for (int jj = jb; jj < je; jj += JT) {
#pragma unroll
                for (int u = 0; u < JT; ++u) {
                    if (jj + u < je) {
                        const double xv = x[jj + u];
#pragma unroll
                        for (int a = 0; a < JT; ++a) acc[a] = fma(w[(a - u + JT) % JT], xv, acc[a]);
                        // next step needs t[|j0 - (jj+u+1)|] in slot (-(u+1)) mod JT
                        int d = j0 - (jj + u + 1);
                        d = d < 0 ? -d : d;
                        w[(2 * JT - 1 - u) % JT] = d < nh ? t[d] : 0.0;
                    }
                }
            }
        }
    }
#pragma unroll
    for (int a = 0; a < JT; ++a) {
        double v = warp_sum(acc[a]);
        const int j = j0 + a;
        if (lane == 0 && j < nh) part[((long long)blk * 2 + side) * nh + j] = v;
    }
}

// psi_b in edge order from the partials (fixed block order).
__global__ void k_bnd_reduce(const double* __restrict__ tb_part, int tb_nchunk, const double* __restrict__ lr_part,
                             int lr_nblk, int nw, int nh, int i_lo, int i_hi, int jlo, int jhi,
                             double* __restrict__ psib) {
    const int n_edge = 2 * nh + 2 * (nw - 2);
    int p = blockIdx.x * blockDim.x + threadIdx.x;
    if (p >= n_edge) return;
    double s = 0.0;
    if (p < 2 * nh) {
        const int side = p < nh ? 0 : 1;
        const int j = p - side * nh;
        if (j < jlo || j >= jhi) return;
        for (int b = 0; b < lr_nblk; ++b) s += lr_part[((long long)b * 2 + side) * nh + j];
    } else {
        const int q = p - 2 * nh;
        const int side = q < nw - 2 ? 0 : 1;
        const int i = q - side * (nw - 2) + 1;
        if (i < i_lo || i >= i_hi) return;
        for (int c = 0; c < tb_nchunk; ++c) s += tb_part[((long long)c * nw + i) * 2 + side];
    }
    psib[p] = s;
}

// On-the-fly variant of k_bnd_tb: G recomputed from (R_i, R_ii, m dZ) with the same device
// function as the table build and the same summation order => bitwise equal to table mode.
template <int GI>
__global__ void __launch_bounds__(256) k_bnd_tb_otf(int row_lo, int nslab, int nw, int nh, double rmin, double dr,
                                                    double dz, const double2* __restrict__ ipair, int ch,
                                                    double* __restrict__ part) {
    extern __shared__ __align__(16) double2 ips[];
    __shared__ double red[8][2 * GI];
    const int n = nw * nh;
    const int c = blockIdx.x, grp = blockIdx.y;
    const long long e0 = (long long)c * ch;
    const int len = (int)min((long long)ch, (long long)n - e0);
    for (int q = threadIdx.x; q < ch; q += blockDim.x) ips[q] = ipair[e0 + q];
    __syncthreads();
    double a0[GI], a1[GI];
#pragma unroll
    for (int t = 0; t < GI; ++t) { a0[t] = 0.0; a1[t] = 0.0; }
    const int s0 = grp * GI;
#pragma unroll
    for (int t = 0; t < GI; ++t) {
        const int sl = s0 + t;
        if (sl < nslab) {
            const int i = row_lo + sl;
            const double Ri = grid_coord(rmin, i, dr);
            for (int q = 2 * threadIdx.x; q < len; q += 2 * blockDim.x) {
                double tv[2];
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    long long e = e0 + q + h;
                    if (e < n) {
                        int ii = (int)(e / nh), m = (int)(e - (long long)ii * nh);
                        double Rs = grid_coord(rmin, ii, dr);
                        tv[h] = (i == ii && m == 0) ? green_self(Ri, dr, dz)
                                                    : green_psi(Ri, __dmul_rn((double)m, dz), Rs, 0.0);
                    } else {
                        tv[h] = 0.0;
                    }
                }
                double2 p0 = ips[q], p1 = ips[q + 1];
                a0[t] = fma(tv[0], p0.x, a0[t]);
                a1[t] = fma(tv[0], p0.y, a1[t]);
                a0[t] = fma(tv[1], p1.x, a0[t]);
                a1[t] = fma(tv[1], p1.y, a1[t]);
            }
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
            double s = 0.0;
            for (int w = 0; w < (int)(blockDim.x >> 5); ++w) s += red[w][threadIdx.x];
            part[((long long)c * nw + row_lo + sl) * 2 + side] = s;
        }
    }
}

constexpr int kTbGI = 8;
constexpr int kLrJT = 16;

cudaError_t launch_boundary(Ctx& c, const double* pcurr, double* psib, cudaStream_t s) {
    const int nslab = c.i_hi - c.i_lo;
    const size_t smem_tb = sizeof(double2) * c.t.tb_ch;
    if (nslab > 0) {
        dim3 grid(c.t.tb_nchunk, c.t.tb_ngroup);
        if (c.mode == EFIT_GREEN_TABLE) {
            k_bnd_tb<kTbGI><<<grid, 256, smem_tb, s>>>(c.T, c.S, nslab, c.i_lo, c.nw * c.nh, c.ipair, c.t.tb_ch,
                                                       c.tb_part, c.nw);
        } else {
            k_bnd_tb_otf<kTbGI><<<grid, 256, smem_tb, s>>>(c.i_lo, nslab, c.nw, c.nh, c.rmin, c.dr, c.dz, c.ipair,
                                                           c.t.tb_ch, c.tb_part);
        }
        cudaError_t e = cudaGetLastError();
        if (e) return e;
    }
    const int ntile = c.jt_hi - c.jt_lo;
    if (ntile > 0) {
        const size_t smem_lr = sizeof(double) * 2 * (size_t)c.t.lr_iib * c.nh;
        dim3 grid(ntile, c.t.lr_nblk, 2);
        k_bnd_lr<kLrJT><<<grid, 256, smem_lr, s>>>(c.Tedge, c.S, pcurr, c.nw, c.nh, c.t.lr_iib, c.jt_lo, c.lr_part);
        cudaError_t e = cudaGetLastError();
        if (e) return e;
    }
    const int jlo = c.jt_lo * 8 * kLrJT, jhi = min(c.nh, c.jt_hi * 8 * kLrJT);
    k_bnd_reduce<<<(c.n_edge + 255) / 256, 256, 0, s>>>(c.tb_part, c.t.tb_nchunk, c.lr_part, c.t.lr_nblk, c.nw,
                                                        c.nh, c.i_lo, c.i_hi, jlo, jhi, psib);
    return cudaGetLastError();
}

// ================================================================================ interior solve

// In-place radix-2 complex FFT (forward, exp(-2 pi i jk/M)) of M = 2^log2m points in shared
// memory; input must already be in bit-reversed order.  Twiddles W[k] = exp(-2 pi i k/M).
__device__ void fft_smem(double2* a, int M, int log2m, const double2* __restrict__ W) {
    for (int st = 1; st <= log2m; ++st) {
        const int half = 1 << (st - 1);
        const int tstride = M >> st;
        for (int b = threadIdx.x; b < M / 2; b += blockDim.x) {
            const int grp = b >> (st - 1);
            const int pos = b & (half - 1);
            const int i0 = (grp << st) + pos;
            const int i1 = i0 + half;
            const double2 w = __ldg(W + pos * tstride);
            const double2 u = a[i0], v = a[i1];
            const double2 t = make_double2(w.x * v.x - w.y * v.y, w.x * v.y + w.y * v.x);
            a[i0] = make_double2(u.x + t.x, u.y + t.y);
            a[i1] = make_double2(u.x - t.x, u.y - t.y);
        }
        __syncthreads();
    }
}

__device__ __forceinline__ int bitrev(int x, int log2m) { return (int)(__brev((unsigned)x) >> (32 - log2m)); }

// Forward DST-I along Z of the right-hand side of two interior rows at once (packed as the real
// and imaginary parts of one complex FFT of the odd extension, length M = 2(n+1)):
//   f_ij = -mu0 R_i I_ij/(dR dZ) - (Dirichlet terms of the edge values psi_b).
// DST_k(x) = -Im(Z_k)/2 for the real-part row, Re(Z_k)/2 for the imaginary-part row.
__global__ void __launch_bounds__(256) k_dst_fwd(const double* __restrict__ pcurr, const double* __restrict__ psib,
                                                 const double* __restrict__ tri_a, int nw, int nh, double rmin,
                                                 double dr, double dz, const double2* __restrict__ W, int M,
                                                 int log2m, double* __restrict__ fhat) {
    extern __shared__ __align__(16) double2 a2[];  // [M]
    const int n = nh - 2, ni = nw - 2;
    const int r0 = 1 + 2 * blockIdx.x;  // first row of the pair
    const double idz2 = 1.0 / (dz * dz);
    const double cellinv = 1.0 / (dr * dz);
    for (int j = threadIdx.x; j < M; j += blockDim.x) {
        double v[2] = {0.0, 0.0};
        int jj = 0;
        double sgn = 0.0;
        if (j >= 1 && j <= n) { jj = j; sgn = 1.0; }
        else if (j >= n + 2) { jj = M - j; sgn = -1.0; }
        if (sgn != 0.0) {
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                const int i = r0 + h;
                if (i > ni) continue;
                const double R = grid_coord(rmin, i, dr);
                double f = -kMu0 * R * pcurr[(long long)i * nh + jj] * cellinv;
                if (i == 1) f -= tri_a[0] * psib[jj];                                   // left edge
                if (i == ni) f -= (2.0 / (dr * dr) - tri_a[ni - 1]) * psib[nh + jj];    // right edge (c_ni)
                if (jj == 1) f -= psib[2 * nh + (i - 1)] * idz2;                        // bottom edge
                if (jj == n) f -= psib[2 * nh + (nw - 2) + (i - 1)] * idz2;             // top edge
                v[h] = sgn * f;
            }
        }
        a2[bitrev(j, log2m)] = make_double2(v[0], v[1]);
    }
    __syncthreads();
    fft_smem(a2, M, log2m, W);
    for (int k = 1 + threadIdx.x; k <= n; k += blockDim.x) {
        const double2 z = a2[k];
        fhat[(long long)(r0 - 1) * n + (k - 1)] = -0.5 * z.y;
        if (r0 + 1 <= ni) fhat[(long long)r0 * n + (k - 1)] = 0.5 * z.x;
    }
}

// Radial tridiagonal solve per sine mode (Thomas with precomputed factors), in place.
__global__ void k_tridiag(double* __restrict__ fhat, const double* __restrict__ tri_a,
                          const double* __restrict__ cp, const double* __restrict__ inv, int ni, int nmode) {
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= nmode) return;
    double d = 0.0;
    for (int i = 0; i < ni; ++i) {
        const long long o = (long long)i * nmode + k;
        d = (fhat[o] - (i > 0 ? tri_a[i] * d : 0.0)) * inv[o];
        fhat[o] = d;
    }
    double x = 0.0;
    for (int i = ni - 1; i >= 0; --i) {
        const long long o = (long long)i * nmode + k;
        x = fhat[o] - (i < ni - 1 ? cp[o] * x : 0.0);
        fhat[o] = x;
    }
}

// Inverse DST-I (same transform, scale 2/(n+1)) of two rows, then either
//   psi_out = psi_p                                  (efit_interior_solve), or
//   psi_inout <- psi_p + psi_ext, eps partial max     (efit_fit_step),
// edges (j = 0, nh-1, and rows 0, nw-1 in the extra last block) take psi_b.
__global__ void __launch_bounds__(256) k_dst_inv(const double* __restrict__ fhat, const double* __restrict__ psib,
                                                 int nw, int nh, const double2* __restrict__ W, int M, int log2m,
                                                 double* __restrict__ psi_out, double* __restrict__ psi_inout,
                                                 const double* __restrict__ psi_ext, double* __restrict__ eps_part,
                                                 unsigned* ticket, const double* __restrict__ axbd,
                                                 double* __restrict__ eps) {
    extern __shared__ __align__(16) double2 a2[];
    __shared__ double wmax[8];
    __shared__ bool last;
    const int n = nh - 2, ni = nw - 2;
    const int npairs = (ni + 1) / 2;
    double dmax = 0.0;
    auto emit = [&](long long g, double pp) {
        if (psi_out) psi_out[g] = pp;
        if (psi_inout) {
            const double nv = pp + psi_ext[g];
            dmax = fmax(dmax, fabs(nv - psi_inout[g]));
            psi_inout[g] = nv;
        }
    };
    if ((int)blockIdx.x < npairs) {
        const int r0 = 1 + 2 * blockIdx.x;
        for (int j = threadIdx.x; j < M; j += blockDim.x) {
            double v[2] = {0.0, 0.0};
            if (j >= 1 && j <= n) {
                v[0] = fhat[(long long)(r0 - 1) * n + (j - 1)];
                if (r0 + 1 <= ni) v[1] = fhat[(long long)r0 * n + (j - 1)];
            } else if (j >= n + 2) {
                const int jj = M - j;
                v[0] = -fhat[(long long)(r0 - 1) * n + (jj - 1)];
                if (r0 + 1 <= ni) v[1] = -fhat[(long long)r0 * n + (jj - 1)];
            }
            a2[bitrev(j, log2m)] = make_double2(v[0], v[1]);
        }
        __syncthreads();
        fft_smem(a2, M, log2m, W);
        const double sc = 2.0 / (double)(n + 1);
        for (int h = 0; h < 2; ++h) {
            const int i = r0 + h;
            if (i > ni) break;
            for (int j = threadIdx.x; j < nh; j += blockDim.x) {
                double pp;
                if (j == 0) pp = psib[2 * nh + (i - 1)];
                else if (j == nh - 1) pp = psib[2 * nh + (nw - 2) + (i - 1)];
                else {
                    const double2 z = a2[j];
                    pp = sc * (h == 0 ? -0.5 * z.y : 0.5 * z.x);
                }
                emit((long long)i * nh + j, pp);
            }
        }
    } else {
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
    __syncthreads();
    if (threadIdx.x == 0) {
        double m = 0.0;
        for (int q = 0; q < (int)(blockDim.x >> 5); ++q) m = fmax(m, wmax[q]);
        eps_part[blockIdx.x] = m;
        __threadfence();
        last = (atomicAdd(ticket, 1u) == gridDim.x - 1);
    }
    __syncthreads();
    if (!last) return;
    __threadfence();
    double m = 0.0;
    for (int b = threadIdx.x; b < (int)gridDim.x; b += blockDim.x) m = fmax(m, __ldcg(eps_part + b));
    m = warp_max(m);
    if (l == 0) wmax[w] = m;
    __syncthreads();
    if (threadIdx.x == 0) {
        double mm = 0.0;
        for (int q = 0; q < (int)(blockDim.x >> 5); ++q) mm = fmax(mm, wmax[q]);
        *eps = mm / fabs(axbd[1] - axbd[0]);
        *ticket = 0u;
    }
}

cudaError_t launch_solve(Ctx& c, const double* pcurr, const double* psib, double* psi_out, double* psi_inout,
                         const double* psi_ext, double* eps, cudaStream_t s) {
    const int npairs = (c.ni + 1) / 2;
    const size_t smem = sizeof(double2) * c.fft_m;
    k_dst_fwd<<<npairs, 256, smem, s>>>(pcurr, psib, c.tri_a, c.nw, c.nh, c.rmin, c.dr, c.dz, c.twiddle, c.fft_m,
                                        c.fft_log2, c.fhat);
    cudaError_t e = cudaGetLastError();
    if (e) return e;
    k_tridiag<<<(c.nmode + 63) / 64, 64, 0, s>>>(c.fhat, c.tri_a, c.tri_cp, c.tri_inv, c.ni, c.nmode);
    e = cudaGetLastError();
    if (e) return e;
    k_dst_inv<<<npairs + 1, 256, smem, s>>>(c.fhat, psib, c.nw, c.nh, c.twiddle, c.fft_m, c.fft_log2, psi_out,
                                            psi_inout, psi_ext, c.eps_part, c.tickets + 1, c.axbd, eps);
    return cudaGetLastError();
}

// (I[g], I[ii][nh-1-m]) pairs for a caller-supplied current (efit_boundary_flux).
__global__ void k_make_pair(const double* __restrict__ I, double2* __restrict__ ip, int nw, int nh) {
    const int n = nw * nh;
    for (int g = blockIdx.x * blockDim.x + threadIdx.x; g < n; g += gridDim.x * blockDim.x) {
        const int ii = g / nh, m = g - (g / nh) * nh;
        ip[g] = make_double2(I[g], I[ii * nh + (nh - 1 - m)]);
    }
}

cudaError_t launch_make_pair(Ctx& c, const double* pcurr, cudaStream_t s) {
    const int n = c.nw * c.nh;
    k_make_pair<<<(n + 255) / 256, 256, 0, s>>>(pcurr, c.ipair, c.nw, c.nh);
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
    if ((e = big((const void*)k_lsq, lsq_smem(c)))) return e;
    if ((e = big((const void*)k_bnd_lr<kLrJT>, sizeof(double) * 2 * (size_t)c.t.lr_iib * c.nh))) return e;
    if ((e = big((const void*)k_bnd_tb<kTbGI>, sizeof(double2) * c.t.tb_ch))) return e;
    if ((e = big((const void*)k_bnd_tb_otf<kTbGI>, sizeof(double2) * c.t.tb_ch))) return e;
    if ((e = big((const void*)k_dst_fwd, sizeof(double2) * c.fft_m))) return e;
    if ((e = big((const void*)k_dst_inv, sizeof(double2) * c.fft_m))) return e;
    return cudaSuccess;
}

}  // namespace efit
