// efit_steps.cu -- the full steps_ normalisation on sm_100a.
//
// steps_ computes "the dimensionless poloidal fluxes and the location of the plasma boundary"
// (P:L107); the algorithm is DESIGN.md reading R4: magnetic axis refined on the bicubic Hermite
// interpolant of psi (central-difference nodal derivatives, index units) by Newton's method,
// X-points found the same way from saddle candidates, the boundary = the first of {limiter contact
// between the X-point heights, lower X-point, upper X-point} met going out from the axis, and the
// plasma mask = the 4-connected component of the axis node in {in-limiter, 0 <= psihat < 1}.
//
// This translation unit is compiled with -fmad=false: every floating-point expression below is a
// sequence of plain IEEE fp64 operations in the written order (that of the reading), so every
// discrete decision (candidate test, Newton acceptance, boundary choice, mask bit) is reproducible
// bit for bit.  Five launches per normalisation (each programmatically behind its predecessor):
//   k_steps_scan   all CTAs: in-limiter argmax partials of s psi + X-point candidate list
//   k_steps_final  one CTA: axis / X-point Newton searches (one warp each), limiter value, boundary
//   k_steps_bits   candidate bitmap {inlim, 0 <= psihat < 1}, 64-bit words (two ballots per warp)
//   k_steps_fill   one CTA: bit-parallel flood fill from the axis node in shared memory (row runs by
//                  carry propagation, column runs by a segmented warp scan, dirty rows / columns only)
//   k_steps_mask   the component as the byte mask read by the basis / response / current kernels
#include <cuda_runtime.h>
#include <float.h>
#include <limits.h>
#include <stdint.h>

#include <cstdio>
#include <utility>

#include "efit_internal.h"

namespace efit {

namespace {

constexpr int kNewtonIters = 20;
constexpr int kMaxXCand = 8;
constexpr int kFillThreads = 1024;

__device__ __forceinline__ void am_merge(double& v, long long& i, double v2, long long i2) {
    if (v2 > v || (v2 == v && i2 < i)) { v = v2; i = i2; }
}

__device__ __forceinline__ void am_warp(double& v, long long& i) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const double v2 = __shfl_xor_sync(0xffffffffu, v, o);
        const long long i2 = __shfl_xor_sync(0xffffffffu, i, o);
        am_merge(v, i, v2, i2);
    }
}

struct Field {
    const double* psi;
    int nw, nh;
    __device__ __forceinline__ double at(int i, int j) const { return __ldg(psi + (long long)i * nh + j); }
};

// Hermite basis on [0, 1]: values at 0 / 1, slopes at 0 / 1, and their first and second derivatives
__device__ __forceinline__ void herm_basis(double t, double h[4], double d[4], double e[4]) {
    const double t2 = t * t;
    h[0] = (2.0 * t - 3.0) * t2 + 1.0;
    h[1] = (3.0 - 2.0 * t) * t2;
    h[2] = ((t - 2.0) * t + 1.0) * t;
    h[3] = (t - 1.0) * t2;
    d[0] = (6.0 * t) * (t - 1.0);
    d[1] = -d[0];
    d[2] = (3.0 * t - 4.0) * t + 1.0;
    d[3] = (3.0 * t - 2.0) * t;
    e[0] = 12.0 * t - 6.0;
    e[1] = -e[0];
    e[2] = 6.0 * t - 4.0;
    e[3] = 6.0 * t - 2.0;
}

// sum_a A[a] (sum_b Q[a][b] B[b]), both sums left to right
__device__ __forceinline__ double herm_form(const double Q[4][4], const double* A, const double* B) {
    double v[4];
#pragma unroll
    for (int a = 0; a < 4; ++a) v[a] = ((Q[a][0] * B[0] + Q[a][1] * B[1]) + Q[a][2] * B[2]) + Q[a][3] * B[3];
    return ((A[0] * v[0] + A[1] * v[1]) + A[2] * v[2]) + A[3] * v[3];
}

// p, pt, pu, ptt, puu, ptu of the interpolant at index coordinates (xt, xu); cell clamped to
// 1 <= ci <= nw-3, 1 <= cj <= nh-3 (both corners interior: central differences defined)
__device__ void herm_eval(const Field& F, double xt, double xu, double out[6]) {
    int ci = (int)floor(xt), cj = (int)floor(xu);
    ci = ci < 1 ? 1 : (ci > F.nw - 3 ? F.nw - 3 : ci);
    cj = cj < 1 ? 1 : (cj > F.nh - 3 ? F.nh - 3 : cj);
    const double t = xt - (double)ci, u = xu - (double)cj;
    double Q[4][4];
#pragma unroll
    for (int a = 0; a < 2; ++a) {
        const int i = ci + a;
#pragma unroll
        for (int b = 0; b < 2; ++b) {
            const int j = cj + b;
            Q[a][b] = F.at(i, j);
            Q[a][2 + b] = 0.5 * (F.at(i, j + 1) - F.at(i, j - 1));
            Q[2 + a][b] = 0.5 * (F.at(i + 1, j) - F.at(i - 1, j));
            Q[2 + a][2 + b] = 0.25 * (((F.at(i + 1, j + 1) - F.at(i + 1, j - 1)) - F.at(i - 1, j + 1)) + F.at(i - 1, j - 1));
        }
    }
    double ht[4], dt[4], et[4], hu[4], du[4], eu[4];
    herm_basis(t, ht, dt, et);
    herm_basis(u, hu, du, eu);
    out[0] = herm_form(Q, ht, hu);
    out[1] = herm_form(Q, dt, hu);
    out[2] = herm_form(Q, ht, du);
    out[3] = herm_form(Q, et, hu);
    out[4] = herm_form(Q, ht, eu);
    out[5] = herm_form(Q, dt, du);
}

// Newton's method for grad p = 0 from (xt, xu): <= 20 steps, step components clamped to [-1/2, 1/2],
// converged when both are below 1e-10.  out = xt, xu, p, det, ptt at the final point.
__device__ bool newton_stationary(const Field& F, double xt, double xu, double out[5]) {
    double d[6];
    bool conv = false;
    for (int it = 0; it < kNewtonIters; ++it) {
        herm_eval(F, xt, xu, d);
        const double det = d[3] * d[4] - d[5] * d[5];
        if (!(det != 0.0)) break;
        double st = (d[4] * d[1] - d[5] * d[2]) / det;
        double su = (d[3] * d[2] - d[5] * d[1]) / det;
        if (!(fabs(st) < 1e300) || !(fabs(su) < 1e300)) break;
        st = st > 0.5 ? 0.5 : st;
        st = st < -0.5 ? -0.5 : st;
        su = su > 0.5 ? 0.5 : su;
        su = su < -0.5 ? -0.5 : su;
        xt = xt - st;
        xu = xu - su;
        if (fabs(st) < 1e-10 && fabs(su) < 1e-10) { conv = true; break; }
    }
    herm_eval(F, xt, xu, d);
    out[0] = xt; out[1] = xu; out[2] = d[0]; out[3] = d[3] * d[4] - d[5] * d[5]; out[4] = d[3];
    return conv;
}

__device__ __forceinline__ double grad2(const Field& F, int i, int j) {
    const double gt = 0.5 * (F.at(i + 1, j) - F.at(i - 1, j));
    const double gu = 0.5 * (F.at(i, j + 1) - F.at(i, j - 1));
    return gt * gt + gu * gu;
}

// X-point candidate test of node (i, j), 2 <= i <= nw-3, 2 <= j <= nh-3, in the limiter: indefinite
// discrete Hessian and |grad|^2 a local minimum over the 8 neighbours (strict against lower node
// indices, <= against higher ones)
__device__ bool xcand(const Field& F, int i, int j, double& key) {
    const double p0 = F.at(i, j);
    const double dtt = (F.at(i + 1, j) - 2.0 * p0) + F.at(i - 1, j);
    const double duu = (F.at(i, j + 1) - 2.0 * p0) + F.at(i, j - 1);
    const double dtu = 0.25 * (((F.at(i + 1, j + 1) - F.at(i + 1, j - 1)) - F.at(i - 1, j + 1)) + F.at(i - 1, j - 1));
    if (!(dtt * duu - dtu * dtu < 0.0)) return false;
    const double g2 = grad2(F, i, j);
    for (int di = -1; di <= 1; ++di)
        for (int dj = -1; dj <= 1; ++dj) {
            if (!di && !dj) continue;
            const double v = grad2(F, i + di, j + dj);
            const bool lower = (di < 0) || (di == 0 && dj < 0);  // neighbour has the lower node index
            if (lower ? !(g2 < v) : !(g2 <= v)) return false;
        }
    key = g2;
    return true;
}

// O8's bilinear value at (R, Z)
__device__ double bilin(const Field& F, double rmin, double dr, double zmin, double dz, double R, double Z) {
    const double x = (R - rmin) / dr, y = (Z - zmin) / dz;
    int i = (int)floor(x), j = (int)floor(y);
    i = i < 0 ? 0 : (i > F.nw - 2 ? F.nw - 2 : i);
    j = j < 0 ? 0 : (j > F.nh - 2 ? F.nh - 2 : j);
    const double t = x - (double)i, u = y - (double)j;
    const double w00 = (1.0 - t) * (1.0 - u), w10 = t * (1.0 - u), w01 = (1.0 - t) * u, w11 = t * u;
    return ((w00 * F.at(i, j) + w10 * F.at(i + 1, j)) + w01 * F.at(i, j + 1)) + w11 * F.at(i + 1, j + 1);
}

struct StepsArgs {
    const double* psi;
    const uint8_t* inlim;
    int nw, nh, sgn;
    double rmin, dr, zmin, dz;
    const double* lim;
    int n_lim;
    double* part;        // [red_blocks][2] (s psi, g) argmax partials of k_steps_scan
    int nparts;
    double2* cand;       // [cap] X-point candidates (|grad|^2, g)
    unsigned* cnt;       // [0] candidates found, [1] axis node g0 (UINT_MAX: no plasma), [2] non-finite psi seen
    int cap;
    double* info;        // [16] (efit.h efit_normalize layout)
    double* axbd;        // [2]
    int* status;
};

// All CTAs: per-block in-limiter argmax of s psi (ties: lowest g), X-point candidates appended to a
// list (at most one per 2 x 2 node block: two 8-neighbours cannot both be local minima under the
// strict/non-strict tie rule, so the list never overflows its ceil(nw/2) ceil(nh/2) slots).
__global__ void __launch_bounds__(256) k_steps_scan(StepsArgs a) {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    __shared__ double sv[8];
    __shared__ long long si[8];
    const Field F{a.psi, a.nw, a.nh};
    const int n = a.nw * a.nh, nh = a.nh;
    const double s = (double)a.sgn;
    double best = -DBL_MAX;
    long long bi = LLONG_MAX;
    bool bad = false;
    for (int g = blockIdx.x * blockDim.x + threadIdx.x; g < n; g += gridDim.x * blockDim.x) {
        const double p = __ldg(a.psi + g);
        if (!isfinite(p)) bad = true;
        if (__ldg(a.inlim + g)) {
            am_merge(best, bi, s * p, (long long)g);
            const int i = g / nh, j = g - (g / nh) * nh;
            double key;
            if (i >= 2 && i <= a.nw - 3 && j >= 2 && j <= nh - 3 && xcand(F, i, j, key)) {
                const unsigned k = atomicAdd(a.cnt, 1u);
                if (k < (unsigned)a.cap) a.cand[k] = make_double2(key, (double)g);
            }
        }
    }
    if (__syncthreads_or(bad) && threadIdx.x == 0) {
        atomicOr(a.status, EFIT_ST_NONFINITE);
        atomicOr(a.cnt + 2, 1u);
    }
    am_warp(best, bi);
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
    if (l == 0) { sv[w] = best; si[w] = bi; }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int q = 1; q < 8; ++q) am_merge(best, bi, sv[q], si[q]);
        a.part[2 * blockIdx.x] = best;
        a.part[2 * blockIdx.x + 1] = (double)bi;
    }
}

constexpr int kFinalWarps = kMaxXCand + 1;  // warp 0: the axis, warps 1..8: X-point candidates
constexpr int kFinalLimStage = 1024;         // limiter vertices staged in shared memory (24 KB)

// One CTA: (3) axis, (4) X-points, (5) limiter value, (6) boundary.  Newton searches run one per
// warp (lane 0) concurrently; the in-limiter test of an X-point is the parity of the crossings over
// the limiter edges (an order-independent count: the same decision as the sequential even-odd rule).
__global__ void __launch_bounds__(32 * kFinalWarps) k_steps_final(StepsArgs a) {
    // limiter vertices (constant: staged before the wait on the predecessor) and, right after it,
    // s psi_bilin at every vertex, so that the X-point in-limiter tests and the limiter value after
    // the Newton searches read shared memory only
    extern __shared__ double lsm[];  // [2 n_lim] vertices (r then z), [n_lim] s psi_bilin
    const bool lstage = a.n_lim <= kFinalLimStage;
    double* vval = lsm + 2 * kFinalLimStage;
    if (lstage)
        for (int k = threadIdx.x; k < 2 * a.n_lim; k += blockDim.x) lsm[k] = __ldg(a.lim + k);
    const double* lim = lstage ? lsm : a.lim;
    asm volatile("griddepcontrol.wait;" ::: "memory");
    __shared__ double sv[kFinalWarps];
    __shared__ long long si[kFinalWarps];
    __shared__ long long selg[kMaxXCand];
    __shared__ double res[kFinalWarps][4];  // xt, xu, p, det (after Newton)
    __shared__ int racc[kFinalWarps];        // converged (+ saddle, near, inside for candidates)
    __shared__ double zlim[2];
    __shared__ int nsel_s;
    const Field F{a.psi, a.nw, a.nh};
    const int nh = a.nh, tid = threadIdx.x, w = tid >> 5, l = tid & 31;
    const double s = (double)a.sgn;
    __syncthreads();  // staged vertices visible
    if (lstage)
        for (int v = tid; v < a.n_lim; v += blockDim.x)
            vval[v] = s * bilin(F, a.rmin, a.dr, a.zmin, a.dz, lim[v], lim[a.n_lim + v]);
    double best = -DBL_MAX;
    long long bi = LLONG_MAX;
    for (int b = tid; b < a.nparts; b += blockDim.x) am_merge(best, bi, a.part[2 * b], (long long)a.part[2 * b + 1]);
    am_warp(best, bi);
    if (l == 0) { sv[w] = best; si[w] = bi; }
    if (tid == 0) nsel_s = 0;
    __syncthreads();
    if (tid == 0) {
        for (int q = 1; q < kFinalWarps; ++q) am_merge(best, bi, sv[q], si[q]);
        si[0] = bi;
    }
    const unsigned ncand_all = a.cnt[0];
    const int ncand = (int)(ncand_all < (unsigned)a.cap ? ncand_all : (unsigned)a.cap);
    for (int q = tid; q < ncand; q += blockDim.x) {  // the 8 smallest (|grad|^2, g): ranks in that order
        const double2 cq = a.cand[q];
        int rank = 0;
        for (int r = 0; r < ncand && rank < kMaxXCand; ++r) {
            const double2 cr = a.cand[r];
            if (cr.x < cq.x || (cr.x == cq.x && cr.y < cq.y)) ++rank;
        }
        if (rank < kMaxXCand) { selg[rank] = (long long)cq.y; atomicMax(&nsel_s, rank + 1); }
    }
    __syncthreads();
    const long long g0 = si[0];
    const int nsel = nsel_s;
    const bool ok0 = (g0 != LLONG_MAX) && a.cnt[2] == 0u;
    if (ok0 && w <= nsel) {
        const long long gs = w == 0 ? g0 : selg[w - 1];
        const int i = (int)(gs / nh), j = (int)(gs - (gs / nh) * nh);
        int acc = 0;
        double o[5] = {0.0, 0.0, 0.0, 0.0, 0.0};
        if (l == 0) {
            if (w > 0 || (a.nw >= 4 && nh >= 4 && i >= 1 && i <= a.nw - 2 && j >= 1 && j <= nh - 2)) {
                const bool conv = newton_stationary(F, (double)i, (double)j, o);
                if (w == 0)
                    acc = conv ? 1 : 0;
                else
                    acc = (conv && o[3] < 0.0 && fabs(o[0] - (double)i) <= 1.5 && fabs(o[1] - (double)j) <= 1.5) ? 1 : 0;
            }
        }
        acc = __shfl_sync(0xffffffffu, acc, 0);
        if (w > 0 && acc) {  // inside the limiter: parity of the edge crossings (O7 rule), lanes over edges
            const double Rx = __shfl_sync(0xffffffffu, a.rmin + o[0] * a.dr, 0);
            const double Zx = __shfl_sync(0xffffffffu, a.zmin + o[1] * a.dz, 0);
            unsigned par = 0u;
            for (int k = l; k < a.n_lim; k += 32) {
                const int k1 = (k + 1 == a.n_lim) ? 0 : k + 1;
                const double r0 = lim[k], z0 = lim[a.n_lim + k], r1 = lim[k1], z1 = lim[a.n_lim + k1];
                if ((z0 > Zx) != (z1 > Zx)) {
                    const double x = ((r1 - r0) * (Zx - z0)) / (z1 - z0) + r0;
                    if (Rx < x) par ^= 1u;
                }
            }
            acc = (__popc(__ballot_sync(0xffffffffu, par != 0u)) & 1) ? 1 : 0;
        }
        if (l == 0) {
            racc[w] = acc;
            res[w][0] = o[0]; res[w][1] = o[1]; res[w][2] = o[2]; res[w][3] = o[3];
            if (w == 0) res[0][3] = o[3] > 0.0 && a.sgn * o[4] < 0.0 ? 1.0 : 0.0;  // maximum of s psi
        }
    }
    __syncthreads();
    if (tid == 0) {
        double* info = a.info;
        for (int k = 0; k < 16; ++k) info[k] = __longlong_as_double(0x7ff8000000000000LL);  // NaN
        double pa = 0.0;
        bool lo = false, hi = false;
        double xlo[3], xhi[3];
        if (ok0) {
            const int i0 = (int)(g0 / nh), j0 = (int)(g0 - (g0 / nh) * nh);
            const double p0 = F.at(i0, j0);
            pa = p0;
            double xa = (double)i0, ya = (double)j0;
            int ref = 0;
            if (racc[0] && res[0][3] == 1.0 && fabs(res[0][0] - (double)i0) <= 1.0 &&
                fabs(res[0][1] - (double)j0) <= 1.0 && s * res[0][2] >= s * p0) {
                pa = res[0][2]; xa = res[0][0]; ya = res[0][1]; ref = 1;
            }
            const double Za = a.zmin + ya * a.dz;
            info[0] = pa; info[2] = a.rmin + xa * a.dr; info[3] = Za; info[4] = (double)ref; info[15] = (double)g0;
            info[14] = (double)nsel;
            for (int q = 0; q < nsel; ++q) {  // candidate order (ties: the earlier one)
                if (!racc[q + 1]) continue;
                const double px = res[q + 1][2];
                if (!(s * (pa - px) > 0.0)) continue;
                const double Rx = a.rmin + res[q + 1][0] * a.dr, Zx = a.zmin + res[q + 1][1] * a.dz;
                if (Zx < Za) {
                    if (!lo || s * px > s * xlo[2]) { lo = true; xlo[0] = Rx; xlo[1] = Zx; xlo[2] = px; }
                } else if (Zx > Za) {
                    if (!hi || s * px > s * xhi[2]) { hi = true; xhi[0] = Rx; xhi[1] = Zx; xhi[2] = px; }
                }
            }
            if (lo) { info[6] = xlo[0]; info[7] = xlo[1]; info[8] = xlo[2]; }
            if (hi) { info[9] = xhi[0]; info[10] = xhi[1]; info[11] = xhi[2]; }
        }
        zlim[0] = lo ? xlo[1] : -DBL_MAX;
        zlim[1] = hi ? xhi[1] : DBL_MAX;
        res[0][2] = pa;
        racc[0] = ok0 ? 1 : 0;
    }
    __syncthreads();
    // (5) limiter value between the X-point heights (ties: lowest vertex)
    double vb = -DBL_MAX;
    long long vi = LLONG_MAX;
    if (racc[0]) {
        const bool lo = zlim[0] != -DBL_MAX, hi = zlim[1] != DBL_MAX;
        for (int v = tid; v < a.n_lim; v += blockDim.x) {
            const double z = lim[a.n_lim + v];
            if (lo && !(z > zlim[0])) continue;
            if (hi && !(z < zlim[1])) continue;
            am_merge(vb, vi, lstage ? vval[v] : s * bilin(F, a.rmin, a.dr, a.zmin, a.dz, lim[v], z), (long long)v);
        }
    }
    am_warp(vb, vi);
    __syncthreads();
    if (l == 0) { sv[w] = vb; si[w] = vi; }
    __syncthreads();
    if (tid == 0) {
        for (int q = 1; q < kFinalWarps; ++q) am_merge(vb, vi, sv[q], si[q]);
        double* info = a.info;
        const double pa = res[0][2];
        // (6) boundary: the largest in s of {limiter, lower X, upper X}, ties in that order
        int kind = -1;
        double pb = 0.0;
        if (racc[0]) {
            if (vi != LLONG_MAX) { kind = 0; pb = s * vb; info[5] = pb; }
            const double plo = info[8], phi = info[11];
            if (plo == plo && (kind < 0 || s * plo > s * pb)) { kind = 1; pb = plo; }
            if (phi == phi && (kind < 0 || s * phi > s * pb)) { kind = 2; pb = phi; }
        }
        info[1] = pb;
        info[12] = (double)kind;
        a.axbd[0] = pa;
        a.axbd[1] = pb;
        const bool plasma = kind >= 0 && s * (pa - pb) > 0.0;
        if (!plasma) atomicOr(a.status, EFIT_ST_NOPLASMA);
        a.cnt[1] = plasma ? (unsigned)g0 : UINT_MAX;
        a.cnt[0] = 0u;  // candidate counter and non-finite flag ready for the next scan
        a.cnt[2] = 0u;
    }
}

// bits[i][k] bit b = node (i, 64k + b) is in the limiter with 0 <= psihat < 1 (one warp per word)
__global__ void __launch_bounds__(256) k_steps_bits(const double* __restrict__ psi, const uint8_t* __restrict__ inlim,
                                                   int nw, int nh, int W, const double* __restrict__ axbd,
                                                   unsigned long long* __restrict__ bits) {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    const long long word = (long long)blockIdx.x * 8 + (threadIdx.x >> 5);
    if (word >= (long long)nw * W) return;
    const int i = (int)(word / W), k = (int)(word - (word / W) * W);
    const double pa = axbd[0], pb = axbd[1];
    uint32_t half[2];
#pragma unroll
    for (int hh = 0; hh < 2; ++hh) {
        const int j = 64 * k + 32 * hh + (threadIdx.x & 31);
        bool in = false;
        if (j < nh) {
            const long long g = (long long)i * nh + j;
            if (__ldg(inlim + g)) {
                const double h = (__ldg(psi + g) - pa) / (pb - pa);
                in = h >= 0.0 && h < 1.0;
            }
        }
        half[hh] = __ballot_sync(0xffffffffu, in);
    }
    if ((threadIdx.x & 31) == 0) bits[word] = (unsigned long long)half[0] | ((unsigned long long)half[1] << 32);
}

// run fill upwards in bit index within a 64-bit word: every bit of c connected through a run of c's
// bits to a seed bit of x (x subset of c); carry = the fill ran out through bit 63
__device__ __forceinline__ unsigned long long fill_up64(unsigned long long c, unsigned long long x, bool& carry) {
    const unsigned long long sum = c + x;
    carry = sum < c;
    return ((sum ^ c) & c) | x;
}

// One CTA: bit-parallel flood fill from the axis node in shared memory.  Rounds of (a) runs along Z
// within each row (one thread per row, carries from word to word) and (b) runs along R within each
// bit column, down then up (one warp per 64-bit column word; 32 row segments: a sequential pass
// inside each segment, the segment transfers (G, P) composed by a warp scan, a second pass with the
// carry-in).  Only rows changed since their last (a) and word columns changed since their last (b)
// are processed (both passes are idempotent on unchanged data); the fill ends when nothing is dirty.
// The component is written back over the candidate bitmap (bits_g) with its size.
template <bool CSMEM>
__global__ void __launch_bounds__(kFillThreads, 1) k_steps_fill(unsigned long long* __restrict__ bits_g, int nw,
                                                               int nh, int W, const unsigned* __restrict__ cnt,
                                                               double* __restrict__ info, int* status) {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    extern __shared__ unsigned long long sm[];
    unsigned long long* R = sm;                                  // [nw][W] reached
    unsigned long long* Cs = sm + (size_t)nw * W;                // [nw][W] candidates (CSMEM)
    unsigned* rdirty = reinterpret_cast<unsigned*>(sm + (CSMEM ? 2 : 1) * (size_t)nw * W);  // [ceil(nw/32)] row bits
    __shared__ unsigned cdirty;  // word-column bits (W <= 32)
    __shared__ unsigned long long wtot[kFillThreads / 32][2];  // per-warp segment-scan totals (G, P)
    __shared__ int cnt_s[32];
    const unsigned long long* C = CSMEM ? Cs : bits_g;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    constexpr int nwarp = kFillThreads / 32;
    const int nwords = nw * W;
    const unsigned g0 = cnt[1];
    for (int q = tid; q < nwords; q += kFillThreads) {
        R[q] = 0ull;
        if (CSMEM) Cs[q] = bits_g[q];
    }
    for (int i = tid; i < (nw + 31) / 32; i += kFillThreads) rdirty[i] = 0u;
    if (tid == 0) cdirty = 0u;
    __syncthreads();
    if (tid == 0 && g0 != UINT_MAX) {
        const int i0 = (int)(g0 / (unsigned)nh), j0 = (int)(g0 - (g0 / (unsigned)nh) * (unsigned)nh);
        const int q = i0 * W + (j0 >> 6);
        R[q] = C[q] & (1ull << (j0 & 63));
        rdirty[i0 >> 5] = 1u << (i0 & 31);
        cdirty = 1u << (j0 >> 6);
    }
    __syncthreads();
#ifdef EFIT_STEPS_DEBUG
    long long t_dbg0 = clock64(), t_dbg[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    int rounds_dbg = 0;
#endif
#ifdef EFIT_STEPS_DEBUG
    long long t_init = clock64() - t_dbg0, t_h[8] = {0, 0, 0, 0, 0, 0, 0, 0};
#endif
    const int WPC = min(4, max(1, nwarp / W));  // warps per column word
    const int L = (nw + 32 * WPC - 1) / (32 * WPC);  // rows per segment
    for (;;) {
        bool work = false;
        unsigned cmask = 0u;  // word columns this thread changed (one warp-aggregated atomic per pass)
        for (int i = tid; i < nw; i += kFillThreads) {  // (a) rows along Z
            if (!((rdirty[i >> 5] >> (i & 31)) & 1u)) continue;
            work = true;
            unsigned long long* r = R + (size_t)i * W;
            const unsigned long long* cr = C + (size_t)i * W;
            bool carry = false;
            for (int k = 0; k < W; ++k) {
                const unsigned long long c = cr[k], old = r[k];
                const unsigned long long x = old | (carry ? (c & 1ull) : 0ull);
                const unsigned long long f = fill_up64(c, x, carry);
                if (f != old) { r[k] = f; cmask |= 1u << k; }
            }
            carry = false;
            for (int k = W - 1; k >= 0; --k) {
                const unsigned long long c = __brevll(cr[k]), old = r[k];
                const unsigned long long x = __brevll(old) | (carry ? (c & 1ull) : 0ull);
                const unsigned long long f = __brevll(fill_up64(c, x, carry));
                if (f != old) { r[k] = f; cmask |= 1u << k; }
            }
        }
        cmask = __reduce_or_sync(0xffffffffu, cmask);
        if (lane == 0 && cmask) atomicOr(&cdirty, cmask);
        __syncthreads();
        const unsigned cd = cdirty;
#ifdef EFIT_STEPS_DEBUG
        if (rounds_dbg < 8) t_h[rounds_dbg] = clock64() - t_dbg0;
#endif
        __syncthreads();
        if (tid == 0) cdirty = 0u;  // every dirty row had its pass: clear (the column passes set new ones)
        for (int i = tid; i < (nw + 31) / 32; i += kFillThreads) rdirty[i] = 0u;
        __syncthreads();
        // (b) word columns along R: WPC warps per column word, lane = one of 32 WPC row segments; the
        // segment transfers are composed by a warp scan, the warps' totals through shared memory
        for (int dir = 0; dir < 2; ++dir) {
            const bool act = warp < W * WPC && ((cd >> (warp / WPC)) & 1u);
            const int k = warp / WPC, part = warp - (warp / WPC) * WPC;
            const int seg = part * 32 + lane;
            const int i0 = min(nw, seg * L), i1 = min(nw, i0 + L);
            unsigned long long gv = 0ull, pv = ~0ull;
            if (act) {
                work = true;
                for (int q = 0; q < i1 - i0; ++q) {
                    const int i = dir == 0 ? i0 + q : i1 - 1 - q;
                    const unsigned long long c = C[(size_t)i * W + k];
                    gv = R[(size_t)i * W + k] | (c & gv);
                    pv &= c;
                }
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {  // inclusive composition in scan order
                    const unsigned long long go = dir == 0 ? __shfl_up_sync(0xffffffffu, gv, d) : __shfl_down_sync(0xffffffffu, gv, d);
                    const unsigned long long po = dir == 0 ? __shfl_up_sync(0xffffffffu, pv, d) : __shfl_down_sync(0xffffffffu, pv, d);
                    if (dir == 0 ? lane >= d : lane + d < 32) { gv |= pv & go; pv &= po; }
                }
                if (lane == (dir == 0 ? 31 : 0)) { wtot[warp][0] = gv; wtot[warp][1] = pv; }
            }
            __syncthreads();
            if (act) {
                unsigned long long cin = 0ull;  // carry into this warp: the totals of the warps before it
                if (dir == 0) {
                    for (int p2 = 0; p2 < part; ++p2) cin = wtot[k * WPC + p2][0] | (wtot[k * WPC + p2][1] & cin);
                } else {
                    for (int p2 = WPC - 1; p2 > part; --p2) cin = wtot[k * WPC + p2][0] | (wtot[k * WPC + p2][1] & cin);
                }
                // exclusive prefix of this lane = the previous lane's inclusive value applied to cin
                unsigned long long ge = dir == 0 ? __shfl_up_sync(0xffffffffu, gv, 1) : __shfl_down_sync(0xffffffffu, gv, 1);
                unsigned long long pe = dir == 0 ? __shfl_up_sync(0xffffffffu, pv, 1) : __shfl_down_sync(0xffffffffu, pv, 1);
                if (lane == (dir == 0 ? 0 : 31)) { ge = 0ull; pe = ~0ull; }
                unsigned long long prev = ge | (pe & cin);
                unsigned long long rmask = 0ull;  // rows i0 + q changed (L <= 64), set with <= 3 atomics
                for (int q = 0; q < i1 - i0; ++q) {
                    const int i = dir == 0 ? i0 + q : i1 - 1 - q;
                    const size_t p = (size_t)i * W + k;
                    const unsigned long long old = R[p];
                    const unsigned long long v = old | (C[p] & prev);
                    if (v != old) { R[p] = v; rmask |= 1ull << (i - i0); }
                    prev = v;
                }
                while (rmask) {  // the changed rows' dirty bits, one atomic per 32-row word touched
                    const int b = __ffsll((long long)rmask) - 1, i = i0 + b, w0 = i >> 5;
                    const int nb = min(32 - (i & 31), 64 - b);
                    const unsigned long long chunk = (nb == 64 ? ~0ull : ((1ull << nb) - 1ull)) & (rmask >> b);
                    atomicOr(&rdirty[w0], (unsigned)(chunk << (i & 31)));
                    rmask &= ~(nb == 64 ? ~0ull : (((1ull << nb) - 1ull) << b));
                }
            }
            __syncthreads();
        }
#ifdef EFIT_STEPS_DEBUG
        if (rounds_dbg < 8) t_dbg[rounds_dbg] = clock64() - t_dbg0;
        ++rounds_dbg;
#endif
        if (!__syncthreads_or(work)) break;
    }
    int c = 0;
    for (int q = tid; q < nwords; q += kFillThreads) {
        bits_g[q] = R[q];
        c += __popcll(R[q]);
    }
    c = __reduce_add_sync(0xffffffffu, c);
    if (lane == 0) cnt_s[warp] = c;
    __syncthreads();
    if (tid == 0) {
        int t = 0;
        for (int q = 0; q < nwarp; ++q) t += cnt_s[q];
        if (g0 != UINT_MAX) info[13] = (double)t;  // no boundary / no plasma: left NaN (as the oracle)
#ifdef EFIT_STEPS_DEBUG
        printf("fill rounds=%d end t=%lld count=%d rounds at %lld %lld %lld %lld %lld\n", rounds_dbg, clock64() - t_dbg0, t,
               t_dbg[0], t_dbg[1], t_dbg[2], t_dbg[3], t_dbg[4]);
        printf("  init %lld, after H: %lld %lld %lld %lld\n", t_init, t_h[0], t_h[1], t_h[2], t_h[3]);
#endif
        if (t == 0) atomicOr(status, EFIT_ST_NOPLASMA);
    }
}

// byte mask from the component bitmap, 16 nodes per thread (one 16-byte store; pmask 256-B aligned)
__global__ void __launch_bounds__(256) k_steps_mask(const unsigned long long* __restrict__ bits, int nw, int nh, int W,
                                                   uint8_t* __restrict__ mask) {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    const unsigned n = (unsigned)nw * (unsigned)nh;
    const unsigned t = blockIdx.x * blockDim.x + threadIdx.x;
    const unsigned g0 = 16u * t;
    if (g0 >= n) return;
    int i = (int)(g0 / (unsigned)nh), j = (int)(g0 - (unsigned)i * (unsigned)nh);
    uint32_t v[4] = {0u, 0u, 0u, 0u};
#pragma unroll
    for (int b = 0; b < 16; ++b) {
        if (g0 + b < n) v[b >> 2] |= (uint32_t)((bits[i * W + (j >> 6)] >> (j & 63)) & 1ull) << (8 * (b & 3));
        if (++j == nh) { j = 0; ++i; }
    }
    if (g0 + 16u <= n) {
        *reinterpret_cast<uint4*>(mask + g0) = make_uint4(v[0], v[1], v[2], v[3]);
    } else {
#pragma unroll
        for (int b = 0; b < 16; ++b)
            if (g0 + b < n) mask[g0 + b] = (uint8_t)(v[b >> 2] >> (8 * (b & 3)));
    }
}

template <typename... KArgs, typename... Args>
cudaError_t launch_pdl_s(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, Args&&... args) {
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

}  // namespace

int steps_words(int nh) { return (nh + 63) / 64; }  // 64-bit words per bitmap row
int steps_cand_cap(int nw, int nh) { return ((nw + 1) / 2) * ((nh + 1) / 2); }

// dynamic shared memory of k_steps_fill; the candidate bitmap is staged too when both maps fit
size_t steps_fill_smem(int nw, int nh, bool* cand_smem) {
    const size_t one = 8 * (size_t)steps_words(nh) * nw;
    const bool both = 2 * one + 4 * (size_t)((nw + 31) / 32) <= 200 * 1024;
    if (cand_smem) *cand_smem = both;
    return (both ? 2 * one : one) + 4 * (size_t)((nw + 31) / 32);  // + the row dirty bits
}

cudaError_t prepare_steps(Ctx& c, int smem_optin) {
    bool cs;
    const size_t sm = steps_fill_smem(c.nw, c.nh, &cs);
    if ((long long)sm > smem_optin) return cudaSuccess;  // reported by efit_set_steps
    cudaError_t e = cudaFuncSetAttribute((const void*)k_steps_fill<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e) return e;
    return cudaFuncSetAttribute((const void*)k_steps_fill<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
}

// full steps_ of psi: c.axbd, c.st_info, c.pmask (the plasma mask used downstream in place of the
// limiter flags).  Five launches: scan (all CTAs) -> final (1 CTA) -> bits -> fill (1 CTA) -> mask.
cudaError_t launch_steps(Ctx& c, const double* psi, cudaStream_t s) {
    StepsArgs a;
    a.psi = psi; a.inlim = c.inlim; a.nw = c.nw; a.nh = c.nh; a.sgn = c.ip_sign;
    a.rmin = c.rmin; a.dr = c.dr; a.zmin = c.zmin; a.dz = c.dz; a.lim = c.lim; a.n_lim = c.n_lim;
    a.part = c.norm_part; a.nparts = c.t.red_blocks; a.cand = c.st_cand; a.cnt = c.st_cnt;
    a.cap = steps_cand_cap(c.nw, c.nh); a.info = c.st_info; a.axbd = c.axbd; a.status = c.status;
    unsigned long long* bits = reinterpret_cast<unsigned long long*>(c.st_bits);
    cudaError_t e = launch_pdl_s(k_steps_scan, dim3(c.t.red_blocks), dim3(256), 0, s, a);
    if (!e) e = launch_pdl_s(k_steps_final, dim3(1), dim3(32 * kFinalWarps), sizeof(double) * 3 * kFinalLimStage, s, a);
    const int W = steps_words(c.nh);
    const long long nwords = (long long)c.nw * W;
    if (!e)
        e = launch_pdl_s(k_steps_bits, dim3((unsigned)((nwords + 7) / 8)), dim3(256), 0, s, psi, (const uint8_t*)c.inlim,
                         c.nw, c.nh, W, (const double*)c.axbd, bits);
    bool cs;
    const size_t sm = steps_fill_smem(c.nw, c.nh, &cs);
    if (!e) {
        if (cs)
            e = launch_pdl_s(k_steps_fill<true>, dim3(1), dim3(kFillThreads), sm, s, bits, c.nw, c.nh, W,
                             (const unsigned*)c.st_cnt, c.st_info, c.status);
        else
            e = launch_pdl_s(k_steps_fill<false>, dim3(1), dim3(kFillThreads), sm, s, bits, c.nw, c.nh, W,
                             (const unsigned*)c.st_cnt, c.st_info, c.status);
    }
    const unsigned n16 = (unsigned)(((long long)c.nw * c.nh + 15) / 16);
    if (!e)
        e = launch_pdl_s(k_steps_mask, dim3((n16 + 255) / 256), dim3(256), 0, s, (const unsigned long long*)bits, c.nw,
                         c.nh, W, c.pmask);
    if (e) return e;
    return cudaGetLastError();
}

// O8 byte mask (limiter rule) for efit_normalize in EFIT_STEPS_LIMITER mode
__global__ void k_mask_o8(const double* __restrict__ psi, const uint8_t* __restrict__ inlim, int n,
                          const double* __restrict__ axbd, uint8_t* __restrict__ mask) {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    const double pa = __ldcg(axbd), pb = __ldcg(axbd + 1);
    for (int g = blockIdx.x * blockDim.x + threadIdx.x; g < n; g += gridDim.x * blockDim.x) {
        bool m = false;
        if (inlim[g]) {
            const double h = (__ldcg(psi + g) - pa) / (pb - pa);
            m = h >= 0.0 && h < 1.0;
        }
        mask[g] = (uint8_t)m;
    }
}

cudaError_t launch_mask_o8(Ctx& c, const double* psi, uint8_t* mask, cudaStream_t s) {
    const int n = c.nw * c.nh;
    cudaError_t e = launch_pdl_s(k_mask_o8, dim3((n + 255) / 256 < 1184 ? (n + 255) / 256 : 1184), dim3(256), 0, s, psi,
                                 (const uint8_t*)c.inlim, n, (const double*)c.axbd, mask);
    if (e) return e;
    return cudaGetLastError();
}

}  // namespace efit
