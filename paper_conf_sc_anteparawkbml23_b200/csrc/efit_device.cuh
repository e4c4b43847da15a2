// efit_device.cuh -- device-side math of the B200 EFIT path (Green's functions, grid,
// basis).  Written for sm_100a from the definitions cited below; shares nothing with the
// CPU oracle.  All fp64.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace efit {

constexpr double kPi = 3.141592653589793238462643383279502884;
constexpr double kMu0 = 4.0e-7 * kPi;     // mu0 = 4 pi 1e-7 (reading Q7)
constexpr double kMu0Over2Pi = 2.0e-7;    // mu0 / (2 pi)
constexpr int kAgmIters = 10;             // enough for m1 >= 1e-15 (quadratic convergence)

// PDL: wait for the programmatic predecessor (no-op for a normal launch).  Dependents are not
// triggered early (implicit trigger at completion): early-launched dependent CTAs would hold SM
// slots while this kernel still has waves to run (measured slower on the C4 step).
__device__ __forceinline__ void griddep() {
    asm volatile("griddepcontrol.wait;" ::: "memory");
}

// Grid coordinates without FMA contraction (R_i = rmin + i*dR rounded twice), so that
// discrete decisions (limiter test, bilinear cell) are reproducible bit for bit.
__device__ __forceinline__ double grid_coord(double lo, int i, double d) {
    return __dadd_rn(lo, __dmul_rn((double)i, d));
}

// Complete elliptic integrals by the arithmetic-geometric mean (Gauss; A&S 17.6):
//   a0 = 1, b0 = sqrt(m1), c0^2 = m;  a' = (a+b)/2, b' = sqrt(ab), c' = (a-b)/2
//   K = pi/(2 a_inf),  E = K (1 - sum_{n>=0} 2^(n-1) c_n^2).
// Returns K and S1 = sum_{n>=1} 2^(n-1) c_n^2, so that
//   (1 - m/2) K - E = K * S1        (no cancellation; all terms positive)
//   E = K (1 - m/2 - S1).
// c1 = (1 - sqrt(m1))/2 is formed as m / (2 (1 + sqrt(m1))) (cancellation-free: it carries the
// far-field O(m) information); later c_n = (a_{n-1} - b_{n-1})/2, whose absolute rounding error
// (~ulp(a)) moves S1 by < 1e-16 relative because c_n^2 <= c_1^4/16.  The loop stops once the
// increment 2^(n-1) c_n^2 no longer changes S1 (quadratic convergence: <= 6 iterations for
// m1 >= 1e-9, the cap covers m1 >= 1e-15).
// Every operation below is an explicit IEEE intrinsic (no FMA contraction left to the compiler),
// so a Green's value is the same bits in every kernel that evaluates it: the table builds and the
// on-the-fly kernels agree bit for bit by construction.
__device__ __forceinline__ void agm_ks1(double m, double m1, double& K, double& S1) {
    double b = __dsqrt_rn(m1);
    double c = __ddiv_rn(m, __dmul_rn(2.0, __dadd_rn(1.0, b)));  // c1
    double a = __dmul_rn(0.5, __dadd_rn(1.0, b));                // a1
    b = __dsqrt_rn(b);                                           // b1 = sqrt(a0 b0) = sqrt(sqrt(m1))
    double s = __dmul_rn(c, c);                                  // 2^0 c1^2
    double p = 1.0;
#pragma unroll 1
    for (int n = 1; n < kAgmIters; ++n) {
        c = __dmul_rn(0.5, __dsub_rn(a, b));                     // c_{n+1}
        const double an = __dmul_rn(0.5, __dadd_rn(a, b));
        b = __dsqrt_rn(__dmul_rn(a, b));
        a = an;
        p = __dmul_rn(p, 2.0);
        const double t = __dmul_rn(__dmul_rn(p, c), c);
        const double s2 = __dadd_rn(s, t);
        if (s2 == s) break;                                      // converged (also covers c == 0)
        s = s2;
    }
    K = __ddiv_rn(kPi, __dmul_rn(2.0, a));
    S1 = s;
}

// Flux per radian at (R, Z) from a 1 A filament at (Rs, Zs):
//   G = (mu0/2pi) sqrt((R+Rs)^2 + dz^2) [(1 - m/2) K(m) - E(m)],  m = 4 R Rs / den.
__device__ __forceinline__ double green_psi(double R, double Z, double Rs, double Zs) {
    const double dz = __dsub_rn(Z, Zs);
    const double dz2 = __dmul_rn(dz, dz);
    const double sp = __dadd_rn(R, Rs), sm = __dsub_rn(R, Rs);
    const double den = __fma_rn(sp, sp, dz2);
    const double inv = __ddiv_rn(1.0, den);
    const double m = __dmul_rn(__dmul_rn(__dmul_rn(4.0, R), Rs), inv);
    const double m1 = __dmul_rn(__fma_rn(sm, sm, dz2), inv);
    double K, S1;
    agm_ks1(m, m1, K, S1);
    return __dmul_rn(__dmul_rn(__dmul_rn(kMu0Over2Pi, __dsqrt_rn(den)), K), S1);
}

// Self term: point-to-cell average of (mu0/2pi) R (ln(8R/rho) - 2) over a dR x dZ cell
// (reading Q5).
__device__ __forceinline__ double green_self(double R, double dR, double dZ) {
    const double p = __dmul_rn(0.5, dR), q = __dmul_rn(0.5, dZ);
    const double pq = __dmul_rn(p, q), p2 = __dmul_rn(p, p), q2 = __dmul_rn(q, q);
    double num = __dmul_rn(pq, log(__dadd_rn(p2, q2)));
    num = __dsub_rn(num, __dmul_rn(3.0, pq));
    num = __dadd_rn(num, __dmul_rn(p2, atan(__ddiv_rn(q, p))));
    num = __dadd_rn(num, __dmul_rn(q2, atan(__ddiv_rn(p, q))));
    const double lnrho = __ddiv_rn(num, __dmul_rn(2.0, pq));
    return __dmul_rn(__dmul_rn(kMu0Over2Pi, R), __dsub_rn(__dsub_rn(log(__dmul_rn(8.0, R)), lnrho), 2.0));
}

// Field of a 1 A filament at (Rs, Zs) measured at (R, Z) (Smythe; a = Rs, z = Z - Zs):
//   B_Z = (mu0/2pi) [K + (a^2 - R^2 - z^2)/((a-R)^2 + z^2) E] / sqrt((a+R)^2 + z^2)
//   B_R = (mu0/2pi) z [-K + (a^2 + R^2 + z^2)/((a-R)^2 + z^2) E] / (R sqrt((a+R)^2 + z^2))
__device__ __forceinline__ void green_field(double R, double Z, double Rs, double Zs,
                                            double& BR, double& BZ) {
    double z = Z - Zs;
    double z2 = z * z;
    double sp = Rs + R, sm = Rs - R;
    double den = sp * sp + z2;
    double dm = sm * sm + z2;
    double m = 4.0 * R * Rs / den;
    double m1 = dm / den;
    double K, S1;
    agm_ks1(m, m1, K, S1);
    double E = K * ((1.0 - 0.5 * m) - S1);
    double isq = 1.0 / sqrt(den);
    BZ = kMu0Over2Pi * isq * (K + (Rs * Rs - R * R - z2) / dm * E);
    BR = kMu0Over2Pi * z * isq / R * (-K + (Rs * Rs + R * R + z2) / dm * E);
}

// Basis evaluation: out[k] = w_k(R) phi_k(psihat), columns [P' (w = R) | FF' (w = mu0/(4 pi^2 R))].
// kind 0: psihat^k.  kind 1: clamped cubic B-splines -- only the 4 non-zero functions on
// the knot span are formed (Cox-de Boor triangle), the rest are zero.
struct BasisParams {
    int kind, n_pp, n_ff, n_knots;
    double knots[20];
};

template <int NB>
__device__ __forceinline__ void basis_eval(const BasisParams& bp, double h, double R, double* out) {
    double wpp = R;
    double wff = kMu0 / (4.0 * kPi * kPi * R);
    if (bp.kind == 0) {
        double p = 1.0;
#pragma unroll
        for (int k = 0; k < NB; ++k) {
            // columns k < n_pp: P' term k;  k >= n_pp: FF' term k - n_pp
            out[k] = 0.0;
        }
        int nmax = bp.n_pp > bp.n_ff ? bp.n_pp : bp.n_ff;
        double pw[NB];
#pragma unroll
        for (int k = 0; k < NB; ++k) {
            pw[k] = p;
            if (k + 1 < nmax) p *= h;
        }
#pragma unroll
        for (int k = 0; k < NB; ++k) {
            if (k < bp.n_pp) out[k] = wpp * pw[k];
            else if (k < bp.n_pp + bp.n_ff) out[k] = wff * pw[k - bp.n_pp];
        }
    } else {
        // knot vector t: 0,0,0,0, k_1..k_n, 1,1,1,1;  span s with t_s <= h < t_{s+1}, 3 <= s <= n+3
        int n = bp.n_knots;
        int s = 3;
        for (int q = 0; q < n; ++q)
            if (h >= bp.knots[q]) s = 4 + q;
        // t(idx) accessor
        auto t = [&](int idx) -> double {
            if (idx <= 3) return 0.0;
            if (idx >= n + 4) return 1.0;
            return bp.knots[idx - 4];
        };
        double N0[4], left[4], right[4];
        N0[0] = 1.0;
        for (int j = 1; j <= 3; ++j) {
            left[j] = h - t(s + 1 - j);
            right[j] = t(s + j) - h;
            double saved = 0.0;
            for (int r = 0; r < j; ++r) {
                double tmp = N0[r] / (right[r + 1] + left[j - r]);
                N0[r] = saved + right[r + 1] * tmp;
                saved = left[j - r] * tmp;
            }
            N0[j] = saved;
        }
        // non-zero functions: indices s-3 .. s  (0-based basis index)
#pragma unroll
        for (int k = 0; k < NB; ++k) out[k] = 0.0;
        int nf = n + 4;
#pragma unroll
        for (int r = 0; r < 4; ++r) {
            int idx = s - 3 + r;
            if (idx >= 0 && idx < nf) {
                if (idx < bp.n_pp) out[idx] = wpp * N0[r];
                if (bp.n_pp + idx < NB) out[bp.n_pp + idx] = wff * N0[r];
            }
        }
    }
}

}  // namespace efit
