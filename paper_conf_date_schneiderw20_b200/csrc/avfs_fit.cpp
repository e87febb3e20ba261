// avfs_fit.cpp -- NEXT-3: offline regression pre-process (§III-C,
// P:L105-L129; Fig. 1 step C).  Host code: it runs once per cell library, not
// on the simulation path.
//
//   x = phi_V(v) = (v - V_min)/(V_max - V_min)
//   z = phi_C(c) = (log2 c - log2 C_min)/(log2 C_max - log2 C_min)
//   y = phi_D(d) = d / d_nom - 1                                  (Eq. 3)
//   X[k] = (x_k^i z_k^j) for i <= deg_v, j <= deg_c, row-major (i, j)  (Eq. 6, reading C9)
//   beta = argmin ||y - X beta||^2 = (X^T X)^-1 X^T y              (Eq. 7, Eq. 8)
// The normal equation is solved by a Cholesky factorisation in FP64.
#include <cmath>
#include <vector>

#include "avfs.h"

extern "C" avfs_status avfs_fit_delay_polynomial(int64_t n, const double* v, const double* c, const double* y,
                                                 int32_t deg_v, int32_t deg_c, double v_min, double v_max,
                                                 double c_min, double c_max, double* beta, double* rms) {
    if (n < 1 || !v || !y || !beta || deg_v < 0 || deg_c < 0 || deg_v > 7 || deg_c > 7) return AVFS_ERR_ARG;
    if (deg_c > 0 && !c) return AVFS_ERR_ARG;
    if (!(v_max > v_min) || !(c_max > c_min) || !(c_min > 0)) return AVFS_ERR_ARG;
    const int m = (deg_v + 1) * (deg_c + 1);
    if (n < m) return AVFS_ERR_ARG;                     // under-determined
    std::vector<double> A((size_t)m * m, 0.0), b(m, 0.0), row(m);
    const double lc0 = std::log2(c_min), lc1 = std::log2(c_max);
    for (int64_t k = 0; k < n; ++k) {
        const double x = (v[k] - v_min) / (v_max - v_min);
        const double z = deg_c > 0 ? (std::log2(c[k]) - lc0) / (lc1 - lc0) : 0.0;
        double xi = 1.0;
        for (int i = 0; i <= deg_v; ++i) {
            double zj = 1.0;
            for (int j = 0; j <= deg_c; ++j) {
                row[i * (deg_c + 1) + j] = xi * zj;
                zj *= z;
            }
            xi *= x;
        }
        for (int a = 0; a < m; ++a) {
            b[a] += row[a] * y[k];
            for (int e = 0; e <= a; ++e) A[(size_t)a * m + e] += row[a] * row[e];
        }
    }
    // Cholesky A = L L^T (lower triangle of A holds X^T X); a pivot that
    // vanishes relative to its column norm means a rank-deficient design
    std::vector<double> diag(m);
    for (int a = 0; a < m; ++a) diag[a] = A[(size_t)a * m + a];
    for (int a = 0; a < m; ++a) {
        for (int e = 0; e <= a; ++e) {
            double s = A[(size_t)a * m + e];
            for (int f = 0; f < e; ++f) s -= A[(size_t)a * m + f] * A[(size_t)e * m + f];
            if (a == e) {
                if (!(s > 1e-12 * diag[a])) return AVFS_ERR_ARG;   // rank deficient design
                A[(size_t)a * m + a] = std::sqrt(s);
            } else {
                A[(size_t)a * m + e] = s / A[(size_t)e * m + e];
            }
        }
    }
    std::vector<double> t(m);
    for (int a = 0; a < m; ++a) {                       // L t = b
        double s = b[a];
        for (int f = 0; f < a; ++f) s -= A[(size_t)a * m + f] * t[f];
        t[a] = s / A[(size_t)a * m + a];
    }
    for (int a = m - 1; a >= 0; --a) {                  // L^T beta = t
        double s = t[a];
        for (int f = a + 1; f < m; ++f) s -= A[(size_t)f * m + a] * beta[f];
        beta[a] = s / A[(size_t)a * m + a];
    }
    if (rms) {
        double ss = 0.0;
        for (int64_t k = 0; k < n; ++k) {
            const double x = (v[k] - v_min) / (v_max - v_min);
            const double z = deg_c > 0 ? (std::log2(c[k]) - lc0) / (lc1 - lc0) : 0.0;
            double f = 0.0;
            for (int i = deg_v; i >= 0; --i) {
                double a = beta[i * (deg_c + 1) + deg_c];
                for (int j = deg_c - 1; j >= 0; --j) a = std::fma(a, z, beta[i * (deg_c + 1) + j]);
                f = (i == deg_v) ? a : std::fma(f, x, a);
            }
            ss += (y[k] - f) * (y[k] - f);
        }
        *rms = std::sqrt(ss / (double)n);
    }
    return AVFS_OK;
}
