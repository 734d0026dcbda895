// siac_math.cpp -- host-side exact constants of the B200 SIAC library (compiled by g++,
// not nvcc: no __int128 code goes through the CUDA front end).
//
// Everything here is computed once per siac_create in exact rational arithmetic (__int128
// numerators/denominators, overflow-checked) and only then rounded to double:
//   * kernel_coefficients(k): c_gamma of K(t) = sum_g c_g psi_{k+1}(t - x_g), x_g = g - k,
//     from the moment conditions  int K = 1, int K t^m = 0 (m = 1..2k);
//   * kernel_cell_table(k): K restricted to each kernel cell [t_i, t_i + 1],
//     t_i = -(3k+1)/2 + i, as a degree-k polynomial in tau = t - (t_i + 1/2)
//     (the cells are the "array of squares" of PAPER.md L398-401);
//   * dubiner_to_centred(k): the orthonormal Dubiner modes written as polynomials in the
//     centred reference coordinates rho = 3r - 1, sigma = 3s - 1 (r, s barycentric on the
//     unit reference triangle), so the GPU evaluates u_T by a bivariate Horner scheme.
// The B-spline is built from its truncated-power form
//     psi_{k+1}(t) = (1/k!) sum_{j=0}^{k+1} (-1)^j C(k+1, j) (t + (k+1)/2 - j)_+^k,
// and the Dubiner modes from the explicit (non-recursive) Jacobi sums.
#include "siac_math.h"

#include <cmath>
#include <cstdint>
#include <stdexcept>
#include <string>
#include <vector>

namespace siac {

typedef __int128 i128;

static inline i128 gcd128(i128 a, i128 b) {
    if (a < 0) a = -a;
    if (b < 0) b = -b;
    while (b != 0) { i128 t = a % b; a = b; b = t; }
    return a;
}

struct Q {  // exact rational, always normalised (den > 0, gcd = 1)
    i128 n, d;
    Q(long long v = 0) : n(v), d(1) {}
    Q(i128 nn, i128 dd, bool) : n(nn), d(dd) { norm(); }
    static Q frac(long long a, long long b) { return Q((i128)a, (i128)b, true); }
    void norm() {
        if (d == 0) throw std::runtime_error("rational division by zero");
        if (d < 0) { n = -n; d = -d; }
        i128 g = gcd128(n, d);
        if (g > 1) { n /= g; d /= g; }
        if (n == 0) d = 1;
    }
    static i128 mul(i128 a, i128 b) {
        i128 r;
        if (__builtin_mul_overflow(a, b, &r)) throw std::runtime_error("rational overflow");
        return r;
    }
    static i128 add(i128 a, i128 b) {
        i128 r;
        if (__builtin_add_overflow(a, b, &r)) throw std::runtime_error("rational overflow");
        return r;
    }
    friend Q operator+(const Q &a, const Q &b) {
        i128 g = gcd128(a.d, b.d);
        i128 da = a.d / g, db = b.d / g;
        return Q(add(mul(a.n, db), mul(b.n, da)), mul(mul(da, db), g), true);
    }
    friend Q operator-(const Q &a) { Q r = a; r.n = -r.n; return r; }
    friend Q operator-(const Q &a, const Q &b) { return a + (-b); }
    friend Q operator*(const Q &a, const Q &b) {
        i128 g1 = gcd128(a.n, b.d), g2 = gcd128(b.n, a.d);
        if (g1 == 0) g1 = 1;
        if (g2 == 0) g2 = 1;
        return Q(mul(a.n / g1, b.n / g2), mul(a.d / g2, b.d / g1), true);
    }
    friend Q operator/(const Q &a, const Q &b) {
        if (b.n == 0) throw std::runtime_error("rational division by zero");
        return a * Q(b.d, b.n, true);
    }
    bool zero() const { return n == 0; }
    double to_double() const {
        // exact when |n|, d < 2^53 (true for every constant of k <= 4); otherwise <= 1 ulp
        const i128 lim = ((i128)1) << 53;
        i128 a = n, b = d;
        while ((a >= lim || a <= -lim) || b >= lim) { a /= 2; b /= 2; if (b == 0) b = 1; }
        return (double)(long long)a / (double)(long long)b;
    }
};

static inline Q qpow(Q a, int e) { Q r(1); for (int i = 0; i < e; ++i) r = r * a; return r; }
static inline long long binom(int n, int k) {
    if (k < 0 || k > n) return 0;
    long long r = 1;
    for (int i = 1; i <= k; ++i) r = r * (n - k + i) / i;
    return r;
}
static inline long long factorial(int n) { long long r = 1; for (int i = 2; i <= n; ++i) r *= i; return r; }

// ---------------------------------------------------------------- 1D polynomials

typedef std::vector<Q> P1;   // coefficients in powers of the variable

static P1 p1_mul(const P1 &a, const P1 &b) {
    P1 r(a.size() + b.size() - 1, Q(0));
    for (size_t i = 0; i < a.size(); ++i)
        for (size_t j = 0; j < b.size(); ++j) r[i + j] = r[i + j] + a[i] * b[j];
    return r;
}
static P1 p1_pow_linear(Q c0, Q c1, int e) {   // (c0 + c1 x)^e
    P1 r(1, Q(1)), lin{c0, c1};
    for (int i = 0; i < e; ++i) r = p1_mul(r, lin);
    return r;
}

// Piece m (m = 0..k) of psi_{k+1} on its knot interval [tau_m, tau_m + 1], tau_m = -(k+1)/2 + m,
// as a polynomial in lambda = t - (tau_m + 1/2) in [-1/2, 1/2]:
//   psi = (1/k!) sum_{j <= m} (-1)^j C(k+1, j) (t - tau_j)^k,   t - tau_j = lambda + (m - j) + 1/2.
static P1 bspline_piece(int k, int m) {
    P1 r(k + 1, Q(0));
    for (int j = 0; j <= m; ++j) {
        Q w = Q((long long)((j % 2) ? -1 : 1) * binom(k + 1, j)) / Q(factorial(k));
        P1 t = p1_pow_linear(Q(m - j) + Q::frac(1, 2), Q(1), k);
        for (int i = 0; i <= k; ++i) r[i] = r[i] + w * t[i];
    }
    return r;
}

// mu_l = int t^l psi_{k+1}(t) dt, piece by piece.
static Q bspline_moment(int k, int l) {
    Q tot(0);
    for (int m = 0; m <= k; ++m) {
        Q centre = Q::frac(-(k + 1), 2) + Q(m) + Q::frac(1, 2);   // t = lambda + centre
        P1 integrand = p1_mul(p1_pow_linear(centre, Q(1), l), bspline_piece(k, m));
        for (size_t i = 0; i < integrand.size(); ++i) {
            if (i % 2) continue;  // odd powers integrate to 0 over [-1/2, 1/2]
            // int_{-1/2}^{1/2} lambda^i = 2 (1/2)^(i+1) / (i+1)
            tot = tot + integrand[i] * Q(2) * qpow(Q::frac(1, 2), (int)i + 1) / Q((long long)i + 1);
        }
    }
    return tot;
}

// c_gamma (gamma = 0..2k): sum_g c_g int psi(t - x_g) t^m dt = delta_{m0}, m = 0..2k.
static std::vector<Q> kernel_coefficients_exact(int k) {
    int n = 2 * k + 1;
    std::vector<Q> mu(n);
    for (int l = 0; l < n; ++l) mu[l] = bspline_moment(k, l);
    std::vector<std::vector<Q>> A(n, std::vector<Q>(n + 1, Q(0)));
    for (int m = 0; m < n; ++m) {
        for (int g = 0; g < n; ++g) {
            Q xg(g - k), s(0);
            for (int l = 0; l <= m; ++l) s = s + Q(binom(m, l)) * qpow(xg, m - l) * mu[l];
            A[m][g] = s;
        }
        A[m][n] = Q(m == 0 ? 1 : 0);
    }
    for (int col = 0; col < n; ++col) {
        int piv = col;
        while (piv < n && A[piv][col].zero()) ++piv;
        if (piv == n) throw std::runtime_error("singular kernel moment system");
        std::swap(A[col], A[piv]);
        Q pv = A[col][col];
        for (int j = col; j <= n; ++j) A[col][j] = A[col][j] / pv;
        for (int r = 0; r < n; ++r) {
            if (r == col || A[r][col].zero()) continue;
            Q f = A[r][col];
            for (int j = col; j <= n; ++j) A[r][j] = A[r][j] - f * A[col][j];
        }
    }
    std::vector<Q> c(n);
    for (int i = 0; i < n; ++i) c[i] = A[i][n];
    return c;
}

// One-sided kernel support (SIAC_BOUNDARY_ONESIDED; reading R4).  The kernel with
// nodes x_g = g - k + lambda is Kt(t - lambda), Kt on the symmetric node grid with moments
// int Kt s^m = (-lambda)^m (m = 0..2k) -- expand (s + lambda)^m in the shifted kernel's
// conditions int K t^m = delta_m0 -- so its coefficients are c(lambda) = A^{-1} b(lambda),
// b_m = (-lambda)^m, with A the symmetric kernel's moment matrix.  Outputs (exact, rounded once):
//   pieces[m*(k+1) + i]: psi_{k+1}'s piece m in the cell-centred variable (bspline_piece);
//   ainv[g*(2k+1) + m]:  (A^{-1})_{g m}.
void onesided_tables(int k, std::vector<double> &pieces, std::vector<double> &ainv) {
    const int n = 2 * k + 1;
    pieces.assign((size_t)(k + 1) * (k + 1), 0.0);
    for (int m = 0; m <= k; ++m) {
        P1 pc = bspline_piece(k, m);
        for (int i = 0; i <= k; ++i) pieces[(size_t)m * (k + 1) + i] = pc[i].to_double();
    }
    std::vector<Q> mu(n);
    for (int l = 0; l < n; ++l) mu[l] = bspline_moment(k, l);
    std::vector<std::vector<Q>> A(n, std::vector<Q>(2 * n, Q(0)));
    for (int m = 0; m < n; ++m) {
        for (int g = 0; g < n; ++g) {
            Q xg(g - k), s(0);
            for (int l = 0; l <= m; ++l) s = s + Q(binom(m, l)) * qpow(xg, m - l) * mu[l];
            A[m][g] = s;
        }
        A[m][n + m] = Q(1);
    }
    for (int col = 0; col < n; ++col) {
        int piv = col;
        while (piv < n && A[piv][col].zero()) ++piv;
        if (piv == n) throw std::runtime_error("singular kernel moment system");
        std::swap(A[col], A[piv]);
        Q pv = A[col][col];
        for (int j = col; j < 2 * n; ++j) A[col][j] = A[col][j] / pv;
        for (int r = 0; r < n; ++r) {
            if (r == col || A[r][col].zero()) continue;
            Q f = A[r][col];
            for (int j = col; j < 2 * n; ++j) A[r][j] = A[r][j] - f * A[col][j];
        }
    }
    // rows of A now hold A^{-1} in columns n..2n-1: (A^{-1})_{g m} = A[g][n + m]
    ainv.assign((size_t)n * n, 0.0);
    for (int g = 0; g < n; ++g)
        for (int m = 0; m < n; ++m) ainv[(size_t)g * n + m] = A[g][n + m].to_double();
}

// table[i*(k+1) + m]: coefficient of tau^m of K on cell i, tau = t - (t_i + 1/2).
// On cell i, psi(t - x_g) is psi's piece i - g (when 0 <= i - g <= k), with the same local
// variable (t_i - x_g = tau_{i-g}).
std::vector<double> kernel_cell_table(int k, std::vector<double> *coeffs_out) {
    std::vector<Q> c = kernel_coefficients_exact(k);
    if (coeffs_out) { coeffs_out->clear(); for (auto &v : c) coeffs_out->push_back(v.to_double()); }
    std::vector<P1> pieces;
    for (int m = 0; m <= k; ++m) pieces.push_back(bspline_piece(k, m));
    int nc = 3 * k + 1;
    std::vector<double> table((size_t)nc * (k + 1));
    for (int i = 0; i < nc; ++i) {
        P1 acc(k + 1, Q(0));
        for (int g = 0; g <= 2 * k; ++g) {
            int m = i - g;
            if (m < 0 || m > k) continue;
            for (int j = 0; j <= k; ++j) acc[j] = acc[j] + c[g] * pieces[m][j];
        }
        for (int j = 0; j <= k; ++j) table[(size_t)i * (k + 1) + j] = acc[j].to_double();
    }
    return table;
}

// ---------------------------------------------------------------- 2D polynomials in (rho, sigma)

struct P2 {   // dense, c[a][b] for rho^a sigma^b, a, b <= D
    int D;
    std::vector<Q> c;
    explicit P2(int D_) : D(D_), c((size_t)(D_ + 1) * (D_ + 1), Q(0)) {}
    Q &at(int a, int b) { return c[(size_t)a * (D + 1) + b]; }
    const Q &at(int a, int b) const { return c[(size_t)a * (D + 1) + b]; }
};
static P2 p2_mul(const P2 &x, const P2 &y) {
    P2 r(x.D);
    for (int a1 = 0; a1 <= x.D; ++a1)
        for (int b1 = 0; b1 <= x.D; ++b1) {
            if (x.at(a1, b1).zero()) continue;
            for (int a2 = 0; a2 + a1 <= x.D; ++a2)
                for (int b2 = 0; b2 + b1 <= x.D; ++b2) {
                    if (y.at(a2, b2).zero()) continue;
                    r.at(a1 + a2, b1 + b2) = r.at(a1 + a2, b1 + b2) + x.at(a1, b1) * y.at(a2, b2);
                }
        }
    return r;
}
static P2 p2_lin(int D, Q c0, Q crho, Q csig) {
    P2 r(D);
    r.at(0, 0) = c0; r.at(1, 0) = crho; r.at(0, 1) = csig;
    return r;
}
static P2 p2_pow(const P2 &x, int e) { P2 r(x.D); r.at(0, 0) = Q(1); for (int i = 0; i < e; ++i) r = p2_mul(r, x); return r; }
static void p2_axpy(P2 &y, Q a, const P2 &x) { for (size_t i = 0; i < y.c.size(); ++i) y.c[i] = y.c[i] + a * x.c[i]; }

// Orthonormal Dubiner mode (p, q) in centred coordinates:
//   xi = 2r - 1 = (2 rho - 1)/3,  eta = (2 sigma - 1)/3,
//   ((1-eta)/2)^p P_p(a) = sum_s C(p,s)^2 ((xi+eta)/2)^s ((1+xi)/2)^(p-s)
//   P_q^(alpha,0)(eta) = sum_s C(q+alpha, q-s) C(q, s) ((eta-1)/2)^s ((eta+1)/2)^(q-s).
// Returned WITHOUT the normalisation sqrt((2p+1)(p+q+1)/2) (irrational; applied in double).
static P2 dubiner_mode_centred(int D, int p, int q) {
    Q third = Q::frac(1, 3);
    // (xi+eta)/2 = (rho + sigma - 1)/3 ; (1+xi)/2 = (rho + 1)/3
    P2 A = p2_lin(D, -third, third, third);
    P2 B = p2_lin(D, third, third, Q(0));
    // (eta-1)/2 = (sigma - 2)/3 ; (eta+1)/2 = (sigma + 1)/3
    P2 Cm = p2_lin(D, Q::frac(-2, 3), Q(0), third);
    P2 Cp = p2_lin(D, third, Q(0), third);
    P2 Qp(D);
    for (int s = 0; s <= p; ++s)
        p2_axpy(Qp, Q(binom(p, s) * binom(p, s)), p2_mul(p2_pow(A, s), p2_pow(B, p - s)));
    int alpha = 2 * p + 1;
    P2 J(D);
    for (int s = 0; s <= q; ++s)
        p2_axpy(J, Q(binom(q + alpha, q - s) * binom(q, s)), p2_mul(p2_pow(Cm, s), p2_pow(Cp, q - s)));
    return p2_mul(Qp, J);
}

// Row-major (nb x nb) matrix R: d[j] = sum_i coeff[i] * R[i*nb + j], where j indexes the
// centred monomials in GPU Horner order (see monomial_order), including the normalisation.
std::vector<double> dubiner_to_centred(int k, std::vector<std::pair<int, int>> *order_out) {
    // Horner order: u = sum_a rho^a * (sum_b d_ab sigma^b); the GPU reads, for a = k..0,
    // the block d_a0 .. d_a,(k-a).  j enumerates (a, b) in that order: a descending, b ascending.
    std::vector<std::pair<int, int>> order;
    for (int a = k; a >= 0; --a)
        for (int b = 0; b <= k - a; ++b) order.push_back({a, b});
    if (order_out) *order_out = order;
    int nb = (k + 1) * (k + 2) / 2;
    std::vector<double> R((size_t)nb * nb, 0.0);
    int i = 0;
    for (int n = 0; n <= k; ++n)
        for (int q = 0; q <= n; ++q, ++i) {
            int p = n - q;
            P2 m = dubiner_mode_centred(k, p, q);
            double norm = std::sqrt((2.0 * p + 1.0) * (p + q + 1.0) / 2.0);
            for (int j = 0; j < nb; ++j) R[(size_t)i * nb + j] = norm * m.at(order[j].first, order[j].second).to_double();
        }
    return R;
}

std::vector<double> monomial_to_centred(int k) {
    std::vector<std::pair<int, int>> order;
    dubiner_to_centred(k, &order);
    const int nb = (k + 1) * (k + 2) / 2;
    std::vector<double> R((size_t)nb * nb, 0.0);
    const Q third = Q::frac(1, 3);
    const P2 rr = p2_lin(k, third, third, Q(0));      // r = (rho + 1)/3
    const P2 ss = p2_lin(k, third, Q(0), third);      // s = (sigma + 1)/3
    int i = 0;
    for (int n = 0; n <= k; ++n)
        for (int b = 0; b <= n; ++b, ++i) {
            const P2 m = p2_mul(p2_pow(rr, n - b), p2_pow(ss, b));
            for (int j = 0; j < nb; ++j) R[(size_t)i * nb + j] = m.at(order[j].first, order[j].second).to_double();
        }
    return R;
}

}  // namespace siac
