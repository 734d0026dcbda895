// siac_jump.cuh -- schedules JUMPX (the default, SIAC_SCHEDULE_DEFAULT) and JUMP: the exact
// decomposition of Eq. (2) reorganised around the spline structure of the kernel, so that almost
// no per-pair quadrature is needed (JUMPX: none).
//
// Why it is exact.  K is a spline of degree k on the unit knots t_m = T0 + m (m = 0..3k+1,
// T0 = -(3k+1)/2), C^{k-1} everywhere and zero outside [t_0, t_{3k+1}] (PAPER.md L196-208,
// L250-254).  Across a knot only the k-th derivative jumps, so with P_i the polynomial of K on
// cell i (P_{-1} = P_{3k+1} = 0)
//     P_m(t) - P_{m-1}(t) = alpha_m (t - t_m)^k,   alpha_m = lead(P_m) - lead(P_{m-1}).
// When h >= the longest edge (the paper's h = s, L430/L440), a triangle's x-range (in z = (y-x)/h
// units) is <= 1, so at most one knot X lies strictly inside it, and on the triangle
//     K(z1) = B1(z1) + C1(z1),  B1 = P_{base},  C1 = sgn alpha_X (z1 - X)^k 1[corner_x],
// where corner_x = T ∩ {z1 on the side of X holding a single vertex} is a triangle: the
// Sutherland-Hodgman clip (Alg. 1) of T against the line z1 = X, on the "alone vertex" side
// (base = the cell on the other side; sgn = +1 if the corner is right of X, -1 if left).
// Likewise for z2.  Eq. (2)'s integral over the pieces of T then splits into four terms:
//     I00 = \int_T B1 B2 u                    -- per-triangle moments mu_ab = \int_T zeta1^a zeta2^b u
//     I10 = \int_{corner_x} C1 B2 u           -- corner_x is the homothetic image of a fixed
//     I01 = \int_{corner_y} B1 C2 u              reference corner about the alone vertex, ratio
//                                                lambda, so \int_{corner} (zeta1 - X)^k zeta2^b u
//                                                = lambda^{k+2} G_b(lambda), G_b a polynomial of
//                                                degree k+b precomputed per triangle at create time
//     I11 = \int_{corner_x ∩ corner_y} C1 C2 u -- JUMP: corner_x clipped by the line z2 = Y (SH),
//                                                fan-triangulated, degree-3k Gauss quadrature;
//                                                JUMPX: a per-triangle interval polynomial in
//                                                (lambda, Y') built at create time (§8.2b).
// zeta = (y - centroid)/h is the per-triangle frame the precomputed data live in; z = zeta +
// delta, delta = (centroid + image shift - x)/h.  Pairs with two or more knots inside a range
// (only when h is smaller than the triangles) take the general per-pair path of siac_device.cuh.
//
// Execution: one warp per tile of 32 Morton-consecutive points (lane = point), exactly like
// schedule TILE for candidate search; for every candidate triangle the whole warp evaluates the
// closed-form terms with warp-uniform record loads (one triangle, 32 stencils), and the rare I11
// terms are queued in shared memory and integrated 32 at a time by the full warp.
#pragma once

#include <type_traits>

#include "siac_device.cuh"

namespace siacjump {

using namespace siacdev;

// ------------------------------------------------------------------ jump record layout (doubles)
// Every field group starts at an even offset so it is read with 16-byte (double2) loads.
//   [0,1]              centroid (physical)
//   [2..7] / [8..13]   axis x / y: zlo, zhi, zmid, zc5 = (zlo+zhi)/2 + 1/2, invL = 1/(zmid-zlo),
//                      invR = 1/(zhi-zmid)
//                      (sorted vertex coordinates in the zeta frame; inv = 0 for a degenerate corner)
//   [OFF_MU ..]        mu[a*(K+1)+b] = \int_T zeta1^a zeta2^b u dzeta, a, b = 0..K (padded to even)
//   [OFF_G ..]         4 corners (x-right, x-left, y-top, y-bottom) x NGP coefficients:
//                      block b (= power of the other coordinate, 0..K) holds G_b[0..K+b]
//   [OFF_XH ..]        per x corner side (0: apex R, 1: apex L): Ay, then the sorted heights
//                      v0 <= v1 <= v2 of its reference corner (A, Mv, C') -- what the cross-term
//                      classification needs at enqueue time (8 doubles)
//   [OFF_GEO ..]       per axis: L, Mv, R (vertices sorted by that coordinate), C' (the point of
//                      edge L-R at coordinate Mv) -- 8 doubles per axis
//   [OFF_MAP ..]       rho = m00 z1 + m01 z2 + r0, sigma = m10 z1 + m11 z2 + s0 (centred reference
//                      coordinates of the record's modes, rho = 3r-1, sigma = 3s-1)
//   [OFF_D ..]         modes d in centred monomials, Horner order (siac_device.cuh, Rec<K>)
// [0, OFF_GEO) is what every (tile, candidate) step reads; the rest only the cross terms.
template <int K> struct JRec {
    static constexpr int NB = (K + 1) * (K + 2) / 2;
    static constexpr int NG = (K + 1) * (3 * K + 2) / 2;
    static constexpr int NGP = (NG + 1) & ~1;
    static constexpr int NMU = (K + 1) * (K + 1);
    static constexpr int OFF_AX = 2;
    static constexpr int OFF_MU = 14;
    static constexpr int OFF_G = OFF_MU + ((NMU + 1) & ~1);
    static constexpr int OFF_XH = OFF_G + 4 * NGP;
    static constexpr int OFF_GEO = OFF_XH + 8;
    static constexpr int OFF_MAP = OFF_GEO + 16;
    static constexpr int OFF_D = OFF_MAP + 6;
    static constexpr int RAW = OFF_D + NB;
    static constexpr int RS = (RAW + 1) & ~1;
};
__host__ __device__ constexpr int g_off(int K, int b) { return b * (K + 1) + b * (b - 1) / 2; }

// ------------------------------------------------------------------ create-time record build

// polynomial in lambda (degree <= D, coefficients p[0..D]) times (c0 + c1 lambda)
template <int D> __device__ __forceinline__ void pmul_lin(double *p, int deg, double c0, double c1) {
    p[deg + 1 < D + 1 ? deg + 1 : D] = 0.0;
    for (int j = deg + 1; j >= 1; --j) p[j] = fma(p[j], c0, p[j - 1] * c1);
    p[0] *= c0;
}

// coefficients in lambda of u(A + lambda d), u = horner2(dm, rho, sigma), rho/sigma affine
template <int K>
__device__ void u_along(const double *dm, double rA, double rD, double sA, double sD, double *ul) {
    double in[K + 2];
    int off = 0;
    for (int j = 0; j <= K; ++j) ul[j] = 0.0;
    int udeg = 0;
    for (int a = K; a >= 0; --a) {
        const int n = K - a;
        for (int j = 0; j <= K + 1; ++j) in[j] = 0.0;
        in[0] = dm[off + n];
        int deg = 0;
        for (int b = n - 1; b >= 0; --b) {
            pmul_lin<K + 1>(in, deg, sA, sD);
            ++deg;
            in[0] += dm[off + b];
        }
        if (a == K) {
            for (int j = 0; j <= deg; ++j) ul[j] = in[j];
            udeg = deg;
        } else {
            double t[K + 2];
            for (int j = 0; j <= K + 1; ++j) t[j] = j <= K ? ul[j] : 0.0;
            pmul_lin<K + 1>(t, udeg, rA, rD);
            udeg = udeg + 1 > deg ? udeg + 1 : deg;
            for (int j = 0; j <= K; ++j) ul[j] = t[j] + (j <= deg ? in[j] : 0.0);
        }
        off += n + 1;
    }
}

// One thread per triangle (binning order).  rec: siacdev::Rec<K> records (same order).
template <int K>
__global__ void k_prep_jump(const double *rec, int64_t nt, double h, double *jrec) {
    using R = Rec<K>;
    using J = JRec<K>;
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= nt) return;
    const double *r = rec + (int64_t)R::RS * t;
    double *o = jrec + (int64_t)J::RS * t;
    const double inv_h = 1.0 / h;
    const double cx = (r[0] + r[2] + r[4]) / 3.0, cy = (r[1] + r[3] + r[5]) / 3.0;
    double zx[3], zy[3];
    for (int v = 0; v < 3; ++v) { zx[v] = (r[2 * v] - cx) * inv_h; zy[v] = (r[2 * v + 1] - cy) * inv_h; }
    // (rho, sigma) = M (z - z_v0) - (1, 1), M = 3 h A^{-1}: affine in zeta
    const double m00 = r[6], m01 = r[7], m10 = r[8], m11 = r[9];
    const double r0 = -fma(m00, zx[0], m01 * zy[0]) - 1.0, s0 = -fma(m10, zx[0], m11 * zy[0]) - 1.0;
    double dm[R::NB];
    for (int j = 0; j < R::NB; ++j) dm[j] = r[R::OFF_D + j];
    o[0] = cx; o[1] = cy;
    // moments over T
    {
        const double e1x = zx[1] - zx[0], e1y = zy[1] - zy[0], e2x = zx[2] - zx[0], e2y = zy[2] - zy[0];
        const double area = 0.5 * fabs(e1x * e2y - e1y * e2x);
        double mu[(K + 1) * (K + 1)];
        for (int i = 0; i < (K + 1) * (K + 1); ++i) mu[i] = 0.0;
        for (int q = 0; q < Rule<K>::NQ; ++q) {
            const double a1 = zx[0] + qr<K>(q) * e1x + qs<K>(q) * e2x;
            const double a2 = zy[0] + qr<K>(q) * e1y + qs<K>(q) * e2y;
            const double u = horner2<K>(dm, fma(m00, a1, fma(m01, a2, r0)), fma(m10, a1, fma(m11, a2, s0)));
            double pa = area * qw<K>(q) * u;
            for (int a = 0; a <= K; ++a) {
                double pb = pa;
                for (int b = 0; b <= K; ++b) { mu[a * (K + 1) + b] += pb; pb *= a2; }
                pa *= a1;
            }
        }
        for (int i = 0; i < (K + 1) * (K + 1); ++i) o[J::OFF_MU + i] = mu[i];
        for (int i = J::OFF_MU + J::NMU; i < J::OFF_G; ++i) o[i] = 0.0;
    }
    for (int ax = 0; ax < 2; ++ax) {
        const double *cA = ax == 0 ? zx : zy;   // coordinate along the cut axis
        int iL = 0, iM = 1, iR = 2;
        if (cA[iL] > cA[iM]) { int s = iL; iL = iM; iM = s; }
        if (cA[iM] > cA[iR]) { int s = iM; iM = iR; iR = s; }
        if (cA[iL] > cA[iM]) { int s = iL; iL = iM; iM = s; }
        const double Lx = zx[iL], Ly = zy[iL], Mx = zx[iM], My = zy[iM], Rx = zx[iR], Ry = zy[iR];
        const double lo = cA[iL], mid = cA[iM], hi = cA[iR];
        const double f = (mid - lo) / (hi - lo);
        const double Cx = Lx + f * (Rx - Lx), Cy = Ly + f * (Ry - Ly);
        double *ad = o + J::OFF_AX + 6 * ax;
        ad[0] = lo; ad[1] = hi; ad[2] = mid; ad[3] = 0.5 * (lo + hi) + 0.5;
        ad[4] = mid > lo ? 1.0 / (mid - lo) : 0.0;
        ad[5] = hi > mid ? 1.0 / (hi - mid) : 0.0;
        double *geo = o + J::OFF_GEO + 8 * ax;
        geo[0] = Lx; geo[1] = Ly; geo[2] = Mx; geo[3] = My; geo[4] = Rx; geo[5] = Ry; geo[6] = Cx; geo[7] = Cy;
        if (ax == 0) {
            for (int side = 0; side < 2; ++side) {   // heights of the reference corner (A, Mv, C')
                const double Ay = side == 0 ? Ry : Ly;
                double v[3] = {Ay, My, Cy};
                if (v[0] > v[1]) { const double tt = v[0]; v[0] = v[1]; v[1] = tt; }
                if (v[1] > v[2]) { const double tt = v[1]; v[1] = v[2]; v[2] = tt; }
                if (v[0] > v[1]) { const double tt = v[0]; v[0] = v[1]; v[1] = tt; }
                double *xh = o + J::OFF_XH + 4 * side;
                xh[0] = Ay; xh[1] = v[0]; xh[2] = v[1]; xh[3] = v[2];
            }
        }
        for (int side = 0; side < 2; ++side) {      // 0: apex = R (right/top), 1: apex = L
            const double Ax = side == 0 ? Rx : Lx, Ay = side == 0 ? Ry : Ly;
            const double e1x = Mx - Ax, e1y = My - Ay, e2x = Cx - Ax, e2y = Cy - Ay;
            const double area = 0.5 * fabs(e1x * e2y - e1y * e2x);
            double g[J::NG];
            for (int i = 0; i < J::NG; ++i) g[i] = 0.0;
            const double rA = fma(m00, Ax, fma(m01, Ay, r0)), sA = fma(m10, Ax, fma(m11, Ay, s0));
            const double aO = ax == 0 ? Ay : Ax;
            for (int q = 0; q < Rule<K>::NQ; ++q) {
                const double dx = qr<K>(q) * e1x + qs<K>(q) * e2x, dy = qr<K>(q) * e1y + qs<K>(q) * e2y;
                const double xiA = (ax == 0 ? Ax + dx : Ay + dy) - mid;   // (xi_axis - Mv_axis)
                double wq = area * qw<K>(q);
                for (int i = 0; i < K; ++i) wq *= xiA;
                double ul[K + 1];
                u_along<K>(dm, rA, fma(m00, dx, m01 * dy), sA, fma(m10, dx, m11 * dy), ul);
                double w[2 * K + 2];
                for (int j = 0; j < 2 * K + 2; ++j) w[j] = j <= K ? ul[j] : 0.0;
                const double dO = ax == 0 ? dy : dx;
                for (int b = 0; b <= K; ++b) {
                    const int deg = K + b;
                    double *gb = g + g_off(K, b);
                    for (int j = 0; j <= deg; ++j) gb[j] = fma(wq, w[j], gb[j]);
                    if (b < K) pmul_lin<2 * K + 1>(w, deg, aO, dO);
                }
            }
            double *go = o + J::OFF_G + (2 * ax + side) * J::NGP;
            for (int i = 0; i < J::NGP; ++i) go[i] = (area > 0.0 && i < J::NG) ? g[i] : 0.0;
        }
    }
    double *mp = o + J::OFF_MAP;
    mp[0] = m00; mp[1] = m01; mp[2] = m10; mp[3] = m11; mp[4] = r0; mp[5] = s0;
    for (int j = 0; j < R::NB; ++j) o[J::OFF_D + j] = dm[j];
    for (int j = J::RAW; j < J::RS; ++j) o[j] = 0.0;
}


// ------------------------------------------------------------------ closed-form cross terms
// I11 = \int_{corner_x ∩ corner_y} (z1 - X)^K (z2 - Y)^K u.  With the homothety about the apex A
// of the x corner (ratio lambda): zeta = A + lambda (w - A), z1 - X = lambda (w1 - M1) and
// z2 - Y = lambda (w2 - Y'), Y' = A2 + (Y - A2) / lambda, so
//     I11 = lambda^{2K+2} F(lambda, Y'),  F = \int_{Cx ∩ H(Y')} (w1 - M1)^K (w2 - Y')^K u(A + lambda (w - A)) dw
// over the fixed reference corner Cx = (A, M, C') clipped (Alg. 1) by the y knot line.  For the
// half-plane above the line (y corner on the top side), F is a polynomial in (lambda, Y') of
// degree K x (3K + 2) on each of the two intervals between the corner's vertex heights (the
// clipped region is a triangle with vertices affine in Y'; the integrand has total degree 3K),
// 0 above the corner and the full-corner integral below it (the corner polynomials G).  Below
// the line (y corner on the bottom side) the same holds with "above" and "below" exchanged; its
// interval polynomials F_below = F_full - F_above (F_full: the unclipped corner, degree K in
// Y') are stored as well, so every in-interval cross term is ONE polynomial evaluation.  The
// interval polynomials are built at create time by Chebyshev interpolation of exact samples
// (each sample: SH clip of Cx + the degree-3K rule), stored as monomials in (mu, s) on
// [-1, 1]^2 and evaluated column-wise in mu (independent short chains) then by Estrin in s.
template <int K> struct XRec {
    static constexpr int NS = 3 * K + 3;          // Y' degree + 1
    static constexpr int NL = K + 1;              // lambda degree + 1
    static constexpr int NLP = (NL + 1) & ~1;     // padded for 16-byte loads
    static constexpr int NP = NS * NLP;           // monomial coefficients m[j * NLP + i]: s^j mu^i
    // per x side: v0 v1 v2 iw0 iw1 0 | interval 0 above, interval 0 below, interval 1 above,
    // interval 1 below (NP each)
    static constexpr int XB = (6 + 4 * NP + 1) & ~1;
    static constexpr int RS = 2 * XB;
    __host__ __device__ static constexpr int poly(int iv, int below) { return 6 + (2 * iv + below) * NP; }
};

// \int over triangle (p0, p1, p2) of (w1 - M1)^K (w2 - Yp)^K u(A + lam (w - A)), degree-3K rule;
// u in centred reference coordinates through the record's affine map mp.
template <int K>
__device__ double corner_piece(double p0x, double p0y, double p1x, double p1y, double p2x, double p2y, double M1,
                               double Yp, double Ax, double Ay, double lam, const double *mp, const double *d) {
    const double e1x = p1x - p0x, e1y = p1y - p0y, e2x = p2x - p0x, e2y = p2y - p0y;
    const double area = 0.5 * fabs(e1x * e2y - e1y * e2x);
    double acc = 0.0;
    for (int q = 0; q < Rule<K>::NQ; ++q) {
        const double w1 = p0x + qr<K>(q) * e1x + qs<K>(q) * e2x;
        const double w2 = p0y + qr<K>(q) * e1y + qs<K>(q) * e2y;
        const double z1 = fma(lam, w1 - Ax, Ax), z2 = fma(lam, w2 - Ay, Ay);
        const double rho = fma(mp[0], z1, fma(mp[1], z2, mp[4]));
        const double sig = fma(mp[2], z1, fma(mp[3], z2, mp[5]));
        double t = (w1 - M1) * (w2 - Yp), tp = 1.0;
        for (int i = 0; i < K; ++i) tp *= t;
        acc = fma(qw<K>(q), tp * horner2<K>(d, rho, sig), acc);
    }
    return area * acc;
}

// Interpolation at Chebyshev nodes -> monomial coefficients, as two small matrices built on the
// host in long double (siac_eval_k.cu): ms[jm * NS + is] maps the NS samples in s to the
// coefficient of s^jm, ml[im * NL + il] the NL samples in lambda to the coefficient of mu^im
// (mu = 2 lambda - 1); nodes cos((2i+1) pi / (2N)).  Passed by value (kernel parameters).
template <int K> struct CrossTabs {
    double ms[XRec<K>::NS * XRec<K>::NS];
    double ml[XRec<K>::NL * XRec<K>::NL];
    double node_s[XRec<K>::NS], node_l[XRec<K>::NL];
};

// (lambda, s) samples f[il][is] -> co[jm * NLP + im] (coefficient of s^jm mu^im), padding 0.
template <int K>
__device__ void samples_to_monomial(const CrossTabs<K> &tb, const double (*f)[XRec<K>::NS], double *co) {
    using X = XRec<K>;
    for (int jm = 0; jm < X::NS; ++jm) {
        double g[X::NL];
        for (int il = 0; il < X::NL; ++il) {
            double acc = 0.0;
            for (int is = 0; is < X::NS; ++is) acc = fma(tb.ms[jm * X::NS + is], f[il][is], acc);
            g[il] = acc;
        }
        for (int im = 0; im < X::NLP; ++im) {
            double acc = 0.0;
            if (im < X::NL)
                for (int il = 0; il < X::NL; ++il) acc = fma(tb.ml[im * X::NL + il], g[il], acc);
            co[jm * X::NLP + im] = acc;
        }
    }
}

// One thread per (triangle, x side, interval): the above and below interval polynomials.
template <int K>
__global__ void k_prep_cross(const double *jrec, int64_t nt, double *xrec, const CrossTabs<K> tb) {
    using J = JRec<K>;
    using X = XRec<K>;
    const int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (idx >= 4 * nt) return;
    const int64_t t = idx >> 2;
    const int sx = (int)(idx >> 1) & 1, iv = (int)idx & 1;
    const double *jr = jrec + (int64_t)J::RS * t;
    const double *geo = jr + J::OFF_GEO;            // x axis: L, M, R, C'
    const double Ax = sx == 0 ? geo[4] : geo[0], Ay = sx == 0 ? geo[5] : geo[1];
    const double Mx = geo[2], My = geo[3], Cx = geo[6], Cy = geo[7];
    double mp[6], d[J::NB];
    for (int i = 0; i < 6; ++i) mp[i] = jr[J::OFF_MAP + i];
    for (int i = 0; i < J::NB; ++i) d[i] = jr[J::OFF_D + i];
    const double *xh = jr + J::OFF_XH + 4 * sx;     // sorted heights (k_prep_jump)
    const double v0 = xh[1], v1 = xh[2], v2 = xh[3];
    double *xo = xrec + (int64_t)X::RS * t + sx * X::XB;
    if (iv == 0) {
        xo[0] = v0; xo[1] = v1; xo[2] = v2;
        xo[3] = v1 > v0 ? 1.0 / (v1 - v0) : 0.0;
        xo[4] = v2 > v1 ? 1.0 / (v2 - v1) : 0.0;
        xo[5] = 0.0;
        for (int i = 6 + 4 * X::NP; i < X::XB; ++i) xo[i] = 0.0;
    }
    double *ca = xo + X::poly(iv, 0), *cb = xo + X::poly(iv, 1);
    const double a = iv == 0 ? v0 : v1, b = iv == 0 ? v1 : v2;
    if (!(b > a)) {
        for (int i = 0; i < X::NP; ++i) { ca[i] = 0.0; cb[i] = 0.0; }
        return;
    }
    double fa[X::NL][X::NS], fb[X::NL][X::NS];
    const double px[3] = {Ax, Mx, Cx}, py[3] = {Ay, My, Cy};
    for (int il = 0; il < X::NL; ++il) {
        const double lam = 0.5 * (tb.node_l[il] + 1.0);
        for (int is = 0; is < X::NS; ++is) {
            const double Yp = a + 0.5 * (tb.node_s[is] + 1.0) * (b - a);
            // Sutherland-Hodgman clip of (A, M, C') by w2 >= Yp, fan from the first vertex
            double qx[4], qy[4];
            int n = 0;
            for (int e = 0; e < 3; ++e) {
                const int e2 = e == 2 ? 0 : e + 1;
                const bool in0 = py[e] >= Yp, in1 = py[e2] >= Yp;
                if (in0) { qx[n] = px[e]; qy[n] = py[e]; ++n; }
                if (in0 != in1) {
                    const double r = (Yp - py[e]) / (py[e2] - py[e]);
                    qx[n] = fma(r, px[e2] - px[e], px[e]); qy[n] = Yp; ++n;
                }
            }
            double F = 0.0;
            for (int j = 1; j + 1 < n; ++j)
                F += corner_piece<K>(qx[0], qy[0], qx[j], qy[j], qx[j + 1], qy[j + 1], Mx, Yp, Ax, Ay, lam, mp, d);
            // the whole corner at the same (lambda, Y'): F_below = F_full - F_above
            const double Ffull = corner_piece<K>(Ax, Ay, Mx, My, Cx, Cy, Mx, Yp, Ax, Ay, lam, mp, d);
            fa[il][is] = F;
            fb[il][is] = Ffull - F;
        }
    }
    samples_to_monomial<K>(tb, fa, ca);
    samples_to_monomial<K>(tb, fb, cb);
}

// ------------------------------------------------------------------ evaluation

#ifndef SIAC_JUMP_WARPS
#define SIAC_JUMP_WARPS 4
#endif
#ifndef SIAC_JUMP_MINB
#define SIAC_JUMP_MINB 4
#endif
#ifndef SIAC_JUMP_PREFETCH
#define SIAC_JUMP_PREFETCH 2      // candidates ahead whose hot record lines are prefetched into L1
#endif
constexpr int WARPS = SIAC_JUMP_WARPS;
constexpr int QCAP = 64;      // cross-term queue: < 32 left over + <= 32 new
constexpr int SCAP = 96;      // staged cross sub-triangles: < 32 left over + <= 64 new

template <int SC> struct WarpSmemT {
    // cross-term queue (one entry per lane with a knot on both axes)
    int qtri[QCAP];
    int qinfo[QCAP];          // lane | sx << 5 | sy << 6 | mx << 7 | my << 12 | row_x << 17
    double qX[QCAP], qY[QCAP];
    double qE[QCAP], qL[QCAP]; // deferred y-corner term: base-x offset e_x, y homothety ratio
    // staged cross sub-triangles (compacted; integrated 32 at a time)
    double s0x[SC], s0y[SC], s1x[SC], s1y[SC], s2x[SC], s2y[SC];
    double sX[SC], sY[SC];
    int stri[SC], sinfo[SC];
    double acc[32];
    double4 cbox[32];
    int klist[32];            // kept candidates of the current chunk (box meets the tile's stencils)
};
using WarpSmem = WarpSmemT<SCAP>;     // schedule JUMP: staged cross sub-triangles

// Schedule JUMPX: cross terms classified at enqueue time (while the record is staged) into two
// queues that are each evaluated 32 at a time without divergence:
//   qp  "poly":  the y knot line cuts the x corner -> one interval polynomial (above / below);
//   qf  "full":  the line misses it -> the whole-corner integral (corner polynomials) or 0.
// Every entry also carries the pair's deferred y-corner term.
struct XQueue {
    int tri[QCAP];
    int info[QCAP];           // lane | sx << 6 | sy << 7 | mx << 8 | my << 13 | row_x << 18 | iv << 23 | full << 24
    double Y[QCAP];           // y knot (zeta frame of the triangle)
    double E[QCAP], L[QCAP];  // deferred y-corner term: base-x offset e_x, y homothety ratio
    double lam[QCAP];         // x corner homothety ratio
};
struct WarpSmemX {
    XQueue qp, qf;
    double acc[32];
    double4 cbox[32];
    int klist[32];
};
template <bool XP> using WarpSmemFor = typename std::conditional<XP, WarpSmemX, WarpSmem>::type;

#ifndef SIAC_JUMP_STAGES
#define SIAC_JUMP_STAGES 2        // records in flight per warp (TMA ring)
#endif
constexpr int NST = SIAC_JUMP_STAGES;
static_assert((NST & (NST - 1)) == 0, "SIAC_JUMP_STAGES must be a power of two");

// Per-warp TMA ring: the hot part [0, OFF_GEO) of the next candidates' records, copied global ->
// shared by cp.async.bulk while the warp works on the current one.
template <int K> struct WarpStage {
    alignas(16) double rec[NST][JRec<K>::OFF_GEO];
    unsigned long long bar[NST];
    int hj[32];               // candidates of the chunk some lane's stencil meets (chunk index)
    unsigned hm[32];          // their lane masks
};

template <int K, int NPT = 32> struct OsSmem {   // one-sided kernels: per-point c[axis][g][point]
    double c[2][2 * K + 1][NPT];
};

struct JumpArgs {
    const double *pts;
    const int *perm;
    int64_t np;
    double *out;
    const double *rec;        // Rec<K> (general fallback)
    const double *jrec;       // JRec<K>
    const double *xrec;       // XRec<K> (closed-form cross terms)
    const int *pcell_start;   // schedule ELEM: CSR of the points sorted by row-major binning cell
    int split;                // warps per point tile (1, 2, 4): the tile's candidate rows are split
    const double4 *bbox;
    const int *cell_start;
    const double *kc;
    double x0, y0, Lx, Ly, inv_h, hw;
    double cw, chh, ex, ey;
    int ncx, ncy, periodic;
    unsigned long long *cnt;  // candidates, pairs, pieces, subtris, corner, cross, cross_subtris, cross_polys
    // one-sided kernels (template OS; reading R4): axes, h, the domain's upper corner,
    // B-spline pieces (piece-major (K+1)^2), their leading-coefficient jumps beta_e (e = 0..K+1)
    // and the inverse moment matrix ((2K+1)^2): c(lambda) = osa . (-lambda)^m
    int os_axes;
    double h, x1d, y1d;
    double osp[25], osb[6], osa[81];
};

__device__ __forceinline__ double2 ld2(const double *p) { return __ldg(reinterpret_cast<const double2 *>(p)); }
// SM = true: p points into shared memory (a TMA-staged record), else global (read-only path)
template <bool SM> __device__ __forceinline__ double2 ldr2(const double *p) {
    if constexpr (SM) return *reinterpret_cast<const double2 *>(p);
    else return ld2(p);
}

// ------------------------------------------------------------------ mbarrier + bulk copy (PTX)
__device__ __forceinline__ unsigned su32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mb_init(unsigned long long *b, int n) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(b)), "r"(n) : "memory");
}
// one thread: arm the barrier with the byte count and start the copy (1D TMA, 16 B granules)
__device__ __forceinline__ void bulk_load(void *dst, const void *src, unsigned bytes, unsigned long long *b) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(su32(dst)), "l"(src), "r"(bytes), "r"(su32(b)) : "memory");
}
__device__ __forceinline__ void mb_wait(unsigned long long *b, unsigned parity) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@!P1 bra WAIT_%=;\n"
        "}\n" ::"r"(su32(b)), "r"(parity)
        : "memory");
}

struct Cut {
    bool cut;      // a knot lies strictly inside the triangle's range on this axis
    bool multi;    // (GEN only) two or more knots inside: the pair takes the general path
    int row;       // row of the base cell in the padded cell table (0 = zero polynomial)
    int m;         // knot index (0..NC) if cut
    int side;      // 0: corner on the high side (apex = max vertex), 1: low side
    double e;      // zeta offset of the base cell: tau = zeta + e (tau = cell-centred kernel variable)
    double X;      // knot position in the zeta frame
    double lam;    // homothety ratio of the corner
};

// Cut structure of one axis for a pair; dd = (centroid + image shift - x)/h - T0 on this axis
// (the triangle's range is (zlo + dd, zhi + dd) in knot-index units, knots at 0..NC).
// GEN = false: the launcher guarantees every triangle extent is <= h (the paper's h = longest
// edge), so the range holds at most one knot strictly inside; it is the integer nearest the
// range's centre (two knots can appear inside only by rounding when an extent equals h, one
// within rounding of each end: either choice drops a sliver that is empty to rounding).  The
// base cell is the one below the knot when the knot is above the middle vertex (corner on the
// high side), else the one above; with no knot inside, the cell holding the range.
template <int K, bool GEN>
__device__ __forceinline__ Cut axis_cut_r(double2 lh, double2 mz, double2 iv, double dd) {
    constexpr int NC = 3 * K + 1;
    const double lo = lh.x + dd, hi = lh.y + dd;
    Cut c;
    c.multi = false;
    if (GEN) {
        const double fl = floor(lo);
        const double mk = fmax(fl + 1.0, 0.0);                  // first real knot above lo
        c.multi = mk + 1.0 < hi && mk + 1.0 <= (double)NC;
        c.cut = mk < hi && mk <= (double)NC;
        c.X = mk - dd;
        const bool hi_side = c.X > mz.x;
        c.side = hi_side ? 0 : 1;
        const double base = c.cut ? (hi_side ? mk - 1.0 : mk) : fl;
        c.row = (base < 0.0 || base >= (double)NC) ? 0 : (int)base + 1;
        c.m = (int)mk;
        c.e = (dd - 0.5) - base;
        c.lam = hi_side ? (hi - mk) * iv.y : (mk - lo) * iv.x;
        return c;
    }
    const double mk = floor(mz.y + dd);                         // knot nearest the range centre
    const int im = (int)mk;
    c.cut = mk > lo && mk < hi && (unsigned)im <= (unsigned)NC;
    c.X = mk - dd;
    const bool hs = c.X > mz.x;
    c.side = hs ? 0 : 1;
    const bool below = c.cut ? hs : mk >= hi;                   // base cell = the one below the knot
    const int ib = below ? im - 1 : im;
    c.row = (unsigned)ib < (unsigned)NC ? ib + 1 : 0;
    c.m = im;
    c.e = (dd - 0.5) - (below ? mk - 1.0 : mk);
    c.lam = hs ? (hi - mk) * iv.y : (mk - lo) * iv.x;
    return c;
}
// the axis data (lo, hi | mid, c5 | invL, invR) read from ad (shared memory if SM)
template <int K, bool GEN, bool SM = false>
__device__ __forceinline__ Cut axis_cut(const double *ad, double dd) {
    return axis_cut_r<K, GEN>(ldr2<SM>(ad), ldr2<SM>(ad + 2), ldr2<SM>(ad + 4), dd);
}

// Taylor coefficients p_a (a = 0..K) of the base cell polynomial at tau = zeta + e, in powers of
// zeta.  kcp: padded cell table, row i+1 = cell i, rows 0 and NC+1 zero.
template <int K> __device__ __forceinline__ void taylor_shift(double *p, double e) {
#pragma unroll
    for (int i = 0; i < K; ++i)
#pragma unroll
        for (int j = K - 1; j >= i; --j) p[j] = fma(e, p[j + 1], p[j]);
}
template <int K>
__device__ __forceinline__ void base_taylor(const double *kcp, int row, double e, double *p) {
    if constexpr ((K & 1) == 1) {     // even row length: 16-byte aligned rows, paired loads
#pragma unroll
        for (int j = 0; j <= K; j += 2) {
            const double2 t = *reinterpret_cast<const double2 *>(kcp + row * (K + 1) + j);
            p[j] = t.x; p[j + 1] = t.y;
        }
    } else {
#pragma unroll
        for (int j = 0; j <= K; ++j) p[j] = kcp[row * (K + 1) + j];
    }
    taylor_shift<K>(p, e);
}

// One-sided kernels (SIAC_BOUNDARY_ONESIDED): the lane's kernel is Kt(t - lambda) with Kt on the
// symmetric knot grid and coefficients c(lambda) (cl = &c[axis][0][lane], stride 32).  Row
// `row` of its padded cell table (cell i = row - 1; rows 0 and NC+1 zero):
//     Kt on cell i = sum_d c_{i-d} piece_d            (piece_d of psi_{k+1}, cell-centred)
template <int K, int NPT = 32>
__device__ __forceinline__ void os_row(const JumpArgs &a, const double *cl, int row, double *p) {
#pragma unroll
    for (int j = 0; j <= K; ++j) p[j] = 0.0;
#pragma unroll
    for (int d = 0; d <= K; ++d) {
        const int g = row - 1 - d;
        const bool ok = g >= 0 && g <= 2 * K;
        const double cg = ok ? cl[(ok ? g : 0) * NPT] : 0.0;
#pragma unroll
        for (int j = 0; j <= K; ++j) p[j] = fma(cg, a.osp[d * (K + 1) + j], p[j]);
    }
}
// jump of Kt's leading coefficient across knot m: sum_e c_{m-e} beta_e
template <int K, int NPT = 32>
__device__ __forceinline__ double os_alpha(const JumpArgs &a, const double *cl, int m) {
    double s = 0.0;
#pragma unroll
    for (int e = 0; e <= K + 1; ++e) {
        const int g = m - e;
        const bool ok = g >= 0 && g <= 2 * K;
        s = fma(ok ? cl[(ok ? g : 0) * NPT] : 0.0, a.osb[e], s);
    }
    return s;
}

// Estrin evaluation of sum_i c[i] x^i (N coefficients): dependency depth log2(N) instead of N.
template <int N> __device__ __forceinline__ double estrin(const double *c, double x) {
    if constexpr (N == 1) {
        return c[0];
    } else {
        constexpr int M = (N + 1) / 2;
        double d[M];
#pragma unroll
        for (int i = 0; i < N / 2; ++i) d[i] = fma(c[2 * i + 1], x, c[2 * i]);
        if constexpr (N % 2 == 1) d[M - 1] = c[N - 1];
        return estrin<M>(d, x * x);
    }
}

// lambda^{K+2} sum_b c_b G_b(lambda), G_b of degree K + b (corner block of NGP doubles):
// w_j = sum_b c_b g_bj first (independent short chains), then one Estrin pass in lambda.
template <int K, bool SM = false>
__device__ __forceinline__ double corner_eval(const double *G, const double *c, double lam) {
    constexpr int NGP = JRec<K>::NGP;
    double g[NGP];
#pragma unroll
    for (int i = 0; i < NGP; i += 2) { const double2 v = ldr2<SM>(G + i); g[i] = v.x; g[i + 1] = v.y; }
    double w[2 * K + 1];
#pragma unroll
    for (int j = 0; j <= 2 * K; ++j) {
        double t = 0.0;
#pragma unroll
        for (int b = K; b >= 0; --b)
            if (j <= K + b) t = fma(c[b], g[g_off(K, b) + j], t);
        w[j] = t;
    }
    const double v = estrin<2 * K + 1>(w, lam);
    const double l2 = lam * lam;
    double lp = (K & 1) ? l2 * lam : l2;            // lambda^{K+2} by squaring
    double sq = l2;
#pragma unroll
    for (int r = K / 2; r > 0; r >>= 1) {
        if (r & 1) lp *= sq;
        sq *= sq;
    }
    return lp * v;
}

// \int over triangle (p0, p1, p2) of (z1 - X)^K (z2 - Y)^K u(z), rule exact for degree 3K
template <int K>
__device__ __forceinline__ double integrate_cross(double p0x, double p0y, double p1x, double p1y, double p2x,
                                                  double p2y, double X, double Y, const double *mp,
                                                  const double *d) {
    const double e1x = p1x - p0x, e1y = p1y - p0y, e2x = p2x - p0x, e2y = p2y - p0y;
    const double area = 0.5 * fabs(e1x * e2y - e1y * e2x);
    const double tx0 = p0x - X, ty0 = p0y - Y;
    const double r0 = fma(mp[0], p0x, fma(mp[1], p0y, mp[4]));
    const double rr = fma(mp[0], e1x, mp[1] * e1y), rs = fma(mp[0], e2x, mp[1] * e2y);
    const double s0 = fma(mp[2], p0x, fma(mp[3], p0y, mp[5]));
    const double sr = fma(mp[2], e1x, mp[3] * e1y), ss = fma(mp[2], e2x, mp[3] * e2y);
    double acc = 0.0;
#pragma unroll
    for (int q = 0; q < Rule<K>::NQ; ++q) {
        const double r = qr<K>(q), s = qs<K>(q);
        const double tx = fma(e2x, s, fma(e1x, r, tx0));
        const double ty = fma(e2y, s, fma(e1y, r, ty0));
        const double rho = fma(rs, s, fma(rr, r, r0));
        const double sig = fma(ss, s, fma(sr, r, s0));
        const double t = tx * ty;
        double tp = t;
#pragma unroll
        for (int i = 1; i < K; ++i) tp *= t;
        acc = fma(qw<K>(q), tp * horner2<K>(d, rho, sig), acc);
    }
    return area * acc;
}

// Clip-and-integrate path for a pair with two or more knots inside an axis range (only when h is
// smaller than the triangle): SH pieces + fan + quadrature (siac_device.cuh).  Out of line so its
// polygon buffers do not burden the hot loop's registers.
struct GenOut {
    double v;
    unsigned pieces, subtris;
};
template <int K, bool COUNT>
__device__ __noinline__ GenOut general_pair(const double *__restrict__ rec, const double *kcp, int tri, double rsx,
                                            double rsy, double x1, double x2, double inv_h,
                                            const double *kcpy = nullptr) {
    const double *rc = rec + (int64_t)Rec<K>::RS * tri;
    double zx[3], zy[3];
#pragma unroll
    for (int v = 0; v < 3; ++v) {
        zx[v] = ((__ldg(rc + 2 * v) + rsx) - x1) * inv_h;
        zy[v] = ((__ldg(rc + 2 * v + 1) + rsy) - x2) * inv_h;
    }
    PairGeom g;
    g.M00 = __ldg(rc + 6); g.M01 = __ldg(rc + 7); g.M10 = __ldg(rc + 8); g.M11 = __ldg(rc + 9);
    g.zv0x = zx[0]; g.zv0y = zy[0];
    double d[Rec<K>::NB];
#pragma unroll
    for (int m = 0; m < Rec<K>::NB; ++m) d[m] = __ldg(rc + Rec<K>::OFF_D + m);
    Counts cn = {0, 0, 0};
    GenOut o;
    o.v = pair_contrib<K, COUNT>(zx, zy, kcp + (K + 1), d, g, cn, kcpy ? kcpy + (K + 1) : nullptr);
    o.pieces = (unsigned)cn.pieces;
    o.subtris = (unsigned)cn.subtris;
    return o;
}

__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

__device__ __forceinline__ int warp_excl_scan(int v, int lane, int &total) {
    int s = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(0xffffffffu, s, o);
        if (lane >= o) s += t;
    }
    total = __shfl_sync(0xffffffffu, s, 31);
    return s - v;
}

// Sum v over lanes with equal key (keys >= 32 ignored), in lane order, into S.acc[key].
template <class SM_>
__device__ __forceinline__ void seg_add(SM_ &S, int key, double v, int lane) {
    const unsigned grp = __match_any_sync(0xffffffffu, key);
    const int leader = __ffs(grp) - 1;
    double sum = (lane == leader) ? v : 0.0;
    unsigned rest = grp & ~(1u << leader);
    while (__any_sync(0xffffffffu, rest != 0)) {
        const int src = rest ? __ffs(rest) - 1 : lane;
        const double w = __shfl_sync(0xffffffffu, v, src);
        if (rest) { if (lane == leader) sum += w; rest &= rest - 1; }
    }
    if (lane == leader && key < (int)(sizeof(S.acc) / sizeof(S.acc[0]))) S.acc[key] += sum;
    __syncwarp();
}

template <class T> __device__ __forceinline__ T pick3(int a, T v0, T v1, T v2) {
    return a == 0 ? v0 : (a == 1 ? v1 : v2);
}

// Clip the top `take` queued cross terms (one per lane): corner_x = the homothetic corner of the
// x knot (apex A, P1 on A-Mv, P2 on A-C'), Sutherland-Hodgman-clipped (Alg. 1) by z2 = Y on the
// y corner's side -- a triangle, a quadrilateral (two fan triangles) or nothing; the fan
// sub-triangles are appended, compacted, to the staging buffer.
template <int K, bool COUNT>
__device__ __forceinline__ void clip_stage(const JumpArgs &a, WarpSmem &S, const double *kcp, const double *alpha,
                                           int &nq, int &ns, int lane, unsigned long long &c_xsub) {
    using J = JRec<K>;
    const int take = min(nq, 32);
    int nsub = 0;
    int ckey = 32 + lane;
    double cval = 0.0;
    double ax_ = 0, ay_ = 0, bx_ = 0, by_ = 0, cx_ = 0, cy_ = 0, dx_ = 0, dy_ = 0;
    int tri = 0, info = 0;
    double X = 0, Y = 0;
    if (lane < take) {
        const int e = nq - 1 - lane;
        tri = S.qtri[e];
        info = S.qinfo[e];
        X = S.qX[e];
        Y = S.qY[e];
        const int sx = (info >> 5) & 1, sy = (info >> 6) & 1;
        const double *jr = a.jrec + (int64_t)J::RS * tri;
        const double2 lh = ld2(jr + J::OFF_AX), iv = ld2(jr + J::OFF_AX + 4);
        const double lam = sx == 0 ? (lh.y - X) * iv.y : (X - lh.x) * iv.x;
        // the pair's y-corner term, deferred from the hot loop (it evaluates one corner per lane)
        {
            const int my = (info >> 12) & 31, rowx = (info >> 17) & 31;
            double pc[K + 1];
            base_taylor<K>(kcp, rowx, S.qE[e], pc);
            const double ay = sy == 0 ? alpha[my] : -alpha[my];
            cval = ay * corner_eval<K>(jr + J::OFF_G + (2 + sy) * J::NGP, pc, S.qL[e]);
            ckey = info & 31;
        }
        const double *geo = jr + J::OFF_GEO;
        const double2 A = ld2(geo + (sx == 0 ? 4 : 0)), M = ld2(geo + 2), Cp = ld2(geo + 6);
        const double v0x = A.x, v0y = A.y;
        const double v1x = fma(lam, M.x - A.x, A.x), v1y = fma(lam, M.y - A.y, A.y);
        const double v2x = fma(lam, Cp.x - A.x, A.x), v2y = fma(lam, Cp.y - A.y, A.y);
        const double sg = sy == 0 ? 1.0 : -1.0;
        const bool k0 = sg * (v0y - Y) >= 0.0, k1 = sg * (v1y - Y) >= 0.0, k2 = sg * (v2y - Y) >= 0.0;
        const int nk = (int)k0 + (int)k1 + (int)k2;
        if (nk == 3) {
            nsub = 1;
            ax_ = v0x; ay_ = v0y; bx_ = v1x; by_ = v1y; cx_ = v2x; cy_ = v2y;
        } else if (nk != 0) {
            // o = the vertex alone on its side (kept if nk == 1, dropped if nk == 2)
            const bool want = nk == 1;
            const int o = (k0 == want) ? 0 : ((k1 == want) ? 1 : 2);
            const int n1 = o == 2 ? 0 : o + 1, n2 = o == 0 ? 2 : o - 1;
            const double ox = pick3(o, v0x, v1x, v2x), oy = pick3(o, v0y, v1y, v2y);
            const double n1x = pick3(n1, v0x, v1x, v2x), n1y = pick3(n1, v0y, v1y, v2y);
            const double n2x = pick3(n2, v0x, v1x, v2x), n2y = pick3(n2, v0y, v1y, v2y);
            const double i1x = fma((Y - oy) / (n1y - oy), n1x - ox, ox);    // on edge o - n1
            const double i2x = fma((Y - oy) / (n2y - oy), n2x - ox, ox);    // on edge o - n2
            if (want) {
                nsub = 1;
                ax_ = ox; ay_ = oy; bx_ = i1x; by_ = Y; cx_ = i2x; cy_ = Y;
            } else {
                nsub = 2;        // quad n1, n2, I2, I1 -> (n1, n2, I2) + (n1, I2, I1)
                ax_ = n1x; ay_ = n1y; bx_ = n2x; by_ = n2y; cx_ = i2x; cy_ = Y; dx_ = i1x; dy_ = Y;
            }
        }
    }
    int total;
    const int off = ns + warp_excl_scan(nsub, lane, total);
    if (nsub >= 1) {
        S.s0x[off] = ax_; S.s0y[off] = ay_; S.s1x[off] = bx_; S.s1y[off] = by_; S.s2x[off] = cx_; S.s2y[off] = cy_;
        S.sX[off] = X; S.sY[off] = Y; S.stri[off] = tri; S.sinfo[off] = info;
    }
    if (nsub == 2) {
        S.s0x[off + 1] = ax_; S.s0y[off + 1] = ay_; S.s1x[off + 1] = cx_; S.s1y[off + 1] = cy_;
        S.s2x[off + 1] = dx_; S.s2y[off + 1] = dy_;
        S.sX[off + 1] = X; S.sY[off + 1] = Y; S.stri[off + 1] = tri; S.sinfo[off + 1] = info;
    }
    nq -= take;
    ns += total;
    if (COUNT) c_xsub += (lane == 0) ? total : 0;
    __syncwarp();
    seg_add(S, ckey, cval, lane);
}

// Integrate the top min(ns, 32) staged cross sub-triangles (one per lane) and add them, times
// sgn_x alpha_mx sgn_y alpha_my, to their points' accumulators.
template <int K>
__device__ __forceinline__ void integrate_stage(const JumpArgs &a, WarpSmem &S, const double *alpha, int &ns,
                                                int lane) {
    using J = JRec<K>;
    const int take = min(ns, 32);
    int key = 32 + lane;
    double v = 0.0;
    if (lane < take) {
        const int e = ns - 1 - lane;
        const int tri = S.stri[e], info = S.sinfo[e];
        key = info & 31;
        const int sx = (info >> 5) & 1, sy = (info >> 6) & 1, mx = (info >> 7) & 31, my = (info >> 12) & 31;
        const double *jr = a.jrec + (int64_t)J::RS * tri;
        double mp[6], d[J::NB];
#pragma unroll
        for (int i = 0; i < 6; i += 2) { const double2 t = ld2(jr + J::OFF_MAP + i); mp[i] = t.x; mp[i + 1] = t.y; }
#pragma unroll
        for (int i = 0; i < J::NB; ++i) d[i] = __ldg(jr + J::OFF_D + i);
        v = integrate_cross<K>(S.s0x[e], S.s0y[e], S.s1x[e], S.s1y[e], S.s2x[e], S.s2y[e], S.sX[e], S.sY[e], mp, d);
        const double cxf = sx == 0 ? alpha[mx] : -alpha[mx];
        const double cyf = sy == 0 ? alpha[my] : -alpha[my];
        v *= cxf * cyf;
    }
    ns -= take;
    __syncwarp();
    seg_add(S, key, v, lane);
}

// sum_{j<NS, i<NL} m[j NLP + i] mu^i s^j: NS independent Horner chains in mu, then Estrin in s
template <int NL, int NLP, int NS>
__device__ __forceinline__ double mono2d(const double *m, double mu, double s) {
    double col[NS];
#pragma unroll
    for (int j = 0; j < NS; ++j) {
        double c[NLP];
#pragma unroll
        for (int i = 0; i < NLP; i += 2) { const double2 t = ld2(m + j * NLP + i); c[i] = t.x; c[i + 1] = t.y; }
        double v = c[NL - 1];
#pragma unroll
        for (int i = NL - 2; i >= 0; --i) v = fma(v, mu, c[i]);
        col[j] = v;
    }
    return estrin<NS>(col, s);
}

// Binomial coefficients of (zeta2 - Y)^K in powers of zeta2: cy[b] = C(K, b) (-Y)^(K-b).
template <int K> __device__ __forceinline__ void ypow_coeffs(double Y, double *cy) {
    double pw = 1.0;
#pragma unroll
    for (int b = K; b >= 0; --b) {
        double bin = 1.0;
#pragma unroll
        for (int r = 0; r < K - b; ++r) bin = bin * (double)(K - r) / (double)(r + 1);
        cy[b] = bin * pw;
        pw *= -Y;
    }
}

// lambda^{2K+2} F_dir(lambda, Y') on interval iv of the x corner of side sx: the y knot Y' in
// the reference corner's frame, s its position in the interval, dir = sy (0 above, 1 below).
template <int K>
__device__ __forceinline__ double cross_poly(const double *xb, double Ay, double lam, double Y, int iv, int dir) {
    using X = XRec<K>;
    const double Yp = fma(Y - Ay, 1.0 / lam, Ay);
    const double va = __ldg(xb + iv), iw = __ldg(xb + 3 + iv);
    const double sv = fma(2.0 * (Yp - va), iw, -1.0);
    double l2k = lam * lam;
#pragma unroll
    for (int i = 0; i < K; ++i) l2k *= lam * lam;
    return l2k * mono2d<X::NL, X::NLP, X::NS>(xb + X::poly(iv, dir), 2.0 * lam - 1.0, sv);
}

// Classification of a cross term (the y knot Y against the x corner of side sx, homothety lam):
// 0 = the line misses the corner on the far side (I11 = 0), 1 = it misses it on the near side
// (I11 = the whole corner), 2 = it cuts interval 0, 3 = it cuts interval 1.  xh: the record's
// (Ay, v0, v1, v2) of that side; the test Y' <> v is written as (Y - Ay) <> lam (v - Ay), lam > 0.
__device__ __forceinline__ int cross_class(const double *xh, double lam, double Y, int sy) {
    const double d = Y - xh[0];
    const bool below_all = d <= lam * (xh[1] - xh[0]);      // Y' <= v0: the line under the corner
    const bool above_all = d >= lam * (xh[3] - xh[0]);      // Y' >= v2
    if (!below_all && !above_all) return d < lam * (xh[2] - xh[0]) ? 2 : 3;
    return (sy == 0 ? below_all : above_all) ? 1 : 0;
}

// I11 / (sgn alpha_x sgn alpha_y) of one pair, evaluated inline (per-element schedule): the
// x corner of side sx with homothety ratio lam, the y knot Y (zeta frame), the y corner on side
// sy; xb = the triangle's XRec block of side sx.  poly: evaluated by an interval polynomial.
template <int K>
__device__ __forceinline__ double cross_I11(const double *jr, const double *xb, double lam, double Y, int sx, int sy,
                                            bool &poly) {
    using J = JRec<K>;
    double xh[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) xh[i] = __ldg(jr + J::OFF_XH + 4 * sx + i);
    const int cls = cross_class(xh, lam, Y, sy);
    poly = cls >= 2;
    if (cls >= 2) return cross_poly<K>(xb, xh[0], lam, Y, cls - 2, sy);
    if (cls == 0) return 0.0;
    double cy[K + 1];
    ypow_coeffs<K>(Y, cy);
    return corner_eval<K>(jr + J::OFF_G + sx * J::NGP, cy, lam);
}

// Evaluate the top min(nq, 32) entries of queue Q (one per lane): the deferred y-corner term
// plus sgn alpha_x sgn alpha_y I11, POLY = true: interval polynomials (qp), else whole corner
// or 0 (qf); added to the owners' accumulators.
template <int K, bool COUNT, bool OS, bool POLY, class SM_, int NPT = 32>
__device__ __forceinline__ void cross_stage(const JumpArgs &a, SM_ &S, XQueue &Q, const double *kcp,
                                            const double *alpha, int &nq, int lane, unsigned long long &c_poly,
                                            const OsSmem<K, NPT> *osm) {
    using J = JRec<K>;
    using X = XRec<K>;
    const int take = min(nq, 32);
    int key = NPT + lane;                       // (>= the number of points: ignored by seg_add)
    double val = 0.0;
    if (lane < take) {
        const int e = nq - 1 - lane;
        const int tri = Q.tri[e], info = Q.info[e];
        const double Y = Q.Y[e], lam = Q.lam[e];
        key = info & 63;
        const int sx = (info >> 6) & 1, sy = (info >> 7) & 1, mx = (info >> 8) & 31, my = (info >> 13) & 31;
        const int rowx = (info >> 18) & 31, iv = (info >> 23) & 1, full = (info >> 24) & 1;
        const double *jr = a.jrec + (int64_t)J::RS * tri;
        double ay, ax, pc[K + 1];
        if constexpr (OS) {          // the owner point's one-sided kernels
            const int ol = info & 63;
            const double amy = os_alpha<K, NPT>(a, &osm->c[1][0][ol], my);
            const double amx = os_alpha<K, NPT>(a, &osm->c[0][0][ol], mx);
            ay = sy == 0 ? amy : -amy;
            ax = sx == 0 ? amx : -amx;
            os_row<K, NPT>(a, &osm->c[0][0][ol], rowx, pc);
            taylor_shift<K>(pc, Q.E[e]);
        } else {
            ay = sy == 0 ? alpha[my] : -alpha[my];
            ax = sx == 0 ? alpha[mx] : -alpha[mx];
            base_taylor<K>(kcp, rowx, Q.E[e], pc);       // (for the deferred y-corner term)
        }
        const double ycorner = ay * corner_eval<K>(jr + J::OFF_G + (2 + sy) * J::NGP, pc, Q.L[e]);
        double I11 = 0.0;
        if constexpr (POLY) {
            const double Ay = __ldg(jr + J::OFF_XH + 4 * sx);
            I11 = cross_poly<K>(a.xrec + (int64_t)X::RS * tri + sx * X::XB, Ay, lam, Y, iv, sy);
            if (COUNT) ++c_poly;
        } else if (full) {
            double cy[K + 1];
            ypow_coeffs<K>(Y, cy);
            I11 = corner_eval<K>(jr + J::OFF_G + sx * J::NGP, cy, lam);
        }
        val = fma(ax * ay, I11, ycorner);
    }
    nq -= take;
    __syncwarp();
    seg_add(S, key, val, lane);
}

#ifndef SIAC_JUMPX_MINB
// 5 blocks/SM (102 registers, small spills) for the default schedule: A/B on one box, 2 reps
// (profiles/r02g_ab_2d_minb5.txt): cfg 5 349.8 vs 354.4 ms, cfg 4 61.1 vs 62.0 ms, cfg 3 12.97
// vs 12.6 ms -- the large problems gain, the small graded one loses a little
#define SIAC_JUMPX_MINB 5
#endif
// OS (one-sided kernels near non-periodic boundaries, with XP only): every lane evaluates its own
// kernel Kt(. - lambda) at the effective point x + lambda h; cell rows and knot jumps are built
// from the lane's coefficients (os_row / os_alpha) instead of the shared table.
template <int K, bool COUNT, bool GEN, bool XP, bool OS = false>
__global__ void __launch_bounds__(WARPS * 32, XP ? SIAC_JUMPX_MINB : SIAC_JUMP_MINB) k_eval_jump(JumpArgs a) {
    static_assert(!OS || XP, "one-sided kernels are implemented for the closed-form cross terms (JUMPX)");
    using J = JRec<K>;
    constexpr int NC = 3 * K + 1;
    __shared__ __align__(16) double kcp[(NC + 2) * (K + 1)];
    __shared__ double alpha[NC + 1];
    extern __shared__ __align__(16) unsigned char jump_dsm[];
    using WS = WarpSmemFor<XP>;
    WS *wsm = reinterpret_cast<WS *>(jump_dsm);
    for (int i = threadIdx.x; i < (NC + 2) * (K + 1); i += blockDim.x) {
        const int row = i / (K + 1);
        kcp[i] = (row == 0 || row == NC + 1) ? 0.0 : a.kc[i - (K + 1)];
    }
    __syncthreads();
    for (int m = threadIdx.x; m <= NC; m += blockDim.x) alpha[m] = kcp[(m + 1) * (K + 1) + K] - kcp[m * (K + 1) + K];
    __syncthreads();

    const int lane = threadIdx.x & 31;
    const int wid = threadIdx.x >> 5;
    WS &S = wsm[wid];
    WarpStage<K> &T = reinterpret_cast<WarpStage<K> *>(wsm + WARPS)[wid];
    OsSmem<K> *osm = OS ? reinterpret_cast<OsSmem<K> *>(reinterpret_cast<WarpStage<K> *>(wsm + WARPS) + WARPS) + wid
                        : nullptr;
    // a.split warps share one tile (small problems: more warps than tiles), each walking a
    // contiguous share of its candidate rows; partial sums are combined in a fixed order
    const int split = a.split;
    const int part = wid % split;
    const int64_t p0 = ((int64_t)blockIdx.x * (WARPS / split) + wid / split) * 32;
    const bool live = p0 < a.np;
    if (split == 1 && !live) return;              // warp-uniform
    if (lane == 0) {
        for (int i = 0; i < NST; ++i) mb_init(&T.bar[i], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    int g = 0;                                    // records streamed so far (ring position)
    unsigned ph = 0;                              // per-slot phase parity
    const bool valid = live && p0 + lane < a.np;
    const int nvalid = __popc(__ballot_sync(0xffffffffu, valid));
    int orig = -1;
    double x1 = 0, x2 = 0;
    if (valid) {
        orig = a.perm[p0 + lane];
        x1 = a.pts[2 * (int64_t)orig];
        x2 = a.pts[2 * (int64_t)orig + 1];
        if (a.periodic & 1) { x1 = x1 - a.Lx * floor((x1 - a.x0) / a.Lx); if (x1 >= a.x0 + a.Lx) x1 -= a.Lx; if (x1 < a.x0) x1 = a.x0; }
        if (a.periodic & 2) { x2 = x2 - a.Ly * floor((x2 - a.y0) / a.Ly); if (x2 >= a.y0 + a.Ly) x2 -= a.Ly; if (x2 < a.y0) x2 = a.y0; }
    }
    if constexpr (OS) {
        // node shift lambda = the smallest |lambda| keeping x + h[-H + lambda, H + lambda] in the
        // domain (0 in the interior); c(lambda) = osa . (-lambda)^m; then the effective point
        constexpr double H = 0.5 * (3 * K + 1);
        double lam[2] = {0.0, 0.0};
        if (valid && (a.os_axes & 1)) lam[0] = fmax(0.0, H - (x1 - a.x0) / a.h) + fmin(0.0, (a.x1d - x1) / a.h - H);
        if (valid && (a.os_axes & 2)) lam[1] = fmax(0.0, H - (x2 - a.y0) / a.h) + fmin(0.0, (a.y1d - x2) / a.h - H);
#pragma unroll
        for (int ax = 0; ax < 2; ++ax) {
            double b[2 * K + 1];
            b[0] = 1.0;
#pragma unroll
            for (int m = 1; m <= 2 * K; ++m) b[m] = -lam[ax] * b[m - 1];
#pragma unroll
            for (int g2 = 0; g2 <= 2 * K; ++g2) {
                double c = 0.0;
#pragma unroll
                for (int m = 2 * K; m >= 0; --m) c = fma(a.osa[g2 * (2 * K + 1) + m], b[m], c);
                osm->c[ax][g2][lane] = c;
            }
        }
        x1 = fma(lam[0], a.h, x1);
        x2 = fma(lam[1], a.h, x2);
        __syncwarp();
    }
    S.acc[lane] = 0.0;
    double tx0 = valid ? x1 : 1e300, tx1 = valid ? x1 : -1e300, ty0 = valid ? x2 : 1e300, ty1 = valid ? x2 : -1e300;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        tx0 = fmin(tx0, __shfl_xor_sync(0xffffffffu, tx0, o));
        tx1 = fmax(tx1, __shfl_xor_sync(0xffffffffu, tx1, o));
        ty0 = fmin(ty0, __shfl_xor_sync(0xffffffffu, ty0, o));
        ty1 = fmax(ty1, __shfl_xor_sync(0xffffffffu, ty1, o));
    }
    const double sx0 = x1 - a.hw, sx1 = x1 + a.hw, sy0 = x2 - a.hw, sy1 = x2 + a.hw;     // own stencil
    const double bx0 = tx0 - a.hw, bx1 = tx1 + a.hw, by0 = ty0 - a.hw, by1 = ty1 + a.hw;  // tile's stencils
    int R0 = (int)floor((by0 - a.ey - a.y0) / a.chh) - 1, R1 = (int)floor((by1 - a.y0) / a.chh) + 1;
    int C0 = (int)floor((bx0 - a.ex - a.x0) / a.cw) - 1, C1 = (int)floor((bx1 - a.x0) / a.cw) + 1;
    if (!(a.periodic & 2)) { R0 = max(R0, 0); R1 = min(R1, a.ncy - 1); }
    if (!(a.periodic & 1)) { C0 = max(C0, 0); C1 = min(C1, a.ncx - 1); }
    if (!live) {
        R0 = 0; R1 = -1;                          // idle warp of a split block: empty walk
    } else if (split > 1) {
        const int nr = R1 - R0 + 1;
        const int r_lo = R0 + (nr * part) / split, r_hi = R0 + (nr * (part + 1)) / split - 1;
        R0 = r_lo; R1 = r_hi;
    }
    __syncwarp();

    double acc = 0.0;
    int nq = 0, ns = 0;       // JUMP: cross-term queue, staged sub-triangles
    int nqp = 0, nqf = 0;     // JUMPX: poly / full cross-term queues
    bool general = false;     // this lane met a pair with several knots on an axis

    unsigned long long c_cand = 0, c_pairs = 0, c_pieces = 0, c_sub = 0, c_corner = 0, c_cross = 0, c_xsub = 0,
                       c_xpoly = 0;
    // Warp-uniform walk over the candidate triangles of the tile: binning-cell row runs of the
    // tile's stencil bounds (Eq. (3)-style, periodic images unwrapped), 32 boxes tested per step,
    // then body(tri, rsx, rsy, hit, hr) for every candidate whose box meets the tile's stencils
    // (stg = true: only those some lane's stencil meets, hr = the record's hot part in shared
    // memory; else hr = nullptr).
    auto candidates = [&](auto stg, auto &&body) {
        for (int R = R0; R <= R1; ++R) {
            int r = R, qy = 0;
            if (a.periodic & 2) { r = ((R % a.ncy) + a.ncy) % a.ncy; qy = (R - r) / a.ncy; }
            const double rsy = qy * a.Ly;
            int C = C0;
            while (C <= C1) {
                int c = C, qx = 0;
                if (a.periodic & 1) { c = ((C % a.ncx) + a.ncx) % a.ncx; qx = (C - c) / a.ncx; }
                const int cend = (a.periodic & 1) ? min(C1, (qx + 1) * a.ncx - 1) : C1;
                const double rsx = qx * a.Lx;
                const int cb = c + (cend - C);
                int t_cur = __ldg(a.cell_start + r * a.ncx + c);
                const int t_end = __ldg(a.cell_start + r * a.ncx + cb + 1);
                C = cend + 1;
                for (; t_cur < t_end; t_cur += 32) {
                    const int n = min(32, t_end - t_cur);
                    bool keep = false;
                    if (lane < n) {
                        double4 b = a.bbox[t_cur + lane];
                        b.x += rsx; b.z += rsx; b.y += rsy; b.w += rsy;
                        S.cbox[lane] = b;
                        keep = (b.x < bx1 && b.z > bx0 && b.y < by1 && b.w > by0);
                    }
                    const unsigned mask = __ballot_sync(0xffffffffu, keep);
                    if (keep) S.klist[__popc(mask & lanemask_lt())] = lane;
                    const int nk = __popc(mask);
                    __syncwarp();
                    if constexpr (decltype(stg)::value) {
                        // exact per-lane stencil tests against the kept boxes; compact the
                        // candidates some lane meets, then stream their records through the ring
                        int nh = 0;
                        for (int i = 0; i < nk; ++i) {
                            const int j = S.klist[i];
                            const double4 b = S.cbox[j];
                            const bool hit = valid && (b.x < sx1 && b.z > sx0 && b.y < sy1 && b.w > sy0);
                            const unsigned hm = __ballot_sync(0xffffffffu, hit);
                            if (COUNT) { c_cand += nvalid; c_pairs += __popc(hm); }
                            if (hm) {
                                if (lane == 0) { T.hj[nh] = j; T.hm[nh] = hm; }
                                ++nh;
                            }
                        }
                        __syncwarp();
                        constexpr unsigned HB = J::OFF_GEO * 8;
                        if (lane == 0) {
                            for (int r = 0; r < min(NST, nh); ++r) {
                                const int sl = (g + r) & (NST - 1);
                                bulk_load(T.rec[sl], a.jrec + (int64_t)J::RS * (t_cur + T.hj[r]), HB, &T.bar[sl]);
                            }
                        }
                        for (int i = 0; i < nh; ++i) {
                            const int sl = (g + i) & (NST - 1);
                            mb_wait(&T.bar[sl], (ph >> sl) & 1u);
                            ph ^= 1u << sl;
                            body(t_cur + T.hj[i], rsx, rsy, ((T.hm[i] >> lane) & 1u) != 0, T.rec[sl]);
                            __syncwarp();
                            if (lane == 0 && i + NST < nh) {
                                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                                bulk_load(T.rec[sl], a.jrec + (int64_t)J::RS * (t_cur + T.hj[i + NST]), HB, &T.bar[sl]);
                            }
                        }
                        g += nh;
                    } else {
                        for (int i = 0; i < nk; ++i) {
                            const int j = S.klist[i];
                            const double4 b = S.cbox[j];
                            const bool hit = valid && (b.x < sx1 && b.z > sx0 && b.y < sy1 && b.w > sy0);
                            body(t_cur + j, rsx, rsy, hit, nullptr);
                        }
                    }
                    __syncwarp();
                }
            }
        }
    };

    // One pair = eval (pure arithmetic on the staged record) + commit (accumulate, queue the
    // cross term).  Every lane evaluates the closed form (no divergence); only lanes whose
    // stencil box meets the triangle's box add it (and queue its cross term): the four terms of a
    // pair cancel to rounding only together, so a pair is taken whole or not at all.
    struct PairV { double v; Cut cx, cy; bool skip; };
    auto pair_eval = [&](double rsx, double rsy, bool hit, const double *hr) -> PairV {
        PairV r;
        const double2 cen = ldr2<true>(hr);
        constexpr double MT0 = 0.5 * (3 * K + 1);      // -T0
        const double dx = fma((cen.x + rsx) - x1, a.inv_h, MT0);
        const double dy = fma((cen.y + rsy) - x2, a.inv_h, MT0);
        const Cut cx = axis_cut<K, GEN, true>(hr + J::OFF_AX, dx);
        const Cut cy = axis_cut<K, GEN, true>(hr + J::OFF_AX + 6, dy);
        bool skip = false;
        if (GEN && (cx.multi || cy.multi)) {
            skip = true;
            general = general || hit;     // integrated in the second pass below
        }
        double p[K + 1], q[K + 1];
        if constexpr (OS) {
            os_row<K>(a, &osm->c[0][0][lane], cx.row, p);
            taylor_shift<K>(p, cx.e);
            os_row<K>(a, &osm->c[1][0][lane], cy.row, q);
            taylor_shift<K>(q, cy.e);
        } else {
            base_taylor<K>(kcp, cx.row, cx.e, p);
            base_taylor<K>(kcp, cy.row, cy.e, q);
        }
        double mu[J::NMU + 1];
#pragma unroll
        for (int i = 0; i < J::NMU; i += 2) {
            const double2 t = ldr2<true>(hr + J::OFF_MU + i);
            mu[i] = t.x; mu[i + 1] = t.y;
        }
        double ve = 0.0, vo = 0.0;                       // two chains (even / odd a)
#pragma unroll
        for (int aa = K; aa >= 0; --aa) {
            double s = 0.0;
#pragma unroll
            for (int bb = K; bb >= 0; --bb) s = fma(q[bb], mu[aa * (K + 1) + bb], s);
            if (aa & 1) vo = fma(p[aa], s, vo);
            else ve = fma(p[aa], s, ve);
        }
        double v = ve + vo;
        // one corner per lane here: the x corner if x is cut, else the y corner; a lane with
        // both cut defers its y corner to the cross-term queue (clip_stage)
        const bool ux = cx.cut;
        const bool uy = !cx.cut && cy.cut;
        const int sdd = ux ? cx.side : cy.side;
        const int mm = ux ? cx.m : (uy ? cy.m : 0);              // uncut: lam = 0 zeroes the corner
        double am;
        if constexpr (OS) am = os_alpha<K>(a, &osm->c[ux ? 0 : 1][0][lane], mm);
        else am = alpha[mm];
        const int sd = ux ? sdd : 2 + sdd;
        const double sg = sdd == 0 ? am : -am;
        double cc[K + 1];
#pragma unroll
        for (int j = 0; j <= K; ++j) cc[j] = ux ? q[j] : p[j];
        const double lam = ux ? cx.lam : (uy ? cy.lam : 0.0);
        r.v = fma(sg, corner_eval<K, true>(hr + J::OFF_G + sd * J::NGP, cc, lam), v);
        r.cx = cx; r.cy = cy; r.skip = skip;
        return r;
    };
    auto pair_commit = [&](int tri, bool hit, const PairV &r, const double *hr) {
        const Cut &cx = r.cx, &cy = r.cy;
        if (hit && !r.skip) acc += r.v;
        const bool cross = hit && !r.skip && cx.cut && cy.cut;
        if (COUNT && hit && !r.skip) c_corner += (int)cx.cut + (int)cy.cut;
        const unsigned cm = __ballot_sync(0xffffffffu, cross);
        if constexpr (XP) {
            // classify each cross term against its x corner's heights (staged record) and
            // append it to the poly or the full queue
            if (cm) {
                int cls = 0;
                if (cross) {
                    const double2 h01 = ldr2<true>(hr + J::OFF_XH + 4 * cx.side);
                    const double2 h23 = ldr2<true>(hr + J::OFF_XH + 4 * cx.side + 2);
                    const double xh[4] = {h01.x, h01.y, h23.x, h23.y};
                    cls = cross_class(xh, cx.lam, cy.X, cy.side);
                }
                const bool isp = cross && cls >= 2;
                const unsigned pm = __ballot_sync(0xffffffffu, isp);
                const unsigned fm = cm & ~pm;
                if (cross) {
                    XQueue &Q = isp ? S.qp : S.qf;
                    const int pos = isp ? nqp + __popc(pm & lanemask_lt()) : nqf + __popc(fm & lanemask_lt());
                    Q.tri[pos] = tri;
                    Q.info[pos] = lane | (cx.side << 6) | (cy.side << 7) | (cx.m << 8) | (cy.m << 13) | (cx.row << 18) |
                                  ((cls == 3) << 23) | ((cls == 1) << 24);
                    Q.Y[pos] = cy.X;
                    Q.E[pos] = cx.e;
                    Q.L[pos] = cy.lam;
                    Q.lam[pos] = cx.lam;
                }
                nqp += __popc(pm);
                nqf += __popc(fm);
                if (COUNT) c_cross += __popc(cm) * (lane == 0);
                __syncwarp();
            }
        } else if (cm) {
            if (cross) {
                const int pos = nq + __popc(cm & lanemask_lt());
                S.qtri[pos] = tri;
                S.qinfo[pos] = lane | (cx.side << 5) | (cy.side << 6) | (cx.m << 7) | (cy.m << 12) | (cx.row << 17);
                S.qX[pos] = cx.X;
                S.qY[pos] = cy.X;
                S.qE[pos] = cx.e;
                S.qL[pos] = cy.lam;
            }
            nq += __popc(cm);
            if (COUNT) c_cross += __popc(cm) * (lane == 0);
            __syncwarp();
        }
    };
    auto flush = [&]() {        // evaluate queued cross terms 32 at a time (warp-uniform counts)
        if constexpr (XP) {
            while (nqp >= 32) cross_stage<K, COUNT, OS, true>(a, S, S.qp, kcp, alpha, nqp, lane, c_xpoly, osm);
            while (nqf >= 32) cross_stage<K, COUNT, OS, false>(a, S, S.qf, kcp, alpha, nqf, lane, c_xpoly, osm);
        } else {
            while (nq >= 32) {
                clip_stage<K, COUNT>(a, S, kcp, alpha, nq, ns, lane, c_xsub);
                while (ns >= 32) integrate_stage<K>(a, S, alpha, ns, lane);
            }
        }
    };
    candidates(std::true_type{},
        [&](int tri, double rsx, double rsy, bool hit, const double *hr) {
            pair_commit(tri, hit, pair_eval(rsx, rsy, hit, hr), hr);
            flush();
        });
    if constexpr (XP) {
        while (nqp > 0) cross_stage<K, COUNT, OS, true>(a, S, S.qp, kcp, alpha, nqp, lane, c_xpoly, osm);
        while (nqf > 0) cross_stage<K, COUNT, OS, false>(a, S, S.qf, kcp, alpha, nqf, lane, c_xpoly, osm);
    } else {
        while (nq > 0) clip_stage<K, COUNT>(a, S, kcp, alpha, nq, ns, lane, c_xsub);
        while (ns > 0) integrate_stage<K>(a, S, alpha, ns, lane);
    }
    __syncwarp();
    // second pass, only for tiles that met pairs with several knots on an axis (h smaller than
    // the triangles): those pairs take the clip-and-integrate path, out of the hot loop
    if (GEN && __any_sync(0xffffffffu, general)) {
        candidates(std::false_type{}, [&](int tri, double rsx, double rsy, bool hit, const double *) {
            if (!hit) return;
            const double *jr = a.jrec + (int64_t)J::RS * tri;
            const double2 cen = ld2(jr);
            constexpr double MT0 = 0.5 * (3 * K + 1);
            const Cut cx = axis_cut<K, GEN>(jr + J::OFF_AX, fma((cen.x + rsx) - x1, a.inv_h, MT0));
            const Cut cy = axis_cut<K, GEN>(jr + J::OFF_AX + 6, fma((cen.y + rsy) - x2, a.inv_h, MT0));
            if (cx.multi || cy.multi) {
                GenOut go;
                if constexpr (OS) {        // the lane's two kernels as padded cell tables
                    double tx[(NC + 2) * (K + 1)], ty[(NC + 2) * (K + 1)];
                    for (int r = 0; r < NC + 2; ++r) {
                        os_row<K>(a, &osm->c[0][0][lane], r, tx + r * (K + 1));
                        os_row<K>(a, &osm->c[1][0][lane], r, ty + r * (K + 1));
                    }
                    go = general_pair<K, COUNT>(a.rec, tx, tri, rsx, rsy, x1, x2, a.inv_h, ty);
                } else {
                    go = general_pair<K, COUNT>(a.rec, kcp, tri, rsx, rsy, x1, x2, a.inv_h);
                }
                acc += go.v;
                if (COUNT) { c_pieces += go.pieces; c_sub += go.subtris; }
            }
        });
    }
    if (split == 1) {
        if (valid) a.out[orig] = acc + S.acc[lane];
    } else {
        __shared__ double psum[WARPS][32];
        psum[wid][lane] = acc + S.acc[lane];
        __syncthreads();
        if (part == 0 && valid) {
            double t = psum[wid][lane];
            for (int q = 1; q < split; ++q) t += psum[wid + q][lane];
            a.out[orig] = t;
        }
    }
    if (COUNT) {
        unsigned long long v[8] = {c_cand, c_pairs, c_pieces, c_sub, c_corner, c_cross, c_xsub, c_xpoly};
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            unsigned long long x = v[i];
            if (i == 2 || i == 3 || i == 4 || i == 7) {
                for (int o = 16; o > 0; o >>= 1) x += __shfl_down_sync(0xffffffffu, x, o);
            }
            if (lane == 0 && x) atomicAdd(a.cnt + i, x);
        }
    }
}


// ------------------------------------------------------------------ per-element schedule (ELEM)
// The paper's per-element method (Alg. 3; search bounds Eq. (3))
// on the same exact decomposition: one warp per triangle (cell order), its stencil-expanded
// bounding box walked over the point grid (row runs of the row-major point CSR, periodic images
// unwrapped), 32 candidate points per step (lane = point), the whole pair contribution --
// moments, both corner terms, the closed-form cross term -- evaluated from the one triangle's
// record (broadcast loads), and scattered to the point with one atomic add per pair (the
// paper's per-patch partial solutions + reduction, L636-652, become atomics; the summation
// order, hence the last bits, is not fixed).
template <int K, bool COUNT, bool GEN>
__global__ void __launch_bounds__(WARPS * 32) k_eval_elem(JumpArgs a, int64_t nt) {
    using J = JRec<K>;
    using X = XRec<K>;
    constexpr int NC = 3 * K + 1;
    __shared__ __align__(16) double kcp[(NC + 2) * (K + 1)];
    __shared__ double alpha[NC + 1];
    for (int i = threadIdx.x; i < (NC + 2) * (K + 1); i += blockDim.x) {
        const int row = i / (K + 1);
        kcp[i] = (row == 0 || row == NC + 1) ? 0.0 : a.kc[i - (K + 1)];
    }
    __syncthreads();
    for (int m = threadIdx.x; m <= NC; m += blockDim.x) alpha[m] = kcp[(m + 1) * (K + 1) + K] - kcp[m * (K + 1) + K];
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int64_t t = (int64_t)blockIdx.x * WARPS + (threadIdx.x >> 5);
    if (t >= nt) return;                           // warp-uniform
    const double *jr = a.jrec + (int64_t)J::RS * t;
    const double4 tb = a.bbox[t];
    // Eq. (3) per-element bounds: floor((min - w/2)/c_e) .. floor((max + w/2)/c_e)
    int C0 = (int)floor((tb.x - a.hw - a.x0) / a.cw), C1 = (int)floor((tb.z + a.hw - a.x0) / a.cw);
    int R0 = (int)floor((tb.y - a.hw - a.y0) / a.chh), R1 = (int)floor((tb.w + a.hw - a.y0) / a.chh);
    if (!(a.periodic & 2)) { R0 = max(R0, 0); R1 = min(R1, a.ncy - 1); }
    if (!(a.periodic & 1)) { C0 = max(C0, 0); C1 = min(C1, a.ncx - 1); }
    const double2 cen = ld2(jr);
    constexpr double MT0 = 0.5 * (3 * K + 1);
    unsigned long long c_cand = 0, c_pairs = 0, c_pieces = 0, c_sub = 0, c_corner = 0, c_cross = 0, c_poly = 0;
    for (int R = R0; R <= R1; ++R) {
        int r = R, qy = 0;
        if (a.periodic & 2) { r = ((R % a.ncy) + a.ncy) % a.ncy; qy = (R - r) / a.ncy; }
        const double rsy = -qy * a.Ly;          // triangle image relative to the wrapped points
        int C = C0;
        while (C <= C1) {
            int c = C, qx = 0;
            if (a.periodic & 1) { c = ((C % a.ncx) + a.ncx) % a.ncx; qx = (C - c) / a.ncx; }
            const int cend = (a.periodic & 1) ? min(C1, (qx + 1) * a.ncx - 1) : C1;
            const double rsx = -qx * a.Lx;
            const int p_beg = __ldg(a.pcell_start + r * a.ncx + c);
            const int p_end = __ldg(a.pcell_start + r * a.ncx + c + (cend - C) + 1);
            C = cend + 1;
            const double bx0 = tb.x + rsx, bx1 = tb.z + rsx, by0 = tb.y + rsy, by1 = tb.w + rsy;
            for (int p0 = p_beg; p0 < p_end; p0 += 32) {
                const int sp = p0 + lane;
                const bool valid = sp < p_end;
                int orig = 0;
                double x1 = 0.0, x2 = 0.0;
                if (valid) {
                    orig = a.perm[sp];
                    x1 = a.pts[2 * (int64_t)orig];
                    x2 = a.pts[2 * (int64_t)orig + 1];
                    if (a.periodic & 1) { x1 = x1 - a.Lx * floor((x1 - a.x0) / a.Lx); if (x1 >= a.x0 + a.Lx) x1 -= a.Lx; if (x1 < a.x0) x1 = a.x0; }
                    if (a.periodic & 2) { x2 = x2 - a.Ly * floor((x2 - a.y0) / a.Ly); if (x2 >= a.y0 + a.Ly) x2 -= a.Ly; if (x2 < a.y0) x2 = a.y0; }
                }
                const bool hit = valid && (bx0 < x1 + a.hw && bx1 > x1 - a.hw && by0 < x2 + a.hw && by1 > x2 - a.hw);
                if (COUNT) { c_cand += valid; c_pairs += hit; }
                if (!__any_sync(0xffffffffu, hit)) continue;
                const double dx = fma((cen.x + rsx) - x1, a.inv_h, MT0);
                const double dy = fma((cen.y + rsy) - x2, a.inv_h, MT0);
                const Cut cx = axis_cut<K, GEN>(jr + J::OFF_AX, dx);
                const Cut cy = axis_cut<K, GEN>(jr + J::OFF_AX + 6, dy);
                double v = 0.0;
                if (GEN && (cx.multi || cy.multi)) {
                    if (hit) {
                        const GenOut go = general_pair<K, COUNT>(a.rec, kcp, (int)t, rsx, rsy, x1, x2, a.inv_h);
                        v = go.v;
                        if (COUNT) { c_pieces += go.pieces; c_sub += go.subtris; }
                    }
                } else {
                    double p[K + 1], q[K + 1];
                    base_taylor<K>(kcp, cx.row, cx.e, p);
                    base_taylor<K>(kcp, cy.row, cy.e, q);
                    double ve = 0.0, vo = 0.0;
#pragma unroll
                    for (int aa = K; aa >= 0; --aa) {
                        double sacc = 0.0;
#pragma unroll
                        for (int bb = K; bb >= 0; --bb) sacc = fma(q[bb], __ldg(jr + J::OFF_MU + aa * (K + 1) + bb), sacc);
                        if (aa & 1) vo = fma(p[aa], sacc, vo);
                        else ve = fma(p[aa], sacc, ve);
                    }
                    v = ve + vo;
                    const double ax = cx.cut ? (cx.side == 0 ? alpha[cx.m] : -alpha[cx.m]) : 0.0;
                    const double ay = cy.cut ? (cy.side == 0 ? alpha[cy.m] : -alpha[cy.m]) : 0.0;
                    if (cx.cut) v = fma(ax, corner_eval<K>(jr + J::OFF_G + cx.side * J::NGP, q, cx.lam), v);
                    if (cy.cut) v = fma(ay, corner_eval<K>(jr + J::OFF_G + (2 + cy.side) * J::NGP, p, cy.lam), v);
                    if (cx.cut && cy.cut) {
                        bool poly = false;
                        const double I11 = cross_I11<K>(jr, a.xrec + (int64_t)X::RS * t + cx.side * X::XB, cx.lam, cy.X,
                                                        cx.side, cy.side, poly);
                        v = fma(ax * ay, I11, v);
                        if (COUNT && hit) { ++c_cross; c_poly += poly; }
                    }
                    if (COUNT && hit) c_corner += (int)cx.cut + (int)cy.cut;
                }
                if (hit) atomicAdd(a.out + orig, v);
            }
        }
    }
    if (COUNT) {
        unsigned long long vv[8] = {c_cand, c_pairs, c_pieces, c_sub, c_corner, c_cross, 0ull, c_poly};
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            unsigned long long x = vv[i];
            for (int o = 16; o > 0; o >>= 1) x += __shfl_down_sync(0xffffffffu, x, o);
            if (lane == 0 && x) atomicAdd(a.cnt + i, x);
        }
    }
}

}  // namespace siacjump
