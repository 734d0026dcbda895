// siac_device.cuh -- device-side building blocks of the B200 SIAC path (sm_100a, FP64).
//
// Geometry is handled in the point-relative, h-scaled "z-frame": for evaluation point x
// and triangle image T + s, z = (y - x)/h, so the kernel's breaklines sit at the exact
// constants t_i = -(3k+1)/2 + i and the (1/h^2) of Eq. (1) cancels the area element:
//     u*(x) = sum over pieces P of  \int_P K_i(z1) K_j(z2) u_T(z) dz.
// A piece is (T + s) ∩ kernel cell (i, j), found by Sutherland-Hodgman clipping against
// the cell lines (Alg. 1), fan-triangulated (L248-249), and each fan
// sub-triangle integrated by a symmetric rule exact for degree 3k (Eq. (2)).
#pragma once

#include <cstdint>
#include "siac_quadrature.h"

namespace siacdev {

// ------------------------------------------------------------------ quadrature tables

template <int K> struct Rule;
template <> struct Rule<1> { static constexpr int NQ = SIAC_NQ_K1; };
template <> struct Rule<2> { static constexpr int NQ = SIAC_NQ_K2; };
template <> struct Rule<3> { static constexpr int NQ = SIAC_NQ_K3; };
template <> struct Rule<4> { static constexpr int NQ = SIAC_NQ_K4; };

template <int K> __device__ __forceinline__ double qr(int q) {
    if constexpr (K == 1) return siac_qr_k1[q];
    else if constexpr (K == 2) return siac_qr_k2[q];
    else if constexpr (K == 3) return siac_qr_k3[q];
    else return siac_qr_k4[q];
}
template <int K> __device__ __forceinline__ double qs(int q) {
    if constexpr (K == 1) return siac_qs_k1[q];
    else if constexpr (K == 2) return siac_qs_k2[q];
    else if constexpr (K == 3) return siac_qs_k3[q];
    else return siac_qs_k4[q];
}
template <int K> __device__ __forceinline__ double qw(int q) {
    if constexpr (K == 1) return siac_qw_k1[q];
    else if constexpr (K == 2) return siac_qw_k2[q];
    else if constexpr (K == 3) return siac_qw_k3[q];
    else return siac_qw_k4[q];
}

// ------------------------------------------------------------------ record layout
// Triangle record (doubles), sorted by anchor cell:
//   [0..5]  v0x v0y v1x v1y v2x v2y         physical vertices (unshifted)
//   [6..9]  M00 M01 M10 M11                  M = 3 h A^{-1}, A = [v1-v0 | v2-v0]:
//                                            (rho, sigma) = M (z - z_v0) - (1, 1)
//   [10..]  d_ab                             u_T in centred coords rho = 3r-1, sigma = 3s-1,
//                                            Horner order (a = k..0, b = 0..k-a)
template <int K> struct Rec {
    static constexpr int NB = (K + 1) * (K + 2) / 2;
    static constexpr int RAW = 10 + NB;
    static constexpr int RS = (RAW + 1) & ~1;        // padded to 16 B
};

// ------------------------------------------------------------------ polynomial evaluation

template <int K> __device__ __forceinline__ double horner1(const double *c, double t) {
    double v = c[K];
#pragma unroll
    for (int m = K - 1; m >= 0; --m) v = fma(v, t, c[m]);
    return v;
}

// u = sum_a rho^a sum_b d_ab sigma^b, d in Horner order (a = K..0, b ascending).
template <int K> __device__ __forceinline__ double horner2(const double *d, double rho, double sig) {
    double u = 0.0;
    int off = 0;
#pragma unroll
    for (int a = K; a >= 0; --a) {
        const int n = K - a;
        double in = d[off + n];
#pragma unroll
        for (int b = n - 1; b >= 0; --b) in = fma(in, sig, d[off + b]);
        u = (a == K) ? in : fma(u, rho, in);
        off += n + 1;
    }
    return u;
}

// ------------------------------------------------------------------ sub-triangle quadrature

struct PairGeom {      // per (point, triangle image) constants
    double M00, M01, M10, M11;   // z -> centred reference map
    double zv0x, zv0y;           // z-frame coordinates of vertex 0
};

// \int over triangle (p0,p1,p2) of K_ci(z1) K_cj(z2) u(z) dz, rule exact for degree 3K.
template <int K>
__device__ __forceinline__ double integrate_subtri(double p0x, double p0y, double p1x, double p1y,
                                                   double p2x, double p2y, const double *kx, const double *ky,
                                                   double cx, double cy, const double *d, const PairGeom &g) {
    const double e1x = p1x - p0x, e1y = p1y - p0y;
    const double e2x = p2x - p0x, e2y = p2y - p0y;
    const double area = 0.5 * fabs(e1x * e2y - e1y * e2x);
    // kernel local variables tau = z - cell centre, affine in the rule's (r, s)
    const double ax0 = p0x - cx, ay0 = p0y - cy;
    // centred reference coordinates, affine in (r, s)
    const double dx0 = p0x - g.zv0x, dy0 = p0y - g.zv0y;
    const double r0 = fma(g.M00, dx0, fma(g.M01, dy0, -1.0));
    const double rr = fma(g.M00, e1x, g.M01 * e1y), rs = fma(g.M00, e2x, g.M01 * e2y);
    const double s0 = fma(g.M10, dx0, fma(g.M11, dy0, -1.0));
    const double sr = fma(g.M10, e1x, g.M11 * e1y), ss = fma(g.M10, e2x, g.M11 * e2y);
    double acc = 0.0;
#pragma unroll
    for (int q = 0; q < Rule<K>::NQ; ++q) {
        const double r = qr<K>(q), s = qs<K>(q);
        const double tx = fma(e2x, s, fma(e1x, r, ax0));
        const double ty = fma(e2y, s, fma(e1y, r, ay0));
        const double rho = fma(rs, s, fma(rr, r, r0));
        const double sig = fma(ss, s, fma(sr, r, s0));
        const double kv = horner1<K>(kx, tx) * horner1<K>(ky, ty);
        acc = fma(qw<K>(q), kv * horner2<K>(d, rho, sig), acc);
    }
    return area * acc;
}

// ------------------------------------------------------------------ Sutherland-Hodgman split

constexpr int PCAP = 10;   // a triangle ∩ 4 half-planes has <= 7 vertices; margin for rounding

// Split convex polygon (px, py, n) by the line coord_AX = X into the closed half-planes
// coord <= X (L) and coord >= X (R).  Each output is exactly Alg. 1's output for that clip
// edge (vertices on the line belong to both; an intersection is added only where an edge
// crosses the line strictly, so no duplicate vertices).  The crossing point is computed
// from the same ordered edge for both outputs, so neighbouring pieces share it bit-exactly.
template <int AX>
__device__ __forceinline__ void split_poly(const double *px, const double *py, int n, double X,
                                           double *lx, double *ly, int &nl, double *rx, double *ry, int &nr) {
    nl = 0;
    nr = 0;
    for (int e = 0; e < n; ++e) {
        const int f = (e + 1 == n) ? 0 : e + 1;
        const double ce = AX ? py[e] : px[e];
        const double cf = AX ? py[f] : px[f];
        if (ce <= X && nl < PCAP) { lx[nl] = px[e]; ly[nl] = py[e]; ++nl; }
        if (ce >= X && nr < PCAP) { rx[nr] = px[e]; ry[nr] = py[e]; ++nr; }
        if ((ce < X && cf > X) || (ce > X && cf < X)) {
            const double t = (X - ce) / (cf - ce);
            double ix, iy;
            if (AX == 0) { ix = X; iy = fma(t, py[f] - py[e], py[e]); }
            else { iy = X; ix = fma(t, px[f] - px[e], px[e]); }
            if (nl < PCAP) { lx[nl] = ix; ly[nl] = iy; ++nl; }
            if (nr < PCAP) { rx[nr] = ix; ry[nr] = iy; ++nr; }
        }
    }
}

__device__ __forceinline__ int clampi(double v, int lo, int hi) {
    v = fmin(fmax(v, (double)lo - 1.0), (double)hi + 1.0);
    int i = (int)floor(v);
    return i < lo ? lo : (i > hi ? hi : i);
}

struct Counts { unsigned long long pairs, pieces, subtris; };

// Contribution of one (point, triangle image) pair: clip the z-frame triangle against the
// kernel cells it overlaps, fan-triangulate, integrate.  kc: (3K+1) x (K+1) cell table.
template <int K, bool COUNT>
__device__ double pair_contrib(const double *zx, const double *zy, const double *kc, const double *d,
                               const PairGeom &g, Counts &cnt) {
    constexpr int NC = 3 * K + 1;
    constexpr double T0 = -0.5 * (3 * K + 1);
    const double xmin = fmin(zx[0], fmin(zx[1], zx[2])), xmax = fmax(zx[0], fmax(zx[1], zx[2]));
    const int ilo = clampi(xmin - T0, 0, NC - 1), ihi = clampi(xmax - T0, 0, NC - 1);
    double ax[PCAP], ay[PCAP];
    int na = 3;
    for (int v = 0; v < 3; ++v) { ax[v] = zx[v]; ay[v] = zy[v]; }
    double tx_[PCAP], ty_[PCAP];
    int nt_;
    if (xmin < T0) {           // drop the part left of the stencil
        double lx[PCAP], ly[PCAP];
        int nl;
        split_poly<0>(ax, ay, na, T0, lx, ly, nl, tx_, ty_, nt_);
        for (int v = 0; v < nt_; ++v) { ax[v] = tx_[v]; ay[v] = ty_[v]; }
        na = nt_;
    }
    double total = 0.0;
    for (int i = ilo; i <= ihi && na >= 3; ++i) {
        const double X1 = T0 + i + 1;
        double cx_[PCAP], cy_[PCAP];
        int nc;
        if (i < ihi || xmax > X1) {
            split_poly<0>(ax, ay, na, X1, cx_, cy_, nc, tx_, ty_, nt_);
            for (int v = 0; v < nt_; ++v) { ax[v] = tx_[v]; ay[v] = ty_[v]; }
            na = nt_;
        } else {
            for (int v = 0; v < na; ++v) { cx_[v] = ax[v]; cy_[v] = ay[v]; }
            nc = na;
            na = 0;
        }
        if (nc < 3) continue;
        double ymin = cy_[0], ymax = cy_[0];
        for (int v = 1; v < nc; ++v) { ymin = fmin(ymin, cy_[v]); ymax = fmax(ymax, cy_[v]); }
        const int jlo = clampi(ymin - T0, 0, NC - 1), jhi = clampi(ymax - T0, 0, NC - 1);
        if (ymin < T0) {       // drop the part below the stencil
            double lx[PCAP], ly[PCAP];
            int nl;
            split_poly<1>(cx_, cy_, nc, T0, lx, ly, nl, tx_, ty_, nt_);
            for (int v = 0; v < nt_; ++v) { cx_[v] = tx_[v]; cy_[v] = ty_[v]; }
            nc = nt_;
        }
        double kx[K + 1];
#pragma unroll
        for (int m = 0; m <= K; ++m) kx[m] = kc[i * (K + 1) + m];
        const double ccx = T0 + i + 0.5;
        for (int j = jlo; j <= jhi && nc >= 3; ++j) {
            const double Y1 = T0 + j + 1;
            double qx_[PCAP], qy_[PCAP];
            int nq;
            if (j < jhi || ymax > Y1) {
                split_poly<1>(cx_, cy_, nc, Y1, qx_, qy_, nq, tx_, ty_, nt_);
                for (int v = 0; v < nt_; ++v) { cx_[v] = tx_[v]; cy_[v] = ty_[v]; }
                nc = nt_;
            } else {
                for (int v = 0; v < nc; ++v) { qx_[v] = cx_[v]; qy_[v] = cy_[v]; }
                nq = nc;
                nc = 0;
            }
            if (nq < 3) continue;
            double ky[K + 1];
#pragma unroll
            for (int m = 0; m <= K; ++m) ky[m] = kc[j * (K + 1) + m];
            const double ccy = T0 + j + 0.5;
            if (COUNT) { cnt.pieces++; cnt.subtris += nq - 2; }
            for (int m = 1; m + 1 < nq; ++m)
                total += integrate_subtri<K>(qx_[0], qy_[0], qx_[m], qy_[m], qx_[m + 1], qy_[m + 1], kx, ky, ccx, ccy, d, g);
        }
    }
    return total;
}

}  // namespace siacdev
