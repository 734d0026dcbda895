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
//   [0..5]   v0x v0y v1x v1y v2x v2y        physical vertices (unshifted)
//   [6..9]   M00 M01 M10 M11                 M = 3 h A^{-1}, A = [v1-v0 | v2-v0]:
//                                            (rho, sigma) = M (z - z_v0) - (1, 1)
//   [10..12] dy/dx of edges 0, 1, 2          edge g runs from vertex g to vertex (g+1)%3
//   [13..15] dx/dy of edges 0, 1, 2          (slopes are scale-invariant: same in the z-frame)
//   [16..]   d_ab                            u_T in centred coords rho = 3r-1, sigma = 3s-1,
//                                            Horner order (a = k..0, b = 0..k-a)
template <int K> struct Rec {
    static constexpr int NB = (K + 1) * (K + 2) / 2;
    static constexpr int OFF_D = 16;
    static constexpr int RAW = OFF_D + NB;
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

// N independent sub-triangles integrated together: the quadrature loop runs over the rule
// points outermost and the N sub-triangles innermost, so their FMA chains interleave
// (instruction-level parallelism for a single warp feeding the FP64 pipe).
#ifndef SIAC_QP_UNROLL
#define SIAC_QP_UNROLL 64
#endif
constexpr int kQpUnroll = SIAC_QP_UNROLL;

template <int K> struct SubTri {
    double p0x, p0y, e1x, e1y, e2x, e2y;
    double kx[K + 1], ky[K + 1];
    double cx, cy;
    double d[(K + 1) * (K + 2) / 2];
    PairGeom g;
};

template <int K, int N>
__device__ __forceinline__ void integrate_subtri_n(const SubTri<K> *t, double *out) {
    double ax0[N], ay0[N], r0[N], rr[N], rs[N], s0[N], sr[N], ss[N], acc[N], area[N];
#pragma unroll
    for (int n = 0; n < N; ++n) {
        const SubTri<K> &T = t[n];
        area[n] = 0.5 * fabs(T.e1x * T.e2y - T.e1y * T.e2x);
        ax0[n] = T.p0x - T.cx;
        ay0[n] = T.p0y - T.cy;
        const double dx0 = T.p0x - T.g.zv0x, dy0 = T.p0y - T.g.zv0y;
        r0[n] = fma(T.g.M00, dx0, fma(T.g.M01, dy0, -1.0));
        rr[n] = fma(T.g.M00, T.e1x, T.g.M01 * T.e1y);
        rs[n] = fma(T.g.M00, T.e2x, T.g.M01 * T.e2y);
        s0[n] = fma(T.g.M10, dx0, fma(T.g.M11, dy0, -1.0));
        sr[n] = fma(T.g.M10, T.e1x, T.g.M11 * T.e1y);
        ss[n] = fma(T.g.M10, T.e2x, T.g.M11 * T.e2y);
        acc[n] = 0.0;
    }
    // rule points in a rolled loop (constant-bank loads): keeps the kernel small enough for
    // the instruction cache, which a fully unrolled 19/33-point loop per sub-triangle is not
#pragma unroll kQpUnroll
    for (int q = 0; q < Rule<K>::NQ; ++q) {
        const double r = qr<K>(q), s = qs<K>(q), w = qw<K>(q);
#pragma unroll
        for (int n = 0; n < N; ++n) {
            const SubTri<K> &T = t[n];
            const double tx = fma(T.e2x, s, fma(T.e1x, r, ax0[n]));
            const double ty = fma(T.e2y, s, fma(T.e1y, r, ay0[n]));
            const double rho = fma(rs[n], s, fma(rr[n], r, r0[n]));
            const double sig = fma(ss[n], s, fma(sr[n], r, s0[n]));
            const double kv = horner1<K>(T.kx, tx) * horner1<K>(T.ky, ty);
            acc[n] = fma(w, kv * horner2<K>(T.d, rho, sig), acc[n]);
        }
    }
#pragma unroll
    for (int n = 0; n < N; ++n) out[n] = area[n] * acc[n];
}

// ------------------------------------------------------------------ Sutherland-Hodgman split

constexpr int PCAP = 10;   // a triangle ∩ 4 half-planes has <= 7 vertices; margin for rounding

// Split convex polygon (px, py, n) by the line coord_AX = X into the closed half-planes
// coord <= X (L) and coord >= X (R).  Each output is exactly Alg. 1's output for that clip
// edge (vertices on the line belong to both; an intersection is added only where an edge
// crosses the line strictly, so no duplicate vertices).  The crossing point is computed
// once from the ordered edge and given to both outputs, so neighbouring pieces share it
// bit-exactly.  Two comparisons per vertex.
template <int AX>
__device__ __forceinline__ void split_poly(const double *px, const double *py, int n, double X,
                                           double *lx, double *ly, int &nl, double *rx, double *ry, int &nr) {
    nl = 0;
    nr = 0;
    const double c0 = AX ? py[0] : px[0];
    const bool le0 = c0 <= X, ge0 = c0 >= X;
    bool le_e = le0, ge_e = ge0;
    double ce = c0;
    for (int e = 0; e < n; ++e) {
        const int f = (e + 1 == n) ? 0 : e + 1;
        const double cf = AX ? py[f] : px[f];
        const bool le_f = (f == 0) ? le0 : (cf <= X);
        const bool ge_f = (f == 0) ? ge0 : (cf >= X);
        if (le_e && nl < PCAP) { lx[nl] = px[e]; ly[nl] = py[e]; ++nl; }
        if (ge_e && nr < PCAP) { rx[nr] = px[e]; ry[nr] = py[e]; ++nr; }
        if ((!ge_e && !le_f) || (!le_e && !ge_f)) {
            const double t = (X - ce) / (cf - ce);
            double ix, iy;
            if (AX == 0) { ix = X; iy = fma(t, py[f] - py[e], py[e]); }
            else { iy = X; ix = fma(t, px[f] - px[e], px[e]); }
            if (nl < PCAP) { lx[nl] = ix; ly[nl] = iy; ++nl; }
            if (nr < PCAP) { rx[nr] = ix; ry[nr] = iy; ++nr; }
        }
        le_e = le_f;
        ge_e = ge_f;
        ce = cf;
    }
}

__device__ __forceinline__ int clampi(double v, int lo, int hi) {
    v = fmin(fmax(v, (double)lo - 1.0), (double)hi + 1.0);
    int i = (int)floor(v);
    return i < lo ? lo : (i > hi ? hi : i);
}

struct Counts { unsigned long long pairs, pieces, subtris; };

// Every non-empty piece (T ∩ kernel cell (i, j)) of the z-frame triangle (zx, zy), in column-
// major cell order, passed to emit(px, py, n, i, j).  Columns are peeled off the remainder
// polygon by vertical splits, rows off each column by horizontal splits (each split is one
// Sutherland-Hodgman pass producing both sides); the parts outside the stencil
// [T0, T0 + 3K+1]^2 are dropped.
template <int K, class EMIT>
__device__ __forceinline__ void gen_pieces(const double *zx, const double *zy, EMIT &emit) {
    constexpr int NC = 3 * K + 1;
    constexpr double T0 = -0.5 * (3 * K + 1);
    const double xmin = fmin(zx[0], fmin(zx[1], zx[2])), xmax = fmax(zx[0], fmax(zx[1], zx[2]));
    const int ilo = clampi(xmin - T0, 0, NC - 1), ihi = clampi(xmax - T0, 0, NC - 1);
    double b0x[PCAP], b0y[PCAP], b1x[PCAP], b1y[PCAP], b2x[PCAP], b2y[PCAP], b3x[PCAP], b3y[PCAP];
    double b4x[PCAP], b4y[PCAP];
    double *ax = b0x, *ay = b0y, *fx = b1x, *fy = b1y;      // x-remainder and its spare buffer
    int na = 3;
    for (int v = 0; v < 3; ++v) { ax[v] = zx[v]; ay[v] = zy[v]; }
    if (xmin < T0) {           // drop the part left of the stencil
        int nl;
        split_poly<0>(ax, ay, na, T0, b4x, b4y, nl, fx, fy, na);
        double *tx = ax, *ty = ay; ax = fx; ay = fy; fx = tx; fy = ty;
    }
    for (int i = ilo; i <= ihi && na >= 3; ++i) {
        const double X1 = T0 + i + 1;
        double *cx = b2x, *cy = b2y;       // column piece
        int nc;
        if (i < ihi || xmax > X1) {
            split_poly<0>(ax, ay, na, X1, cx, cy, nc, fx, fy, na);
            double *tx = ax, *ty = ay; ax = fx; ay = fy; fx = tx; fy = ty;
        } else {
            cx = ax; cy = ay; nc = na; na = 0;
        }
        if (nc < 3) continue;
        double ymin = cy[0], ymax = cy[0];
        for (int v = 1; v < nc; ++v) { ymin = fmin(ymin, cy[v]); ymax = fmax(ymax, cy[v]); }
        const int jlo = clampi(ymin - T0, 0, NC - 1), jhi = clampi(ymax - T0, 0, NC - 1);
        double *gx = (cx == b2x) ? b3x : b2x, *gy = (cx == b2x) ? b3y : b2y;   // spare for the y-remainder
        if (ymin < T0) {       // drop the part below the stencil
            int nl;
            split_poly<1>(cx, cy, nc, T0, b4x, b4y, nl, gx, gy, nc);
            double *tx = cx, *ty = cy; cx = gx; cy = gy; gx = tx; gy = ty;
        }
        for (int j = jlo; j <= jhi && nc >= 3; ++j) {
            const double Y1 = T0 + j + 1;
            if (j < jhi || ymax > Y1) {
                int nq;
                split_poly<1>(cx, cy, nc, Y1, b4x, b4y, nq, gx, gy, nc);
                double *tx = cx, *ty = cy; cx = gx; cy = gy; gx = tx; gy = ty;
                if (nq >= 3) emit(b4x, b4y, nq, i, j);
            } else {
                if (nc >= 3) emit(cx, cy, nc, i, j);
                nc = 0;
            }
        }
    }
}

// Contribution of one (point, triangle image) pair, integrated inline (thread-per-point
// schedule).  kc: (3K+1) x (K+1) cell table; kcy: the y axis' table if it differs (one-sided
// kernels), else nullptr.
template <int K, bool COUNT>
__device__ double pair_contrib(const double *zx, const double *zy, const double *kc, const double *d,
                               const PairGeom &g, Counts &cnt, const double *kcy = nullptr) {
    if (kcy == nullptr) kcy = kc;
    constexpr double T0 = -0.5 * (3 * K + 1);
    double total = 0.0;
    auto emit = [&](const double *qx, const double *qy, int nq, int i, int j) {
        double kx[K + 1], ky[K + 1];
#pragma unroll
        for (int m = 0; m <= K; ++m) { kx[m] = kc[i * (K + 1) + m]; ky[m] = kcy[j * (K + 1) + m]; }
        if (COUNT) { cnt.pieces++; cnt.subtris += nq - 2; }
        for (int m = 1; m + 1 < nq; ++m)
            total += integrate_subtri<K>(qx[0], qy[0], qx[m], qy[m], qx[m + 1], qy[m + 1], kx, ky, T0 + i + 0.5,
                                         T0 + j + 0.5, d, g);
    };
    gen_pieces<K>(zx, zy, emit);
    return total;
}

}  // namespace siacdev
