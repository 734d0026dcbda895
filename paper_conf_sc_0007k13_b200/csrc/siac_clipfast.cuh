// siac_clipfast.cuh -- register-only Sutherland-Hodgman for the common pair geometry.
//
// When h >= the longest triangle edge (the paper's choice, h = s), a
// triangle's open x-range contains at most one kernel line (an interior breakline or a
// stencil edge) and likewise in y.  The pieces T ∩ cell are then produced by at most one
// vertical and one horizontal Sutherland-Hodgman split (Alg. 1), which this file
// evaluates in closed form on registers:
//   split of a convex n-gon (n = 3, 4) by an axis line: vertices with coord <= X form one
//   contiguous run; the "alone" vertex (or the run start, for a 2/2 quad split) fixes the
//   output layout, so every output vertex is an input vertex picked by a select or an edge
//   intersection.  Intersections are evaluated from the ORIGINAL triangle edge they lie on
//   (anchor vertex + slope from the record) or are exact line corners, so a point shared by
//   two pieces is computed once, identically.
// A vertex exactly on a line is classified "<= X"; the pieces are then still exact (the
// other side gains a duplicate vertex, i.e. a zero-area fan triangle).
// Pairs with more than one line per axis (h smaller than the triangles) use the general
// splitter siacdev::gen_pieces.
#pragma once

#include "siac_device.cuh"

namespace siacfast {

struct TriZ {
    double x[3], y[3];        // z-frame vertices
    double syx[3], sxy[3];    // dy/dx, dx/dy of original edge g (vertex g -> g+1)
};

template <class T> __device__ __forceinline__ T pick3(int a, T v0, T v1, T v2) {
    return a == 0 ? v0 : (a == 1 ? v1 : v2);
}
template <class T> __device__ __forceinline__ T pick4(int a, T v0, T v1, T v2, T v3) {
    return a < 2 ? (a == 0 ? v0 : v1) : (a == 2 ? v2 : v3);
}

// A polygon piece in registers: up to 5 vertices, edge tags (tag[e] = edge e -> e+1):
// 0..2 original triangle edge, 3 = the vertical cut line.
struct Poly {
    double x[5], y[5];
    int tag[5];
    int n;
};

// x where the edge with tag t crosses the horizontal line Y (t = 3: the vertical cut X)
__device__ __forceinline__ double cross_y(const TriZ &T, int t, double Y, double X) {
    if (t == 3) return X;
    const double ax = pick3(t, T.x[0], T.x[1], T.x[2]);
    const double ay = pick3(t, T.y[0], T.y[1], T.y[2]);
    const double s = pick3(t, T.sxy[0], T.sxy[1], T.sxy[2]);
    return fma(Y - ay, s, ax);
}

// Split the triangle by the vertical line X into two parts A and B (A.n / B.n = 0 when
// empty); a_lo tells whether A is the part with x <= X.  Outputs are fixed variables (no
// runtime-selected references) so everything stays in registers.
__device__ __forceinline__ void split_tri_x(const TriZ &T, double X, Poly &A, Poly &B, bool &a_lo) {
    const bool b0 = T.x[0] <= X, b1 = T.x[1] <= X, b2 = T.x[2] <= X;
    const int nb = (int)b0 + (int)b1 + (int)b2;
    if (nb == 3 || nb == 0) {
#pragma unroll
        for (int v = 0; v < 3; ++v) { A.x[v] = T.x[v]; A.y[v] = T.y[v]; A.tag[v] = v; }
        A.n = 3;
        B.n = 0;
        a_lo = (nb == 3);
        return;
    }
    // alone vertex a: the one on the minority side; A = its triangle, B = the quad
    const int a = (nb == 1) ? (b0 ? 0 : (b1 ? 1 : 2)) : (!b0 ? 0 : (!b1 ? 1 : 2));
    const int bI = a == 2 ? 0 : a + 1, cI = a == 0 ? 2 : a - 1;
    const double Ax = pick3(a, T.x[0], T.x[1], T.x[2]), Ay = pick3(a, T.y[0], T.y[1], T.y[2]);
    const double Bx = pick3(bI, T.x[0], T.x[1], T.x[2]), By = pick3(bI, T.y[0], T.y[1], T.y[2]);
    const double Cx = pick3(cI, T.x[0], T.x[1], T.x[2]), Cy = pick3(cI, T.y[0], T.y[1], T.y[2]);
    // edge AB is original edge a (anchor A); edge CA is original edge cI (anchor C)
    const double sAB = pick3(a, T.syx[0], T.syx[1], T.syx[2]);
    const double sCA = pick3(cI, T.syx[0], T.syx[1], T.syx[2]);
    const double yAB = fma(X - Ax, sAB, Ay);
    const double yCA = fma(X - Cx, sCA, Cy);
    a_lo = (nb == 1);
    A.x[0] = Ax; A.y[0] = Ay;  A.tag[0] = a;
    A.x[1] = X;  A.y[1] = yAB; A.tag[1] = 3;
    A.x[2] = X;  A.y[2] = yCA; A.tag[2] = cI;
    A.n = 3;
    B.x[0] = X;  B.y[0] = yAB; B.tag[0] = a;
    B.x[1] = Bx; B.y[1] = By;  B.tag[1] = bI;
    B.x[2] = Cx; B.y[2] = Cy;  B.tag[2] = cI;
    B.x[3] = X;  B.y[3] = yCA; B.tag[3] = 3;
    B.n = 4;
}

// Split polygon P (3 or 4 vertices) by the horizontal line Y into parts A and B; a_lo tells
// whether A is the part with y <= Y.  Returns false if the classification is not a single
// contiguous run (only possible for a numerically degenerate quad).
__device__ __forceinline__ bool split_poly_y(const TriZ &T, const Poly &P, double Y, double X, Poly &A, Poly &B,
                                             bool &a_lo) {
    const int n = P.n;
    bool b[4];
    int nb = 0;
#pragma unroll
    for (int v = 0; v < 4; ++v) { b[v] = (v < n) && (P.y[v] <= Y); nb += (int)b[v]; }
    if (nb == 0 || nb == n) {
        A = P;
        B.n = 0;
        a_lo = (nb == n);
        return true;
    }
    if (n == 3) {
        const int a = (nb == 1) ? (b[0] ? 0 : (b[1] ? 1 : 2)) : (!b[0] ? 0 : (!b[1] ? 1 : 2));
        const int bI = a == 2 ? 0 : a + 1, cI = a == 0 ? 2 : a - 1;
        const double Ax = pick3(a, P.x[0], P.x[1], P.x[2]), Ay = pick3(a, P.y[0], P.y[1], P.y[2]);
        const double Bx = pick3(bI, P.x[0], P.x[1], P.x[2]), By = pick3(bI, P.y[0], P.y[1], P.y[2]);
        const double Cx = pick3(cI, P.x[0], P.x[1], P.x[2]), Cy = pick3(cI, P.y[0], P.y[1], P.y[2]);
        const int tAB = pick3(a, P.tag[0], P.tag[1], P.tag[2]);
        const int tBC = pick3(bI, P.tag[0], P.tag[1], P.tag[2]);
        const int tCA = pick3(cI, P.tag[0], P.tag[1], P.tag[2]);
        const double xAB = cross_y(T, tAB, Y, X), xCA = cross_y(T, tCA, Y, X);
        a_lo = (nb == 1);
        A.x[0] = Ax;  A.y[0] = Ay; A.tag[0] = tAB;
        A.x[1] = xAB; A.y[1] = Y;  A.tag[1] = 4;
        A.x[2] = xCA; A.y[2] = Y;  A.tag[2] = tCA;
        A.n = 3;
        B.x[0] = xAB; B.y[0] = Y;  B.tag[0] = tAB;
        B.x[1] = Bx;  B.y[1] = By; B.tag[1] = tBC;
        B.x[2] = Cx;  B.y[2] = Cy; B.tag[2] = tCA;
        B.x[3] = xCA; B.y[3] = Y;  B.tag[3] = 4;
        B.n = 4;
        return true;
    }
    // n == 4
    if (nb == 2) {
        if (b[0] == b[2]) return false;     // 1010 / 0101: not a contiguous run
        // run start p: below vertex whose predecessor is above; A = below quad
        const int p = (b[0] && !b[3]) ? 0 : ((b[1] && !b[0]) ? 1 : ((b[2] && !b[1]) ? 2 : 3));
        const int q = (p + 1) & 3, r = (p + 2) & 3, s = (p + 3) & 3;
        const double Px = pick4(p, P.x[0], P.x[1], P.x[2], P.x[3]), Py = pick4(p, P.y[0], P.y[1], P.y[2], P.y[3]);
        const double Qx = pick4(q, P.x[0], P.x[1], P.x[2], P.x[3]), Qy = pick4(q, P.y[0], P.y[1], P.y[2], P.y[3]);
        const double Rx = pick4(r, P.x[0], P.x[1], P.x[2], P.x[3]), Ry = pick4(r, P.y[0], P.y[1], P.y[2], P.y[3]);
        const double Sx = pick4(s, P.x[0], P.x[1], P.x[2], P.x[3]), Sy = pick4(s, P.y[0], P.y[1], P.y[2], P.y[3]);
        const int tP = pick4(p, P.tag[0], P.tag[1], P.tag[2], P.tag[3]);   // edge P->Q
        const int tQ = pick4(q, P.tag[0], P.tag[1], P.tag[2], P.tag[3]);   // edge Q->R (crossing)
        const int tR = pick4(r, P.tag[0], P.tag[1], P.tag[2], P.tag[3]);   // edge R->S
        const int tS = pick4(s, P.tag[0], P.tag[1], P.tag[2], P.tag[3]);   // edge S->P (crossing)
        const double xQ = cross_y(T, tQ, Y, X), xS = cross_y(T, tS, Y, X);
        a_lo = true;
        A.x[0] = Px; A.y[0] = Py; A.tag[0] = tP;
        A.x[1] = Qx; A.y[1] = Qy; A.tag[1] = tQ;
        A.x[2] = xQ; A.y[2] = Y;  A.tag[2] = 4;
        A.x[3] = xS; A.y[3] = Y;  A.tag[3] = tS;
        A.n = 4;
        B.x[0] = xQ; B.y[0] = Y;  B.tag[0] = tQ;
        B.x[1] = Rx; B.y[1] = Ry; B.tag[1] = tR;
        B.x[2] = Sx; B.y[2] = Sy; B.tag[2] = tS;
        B.x[3] = xS; B.y[3] = Y;  B.tag[3] = 4;
        B.n = 4;
        return true;
    }
    // nb == 1 or 3: the alone vertex a -> triangle A on its side, pentagon B on the other
    const bool want = (nb == 1);
    const int a = (b[0] == want) ? 0 : ((b[1] == want) ? 1 : ((b[2] == want) ? 2 : 3));
    const int bI = (a + 1) & 3, cI = (a + 2) & 3, dI = (a + 3) & 3;
    const double Ax = pick4(a, P.x[0], P.x[1], P.x[2], P.x[3]), Ay = pick4(a, P.y[0], P.y[1], P.y[2], P.y[3]);
    const double Bx = pick4(bI, P.x[0], P.x[1], P.x[2], P.x[3]), By = pick4(bI, P.y[0], P.y[1], P.y[2], P.y[3]);
    const double Cx = pick4(cI, P.x[0], P.x[1], P.x[2], P.x[3]), Cy = pick4(cI, P.y[0], P.y[1], P.y[2], P.y[3]);
    const double Dx = pick4(dI, P.x[0], P.x[1], P.x[2], P.x[3]), Dy = pick4(dI, P.y[0], P.y[1], P.y[2], P.y[3]);
    const int tA = pick4(a, P.tag[0], P.tag[1], P.tag[2], P.tag[3]);
    const int tB = pick4(bI, P.tag[0], P.tag[1], P.tag[2], P.tag[3]);
    const int tC = pick4(cI, P.tag[0], P.tag[1], P.tag[2], P.tag[3]);
    const int tD = pick4(dI, P.tag[0], P.tag[1], P.tag[2], P.tag[3]);
    const double xAB = cross_y(T, tA, Y, X), xDA = cross_y(T, tD, Y, X);
    a_lo = want;
    A.x[0] = Ax;  A.y[0] = Ay; A.tag[0] = tA;
    A.x[1] = xAB; A.y[1] = Y;  A.tag[1] = 4;
    A.x[2] = xDA; A.y[2] = Y;  A.tag[2] = tD;
    A.n = 3;
    B.x[0] = xAB; B.y[0] = Y;  B.tag[0] = tA;
    B.x[1] = Bx;  B.y[1] = By; B.tag[1] = tB;
    B.x[2] = Cx;  B.y[2] = Cy; B.tag[2] = tC;
    B.x[3] = Dx;  B.y[3] = Dy; B.tag[3] = tD;
    B.x[4] = xDA; B.y[4] = Y;  B.tag[4] = 4;
    B.n = 5;
    return true;
}

// Cut structure of one axis: the kernel lines strictly inside (lo, hi) (in z units).
// Returns the number of such lines (capped at 2); m = index of the (first) line,
// c = the single column when there is no line.
template <int K>
__device__ __forceinline__ int axis_cuts(double lo, double hi, int &m, int &c) {
    constexpr int NC = 3 * K + 1;
    constexpr double T0 = -0.5 * (3 * K + 1);
    const double a = lo - T0, b = hi - T0;
    int mlo = (int)floor(fmax(a, -1.0)) + 1;          // first integer > a
    int mhi = (int)ceil(fmin(b, (double)NC + 1)) - 1;  // last integer < b
    mlo = max(mlo, 0);
    mhi = min(mhi, NC);
    m = mlo;
    c = min(max((int)floor(fmax(a, -1.0)), 0), NC - 1);
    const int cnt = mhi - mlo + 1;
    return cnt < 0 ? 0 : (cnt > 2 ? 2 : cnt);
}

// Split one x-part by the horizontal cut (if any) and emit its pieces.  Returns false if
// the split found a degenerate quad (caller falls back).
template <class EMIT>
__device__ __forceinline__ bool emit_col(const TriZ &T, const Poly &P, int ci, bool ny, double X, double Y,
                                         int rowL, int rowH, EMIT &emit) {
    if (P.n < 3 || ci < 0) return true;
    if (!ny) { emit(P, ci, rowL); return true; }
    Poly A, B;
    bool a_lo;
    if (!split_poly_y(T, P, Y, X, A, B, a_lo)) return false;
    const int ra = a_lo ? rowL : rowH, rb = a_lo ? rowH : rowL;
    if (A.n >= 3 && ra >= 0) emit(A, ci, ra);
    if (B.n >= 3 && rb >= 0) emit(B, ci, rb);
    return true;
}

// Emit every non-empty piece of triangle T (common geometry only); returns false if an axis
// has two or more lines inside the triangle's range or a split degenerates -- the caller
// must then discard whatever was emitted and use the general splitter.  emit(Poly, ci, cj).
template <int K, class EMIT>
__device__ __forceinline__ bool gen_pieces_fast(const TriZ &T, EMIT &emit) {
    constexpr int NC = 3 * K + 1;
    constexpr double T0 = -0.5 * (3 * K + 1);
    const double xmin = fmin(T.x[0], fmin(T.x[1], T.x[2])), xmax = fmax(T.x[0], fmax(T.x[1], T.x[2]));
    const double ymin = fmin(T.y[0], fmin(T.y[1], T.y[2])), ymax = fmax(T.y[0], fmax(T.y[1], T.y[2]));
    int mx, cx, my, cy;
    const int nx = axis_cuts<K>(xmin, xmax, mx, cx);
    const int ny = axis_cuts<K>(ymin, ymax, my, cy);
    if (nx > 1 || ny > 1) return false;
    const double X = T0 + mx, Y = T0 + my;
    // columns of the two x-parts (-1 = outside the stencil) and rows of the y-parts
    const int colL = nx ? mx - 1 : cx, colH = nx ? (mx < NC ? mx : -1) : -1;
    const int rowL = ny ? my - 1 : cy, rowH = ny ? (my < NC ? my : -1) : -1;
    if (nx) {
        Poly A, B;
        bool a_lo;
        split_tri_x(T, X, A, B, a_lo);
        if (!emit_col(T, A, a_lo ? colL : colH, ny, X, Y, rowL, rowH, emit)) return false;
        if (!emit_col(T, B, a_lo ? colH : colL, ny, X, Y, rowL, rowH, emit)) return false;
    } else {
        Poly P;
#pragma unroll
        for (int v = 0; v < 3; ++v) { P.x[v] = T.x[v]; P.y[v] = T.y[v]; P.tag[v] = v; }
        P.n = 3;
        if (!emit_col(T, P, colL, ny, X, Y, rowL, rowH, emit)) return false;
    }
    return true;
}

}  // namespace siacfast
