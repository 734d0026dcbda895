/*
 * siac_oracle3d.c -- TEST INFRASTRUCTURE ONLY.  The plain, slow CPU oracle for SIAC filtering
 * on TETRAHEDRAL meshes ("extension of these ideas to
 * 3D over unstructured tetrahedral meshes").  Only tests/ may load it; the CUDA path
 * (paper_conf_sc_0007k13_b200/csrc/siac3d.cu) shares no code with it.
 *
 * What it computes: the 3D form of Eq. (1) (L213-235; "the convolution stencil is the tensor
 * product of one-dimensional kernels", L212-214):
 *     u*(x) = (1/h^3) sum_T sum_s \int_{T+s} K((y1-x1)/h) K((y2-x2)/h) K((y3-x3)/h) u_T(y-s) dy
 * with the same 1D kernel K as the 2D oracle (siac_oracle.c: oracle_kernel, Cox-de Boor).
 *
 * How (the 2D oracle's slab/strip method, one dimension up; a different decomposition from the
 * GPU's tetrahedron splitting): the x-integrand g(x) = K(x) \int\int_{T cap {x}} K K u dy dz
 * is a polynomial between consecutive x-breakpoints -- tet vertices, kernel x-planes, the x
 * where a tet edge crosses a kernel y- or z-plane, and the x where a tet face crosses a kernel
 * line {y = Y_j, z = Z_l} (extra breakpoints are harmless) -- so Gauss-Legendre in x on every
 * slab is exact.  At each x-node the cross-section is a convex polygon (3 or 4 vertices), whose
 * (y, z) integral is computed exactly by the 2D method: y-slabs between the polygon's vertex
 * y's, kernel y-lines and the y where polygon edges cross kernel z-lines; each y-slab's z-range
 * (two polygon edges) split at the kernel z-lines into strips; Gauss-Legendre in y and along z.
 * Sums are Neumaier-compensated.
 */
#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define MAXK3 4
#define MAXBR (3 * MAXK3 + 2)

double oracle_kernel(int k, const double *c, double t);   /* siac_oracle.c */

typedef struct { double s, c; } nsum3;
static inline void nadd3(nsum3 *a, double v)
{
    double t = a->s + v;
    if (fabs(a->s) >= fabs(v)) a->c += (a->s - t) + v;
    else a->c += (v - t) + a->s;
    a->s = t;
}

static int cmp_d(const void *a, const void *b)
{
    double x = *(const double *)a, y = *(const double *)b;
    return (x > y) - (x < y);
}

typedef struct {
    int k;
    double h;
    const double *kc;
    const double *V;          /* nv x 3 */
    const int *T;             /* nt x 4 */
    long nt;
    int field_mode;           /* 0: per-tet monomials r^a s^b t^c (nt x nb); 1: global y1^i y2^j y3^l */
    const double *field;
    int field_deg;            /* mode 1: a[(i*(d+1)+j)*(d+1)+l] */
    int n;                    /* Gauss-Legendre points per direction */
    const double *gx, *gw;
} prob3;

/* u_T at the physical point y (already shifted back into the mesh). */
static double field3(const prob3 *P, long t, double y1, double y2, double y3)
{
    if (P->field_mode == 1) {
        const int d = P->field_deg;
        double s = 0.0, p1 = 1.0;
        for (int i = 0; i <= d; ++i, p1 *= y1) {
            double p2 = 1.0;
            for (int j = 0; j <= d; ++j, p2 *= y2) {
                double p3 = 1.0;
                for (int l = 0; l <= d; ++l, p3 *= y3) s += P->field[(i * (d + 1) + j) * (d + 1) + l] * p1 * p2 * p3;
            }
        }
        return s;
    }
    /* y = v0 + r (v1-v0) + s (v2-v0) + t (v3-v0): Cramer's rule */
    const double *v0 = P->V + 3 * (long)P->T[4 * t], *v1 = P->V + 3 * (long)P->T[4 * t + 1];
    const double *v2 = P->V + 3 * (long)P->T[4 * t + 2], *v3 = P->V + 3 * (long)P->T[4 * t + 3];
    double a[3][3], b[3];
    for (int i = 0; i < 3; ++i) {
        a[i][0] = v1[i] - v0[i]; a[i][1] = v2[i] - v0[i]; a[i][2] = v3[i] - v0[i];
    }
    b[0] = y1 - v0[0]; b[1] = y2 - v0[1]; b[2] = y3 - v0[2];
    const double det = a[0][0] * (a[1][1] * a[2][2] - a[1][2] * a[2][1]) - a[0][1] * (a[1][0] * a[2][2] - a[1][2] * a[2][0]) +
                       a[0][2] * (a[1][0] * a[2][1] - a[1][1] * a[2][0]);
    double rst[3];
    for (int c = 0; c < 3; ++c) {
        double m[3][3];
        memcpy(m, a, sizeof(m));
        for (int i = 0; i < 3; ++i) m[i][c] = b[i];
        rst[c] = (m[0][0] * (m[1][1] * m[2][2] - m[1][2] * m[2][1]) - m[0][1] * (m[1][0] * m[2][2] - m[1][2] * m[2][0]) +
                  m[0][2] * (m[1][0] * m[2][1] - m[1][1] * m[2][0])) / det;
    }
    /* modes ordered by n = a+b+c, then c, then b (a = n-b-c) */
    const double *cf = P->field + (long)((P->k + 1) * (P->k + 2) * (P->k + 3) / 6) * t;
    double u = 0.0;
    int idx = 0;
    for (int nn = 0; nn <= P->k; ++nn)
        for (int cc = 0; cc <= nn; ++cc)
            for (int bb = 0; bb <= nn - cc; ++bb, ++idx) {
                const int aa = nn - bb - cc;
                u += cf[idx] * pow(rst[0], aa) * pow(rst[1], bb) * pow(rst[2], cc);
            }
    return u;
}

/* \int\int over the convex polygon (py[i], pz[i]), i < m (any vertex order), of
 * K((y - x2)/h) K((z - x3)/h) u_T(x, y, z) dy dz, by y-slabs and z-strips. */
static double section_integral(const prob3 *P, long t, double xs, double sx, double sy, double sz, double x2,
                               double x3, const double *py, const double *pz, int m, const double *Yb,
                               const double *Zb, double *area)
{
    const int k = P->k, nbr = 3 * k + 2;
    const double h = P->h;
    double ymin = 1e300, ymax = -1e300;
    for (int i = 0; i < m; ++i) { ymin = fmin(ymin, py[i]); ymax = fmax(ymax, py[i]); }
    const double lo = fmax(ymin, Yb[0]), hi = fmin(ymax, Yb[nbr - 1]);
    if (!(lo < hi)) return 0.0;
    double br[4 + MAXBR + 4 * MAXBR + 2];
    int nb = 0;
    br[nb++] = lo;
    br[nb++] = hi;
    for (int i = 0; i < m; ++i)
        if (py[i] > lo && py[i] < hi) br[nb++] = py[i];
    for (int j = 0; j < nbr; ++j)
        if (Yb[j] > lo && Yb[j] < hi) br[nb++] = Yb[j];
    for (int i = 0; i < m; ++i) {             /* polygon edges crossing kernel z-lines */
        const double ay = py[i], az = pz[i], by = py[(i + 1) % m], bz = pz[(i + 1) % m];
        if (az == bz) continue;
        for (int j = 0; j < nbr; ++j) {
            const double Z = Zb[j];
            if ((Z > az && Z < bz) || (Z < az && Z > bz)) {
                const double yc = ay + (Z - az) / (bz - az) * (by - ay);
                if (yc > lo && yc < hi) br[nb++] = yc;
            }
        }
    }
    qsort(br, nb, sizeof(double), cmp_d);
    nsum3 acc = {0, 0}, ar = {0, 0};
    for (int sl = 0; sl + 1 < nb; ++sl) {
        const double a = br[sl], b = br[sl + 1];
        if (!(b > a)) continue;
        const double ym = 0.5 * (a + b);
        /* z-extent at ym: the lowest and highest crossing of the polygon's edges (edge lines) */
        double zlo = 1e300, zhi = -1e300, mlo = 0, qlo = 0, mhi = 0, qhi = 0;
        int ncross = 0;
        for (int i = 0; i < m; ++i) {
            const double ay = py[i], az = pz[i], by = py[(i + 1) % m], bz = pz[(i + 1) % m];
            const double el = fmin(ay, by), er = fmax(ay, by);
            if (!(el < er) || el > a || er < b) continue;
            const double sl_ = (bz - az) / (by - ay), q = az - sl_ * ay;
            const double zm = sl_ * ym + q;
            if (zm < zlo) { zlo = zm; mlo = sl_; qlo = q; }
            if (zm > zhi) { zhi = zm; mhi = sl_; qhi = q; }
            ++ncross;
        }
        if (ncross < 2 || !(zhi > zlo)) continue;
        for (int iy = 0; iy < P->n; ++iy) {
            const double y = a + 0.5 * (b - a) * (1.0 + P->gx[iy]);
            const double wy = 0.5 * (b - a) * P->gw[iy];
            const double zl = fmax(mlo * y + qlo, Zb[0]), zh = fmin(mhi * y + qhi, Zb[nbr - 1]);
            if (!(zh > zl)) continue;
            const double ky = oracle_kernel(k, P->kc, (y - x2) / h);
            /* z-strips at the kernel z-lines inside (zl, zh) */
            double zb[MAXBR + 2];
            int nz = 0;
            zb[nz++] = zl;
            for (int j = 0; j < nbr; ++j)
                if (Zb[j] > zl && Zb[j] < zh) zb[nz++] = Zb[j];
            zb[nz++] = zh;
            for (int st = 0; st + 1 < nz; ++st) {
                const double c0 = zb[st], c1 = zb[st + 1];
                nadd3(&ar, wy * (c1 - c0));
                for (int iz = 0; iz < P->n; ++iz) {
                    const double z = c0 + 0.5 * (c1 - c0) * (1.0 + P->gx[iz]);
                    const double wz = 0.5 * (c1 - c0) * P->gw[iz];
                    const double kz = oracle_kernel(k, P->kc, (z - x3) / h);
                    nadd3(&acc, wy * wz * ky * kz * field3(P, t, xs - sx, y - sy, z - sz));
                }
            }
        }
    }
    *area = ar.s + ar.c;
    return acc.s + acc.c;
}

/* cross-section of tetrahedron p[4][3] at x = xs: 3 or 4 points ordered around their centroid */
static int tet_section(double p[4][3], double xs, double *py, double *pz)
{
    static const int E[6][2] = {{0, 1}, {0, 2}, {0, 3}, {1, 2}, {1, 3}, {2, 3}};
    int m = 0;
    for (int e = 0; e < 6 && m < 4; ++e) {
        const double *a = p[E[e][0]], *b = p[E[e][1]];
        if ((a[0] - xs) * (b[0] - xs) < 0.0) {
            const double r = (xs - a[0]) / (b[0] - a[0]);
            py[m] = a[1] + r * (b[1] - a[1]);
            pz[m] = a[2] + r * (b[2] - a[2]);
            ++m;
        }
    }
    if (m < 3) return 0;
    double cy = 0, cz = 0;
    for (int i = 0; i < m; ++i) { cy += py[i]; cz += pz[i]; }
    cy /= m; cz /= m;
    /* insertion sort by angle */
    for (int i = 1; i < m; ++i) {
        const double yy = py[i], zz = pz[i], ai = atan2(zz - cz, yy - cy);
        int j = i - 1;
        while (j >= 0 && atan2(pz[j] - cz, py[j] - cy) > ai) { py[j + 1] = py[j]; pz[j + 1] = pz[j]; --j; }
        py[j + 1] = yy; pz[j + 1] = zz;
    }
    return m;
}

static void pair_integral3(const prob3 *P, long t, const double *shift, const double *x, nsum3 *acc, nsum3 *vol)
{
    const int k = P->k, nbr = 3 * k + 2;
    const double h = P->h;
    double Xb[MAXBR], Yb[MAXBR], Zb[MAXBR];
    for (int m = 0; m < nbr; ++m) {
        const double tm = -0.5 * (3 * k + 1) + m;
        Xb[m] = x[0] + h * tm; Yb[m] = x[1] + h * tm; Zb[m] = x[2] + h * tm;
    }
    double p[4][3];
    for (int i = 0; i < 4; ++i)
        for (int d = 0; d < 3; ++d) p[i][d] = P->V[3 * (long)P->T[4 * t + i] + d] + shift[d];
    double xmin = 1e300, xmax = -1e300;
    for (int i = 0; i < 4; ++i) { xmin = fmin(xmin, p[i][0]); xmax = fmax(xmax, p[i][0]); }
    const double lo = fmax(xmin, Xb[0]), hi = fmin(xmax, Xb[nbr - 1]);
    if (!(lo < hi)) return;
    double br[2 + 4 + MAXBR + 6 * 2 * MAXBR + 4 * MAXBR * MAXBR];
    int nb = 0;
    br[nb++] = lo;
    br[nb++] = hi;
    for (int i = 0; i < 4; ++i)
        if (p[i][0] > lo && p[i][0] < hi) br[nb++] = p[i][0];
    for (int m = 0; m < nbr; ++m)
        if (Xb[m] > lo && Xb[m] < hi) br[nb++] = Xb[m];
    static const int E[6][2] = {{0, 1}, {0, 2}, {0, 3}, {1, 2}, {1, 3}, {2, 3}};
    for (int e = 0; e < 6; ++e) {                   /* edges crossing kernel y- and z-planes */
        const double *a = p[E[e][0]], *b = p[E[e][1]];
        for (int d = 1; d <= 2; ++d) {
            if (a[d] == b[d]) continue;
            const double *pl = d == 1 ? Yb : Zb;
            for (int m = 0; m < nbr; ++m) {
                const double c = pl[m];
                if ((c > a[d] && c < b[d]) || (c < a[d] && c > b[d])) {
                    const double xc = a[0] + (c - a[d]) / (b[d] - a[d]) * (b[0] - a[0]);
                    if (xc > lo && xc < hi) br[nb++] = xc;
                }
            }
        }
    }
    double ymn = 1e300, ymx = -1e300, zmn = 1e300, zmx = -1e300;
    for (int i = 0; i < 4; ++i) {
        ymn = fmin(ymn, p[i][1]); ymx = fmax(ymx, p[i][1]); zmn = fmin(zmn, p[i][2]); zmx = fmax(zmx, p[i][2]);
    }
    static const int F[4][3] = {{1, 2, 3}, {0, 2, 3}, {0, 1, 3}, {0, 1, 2}};
    for (int f = 0; f < 4; ++f) {                   /* faces crossing kernel lines {y = Y, z = Z} */
        const double *a = p[F[f][0]], *b = p[F[f][1]], *c = p[F[f][2]];
        const double u1[3] = {b[0] - a[0], b[1] - a[1], b[2] - a[2]}, u2[3] = {c[0] - a[0], c[1] - a[1], c[2] - a[2]};
        const double nx = u1[1] * u2[2] - u1[2] * u2[1], ny = u1[2] * u2[0] - u1[0] * u2[2], nz = u1[0] * u2[1] - u1[1] * u2[0];
        if (nx == 0.0) continue;
        const double dd = nx * a[0] + ny * a[1] + nz * a[2];
        for (int j = 0; j < nbr; ++j)
            for (int l = 0; l < nbr; ++l) {
                if (Yb[j] < ymn || Yb[j] > ymx || Zb[l] < zmn || Zb[l] > zmx) continue;  /* line misses the tet */
                const double xc = (dd - ny * Yb[j] - nz * Zb[l]) / nx;
                if (xc > lo && xc < hi) br[nb++] = xc;
            }
    }
    qsort(br, nb, sizeof(double), cmp_d);
    for (int sl = 0; sl + 1 < nb; ++sl) {
        const double a = br[sl], b = br[sl + 1];
        if (!(b > a)) continue;
        for (int ix = 0; ix < P->n; ++ix) {
            const double xs = a + 0.5 * (b - a) * (1.0 + P->gx[ix]);
            const double wx = 0.5 * (b - a) * P->gw[ix];
            double py[4], pz[4];
            const int m = tet_section(p, xs, py, pz);
            if (m < 3) continue;
            double area = 0.0;
            const double s2 = section_integral(P, t, xs, shift[0], shift[1], shift[2], x[1], x[2], py, pz, m, Yb, Zb, &area);
            nadd3(acc, wx * oracle_kernel(k, P->kc, (xs - x[0]) / h) * s2);
            nadd3(vol, wx * area);
        }
    }
}

/* u*(x) at np points (pts np x 3).  periodic: bit d = axis d periodic on domain[d]..domain[d+3].
 * vol_out (nullable): per point the volume of all integrated pieces (W^3 when the mesh covers
 * the stencil).  n: Gauss-Legendre points per direction, nodes gx / weights gw on [-1, 1]. */
int oracle_siac_eval3(int k, double h, int periodic, const double *domain, const double *V, long nv, const int *T,
                      long nt, int field_mode, const double *field, int field_deg, const double *kc, int n,
                      const double *gx, const double *gw, const double *pts, long np, double *out, double *vol_out,
                      int nthreads)
{
    (void)nv;
    if (k < 1 || k > MAXK3 || n < 1 || n > 64) return -1;
    prob3 P = {k, h, kc, V, T, nt, field_mode, field, field_deg, n, gx, gw};
    const double W = (3 * k + 1) * h;
    double L[3];
    for (int d = 0; d < 3; ++d) L[d] = domain[d + 3] - domain[d];
    double *bb = (double *)malloc(sizeof(double) * 6 * (nt > 0 ? nt : 1));
    for (long t = 0; t < nt; ++t)
        for (int d = 0; d < 3; ++d) {
            double lo = 1e300, hi = -1e300;
            for (int i = 0; i < 4; ++i) {
                const double v = V[3 * (long)T[4 * t + i] + d];
                lo = fmin(lo, v); hi = fmax(hi, v);
            }
            bb[6 * t + d] = lo; bb[6 * t + 3 + d] = hi;
        }
#ifdef _OPENMP
    if (nthreads > 0) omp_set_num_threads(nthreads);
#else
    (void)nthreads;
#endif
#pragma omp parallel for schedule(dynamic, 1)
    for (long p = 0; p < np; ++p) {
        double x[3];
        for (int d = 0; d < 3; ++d) {
            x[d] = pts[3 * p + d];
            if (periodic & (1 << d)) x[d] = domain[d] + (x[d] - domain[d]) - L[d] * floor((x[d] - domain[d]) / L[d]);
        }
        nsum3 acc = {0, 0}, vol = {0, 0};
        const int r0 = (periodic & 1) ? 1 : 0, r1 = (periodic & 2) ? 1 : 0, r2 = (periodic & 4) ? 1 : 0;
        for (int i = -r0; i <= r0; ++i)
            for (int j = -r1; j <= r1; ++j)
                for (int l = -r2; l <= r2; ++l) {
                    const double s[3] = {i * L[0], j * L[1], l * L[2]};
                    for (long t = 0; t < nt; ++t) {
                        int out_of = 0;
                        for (int d = 0; d < 3; ++d)
                            if (bb[6 * t + 3 + d] + s[d] <= x[d] - 0.5 * W || bb[6 * t + d] + s[d] >= x[d] + 0.5 * W) out_of = 1;
                        if (!out_of) pair_integral3(&P, t, s, x, &acc, &vol);
                    }
                }
        out[p] = (acc.s + acc.c) / (h * h * h);
        if (vol_out) vol_out[p] = vol.s + vol.c;
    }
    free(bb);
    return 0;
}
