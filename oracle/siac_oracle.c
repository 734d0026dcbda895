/*
 * siac_oracle.c -- TEST INFRASTRUCTURE ONLY.  The plain, slow CPU oracle for the SIAC
 * post-processor.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  The product path (include/siac.h,
 * paper_conf_sc_0007k13_b200/csrc) shares no code with it.
 *
 * What it computes (§2.2, Eq. (1), and Eq. (2)):
 *
 *     u*(x) = (1/h^2) sum_T sum_{s in S} \int_{T+s} K((y1-x1)/h) K((y2-x2)/h) u_T(y-s) dy
 *
 * with K(t) = sum_{g=0}^{2k} c_g psi_{k+1}(t - x_g), x_g = -k + g,
 * psi_{k+1} the centred B-spline of order k+1 (degree k) on unit knots, S the periodic
 * image shifts ("the stencil ... wraps around the domain for periodic
 * solutions") and c_g supplied by oracle/__init__.py (exact rational moment solve).
 *
 * How: the paper computes the integral "exactly" by splitting each triangle into pieces
 * "over which there is no break in regularity" (L236-249).  This oracle uses a different
 * exact split than the GPU path (which clips with Sutherland-Hodgman and fans into
 * sub-triangles): vertical SLABS between consecutive x-breakpoints (triangle vertices,
 * kernel x-breaklines, and the x where triangle edges cross kernel y-breaklines), each
 * slab cut into STRIPS by the kernel y-breaklines.  On each strip the integrand is a
 * polynomial; a tensor Gauss-Legendre rule on the map y2 = g(x) + (q(x)-g(x))(1+eta)/2 is
 * exact for it when nx, ny satisfy the degree bounds computed in oracle/__init__.py.
 * K is evaluated by the Cox-de Boor recursion on its knots, u_T by the Jacobi
 * three-term recurrences of the Dubiner basis.  Sums are Neumaier-compensated.
 */
#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define MAXK 8
#define MAXB ((MAXK + 1) * (MAXK + 2) / 2)
#define MAXPOLY 24

/* ------------------------------------------------------------------ B-spline, kernel */

/* Centred cardinal B-spline of order k+1 (degree k), knots -(k+1)/2 + j, j = 0..k+1,
 * by the Cox-de Boor recursion ("psi^(k+1) is the B-spline of order k+1"). */
double oracle_bspline(int k, double t)
{
    double knot[MAXK + 3];
    double B[MAXK + 2];
    for (int j = 0; j <= k + 1; ++j) knot[j] = -0.5 * (k + 1) + j;
    for (int j = 0; j <= k; ++j) B[j] = (knot[j] <= t && t < knot[j + 1]) ? 1.0 : 0.0;
    for (int d = 1; d <= k; ++d) {
        for (int j = 0; j + d <= k; ++j) {
            double left = (t - knot[j]) / (knot[j + d] - knot[j]) * B[j];
            double right = (knot[j + d + 1] - t) / (knot[j + d + 1] - knot[j + 1]) * B[j + 1];
            B[j] = left + right;
        }
    }
    return B[0];
}

/* K(t) = sum_{g=0}^{2k} c_g psi(t - x_g), x_g = -r/2 + g, r = 2k. */
double oracle_kernel(int k, const double *c, double t)
{
    double s = 0.0;
    for (int g = 0; g <= 2 * k; ++g) s += c[g] * oracle_bspline(k, t - (double)(g - k));
    return s;
}

/* The one-sided kernel of ref [21] (reading R4): the same 2k+1
 * B-splines with every node shifted by lambda, x_g = -k + g + lambda, and coefficients c_g
 * (supplied by oracle/__init__.py: the exact solution of the moment system at these nodes).
 * lambda = 0 is the symmetric kernel. */
double oracle_kernel_shifted(int k, const double *c, double lam, double t)
{
    double s = 0.0;
    for (int g = 0; g <= 2 * k; ++g) s += c[g] * oracle_bspline(k, t - ((double)(g - k) + lam));
    return s;
}

/* ------------------------------------------------------------------ Dubiner basis */

/* Jacobi P_n^(alpha,0)(x) by the three-term recurrence (Abramowitz & Stegun 22.7.1). */
static double jacobi_a0(int n, double alpha, double x)
{
    if (n == 0) return 1.0;
    double p0 = 1.0;
    double p1 = (alpha + 1.0) + (alpha + 2.0) * (x - 1.0) / 2.0;
    for (int m = 1; m < n; ++m) {
        double a1 = 2.0 * (m + 1) * (m + alpha + 1) * (2 * m + alpha);
        double a2 = (2 * m + alpha + 1) * (alpha * alpha);
        double a3 = (2 * m + alpha) * (2 * m + alpha + 1) * (2 * m + alpha + 2);
        double a4 = 2.0 * (m + alpha) * m * (2 * m + alpha + 2);
        double p2 = ((a2 + a3 * x) * p1 - a4 * p0) / a1;
        p0 = p1;
        p1 = p2;
    }
    return p1;
}

/* Orthonormal Dubiner modes on {xi,eta >= -1, xi+eta <= 0}, ordered by total degree
 * then q (SURVEY §8(b) basis convention, Q8):
 *   phi_pq = sqrt((2p+1)(p+q+1)/2) * [((1-eta)/2)^p P_p(a)] * P_q^(2p+1,0)(eta),
 *   a = 2(1+xi)/(1-eta) - 1.
 * The bracket is the collapsed Legendre polynomial Q_p, computed without dividing by
 * (1-eta): Q_0 = 1, Q_1 = xi + (1+eta)/2,
 *   (n+1) Q_{n+1} = (2n+1) (xi + (1+eta)/2) Q_n - n ((1-eta)/2)^2 Q_{n-1}. */
void oracle_dubiner(int k, double xi, double eta, double *phi)
{
    double Q[MAXK + 2];
    double ab = xi + 0.5 * (1.0 + eta);   /* a * (1-eta)/2 */
    double b = 0.5 * (1.0 - eta);
    Q[0] = 1.0;
    if (k >= 1) Q[1] = ab;
    for (int n = 1; n < k; ++n) Q[n + 1] = ((2 * n + 1) * ab * Q[n] - n * b * b * Q[n - 1]) / (n + 1);
    int idx = 0;
    for (int n = 0; n <= k; ++n) {
        for (int q = 0; q <= n; ++q) {
            int p = n - q;
            double norm = sqrt((2.0 * p + 1.0) * (p + q + 1.0) / 2.0);
            phi[idx++] = norm * Q[p] * jacobi_a0(q, 2.0 * p + 1.0, eta);
        }
    }
}

/* ------------------------------------------------------------------ compensated sum */

typedef struct { double s, c; } nsum;
static inline void nadd(nsum *a, double v)
{
    double t = a->s + v;
    if (fabs(a->s) >= fabs(v)) a->c += (a->s - t) + v;
    else a->c += (v - t) + a->s;
    a->s = t;
}

/* ------------------------------------------------------------------ problem */

typedef struct {
    int k;
    double h;
    const double *kc;            /* 2k+1 kernel coefficients */
    const double *V;             /* nv x 2 */
    const int *T;                /* nt x 3 */
    long nt;
    int field_mode;              /* 0: dG Dubiner modes (nt x nb); 1: global polynomial;
                                    2: per-triangle monomials r^a s^b of the unit reference
                                       triangle (nt x nb, ordered by a+b, then b) */
    const double *field;
    int field_deg;               /* mode 1: coefficients a[i*(deg+1)+j] of y1^i y2^j */
    int nx, ny;                  /* Gauss-Legendre sizes in x and along the strip */
    const double *gx, *gwx, *gy, *gwy;
} problem;

/* u at physical point y (already shifted back into the mesh: y = y_image - s) on triangle t */
static double field_value(const problem *P, long t, double y1, double y2)
{
    if (P->field_mode == 1) {
        double s = 0.0;
        int d = P->field_deg;
        for (int i = 0; i <= d; ++i)
            for (int j = 0; j <= d; ++j)
                s += P->field[i * (d + 1) + j] * pow(y1, i) * pow(y2, j);
        return s;
    }
    const double *v0 = P->V + 2 * (long)P->T[3 * t + 0];
    const double *v1 = P->V + 2 * (long)P->T[3 * t + 1];
    const double *v2 = P->V + 2 * (long)P->T[3 * t + 2];
    /* y = v0 + r (v1-v0) + s (v2-v0), xi = 2r-1, eta = 2s-1 (vertices 0,1,2 -> (-1,-1),(1,-1),(-1,1)) */
    double a11 = v1[0] - v0[0], a12 = v2[0] - v0[0];
    double a21 = v1[1] - v0[1], a22 = v2[1] - v0[1];
    double det = a11 * a22 - a12 * a21;
    double d1 = y1 - v0[0], d2 = y2 - v0[1];
    double r = (a22 * d1 - a12 * d2) / det;
    double s = (-a21 * d1 + a11 * d2) / det;
    double phi[MAXB];
    int nb = (P->k + 1) * (P->k + 2) / 2;
    if (P->field_mode == 2) {            /* phi_i = r^(n-b) s^b, i by n = a+b then b */
        int i = 0;
        for (int n = 0; n <= P->k; ++n)
            for (int b = 0; b <= n; ++b) phi[i++] = pow(r, n - b) * pow(s, b);
    } else {
        oracle_dubiner(P->k, 2.0 * r - 1.0, 2.0 * s - 1.0, phi);
    }
    const double *c = P->field + (long)nb * t;
    double u = 0.0;
    for (int i = 0; i < nb; ++i) u += c[i] * phi[i];
    return u;
}

static int cmp_double(const void *a, const void *b)
{
    double x = *(const double *)a, y = *(const double *)b;
    return (x > y) - (x < y);
}

/* A strip boundary: y = m*x + q (a triangle edge line) or y = q (a kernel breakline). */
typedef struct { double m, q; } line;
static inline double line_at(line L, double x) { return L.m * x + L.q; }

/* Integral of Kx((y1-x1)/h) Ky((y2-x2)/h) u_t(y - s) over (T_t + s) for point x, with
 * Kx / Ky the kernels of coefficients kcx / kcy and node shifts lamx / lamy (0, P->kc: the
 * symmetric kernel).  Adds the integral to *acc and the covered area to *area. */
static void pair_integral(const problem *P, long t, double sx, double sy,
                          double x1, double x2, const double *kcx, const double *kcy,
                          double lamx, double lamy, nsum *acc, nsum *area)
{
    const int k = P->k;
    const double h = P->h;
    const int nbr = 3 * k + 2;                /* breaklines t_m = -(3k+1)/2 + lam + m, m = 0..3k+1 */
    double Xb[3 * MAXK + 2], Yb[3 * MAXK + 2];
    for (int m = 0; m < nbr; ++m) {
        double tm = -0.5 * (3 * k + 1) + m;
        Xb[m] = x1 + h * (tm + lamx);
        Yb[m] = x2 + h * (tm + lamy);
    }
    double px[3], py[3];
    for (int i = 0; i < 3; ++i) {
        px[i] = P->V[2 * (long)P->T[3 * t + i] + 0] + sx;
        py[i] = P->V[2 * (long)P->T[3 * t + i] + 1] + sy;
    }
    double xmin = fmin(px[0], fmin(px[1], px[2])), xmax = fmax(px[0], fmax(px[1], px[2]));
    double lo_x = fmax(xmin, Xb[0]), hi_x = fmin(xmax, Xb[nbr - 1]);
    if (!(lo_x < hi_x)) return;

    /* x-breakpoints: the 2 ends, <= 3 vertices, <= nbr kernel x-breaklines and <= 3 nbr
     * crossings of the 3 edges with the nbr kernel y-breaklines */
    double bx[5 + 4 * (3 * MAXK + 2)];
    int nbx = 0;
    bx[nbx++] = lo_x;
    bx[nbx++] = hi_x;
    for (int i = 0; i < 3; ++i)
        if (px[i] > lo_x && px[i] < hi_x) bx[nbx++] = px[i];
    for (int m = 0; m < nbr; ++m)
        if (Xb[m] > lo_x && Xb[m] < hi_x) bx[nbx++] = Xb[m];
    for (int e = 0; e < 3; ++e) {
        double ax = px[e], ay = py[e], bxx = px[(e + 1) % 3], byy = py[(e + 1) % 3];
        if (ay == byy) continue;
        for (int m = 0; m < nbr; ++m) {
            double Y = Yb[m];
            if ((Y > ay && Y < byy) || (Y < ay && Y > byy)) {
                double xc = ax + (Y - ay) / (byy - ay) * (bxx - ax);
                if (xc > lo_x && xc < hi_x) bx[nbx++] = xc;
            }
        }
    }
    qsort(bx, nbx, sizeof(double), cmp_double);

    for (int sl = 0; sl + 1 < nbx; ++sl) {
        double a = bx[sl], b = bx[sl + 1];
        if (!(b > a)) continue;
        double xm = 0.5 * (a + b);
        /* the two non-vertical edges spanning [a, b] bound the triangle's cross-section */
        line bot = {0, 0}, top = {0, 0};
        int nspan = 0;
        double ylo = 0, yhi = 0;
        for (int e = 0; e < 3; ++e) {
            double ax = px[e], ay = py[e], bxx = px[(e + 1) % 3], byy = py[(e + 1) % 3];
            double el = fmin(ax, bxx), er = fmax(ax, bxx);
            if (!(el < er) || el > a || er < b) continue;
            line L;
            L.m = (byy - ay) / (bxx - ax);
            L.q = ay - L.m * ax;
            double ym = line_at(L, xm);
            if (nspan == 0) { bot = top = L; ylo = yhi = ym; }
            else {
                if (ym < ylo) { bot = L; ylo = ym; }
                if (ym > yhi) { top = L; yhi = ym; }
            }
            ++nspan;
        }
        if (nspan < 2 || !(yhi > ylo)) continue;
        /* strip boundaries: bottom edge, interior kernel y-breaklines, top edge, clipped to
         * the stencil's y-extent [Yb[0], Yb[nbr-1]] */
        line bnd[3 * MAXK + 4];
        int nb = 0;
        line c0 = bot;
        if (Yb[0] > ylo) { c0.m = 0; c0.q = Yb[0]; }
        if (c0.m == 0 && c0.q >= yhi) continue;
        bnd[nb++] = c0;
        for (int m = 1; m < nbr - 1; ++m)
            if (Yb[m] > ylo && Yb[m] < yhi && Yb[m] > Yb[0]) { bnd[nb].m = 0; bnd[nb].q = Yb[m]; ++nb; }
        line c1 = top;
        if (Yb[nbr - 1] < yhi) { c1.m = 0; c1.q = Yb[nbr - 1]; }
        if (line_at(c1, xm) <= line_at(bnd[0], xm)) continue;
        bnd[nb++] = c1;

        for (int st = 0; st + 1 < nb; ++st) {
            line g = bnd[st], q = bnd[st + 1];
            for (int i = 0; i < P->nx; ++i) {
                double x = a + 0.5 * (b - a) * (1.0 + P->gx[i]);
                double wx = 0.5 * (b - a) * P->gwx[i];
                double yg = line_at(g, x), yq = line_at(q, x);
                double jy = 0.5 * (yq - yg);
                double kx = oracle_kernel_shifted(k, kcx, lamx, (x - x1) / h);
                nadd(area, wx * 2.0 * jy);
                for (int j = 0; j < P->ny; ++j) {
                    double y = yg + jy * (1.0 + P->gy[j]);
                    double ky = oracle_kernel_shifted(k, kcy, lamy, (y - x2) / h);
                    double u = field_value(P, t, x - sx, y - sy);
                    nadd(acc, wx * jy * P->gwy[j] * kx * ky * u);
                }
            }
        }
    }
}

/* ------------------------------------------------------------------ driver */

/* Evaluate u*(x) at np points.  periodic: bit0 x, bit1 y.  domain = {x0, y0, x1, y1}.
 * use_grid = 0: every triangle and every image shift is tested (brute force);
 * use_grid = 1: triangles are found through a bucket grid (each triangle is listed in every
 * bucket its bounding box touches; duplicates are skipped with a per-query stamp).
 * area_out (nullable): per point, the area of all integrated strips (the stencil area W^2
 * when the mesh covers the stencil).
 * pt_lam, pt_coef (nullable, the one-sided kernel): per point the node shifts (lambda_x,
 * lambda_y) and the 2 x (2k+1) coefficients (x kernel, then y kernel); NULL = the symmetric
 * kernel kc on both axes.  Returns 0 on success. */
int oracle_siac_eval(int k, double h, int periodic, const double *domain,
                     const double *V, long nv, const int *T, long nt,
                     int field_mode, const double *field, int field_deg,
                     const double *kc, int nx, const double *gx, const double *gwx,
                     int ny, const double *gy, const double *gwy,
                     const double *pts, long np, double *out, double *area_out,
                     int use_grid, int nthreads, const double *pt_lam, const double *pt_coef)
{
    (void)nv;
    if (k < 1 || k > MAXK || nx > 64 || ny > 64) return -1;
    problem P = {k, h, kc, V, T, nt, field_mode, field, field_deg, nx, ny, gx, gwx, gy, gwy};
    const double Lx = domain[2] - domain[0], Ly = domain[3] - domain[1];
    const double W = (3 * k + 1) * h;            /* Supp{K} = (3k+1)h */
    const int sxr = (periodic & 1) ? 1 : 0, syr = (periodic & 2) ? 1 : 0;

    /* triangle bounding boxes */
    double *bb = (double *)malloc(sizeof(double) * 4 * (nt > 0 ? nt : 1));
    for (long t = 0; t < nt; ++t) {
        double x0 = 1e300, y0 = 1e300, x1 = -1e300, y1 = -1e300;
        for (int i = 0; i < 3; ++i) {
            double x = V[2 * (long)T[3 * t + i]], y = V[2 * (long)T[3 * t + i] + 1];
            x0 = fmin(x0, x); x1 = fmax(x1, x); y0 = fmin(y0, y); y1 = fmax(y1, y);
        }
        bb[4 * t] = x0; bb[4 * t + 1] = y0; bb[4 * t + 2] = x1; bb[4 * t + 3] = y1;
    }
    /* bucket grid over the domain, bucket size ~ h */
    int gnx = 1, gny = 1;
    long *bstart = NULL, *blist = NULL;
    if (use_grid) {
        gnx = (int)fmax(1.0, floor(Lx / h));
        gny = (int)fmax(1.0, floor(Ly / h));
        long ncell = (long)gnx * gny;
        bstart = (long *)calloc(ncell + 1, sizeof(long));
        for (int pass = 0; pass < 2; ++pass) {
            long *fill = pass ? (long *)calloc(ncell, sizeof(long)) : NULL;
            for (long t = 0; t < nt; ++t) {
                int i0 = (int)floor((bb[4 * t] - domain[0]) / Lx * gnx), i1 = (int)floor((bb[4 * t + 2] - domain[0]) / Lx * gnx);
                int j0 = (int)floor((bb[4 * t + 1] - domain[1]) / Ly * gny), j1 = (int)floor((bb[4 * t + 3] - domain[1]) / Ly * gny);
                i0 = i0 < 0 ? 0 : (i0 >= gnx ? gnx - 1 : i0); i1 = i1 < 0 ? 0 : (i1 >= gnx ? gnx - 1 : i1);
                j0 = j0 < 0 ? 0 : (j0 >= gny ? gny - 1 : j0); j1 = j1 < 0 ? 0 : (j1 >= gny ? gny - 1 : j1);
                for (int j = j0; j <= j1; ++j)
                    for (int i = i0; i <= i1; ++i) {
                        long c = (long)j * gnx + i;
                        if (pass == 0) bstart[c + 1]++;
                        else blist[bstart[c] + fill[c]++] = t;
                    }
            }
            if (pass == 0) {
                for (long c = 0; c < ncell; ++c) bstart[c + 1] += bstart[c];
                blist = (long *)malloc(sizeof(long) * (bstart[ncell] > 0 ? bstart[ncell] : 1));
            } else free(fill);
        }
    }

#ifdef _OPENMP
    if (nthreads > 0) omp_set_num_threads(nthreads);
#else
    (void)nthreads;
#endif
#pragma omp parallel
    {
        long *stamp = use_grid ? (long *)calloc(nt > 0 ? nt : 1, sizeof(long)) : NULL;
        long query = 0;
#pragma omp for schedule(dynamic, 4)
        for (long p = 0; p < np; ++p) {
            double x1 = pts[2 * p], x2 = pts[2 * p + 1];
            /* periodic axes: wrap the point into [x0, x1) (the convolution is periodic) */
            if (periodic & 1) x1 = domain[0] + (x1 - domain[0]) - Lx * floor((x1 - domain[0]) / Lx);
            if (periodic & 2) x2 = domain[1] + (x2 - domain[1]) - Ly * floor((x2 - domain[1]) / Ly);
            nsum acc = {0, 0}, area = {0, 0};
            const double lamx = pt_lam ? pt_lam[2 * p] : 0.0, lamy = pt_lam ? pt_lam[2 * p + 1] : 0.0;
            const double *kcx = pt_coef ? pt_coef + (long)2 * (2 * k + 1) * p : kc;
            const double *kcy = pt_coef ? kcx + (2 * k + 1) : kc;
            for (int si = -sxr; si <= sxr; ++si)
                for (int sj = -syr; sj <= syr; ++sj) {
                    double sx = si * Lx, sy = sj * Ly;
                    /* stencil box (moved by the node shift) pulled back by the image shift:
                     * images T+s meet the box iff T meets box-s */
                    double qx0 = x1 + h * lamx - 0.5 * W - sx, qx1 = x1 + h * lamx + 0.5 * W - sx;
                    double qy0 = x2 + h * lamy - 0.5 * W - sy, qy1 = x2 + h * lamy + 0.5 * W - sy;
                    if (!use_grid) {
                        for (long t = 0; t < nt; ++t) {
                            if (bb[4 * t + 2] <= qx0 || bb[4 * t] >= qx1 || bb[4 * t + 3] <= qy0 || bb[4 * t + 1] >= qy1) continue;
                            pair_integral(&P, t, sx, sy, x1, x2, kcx, kcy, lamx, lamy, &acc, &area);
                        }
                    } else {
                        ++query;
                        int i0 = (int)floor((qx0 - domain[0]) / Lx * gnx), i1 = (int)floor((qx1 - domain[0]) / Lx * gnx);
                        int j0 = (int)floor((qy0 - domain[1]) / Ly * gny), j1 = (int)floor((qy1 - domain[1]) / Ly * gny);
                        i0 = i0 < 0 ? 0 : i0; j0 = j0 < 0 ? 0 : j0;
                        i1 = i1 >= gnx ? gnx - 1 : i1; j1 = j1 >= gny ? gny - 1 : j1;
                        for (int j = j0; j <= j1; ++j)
                            for (int i = i0; i <= i1; ++i) {
                                long c = (long)j * gnx + i;
                                for (long e = bstart[c]; e < bstart[c + 1]; ++e) {
                                    long t = blist[e];
                                    if (stamp[t] == query) continue;
                                    stamp[t] = query;
                                    if (bb[4 * t + 2] <= qx0 || bb[4 * t] >= qx1 || bb[4 * t + 3] <= qy0 || bb[4 * t + 1] >= qy1) continue;
                                    pair_integral(&P, t, sx, sy, x1, x2, kcx, kcy, lamx, lamy, &acc, &area);
                                }
                            }
                    }
                }
            out[p] = (acc.s + acc.c) / (h * h);
            if (area_out) area_out[p] = area.s + area.c;
        }
        free(stamp);
    }
    free(bb);
    free(bstart);
    free(blist);
    return 0;
}

/* exported for pins: K(t) at many t */
void oracle_kernel_many(int k, const double *c, const double *t, long n, double *out)
{
    for (long i = 0; i < n; ++i) out[i] = oracle_kernel(k, c, t[i]);
}

void oracle_kernel_shifted_many(int k, const double *c, double lam, const double *t, long n, double *out)
{
    for (long i = 0; i < n; ++i) out[i] = oracle_kernel_shifted(k, c, lam, t[i]);
}

void oracle_bspline_many(int k, const double *t, long n, double *out)
{
    for (long i = 0; i < n; ++i) out[i] = oracle_bspline(k, t[i]);
}

void oracle_dubiner_many(int k, const double *xi, const double *eta, long n, double *out)
{
    int nb = (k + 1) * (k + 2) / 2;
    for (long i = 0; i < n; ++i) oracle_dubiner(k, xi[i], eta[i], out + (long)nb * i);
}
