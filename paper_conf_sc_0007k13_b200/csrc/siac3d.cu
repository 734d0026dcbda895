// siac3d.cu -- SIAC filtering on TETRAHEDRAL meshes (PAPER.md L946-950:
// "extension of these ideas to 3D over unstructured tetrahedral meshes"), the 3D form of
// Eq. (1): u*(x) = (1/h^3) \int K((y1-x1)/h) K((y2-x2)/h) K((y3-x3)/h) u_h(y) dy (the stencil is
// the tensor product of 1D kernels, L212-214), computed exactly as in Eq. (2): every tetrahedron
// the stencil touches is cut by the kernel breakplanes into pieces inside single kernel cells,
// and each piece is integrated by a rule exact for the integrand's degree 4k (K K K u).
//
// B200 design (direct method; the 2D library's spline-jump decomposition is not carried over):
//   siac3_create: H2D of V, T, modes; k_prep3 (per-tetrahedron record: vertices, inverse affine
//     map, modes in the reference monomial basis; bounding box; anchor cell = bbox-min cell of a
//     uniform grid); CUB radix sort by anchor cell; k_gather3; CSR cell_start.
//   siac3_eval_async: k_point_keys3 (periodic wrap, 30-bit Morton key) + CUB sort -> k_eval3w
//     (default), one warp per 32-point tile in Morton order: the cells of the tile's stencil box
//     (extended by the largest tetrahedron extent), box tests per candidate image, then per lane a
//     depth-first stack that splits the tetrahedron by every kernel plane strictly crossing it (a
//     plane cut yields a tetrahedron plus a prism, or two prisms; prisms are cut into 3
//     tetrahedra) until every piece lies in one kernel cell; the pieces are queued in shared
//     memory and integrated 32 at a time by a collapsed Gauss(-Jacobi) rule; one write per point.
//     k_eval3 (schedule 1) is the thread-per-point mapping of the same steps.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <functional>
#include <string>
#include <vector>

#include <cub/device/device_radix_sort.cuh>

#include "../../include/siac.h"
#include "siac_internal.h"
#include "siac_math.h"

namespace {

struct Fail3 {
    siac_status st;
    std::string msg;
};
#define CK3(call)                                                                              \
    do {                                                                                       \
        cudaError_t e_ = (call);                                                               \
        if (e_ != cudaSuccess)                                                                 \
            throw Fail3{SIAC_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e_)};       \
    } while (0)
inline void need3(bool ok, const char *msg) {
    if (!ok) throw Fail3{SIAC_EINVAL, std::string(msg)};
}

constexpr int MAXQ3 = 343;        // quadrature points (k = 3: 7^3)
constexpr int STACK3 = 64;        // depth-first split stack (tetrahedra); overflow is reported

template <int K> struct Rec3 {
    static constexpr int NB = (K + 1) * (K + 2) * (K + 3) / 6;
    static constexpr int OFF_AINV = 12;       // rst = Ainv (y - v0), row-major 3x3
    static constexpr int OFF_C = 21;          // modes, order: n = a+b+c, then c, then b
    static constexpr int RS = (OFF_C + NB + 1) & ~1;
};
inline int rec3_size(int k) {
    const int nb = (k + 1) * (k + 2) * (k + 3) / 6;
    return (21 + nb + 1) & ~1;
}

struct Prep3Args {
    const double *V;
    const int *T;
    const double *C;
    int64_t nt;
    int nb, rs;
    double x0[3], cell[3];
    int nc[3];
    double *rec;
    double *bbox;     // nt x 6: lo xyz, hi xyz
    unsigned long long *key;
    int *idx;
    int *bad;         // validation flags (bit 0: index out of range, bit 1: degenerate, bit 2: non-finite)
    int64_t nv;
};

__global__ void k_prep3(Prep3Args a) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= a.nt) return;
    int vi[4];
    int bad = 0;
    for (int i = 0; i < 4; ++i) {
        vi[i] = a.T[4 * t + i];
        if (vi[i] < 0 || vi[i] >= a.nv) { bad |= 1; vi[i] = 0; }
    }
    double v[4][3];
    for (int i = 0; i < 4; ++i)
        for (int d = 0; d < 3; ++d) {
            v[i][d] = a.V[3 * (int64_t)vi[i] + d];
            if (!isfinite(v[i][d])) bad |= 4;
        }
    double *r = a.rec + (int64_t)a.rs * t;
    for (int i = 0; i < 4; ++i)
        for (int d = 0; d < 3; ++d) r[3 * i + d] = v[i][d];
    // A = [v1-v0, v2-v0, v3-v0] (columns); Ainv by the adjugate
    double A[3][3];
    for (int d = 0; d < 3; ++d) { A[d][0] = v[1][d] - v[0][d]; A[d][1] = v[2][d] - v[0][d]; A[d][2] = v[3][d] - v[0][d]; }
    const double c00 = A[1][1] * A[2][2] - A[1][2] * A[2][1], c01 = A[1][2] * A[2][0] - A[1][0] * A[2][2],
                 c02 = A[1][0] * A[2][1] - A[1][1] * A[2][0];
    const double det = A[0][0] * c00 + A[0][1] * c01 + A[0][2] * c02;
    double scale = 0.0;
    for (int i = 0; i < 3; ++i)
        for (int j = 0; j < 3; ++j) scale = fmax(scale, fabs(A[i][j]));
    if (!(fabs(det) > 1e-14 * scale * scale * scale)) bad |= 2;
    const double id = 1.0 / det;
    double *ai = r + 12;
    ai[0] = c00 * id; ai[1] = (A[0][2] * A[2][1] - A[0][1] * A[2][2]) * id; ai[2] = (A[0][1] * A[1][2] - A[0][2] * A[1][1]) * id;
    ai[3] = c01 * id; ai[4] = (A[0][0] * A[2][2] - A[0][2] * A[2][0]) * id; ai[5] = (A[0][2] * A[1][0] - A[0][0] * A[1][2]) * id;
    ai[6] = c02 * id; ai[7] = (A[0][1] * A[2][0] - A[0][0] * A[2][1]) * id; ai[8] = (A[0][0] * A[1][1] - A[0][1] * A[1][0]) * id;
    for (int j = 0; j < a.nb; ++j) {
        const double c = a.C[(int64_t)a.nb * t + j];
        if (!isfinite(c)) bad |= 4;
        r[21 + j] = c;
    }
    for (int j = 21 + a.nb; j < a.rs; ++j) r[j] = 0.0;
    double lo[3], hi[3];
    unsigned long long key = 0;
    unsigned cidx[3];
    for (int d = 0; d < 3; ++d) {
        lo[d] = fmin(fmin(v[0][d], v[1][d]), fmin(v[2][d], v[3][d]));
        hi[d] = fmax(fmax(v[0][d], v[1][d]), fmax(v[2][d], v[3][d]));
        int c = (int)floor((lo[d] - a.x0[d]) / a.cell[d]);
        c = c < 0 ? 0 : (c >= a.nc[d] ? a.nc[d] - 1 : c);
        cidx[d] = (unsigned)c;
    }
    key = ((unsigned long long)cidx[2] * a.nc[1] + cidx[1]) * a.nc[0] + cidx[0];
    for (int d = 0; d < 3; ++d) { a.bbox[6 * t + d] = lo[d]; a.bbox[6 * t + 3 + d] = hi[d]; }
    a.key[t] = key;
    a.idx[t] = (int)t;
    if (bad) atomicOr(a.bad, bad);
}

__global__ void k_gather3(const double *rec_u, const double *bb_u, const int *idx, int64_t nt, int rs, double *rec,
                          double *bbox) {
    const int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= nt) return;
    const int t = idx[s];
    for (int j = 0; j < rs; ++j) rec[(int64_t)rs * s + j] = rec_u[(int64_t)rs * t + j];
    for (int j = 0; j < 6; ++j) bbox[6 * s + j] = bb_u[6 * t + j];
}

__global__ void k_cell_start3(const unsigned long long *keys, int64_t nt, int64_t ncell, int *cs) {
    const int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (c > ncell) return;
    int64_t lo = 0, hi = nt;
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if ((int64_t)keys[mid] < c) lo = mid + 1;
        else hi = mid;
    }
    cs[c] = (int)lo;
}

__device__ __forceinline__ unsigned spread10(unsigned v) {
    v &= 0x3ff;
    v = (v | (v << 16)) & 0x030000FF;
    v = (v | (v << 8)) & 0x0300F00F;
    v = (v | (v << 4)) & 0x030C30C3;
    v = (v | (v << 2)) & 0x09249249;
    return v;
}

struct Eval3Args {
    const double *pts;
    const int *perm;
    int64_t np;
    double *out;
    const double *rec;
    const double *bbox;
    const int *cell_start;
    const double *kc;         // (3K+1) x (K+1) kernel cell table
    const double *qr;         // quadrature: nq x 4 (xi, eta, zeta, w), weights sum to 1/6
    int nq;
    double x0[3], L[3], cell[3], ext[3];
    int nc[3];
    int periodic;
    double h, inv_h, hw;
    unsigned long long *cnt;  // pairs, pieces
    int split;                // k_eval3w: warps per point tile (1, 2, 4), each walking a share of the cells
};

__global__ void k_point_keys3(const double *pts, int64_t np, double x0, double y0, double z0, double Lx, double Ly,
                              double Lz, unsigned *key, int *idx) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= np) return;
    const double L[3] = {Lx, Ly, Lz}, o[3] = {x0, y0, z0};
    unsigned c[3];
    for (int d = 0; d < 3; ++d) {
        double u = (pts[3 * i + d] - o[d]) / L[d];
        u = u - floor(u);
        int q = (int)(u * 1024.0);
        c[d] = (unsigned)(q < 0 ? 0 : (q > 1023 ? 1023 : q));
    }
    key[i] = spread10(c[0]) | (spread10(c[1]) << 1) | (spread10(c[2]) << 2);
    idx[i] = (int)i;
}

struct Tet { double p[4][3]; };

template <int K>
__device__ __forceinline__ double horner1(const double *c, double t) {
    double v = c[K];
#pragma unroll
    for (int i = K - 1; i >= 0; --i) v = fma(v, t, c[i]);
    return v;
}

// u at reference coordinates (r, s, t): sum of c_abc r^a s^b t^c, modes by n, then c, then b
template <int K>
__device__ __forceinline__ double umono(const double *c, double r, double s, double t) {
    double rp[K + 1], sp[K + 1], tp[K + 1];
    rp[0] = sp[0] = tp[0] = 1.0;
#pragma unroll
    for (int i = 1; i <= K; ++i) { rp[i] = rp[i - 1] * r; sp[i] = sp[i - 1] * s; tp[i] = tp[i - 1] * t; }
    double u = 0.0;
    int idx = 0;
#pragma unroll
    for (int n = 0; n <= K; ++n)
#pragma unroll
        for (int cc = 0; cc <= n; ++cc)
#pragma unroll
            for (int bb = 0; bb <= n - cc; ++bb, ++idx) u = fma(c[idx], rp[n - bb - cc] * sp[bb] * tp[cc], u);
    return u;
}

// One thread per point.  z-units: z = (y - x) / h, kernel cells [T0 + i, T0 + i + 1].
template <int K, bool COUNT>
__global__ void __launch_bounds__(128) k_eval3(Eval3Args a) {
    using R = Rec3<K>;
    constexpr int NC = 3 * K + 1;
    constexpr double T0 = -0.5 * (3 * K + 1);
    __shared__ double kc[NC * (K + 1)];
    __shared__ double qr[MAXQ3 * 4];
    for (int i = threadIdx.x; i < NC * (K + 1); i += blockDim.x) kc[i] = a.kc[i];
    for (int i = threadIdx.x; i < a.nq * 4; i += blockDim.x) qr[i] = a.qr[i];
    __syncthreads();
    const int64_t sp = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (sp >= a.np) return;
    const int orig = a.perm[sp];
    double x[3];
    for (int d = 0; d < 3; ++d) {
        x[d] = a.pts[3 * (int64_t)orig + d];
        if (a.periodic & (1 << d)) {
            x[d] = x[d] - a.L[d] * floor((x[d] - a.x0[d]) / a.L[d]);
            if (x[d] >= a.x0[d] + a.L[d]) x[d] -= a.L[d];
            if (x[d] < a.x0[d]) x[d] = a.x0[d];
        }
    }
    int lo[3], hi[3];
    for (int d = 0; d < 3; ++d) {
        lo[d] = (int)floor((x[d] - a.hw - a.ext[d] - a.x0[d]) / a.cell[d]) - 1;
        hi[d] = (int)floor((x[d] + a.hw - a.x0[d]) / a.cell[d]) + 1;
        if (!(a.periodic & (1 << d))) { lo[d] = max(lo[d], 0); hi[d] = min(hi[d], a.nc[d] - 1); }
    }
    double acc = 0.0;
    unsigned long long c_pairs = 0, c_pieces = 0;
    bool overflow = false;
    Tet stack[STACK3];
    for (int I2 = lo[2]; I2 <= hi[2]; ++I2)
        for (int I1 = lo[1]; I1 <= hi[1]; ++I1)
            for (int I0 = lo[0]; I0 <= hi[0]; ++I0) {
                const int I[3] = {I0, I1, I2};
                int cidx[3];
                double sh[3];
                for (int d = 0; d < 3; ++d) {
                    cidx[d] = I[d];
                    int q = 0;
                    if (a.periodic & (1 << d)) { cidx[d] = ((I[d] % a.nc[d]) + a.nc[d]) % a.nc[d]; q = (I[d] - cidx[d]) / a.nc[d]; }
                    sh[d] = q * a.L[d];
                }
                const int cell = (cidx[2] * a.nc[1] + cidx[1]) * a.nc[0] + cidx[0];
                const int t0 = __ldg(a.cell_start + cell), t1 = __ldg(a.cell_start + cell + 1);
                for (int t = t0; t < t1; ++t) {
                    const double *bb = a.bbox + 6 * (int64_t)t;
                    bool meet = true;
                    for (int d = 0; d < 3; ++d)
                        meet = meet && (__ldg(bb + d) + sh[d] < x[d] + a.hw) && (__ldg(bb + 3 + d) + sh[d] > x[d] - a.hw);
                    if (!meet) continue;
                    if (COUNT) ++c_pairs;
                    const double *rc = a.rec + (int64_t)R::RS * t;
                    // affine map z -> reference (r, s, t): rst = M z + r0, M = h Ainv, r0 = Ainv (x - sh - v0)
                    double M[9], r0[3], cf[R::NB];
                    double d0[3];
                    for (int d = 0; d < 3; ++d) d0[d] = x[d] - sh[d] - __ldg(rc + d);
                    for (int i = 0; i < 3; ++i) {
                        r0[i] = 0.0;
                        for (int j = 0; j < 3; ++j) {
                            const double ai = __ldg(rc + R::OFF_AINV + 3 * i + j);
                            M[3 * i + j] = a.h * ai;
                            r0[i] = fma(ai, d0[j], r0[i]);
                        }
                    }
#pragma unroll
                    for (int j = 0; j < R::NB; ++j) cf[j] = __ldg(rc + R::OFF_C + j);
                    int ns = 1;
                    for (int i = 0; i < 4; ++i)
                        for (int d = 0; d < 3; ++d) stack[0].p[i][d] = ((__ldg(rc + 3 * i + d) + sh[d]) - x[d]) * a.inv_h;
                    while (ns > 0) {
                        const Tet tt = stack[--ns];
                        bool outside = false;             // a piece outside the support on an axis: K = 0, drop
                        for (int d = 0; d < 3; ++d) {
                            const double mn = fmin(fmin(tt.p[0][d], tt.p[1][d]), fmin(tt.p[2][d], tt.p[3][d]));
                            const double mx = fmax(fmax(tt.p[0][d], tt.p[1][d]), fmax(tt.p[2][d], tt.p[3][d]));
                            outside = outside || mx <= T0 || mn >= -T0;
                        }
                        if (outside) continue;
                        // the first kernel plane strictly crossing the piece (axes x, y, z in order)
                        int ax = -1;
                        double cut = 0.0;
                        for (int d = 0; d < 3 && ax < 0; ++d) {
                            double mn = tt.p[0][d], mx = tt.p[0][d];
                            for (int i = 1; i < 4; ++i) { mn = fmin(mn, tt.p[i][d]); mx = fmax(mx, tt.p[i][d]); }
                            // the first kernel plane (t_0 = T0 .. t_NC = -T0, incl. the support ends)
                            // strictly above the piece's minimum; a plane inside the piece cuts it
                            const double kn = fmax(floor(mn - T0) + 1.0 + T0, T0);
                            if (kn < mx && kn <= -T0) { ax = d; cut = kn; }
                        }
                        if (ax < 0) {
                            // one kernel cell: integrate K K K u over the piece (if inside the support)
                            double cen[3];
                            for (int d = 0; d < 3; ++d) cen[d] = 0.25 * (tt.p[0][d] + tt.p[1][d] + tt.p[2][d] + tt.p[3][d]);
                            int ci[3];
                            bool inside = true;
                            for (int d = 0; d < 3; ++d) {
                                ci[d] = (int)floor(cen[d] - T0);
                                inside = inside && ci[d] >= 0 && ci[d] < NC;
                            }
                            if (!inside) continue;
                            double e[3][3];
                            for (int j = 0; j < 3; ++j)
                                for (int d = 0; d < 3; ++d) e[j][d] = tt.p[j + 1][d] - tt.p[0][d];
                            const double vol6 = fabs(e[0][0] * (e[1][1] * e[2][2] - e[1][2] * e[2][1]) -
                                                     e[0][1] * (e[1][0] * e[2][2] - e[1][2] * e[2][0]) +
                                                     e[0][2] * (e[1][0] * e[2][1] - e[1][1] * e[2][0]));
                            if (!(vol6 > 0.0)) continue;
                            if (COUNT) ++c_pieces;
                            const double *kx = kc + ci[0] * (K + 1), *ky = kc + ci[1] * (K + 1), *kz = kc + ci[2] * (K + 1);
                            double s = 0.0;
                            for (int q = 0; q < a.nq; ++q) {
                                const double xi = qr[4 * q], et = qr[4 * q + 1], ze = qr[4 * q + 2], w = qr[4 * q + 3];
                                double z[3];
                                for (int d = 0; d < 3; ++d) z[d] = fma(ze, e[2][d], fma(et, e[1][d], fma(xi, e[0][d], tt.p[0][d])));
                                const double kv = horner1<K>(kx, z[0] - (T0 + ci[0] + 0.5)) *
                                                  horner1<K>(ky, z[1] - (T0 + ci[1] + 0.5)) *
                                                  horner1<K>(kz, z[2] - (T0 + ci[2] + 0.5));
                                const double rr = fma(M[0], z[0], fma(M[1], z[1], fma(M[2], z[2], r0[0])));
                                const double ss = fma(M[3], z[0], fma(M[4], z[1], fma(M[5], z[2], r0[1])));
                                const double tq = fma(M[6], z[0], fma(M[7], z[1], fma(M[8], z[2], r0[2])));
                                s = fma(w * kv, umono<K>(cf, rr, ss, tq), s);
                            }
                            acc = fma(vol6, s, acc);
                            continue;
                        }
                        // split by the plane z_ax = cut: vertices on the low side (<= cut) and high side
                        int lowi[4], highi[4], nl = 0, nh = 0;
                        for (int i = 0; i < 4; ++i) {
                            if (tt.p[i][ax] <= cut) lowi[nl++] = i;
                            else highi[nh++] = i;
                        }
                        auto isect = [&](int i, int j, double *o) {     // point of edge i-j on the plane
                            const double r = (cut - tt.p[i][ax]) / (tt.p[j][ax] - tt.p[i][ax]);
                            for (int d = 0; d < 3; ++d) o[d] = fma(r, tt.p[j][d] - tt.p[i][d], tt.p[i][d]);
                            o[ax] = cut;
                        };
                        auto push = [&](const double *q0, const double *q1, const double *q2, const double *q3) {
                            if (ns >= STACK3) { overflow = true; return; }
                            {
                                for (int d = 0; d < 3; ++d) {
                                    stack[ns].p[0][d] = q0[d]; stack[ns].p[1][d] = q1[d];
                                    stack[ns].p[2][d] = q2[d]; stack[ns].p[3][d] = q3[d];
                                }
                                ++ns;
                            }
                        };
                        // a prism (triangle a0 a1 a2 -> b0 b1 b2, edges a_i b_i) as 3 tetrahedra
                        auto push_prism = [&](const double *a0, const double *a1, const double *a2, const double *b0,
                                              const double *b1, const double *b2) {
                            push(a0, a1, a2, b2);
                            push(a0, a1, b1, b2);
                            push(a0, b0, b1, b2);
                        };
                        if (nl == 1 || nh == 1) {
                            const int o = nl == 1 ? lowi[0] : highi[0];       // the lone vertex
                            const int *rest = nl == 1 ? highi : lowi;
                            double q[3][3];
                            for (int j = 0; j < 3; ++j) isect(o, rest[j], q[j]);
                            push(tt.p[o], q[0], q[1], q[2]);
                            push_prism(q[0], q[1], q[2], tt.p[rest[0]], tt.p[rest[1]], tt.p[rest[2]]);
                        } else {                                               // 2 - 2
                            const int l0 = lowi[0], l1 = lowi[1], h0 = highi[0], h1 = highi[1];
                            double q00[3], q01[3], q10[3], q11[3];
                            isect(l0, h0, q00); isect(l0, h1, q01); isect(l1, h0, q10); isect(l1, h1, q11);
                            // low side: prism (l0, q00, q01) -> (l1, q10, q11); high side: (h0, q00, q10) -> (h1, q01, q11)
                            push_prism(tt.p[l0], q00, q01, tt.p[l1], q10, q11);
                            push_prism(tt.p[h0], q00, q10, tt.p[h1], q01, q11);
                        }
                    }
                }
            }
    a.out[orig] = acc;
    if (overflow) atomicOr(a.cnt + 2, 1ull);       // the host reports it (siac3_eval / siac3_stats)
    if (COUNT) {
        atomicAdd(a.cnt + 0, c_pairs);
        atomicAdd(a.cnt + 1, c_pieces);
    }
}

// ------------------------------------------------------------------ warp per point tile (default)
// The same decomposition and rule as k_eval3, mapped for SIMD efficiency: one warp owns a tile of
// 32 Morton-consecutive points (each point written by exactly one warp: the buffered stencil of
// PAPER.md L340-347, no races); the candidate tetrahedra of the tile's stencil box are walked
// warp-uniformly (32 boxes tested per step, ballot); for each candidate the lanes whose stencil
// meets it split it depth-first (divergent but cheap), and every leaf piece is appended to the
// warp's shared-memory piece queue; the quadrature -- the dominant cost, (2k+1)^3 points per
// piece -- runs 32 queued pieces at a time, one per lane, in lock step.  Piece values are added
// to their owner points in lane order (deterministic).
// Device-side bounds checks (debug builds: -DSIAC_DEVICE_CHECKS=1, e.g. tools/build_variant.py);
// a failed check prints its condition and traps.
#ifndef SIAC_DEVICE_CHECKS
#define SIAC_DEVICE_CHECKS 0
#endif
#define CHK3(c)                                                                                   \
    do {                                                                                          \
        if (SIAC_DEVICE_CHECKS && !(c)) {                                                         \
            printf("siac3d device check failed: %s (line %d)\n", #c, __LINE__);                   \
            __trap();                                                                             \
        }                                                                                         \
    } while (0)

constexpr int TW3 = 4;            // warps per block
constexpr int QC3 = 64;           // piece queue per warp: < 32 left over + <= 32 new

struct PieceQ3 {
    double p[12][QC3];            // vertex 0 (3) and edges v1-v0, v2-v0, v3-v0 (9), z-units of the owner
    double r0[3][QC3];            // reference coordinates of the owner's z = 0: Ainv (x - shift - v0)
    double vol6[QC3];             // 6 |volume| (z-units)
    int tet[QC3];
    int info[QC3];                // owner lane | cell x << 5 | cell y << 9 | cell z << 13
    double acc[32];               // per-owner sums of the flushed pieces
};

// Pending pieces of the current candidate tetrahedron shared by the warp's lanes: a lane that has
// finished its own pair takes pieces split off by the others (the split work is balanced across the
// warp; a lane's own overflow goes to its local-memory stack).
constexpr int WQ3 = 64;
struct WorkQ3 {
    double p[12][WQ3];            // the 4 vertices (z-units of the owner point)
    int owner[WQ3];               // owner lane
    double r0[3][32];             // per owner lane: reference coordinates of its z = 0 (this candidate)
};

__device__ __forceinline__ unsigned lanemask_lt3() {
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

template <int K>
__device__ __forceinline__ void flush3(const Eval3Args &a, PieceQ3 &Q, const double *kc, const double *qr, int &nq,
                                       int lane) {
    using R = Rec3<K>;
    constexpr double T0 = -0.5 * (3 * K + 1);
    const int take = min(nq, 32);
    int key = 32;                 // no owner
    double v = 0.0;
    if (lane < take) {
        const int e = nq - 1 - lane;
        CHK3(e >= 0 && e < QC3);
        const int info = Q.info[e];
        key = info & 31;
        const int ci[3] = {(info >> 5) & 15, (info >> 9) & 15, (info >> 13) & 15};
        CHK3(ci[0] < 3 * K + 1 && ci[1] < 3 * K + 1 && ci[2] < 3 * K + 1 && Q.tet[e] >= 0);
        const double *rc = a.rec + (int64_t)R::RS * Q.tet[e];
        double M[9], cf[R::NB];
#pragma unroll
        for (int j = 0; j < 9; ++j) M[j] = a.h * __ldg(rc + R::OFF_AINV + j);
#pragma unroll
        for (int j = 0; j < R::NB; ++j) cf[j] = __ldg(rc + R::OFF_C + j);
        // z(xi, eta, zeta) = p0 + xi E0 + eta E1 + zeta E2;  rst = r0 + M z = A + xi B0 + eta B1 + zeta B2;
        // the kernel factors are evaluated in cell-centred variables (p0 shifted by the cell centre)
        double pc[3], E[3][3], A[3], B[3][3];
#pragma unroll
        for (int d = 0; d < 3; ++d) {
            pc[d] = Q.p[d][e];
#pragma unroll
            for (int j = 0; j < 3; ++j) E[j][d] = Q.p[3 + 3 * j + d][e];
        }
#pragma unroll
        for (int i = 0; i < 3; ++i) {
            A[i] = fma(M[3 * i], pc[0], fma(M[3 * i + 1], pc[1], fma(M[3 * i + 2], pc[2], Q.r0[i][e])));
#pragma unroll
            for (int j = 0; j < 3; ++j) B[j][i] = fma(M[3 * i], E[j][0], fma(M[3 * i + 1], E[j][1], M[3 * i + 2] * E[j][2]));
        }
        double kr[3][K + 1];
#pragma unroll
        for (int d = 0; d < 3; ++d) {
            pc[d] -= T0 + ci[d] + 0.5;
#pragma unroll
            for (int j = 0; j <= K; ++j) kr[d][j] = kc[ci[d] * (K + 1) + j];
        }
        double s = 0.0;
        for (int q = 0; q < a.nq; ++q) {
            const double2 xe = *reinterpret_cast<const double2 *>(qr + 4 * q);
            const double2 zw = *reinterpret_cast<const double2 *>(qr + 4 * q + 2);
            double kv = 1.0;
#pragma unroll
            for (int d = 0; d < 3; ++d)
                kv *= horner1<K>(kr[d], fma(zw.x, E[2][d], fma(xe.y, E[1][d], fma(xe.x, E[0][d], pc[d]))));
            const double rr = fma(zw.x, B[2][0], fma(xe.y, B[1][0], fma(xe.x, B[0][0], A[0])));
            const double ss = fma(zw.x, B[2][1], fma(xe.y, B[1][1], fma(xe.x, B[0][1], A[1])));
            const double tt = fma(zw.x, B[2][2], fma(xe.y, B[1][2], fma(xe.x, B[0][2], A[2])));
            s = fma(zw.y * kv, umono<K>(cf, rr, ss, tt), s);
        }
        v = Q.vol6[e] * s;
    }
    nq -= take;
    // per-owner sums in lane order (deterministic): the group leader adds the others' values
    const unsigned grp = __match_any_sync(0xffffffffu, key);
    const int leader = __ffs(grp) - 1;
    double sum = v;
    unsigned rest = grp & ~(1u << leader);
    while (__any_sync(0xffffffffu, rest != 0)) {
        const int src = rest ? __ffs(rest) - 1 : lane;
        const double w = __shfl_sync(0xffffffffu, v, src);
        if (rest) { sum += w; rest &= rest - 1; }
    }
    if (lane == leader && key < 32) Q.acc[key] += sum;
    __syncwarp();
}

template <int K, bool COUNT, int MINB>
__global__ void __launch_bounds__(TW3 * 32, MINB) k_eval3w(Eval3Args a) {
    using R = Rec3<K>;
    constexpr int NC = 3 * K + 1;
    constexpr double T0 = -0.5 * (3 * K + 1);
    constexpr int NKC = (NC * (K + 1) + 1) & ~1;
    extern __shared__ __align__(16) double sm3[];
    double *kc = sm3;
    double *qr = kc + NKC;
    PieceQ3 *qs = reinterpret_cast<PieceQ3 *>(qr + ((4 * a.nq + 1) & ~1));
    for (int i = threadIdx.x; i < NC * (K + 1); i += blockDim.x) kc[i] = a.kc[i];
    for (int i = threadIdx.x; i < a.nq * 4; i += blockDim.x) qr[i] = a.qr[i];
    __syncthreads();
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    PieceQ3 &Q = qs[wid];
    WorkQ3 &W = reinterpret_cast<WorkQ3 *>(qs + TW3)[wid];
    // a.split warps share one tile (small problems: fewer tiles than resident warps), each walking
    // a contiguous share of the tile's candidate cells; their sums are combined in a fixed order
    const int split = a.split, part = wid % split;
    const int64_t p0 = ((int64_t)blockIdx.x * (TW3 / split) + wid / split) * 32;
    const bool live = p0 < a.np;
    if (split == 1 && !live) return;              // warp-uniform; no block barrier below for split == 1
    const bool valid = live && p0 + lane < a.np;
    int orig = -1;
    double x[3] = {0.0, 0.0, 0.0};
    if (valid) {
        orig = a.perm[p0 + lane];
        for (int d = 0; d < 3; ++d) {
            x[d] = a.pts[3 * (int64_t)orig + d];
            if (a.periodic & (1 << d)) {
                x[d] = x[d] - a.L[d] * floor((x[d] - a.x0[d]) / a.L[d]);
                if (x[d] >= a.x0[d] + a.L[d]) x[d] -= a.L[d];
                if (x[d] < a.x0[d]) x[d] = a.x0[d];
            }
        }
    }
    Q.acc[lane] = 0.0;
    int lo[3], hi[3];
    double tb0[3], tb1[3];
#pragma unroll
    for (int d = 0; d < 3; ++d) {
        double mn = valid ? x[d] : 1e300, mx = valid ? x[d] : -1e300;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            mn = fmin(mn, __shfl_xor_sync(0xffffffffu, mn, o));
            mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        }
        tb0[d] = mn - a.hw;       // the tile's stencil box
        tb1[d] = mx + a.hw;
        lo[d] = (int)floor((tb0[d] - a.ext[d] - a.x0[d]) / a.cell[d]) - 1;
        hi[d] = (int)floor((tb1[d] - a.x0[d]) / a.cell[d]) + 1;
        if (!(a.periodic & (1 << d))) { lo[d] = max(lo[d], 0); hi[d] = min(hi[d], a.nc[d] - 1); }
    }
    __syncwarp();
    int nq = 0;
    unsigned long long c_pairs = 0, c_pieces = 0;
    bool overflow = false;
    Tet stack[STACK3];
    int stack_own[STACK3];
    const int nx = hi[0] - lo[0] + 1, ny = hi[1] - lo[1] + 1;
    const int nz = hi[2] - lo[2] + 1;             // (empty when a non-periodic axis clamps the range away)
    const int64_t ncl = (live && nx > 0 && ny > 0 && nz > 0) ? (int64_t)nx * ny * nz : 0;
    const int64_t cl0 = ncl * part / split, cl1 = ncl * (part + 1) / split;
    for (int64_t cl = cl0; cl < cl1; ++cl) {
                const int I[3] = {lo[0] + (int)(cl % nx), lo[1] + (int)((cl / nx) % ny), lo[2] + (int)(cl / ((int64_t)nx * ny))};
                int cidx[3];
                double sh[3];
#pragma unroll
                for (int d = 0; d < 3; ++d) {
                    cidx[d] = I[d];
                    int q = 0;
                    if (a.periodic & (1 << d)) { cidx[d] = ((I[d] % a.nc[d]) + a.nc[d]) % a.nc[d]; q = (I[d] - cidx[d]) / a.nc[d]; }
                    sh[d] = q * a.L[d];
                }
                const int cell = (cidx[2] * a.nc[1] + cidx[1]) * a.nc[0] + cidx[0];
                CHK3(cidx[0] >= 0 && cidx[0] < a.nc[0] && cidx[1] >= 0 && cidx[1] < a.nc[1] && cidx[2] >= 0 && cidx[2] < a.nc[2]);
                const int t0 = __ldg(a.cell_start + cell), t1 = __ldg(a.cell_start + cell + 1);
                for (int tb = t0; tb < t1; tb += 32) {
                    bool keep = false;
                    if (tb + lane < t1) {
                        const double *bb = a.bbox + 6 * (int64_t)(tb + lane);
                        keep = true;
#pragma unroll
                        for (int d = 0; d < 3; ++d)
                            keep = keep && (__ldg(bb + d) + sh[d] < tb1[d]) && (__ldg(bb + 3 + d) + sh[d] > tb0[d]);
                    }
                    unsigned km = __ballot_sync(0xffffffffu, keep);
                    while (km) {
                        const int t = tb + __ffs(km) - 1;
                        km &= km - 1;
                        const double *bb = a.bbox + 6 * (int64_t)t;
                        bool hit = valid;
#pragma unroll
                        for (int d = 0; d < 3; ++d)
                            hit = hit && (__ldg(bb + d) + sh[d] < x[d] + a.hw) && (__ldg(bb + 3 + d) + sh[d] > x[d] - a.hw);
                        if (!__any_sync(0xffffffffu, hit)) continue;
                        if (COUNT) c_pairs += hit;
                        const double *rc = a.rec + (int64_t)R::RS * t;
                        int ns = 0, wn = 0;       // local stack depth; shared work-queue length (warp-uniform)
                        bool have = false;        // tt holds a piece to process (the pair's tetrahedron first)
                        int own = lane;           // owner lane of tt
                        Tet tt;
                        __syncwarp();             // the previous candidate's leaves have read W.r0
                        if (hit) {
                            double d0[3];
#pragma unroll
                            for (int d = 0; d < 3; ++d) d0[d] = x[d] - sh[d] - __ldg(rc + d);
#pragma unroll
                            for (int i = 0; i < 3; ++i) {
                                double r = 0.0;
#pragma unroll
                                for (int j = 0; j < 3; ++j) r = fma(__ldg(rc + R::OFF_AINV + 3 * i + j), d0[j], r);
                                W.r0[i][lane] = r;
                            }
                            for (int i = 0; i < 4; ++i)
                                for (int d = 0; d < 3; ++d) tt.p[i][d] = ((__ldg(rc + 3 * i + d) + sh[d]) - x[d]) * a.inv_h;
                            have = true;
                        }
                        while (true) {
                            // refill: own local stack first, then idle lanes take pieces of the shared queue
                            if (!have && ns > 0) { --ns; tt = stack[ns]; own = stack_own[ns]; have = true; }
                            const unsigned idle = __ballot_sync(0xffffffffu, !have);
                            const int take = min(__popc(idle), wn);
                            if (take > 0) {                   // warp-uniform
                                __syncwarp();                 // W (pieces, owners' r0) written by other lanes is visible
                                if (!have) {
                                    const int rk = __popc(idle & lanemask_lt3());
                                    if (rk < take) {
                                        const int e = wn - 1 - rk;
#pragma unroll
                                        for (int i = 0; i < 4; ++i)
#pragma unroll
                                            for (int d = 0; d < 3; ++d) tt.p[i][d] = W.p[3 * i + d][e];
                                        own = W.owner[e];
                                        have = true;
                                    }
                                }
                                __syncwarp();                 // slots [wn - take, wn) are read before they are refilled
                            }
                            wn -= take;
                            if (!__any_sync(0xffffffffu, have)) break;
                            bool leaf = false;
                            double vol6 = 0.0;
                            int ci[3] = {0, 0, 0};
                            bool split = false;
                            int ax = -1, npush = 0;
                            double cut = 0.0;
                            if (have) {
                                have = false;
                                double mn[3], mx[3];
                                bool outside = false;
#pragma unroll
                                for (int d = 0; d < 3; ++d) {
                                    mn[d] = fmin(fmin(tt.p[0][d], tt.p[1][d]), fmin(tt.p[2][d], tt.p[3][d]));
                                    mx[d] = fmax(fmax(tt.p[0][d], tt.p[1][d]), fmax(tt.p[2][d], tt.p[3][d]));
                                    outside = outside || mx[d] <= T0 || mn[d] >= -T0;   // K = 0 there: drop
                                }
#pragma unroll
                                for (int d = 2; d >= 0; --d) {      // the first axis (x, y, z order) cut by a kernel plane
                                    const double kn = fmax(floor(mn[d] - T0) + 1.0 + T0, T0);
                                    if (kn < mx[d] && kn <= -T0) { ax = d; cut = kn; }
                                }
                                if (outside) {
                                } else if (ax < 0) {
                                    // the centroid's cell; a piece whose centroid lies outside the
                                    // support is dropped (a plane within rounding of its lower end is
                                    // not found by the search above, e.g. [2 - 1e-16, 2.5] at k = 1)
                                    bool inside = true;
                                    for (int d = 0; d < 3; ++d) {
                                        const double cen = 0.25 * (tt.p[0][d] + tt.p[1][d] + tt.p[2][d] + tt.p[3][d]);
                                        ci[d] = (int)floor(cen - T0);
                                        inside = inside && ci[d] >= 0 && ci[d] < NC;
                                    }
                                    double e[3][3];
                                    for (int j = 0; j < 3; ++j)
                                        for (int d = 0; d < 3; ++d) e[j][d] = tt.p[j + 1][d] - tt.p[0][d];
                                    vol6 = fabs(e[0][0] * (e[1][1] * e[2][2] - e[1][2] * e[2][1]) -
                                                e[0][1] * (e[1][0] * e[2][2] - e[1][2] * e[2][0]) +
                                                e[0][2] * (e[1][0] * e[2][1] - e[1][1] * e[2][0]));
                                    leaf = inside && vol6 > 0.0;
                                } else {
                                    split = true;
                                    int nl = 0;
                                    for (int i = 0; i < 4; ++i) nl += tt.p[i][ax] <= cut;
                                    // a side beyond a support end plane (cut = T0: the low side, cut =
                                    // -T0: the high side) is outside the support: not emitted
                                    const int nlo = cut > T0 ? (nl == 1 ? 1 : 3) : 0;      // tets on the low side
                                    const int nhi = cut < -T0 ? (nl == 3 ? 1 : 3) : 0;     // (2-2: 3 and 3)
                                    npush = nlo + nhi - 1;                                // all but the last child
                                }
                            }
                            // children go to the shared queue while it has room (a prefix of the lanes),
                            // the rest to their lanes' local stacks
                            int excl = npush;
#pragma unroll
                            for (int o = 1; o < 32; o <<= 1) {
                                const int v = __shfl_up_sync(0xffffffffu, excl, o);
                                if (lane >= o) excl += v;
                            }
                            excl -= npush;
                            const bool fits = wn + excl + npush <= WQ3;
                            const int pushed = __reduce_add_sync(0xffffffffu, (split && fits) ? npush : 0);
                            if (split) {
                                Tet pend;
                                bool haspend = false;
                                int slot = wn + excl;
                                const Tet src = tt;
                                int lowi[4], highi[4], nl = 0, nh = 0;
                                for (int i = 0; i < 4; ++i) {
                                    if (src.p[i][ax] <= cut) lowi[nl++] = i;
                                    else highi[nh++] = i;
                                }
                                auto isect = [&](int i, int j, double *o) {
                                    const double r = (cut - src.p[i][ax]) / (src.p[j][ax] - src.p[i][ax]);
                                    for (int d = 0; d < 3; ++d) o[d] = fma(r, src.p[j][d] - src.p[i][d], src.p[i][d]);
                                    o[ax] = cut;
                                };
                                auto push = [&](const double *q0, const double *q1, const double *q2, const double *q3) {
                                    if (haspend) {
                                        if (fits) {
                                            CHK3(slot < WQ3);
#pragma unroll
                                            for (int i = 0; i < 4; ++i)
#pragma unroll
                                                for (int d = 0; d < 3; ++d) W.p[3 * i + d][slot] = pend.p[i][d];
                                            W.owner[slot] = own;
                                            ++slot;
                                        } else if (ns >= STACK3) {
                                            overflow = true;
                                        } else {
                                            stack[ns] = pend;
                                            stack_own[ns] = own;
                                            ++ns;
                                        }
                                    }
                                    for (int d = 0; d < 3; ++d) {
                                        pend.p[0][d] = q0[d]; pend.p[1][d] = q1[d];
                                        pend.p[2][d] = q2[d]; pend.p[3][d] = q3[d];
                                    }
                                    haspend = true;
                                };
                                auto push_prism = [&](const double *a0, const double *a1, const double *a2,
                                                      const double *b0, const double *b1, const double *b2) {
                                    push(a0, a1, a2, b2);
                                    push(a0, a1, b1, b2);
                                    push(a0, b0, b1, b2);
                                };
                                const bool keep_lo = cut > T0, keep_hi = cut < -T0;
                                if (nl == 1 || nh == 1) {
                                    const int o = nl == 1 ? lowi[0] : highi[0];
                                    const int *rest = nl == 1 ? highi : lowi;
                                    double q[3][3];
                                    for (int j = 0; j < 3; ++j) isect(o, rest[j], q[j]);
                                    if (nl == 1 ? keep_lo : keep_hi) push(src.p[o], q[0], q[1], q[2]);
                                    if (nl == 1 ? keep_hi : keep_lo)
                                        push_prism(q[0], q[1], q[2], src.p[rest[0]], src.p[rest[1]], src.p[rest[2]]);
                                } else {
                                    const int l0 = lowi[0], l1 = lowi[1], h0 = highi[0], h1 = highi[1];
                                    double q00[3], q01[3], q10[3], q11[3];
                                    isect(l0, h0, q00); isect(l0, h1, q01); isect(l1, h0, q10); isect(l1, h1, q11);
                                    if (keep_lo) push_prism(src.p[l0], q00, q01, src.p[l1], q10, q11);
                                    if (keep_hi) push_prism(src.p[h0], q00, q10, src.p[h1], q01, q11);
                                }
                                tt = pend;
                                have = haspend;
                            }
                            wn += pushed;
                            double r0[3] = {0.0, 0.0, 0.0};
                            if (leaf) {
#pragma unroll
                                for (int d = 0; d < 3; ++d) r0[d] = W.r0[d][own];
                            }
                            const unsigned lm = __ballot_sync(0xffffffffu, leaf);
                            if (leaf) {
                                const int pos = nq + __popc(lm & lanemask_lt3());
                                CHK3(pos < QC3 && ci[0] >= 0 && ci[0] < NC && ci[1] >= 0 && ci[1] < NC && ci[2] >= 0 && ci[2] < NC);
#pragma unroll
                                for (int d = 0; d < 3; ++d) {
                                    Q.p[d][pos] = tt.p[0][d];
#pragma unroll
                                    for (int j = 0; j < 3; ++j) Q.p[3 + 3 * j + d][pos] = tt.p[j + 1][d] - tt.p[0][d];
                                    Q.r0[d][pos] = r0[d];
                                }
                                Q.vol6[pos] = vol6;
                                Q.tet[pos] = t;
                                Q.info[pos] = own | (ci[0] << 5) | (ci[1] << 9) | (ci[2] << 13);
                            }
                            nq += __popc(lm);
                            if (COUNT) c_pieces += leaf;
                            if (nq >= 32) {
                                __syncwarp();
                                flush3<K>(a, Q, kc, qr, nq, lane);
                            }
                        }
                    }
                }
            }
    while (nq > 0) {
        __syncwarp();
        flush3<K>(a, Q, kc, qr, nq, lane);
    }
    __syncwarp();
    if (split == 1) {
        if (valid) a.out[orig] = Q.acc[lane];
    } else {
        __syncthreads();
        if (part == 0 && valid) {
            double v = Q.acc[lane];
            for (int q = 1; q < split; ++q) {
                CHK3(wid + q < TW3);
                v += qs[wid + q].acc[lane];
            }
            a.out[orig] = v;
        }
    }
    if (__any_sync(0xffffffffu, overflow) && lane == 0) atomicOr(a.cnt + 2, 1ull);
    if (COUNT) {
        atomicAdd(a.cnt + 0, c_pairs);
        atomicAdd(a.cnt + 1, c_pieces);
    }
}

// Launch k_eval3w: when the point tiles do not fill one wave of resident warps, each tile's cells
// are split over 2 or 4 warps (a.split) so that more warps share the work.
template <int K, bool COUNT, int MINB>
void launch3w_mb(int64_t ntiles, int num_sms, size_t sm, cudaStream_t st, Eval3Args a) {
    auto kern = k_eval3w<K, COUNT, MINB>;
    CK3(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
    int per_sm = 0;
    CK3(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, 32 * TW3, sm));
    const int64_t resident = (int64_t)std::max(per_sm, 1) * num_sms * TW3;
    a.split = 1;
    while (a.split < TW3 && ntiles * a.split * 2 <= resident) a.split *= 2;
    if (const char *e = getenv("SIAC3_SPLIT")) a.split = std::max(1, std::min(TW3, atoi(e)));   // (experiments)
    const int tpb = TW3 / a.split;
    kern<<<(unsigned)((ntiles + tpb - 1) / tpb), 32 * TW3, sm, st>>>(a);
}
template <int K, bool COUNT>
void launch3w(int minb, int64_t ntiles, int num_sms, size_t sm, cudaStream_t st, const Eval3Args &a) {
    // measured (tools/gpu_wq3.sh, with the shared work queue): 3 blocks/SM (168 registers) at k = 1
    // (709 vs 739 ms at 4 blocks), the unbounded variant at k = 2, 3 (the quadrature's registers:
    // 5.6 s unbounded vs 6.4 s at 3 blocks/SM, k = 2, before the work queue)
    if (minb == 0) minb = K == 1 ? 3 : 1;
    if (minb >= 4) launch3w_mb<K, COUNT, 4>(ntiles, num_sms, sm, st, a);
    else if (minb == 3) launch3w_mb<K, COUNT, 3>(ntiles, num_sms, sm, st, a);
    else launch3w_mb<K, COUNT, 1>(ntiles, num_sms, sm, st, a);
}

inline size_t smem3w(int k, int nq) {
    const int nc = 3 * k + 1;
    return sizeof(double) * (((nc * (k + 1) + 1) & ~1) + ((4 * nq + 1) & ~1)) + TW3 * (sizeof(PieceQ3) + sizeof(WorkQ3));
}

// Gauss-Jacobi rule for the weight (1-x)^alpha on [-1, 1] (Golub-Welsch, Jacobi eigenvalue
// iterations in long double), mapped to [0, 1] with weight (1-b)^alpha.
void gauss_jacobi01(int n, int alpha, std::vector<long double> &x, std::vector<long double> &w) {
    std::vector<long double> J((size_t)n * n, 0.0L), Vv((size_t)n * n, 0.0L);
    const long double al = alpha;
    for (int i = 0; i < n; ++i) {
        const long double s = 2.0L * i + al;
        J[(size_t)i * n + i] = (i == 0) ? (-al) / (al + 2.0L) : (-al * al) / (s * (s + 2.0L));
        if (i + 1 < n) {
            const long double k1 = i + 1, s1 = 2.0L * k1 + al;
            const long double b = sqrtl(4.0L * k1 * (k1 + al) * k1 * (k1 + al) / (s1 * s1 * (s1 + 1.0L) * (s1 - 1.0L)));
            J[(size_t)i * n + i + 1] = J[(size_t)(i + 1) * n + i] = b;
        }
        Vv[(size_t)i * n + i] = 1.0L;
    }
    for (int sweep = 0; sweep < 100; ++sweep) {        // cyclic Jacobi rotations
        long double off = 0.0L;
        for (int p = 0; p < n; ++p)
            for (int q = p + 1; q < n; ++q) off += J[(size_t)p * n + q] * J[(size_t)p * n + q];
        if (off < 1e-40L) break;
        for (int p = 0; p < n; ++p)
            for (int q = p + 1; q < n; ++q) {
                const long double apq = J[(size_t)p * n + q];
                if (fabsl(apq) < 1e-300L) continue;
                const long double theta = (J[(size_t)q * n + q] - J[(size_t)p * n + p]) / (2.0L * apq);
                const long double tt = (theta >= 0 ? 1.0L : -1.0L) / (fabsl(theta) + sqrtl(theta * theta + 1.0L));
                const long double c = 1.0L / sqrtl(tt * tt + 1.0L), s = tt * c;
                for (int k = 0; k < n; ++k) {
                    const long double jkp = J[(size_t)k * n + p], jkq = J[(size_t)k * n + q];
                    J[(size_t)k * n + p] = c * jkp - s * jkq;
                    J[(size_t)k * n + q] = s * jkp + c * jkq;
                }
                for (int k = 0; k < n; ++k) {
                    const long double jpk = J[(size_t)p * n + k], jqk = J[(size_t)q * n + k];
                    J[(size_t)p * n + k] = c * jpk - s * jqk;
                    J[(size_t)q * n + k] = s * jpk + c * jqk;
                }
                for (int k = 0; k < n; ++k) {
                    const long double vkp = Vv[(size_t)k * n + p], vkq = Vv[(size_t)k * n + q];
                    Vv[(size_t)k * n + p] = c * vkp - s * vkq;
                    Vv[(size_t)k * n + q] = s * vkp + c * vkq;
                }
            }
    }
    // mu0 = int_{-1}^{1} (1-x)^alpha dx = 2^(alpha+1) / (alpha+1); mapped weight * 2^-(alpha+1)
    x.resize(n);
    w.resize(n);
    for (int i = 0; i < n; ++i) {
        x[i] = 0.5L * (1.0L + J[(size_t)i * n + i]);
        w[i] = (1.0L / (al + 1.0L)) * Vv[(size_t)0 * n + i] * Vv[(size_t)0 * n + i];
    }
}

// Collapsed rule on the unit tetrahedron exact for total degree <= 2n - 1:
// r = a (1 - b)(1 - c), s = b (1 - c), t = c; Gauss-Legendre in a, Gauss-Jacobi (1-b)^1, (1-c)^2.
std::vector<double> tet_rule(int n) {
    std::vector<long double> xa, wa, xb, wb, xc, wc;
    gauss_jacobi01(n, 0, xa, wa);
    gauss_jacobi01(n, 1, xb, wb);
    gauss_jacobi01(n, 2, xc, wc);
    std::vector<double> q;
    for (int i = 0; i < n; ++i)
        for (int j = 0; j < n; ++j)
            for (int l = 0; l < n; ++l) {
                const long double r = xa[i] * (1.0L - xb[j]) * (1.0L - xc[l]), s = xb[j] * (1.0L - xc[l]), t = xc[l];
                q.push_back((double)r); q.push_back((double)s); q.push_back((double)t);
                q.push_back((double)(wa[i] * wb[j] * wc[l]));
            }
    return q;
}

siac_status run3(std::string *err, const std::function<void()> &fn) {
    try {
        fn();
        return SIAC_OK;
    } catch (const Fail3 &f) {
        *err = f.msg;
        return f.st;
    } catch (const std::bad_alloc &) {
        *err = "host allocation failed";
        return SIAC_ENOMEM;
    } catch (const std::exception &e) {
        *err = std::string("internal error: ") + e.what();
        return SIAC_EINTERNAL;
    }
}

inline unsigned nblk3(int64_t n, int bs) { return (unsigned)((n + bs - 1) / bs); }

}  // namespace

struct siac3_ctx {
    int device = 0, k = 1, periodic = 7, rs = 0;
    double h = 0, dom[6] = {0, 0, 0, 1, 1, 1}, cell[3] = {1, 1, 1}, ext[3] = {0, 0, 0};
    int nc[3] = {1, 1, 1};
    int64_t nt = 0;
    cudaStream_t stream = nullptr;
    double *d_rec = nullptr, *d_bbox = nullptr, *d_kc = nullptr, *d_qr = nullptr;
    int *d_cs = nullptr;
    int nq = 0;
    int64_t cap = 0;
    unsigned *d_keys[2] = {nullptr, nullptr};
    int *d_idx[2] = {nullptr, nullptr};
    void *d_cub = nullptr;
    size_t cub_bytes = 0;
    double *d_hp = nullptr, *d_ho = nullptr;
    int64_t cap_h = 0;
    unsigned long long *d_cnt = nullptr;
    bool counting = false;
    int schedule = 0;         // 0: warp per point tile (k_eval3w, default), 1: thread per point (k_eval3)
    int num_sms = 148;
    int minb = 0;             // k_eval3w __launch_bounds__ min blocks; 0 = per degree (env SIAC3_MINB: experiments)
    std::string err;
};

static thread_local std::string g_err3;

static void free3(siac3_ctx *c) {
    if (!c) return;
    cudaSetDevice(c->device);
    void *ps[] = {c->d_rec, c->d_bbox, c->d_kc, c->d_qr, c->d_cs, c->d_keys[0], c->d_keys[1], c->d_idx[0], c->d_idx[1],
                  c->d_cub, c->d_hp, c->d_ho, c->d_cnt};
    for (void *p : ps)
        if (p) cudaFree(p);
    if (c->stream) cudaStreamDestroy(c->stream);
    delete c;
}

extern "C" {

siac_status siac3_create(siac3_ctx **out, const double *V, int64_t nv, const int32_t *T, int64_t nt, const double *C,
                         const siac3_params *p) {
    if (out) *out = nullptr;
    siac3_ctx *c = nullptr;
    const siac_status st = run3(&g_err3, [&]() {
        need3(out != nullptr && p != nullptr, "out and params must be non-NULL");
        need3(p->k >= 1 && p->k <= 3, "k must be in 1..3 for tetrahedral meshes");
        need3(std::isfinite(p->h) && p->h > 0, "h must be finite and > 0");
        need3(nv >= 0 && nt >= 0 && nt <= 0x3fffffff, "bad sizes");
        need3(nt == 0 || (V && T && C), "NULL mesh arrays");
        need3((p->periodic & ~7) == 0, "periodic must be a combination of bits 0..2");
        const double W = (3 * p->k + 1) * p->h;
        for (int d = 0; d < 3; ++d) {
            need3(std::isfinite(p->domain[d]) && std::isfinite(p->domain[d + 3]) && p->domain[d + 3] > p->domain[d],
                  "empty or inverted domain");
            need3(!(p->periodic & (1 << d)) || W <= (p->domain[d + 3] - p->domain[d]) * (1 + 1e-12),
                  "(3k+1)h exceeds a periodic extent");
        }
        int ndev = 0;
        if (cudaGetDeviceCount(&ndev) != cudaSuccess || p->device < 0 || p->device >= ndev)
            throw Fail3{SIAC_EDEVICE, "no CUDA device with that ordinal"};
        int major = 0;
        CK3(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, p->device));
        if (major < 10) throw Fail3{SIAC_EDEVICE, "device is not sm_100 class"};
        CK3(cudaSetDevice(p->device));
        int nsm = 0;
        CK3(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, p->device));
        c = new siac3_ctx();
        c->num_sms = nsm;
        if (const char *e = getenv("SIAC3_MINB")) c->minb = atoi(e);
        c->device = p->device;
        c->k = p->k;
        c->h = p->h;
        c->periodic = p->periodic;
        for (int d = 0; d < 6; ++d) c->dom[d] = p->domain[d];
        c->nt = nt;
        CK3(cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking));
        const int nb = (p->k + 1) * (p->k + 2) * (p->k + 3) / 6;
        c->rs = rec3_size(p->k);
        // max tetrahedron extents (host; also the validation of the vertex range)
        for (int64_t t = 0; t < nt; ++t)
            for (int d = 0; d < 3; ++d) {
                double lo = 1e300, hi = -1e300;
                for (int i = 0; i < 4; ++i) {
                    const int vi = T[4 * t + i];
                    need3(vi >= 0 && vi < nv, "tetrahedron index out of range");
                    lo = std::min(lo, V[3 * (int64_t)vi + d]);
                    hi = std::max(hi, V[3 * (int64_t)vi + d]);
                }
                c->ext[d] = std::max(c->ext[d], hi - lo);
            }
        for (int d = 0; d < 3; ++d) {
            const double L = p->domain[d + 3] - p->domain[d];
            c->nc[d] = (int)std::max(1.0, std::min(256.0, std::floor(L / (0.5 * p->h))));
            c->cell[d] = L / c->nc[d];
        }
        const int64_t ncell = (int64_t)c->nc[0] * c->nc[1] * c->nc[2];
        std::vector<double> kc = siac::kernel_cell_table(p->k);
        // the integrand K(z1) K(z2) K(z3) u has total degree 4k: n^3 points, exact for 2n - 1 >= 4k
        const int nqd = 2 * p->k + 1;
        std::vector<double> q = tet_rule(nqd);
        c->nq = (int)(q.size() / 4);
        CK3(cudaMalloc(&c->d_kc, sizeof(double) * kc.size()));
        CK3(cudaMalloc(&c->d_qr, sizeof(double) * q.size()));
        CK3(cudaMemcpy(c->d_kc, kc.data(), sizeof(double) * kc.size(), cudaMemcpyHostToDevice));
        CK3(cudaMemcpy(c->d_qr, q.data(), sizeof(double) * q.size(), cudaMemcpyHostToDevice));
        CK3(cudaMalloc(&c->d_cnt, 3 * sizeof(unsigned long long)));
        CK3(cudaMemset(c->d_cnt, 0, 3 * sizeof(unsigned long long)));
        CK3(cudaMalloc(&c->d_cs, sizeof(int) * (ncell + 1)));
        if (nt == 0) {
            CK3(cudaMemset(c->d_cs, 0, sizeof(int) * (ncell + 1)));
            return;
        }
        double *dV = nullptr, *dC = nullptr, *rec_u = nullptr, *bb_u = nullptr;
        int *dT = nullptr, *idx[2] = {nullptr, nullptr}, *dbad = nullptr;
        unsigned long long *keys[2] = {nullptr, nullptr};
        void *tmp = nullptr;
        auto cleanup = [&]() {
            void *ps[] = {dV, dC, rec_u, bb_u, dT, idx[0], idx[1], dbad, keys[0], keys[1], tmp};
            for (void *pp : ps)
                if (pp) cudaFree(pp);
        };
        try {
            CK3(cudaMalloc(&dV, sizeof(double) * 3 * std::max<int64_t>(nv, 1)));
            CK3(cudaMalloc(&dT, sizeof(int) * 4 * nt));
            CK3(cudaMalloc(&dC, sizeof(double) * nb * nt));
            CK3(cudaMalloc(&rec_u, sizeof(double) * c->rs * nt));
            CK3(cudaMalloc(&bb_u, sizeof(double) * 6 * nt));
            CK3(cudaMalloc(&dbad, sizeof(int)));
            for (int b = 0; b < 2; ++b) {
                CK3(cudaMalloc(&keys[b], sizeof(unsigned long long) * nt));
                CK3(cudaMalloc(&idx[b], sizeof(int) * nt));
            }
            CK3(cudaMalloc(&c->d_rec, sizeof(double) * c->rs * nt));
            CK3(cudaMalloc(&c->d_bbox, sizeof(double) * 6 * nt));
            cudaStream_t cs = c->stream;
            CK3(cudaMemcpyAsync(dV, V, sizeof(double) * 3 * nv, cudaMemcpyHostToDevice, cs));
            CK3(cudaMemcpyAsync(dT, T, sizeof(int) * 4 * nt, cudaMemcpyHostToDevice, cs));
            CK3(cudaMemcpyAsync(dC, C, sizeof(double) * nb * nt, cudaMemcpyHostToDevice, cs));
            CK3(cudaMemsetAsync(dbad, 0, sizeof(int), cs));
            Prep3Args pa;
            pa.V = dV; pa.T = dT; pa.C = dC; pa.nt = nt; pa.nb = nb; pa.rs = c->rs; pa.nv = nv;
            for (int d = 0; d < 3; ++d) { pa.x0[d] = p->domain[d]; pa.cell[d] = c->cell[d]; pa.nc[d] = c->nc[d]; }
            pa.rec = rec_u; pa.bbox = bb_u; pa.key = keys[0]; pa.idx = idx[0]; pa.bad = dbad;
            k_prep3<<<nblk3(nt, 128), 128, 0, cs>>>(pa);
            CK3(cudaGetLastError());
            int bad = 0;
            CK3(cudaMemcpyAsync(&bad, dbad, sizeof(int), cudaMemcpyDeviceToHost, cs));
            CK3(cudaStreamSynchronize(cs));
            need3(!(bad & 4), "non-finite vertex coordinate or coefficient");
            need3(!(bad & 2), "zero-volume tetrahedron");
            need3(!(bad & 1), "tetrahedron index out of range");
            cub::DoubleBuffer<unsigned long long> kb(keys[0], keys[1]);
            cub::DoubleBuffer<int> vb(idx[0], idx[1]);
            size_t bytes = 0;
            int end_bit = 1;
            while ((1ull << end_bit) <= (unsigned long long)ncell && end_bit < 63) ++end_bit;
            CK3(cub::DeviceRadixSort::SortPairs(nullptr, bytes, kb, vb, (int)nt, 0, end_bit, cs));
            CK3(cudaMalloc(&tmp, bytes));
            CK3(cub::DeviceRadixSort::SortPairs(tmp, bytes, kb, vb, (int)nt, 0, end_bit, cs));
            k_gather3<<<nblk3(nt, 256), 256, 0, cs>>>(rec_u, bb_u, vb.Current(), nt, c->rs, c->d_rec, c->d_bbox);
            CK3(cudaGetLastError());
            k_cell_start3<<<nblk3(ncell + 1, 256), 256, 0, cs>>>(kb.Current(), nt, ncell, c->d_cs);
            CK3(cudaGetLastError());
            CK3(cudaStreamSynchronize(cs));
        } catch (...) {
            cleanup();
            throw;
        }
        cleanup();
    });
    if (st != SIAC_OK) {
        free3(c);
        return st;
    }
    *out = c;
    return SIAC_OK;
}

siac_status siac3_eval_async(siac3_ctx *ctx, const double *d_pts, int64_t np, double *d_out, void *stream) {
    if (!ctx) { g_err3 = "NULL context"; return SIAC_EINVAL; }
    return run3(&ctx->err, [&]() {
        need3(np >= 0 && np <= 0x7fffffff, "bad n_points");
        if (np == 0) return;
        need3(d_pts && d_out, "NULL device pointers");
        CK3(cudaSetDevice(ctx->device));
        cudaStream_t st = (cudaStream_t)stream;
        if (np > ctx->cap) {
            for (int b = 0; b < 2; ++b) {
                if (ctx->d_keys[b]) cudaFree(ctx->d_keys[b]);
                if (ctx->d_idx[b]) cudaFree(ctx->d_idx[b]);
                ctx->d_keys[b] = nullptr; ctx->d_idx[b] = nullptr;
            }
            if (ctx->d_cub) cudaFree(ctx->d_cub);
            ctx->d_cub = nullptr;
            ctx->cap = 0;
            for (int b = 0; b < 2; ++b) {
                CK3(cudaMalloc(&ctx->d_keys[b], sizeof(unsigned) * np));
                CK3(cudaMalloc(&ctx->d_idx[b], sizeof(int) * np));
            }
            cub::DoubleBuffer<unsigned> kb(ctx->d_keys[0], ctx->d_keys[1]);
            cub::DoubleBuffer<int> vb(ctx->d_idx[0], ctx->d_idx[1]);
            size_t bytes = 0;
            CK3(cub::DeviceRadixSort::SortPairs(nullptr, bytes, kb, vb, (int)np));
            CK3(cudaMalloc(&ctx->d_cub, bytes));
            ctx->cub_bytes = bytes;
            ctx->cap = np;
        }
        const double *dm = ctx->dom;
        k_point_keys3<<<nblk3(np, 256), 256, 0, st>>>(d_pts, np, dm[0], dm[1], dm[2], dm[3] - dm[0], dm[4] - dm[1],
                                                      dm[5] - dm[2], ctx->d_keys[0], ctx->d_idx[0]);
        CK3(cudaGetLastError());
        cub::DoubleBuffer<unsigned> kb(ctx->d_keys[0], ctx->d_keys[1]);
        cub::DoubleBuffer<int> vb(ctx->d_idx[0], ctx->d_idx[1]);
        CK3(cub::DeviceRadixSort::SortPairs(ctx->d_cub, ctx->cub_bytes, kb, vb, (int)np, 0, 30, st));
        Eval3Args a;
        a.pts = d_pts; a.perm = vb.Current(); a.np = np; a.out = d_out; a.rec = ctx->d_rec; a.bbox = ctx->d_bbox;
        a.cell_start = ctx->d_cs; a.kc = ctx->d_kc; a.qr = ctx->d_qr; a.nq = ctx->nq;
        for (int d = 0; d < 3; ++d) {
            a.x0[d] = dm[d]; a.L[d] = dm[d + 3] - dm[d]; a.cell[d] = ctx->cell[d]; a.ext[d] = ctx->ext[d]; a.nc[d] = ctx->nc[d];
        }
        a.periodic = ctx->periodic;
        a.h = ctx->h; a.inv_h = 1.0 / ctx->h; a.hw = 0.5 * (3 * ctx->k + 1) * ctx->h;
        a.cnt = ctx->d_cnt;
        if (ctx->counting) CK3(cudaMemsetAsync(ctx->d_cnt, 0, 2 * sizeof(unsigned long long), st));
        const unsigned grid = nblk3(np, 128);
        const int64_t ntiles = (np + 31) / 32;
        a.split = 1;
        if (ctx->nt == 0) {
            CK3(cudaMemsetAsync(d_out, 0, sizeof(double) * np, st));
            return;
        }
#define SIAC3_LAUNCH(KK)                                                                       \
    do {                                                                                       \
        if (ctx->schedule == 1) {                                                              \
            if (ctx->counting) k_eval3<KK, true><<<grid, 128, 0, st>>>(a);                    \
            else k_eval3<KK, false><<<grid, 128, 0, st>>>(a);                                 \
        } else {                                                                               \
            const size_t sm = smem3w(KK, a.nq);                                                \
            if (ctx->counting) launch3w<KK, true>(ctx->minb, ntiles, ctx->num_sms, sm, st, a); \
            else launch3w<KK, false>(ctx->minb, ntiles, ctx->num_sms, sm, st, a);              \
        }                                                                                      \
    } while (0)
        if (ctx->k == 1) SIAC3_LAUNCH(1);
        else if (ctx->k == 2) SIAC3_LAUNCH(2);
        else SIAC3_LAUNCH(3);
#undef SIAC3_LAUNCH
        CK3(cudaGetLastError());
    });
}

siac_status siac3_eval(siac3_ctx *ctx, const double *pts, int64_t np, double *out) {
    if (!ctx) { g_err3 = "NULL context"; return SIAC_EINVAL; }
    const siac_status s0 = run3(&ctx->err, [&]() {
        need3(np >= 0, "negative n_points");
        if (np == 0) return;
        need3(pts && out, "NULL host pointers");
        CK3(cudaSetDevice(ctx->device));
        if (np > ctx->cap_h) {
            if (ctx->d_hp) cudaFree(ctx->d_hp);
            if (ctx->d_ho) cudaFree(ctx->d_ho);
            ctx->d_hp = ctx->d_ho = nullptr;
            ctx->cap_h = 0;
            CK3(cudaMalloc(&ctx->d_hp, sizeof(double) * 3 * np));
            CK3(cudaMalloc(&ctx->d_ho, sizeof(double) * np));
            ctx->cap_h = np;
        }
        CK3(cudaMemcpyAsync(ctx->d_hp, pts, sizeof(double) * 3 * np, cudaMemcpyHostToDevice, ctx->stream));
    });
    if (s0 != SIAC_OK || np == 0) return s0;
    const siac_status s1 = siac3_eval_async(ctx, ctx->d_hp, np, ctx->d_ho, ctx->stream);
    if (s1 != SIAC_OK) return s1;
    return run3(&ctx->err, [&]() {
        CK3(cudaMemcpyAsync(out, ctx->d_ho, sizeof(double) * np, cudaMemcpyDeviceToHost, ctx->stream));
        unsigned long long ovf = 0;
        CK3(cudaMemcpyAsync(&ovf, ctx->d_cnt + 2, sizeof(ovf), cudaMemcpyDeviceToHost, ctx->stream));
        CK3(cudaStreamSynchronize(ctx->stream));
        if (ovf) throw Fail3{SIAC_EINTERNAL, "piece stack overflow (h much smaller than the tetrahedra)"};
    });
}

siac_status siac3_set_schedule(siac3_ctx *ctx, int32_t schedule) {
    if (!ctx) { g_err3 = "NULL context"; return SIAC_EINVAL; }
    if (schedule < 0 || schedule > 1) { ctx->err = "schedule must be 0 (warp per point tile) or 1 (thread per point)"; return SIAC_EINVAL; }
    ctx->schedule = schedule;
    return SIAC_OK;
}

siac_status siac3_set_counting(siac3_ctx *ctx, int32_t enable) {
    if (!ctx) { g_err3 = "NULL context"; return SIAC_EINVAL; }
    ctx->counting = enable != 0;
    return SIAC_OK;
}

siac_status siac3_stats(const siac3_ctx *ctx, int64_t *pairs, int64_t *pieces) {
    if (!ctx) { g_err3 = "NULL context"; return SIAC_EINVAL; }
    siac3_ctx *c = const_cast<siac3_ctx *>(ctx);
    return run3(&c->err, [&]() {
        CK3(cudaSetDevice(c->device));
        unsigned long long h[3];
        CK3(cudaDeviceSynchronize());
        CK3(cudaMemcpy(h, c->d_cnt, sizeof(h), cudaMemcpyDeviceToHost));
        if (pairs) *pairs = (int64_t)h[0];
        if (pieces) *pieces = (int64_t)h[1];
        if (h[2]) throw Fail3{SIAC_EINTERNAL, "piece stack overflow in an evaluation (h much smaller than the tetrahedra)"};
    });
}

siac_status siac3_tet_rule(int32_t n, double *out) {
    return run3(&g_err3, [&]() {
        need3(n >= 1 && n <= 16 && out, "n must be in 1..16");
        std::vector<double> q = tet_rule(n);
        std::copy(q.begin(), q.end(), out);
    });
}

void siac3_destroy(siac3_ctx *ctx) { free3(ctx); }

const char *siac3_last_error(const siac3_ctx *ctx) { return ctx ? ctx->err.c_str() : g_err3.c_str(); }

}  // extern "C"
