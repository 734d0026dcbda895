// siac_eval_k.cu -- the evaluation kernels of one dG degree k and one schedule, and their
// launchers (siac_internal.h).  Compiled once per (k, schedule) with -DSIAC_K=k -DSIAC_PART=p
// (p = 0 jump + its create-time prep, 1 point, 2 tile, 3 warp-specialized) so the sixteen
// translation units build in parallel.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <vector>

#include "siac_device.cuh"
#include "siac_internal.h"
#if SIAC_PART == 0
#include "siac_jump.cuh"
#elif SIAC_PART == 2
#include "siac_tile.cuh"
#elif SIAC_PART == 3
#include "siac_ws.cuh"
#endif

#ifndef SIAC_K
#error "compile with -DSIAC_K=1..4"
#endif
#ifndef SIAC_PART
#error "compile with -DSIAC_PART=0..3"
#endif

using namespace siacdev;

namespace {

#define CK(call)                                       \
    do {                                               \
        cudaError_t e_ = (call);                       \
        if (e_ != cudaSuccess) return e_;              \
    } while (0)

__device__ __forceinline__ double wrap_coord(double v, double lo, double L) {
    double w = v - L * floor((v - lo) / L);
    if (w >= lo + L) w -= L;   // guard rounding
    if (w < lo) w = lo;
    return w;
}

#if SIAC_PART == 1
// v1: one thread per point (points in Morton order); candidates from the binning cells.
template <int K, bool COUNT>
__global__ void __launch_bounds__(128) k_eval_v1(EvalArgs a) {
    constexpr int RS = Rec<K>::RS;
    constexpr int NB = Rec<K>::NB;
    __shared__ double kc[(3 * K + 1) * (K + 1)];
    for (int i = threadIdx.x; i < (3 * K + 1) * (K + 1); i += blockDim.x) kc[i] = a.kc[i];
    __syncthreads();
    const int64_t sp = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    Counts cnt = {0, 0, 0};
    unsigned long long ncand = 0;
    if (sp < a.np) {
        const int orig = a.perm[sp];
        double x1 = a.pts[2 * (int64_t)orig], x2 = a.pts[2 * (int64_t)orig + 1];
        if (a.periodic & 1) x1 = wrap_coord(x1, a.x0, a.Lx);
        if (a.periodic & 2) x2 = wrap_coord(x2, a.y0, a.Ly);
        // Eq. (3)-style cell bounds of the stencil, extended by the max triangle extent
        // (anchors are bbox-min corners) and one guard cell each side.
        int R0 = (int)floor((x2 - a.hw - a.ey - a.y0) / a.chh) - 1;
        int R1 = (int)floor((x2 + a.hw - a.y0) / a.chh) + 1;
        int C0 = (int)floor((x1 - a.hw - a.ex - a.x0) / a.cw) - 1;
        int C1 = (int)floor((x1 + a.hw - a.x0) / a.cw) + 1;
        if (!(a.periodic & 2)) { R0 = max(R0, 0); R1 = min(R1, a.ncy - 1); }
        if (!(a.periodic & 1)) { C0 = max(C0, 0); C1 = min(C1, a.ncx - 1); }
        double acc = 0.0;
        const double sx0 = x1 - a.hw, sx1 = x1 + a.hw, sy0 = x2 - a.hw, sy1 = x2 + a.hw;
        for (int R = R0; R <= R1; ++R) {
            int r = R, qy = 0;
            if (a.periodic & 2) { r = ((R % a.ncy) + a.ncy) % a.ncy; qy = (R - r) / a.ncy; }
            const double sy = qy * a.Ly;
            int C = C0;
            while (C <= C1) {
                int c = C, qx = 0;
                if (a.periodic & 1) { c = ((C % a.ncx) + a.ncx) % a.ncx; qx = (C - c) / a.ncx; }
                const int cend = (a.periodic & 1) ? min(C1, (qx + 1) * a.ncx - 1) : C1;
                const double sx = qx * a.Lx;
                const int cb = c + (cend - C);
                const int t0 = a.cell_start[r * a.ncx + c], t1 = a.cell_start[r * a.ncx + cb + 1];
                for (int t = t0; t < t1; ++t) {
                    if (COUNT) ++ncand;
                    const double4 b = a.bbox[t];
                    if (!(b.x + sx < sx1 && b.z + sx > sx0 && b.y + sy < sy1 && b.w + sy > sy0)) continue;
                    if (COUNT) cnt.pairs++;
                    const double *rc = a.rec + (int64_t)RS * t;
                    double zx[3], zy[3];
#pragma unroll
                    for (int v = 0; v < 3; ++v) {
                        zx[v] = ((rc[2 * v] + sx) - x1) * a.inv_h;
                        zy[v] = ((rc[2 * v + 1] + sy) - x2) * a.inv_h;
                    }
                    PairGeom g;
                    g.M00 = rc[6]; g.M01 = rc[7]; g.M10 = rc[8]; g.M11 = rc[9];
                    g.zv0x = zx[0]; g.zv0y = zy[0];
                    double d[NB];
#pragma unroll
                    for (int m = 0; m < NB; ++m) d[m] = rc[Rec<K>::OFF_D + m];
                    acc += pair_contrib<K, COUNT>(zx, zy, kc, d, g, cnt);
                }
                C = cend + 1;
            }
        }
        a.out[orig] = acc;
    }
    if (COUNT) {
        unsigned long long v0 = ncand, v1 = cnt.pairs, v2 = cnt.pieces, v3 = cnt.subtris;
        for (int o = 16; o > 0; o >>= 1) {
            v0 += __shfl_down_sync(0xffffffffu, v0, o);
            v1 += __shfl_down_sync(0xffffffffu, v1, o);
            v2 += __shfl_down_sync(0xffffffffu, v2, o);
            v3 += __shfl_down_sync(0xffffffffu, v3, o);
        }
        if ((threadIdx.x & 31) == 0) {
            atomicAdd(a.cnt + 0, v0); atomicAdd(a.cnt + 1, v1);
            atomicAdd(a.cnt + 2, v2); atomicAdd(a.cnt + 3, v3);
        }
    }
}

#endif

#if SIAC_PART == 0
template <int K>
cudaError_t launch_part(const EvalArgs &a, bool count, int *, int num_sms, cudaStream_t st) {

    siacjump::JumpArgs j;
    j.pts = a.pts; j.perm = a.perm; j.np = a.np; j.out = a.out; j.rec = a.rec; j.jrec = a.jrec; j.xrec = a.xrec;
    j.bbox = a.bbox;
    j.cell_start = a.cell_start; j.kc = a.kc; j.x0 = a.x0; j.y0 = a.y0; j.Lx = a.Lx; j.Ly = a.Ly;
    j.inv_h = a.inv_h; j.hw = a.hw; j.cw = a.cw; j.chh = a.chh; j.ex = a.ex; j.ey = a.ey;
    j.ncx = a.ncx; j.ncy = a.ncy; j.periodic = a.periodic; j.cnt = a.cnt;
    // one-sided kernels near the non-periodic boundaries (schedule JUMPX only)
    const bool os = a.os_axes != 0;
    if (os && !a.xpoly) return cudaErrorInvalidValue;
    j.os_axes = a.os_axes; j.h = a.h; j.x1d = a.x1d; j.y1d = a.y1d;
    for (int i = 0; i < 25; ++i) j.osp[i] = 0.0;
    for (int i = 0; i < 6; ++i) j.osb[i] = 0.0;
    for (int i = 0; i < 81; ++i) j.osa[i] = 0.0;
    if (os) {
        for (int i = 0; i < (K + 1) * (K + 1); ++i) j.osp[i] = a.os_pieces[i];
        for (int e = 0; e <= K + 1; ++e)      // beta_e = lead(piece e) - lead(piece e-1)
            j.osb[e] = (e <= K ? a.os_pieces[e * (K + 1) + K] : 0.0) - (e >= 1 ? a.os_pieces[(e - 1) * (K + 1) + K] : 0.0);
        for (int i = 0; i < (2 * K + 1) * (2 * K + 1); ++i) j.osa[i] = a.os_ainv[i];
    }
    const int64_t ntiles = (a.np + 31) / 32;
    // fewer tiles than ~two waves of resident warps: split each tile's rows over 2 or 4 warps
    int split = 1;
    while (split < 4 && split < siacjump::WARPS && ntiles * split < (int64_t)num_sms * 16 * 2) split *= 2;
    j.split = split;
    const int tpb = siacjump::WARPS / split;
    const unsigned grid = (unsigned)((ntiles + tpb - 1) / tpb);
    const size_t smem = ((a.xpoly ? sizeof(siacjump::WarpSmemX) : sizeof(siacjump::WarpSmem)) +
                         sizeof(siacjump::WarpStage<K>) + (os ? sizeof(siacjump::OsSmem<K>) : 0)) * siacjump::WARPS;
    // GEN: some triangle is wider than h (in x or y), so a pair may see two knots on an axis
    const bool gen = std::max(a.ex, a.ey) > a.h * (1.0 + 1e-9);
#define SIAC_LAUNCH_JUMP(C, G, XP, OS)                                                                         \
do {                                                                                                           \
    CK(cudaFuncSetAttribute(siacjump::k_eval_jump<K, C, G, XP, OS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)); \
    siacjump::k_eval_jump<K, C, G, XP, OS><<<grid, siacjump::WARPS * 32, smem, st>>>(j);                      \
} while (0)
#define SIAC_LAUNCH_JUMP2(C, G)                                                                                \
do {                                                                                                           \
    if (os) SIAC_LAUNCH_JUMP(C, G, true, true);                                                                \
    else if (a.xpoly) SIAC_LAUNCH_JUMP(C, G, true, false);                                                     \
    else SIAC_LAUNCH_JUMP(C, G, false, false);                                                                 \
} while (0)
    if (count) { if (gen) SIAC_LAUNCH_JUMP2(true, true); else SIAC_LAUNCH_JUMP2(true, false); }
    else { if (gen) SIAC_LAUNCH_JUMP2(false, true); else SIAC_LAUNCH_JUMP2(false, false); }
#undef SIAC_LAUNCH_JUMP2
#undef SIAC_LAUNCH_JUMP
    return cudaGetLastError();

}
#elif SIAC_PART == 1
template <int K>
cudaError_t launch_part(const EvalArgs &a, bool count, int *, int, cudaStream_t st) {

    const int bs = 128;
    const unsigned grid = (unsigned)((a.np + bs - 1) / bs);
    if (count) k_eval_v1<K, true><<<grid, bs, 0, st>>>(a);
    else k_eval_v1<K, false><<<grid, bs, 0, st>>>(a);
    return cudaGetLastError();

}
#elif SIAC_PART == 2
template <int K>
cudaError_t launch_part(const EvalArgs &a, bool count, int *, int, cudaStream_t st) {
    siactile::TileArgs t;
    t.pts = a.pts; t.perm = a.perm; t.np = a.np; t.out = a.out; t.rec = a.rec; t.bbox = a.bbox;
    t.cell_start = a.cell_start; t.kc = a.kc; t.x0 = a.x0; t.y0 = a.y0; t.Lx = a.Lx; t.Ly = a.Ly;
    t.inv_h = a.inv_h; t.hw = a.hw; t.cw = a.cw; t.chh = a.chh; t.ex = a.ex; t.ey = a.ey;
    t.ncx = a.ncx; t.ncy = a.ncy; t.periodic = a.periodic; t.cnt = a.cnt;
    const int64_t ntiles = (a.np + 31) / 32;
    const unsigned grid = (unsigned)((ntiles + siactile::WARPS - 1) / siactile::WARPS);
    const size_t smem = sizeof(siactile::WarpSmem) * siactile::WARPS;
    if (count) CK(cudaFuncSetAttribute(siactile::k_eval_tile<K, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    else CK(cudaFuncSetAttribute(siactile::k_eval_tile<K, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    if (count) siactile::k_eval_tile<K, true><<<grid, siactile::WARPS * 32, smem, st>>>(t);
    else siactile::k_eval_tile<K, false><<<grid, siactile::WARPS * 32, smem, st>>>(t);
    return cudaGetLastError();
}
#else
template <int K>
cudaError_t launch_part(const EvalArgs &a, bool count, int *tile_counter, int num_sms, cudaStream_t st) {

    siacws::WsArgs w;
    w.pts = a.pts; w.perm = a.perm; w.np = a.np; w.out = a.out; w.rec = a.rec; w.bbox = a.bbox;
    w.cell_start = a.cell_start; w.kc = a.kc; w.x0 = a.x0; w.y0 = a.y0; w.Lx = a.Lx; w.Ly = a.Ly;
    w.inv_h = a.inv_h; w.hw = a.hw; w.cw = a.cw; w.chh = a.chh; w.ex = a.ex; w.ey = a.ey;
    w.ncx = a.ncx; w.ncy = a.ncy; w.periodic = a.periodic; w.cnt = a.cnt; w.tile_counter = tile_counter;
    CK(cudaMemsetAsync(tile_counter, 0, sizeof(int), st));
    const size_t smem = sizeof(siacws::Smem<K>);
    const int64_t ntiles = (a.np + 31) / 32;
    const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(num_sms, ntiles));
    if (count) {
        CK(cudaFuncSetAttribute(siacws::k_eval_ws<K, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        siacws::k_eval_ws<K, true><<<grid, siacws::NWARPS * 32, smem, st>>>(w);
    } else {
        CK(cudaFuncSetAttribute(siacws::k_eval_ws<K, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        siacws::k_eval_ws<K, false><<<grid, siacws::NWARPS * 32, smem, st>>>(w);
    }
    return cudaGetLastError();

}
#endif

}  // namespace

#define SIAC_CAT2(a, b) a##b
#define SIAC_CAT(a, b) SIAC_CAT2(a, b)

#define SIAC_FN(k, p) SIAC_CAT(SIAC_CAT(SIAC_CAT(siac_launch_eval_k, k), _p), p)
cudaError_t SIAC_FN(SIAC_K, SIAC_PART)(const EvalArgs &a, bool count, int *tile_counter, int num_sms,
                                      cudaStream_t st) {
    return launch_part<SIAC_K>(a, count, tile_counter, num_sms, st);
}

#if SIAC_PART == 0
cudaError_t SIAC_CAT(siac_prep_jump_k, SIAC_K)(const double *rec, int64_t nt, double h, double *jrec, cudaStream_t st) {
    siacjump::k_prep_jump<SIAC_K><<<(unsigned)((nt + 127) / 128), 128, 0, st>>>(rec, nt, h, jrec);
    return cudaGetLastError();
}
// Chebyshev interpolation -> monomial matrices (long double): for N nodes x_i = cos((2i+1)pi/2N),
// the interpolant's Chebyshev coefficients are a_j = (w_j) sum_i f_i cos(j (2i+1) pi / 2N)
// (w_0 = 1/N, else 2/N) and T_j = sum_m t_jm x^m (T_0 = 1, T_1 = x, T_j = 2x T_{j-1} - T_{j-2}),
// so the coefficient of x^m is sum_i f_i sum_j t_jm w_j cos(j (2i+1) pi / 2N).
static void cheb_mono_matrix(int N, double *mat, double *nodes) {
    const long double pi = 3.141592653589793238462643383279502884L;
    std::vector<long double> t((size_t)N * N, 0.0L);
    t[0] = 1.0L;
    if (N > 1) t[(size_t)1 * N + 1] = 1.0L;
    for (int j = 2; j < N; ++j)
        for (int m = 0; m < N; ++m)
            t[(size_t)j * N + m] = (m > 0 ? 2.0L * t[(size_t)(j - 1) * N + m - 1] : 0.0L) - t[(size_t)(j - 2) * N + m];
    for (int i = 0; i < N; ++i) nodes[i] = (double)cosl(pi * (2 * i + 1) / (2.0L * N));
    for (int m = 0; m < N; ++m)
        for (int i = 0; i < N; ++i) {
            long double acc = 0.0L;
            for (int j = m; j < N; ++j)
                acc += t[(size_t)j * N + m] * (j == 0 ? 1.0L : 2.0L) / N * cosl(pi * j * (2 * i + 1) / (2.0L * N));
            mat[(size_t)m * N + i] = (double)acc;
        }
}

cudaError_t SIAC_CAT(siac_prep_cross_k, SIAC_K)(const double *jrec, int64_t nt, double *xrec, cudaStream_t st) {
    using X = siacjump::XRec<SIAC_K>;
    siacjump::CrossTabs<SIAC_K> tb;
    cheb_mono_matrix(X::NS, tb.ms, tb.node_s);
    cheb_mono_matrix(X::NL, tb.ml, tb.node_l);
    siacjump::k_prep_cross<SIAC_K><<<(unsigned)((4 * nt + 127) / 128), 128, 0, st>>>(jrec, nt, xrec, tb);
    return cudaGetLastError();
}
int SIAC_CAT(siac_xrec_doubles_k, SIAC_K)() { return siacjump::XRec<SIAC_K>::RS; }
cudaError_t SIAC_CAT(siac_launch_elem_k, SIAC_K)(const EvalArgs &a, bool count, int *, int, cudaStream_t st) {
    if (a.nt == 0) return cudaSuccess;
    siacjump::JumpArgs j;
    j.pts = a.pts; j.perm = a.perm; j.np = a.np; j.out = a.out; j.rec = a.rec; j.jrec = a.jrec; j.xrec = a.xrec;
    j.pcell_start = a.pcell_start; j.bbox = a.bbox; j.cell_start = a.cell_start; j.kc = a.kc; j.split = 1;
    j.x0 = a.x0; j.y0 = a.y0; j.Lx = a.Lx; j.Ly = a.Ly; j.inv_h = a.inv_h; j.hw = a.hw; j.cw = a.cw; j.chh = a.chh;
    j.ex = a.ex; j.ey = a.ey; j.ncx = a.ncx; j.ncy = a.ncy; j.periodic = a.periodic; j.cnt = a.cnt;
    const unsigned grid = (unsigned)((a.nt + siacjump::WARPS - 1) / siacjump::WARPS);
    const bool gen = std::max(a.ex, a.ey) > a.h * (1.0 + 1e-9);
    constexpr int K = SIAC_K;
    if (count) { if (gen) siacjump::k_eval_elem<K, true, true><<<grid, siacjump::WARPS * 32, 0, st>>>(j, a.nt);
                 else siacjump::k_eval_elem<K, true, false><<<grid, siacjump::WARPS * 32, 0, st>>>(j, a.nt); }
    else { if (gen) siacjump::k_eval_elem<K, false, true><<<grid, siacjump::WARPS * 32, 0, st>>>(j, a.nt);
           else siacjump::k_eval_elem<K, false, false><<<grid, siacjump::WARPS * 32, 0, st>>>(j, a.nt); }
    return cudaGetLastError();
}
#endif
