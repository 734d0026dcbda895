// siac_tile.cuh -- the warp-per-point-tile evaluation kernel (schedule TILE: the direct clip-and-integrate method; the default is JUMPX, siac_jump.cuh).
//
// One warp owns a tile of 32 Morton-consecutive evaluation points (buffered stencil:
// every point is written by exactly one warp, so no write races).
// The warp streams three decoupled stages through shared-memory stacks so that the
// divergent geometry never starves the FP64 quadrature:
//   A  candidates -> pairs: triangles from the binning cells covering the tile's stencils
//      (Eq. (3)-style bounds, L434-481), 32 at a time; each lane tests its point's stencil
//      square against each candidate's box (+ periodic image shift), ballot-compacted into
//      a pair stack;
//   B  pairs -> sub-triangles: each lane pops one pair and splits its triangle along the
//      kernel lines (Sutherland-Hodgman passes, Alg. 1; siacdev::gen_pieces) into the
//      pieces T ∩ cell, fan-triangulated; the sub-triangles are staged in shared memory
//      (up to SLOTS per lane; a rare overflow -- only when h is much smaller than the
//      triangles -- is integrated inline by its lane);
//   C  sub-triangles -> values: the staged sub-triangles are compacted across lanes and
//      integrated 32 at a time with the degree-3k rule (full-warp FP64 work); lanes holding
//      the same point are summed by a __match_any_sync segmented reduction, in lane order,
//      into the tile's accumulators (deterministic).
#pragma once

#include "siac_clipfast.cuh"
#include "siac_device.cuh"

namespace siactile {

using namespace siacdev;

#ifndef SIAC_TILE_WARPS
#define SIAC_TILE_WARPS 4
#endif
#ifndef SIAC_TILE_SLOTS
#define SIAC_TILE_SLOTS 8
#endif
#ifndef SIAC_TILE_MINB
#define SIAC_TILE_MINB 3
#endif
constexpr int WARPS = SIAC_TILE_WARPS;   // warps per block
constexpr int SLOTS = SIAC_TILE_SLOTS;   // sub-triangles a lane may stage per generation step
constexpr int PSTACK = 64;      // pair stack: 31 left over + 32 new

// Triangle record layout: siacdev::Rec (siac_device.cuh).
template <int K> using Rec2 = Rec<K>;

struct WarpSmem {
    // staged sub-triangles, index slot * 32 + lane (bank-friendly per slot)
    double sx0[SLOTS * 32], sy0[SLOTS * 32], sx1[SLOTS * 32], sy1[SLOTS * 32], sx2[SLOTS * 32], sy2[SLOTS * 32];
    int scell[SLOTS * 32];      // ci | cj << 5
    int smap[SLOTS * 32];       // compacted index -> slot << 5 | lane
    int gtri[32];               // per generating lane: triangle (binning order)
    int ginfo[32];              // per generating lane: point slot | shift code << 5
    int ptri[PSTACK];
    int pinfo[PSTACK];          // point slot | shift code << 5
    double px[32], py[32];
    double acc[32];
    double4 cbox[32];
};

struct TileArgs {
    const double *pts;
    const int *perm;
    int64_t np;
    double *out;
    const double *rec;
    const double4 *bbox;
    const int *cell_start;
    const double *kc;
    double x0, y0, Lx, Ly, inv_h, hw;
    double cw, chh, ex, ey;
    int ncx, ncy, periodic;
    unsigned long long *cnt;
};

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

// Sum v over lanes with equal key (keys >= 32 are ignored), in lane order, into S.acc[key].
__device__ __forceinline__ void seg_add(WarpSmem &S, int key, double v, int lane) {
    const unsigned grp = __match_any_sync(0xffffffffu, key);
    const int leader = __ffs(grp) - 1;
    double sum = (lane == leader) ? v : 0.0;
    unsigned rest = grp & ~(1u << leader);
    while (__any_sync(0xffffffffu, rest != 0)) {
        const int src = rest ? __ffs(rest) - 1 : lane;
        const double w = __shfl_sync(0xffffffffu, v, src);
        if (rest) { if (lane == leader) sum += w; rest &= rest - 1; }
    }
    if (lane == leader && key < 32) S.acc[key] += sum;
    __syncwarp();
}

// Integrand data of a pair: record fields + the pair's z-frame offset of vertex 0.
template <int K>
__device__ __forceinline__ void pair_data(const TileArgs &a, const WarpSmem &S, int tri, int pinfo, PairGeom &g,
                                          double *d) {
    const double *__restrict__ rc = a.rec + (int64_t)Rec<K>::RS * tri;
    const int slot = pinfo & 31, code = pinfo >> 5;
    const double psx = (double)(code % 3 - 1) * a.Lx, psy = (double)(code / 3 - 1) * a.Ly;
    g.zv0x = ((__ldg(rc + 0) + psx) - S.px[slot]) * a.inv_h;
    g.zv0y = ((__ldg(rc + 1) + psy) - S.py[slot]) * a.inv_h;
    g.M00 = __ldg(rc + 6); g.M01 = __ldg(rc + 7); g.M10 = __ldg(rc + 8); g.M11 = __ldg(rc + 9);
#pragma unroll
    for (int m = 0; m < Rec<K>::NB; ++m) d[m] = __ldg(rc + Rec<K>::OFF_D + m);
}

// General splitter for pairs outside the fast path (h smaller than the triangles, or a
// degenerate split): stages up to SLOTS sub-triangles, integrates any overflow inline.
// Kept out of line so its register demand does not burden the hot path.
template <int K>
__device__ __noinline__ void gen_general(const TileArgs &a, WarpSmem &S, const double *kc, int lane, int tri,
                                         int pinfo, const double *zx, const double *zy, int &cnt, double &extra,
                                         unsigned long long &pieces, unsigned long long &subtris) {
    constexpr int NB = Rec<K>::NB;
    constexpr double T0 = -0.5 * (3 * K + 1);
    bool have_pd = false;
    PairGeom g;
    double d[NB];
    auto emit = [&](const double *qx, const double *qy, int nq, int i, int j) {
        pieces++;
        subtris += nq - 2;
        for (int m = 1; m + 1 < nq; ++m) {
            if (cnt < SLOTS) {
                const int q = cnt * 32 + lane;
                S.sx0[q] = qx[0]; S.sy0[q] = qy[0];
                S.sx1[q] = qx[m]; S.sy1[q] = qy[m];
                S.sx2[q] = qx[m + 1]; S.sy2[q] = qy[m + 1];
                S.scell[q] = i | (j << 5);
                ++cnt;
            } else {
                if (!have_pd) { pair_data<K>(a, S, tri, pinfo, g, d); have_pd = true; }
                double kx[K + 1], ky[K + 1];
#pragma unroll
                for (int mm = 0; mm <= K; ++mm) { kx[mm] = kc[i * (K + 1) + mm]; ky[mm] = kc[j * (K + 1) + mm]; }
                extra += integrate_subtri<K>(qx[0], qy[0], qx[m], qy[m], qx[m + 1], qy[m + 1], kx, ky,
                                             T0 + i + 0.5, T0 + j + 0.5, d, g);
            }
        }
    };
    gen_pieces<K>(zx, zy, emit);
}

template <int K, bool COUNT>
__global__ void __launch_bounds__(WARPS * 32, SIAC_TILE_MINB) k_eval_tile(TileArgs a) {
    constexpr int NC = 3 * K + 1;
    constexpr int NB = Rec<K>::NB;
    constexpr double T0 = -0.5 * (3 * K + 1);
    __shared__ double kc[NC * (K + 1)];
    extern __shared__ __align__(16) unsigned char tile_dsm[];
    WarpSmem *wsm = reinterpret_cast<WarpSmem *>(tile_dsm);
    for (int i = threadIdx.x; i < NC * (K + 1); i += blockDim.x) kc[i] = a.kc[i];
    __syncthreads();

    const int lane = threadIdx.x & 31;
    const int wid = threadIdx.x >> 5;
    WarpSmem &S = wsm[wid];
    const int64_t p0 = ((int64_t)blockIdx.x * WARPS + wid) * 32;
    if (p0 >= a.np) return;                       // warp-uniform
    const bool valid = p0 + lane < a.np;
    int orig = -1;
    double x1 = 0, x2 = 0;
    if (valid) {
        orig = a.perm[p0 + lane];
        x1 = a.pts[2 * (int64_t)orig];
        x2 = a.pts[2 * (int64_t)orig + 1];
        if (a.periodic & 1) { x1 = x1 - a.Lx * floor((x1 - a.x0) / a.Lx); if (x1 >= a.x0 + a.Lx) x1 -= a.Lx; if (x1 < a.x0) x1 = a.x0; }
        if (a.periodic & 2) { x2 = x2 - a.Ly * floor((x2 - a.y0) / a.Ly); if (x2 >= a.y0 + a.Ly) x2 -= a.Ly; if (x2 < a.y0) x2 = a.y0; }
    }
    S.px[lane] = x1;
    S.py[lane] = x2;
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
    __syncwarp();

    // warp-uniform candidate iterator
    int R = R0, C = C0;
    int t_cur = 0, t_end = 0, code = 4;
    double rsx = 0, rsy = 0;
    unsigned chunk_mask = 0;
    int chunk_base = 0, chunk_code = 4;
    bool cand_done = (R0 > R1) || (C0 > C1);
    int npair = 0;
    unsigned long long c_cand = 0, c_pairs = 0, c_pieces = 0, c_sub = 0;

    while (true) {
        // ================= A: candidates -> pairs (until >= 32 stacked)
        while (npair < 32 && !cand_done) {
            if (chunk_mask == 0) {
                while (t_cur >= t_end && R <= R1) {
                    if (C > C1) { ++R; C = C0; continue; }
                    int r = R, qy = 0;
                    if (a.periodic & 2) { r = ((R % a.ncy) + a.ncy) % a.ncy; qy = (R - r) / a.ncy; }
                    int c = C, qx = 0;
                    if (a.periodic & 1) { c = ((C % a.ncx) + a.ncx) % a.ncx; qx = (C - c) / a.ncx; }
                    const int cend = (a.periodic & 1) ? min(C1, (qx + 1) * a.ncx - 1) : C1;
                    const int cb = c + (cend - C);
                    t_cur = a.cell_start[r * a.ncx + c];
                    t_end = a.cell_start[r * a.ncx + cb + 1];
                    code = (qx + 1) + 3 * (qy + 1);
                    rsx = qx * a.Lx;
                    rsy = qy * a.Ly;
                    C = cend + 1;
                }
                if (t_cur >= t_end) { cand_done = true; break; }
                const int n = min(32, t_end - t_cur);
                bool keep = false;
                if (lane < n) {
                    double4 b = a.bbox[t_cur + lane];
                    b.x += rsx; b.z += rsx; b.y += rsy; b.w += rsy;
                    S.cbox[lane] = b;
                    keep = (b.x < bx1 && b.z > bx0 && b.y < by1 && b.w > by0);
                }
                chunk_mask = __ballot_sync(0xffffffffu, keep);
                chunk_base = t_cur;
                chunk_code = code;
                t_cur += n;
                __syncwarp();
                continue;
            }
            const int j = __ffs(chunk_mask) - 1;
            chunk_mask &= chunk_mask - 1;
            const double4 b = S.cbox[j];
            const bool hit = valid && (b.x < sx1 && b.z > sx0 && b.y < sy1 && b.w > sy0);
            const unsigned m = __ballot_sync(0xffffffffu, hit);
            if (COUNT) { c_cand += __popc(__ballot_sync(0xffffffffu, valid)); c_pairs += __popc(m); }
            if (hit) {
                const int pos = npair + __popc(m & lanemask_lt());
                S.ptri[pos] = chunk_base + j;
                S.pinfo[pos] = lane | (chunk_code << 5);
            }
            npair += __popc(m);
            __syncwarp();
        }
        if (npair == 0) break;     // cand_done as well

        // ================= B: every lane takes one pair and stages all of its sub-triangles
        const int take = min(npair, 32);
        int cnt = 0;
        double extra = 0.0;       // sub-triangles beyond SLOTS (tiny h only), integrated inline
        int my_pinfo = 32;        // key for the overflow reduction (32 = none)
        if (lane < take) {
            const int e = npair - 1 - lane;
            const int tri = S.ptri[e];
            const int pinfo = S.pinfo[e];
            S.gtri[lane] = tri;
            S.ginfo[lane] = pinfo;
            my_pinfo = pinfo & 31;
            const int slot = pinfo & 31, pcode = pinfo >> 5;
            const double *__restrict__ rc = a.rec + (int64_t)Rec<K>::RS * tri;
            const double psx = (double)(pcode % 3 - 1) * a.Lx, psy = (double)(pcode / 3 - 1) * a.Ly;
            const double px = S.px[slot], py = S.py[slot];
            siacfast::TriZ TZ;
#pragma unroll
            for (int v = 0; v < 3; ++v) {
                TZ.x[v] = ((__ldg(rc + 2 * v) + psx) - px) * a.inv_h;
                TZ.y[v] = ((__ldg(rc + 2 * v + 1) + psy) - py) * a.inv_h;
                TZ.syx[v] = __ldg(rc + 10 + v);
                TZ.sxy[v] = __ldg(rc + 13 + v);
            }
            unsigned long long f_pieces = 0, f_sub = 0;
            auto emit_fast = [&](const siacfast::Poly &P, int i, int j) {
                if (COUNT) { f_pieces++; f_sub += P.n - 2; }
#pragma unroll
                for (int m = 1; m < 4; ++m) {
                    if (m + 1 < P.n) {     // cnt <= 7 here: at most 7 fan triangles per pair
                        const int q = cnt * 32 + lane;
                        S.sx0[q] = P.x[0]; S.sy0[q] = P.y[0];
                        S.sx1[q] = P.x[m]; S.sy1[q] = P.y[m];
                        S.sx2[q] = P.x[m + 1]; S.sy2[q] = P.y[m + 1];
                        S.scell[q] = i | (j << 5);
                        ++cnt;
                    }
                }
            };
            if (siacfast::gen_pieces_fast<K>(TZ, emit_fast)) {
                if (COUNT) { c_pieces += f_pieces; c_sub += f_sub; }
            } else {
                cnt = 0;                 // discard the partial fast emission
                unsigned long long gp = 0, gs = 0;
                gen_general<K>(a, S, kc, lane, tri, pinfo, TZ.x, TZ.y, cnt, extra, gp, gs);
                if (COUNT) { c_pieces += gp; c_sub += gs; }
            }
        }
        npair -= take;
        __syncwarp();
        if (__any_sync(0xffffffffu, extra != 0.0)) seg_add(S, extra != 0.0 ? my_pinfo : 32 + lane, extra, lane);

        // ================= C: integrate every staged sub-triangle, 32 at a time
        int total;
        {
            const int off = warp_excl_scan(cnt, lane, total);
            for (int m = 0; m < cnt; ++m) S.smap[off + m] = (m << 5) | lane;
            __syncwarp();
        }
        for (int base = 0; base < total; base += 32) {
            const int gi = base + lane;
            const bool act = gi < total;
            int key = 32 + lane;
            double v = 0.0;
            if (act) {
                const int mp = S.smap[gi];
                const int l = mp & 31;
                const int q = (mp >> 5) * 32 + l;
                const int tri = S.gtri[l], pinfo = S.ginfo[l];
                key = pinfo & 31;
                PairGeom g;
                double d[NB];
                pair_data<K>(a, S, tri, pinfo, g, d);
                const int cell = S.scell[q];
                const int ci = cell & 31, cj = cell >> 5;
                double kx[K + 1], ky[K + 1];
#pragma unroll
                for (int m = 0; m <= K; ++m) { kx[m] = kc[ci * (K + 1) + m]; ky[m] = kc[cj * (K + 1) + m]; }
                v = integrate_subtri<K>(S.sx0[q], S.sy0[q], S.sx1[q], S.sy1[q], S.sx2[q], S.sy2[q], kx, ky,
                                        T0 + ci + 0.5, T0 + cj + 0.5, d, g);
            }
            seg_add(S, key, v, lane);
        }
    }
    if (valid) a.out[orig] = S.acc[lane];
    if (COUNT) {
        if (lane == 0) { atomicAdd(a.cnt + 0, c_cand); atomicAdd(a.cnt + 1, c_pairs); }
        unsigned long long v2 = c_pieces, v3 = c_sub;
        for (int o = 16; o > 0; o >>= 1) {
            v2 += __shfl_down_sync(0xffffffffu, v2, o);
            v3 += __shfl_down_sync(0xffffffffu, v3, o);
        }
        if (lane == 0) { atomicAdd(a.cnt + 2, v2); atomicAdd(a.cnt + 3, v3); }
    }
}

}  // namespace siactile
