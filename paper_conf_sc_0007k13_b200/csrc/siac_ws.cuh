// siac_ws.cuh -- warp-specialized evaluation kernel (schedule WS: the direct method with producer/consumer warps; the default is JUMPX, siac_jump.cuh).
//
// The SIAC sum for a point is a stream of fan sub-triangles whose geometry (candidate
// search, Sutherland-Hodgman clipping, Alg. 1 / L369-407) is divergent, branchy
// integer/compare work, while the quadrature of each sub-triangle (Eq. (2)) is
// straight-line FP64 FMA work.  One persistent block per SM runs NPAIR producer/consumer
// warp pairs that overlap the two on every SM sub-partition:
//   producer warp  tiles of 32 Morton-ordered points (dynamic tile counter); per tile:
//                  A  candidate triangles from the binning cells of the tile's stencils,
//                     ballot-tested per point (pairs stacked in shared memory);
//                  B  32 pairs per batch, one per lane: register-only closed-form clipping
//                     (siacfast), fan sub-triangles + per-pair integrand data staged in a
//                     shared-memory batch buffer (double-buffered);
//   consumer warp  waits for a full batch (mbarrier), integrates its sub-triangles 32 at a
//                  time with the degree-3k rule, sums them per point (segmented, lane
//                  order, deterministic) into the batch's result slots and releases it;
//                  the producer folds each batch's per-point results into the tile
//                  accumulators in batch order when it reuses the buffer.
// Every point is owned by exactly one producer warp (buffered stencil, L340-347): no
// global atomics on results.
#pragma once

#include "siac_clipfast.cuh"
#include "siac_device.cuh"

namespace siacws {

using namespace siacdev;

#ifndef SIAC_WS_SUSPEND_NS
#define SIAC_WS_SUSPEND_NS 1000000
#endif
#ifndef SIAC_WS_NPROD
#define SIAC_WS_NPROD 4
#endif
#ifndef SIAC_WS_CPP
#define SIAC_WS_CPP 1
#endif
constexpr int NPAIR = SIAC_WS_NPROD;   // producer warps per block (each with NBUF batch buffers)
constexpr int CPP = SIAC_WS_CPP;       // consumer warps per producer (1: alternates buffers; 2: one per buffer)
constexpr int NWARPS = NPAIR * (1 + CPP);
constexpr int NBUF = 2;                // batch buffers per pair
constexpr int SLOTS = 8;               // staged sub-triangles per lane per batch
constexpr int PSTACK = 64;

template <int K> struct Buf {
    static constexpr int NB = (K + 1) * (K + 2) / 2;
    static constexpr int PD = 2;               // zv0x zv0y (the rest is read from the record)
    double sx0[SLOTS * 32], sy0[SLOTS * 32], sx1[SLOTS * 32], sy1[SLOTS * 32], sx2[SLOTS * 32], sy2[SLOTS * 32];
    double pd[PD][32];
    double sres[SLOTS * 32];                   // value of each staged sub-triangle
    double res[32];
    int scell[SLOTS * 32];
    int smap[SLOTS * 32];
    int pkey[32];
    int ptri[32];                              // record index of each generating lane's pair
    int pcnt[32];                              // staged sub-triangles per generating lane
    int count, flag;
    int pad_[2];
};

struct Prod {
    double px[32], py[32], acc[32];
    double4 cbox[32];
    int ptri[PSTACK], pinfo[PSTACK];
};

template <int K> struct Smem {
    Buf<K> buf[NPAIR][NBUF];
    Prod prod[NPAIR];
    unsigned long long full[NPAIR][NBUF], empty[NPAIR][NBUF];
};

struct WsArgs {
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
    int *tile_counter;
};

// ------------------------------------------------------------------ mbarrier helpers (PTX)

__device__ __forceinline__ unsigned smem_u32(const void *p) {
    return (unsigned)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(unsigned long long *bar, int count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
// Blocking wait for the phase with the given parity.  try_wait suspends the warp for up to
// the hint (ns) instead of spinning, so waiting warps do not steal issue slots from the
// working warps on the same sub-partition.
__device__ __forceinline__ void mbar_wait(unsigned long long *bar, int parity) {
    const unsigned addr = smem_u32(bar);
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1, %2;\n"
        "@!P1 bra WAIT_%=;\n"
        "}\n" ::"r"(addr),
        "r"(parity), "r"(SIAC_WS_SUSPEND_NS)
        : "memory");
}

// consumer-side wait (separate function so profiles attribute the two waits separately)
__device__ __noinline__ static void mbar_wait_full(unsigned long long *bar, int parity) { mbar_wait(bar, parity); }

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

// Sum v over lanes with equal key (keys >= 32 ignored), in lane order, into dst[key].
__device__ __forceinline__ void seg_add(double *dst, int key, double v, int lane) {
    const unsigned grp = __match_any_sync(0xffffffffu, key);
    const int leader = __ffs(grp) - 1;
    double sum = (lane == leader) ? v : 0.0;
    unsigned rest = grp & ~(1u << leader);
    while (__any_sync(0xffffffffu, rest != 0)) {
        const int src = rest ? __ffs(rest) - 1 : lane;
        const double w = __shfl_sync(0xffffffffu, v, src);
        if (rest) { if (lane == leader) sum += w; rest &= rest - 1; }
    }
    if (lane == leader && key < 32) dst[key] += sum;
    __syncwarp();
}

// ------------------------------------------------------------------ general (rare) splitter

// Pairs outside the closed-form path: stage up to SLOTS sub-triangles, integrate any
// overflow inline (returned in extra).  Out of line: keeps its registers off the hot path.
template <int K>
__device__ __noinline__ void gen_general(Buf<K> &B, const double *kc, int lane, const double *zx, const double *zy,
                                         const PairGeom &g, const double *d, int &cnt, double &extra,
                                         unsigned long long &pieces, unsigned long long &subtris) {
    constexpr double T0 = -0.5 * (3 * K + 1);
    auto emit = [&](const double *qx, const double *qy, int nq, int i, int j) {
        pieces++;
        subtris += nq - 2;
        for (int m = 1; m + 1 < nq; ++m) {
            if (cnt < SLOTS) {
                const int q = cnt * 32 + lane;
                B.sx0[q] = qx[0]; B.sy0[q] = qy[0];
                B.sx1[q] = qx[m]; B.sy1[q] = qy[m];
                B.sx2[q] = qx[m + 1]; B.sy2[q] = qy[m + 1];
                B.scell[q] = i | (j << 5);
                ++cnt;
            } else {
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

// ------------------------------------------------------------------ producer

template <int K, bool COUNT>
__device__ __forceinline__ void producer(const WsArgs &a, Smem<K> &SM, const double *kc, int p, int lane) {
    constexpr int NB = Rec<K>::NB;
    Prod &S = SM.prod[p];
    int use[NBUF] = {0, 0};
    bool pending[NBUF] = {false, false};
    int b = 0;
    unsigned long long c_cand = 0, c_pairs = 0, c_pieces = 0, c_sub = 0;
    const int64_t ntiles = (a.np + 31) / 32;

    while (true) {
        int tile = 0;
        if (lane == 0) tile = atomicAdd(a.tile_counter, 1);
        tile = __shfl_sync(0xffffffffu, tile, 0);
        if (tile >= ntiles) break;
        const int64_t p0 = (int64_t)tile * 32;
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
        const double sx0 = x1 - a.hw, sx1 = x1 + a.hw, sy0 = x2 - a.hw, sy1 = x2 + a.hw;
        const double bx0 = tx0 - a.hw, bx1 = tx1 + a.hw, by0 = ty0 - a.hw, by1 = ty1 + a.hw;
        int R0 = (int)floor((by0 - a.ey - a.y0) / a.chh) - 1, R1 = (int)floor((by1 - a.y0) / a.chh) + 1;
        int C0 = (int)floor((bx0 - a.ex - a.x0) / a.cw) - 1, C1 = (int)floor((bx1 - a.x0) / a.cw) + 1;
        if (!(a.periodic & 2)) { R0 = max(R0, 0); R1 = min(R1, a.ncy - 1); }
        if (!(a.periodic & 1)) { C0 = max(C0, 0); C1 = min(C1, a.ncx - 1); }
        __syncwarp();

        int R = R0, C = C0;
        int t_cur = 0, t_end = 0, code = 4;
        double rsx = 0, rsy = 0;
        unsigned chunk_mask = 0;
        int chunk_base = 0, chunk_code = 4;
        bool cand_done = (R0 > R1) || (C0 > C1);
        int npair = 0;

        while (true) {
            // ---------------- A: candidates -> pairs
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
                        t_cur = __ldg(a.cell_start + r * a.ncx + c);
                        t_end = __ldg(a.cell_start + r * a.ncx + cb + 1);
                        code = (qx + 1) + 3 * (qy + 1);
                        rsx = qx * a.Lx;
                        rsy = qy * a.Ly;
                        C = cend + 1;
                    }
                    if (t_cur >= t_end) { cand_done = true; break; }
                    const int n = min(32, t_end - t_cur);
                    bool keep = false;
                    if (lane < n) {
                        double4 bb = a.bbox[t_cur + lane];
                        bb.x += rsx; bb.z += rsx; bb.y += rsy; bb.w += rsy;
                        S.cbox[lane] = bb;
                        keep = (bb.x < bx1 && bb.z > bx0 && bb.y < by1 && bb.w > by0);
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
                const double4 bb = S.cbox[j];
                const bool hit = valid && (bb.x < sx1 && bb.z > sx0 && bb.y < sy1 && bb.w > sy0);
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
            if (npair == 0) break;

            // ---------------- acquire batch buffer b; fold its previous results
            mbar_wait(&SM.empty[p][b], (use[b] & 1) ^ 1);
            Buf<K> &B = SM.buf[p][b];
            if (pending[b]) { S.acc[lane] += B.res[lane]; pending[b] = false; }

            // ---------------- B: one pair per lane -> staged sub-triangles
            const int take = min(npair, 32);
            int cnt = 0;
            double extra = 0.0;
            int key = 32 + lane;
            if (lane < take) {
                const int e = npair - 1 - lane;
                const int tri = S.ptri[e];
                const int pinfo = S.pinfo[e];
                const int slot = pinfo & 31, pcode = pinfo >> 5;
                key = slot;
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
                // integrand data of the pair for the consumer: z-frame vertex 0 + record index
                B.pd[0][lane] = TZ.x[0];
                B.pd[1][lane] = TZ.y[0];
                B.ptri[lane] = tri;
                B.pkey[lane] = slot;
                unsigned long long f_pieces = 0, f_sub = 0;
                auto emit_fast = [&](const siacfast::Poly &P, int i, int j) {
                    if (COUNT) { f_pieces++; f_sub += P.n - 2; }
#pragma unroll
                    for (int m = 1; m < 4; ++m) {
                        if (m + 1 < P.n) {     // <= 7 fan triangles per pair on this path
                            const int q = cnt * 32 + lane;
                            B.sx0[q] = P.x[0]; B.sy0[q] = P.y[0];
                            B.sx1[q] = P.x[m]; B.sy1[q] = P.y[m];
                            B.sx2[q] = P.x[m + 1]; B.sy2[q] = P.y[m + 1];
                            B.scell[q] = i | (j << 5);
                            ++cnt;
                        }
                    }
                };
                if (siacfast::gen_pieces_fast<K>(TZ, emit_fast)) {
                    if (COUNT) { c_pieces += f_pieces; c_sub += f_sub; }
                } else {
                    cnt = 0;           // discard the partial fast emission
                    PairGeom g;
                    g.M00 = __ldg(rc + 6); g.M01 = __ldg(rc + 7); g.M10 = __ldg(rc + 8); g.M11 = __ldg(rc + 9);
                    g.zv0x = TZ.x[0]; g.zv0y = TZ.y[0];
                    double d[NB];
#pragma unroll
                    for (int f = 0; f < NB; ++f) d[f] = __ldg(rc + Rec<K>::OFF_D + f);
                    unsigned long long gp = 0, gs = 0;
                    gen_general<K>(B, kc, lane, TZ.x, TZ.y, g, d, cnt, extra, gp, gs);
                    if (COUNT) { c_pieces += gp; c_sub += gs; }
                }
            }
            npair -= take;
            B.pcnt[lane] = cnt;
            if (lane >= take) B.pkey[lane] = 32 + lane;
            int total;
            const int off = warp_excl_scan(cnt, lane, total);
            for (int m = 0; m < cnt; ++m) B.smap[off + m] = (m << 5) | lane;
            if (lane == 0) { B.count = total; B.flag = 0; }
            __syncwarp();
            if (__any_sync(0xffffffffu, extra != 0.0)) seg_add(S.acc, extra != 0.0 ? key : 32 + lane, extra, lane);
            mbar_arrive(&SM.full[p][b]);
            pending[b] = true;
            ++use[b];
            b ^= 1;
        }
        // tile done: collect outstanding batches (in issue order), write the values
        for (int k2 = 0; k2 < NBUF; ++k2) {
            const int bb = (b + k2) % NBUF;       // oldest first
            if (pending[bb]) {
                mbar_wait(&SM.empty[p][bb], (use[bb] & 1) ^ 1);
                S.acc[lane] += SM.buf[p][bb].res[lane];
                pending[bb] = false;
            }
        }
        __syncwarp();
        if (valid) a.out[orig] = S.acc[lane];
    }
    // termination batch on every buffer (each consumer reads at least one of them)
    for (int k2 = 0; k2 < NBUF; ++k2) {
        const int bb = (b + k2) % NBUF;
        mbar_wait(&SM.empty[p][bb], (use[bb] & 1) ^ 1);
        if (lane == 0) { SM.buf[p][bb].flag = 1; SM.buf[p][bb].count = 0; }
        __syncwarp();
        mbar_arrive(&SM.full[p][bb]);
        ++use[bb];
    }
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

// ------------------------------------------------------------------ consumer

#ifndef SIAC_WS_ILP
#define SIAC_WS_ILP 1
#endif

template <int K>
__device__ __forceinline__ void load_subtri(const Buf<K> &B, const double *__restrict__ rec, const double *kc, int gi,
                                            SubTri<K> &t, int &q) {
    constexpr int NB = Rec<K>::NB;
    constexpr double T0 = -0.5 * (3 * K + 1);
    const int mp = B.smap[gi];
    const int l = mp & 31;
    q = (mp >> 5) * 32 + l;
    const double *__restrict__ rc = rec + (int64_t)Rec<K>::RS * B.ptri[l];
    t.g.M00 = __ldg(rc + 6); t.g.M01 = __ldg(rc + 7); t.g.M10 = __ldg(rc + 8); t.g.M11 = __ldg(rc + 9);
    t.g.zv0x = B.pd[0][l]; t.g.zv0y = B.pd[1][l];
#pragma unroll
    for (int f = 0; f < NB; ++f) t.d[f] = __ldg(rc + Rec<K>::OFF_D + f);
    const int cell = B.scell[q];
    const int ci = cell & 31, cj = cell >> 5;
#pragma unroll
    for (int m = 0; m <= K; ++m) { t.kx[m] = kc[ci * (K + 1) + m]; t.ky[m] = kc[cj * (K + 1) + m]; }
    t.cx = T0 + ci + 0.5;
    t.cy = T0 + cj + 0.5;
    t.p0x = B.sx0[q]; t.p0y = B.sy0[q];
    t.e1x = B.sx1[q] - t.p0x; t.e1y = B.sy1[q] - t.p0y;
    t.e2x = B.sx2[q] - t.p0x; t.e2y = B.sy2[q] - t.p0y;
}

template <int K>
__device__ __forceinline__ void consumer(Smem<K> &SM, const double *__restrict__ rec, const double *kc, int p, int j,
                                         int lane) {
    constexpr int ILP = SIAC_WS_ILP;
    int use[NBUF] = {0, 0};
    int b = (CPP == 1) ? 0 : j;
    while (true) {
        mbar_wait_full(&SM.full[p][b], use[b] & 1);
        Buf<K> &B = SM.buf[p][b];
        if (B.flag) break;
#ifndef SIAC_WS_EXP
#define SIAC_WS_EXP 0
#endif
        // experiments: 1 = skip the quadrature (producer-bound timing); 2 = integrate each
        // batch three times (consumer-bound timing)
        const int total = (SIAC_WS_EXP == 1) ? 0 : B.count;
        for (int rep = 0; rep < (SIAC_WS_EXP == 2 ? 3 : 1); ++rep) {
        int base = 0;
        // full rounds of ILP x 32 sub-triangles: every lane integrates ILP of them together
        for (; total - base >= ILP * 32; base += ILP * 32) {
            SubTri<K> t[ILP];
            int q[ILP];
            double v[ILP];
#pragma unroll
            for (int n = 0; n < ILP; ++n) load_subtri<K>(B, rec, kc, base + n * 32 + lane, t[n], q[n]);
            integrate_subtri_n<K, ILP>(t, v);
#pragma unroll
            for (int n = 0; n < ILP; ++n) B.sres[q[n]] = v[n];
        }
        // remainder, one per lane
        for (; base < total; base += 32) {
            const int gi = base + lane;
            if (gi < total) {
                SubTri<K> t[1];
                int q;
                double v[1];
                load_subtri<K>(B, rec, kc, gi, t[0], q);
                integrate_subtri_n<K, 1>(t, v);
                B.sres[q] = v[0];
            }
        }
        }
        __syncwarp();
        // per pair (generating lane) sums in slot order, then per point (lane order)
        double ps = 0.0;
        const int c = B.pcnt[lane];
        for (int m = 0; m < c; ++m) ps += B.sres[m * 32 + lane];
        B.res[lane] = 0.0;
        __syncwarp();
        seg_add(B.res, B.pkey[lane], ps, lane);
        mbar_arrive(&SM.empty[p][b]);
        ++use[b];
        if (CPP == 1) b ^= 1;
    }
}

template <int K, bool COUNT>
__global__ void __launch_bounds__(NWARPS * 32, 1) k_eval_ws(WsArgs a) {
    constexpr int NC = 3 * K + 1;
    __shared__ double kc[NC * (K + 1)];
    extern __shared__ __align__(16) unsigned char ws_dsm[];
    Smem<K> &SM = *reinterpret_cast<Smem<K> *>(ws_dsm);
    for (int i = threadIdx.x; i < NC * (K + 1); i += blockDim.x) kc[i] = a.kc[i];
    if (threadIdx.x == 0) {
        for (int p = 0; p < NPAIR; ++p)
            for (int b = 0; b < NBUF; ++b) {
                mbar_init(&SM.full[p][b], 32);     // all producer lanes arrive
                mbar_init(&SM.empty[p][b], 32);
            }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (warp < NPAIR) producer<K, COUNT>(a, SM, kc, warp, lane);
    else consumer<K>(SM, a.rec, kc, (warp - NPAIR) / CPP, (warp - NPAIR) % CPP, lane);
}

}  // namespace siacws
