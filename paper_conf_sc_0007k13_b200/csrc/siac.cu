// siac.cu -- C ABI (include/siac.h) and kernels of the B200 SIAC post-processor.
//
// Pipeline:
//   siac_create:  host validation + exact constants (siac_math.hpp) -> H2D of V, T, C ->
//                 k_prep (per-triangle record, bbox, anchor cell) -> CUB radix sort by anchor
//                 cell -> k_gather (records in cell order) -> k_cell_start (CSR offsets).
//                 -> k_prep_jump (moments, corner polynomials) -> k_prep_cross (interval
//                 polynomials of the clipped reference corners), all on the context's stream.
//   siac_eval_async: k_point_keys (periodic wrap, Morton key of a grid finer than the binning
//                 cells) -> CUB radix sort -> the schedule's evaluation kernel (default
//                 k_eval_jump<K,..,JUMPX>: candidate triangles from the cells of each 32-point
//                 tile's Eq. (3)-style bounds, the spline-jump decomposition of Eq. (2) in closed
//                 form per pair, one accumulator per point, written in input order).
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <functional>
#include <string>
#include <vector>

#include <cub/device/device_radix_sort.cuh>

#include "../../include/siac.h"
#include "siac_device.cuh"
#include "siac_jump.cuh"
#include "siac_internal.h"
#include "siac_math.h"

#define SIAC_VERSION "siac-b200 0.1 (sm_100a, fp64)"

using namespace siacdev;

struct siac_ctx {
    int device = 0;
    cudaStream_t stream = nullptr;   // the context's own non-blocking stream (create, siac_eval)
    int k = 1;
    int basis = 0, boundary = 0;
    std::vector<double> os_pieces, os_ainv;   // one-sided kernel tables (siac::onesided_tables)
    siac_create_info cinfo = {};
    double h = 0, inv_h = 0;
    int periodic = 0;
    double dom[4] = {0, 0, 1, 1};
    int64_t nt = 0;
    // binning grid
    int ncx = 1, ncy = 1;
    double cw = 1, chh = 1;      // cell width / height
    double ex = 0, ey = 0;       // max triangle bbox extents
    // device mesh
    double *d_rec = nullptr;
    double *d_jrec = nullptr;    // schedule JUMP records (siac_jump.cuh)
    double *d_xrec = nullptr;    // closed-form cross-term polynomials (schedule JUMP-X)
    int *d_pcell = nullptr;      // schedule ELEM: point CSR by row-major binning cell
    double4 *d_bbox = nullptr;
    int *d_cell_start = nullptr;
    double *d_kc = nullptr;
    // eval scratch
    int64_t cap = 0;
    uint32_t *d_keys[2] = {nullptr, nullptr};
    int *d_idx[2] = {nullptr, nullptr};
    void *d_cub = nullptr;
    size_t cub_bytes = 0;
    int64_t cap_host = 0;
    int64_t scratch_bytes = 0;
    double *d_hpts = nullptr, *d_hout = nullptr;
    // counters
    int schedule = 0;            // 0 = default (= 5), 1 = thread-per-point, 2 = warp-per-tile, 3 = warp-specialized, 4 = jump, 5 = jump-x, 6 = per-element
    int *d_tile_counter = nullptr;
    int num_sms = 148;
    bool counting = false;
    unsigned long long *d_cnt = nullptr;
    int64_t last_np = 0;
    // CUDA graphs of whole evaluations (siac_set_graphs): one per (points, n, values, schedule)
    bool graphs = false;
    struct GraphEntry {
        const double *pts;
        int64_t np;
        double *out;
        int schedule;
        cudaGraphExec_t exec;
    };
    std::vector<GraphEntry> gcache;
    // main-kernel timing (CUDA events on the evaluation stream)
    bool timing = false;
    std::vector<std::pair<cudaEvent_t, cudaEvent_t>> ev;
    size_t ev_used = 0;
    std::string err;
};

static thread_local std::string g_err;
void siac_set_thread_error(const std::string &msg) { g_err = msg; }   // siac_io.cu (siac_internal.h)

namespace {

struct Fail {
    siac_status st;
    std::string msg;
};

#define CK(call)                                                                               \
    do {                                                                                       \
        cudaError_t e_ = (call);                                                               \
        if (e_ != cudaSuccess)                                                                 \
            throw Fail{SIAC_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e_)};        \
    } while (0)

// (const char *: the hot validation loops must not build a std::string per check)
inline void need(bool ok, const char *msg) {
    if (__builtin_expect(!ok, 0)) throw Fail{SIAC_EINVAL, std::string(msg)};
}

// ------------------------------------------------------------------ create kernels

struct PrepArgs {
    const double *V;
    const int *T;
    const double *C;
    const double *R;        // nb x nb Dubiner -> centred monomial (row = mode)
    int64_t nt;
    int nb, rs;
    double h, x0, y0, cw, chh;
    int ncx, ncy;
    double *rec;            // unsorted records
    double4 *bbox;
    uint32_t *key;
    int *idx;
};

__global__ void k_prep(PrepArgs a) {
    int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= a.nt) return;
    const int i0 = a.T[3 * t], i1 = a.T[3 * t + 1], i2 = a.T[3 * t + 2];
    const double v0x = a.V[2 * i0], v0y = a.V[2 * i0 + 1];
    const double v1x = a.V[2 * i1], v1y = a.V[2 * i1 + 1];
    const double v2x = a.V[2 * i2], v2y = a.V[2 * i2 + 1];
    double *r = a.rec + (int64_t)a.rs * t;
    r[0] = v0x; r[1] = v0y; r[2] = v1x; r[3] = v1y; r[4] = v2x; r[5] = v2y;
    const double a11 = v1x - v0x, a12 = v2x - v0x, a21 = v1y - v0y, a22 = v2y - v0y;
    const double det = a11 * a22 - a12 * a21;
    const double f = 3.0 * a.h / det;
    r[6] = f * a22; r[7] = -f * a12; r[8] = -f * a21; r[9] = f * a11;
    const double vx[3] = {v0x, v1x, v2x}, vy[3] = {v0y, v1y, v2y};
    for (int g = 0; g < 3; ++g) {
        const double dx = vx[(g + 1) % 3] - vx[g], dy = vy[(g + 1) % 3] - vy[g];
        r[10 + g] = dy / dx;         // +-inf for a vertical edge (never used for vertical lines)
        r[13 + g] = dx / dy;
    }
    const double *c = a.C + (int64_t)a.nb * t;
    for (int j = 0; j < a.nb; ++j) {
        double s = 0.0;
        for (int i = 0; i < a.nb; ++i) s = fma(c[i], a.R[i * a.nb + j], s);
        r[16 + j] = s;
    }
    for (int j = 16 + a.nb; j < a.rs; ++j) r[j] = 0.0;
    const double bx0 = fmin(v0x, fmin(v1x, v2x)), bx1 = fmax(v0x, fmax(v1x, v2x));
    const double by0 = fmin(v0y, fmin(v1y, v2y)), by1 = fmax(v0y, fmax(v1y, v2y));
    a.bbox[t] = make_double4(bx0, by0, bx1, by1);
    int cx = (int)floor((bx0 - a.x0) / a.cw), cy = (int)floor((by0 - a.y0) / a.chh);
    cx = cx < 0 ? 0 : (cx >= a.ncx ? a.ncx - 1 : cx);
    cy = cy < 0 ? 0 : (cy >= a.ncy ? a.ncy - 1 : cy);
    a.key[t] = (uint32_t)cy * (uint32_t)a.ncx + (uint32_t)cx;
    a.idx[t] = (int)t;
}

__global__ void k_gather(const double *rec_u, const double4 *bbox_u, const int *idx, int64_t nt, int rs,
                         double *rec, double4 *bbox) {
    int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= nt) return;
    const int t = idx[s];
    for (int j = 0; j < rs; ++j) rec[(int64_t)rs * s + j] = rec_u[(int64_t)rs * t + j];
    bbox[s] = bbox_u[t];
}

// cell_start[c] = first sorted position whose key >= c (c = 0..ncell)
__global__ void k_cell_start(const uint32_t *keys, int64_t nt, int64_t ncell, int *cell_start) {
    int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (c > ncell) return;
    int64_t lo = 0, hi = nt;
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if ((int64_t)keys[mid] < c) lo = mid + 1;
        else hi = mid;
    }
    cell_start[c] = (int)lo;
}

// ------------------------------------------------------------------ eval kernels



__device__ __forceinline__ uint32_t spread16(uint32_t v) {
    v &= 0xFFFF;
    v = (v | (v << 8)) & 0x00FF00FF;
    v = (v | (v << 4)) & 0x0F0F0F0F;
    v = (v | (v << 2)) & 0x33333333;
    v = (v | (v << 1)) & 0x55555555;
    return v;
}

__device__ __forceinline__ double wrap_coord(double v, double lo, double L) {
    double w = v - L * floor((v - lo) / L);
    if (w >= lo + L) w -= L;   // guard rounding
    if (w < lo) w = lo;
    return w;
}

__global__ void k_point_keys(const double *pts, int64_t np, double x0, double y0, double Lx, double Ly,
                             int periodic, double cw, double chh, int ncx, int ncy, uint32_t *key, int *idx,
                             int rowmajor) {
    int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= np) return;
    double x = pts[2 * i], y = pts[2 * i + 1];
    if (periodic & 1) x = wrap_coord(x, x0, Lx);
    if (periodic & 2) y = wrap_coord(y, y0, Ly);
    int cx = (int)fmin(fmax(floor((x - x0) / cw), 0.0), (double)(ncx - 1));
    int cy = (int)fmin(fmax(floor((y - y0) / chh), 0.0), (double)(ncy - 1));
    key[i] = rowmajor ? (uint32_t)cy * (uint32_t)ncx + (uint32_t)cx : spread16((uint32_t)cx) | (spread16((uint32_t)cy) << 1);
    idx[i] = (int)i;
}

inline unsigned nblk(int64_t n, int bs) { return (unsigned)((n + bs - 1) / bs); }

void clear_graphs(siac_ctx *c);

void ensure_scratch(siac_ctx *c, int64_t np) {
    if (np <= c->cap) return;
    clear_graphs(c);                 // captured graphs point at the old scratch buffers
    int64_t cap = std::max<int64_t>(np, c->cap * 3 / 2);
    for (int b = 0; b < 2; ++b) {
        if (c->d_keys[b]) cudaFree(c->d_keys[b]);
        if (c->d_idx[b]) cudaFree(c->d_idx[b]);
        c->d_keys[b] = nullptr; c->d_idx[b] = nullptr;
    }
    if (c->d_cub) cudaFree(c->d_cub);
    c->d_cub = nullptr;
    c->cap = 0;
    for (int b = 0; b < 2; ++b) {
        CK(cudaMalloc(&c->d_keys[b], sizeof(uint32_t) * cap));
        CK(cudaMalloc(&c->d_idx[b], sizeof(int) * cap));
    }
    cub::DoubleBuffer<uint32_t> kb(c->d_keys[0], c->d_keys[1]);
    cub::DoubleBuffer<int> vb(c->d_idx[0], c->d_idx[1]);
    size_t bytes = 0;
    CK(cub::DeviceRadixSort::SortPairs(nullptr, bytes, kb, vb, (int)cap));
    CK(cudaMalloc(&c->d_cub, bytes));
    c->cub_bytes = bytes;
    c->cap = cap;
}

void eval_device(siac_ctx *c, const double *d_pts, int64_t np, double *d_out, cudaStream_t st) {
    CK(cudaSetDevice(c->device));
    need(np <= (int64_t)0x7fffffff, "n_points must be < 2^31");
    ensure_scratch(c, np);
    const double Lx = c->dom[2] - c->dom[0], Ly = c->dom[3] - c->dom[1];
    const bool elem = c->schedule == 6;          // per-element: points in row-major cell order
#ifndef SIAC_TILE_REFINE
#define SIAC_TILE_REFINE 4
#endif
    // point tiles: Morton order of a grid SIAC_TILE_REFINE x finer than the binning cells (more
    // compact 32-point tiles -> fewer candidates per tile); per-element: row-major binning cells
    const int rf = elem ? 1 : std::max(1, std::min(SIAC_TILE_REFINE, 65536 / std::max(c->ncx, c->ncy)));
    k_point_keys<<<nblk(np, 256), 256, 0, st>>>(d_pts, np, c->dom[0], c->dom[1], Lx, Ly, c->periodic, c->cw / rf,
                                                c->chh / rf, c->ncx * rf, c->ncy * rf, c->d_keys[0], c->d_idx[0],
                                                elem ? 1 : 0);
    CK(cudaGetLastError());
    cub::DoubleBuffer<uint32_t> kb(c->d_keys[0], c->d_keys[1]);
    cub::DoubleBuffer<int> vb(c->d_idx[0], c->d_idx[1]);
    int end_bit = 1;
    while ((1ull << end_bit) <= (unsigned long long)std::max(c->ncx, c->ncy) * rf && end_bit < 16) ++end_bit;
    int key_bits = 2 * end_bit;
    if (elem) {
        key_bits = 1;
        while ((1ull << key_bits) < (unsigned long long)c->ncx * c->ncy && key_bits < 32) ++key_bits;
    }
    CK(cub::DeviceRadixSort::SortPairs(c->d_cub, c->cub_bytes, kb, vb, (int)np, 0, key_bits, st));
    EvalArgs a;
    a.pts = d_pts; a.perm = vb.Current(); a.np = np; a.out = d_out;
    a.rec = c->d_rec; a.jrec = c->d_jrec; a.xrec = c->d_xrec; a.bbox = c->d_bbox; a.cell_start = c->d_cell_start;
    a.kc = c->d_kc;
    a.xpoly = (c->schedule == 0 || c->schedule == 5) ? 1 : 0;
    a.nt = c->nt;
    a.pcell_start = nullptr;
    if (elem) {
        const int64_t ncell = (int64_t)c->ncx * c->ncy;
        if (!c->d_pcell) CK(cudaMalloc(&c->d_pcell, sizeof(int) * (ncell + 1)));
        k_cell_start<<<nblk(ncell + 1, 256), 256, 0, st>>>(kb.Current(), np, ncell, c->d_pcell);
        CK(cudaGetLastError());
        CK(cudaMemsetAsync(d_out, 0, sizeof(double) * np, st));    // the pairs scatter-add
        a.pcell_start = c->d_pcell;
    }
    a.x0 = c->dom[0]; a.y0 = c->dom[1]; a.Lx = Lx; a.Ly = Ly;
    a.h = c->h; a.inv_h = c->inv_h; a.hw = 0.5 * (3 * c->k + 1) * c->h;
    a.cw = c->cw; a.chh = c->chh; a.ex = c->ex; a.ey = c->ey;
    a.ncx = c->ncx; a.ncy = c->ncy; a.periodic = c->periodic;
    a.cnt = c->d_cnt;
    a.os_axes = c->boundary == SIAC_BOUNDARY_ONESIDED ? (~c->periodic & 3) : 0;
    a.x1d = c->dom[2]; a.y1d = c->dom[3];
    a.os_pieces = c->os_pieces.data(); a.os_ainv = c->os_ainv.data();
    need(a.os_axes == 0 || c->schedule == 0 || c->schedule == 5,
         "SIAC_BOUNDARY_ONESIDED is implemented by the default schedule (JUMPX) only");
    if (c->counting) CK(cudaMemsetAsync(c->d_cnt, 0, 8 * sizeof(unsigned long long), st));
    cudaEvent_t ev_stop = nullptr;
    if (c->timing) {
        if (c->ev_used == c->ev.size()) {
            cudaEvent_t e0, e1;
            CK(cudaEventCreate(&e0));
            CK(cudaEventCreate(&e1));
            c->ev.push_back({e0, e1});
        }
        CK(cudaEventRecord(c->ev[c->ev_used].first, st));
        ev_stop = c->ev[c->ev_used].second;
        ++c->ev_used;
    }
    // schedule -> part: 0 (default) / 5 = jump-x and 4 = jump (p0), 1 = point (p1), 2 = tile (p2), 3 = ws (p3)
    static const siac_launch_fn table[4][4] = {
        {siac_launch_eval_k1_p0, siac_launch_eval_k1_p1, siac_launch_eval_k1_p2, siac_launch_eval_k1_p3},
        {siac_launch_eval_k2_p0, siac_launch_eval_k2_p1, siac_launch_eval_k2_p2, siac_launch_eval_k2_p3},
        {siac_launch_eval_k3_p0, siac_launch_eval_k3_p1, siac_launch_eval_k3_p2, siac_launch_eval_k3_p3},
        {siac_launch_eval_k4_p0, siac_launch_eval_k4_p1, siac_launch_eval_k4_p2, siac_launch_eval_k4_p3}};
    if (c->k < 1 || c->k > 4) throw Fail{SIAC_EINTERNAL, "bad k"};
    const int part = (c->schedule == 0 || c->schedule >= 4) ? 0 : c->schedule;
    static const siac_launch_fn elem_table[4] = {siac_launch_elem_k1, siac_launch_elem_k2, siac_launch_elem_k3,
                                                 siac_launch_elem_k4};
    const cudaError_t e = elem ? elem_table[c->k - 1](a, c->counting, c->d_tile_counter, c->num_sms, st)
                               : table[c->k - 1][part](a, c->counting, c->d_tile_counter, c->num_sms, st);
    CK(e);
    CK(cudaGetLastError());
    if (ev_stop) CK(cudaEventRecord(ev_stop, st));
    c->last_np = np;
}

// DFMA throughput probe: 8 independent FMA chains per thread, every SM full.
__global__ void __launch_bounds__(512) k_dfma_probe(double *out, int iters, double m, double cst) {
    double a[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) a[j] = 1e-9 * threadIdx.x + j;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j) a[j] = fma(a[j], m, cst);
    }
    double s = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) s += a[j];
    if (s == 1234.5678) out[blockIdx.x] = s;   // never true; keeps the chains alive
}

void clear_graphs(siac_ctx *c) {
    for (auto &g : c->gcache) cudaGraphExecDestroy(g.exec);
    c->gcache.clear();
}

void free_ctx(siac_ctx *c) {
    if (!c) return;
    cudaSetDevice(c->device);
    clear_graphs(c);
    for (auto &e : c->ev) { cudaEventDestroy(e.first); cudaEventDestroy(e.second); }
    void *ptrs[] = {c->d_rec, c->d_jrec, c->d_xrec, c->d_pcell, c->d_bbox, c->d_cell_start, c->d_kc, c->d_keys[0], c->d_keys[1],
                    c->d_idx[0], c->d_idx[1], c->d_cub, c->d_hpts, c->d_hout, c->d_cnt, c->d_tile_counter};
    for (void *p : ptrs)
        if (p) cudaFree(p);
    if (c->stream) cudaStreamDestroy(c->stream);
    delete c;
}

// ------------------------------------------------------------------ C ABI

siac_status run_guarded(std::string *err, const std::function<void()> &fn) {
    try {
        fn();
        return SIAC_OK;
    } catch (const Fail &f) {
        *err = f.msg;
        return f.st;
    } catch (const std::bad_alloc &) {
        *err = "host allocation failed";
        return SIAC_ENOMEM;
    } catch (const std::exception &e) {
        *err = std::string("internal error: ") + e.what();
        return SIAC_EINTERNAL;
    } catch (...) {
        *err = "unknown internal error";
        return SIAC_EINTERNAL;
    }
}
}  // namespace

extern "C" {

const char *siac_version(void) { return SIAC_VERSION; }

const char *siac_last_error(const siac_ctx *ctx) { return ctx ? ctx->err.c_str() : g_err.c_str(); }

siac_status siac_create(siac_ctx **out, const double *V, int64_t nv, const int32_t *T, int64_t nt,
                        const double *C, const siac_params *p) {
    if (out) *out = nullptr;
    siac_ctx *c = nullptr;
    const auto t_start = std::chrono::steady_clock::now();
    auto ms_since = [](std::chrono::steady_clock::time_point t0) {
        return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    };
    siac_status st = run_guarded(&g_err, [&]() {
        need(out != nullptr && p != nullptr, "out and params must be non-NULL");
        need(p->k >= 1 && p->k <= 4, "k must be in 1..4");
        need(std::isfinite(p->h) && p->h > 0, "h must be finite and > 0");
        need(nv >= 0 && nt >= 0, "negative sizes");
        need(nt == 0 || (V && T && C), "NULL mesh arrays");
        need((p->periodic & ~3) == 0, "periodic must be a combination of SIAC_PERIODIC_X|Y");
        need(p->basis == SIAC_BASIS_DUBINER_ORTHONORMAL || p->basis == SIAC_BASIS_MONOMIAL_REF, "unknown basis");
        need(p->boundary == SIAC_BOUNDARY_ZERO || p->boundary == SIAC_BOUNDARY_ONESIDED, "unknown boundary");
        for (int i = 0; i < 4; ++i) need(std::isfinite(p->domain[i]), "non-finite domain");
        const double Lx = p->domain[2] - p->domain[0], Ly = p->domain[3] - p->domain[1];
        need(Lx > 0 && Ly > 0, "empty or inverted domain");
        const int k = p->k;
        const double W = (3 * k + 1) * p->h;
        need(!(p->periodic & 1) || W <= Lx * (1 + 1e-12), "(3k+1)h exceeds the periodic x-extent");
        need(!(p->periodic & 2) || W <= Ly * (1 + 1e-12), "(3k+1)h exceeds the periodic y-extent");
        if (p->boundary == SIAC_BOUNDARY_ONESIDED) {
            need((p->periodic & 1) || W <= Lx * (1 + 1e-12), "one-sided kernel: (3k+1)h exceeds the x-extent");
            need((p->periodic & 2) || W <= Ly * (1 + 1e-12), "one-sided kernel: (3k+1)h exceeds the y-extent");
        }
        need(nt <= (int64_t)0x3fffffff, "too many triangles");
        const int nb = (k + 1) * (k + 2) / 2;
        // host validation pass
        const double tolx = 1e-9 * Lx, toly = 1e-9 * Ly;
        for (int64_t i = 0; i < nv; ++i) {
            need(std::isfinite(V[2 * i]) && std::isfinite(V[2 * i + 1]), "non-finite vertex coordinate");
            if (p->periodic & 1)
                need(V[2 * i] >= p->domain[0] - tolx && V[2 * i] <= p->domain[2] + tolx, "vertex outside the periodic x-range");
            if (p->periodic & 2)
                need(V[2 * i + 1] >= p->domain[1] - toly && V[2 * i + 1] <= p->domain[3] + toly, "vertex outside the periodic y-range");
        }
        double ex = 0, ey = 0;
        for (int64_t t = 0; t < nt; ++t) {
            int a = T[3 * t], b = T[3 * t + 1], d = T[3 * t + 2];
            need(a >= 0 && a < nv && b >= 0 && b < nv && d >= 0 && d < nv, "triangle index out of range");
            const double ax = V[2 * a], ay = V[2 * a + 1], bx = V[2 * b], by = V[2 * b + 1], dx = V[2 * d], dy = V[2 * d + 1];
            const double det = (bx - ax) * (dy - ay) - (dx - ax) * (by - ay);
            const double sx = std::max({ax, bx, dx}) - std::min({ax, bx, dx});
            const double sy = std::max({ay, by, dy}) - std::min({ay, by, dy});
            need(std::fabs(det) > 1e-14 * sx * sy && det != 0.0, "zero-area triangle");
            ex = std::max(ex, sx);
            ey = std::max(ey, sy);
            for (int j = 0; j < nb; ++j) need(std::isfinite(C[nb * t + j]), "non-finite coefficient");
        }
        int ndev = 0;
        if (cudaGetDeviceCount(&ndev) != cudaSuccess || p->device < 0 || p->device >= ndev)
            throw Fail{SIAC_EDEVICE, "no CUDA device with that ordinal"};
        int major = 0, nsm = 0;
        CK(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, p->device));
        CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, p->device));
        if (major < 10) {
            cudaDeviceProp prop;
            CK(cudaGetDeviceProperties(&prop, p->device));
            throw Fail{SIAC_EDEVICE, std::string("device is not sm_100 class: ") + prop.name};
        }
        CK(cudaSetDevice(p->device));

        c = new siac_ctx();
        c->device = p->device;
        CK(cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking));
        c->basis = p->basis;
        c->boundary = p->boundary;
        if (p->boundary == SIAC_BOUNDARY_ONESIDED) siac::onesided_tables(k, c->os_pieces, c->os_ainv);
        c->k = k;
        c->h = p->h;
        c->inv_h = 1.0 / p->h;
        c->periodic = p->periodic;
        for (int i = 0; i < 4; ++i) c->dom[i] = p->domain[i];
        c->nt = nt;
        c->ex = ex;
        c->ey = ey;
        const double cf = p->cell_factor > 0 ? p->cell_factor : 0.5;
        c->ncx = (int)std::max(1.0, std::min(4096.0, std::floor(Lx / (cf * p->h))));
        c->ncy = (int)std::max(1.0, std::min(4096.0, std::floor(Ly / (cf * p->h))));
        c->cw = Lx / c->ncx;
        c->chh = Ly / c->ncy;
        // exact constants
        std::vector<double> kc = siac::kernel_cell_table(k);
        std::vector<double> R = p->basis == SIAC_BASIS_MONOMIAL_REF ? siac::monomial_to_centred(k)
                                                                    : siac::dubiner_to_centred(k);
        c->cinfo.host_ms = ms_since(t_start);
        cudaStream_t cs = c->stream;
        cudaEvent_t ev[5] = {};
        for (auto &e : ev) CK(cudaEventCreate(&e));
        struct EvGuard { cudaEvent_t *e; ~EvGuard() { for (int i = 0; i < 5; ++i) if (e[i]) cudaEventDestroy(e[i]); } } evg{ev};
        CK(cudaMalloc(&c->d_kc, sizeof(double) * kc.size()));
        CK(cudaMemcpy(c->d_kc, kc.data(), sizeof(double) * kc.size(), cudaMemcpyHostToDevice));
        CK(cudaMalloc(&c->d_cnt, 8 * sizeof(unsigned long long)));
        CK(cudaMalloc(&c->d_tile_counter, sizeof(int)));
        c->num_sms = nsm;
        CK(cudaMemsetAsync(c->d_cnt, 0, 8 * sizeof(unsigned long long), c->stream));
        const int64_t ncell = (int64_t)c->ncx * c->ncy;
        CK(cudaMalloc(&c->d_cell_start, sizeof(int) * (ncell + 1)));
        if (nt == 0) {
            CK(cudaMemsetAsync(c->d_cell_start, 0, sizeof(int) * (ncell + 1), c->stream));
            CK(cudaStreamSynchronize(c->stream));
            c->cinfo.device_bytes = (int64_t)(sizeof(int) * (ncell + 1) + sizeof(double) * kc.size() + 64 + 4);
            c->cinfo.total_ms = ms_since(t_start);
            return;
        }
        const int rs = (16 + nb + 1) & ~1;
        double *dV = nullptr, *dC = nullptr, *dR = nullptr, *rec_u = nullptr;
        int *dT = nullptr;
        double4 *bb_u = nullptr;
        uint32_t *keys[2] = {nullptr, nullptr};
        int *idx[2] = {nullptr, nullptr};
        void *tmp = nullptr;
        auto cleanup = [&]() {
            void *ps[] = {dV, dC, dR, rec_u, dT, bb_u, keys[0], keys[1], idx[0], idx[1], tmp};
            for (void *q : ps)
                if (q) cudaFree(q);
        };
        try {
            CK(cudaMalloc(&dV, sizeof(double) * 2 * std::max<int64_t>(nv, 1)));
            CK(cudaMalloc(&dT, sizeof(int) * 3 * nt));
            CK(cudaMalloc(&dC, sizeof(double) * nb * nt));
            CK(cudaMalloc(&dR, sizeof(double) * nb * nb));
            CK(cudaMalloc(&rec_u, sizeof(double) * rs * nt));
            CK(cudaMalloc(&bb_u, sizeof(double4) * nt));
            for (int b = 0; b < 2; ++b) {
                CK(cudaMalloc(&keys[b], sizeof(uint32_t) * nt));
                CK(cudaMalloc(&idx[b], sizeof(int) * nt));
            }
            CK(cudaMalloc(&c->d_rec, sizeof(double) * rs * nt));
            CK(cudaMalloc(&c->d_bbox, sizeof(double4) * nt));
            cub::DoubleBuffer<uint32_t> kb(keys[0], keys[1]);
            cub::DoubleBuffer<int> vb(idx[0], idx[1]);
            size_t bytes = 0;
            CK(cub::DeviceRadixSort::SortPairs(nullptr, bytes, kb, vb, (int)nt));
            CK(cudaMalloc(&tmp, bytes));
            CK(cudaEventRecord(ev[0], cs));
            CK(cudaMemcpyAsync(dV, V, sizeof(double) * 2 * nv, cudaMemcpyHostToDevice, cs));
            CK(cudaMemcpyAsync(dT, T, sizeof(int) * 3 * nt, cudaMemcpyHostToDevice, cs));
            CK(cudaMemcpyAsync(dC, C, sizeof(double) * nb * nt, cudaMemcpyHostToDevice, cs));
            CK(cudaMemcpyAsync(dR, R.data(), sizeof(double) * nb * nb, cudaMemcpyHostToDevice, cs));
            CK(cudaEventRecord(ev[1], cs));
            PrepArgs pa{dV, dT, dC, dR, nt, nb, rs, p->h, p->domain[0], p->domain[1], c->cw, c->chh,
                        c->ncx, c->ncy, rec_u, bb_u, keys[0], idx[0]};
            k_prep<<<nblk(nt, 256), 256, 0, cs>>>(pa);
            CK(cudaGetLastError());
            CK(cub::DeviceRadixSort::SortPairs(tmp, bytes, kb, vb, (int)nt, 0, sizeof(uint32_t) * 8, cs));
            k_gather<<<nblk(nt, 256), 256, 0, cs>>>(rec_u, bb_u, vb.Current(), nt, rs, c->d_rec, c->d_bbox);
            CK(cudaGetLastError());
            k_cell_start<<<nblk(ncell + 1, 256), 256, 0, cs>>>(kb.Current(), nt, ncell, c->d_cell_start);
            CK(cudaGetLastError());
            CK(cudaEventRecord(ev[2], cs));
            // schedule JUMP: per-triangle moments and corner polynomials (siac_jump.cuh)
            int jrs = 0;
            switch (k) {
                case 1: jrs = siacjump::JRec<1>::RS; break;
                case 2: jrs = siacjump::JRec<2>::RS; break;
                case 3: jrs = siacjump::JRec<3>::RS; break;
                default: jrs = siacjump::JRec<4>::RS; break;
            }
            CK(cudaMalloc(&c->d_jrec, sizeof(double) * jrs * nt));
            switch (k) {
                case 1: CK(siac_prep_jump_k1(c->d_rec, nt, p->h, c->d_jrec, cs)); break;
                case 2: CK(siac_prep_jump_k2(c->d_rec, nt, p->h, c->d_jrec, cs)); break;
                case 3: CK(siac_prep_jump_k3(c->d_rec, nt, p->h, c->d_jrec, cs)); break;
                default: CK(siac_prep_jump_k4(c->d_rec, nt, p->h, c->d_jrec, cs)); break;
            }
            CK(cudaEventRecord(ev[3], cs));
            // closed-form cross terms (interval polynomials of the reference corners)
            int xrs = 0;
            switch (k) {
                case 1: xrs = siac_xrec_doubles_k1(); break;
                case 2: xrs = siac_xrec_doubles_k2(); break;
                case 3: xrs = siac_xrec_doubles_k3(); break;
                default: xrs = siac_xrec_doubles_k4(); break;
            }
            CK(cudaMalloc(&c->d_xrec, sizeof(double) * xrs * nt));
            switch (k) {
                case 1: CK(siac_prep_cross_k1(c->d_jrec, nt, c->d_xrec, cs)); break;
                case 2: CK(siac_prep_cross_k2(c->d_jrec, nt, c->d_xrec, cs)); break;
                case 3: CK(siac_prep_cross_k3(c->d_jrec, nt, c->d_xrec, cs)); break;
                default: CK(siac_prep_cross_k4(c->d_jrec, nt, c->d_xrec, cs)); break;
            }
            CK(cudaGetLastError());
            CK(cudaEventRecord(ev[4], cs));
            CK(cudaStreamSynchronize(cs));
            float t01 = 0, t12 = 0, t23 = 0, t34 = 0;
            CK(cudaEventElapsedTime(&t01, ev[0], ev[1]));
            CK(cudaEventElapsedTime(&t12, ev[1], ev[2]));
            CK(cudaEventElapsedTime(&t23, ev[2], ev[3]));
            CK(cudaEventElapsedTime(&t34, ev[3], ev[4]));
            c->cinfo.h2d_ms = t01;
            c->cinfo.index_ms = t12;
            c->cinfo.jump_ms = t23;
            c->cinfo.cross_ms = t34;
            const int64_t per_tri = (int64_t)sizeof(double) * (rs + jrs + xrs) + (int64_t)sizeof(double4);
            c->cinfo.bytes_per_triangle = per_tri;
            c->cinfo.device_bytes = per_tri * nt + (int64_t)sizeof(int) * (ncell + 1) +
                                    (int64_t)(sizeof(double) * kc.size()) + 64 + 4;
        } catch (...) {
            cleanup();
            throw;
        }
        cleanup();
        c->cinfo.total_ms = ms_since(t_start);
    });
    if (st != SIAC_OK) {
        free_ctx(c);
        return st;
    }
    *out = c;
    return SIAC_OK;
}

siac_status siac_eval_async(siac_ctx *ctx, const double *d_pts, int64_t np, double *d_out, void *stream) {
    if (!ctx) { g_err = "NULL context"; return SIAC_EINVAL; }
    return run_guarded(&ctx->err, [&]() {
        need(np >= 0, "negative n_points");
        if (np == 0) return;
        need(d_pts && d_out, "NULL device pointers");
        cudaStream_t st = (cudaStream_t)stream;
        if (!ctx->graphs || ctx->counting || ctx->timing || st == nullptr) {
            eval_device(ctx, d_pts, np, d_out, st);
            return;
        }
        // replay a captured graph of the whole evaluation (keys, sort, kernels) when the same
        // buffers come back: launch-bound small evaluations pay one graph launch
        CK(cudaSetDevice(ctx->device));
        ensure_scratch(ctx, np);
        if (ctx->schedule == 6 && !ctx->d_pcell)
            CK(cudaMalloc(&ctx->d_pcell, sizeof(int) * ((int64_t)ctx->ncx * ctx->ncy + 1)));
        for (auto &g : ctx->gcache)
            if (g.pts == d_pts && g.np == np && g.out == d_out && g.schedule == ctx->schedule) {
                CK(cudaGraphLaunch(g.exec, st));
                return;
            }
        // The very first evaluation of a context runs directly (it sets the kernels' shared-memory
        // attributes and loads the modules, which must not happen inside a capture) and is this
        // call's result; the graph captured right after is only instantiated, not launched.
        const bool first = ctx->gcache.empty();
        if (first) eval_device(ctx, d_pts, np, d_out, st);
        cudaGraph_t graph = nullptr;
        CK(cudaStreamBeginCapture(st, cudaStreamCaptureModeRelaxed));
        try {
            eval_device(ctx, d_pts, np, d_out, st);
        } catch (...) {
            cudaStreamEndCapture(st, &graph);
            if (graph) cudaGraphDestroy(graph);
            throw;
        }
        CK(cudaStreamEndCapture(st, &graph));
        cudaGraphExec_t exec = nullptr;
        const cudaError_t ie = cudaGraphInstantiate(&exec, graph, 0);
        cudaGraphDestroy(graph);
        CK(ie);
        if (ctx->gcache.size() >= 8) {
            cudaGraphExecDestroy(ctx->gcache.front().exec);
            ctx->gcache.erase(ctx->gcache.begin());
        }
        ctx->gcache.push_back({d_pts, np, d_out, ctx->schedule, exec});
        if (!first) CK(cudaGraphLaunch(exec, st));
    });
}

siac_status siac_set_graphs(siac_ctx *ctx, int32_t enable) {
    if (!ctx) { g_err = "NULL context"; return SIAC_EINVAL; }
    ctx->graphs = enable != 0;
    if (!ctx->graphs) {
        cudaSetDevice(ctx->device);
        clear_graphs(ctx);
    }
    return SIAC_OK;
}

siac_status siac_eval(siac_ctx *ctx, const double *pts, int64_t np, double *out) {
    if (!ctx) { g_err = "NULL context"; return SIAC_EINVAL; }
    return run_guarded(&ctx->err, [&]() {
        need(np >= 0, "negative n_points");
        if (np == 0) return;
        need(pts && out, "NULL host pointers");
        CK(cudaSetDevice(ctx->device));
        if (np > ctx->cap_host) {
            if (ctx->d_hpts) cudaFree(ctx->d_hpts);
            if (ctx->d_hout) cudaFree(ctx->d_hout);
            ctx->d_hpts = ctx->d_hout = nullptr;
            ctx->cap_host = 0;
            CK(cudaMalloc(&ctx->d_hpts, sizeof(double) * 2 * np));
            CK(cudaMalloc(&ctx->d_hout, sizeof(double) * np));
            ctx->cap_host = np;
        }
        cudaStream_t st = ctx->stream;
        CK(cudaMemcpyAsync(ctx->d_hpts, pts, sizeof(double) * 2 * np, cudaMemcpyHostToDevice, st));
        eval_device(ctx, ctx->d_hpts, np, ctx->d_hout, st);
        CK(cudaMemcpyAsync(out, ctx->d_hout, sizeof(double) * np, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
    });
}

siac_status siac_set_counting(siac_ctx *ctx, int32_t enable) {
    if (!ctx) { g_err = "NULL context"; return SIAC_EINVAL; }
    ctx->counting = enable != 0;
    return SIAC_OK;
}

siac_status siac_get_create_info(const siac_ctx *ctx, siac_create_info *out) {
    if (!ctx || !out) { g_err = "NULL argument"; return SIAC_EINVAL; }
    *out = ctx->cinfo;
    return SIAC_OK;
}

siac_status siac_stats(const siac_ctx *cctx, siac_counters *out) {
    if (!cctx || !out) { g_err = "NULL argument"; return SIAC_EINVAL; }
    siac_ctx *ctx = const_cast<siac_ctx *>(cctx);     // only the error message is written
    return run_guarded(&ctx->err, [&]() {
        CK(cudaSetDevice(ctx->device));
        unsigned long long h[8];
        CK(cudaDeviceSynchronize());
        CK(cudaMemcpy(h, ctx->d_cnt, sizeof(h), cudaMemcpyDeviceToHost));
        out->n_points = ctx->last_np;
        out->candidates = (int64_t)h[0];
        out->pairs = (int64_t)h[1];
        out->pieces = (int64_t)h[2];
        out->subtris = (int64_t)h[3];
        out->corner_terms = (int64_t)h[4];
        out->cross_terms = (int64_t)h[5];
        out->cross_subtris = (int64_t)h[6];
        out->cross_polys = (int64_t)h[7];
    });
}

siac_status siac_set_schedule(siac_ctx *ctx, int32_t schedule) {
    if (!ctx) { g_err = "NULL context"; return SIAC_EINVAL; }
    if (schedule < 0 || schedule > 6) { ctx->err = "unknown schedule"; return SIAC_EINVAL; }
    ctx->schedule = schedule;
    return SIAC_OK;
}

siac_status siac_set_timing(siac_ctx *ctx, int32_t enable) {
    if (!ctx) { g_err = "NULL context"; return SIAC_EINVAL; }
    ctx->timing = enable != 0;
    return SIAC_OK;
}

siac_status siac_timing(siac_ctx *ctx, double *ms_total, int64_t *n) {
    if (!ctx || !ms_total || !n) { g_err = "NULL argument"; return SIAC_EINVAL; }
    return run_guarded(&ctx->err, [&]() {
        CK(cudaSetDevice(ctx->device));
        double tot = 0;
        for (size_t i = 0; i < ctx->ev_used; ++i) {
            float ms = 0;
            CK(cudaEventSynchronize(ctx->ev[i].second));
            CK(cudaEventElapsedTime(&ms, ctx->ev[i].first, ctx->ev[i].second));
            tot += ms;
        }
        *ms_total = tot;
        *n = (int64_t)ctx->ev_used;
        ctx->ev_used = 0;
    });
}

siac_status siac_probe_fp64(int32_t device, double *tflops) {
    if (!tflops) { g_err = "NULL argument"; return SIAC_EINVAL; }
    return run_guarded(&g_err, [&]() {
        CK(cudaSetDevice(device));
        cudaDeviceProp prop;
        CK(cudaGetDeviceProperties(&prop, device));
        const int blocks = prop.multiProcessorCount * 4, threads = 512, iters = 1 << 14;
        double *d = nullptr;
        CK(cudaMalloc(&d, sizeof(double) * blocks));
        cudaEvent_t e0, e1;
        CK(cudaEventCreate(&e0));
        CK(cudaEventCreate(&e1));
        float best = 1e30f;
        for (int rep = 0; rep < 6; ++rep) {
            CK(cudaEventRecord(e0));
            k_dfma_probe<<<blocks, threads>>>(d, iters, 0.9999999, 1e-7);
            CK(cudaEventRecord(e1));
            CK(cudaEventSynchronize(e1));
            float ms = 0;
            CK(cudaEventElapsedTime(&ms, e0, e1));
            if (rep > 0) best = std::min(best, ms);
        }
        CK(cudaGetLastError());
        cudaEventDestroy(e0);
        cudaEventDestroy(e1);
        cudaFree(d);
        const double flops = 2.0 * 8.0 * iters * (double)blocks * threads;
        *tflops = flops / (best * 1e-3) / 1e12;
    });
}

siac_status siac_info(const siac_ctx *ctx, int64_t *n_triangles, int32_t *gx, int32_t *gy, double *cw, double *ch) {
    if (!ctx) { g_err = "NULL context"; return SIAC_EINVAL; }
    if (n_triangles) *n_triangles = ctx->nt;
    if (gx) *gx = ctx->ncx;
    if (gy) *gy = ctx->ncy;
    if (cw) *cw = ctx->cw;
    if (ch) *ch = ctx->chh;
    return SIAC_OK;
}

siac_status siac_host_tables(int32_t k, double *cell_table, double *basis_matrix) {
    return run_guarded(&g_err, [&]() {
        need(k >= 1 && k <= 4, "k must be in 1..4");
        if (cell_table) {
            std::vector<double> t = siac::kernel_cell_table(k);
            std::copy(t.begin(), t.end(), cell_table);
        }
        if (basis_matrix) {
            std::vector<double> R = siac::dubiner_to_centred(k);
            std::copy(R.begin(), R.end(), basis_matrix);
        }
    });
}

siac_status siac_debug_records(siac_ctx *ctx, int32_t which, int64_t n, double *out, int32_t *rd) {
    if (!ctx) { g_err = "NULL context"; return SIAC_EINVAL; }
    return run_guarded(&ctx->err, [&]() {
        need(which >= 0 && which <= 2, "which must be 0, 1 or 2");
        const int nb = (ctx->k + 1) * (ctx->k + 2) / 2;
        int rs = (16 + nb + 1) & ~1;
        const double *src = ctx->d_rec;
        if (which == 1) {
            static const int jrs[4] = {siacjump::JRec<1>::RS, siacjump::JRec<2>::RS, siacjump::JRec<3>::RS,
                                       siacjump::JRec<4>::RS};
            rs = jrs[ctx->k - 1];
            src = ctx->d_jrec;
        } else if (which == 2) {
            const int xrs[4] = {siac_xrec_doubles_k1(), siac_xrec_doubles_k2(), siac_xrec_doubles_k3(),
                                siac_xrec_doubles_k4()};
            rs = xrs[ctx->k - 1];
            src = ctx->d_xrec;
        }
        if (rd) *rd = rs;
        need(n >= 0 && n <= ctx->nt, "n out of range");
        if (n > 0 && out) {
            CK(cudaSetDevice(ctx->device));
            CK(cudaMemcpy(out, src, sizeof(double) * rs * n, cudaMemcpyDeviceToHost));
        }
    });
}

void siac_destroy(siac_ctx *ctx) { free_ctx(ctx); }

}  // extern "C"
