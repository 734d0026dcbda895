// siac_internal.h -- interface between the host TU (siac.cu) and the per-degree kernel TUs
// (siac_eval_k.cu compiled once per k with -DSIAC_K=k, in parallel).
#pragma once

#include <cuda_runtime.h>
#include <cstdint>
#include <string>

// message returned by siac_last_error(NULL) on this thread (defined in siac.cu)
void siac_set_thread_error(const std::string &msg);

struct EvalArgs {            // arguments of every evaluation schedule
    const double *pts;        // input order, np x 2
    const int *perm;          // sorted position -> input index
    int64_t np;
    double *out;
    const double *rec;
    const double *jrec;
    const double *xrec;       // closed-form cross terms (schedule JUMP-X)
    const double4 *bbox;
    const int *cell_start;
    const double *kc;
    double x0, y0, Lx, Ly, h, inv_h, hw;   // hw = W/2 (physical)
    double cw, chh, ex, ey;
    int ncx, ncy, periodic;
    int xpoly;                // jump schedule: 1 = closed-form cross terms, 0 = clipped + quadrature
    const int *pcell_start;   // schedule ELEM: point CSR by row-major binning cell
    int64_t nt;               // number of triangles
    unsigned long long *cnt;  // [candidates, pairs, pieces, subtris, corner, cross, cross_subtris, cross_polys]
    // one-sided kernels (SIAC_BOUNDARY_ONESIDED; reading R4): axes (bit0 x, bit1 y)
    // whose stencil shifts near the boundary, the domain's upper corner, and the host tables of
    // siac::onesided_tables (B-spline pieces, inverse moment matrix) copied into the launch
    int os_axes;
    double x1d, y1d;
    const double *os_pieces, *os_ainv;
};

// per (k, schedule part): p0 = jump, p1 = point, p2 = tile, p3 = warp-specialized
#define SIAC_DECL_KP(k, p)                                                                      \
    cudaError_t siac_launch_eval_k##k##_p##p(const EvalArgs &a, bool count, int *tile_counter, \
                                             int num_sms, cudaStream_t st);
#define SIAC_DECL_K(k)                                                                          \
    SIAC_DECL_KP(k, 0) SIAC_DECL_KP(k, 1) SIAC_DECL_KP(k, 2) SIAC_DECL_KP(k, 3)                 \
    cudaError_t siac_prep_jump_k##k(const double *rec, int64_t nt, double h, double *jrec, cudaStream_t st); \
    cudaError_t siac_prep_cross_k##k(const double *jrec, int64_t nt, double *xrec, cudaStream_t st);         \
    cudaError_t siac_launch_elem_k##k(const EvalArgs &a, bool count, int *, int, cudaStream_t st); \
    int siac_xrec_doubles_k##k();
SIAC_DECL_K(1)
SIAC_DECL_K(2)
SIAC_DECL_K(3)
SIAC_DECL_K(4)
#undef SIAC_DECL_K
#undef SIAC_DECL_KP

typedef cudaError_t (*siac_launch_fn)(const EvalArgs &, bool, int *, int, cudaStream_t);
