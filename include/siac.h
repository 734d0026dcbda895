/*
 * siac.h -- C ABI of the B200 SIAC post-processor (libsiac_b200.so).
 *
 * What it computes (King & Kirby, SC'13; /root/reference/PAPER.md):
 *   For every evaluation point x, the SIAC-filtered value of a 2D dG solution u_h,
 *       u*(x) = (1/h^2) \int\int K((y1-x1)/h) K((y2-x2)/h) u_h(y) dy          (Eq. (1))
 *   K(t) = sum_{g=0}^{2k} c_g psi_{k+1}(t - x_g), x_g = -k + g, psi_{k+1} the centred
 *   B-spline of order k+1 (L196-208); Supp K = (3k+1) (L250-254).  Each triangle the
 *   stencil touches is split along the kernel breaklines into pieces on which the integrand
 *   is polynomial, the pieces are triangulated and integrated exactly by Gauss quadrature
 *   (Eq. (2); Sutherland-Hodgman clipping, Alg. 1).  Periodic axes
 *   wrap the stencil around the domain (L280-282).
 *
 * Conventions
 *   - All functions are extern "C", never throw, and return siac_status (0 = OK).
 *   - Precision: IEEE FP64 throughout; results differ from the exact integral only by
 *     rounding (any summation order).
 *   - Ownership: siac_create deep-copies every input (the caller may free them on return);
 *     the context owns all device memory until siac_destroy.  siac_eval / siac_eval_async
 *     write n_points doubles to caller-owned memory, in input order.
 *   - Errors: on failure a message is available from siac_last_error(ctx) (ctx may be NULL
 *     for errors of siac_create; the message is then thread-local).  No partial results are
 *     promised on failure.  CUDA errors are reported as SIAC_ECUDA with cudaGetErrorString.
 *   - Thread safety: one host thread at a time per context, and at most one evaluation in
 *     flight per context (scratch buffers are per context).  Different contexts on
 *     different devices may be used concurrently (one per rank in multi-GPU runs).
 *   - No CPU fallback: every evaluation step runs in CUDA kernels on the context's device.
 */
#ifndef SIAC_H
#define SIAC_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct siac_ctx siac_ctx;

typedef enum {
    SIAC_OK = 0,
    SIAC_EINVAL = -1,     /* invalid argument (message says which) */
    SIAC_ENOMEM = -2,     /* host or device allocation failed */
    SIAC_ECUDA = -3,      /* a CUDA runtime call or kernel failed */
    SIAC_EDEVICE = -4,    /* no usable sm_100 device at params->device */
    SIAC_EINTERNAL = -5   /* internal invariant violated (bug) */
} siac_status;

/* Periodicity bits (all the paper's tests are periodic, L715). */
#define SIAC_PERIODIC_X 1
#define SIAC_PERIODIC_Y 2

/* Modal basis of the coefficients siac_create reads ("an array of the
 * polynomial modes"; the basis is not named). */
typedef enum {
    SIAC_BASIS_DUBINER_ORTHONORMAL = 0,  /* default; see siac_create */
    SIAC_BASIS_MONOMIAL_REF = 1          /* u = sum c_i r^a s^b on the unit reference triangle
                                            (point = v0 + r (v1 - v0) + s (v2 - v0)); mode i
                                            ordered like the Dubiner modes: by n = a + b, then b */
} siac_basis;

/* What the stencil does on a NON-periodic axis near the domain boundary (PAPER.md L280-283:
 * "the stencil either wraps around the domain for periodic solutions, or an asymmetric
 * (one-sided) stencil is used [21]").  Periodic axes always wrap. */
typedef enum {
    SIAC_BOUNDARY_ZERO = 0,      /* symmetric kernel everywhere, u_h = 0 outside the mesh */
    SIAC_BOUNDARY_ONESIDED = 1   /* position-dependent one-sided kernel (ref [21], Ryan & Shu
                                    2003; reading R4): the 2k+1 B-spline nodes are
                                    shifted by lambda(x) so the support stays inside
                                    [x0, x1] x [y0, y1], and the coefficients c_g(lambda)
                                    re-solve the same moment conditions (degree-2k
                                    reproduction); needs W = (3k+1)h <= the extent */
} siac_boundary;

typedef struct {
    int32_t k;          /* dG degree = B-spline degree; 1..4 (paper tested 1..3, L716-718) */
    double  h;          /* kernel scaling > 0; the paper uses the longest edge s (L430, L440) */
    int32_t periodic;   /* SIAC_PERIODIC_X | SIAC_PERIODIC_Y; non-periodic axes: see boundary */
    double  domain[4];  /* x0, y0, x1, y1; the paper uses [0,1]^2 (L428) */
    int32_t device;     /* CUDA device ordinal */
    double  cell_factor;/* binning cell size / h; 0 -> default 0.5 (paper c_e = s/2, L505-508) */
    int32_t basis;      /* siac_basis of `coeffs` (0 = orthonormal Dubiner) */
    int32_t boundary;   /* siac_boundary for the non-periodic axes (0 = zero extension) */
} siac_params;

typedef struct {        /* geometry counts of the last evaluation (see siac_set_counting) */
    int64_t n_points;
    int64_t candidates; /* (point, triangle image) bounding-box tests */
    int64_t pairs;      /* (point, triangle image) pairs whose boxes overlap */
    int64_t pieces;     /* non-empty clipped polygons (triangle image ∩ kernel cell) integrated
                           piece by piece (schedules POINT/TILE/WS; JUMP: general-path pairs only) */
    int64_t subtris;    /* fan sub-triangles of those pieces = sum over pieces of (vertices - 2) */
    int64_t corner_terms;  /* JUMP: closed-form corner terms (one per pair and axis with a knot) */
    int64_t cross_terms;   /* JUMP: pairs with a knot on both axes (clipped corner-corner terms) */
    int64_t cross_subtris; /* JUMP: fan sub-triangles integrated for the cross terms */
    int64_t cross_polys;   /* JUMPX: cross terms evaluated by an interval polynomial (the rest are
                              empty or whole-corner terms) */
} siac_counters;

/*
 * siac_create -- ingest a mesh and its dG modes onto the device and build the spatial index.
 *   vertices_xy  host, n_vertices x 2 doubles, row-major (x, y).  On periodic axes every
 *                vertex must lie in [x0, x1] (tolerance 1e-9 of the extent).
 *   triangles    host, n_triangles x 3 int32, 0-based vertex indices; any orientation.
 *   coeffs       host, n_triangles x (k+1)(k+2)/2 doubles: modal coefficients in
 *                params->basis; default: the orthonormal
 *                Dubiner basis on the reference triangle {xi, eta >= -1, xi + eta <= 0},
 *                triangle vertices 0, 1, 2 mapped to (-1,-1), (1,-1), (-1,1);
 *                phi_pq = sqrt((2p+1)(p+q+1)/2) P_p(a) ((1-eta)/2)^p P_q^(2p+1,0)(eta),
 *                a = 2(1+xi)/(1-eta) - 1; modes ordered by p+q, then q (PAPER.md L209-212,
 *                L716-718: "an array of the polynomial modes"; basis per SURVEY Q8).
 *   params       see siac_params.
 *   *out         receives the context (NULL on failure).
 * Errors: SIAC_EINVAL for k outside 1..4, h <= 0 or non-finite, (3k+1)h larger than a
 *   periodic extent (or, with SIAC_BOUNDARY_ONESIDED, than a non-periodic extent), an unknown
 *   basis or boundary, an empty or inverted domain, out-of-range indices, zero-area triangles,
 *   non-finite coordinates or coefficients, vertices outside a periodic axis; SIAC_EDEVICE,
 *   SIAC_ENOMEM, SIAC_ECUDA.  n_triangles == 0 is allowed (every value is then 0).
 */
siac_status siac_create(siac_ctx **out,
                        const double *vertices_xy, int64_t n_vertices,
                        const int32_t *triangles, int64_t n_triangles,
                        const double *coeffs, const siac_params *params);

/*
 * siac_eval -- blocking evaluation with HOST buffers.
 *   points_xy   host, n_points x 2 doubles (x, y); any location (periodic axes wrap).
 *   values_out  host, n_points doubles, written in input order.
 * Includes the host->device copy of the points and the device->host copy of the values, all
 * stream-ordered on the context's own stream (pinned host buffers copy at full PCIe rate;
 * the copies cannot overlap the kernel: the point sort needs every point and the values are
 * written in input order).  n_points == 0 is a no-op returning SIAC_OK.
 */
siac_status siac_eval(siac_ctx *ctx, const double *points_xy, int64_t n_points, double *values_out);

/*
 * siac_eval_async -- stream-ordered evaluation with DEVICE buffers on the context's device.
 *   d_points_xy   device, n_points x 2 doubles; must stay valid until the stream passes.
 *   d_values_out  device, n_points doubles (input order).
 *   cuda_stream   a cudaStream_t (NULL = legacy default stream).
 * Returns after enqueueing (the first call for a given size may allocate scratch memory,
 * which synchronises the device).
 */
siac_status siac_eval_async(siac_ctx *ctx, const double *d_points_xy, int64_t n_points,
                            double *d_values_out, void *cuda_stream);

/* CUDA graphs for repeated evaluations (default off).  When enabled, siac_eval_async on a
 * non-NULL stream captures the whole evaluation (point keys, sort, evaluation kernel) into a
 * CUDA graph the first time it sees a (d_points_xy, n_points, d_values_out, schedule)
 * combination and replays it afterwards (up to 8 cached graphs per context, least recently
 * created evicted first): launch-bound small evaluations cost one graph launch.  The caller
 * must not free or reallocate those buffers while graphs are enabled; disabling (enable = 0)
 * drops every cached graph.  Counting, timing and the NULL stream bypass the graphs.  Results
 * are bitwise those of the direct path. */
siac_status siac_set_graphs(siac_ctx *ctx, int32_t enable);

/* Evaluation schedule (same result up to rounding):
 *   SIAC_SCHEDULE_DEFAULT (0) the fastest measured schedule (currently SIAC_SCHEDULE_JUMPX);
 *   SIAC_SCHEDULE_POINT   (1) one thread per point, clip and integrate inline (the paper's
 *                         per-point evaluation, Alg. 2, one thread per point);
 *   SIAC_SCHEDULE_TILE    (2) one warp per tile of 32 Morton-ordered points: ballot-compacted
 *                         candidate tests, register-only Sutherland-Hodgman splits, sub-triangles
 *                         staged in shared memory and integrated 32 at a time by the full warp;
 *   SIAC_SCHEDULE_WS      (3) persistent warp-specialized variant of TILE: producer warps clip,
 *                         paired consumer warps integrate double-buffered batches (mbarriers);
 *   SIAC_SCHEDULE_JUMP    (4) the same exact decomposition (Eq. (2)) reorganised with the spline
 *                         jumps of K: K = base cell polynomial + alpha (t - X)^k on the triangle's
 *                         one-vertex side of a knot X, so each pair is the whole-triangle moment
 *                         term + closed-form corner polynomials (precomputed per triangle at
 *                         create time) + one clipped corner-corner piece integrated by quadrature
 *                         when both axes have a knot (csrc/siac_jump.cuh).  Pairs with two knots
 *                         on an axis (h < triangle size) use the clip-and-integrate path;
 *   SIAC_SCHEDULE_JUMPX   (5) JUMP with the corner-corner pieces in closed form too: the x corner
 *                         clipped by the y knot line is the homothetic image of a fixed reference
 *                         corner clipped by a horizontal line, whose integral is a polynomial in
 *                         (homothety ratio, line height) on each of two height intervals, built
 *                         per triangle at create time (Chebyshev interpolation of exact samples);
 *   SIAC_SCHEDULE_ELEM    (6) the paper's per-element method (Alg. 3) on the JUMPX
 *                         decomposition: one warp per triangle walks the point grid within its
 *                         Eq. (3) bounds (L434-498), lane = candidate point, and scatter-adds each
 *                         pair's contribution (atomics: the summation order, hence the last bits,
 *                         varies between runs; every other schedule is bitwise deterministic). */
#define SIAC_SCHEDULE_DEFAULT 0
#define SIAC_SCHEDULE_POINT 1
#define SIAC_SCHEDULE_TILE 2
#define SIAC_SCHEDULE_WS 3
#define SIAC_SCHEDULE_JUMP 4
#define SIAC_SCHEDULE_JUMPX 5
#define SIAC_SCHEDULE_ELEM 6
siac_status siac_set_schedule(siac_ctx *ctx, int32_t schedule);

/* Enable (1) / disable (0) geometry counting in later evaluations (adds atomics; off by default). */
siac_status siac_set_counting(siac_ctx *ctx, int32_t enable);

/* ---- Steps either side of the path ("grid points ... used at the end of
 * the simulation for such things as error calculations").  They need no
 * context; device pointers are stream-ordered on `cuda_stream` (NULL = legacy default stream)
 * and must stay valid until the stream passes the call.  Errors: SIAC_EINVAL for bad sizes or
 * NULL pointers, SIAC_ECUDA for launch failures; message via siac_last_error(NULL). */

/* Host: the collapsed Gauss-Legendre rule with n_quad^2 nodes (n_quad in 1..64) used by
 * siac_project_async, exact to total degree 2 n_quad - 2.
 *   rs_out  host, n_quad^2 x 2 doubles: node (r, s) on the unit triangle (point = v0 +
 *           r (v1 - v0) + s (v2 - v0)); node q = i * n_quad + j.
 *   w_out   host, n_quad^2 doubles: weights on the reference triangle (area 2; sum = 2). */
siac_status siac_projection_rule(int32_t n_quad, double *rs_out, double *w_out);

/* Device: points_out[(t * n_nodes + q)] = v0 + r_q (v1 - v0) + s_q (v2 - v0) of triangle t.
 *   d_vertices_xy  n_vertices x 2;  d_triangles  n_triangles x 3 (0-based, unchecked here);
 *   d_rs           n_nodes x 2 reference nodes;  d_points_out  n_triangles * n_nodes x 2. */
siac_status siac_map_points_async(const double *d_vertices_xy, const int32_t *d_triangles, int64_t n_triangles,
                                  const double *d_rs, int32_t n_nodes, double *d_points_out, void *cuda_stream);

/* Device: L2 projection onto P_k (orthonormal Dubiner, SIAC_BASIS_DUBINER_ORTHONORMAL, the
 * layout siac_create reads) of a field sampled at the siac_projection_rule nodes:
 *   d_f             n_triangles x n_quad^2 values, element-major (node order of the rule);
 *   d_coeffs_out    n_triangles x (k+1)(k+2)/2 modes.
 * c_i = sum_q w_q phi_i(node_q) f_q (the element mass matrix on the reference triangle is the
 * identity for this basis).  Exact for f in P_{2 n_quad - 2 - k}; k in 1..4, n_quad in k+1..32. */
siac_status siac_project_async(int32_t k, int32_t n_quad, const double *d_f, int64_t n_triangles,
                               double *d_coeffs_out, void *cuda_stream);

/* Device: error norms of e = u - ref over n values, deterministic (fixed reduction order):
 *   d_weights  n weights (e.g. quadrature weight x element area) or NULL (all 1);
 *   d_out      3 doubles: sqrt(sum w e^2), max |e|, sum w. */
siac_status siac_error_norms_async(const double *d_u, const double *d_ref, const double *d_weights, int64_t n,
                                   double *d_out, void *cuda_stream);

/* Counters of the last evaluation run with counting enabled (synchronises the device). */
siac_status siac_stats(const siac_ctx *ctx, siac_counters *out);

/* Cost and footprint of siac_create (create is excluded from points/s and
 * "reported separately"; the element data are built once and reused by every evaluation,
 * PAPER.md L586-594).  Device times are CUDA-event times on the context's stream. */
typedef struct {
    double  total_ms;        /* wall clock of siac_create (host + device, until synchronised) */
    double  host_ms;         /* host validation pass + exact constants */
    double  h2d_ms;          /* vertices, triangles and modes host -> device */
    double  index_ms;        /* k_prep + CUB sort by anchor cell + k_gather + k_cell_start */
    double  jump_ms;         /* k_prep_jump: per-triangle moments and corner polynomials */
    double  cross_ms;        /* k_prep_cross: interval polynomials of the clipped corners */
    int64_t device_bytes;    /* device memory the context keeps after siac_create */
    int64_t bytes_per_triangle;  /* resident per-triangle data (records + box) */
} siac_create_info;
siac_status siac_get_create_info(const siac_ctx *ctx, siac_create_info *out);

/* Enable (1) / disable (0) CUDA-event timing of the main evaluation kernel (k_eval) on the
 * evaluation stream.  While enabled, every evaluation records one event pair around it. */
siac_status siac_set_timing(siac_ctx *ctx, int32_t enable);

/* Sum of the main-kernel durations (ms) and number of timed launches since the last call;
 * synchronises on the recorded events and resets the accumulator. */
siac_status siac_timing(siac_ctx *ctx, double *kernel_ms_total, int64_t *n_launches);

/* FP64 FMA throughput probe on `device`: a DFMA-chain kernel filling every SM; writes the
 * achieved TFLOP/s (2 flops per DFMA) to *tflops.  Used as the measured roofline peak. */
siac_status siac_probe_fp64(int32_t device, double *tflops);

/* Mesh-side info: n_triangles, binning grid size, cells, max bbox extents. */
siac_status siac_info(const siac_ctx *ctx, int64_t *n_triangles, int32_t *grid_nx, int32_t *grid_ny,
                      double *cell_w, double *cell_h);

/* Host-side exact constants (diagnostics and CPU tests; no device needed):
 *   cell_table    (3k+1) x (k+1) doubles: K on kernel cell i as sum_m T[i][m] tau^m,
 *                 tau = t - (t_i + 1/2), t_i = -(3k+1)/2 + i;
 *   basis_matrix  nb x nb doubles, nb = (k+1)(k+2)/2: row i = Dubiner mode i written in the
 *                 centred monomials rho^a sigma^b (rho = 3r-1, sigma = 3s-1), columns in the
 *                 device Horner order (a = k..0, b = 0..k-a).
 * Either pointer may be NULL. */
siac_status siac_host_tables(int32_t k, double *cell_table, double *basis_matrix);

/* Copy the first n device triangle records, in binning order, to host memory `out`
 * (n * record_doubles); *record_doubles receives the record length.  which = 0: the mesh
 * record (csrc/siac_device.cuh Rec), 1: the jump record (csrc/siac_jump.cuh JRec), 2: the
 * closed-form cross-term record (XRec).  Diagnostics only. */
siac_status siac_debug_records(siac_ctx *ctx, int32_t which, int64_t n, double *out, int32_t *record_doubles);

/* ---- Tetrahedral meshes ("extension of these ideas to
 * 3D over unstructured tetrahedral meshes").  The 3D form of Eq. (1) -- the stencil is the tensor
 * product of three 1D kernels (L212-214) -- integrated exactly as in Eq. (2): each tetrahedron
 * the stencil touches is cut by the kernel breakplanes into pieces inside single kernel cells
 * (depth-first plane splits; a cut tetrahedron is a tetrahedron + a prism or two prisms, a prism
 * 3 tetrahedra), each piece integrated by a collapsed Gauss-Jacobi rule exact for degree 4k
 * (three kernel factors of degree k and u of degree k).
 * Direct method (warp per point tile, siac3_set_schedule); conventions as for the 2D calls above. */
typedef struct siac3_ctx siac3_ctx;
typedef struct {
    int32_t k;          /* dG degree 1..3 */
    double  h;          /* kernel scaling > 0 */
    int32_t periodic;   /* bit d (0..2): axis d periodic; non-periodic axes use zero extension */
    double  domain[6];  /* x0, y0, z0, x1, y1, z1 */
    int32_t device;
} siac3_params;

/* vertices_xyz  host, n_vertices x 3 doubles;  tets  host, n_tets x 4 int32 (0-based, any
 *               orientation);  coeffs  host, n_tets x (k+1)(k+2)(k+3)/6 doubles: coefficients of
 *               the monomials r^a s^b t^c of the unit reference tetrahedron, point = v0 +
 *               r (v1 - v0) + s (v2 - v0) + t (v3 - v0), modes ordered by a+b+c, then c, then b.
 * Errors: SIAC_EINVAL (k outside 1..3, h, domain, (3k+1)h larger than a periodic extent, indices,
 *   zero-volume tetrahedra, non-finite data), SIAC_EDEVICE, SIAC_ENOMEM, SIAC_ECUDA. */
siac_status siac3_create(siac3_ctx **out, const double *vertices_xyz, int64_t n_vertices,
                         const int32_t *tets, int64_t n_tets, const double *coeffs, const siac3_params *params);
/* host buffers, blocking: points_xyz n_points x 3 -> values_out n_points (input order).  Reports
 * SIAC_EINTERNAL if a piece stack overflowed (h much smaller than the tetrahedra). */
siac_status siac3_eval(siac3_ctx *ctx, const double *points_xyz, int64_t n_points, double *values_out);
/* device buffers, stream-ordered (cuda_stream NULL = legacy default stream). */
siac_status siac3_eval_async(siac3_ctx *ctx, const double *d_points_xyz, int64_t n_points, double *d_values_out,
                             void *cuda_stream);
/* Evaluation mapping for later evaluations (same decomposition, rule and result up to rounding
 * order): 0 (default) = warp per 32-point tile -- the tile's candidate tetrahedra walked
 * warp-uniformly, the pieces split per lane and queued in shared memory, the quadrature run 32
 * pieces at a time in lock step; 1 = thread per point (the paper's per-point mapping, Alg. 2,
 * PAPER.md L552-565).  SIAC_EINVAL for other values. */
siac_status siac3_set_schedule(siac3_ctx *ctx, int32_t schedule);
/* counting of (point, tetrahedron image) pairs and integrated pieces in later evaluations */
siac_status siac3_set_counting(siac3_ctx *ctx, int32_t enable);
siac_status siac3_stats(const siac3_ctx *ctx, int64_t *pairs, int64_t *pieces);
/* host: the collapsed rule on the unit tetrahedron with n^3 points, exact for degree 2n-1:
 * out n^3 x 4 doubles (r, s, t, weight); weights sum to 1/6. */
siac_status siac3_tet_rule(int32_t n, double *out);
void        siac3_destroy(siac3_ctx *ctx);
const char *siac3_last_error(const siac3_ctx *ctx);

/* Free everything the context owns.  NULL-safe. */
void siac_destroy(siac_ctx *ctx);

/* Last error message for ctx (or the calling thread's last siac_create error if ctx is NULL). */
const char *siac_last_error(const siac_ctx *ctx);

/* Library version string. */
const char *siac_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SIAC_H */
