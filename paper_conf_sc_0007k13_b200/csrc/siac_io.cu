// siac_io.cu -- the GPU steps either side of the SIAC path: L2 projection
// of a field into the dG modes the filter consumes, the mapping of reference nodes to element
// points, and error norms of filtered values ("grid points ... used at the end of the
// simulation for such things as error calculations").
//
//   siac_projection_rule     collapsed Gauss-Legendre rule on the unit triangle (host)
//   siac_map_points_async    x = v0 + r (v1 - v0) + s (v2 - v0) for every (element, node)
//   siac_project_async       c_i = sum_q W_q phi_i(node_q) f(element, q): orthonormal Dubiner
//                            modes (the element mass matrix is |T|/2 I on the reference
//                            triangle of area 2, so the projection is one weighted sum)
//   siac_error_norms_async   sqrt(sum w e^2), max |e|, sum w with e = u - ref, deterministic
//                            two-pass reduction (fixed grid, fixed order)
#include <cuda_runtime.h>

#include <cmath>
#include <map>
#include <mutex>
#include <string>
#include <tuple>
#include <vector>

#include "../../include/siac.h"
#include "siac_internal.h"
#include "siac_math.h"

namespace {

siac_status io_fail(siac_status st, const std::string &msg) {
    siac_set_thread_error(msg);
    return st;
}

#define IOCK(call)                                                                            \
    do {                                                                                      \
        cudaError_t e_ = (call);                                                              \
        if (e_ != cudaSuccess) return io_fail(SIAC_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e_)); \
    } while (0)

// Gauss-Legendre nodes/weights on [-1, 1] by Newton iteration on P_n (long double).
void gauss_legendre(int n, std::vector<long double> &x, std::vector<long double> &w) {
    const long double pi = 3.141592653589793238462643383279502884L;
    x.assign(n, 0.0L);
    w.assign(n, 0.0L);
    for (int i = 0; i < n; ++i) {
        long double z = cosl(pi * (i + 0.75L) / (n + 0.5L)), dp = 0.0L;
        for (int it = 0; it < 100; ++it) {
            long double p0 = 1.0L, p1 = z;
            for (int j = 2; j <= n; ++j) {
                const long double p2 = ((2 * j - 1) * z * p1 - (j - 1) * p0) / j;
                p0 = p1;
                p1 = p2;
            }
            if (n == 1) { p1 = z; p0 = 1.0L; }
            dp = n * (z * p1 - p0) / (z * z - 1.0L);
            const long double dz = p1 / dp;
            z -= dz;
            if (fabsl(dz) < 1e-30L) break;
        }
        long double p0 = 1.0L, p1 = z;
        for (int j = 2; j <= n; ++j) {
            const long double p2 = ((2 * j - 1) * z * p1 - (j - 1) * p0) / j;
            p0 = p1;
            p1 = p2;
        }
        dp = n * (z * p1 - p0) / (z * z - 1.0L);
        x[i] = z;
        w[i] = 2.0L / ((1.0L - z * z) * dp * dp);
    }
}

// Collapsed (Duffy) rule: n^2 nodes (r, s) on the unit triangle; weights of the reference
// triangle {xi, eta >= -1, xi + eta <= 0} (area 2), exact to total degree 2n - 2.
void collapsed_rule(int n, std::vector<double> &rs, std::vector<double> &w) {
    std::vector<long double> g, gw;
    gauss_legendre(n, g, gw);
    rs.resize(2 * (size_t)n * n);
    w.resize((size_t)n * n);
    for (int i = 0; i < n; ++i)
        for (int j = 0; j < n; ++j) {
            const long double a = g[i], b = g[j];
            const long double xi = (1.0L + a) * (1.0L - b) / 2.0L - 1.0L, eta = b;
            const size_t q = (size_t)i * n + j;
            rs[2 * q] = (double)((xi + 1.0L) / 2.0L);
            rs[2 * q + 1] = (double)((eta + 1.0L) / 2.0L);
            w[q] = (double)(gw[i] * gw[j] * (1.0L - b) / 2.0L);
        }
}

// Device table M[q * nb + i] = W_q phi_i(node_q), cached per (device, k, n_quad).
std::mutex g_mu;
std::map<std::tuple<int, int, int>, double *> g_tables;

siac_status projection_table(int k, int n_quad, const double **out) {
    int dev = 0;
    IOCK(cudaGetDevice(&dev));
    std::lock_guard<std::mutex> lock(g_mu);
    auto key = std::make_tuple(dev, k, n_quad);
    auto it = g_tables.find(key);
    if (it != g_tables.end()) { *out = it->second; return SIAC_OK; }
    std::vector<double> rs, w;
    collapsed_rule(n_quad, rs, w);
    std::vector<std::pair<int, int>> order;
    const std::vector<double> R = siac::dubiner_to_centred(k, &order);   // mode i -> centred monomials
    const int nb = (k + 1) * (k + 2) / 2, nq = n_quad * n_quad;
    std::vector<double> M((size_t)nq * nb);
    for (int q = 0; q < nq; ++q) {
        const double rho = 3.0 * rs[2 * q] - 1.0, sig = 3.0 * rs[2 * q + 1] - 1.0;
        for (int i = 0; i < nb; ++i) {
            double v = 0.0;
            for (int j = 0; j < nb; ++j)
                v += R[(size_t)i * nb + j] * std::pow(rho, order[j].first) * std::pow(sig, order[j].second);
            M[(size_t)q * nb + i] = w[q] * v;
        }
    }
    double *d = nullptr;
    IOCK(cudaMalloc(&d, sizeof(double) * M.size()));
    IOCK(cudaMemcpy(d, M.data(), sizeof(double) * M.size(), cudaMemcpyHostToDevice));
    g_tables[key] = d;
    *out = d;
    return SIAC_OK;
}

__global__ void k_map_points(const double *V, const int *T, int64_t nt, const double *rs, int nq, double *out) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= nt * nq) return;
    const int64_t t = i / nq;
    const int q = (int)(i - t * nq);
    const int a = T[3 * t], b = T[3 * t + 1], c = T[3 * t + 2];
    const double r = rs[2 * q], s = rs[2 * q + 1];
    const double x0 = V[2 * a], y0 = V[2 * a + 1];
    out[2 * i] = fma(s, V[2 * c] - x0, fma(r, V[2 * b] - x0, x0));
    out[2 * i + 1] = fma(s, V[2 * c + 1] - y0, fma(r, V[2 * b + 1] - y0, y0));
}

// One warp per element: lanes stride the nodes (coalesced f reads), nb partial sums per lane,
// butterfly reductions in a fixed order, lane i writes mode i.
template <int NB>
__global__ void __launch_bounds__(256) k_project(const double *f, int64_t nt, int nq, const double *M, double *c) {
    extern __shared__ double sM[];
    for (int i = threadIdx.x; i < nq * NB; i += blockDim.x) sM[i] = M[i];
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int64_t t = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    if (t >= nt) return;
    double acc[NB];
#pragma unroll
    for (int i = 0; i < NB; ++i) acc[i] = 0.0;
    for (int q = lane; q < nq; q += 32) {
        const double fv = f[t * nq + q];
#pragma unroll
        for (int i = 0; i < NB; ++i) acc[i] = fma(sM[q * NB + i], fv, acc[i]);
    }
    double mine = 0.0;
#pragma unroll
    for (int i = 0; i < NB; ++i) {
        double v = acc[i];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if (lane == i) mine = v;
    }
    if (lane < NB) c[t * NB + lane] = mine;
}

constexpr int ERR_BLOCKS = 296, ERR_THREADS = 256;

__global__ void __launch_bounds__(ERR_THREADS) k_err_partial(const double *u, const double *ref, const double *w,
                                                             int64_t n, double *part) {
    __shared__ double s2[ERR_THREADS], smax[ERR_THREADS], sw[ERR_THREADS];
    double a2 = 0.0, am = 0.0, aw = 0.0;
    for (int64_t i = (int64_t)blockIdx.x * ERR_THREADS + threadIdx.x; i < n; i += (int64_t)ERR_BLOCKS * ERR_THREADS) {
        const double e = u[i] - ref[i];
        const double wi = w ? w[i] : 1.0;
        a2 = fma(wi * e, e, a2);
        am = fmax(am, fabs(e));
        aw += wi;
    }
    s2[threadIdx.x] = a2; smax[threadIdx.x] = am; sw[threadIdx.x] = aw;
    __syncthreads();
    for (int o = ERR_THREADS / 2; o > 0; o >>= 1) {
        if (threadIdx.x < o) {
            s2[threadIdx.x] += s2[threadIdx.x + o];
            smax[threadIdx.x] = fmax(smax[threadIdx.x], smax[threadIdx.x + o]);
            sw[threadIdx.x] += sw[threadIdx.x + o];
        }
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        part[3 * blockIdx.x] = s2[0];
        part[3 * blockIdx.x + 1] = smax[0];
        part[3 * blockIdx.x + 2] = sw[0];
    }
}

__global__ void k_err_final(const double *part, double *out) {
    if (threadIdx.x != 0) return;
    double a2 = 0.0, am = 0.0, aw = 0.0;
    for (int b = 0; b < ERR_BLOCKS; ++b) {
        a2 += part[3 * b];
        am = fmax(am, part[3 * b + 1]);
        aw += part[3 * b + 2];
    }
    out[0] = sqrt(a2);
    out[1] = am;
    out[2] = aw;
}

}  // namespace

extern "C" {

siac_status siac_projection_rule(int32_t n_quad, double *rs_out, double *w_out) {
    if (n_quad < 1 || n_quad > 64 || !rs_out || !w_out) return io_fail(SIAC_EINVAL, "siac_projection_rule: bad arguments");
    std::vector<double> rs, w;
    collapsed_rule(n_quad, rs, w);
    for (size_t i = 0; i < rs.size(); ++i) rs_out[i] = rs[i];
    for (size_t i = 0; i < w.size(); ++i) w_out[i] = w[i];
    return SIAC_OK;
}

siac_status siac_map_points_async(const double *d_vertices_xy, const int32_t *d_triangles, int64_t n_triangles,
                                  const double *d_rs, int32_t n_nodes, double *d_points_out, void *stream) {
    if (n_triangles < 0 || n_nodes < 1) return io_fail(SIAC_EINVAL, "siac_map_points_async: bad sizes");
    if (n_triangles == 0) return SIAC_OK;
    if (!d_vertices_xy || !d_triangles || !d_rs || !d_points_out) return io_fail(SIAC_EINVAL, "siac_map_points_async: NULL pointer");
    const int64_t n = n_triangles * n_nodes;
    k_map_points<<<(unsigned)((n + 255) / 256), 256, 0, (cudaStream_t)stream>>>(d_vertices_xy, d_triangles, n_triangles,
                                                                                d_rs, n_nodes, d_points_out);
    IOCK(cudaGetLastError());
    return SIAC_OK;
}

siac_status siac_project_async(int32_t k, int32_t n_quad, const double *d_f, int64_t n_triangles, double *d_coeffs_out,
                               void *stream) {
    if (k < 1 || k > 4) return io_fail(SIAC_EINVAL, "siac_project_async: k must be in 1..4");
    if (n_quad < k + 1 || n_quad > 32) return io_fail(SIAC_EINVAL, "siac_project_async: n_quad must be in k+1..32");
    if (n_triangles < 0) return io_fail(SIAC_EINVAL, "siac_project_async: negative n_triangles");
    if (n_triangles == 0) return SIAC_OK;
    if (!d_f || !d_coeffs_out) return io_fail(SIAC_EINVAL, "siac_project_async: NULL pointer");
    const double *M = nullptr;
    const siac_status st = projection_table(k, n_quad, &M);
    if (st != SIAC_OK) return st;
    const int nq = n_quad * n_quad, nb = (k + 1) * (k + 2) / 2;
    const unsigned grid = (unsigned)((n_triangles + 7) / 8);
    const size_t smem = sizeof(double) * nq * nb;
    cudaStream_t s = (cudaStream_t)stream;
    switch (k) {
        case 1:
            IOCK(cudaFuncSetAttribute(k_project<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            k_project<3><<<grid, 256, smem, s>>>(d_f, n_triangles, nq, M, d_coeffs_out);
            break;
        case 2:
            IOCK(cudaFuncSetAttribute(k_project<6>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            k_project<6><<<grid, 256, smem, s>>>(d_f, n_triangles, nq, M, d_coeffs_out);
            break;
        case 3:
            IOCK(cudaFuncSetAttribute(k_project<10>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            k_project<10><<<grid, 256, smem, s>>>(d_f, n_triangles, nq, M, d_coeffs_out);
            break;
        default:
            IOCK(cudaFuncSetAttribute(k_project<15>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            k_project<15><<<grid, 256, smem, s>>>(d_f, n_triangles, nq, M, d_coeffs_out);
            break;
    }
    (void)nb;
    IOCK(cudaGetLastError());
    return SIAC_OK;
}

siac_status siac_error_norms_async(const double *d_u, const double *d_ref, const double *d_weights, int64_t n,
                                   double *d_out, void *stream) {
    if (n < 0 || !d_out) return io_fail(SIAC_EINVAL, "siac_error_norms_async: bad arguments");
    if (n > 0 && (!d_u || !d_ref)) return io_fail(SIAC_EINVAL, "siac_error_norms_async: NULL pointer");
    cudaStream_t s = (cudaStream_t)stream;
    double *part = nullptr;
    IOCK(cudaMallocAsync(&part, sizeof(double) * 3 * ERR_BLOCKS, s));
    k_err_partial<<<ERR_BLOCKS, ERR_THREADS, 0, s>>>(d_u, d_ref, d_weights, n, part);
    k_err_final<<<1, 32, 0, s>>>(part, d_out);
    IOCK(cudaGetLastError());
    IOCK(cudaFreeAsync(part, s));
    return SIAC_OK;
}

}  // extern "C"
