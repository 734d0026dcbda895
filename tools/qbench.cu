// qbench.cu -- microbenchmark: FP64 throughput of the sub-triangle quadrature alone
// (no clipping, no staging), to find the ceiling of the consumer stage.
// nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I paper_conf_sc_0007k13_b200/csrc
//      -DQB_N=2 -o qbench tools/qbench.cu
#include <cstdio>
#include <cuda_runtime.h>

#include "siac_device.cuh"

using namespace siacdev;

#ifndef QB_N
#define QB_N 1
#endif
#ifndef QB_K
#define QB_K 3
#endif
#ifndef QB_THREADS
#define QB_THREADS 256
#endif
#ifndef QB_MINB
#define QB_MINB 2
#endif

__global__ void __launch_bounds__(QB_THREADS, QB_MINB) qbench(const double *__restrict__ dat, int iters, double *out) {
    constexpr int K = QB_K;
    constexpr int NB = (K + 1) * (K + 2) / 2;
    const int tid = blockIdx.x * blockDim.x + threadIdx.x;
    SubTri<K> t[QB_N];
    double accum = 0.0;
#pragma unroll
    for (int n = 0; n < QB_N; ++n) {
        const double *p = dat + ((tid * QB_N + n) & 1023) * 40;
        t[n].p0x = p[0]; t[n].p0y = p[1]; t[n].e1x = p[2]; t[n].e1y = p[3]; t[n].e2x = p[4]; t[n].e2y = p[5];
        for (int m = 0; m <= K; ++m) { t[n].kx[m] = p[6 + m]; t[n].ky[m] = p[11 + m]; }
        t[n].cx = p[16]; t[n].cy = p[17];
        for (int m = 0; m < NB; ++m) t[n].d[m] = p[18 + m];
        t[n].g.M00 = p[34]; t[n].g.M01 = p[35]; t[n].g.M10 = p[36]; t[n].g.M11 = p[37]; t[n].g.zv0x = p[38]; t[n].g.zv0y = p[39];
    }
    for (int it = 0; it < iters; ++it) {
        double v[QB_N];
        integrate_subtri_n<K, QB_N>(t, v);
#pragma unroll
        for (int n = 0; n < QB_N; ++n) { accum += v[n]; t[n].p0x += 1e-12 * v[n]; }
    }
    if (accum == 12345.678) out[tid] = accum;
}

int main() {
    double *dat, *out;
    cudaMalloc(&dat, 1024 * 40 * sizeof(double));
    cudaMalloc(&out, 1 << 24);
    double h[1024 * 40];
    for (int i = 0; i < 1024 * 40; ++i) h[i] = 0.1 + 1e-3 * (i % 97);
    cudaMemcpy(dat, h, sizeof(h), cudaMemcpyHostToDevice);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int blocks_per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks_per_sm, qbench, QB_THREADS, 0);
    const int grid = sms * blocks_per_sm;
    const int iters = 200;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    qbench<<<grid, QB_THREADS>>>(dat, 10, out);
    cudaEventRecord(e0);
    qbench<<<grid, QB_THREADS>>>(dat, iters, out);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    constexpr int K = QB_K;
    const int nq = Rule<K>::NQ;
    const int nb = (K + 1) * (K + 2) / 2;
    const double subtris = (double)grid * QB_THREADS * QB_N * iters;
    const double flops = subtris * nq * 2.0 * (nb + 2 * K + 8);
    printf("K=%d N=%d threads=%d blocks/SM=%d warps/SM=%d: %.3f ms, %.3e subtri/s, %.2f TFLOP/s (model)  err=%s\n", K,
           QB_N, QB_THREADS, blocks_per_sm, blocks_per_sm * QB_THREADS / 32, ms, subtris / (ms * 1e-3),
           flops / (ms * 1e-3) / 1e12, cudaGetErrorString(cudaGetLastError()));
    return 0;
}
