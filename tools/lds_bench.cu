// Microbenchmark: shared-memory wavefronts and throughput of warp-uniform (broadcast) loads of
// 32/64/128-bit width, and of lane-distinct 128-bit loads.  Build:
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tools/bin/lds_bench tools/lds_bench.cu
// Run under ncu with --metrics l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,gpu__time_duration.sum
#include <cstdio>
#include <cuda_runtime.h>

template <int MODE>
__global__ void __launch_bounds__(128) k_lds(double *out, int iters) {
    __shared__ __align__(16) double buf[1024];
    for (int i = threadIdx.x; i < 1024; i += blockDim.x) buf[i] = 1.0 + i * 1e-3;
    __syncthreads();
    double acc0 = 0, acc1 = 0;
    const int lane = threadIdx.x & 31;
    int base = 0;
    for (int it = 0; it < iters; ++it) {
        // 16 loads of 16 bytes (uniform address unless MODE 3) per iteration
#pragma unroll
        for (int j = 0; j < 16; ++j) {
            const int off = (base + 8 * j) & 1000;
            if (MODE == 0) {        // 4 x 32-bit uniform
                const float *f = reinterpret_cast<const float *>(buf + off);
                acc0 += f[0] + f[3] + f[6] + f[9];
            } else if (MODE == 1) { // 2 x 64-bit uniform
                acc0 += buf[off]; acc1 += buf[off + 1];
            } else if (MODE == 2) { // 1 x 128-bit uniform
                const double2 v = *reinterpret_cast<const double2 *>(buf + off);
                acc0 += v.x; acc1 += v.y;
            } else if (MODE == 3) { // 1 x 128-bit, 4 distinct addresses (lane & 3), 176 B apart
                const double2 v = *reinterpret_cast<const double2 *>(buf + ((off & 511) + 22 * (lane & 3)));
                acc0 += v.x; acc1 += v.y;
            } else if (MODE == 4) { // 1 x 128-bit, 2 distinct addresses
                const double2 v = *reinterpret_cast<const double2 *>(buf + ((off & 511) + 22 * (lane & 1)));
                acc0 += v.x; acc1 += v.y;
            } else if (MODE == 5) { // 1 x 128-bit, 13 distinct rows of 4 doubles (lane % 13)
                const double2 v = *reinterpret_cast<const double2 *>(buf + ((off & 511) + 4 * (lane % 13)));
                acc0 += v.x; acc1 += v.y;
            } else if (MODE == 6) { // 4 distinct contiguous 16 B chunks (lane & 3)
                const double2 v = *reinterpret_cast<const double2 *>(buf + ((off & 511) + 2 * (lane & 3)));
                acc0 += v.x; acc1 += v.y;
            } else if (MODE == 7) { // 13 distinct contiguous 16 B chunks (lane % 13)
                const double2 v = *reinterpret_cast<const double2 *>(buf + ((off & 511) + 2 * (lane % 13)));
                acc0 += v.x; acc1 += v.y;
            } else if (MODE == 8) { // 4 distinct chunks, 4 per half-warp-contiguous pattern: (lane >> 3)
                const double2 v = *reinterpret_cast<const double2 *>(buf + ((off & 511) + 2 * (lane >> 3)));
                acc0 += v.x; acc1 += v.y;
            } else {                // 64-bit loads, 13 distinct contiguous doubles (lane % 13)
                acc0 += buf[(off & 511) + (lane % 13)];
                acc1 += buf[(off & 511) + 16 + (lane % 13)];
            }
        }
        base += 2;
    }
    if (acc0 + acc1 == 1234.5) out[threadIdx.x] = acc0;
}

int main() {
    double *d;
    cudaMalloc(&d, 1024 * sizeof(double));
    const int iters = 4096, grid = 148 * 8;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const char *names[10] = {"4x LDS.32 uniform", "2x LDS.64 uniform", "1x LDS.128 uniform", "1x LDS.128 4 addrs",
                             "1x LDS.128 2 addrs", "1x LDS.128 13 rows", "128 4 contiguous", "128 13 contiguous",
                             "128 4 contig lane>>3", "2x LDS.64 13 contig"};
    for (int m = 0; m < 10; ++m) {
        for (int rep = 0; rep < 2; ++rep) {
            cudaEventRecord(e0);
            if (m == 0) k_lds<0><<<grid, 128>>>(d, iters);
            if (m == 1) k_lds<1><<<grid, 128>>>(d, iters);
            if (m == 2) k_lds<2><<<grid, 128>>>(d, iters);
            if (m == 3) k_lds<3><<<grid, 128>>>(d, iters);
            if (m == 4) k_lds<4><<<grid, 128>>>(d, iters);
            if (m == 5) k_lds<5><<<grid, 128>>>(d, iters);
            if (m == 6) k_lds<6><<<grid, 128>>>(d, iters);
            if (m == 7) k_lds<7><<<grid, 128>>>(d, iters);
            if (m == 8) k_lds<8><<<grid, 128>>>(d, iters);
            if (m == 9) k_lds<9><<<grid, 128>>>(d, iters);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
        }
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        const double bytes16 = (double)grid * 4 * iters * 16;   // warp-level 16-byte loads
        printf("%-22s %8.3f ms  %.3f G warp-16B-loads/s\n", names[m], ms, bytes16 / ms / 1e6);
    }
    return 0;
}
