// fp64_mix_probe.cu -- do DMMA (FP64 tensor) and DFMA (FP64 SIMT) issue from
// separate pipes on sm_100a?  Warps [0, nd) run DMMA.8x8x4, the rest DFMA,
// from registers; the combined FLOP rate tells whether a hybrid DGEMM pays.
#include <cstdio>
#include <cuda_runtime.h>

__global__ void mix(double *out, int iters, int nd) {
    const int warp = threadIdx.x >> 5;
    double a = threadIdx.x * 1e-3, b = 1.0 + blockIdx.x * 1e-6, s = 0;
    if (warp < nd) {
        double c[16][2];
#pragma unroll
        for (int i = 0; i < 16; ++i) c[i][0] = c[i][1] = 0.0;
        for (int it = 0; it < iters; ++it) {
#pragma unroll
            for (int i = 0; i < 16; ++i)
                asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                             : "+d"(c[i][0]), "+d"(c[i][1]) : "d"(a), "d"(b));
        }
#pragma unroll
        for (int i = 0; i < 16; ++i) s += c[i][0] + c[i][1];
    } else {
        double c[16];
#pragma unroll
        for (int i = 0; i < 16; ++i) c[i] = i;
        for (int it = 0; it < iters * 8; ++it) {   // 8x the loop count: one DMMA = 8 DFMA per lane
#pragma unroll
            for (int i = 0; i < 16; ++i) c[i] = fma(a, c[i], b);
        }
#pragma unroll
        for (int i = 0; i < 16; ++i) s += c[i];
    }
    if (s == 12345.678) out[0] = s;
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    double *o;
    cudaMalloc(&o, 8);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int iters = 4000, threads = 256;
    printf("{");
    for (int nd : {8, 0, 4, 6, 2}) {
        mix<<<sms, threads>>>(o, 10, nd);
        cudaEventRecord(e0);
        mix<<<sms, threads>>>(o, iters, nd);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        // DMMA warp: 16 * iters * 512 flop; DFMA warp: 16 * iters*8 * 32 lanes * 2 flop = same per warp
        double flops = 512.0 * 16 * iters * (threads / 32) * sms;
        printf("%s\"dmma_warps_%d_of_8_tflops\":%.2f", nd == 8 ? "" : ",", nd, flops / ms / 1e9);
    }
    printf(",\"err\":\"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
}
