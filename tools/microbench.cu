// microbench.cu -- FP64 pipe peaks on the B200 (the K1 roofline denominator).
// DMMA.8x8x4 (mma.sync m8n8k4 f64) and DFMA throughput from registers,
// 148 x 2 CTAs x 256 threads, CUDA-event timed.  Build: nvcc -arch=sm_100a.
#include <cstdio>
#include <cuda_runtime.h>

__global__ void dmma_peak(double *out, int iters) {
    double a = threadIdx.x * 1e-3, b = 1.0 + blockIdx.x * 1e-6;
    double c[16][2];
#pragma unroll
    for (int i = 0; i < 16; ++i) c[i][0] = c[i][1] = 0.0;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < 16; ++i)
            asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                         : "+d"(c[i][0]), "+d"(c[i][1]) : "d"(a), "d"(b));
    }
    double s = 0;
#pragma unroll
    for (int i = 0; i < 16; ++i) s += c[i][0] + c[i][1];
    if (s == 12345.678) out[0] = s;
}

__global__ void dfma_peak(double *out, int iters) {
    double a = threadIdx.x * 1e-3, b = 1.0 + blockIdx.x * 1e-6;
    double c[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) c[i] = i;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < 16; ++i) c[i] = fma(a, c[i], b);
    }
    double s = 0;
#pragma unroll
    for (int i = 0; i < 16; ++i) s += c[i];
    if (s == 12345.678) out[0] = s;
}

int main() {
    cudaDeviceProp p;
    cudaGetDeviceProperties(&p, 0);
    int sms = p.multiProcessorCount;
    double *out;
    cudaMalloc(&out, 8);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    int clk = 0;
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    printf("{\"device\":\"%s\",\"sms\":%d,\"clock_khz\":%d", p.name, sms, clk);
    for (int bps : {1, 2, 4}) {
        int iters = 20000;
        dim3 grid(sms * bps);
        dmma_peak<<<grid, 256>>>(out, 100);
        cudaEventRecord(e0);
        dmma_peak<<<grid, 256>>>(out, iters);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        double flops = 2.0 * 256.0 * 16 * iters * (grid.x * 256 / 32);
        printf(",\"dmma_tflops_bps%d\":%.2f", bps, flops / ms / 1e9);
        dfma_peak<<<grid, 256>>>(out, 100);
        cudaEventRecord(e0);
        dfma_peak<<<grid, 256>>>(out, iters);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
        flops = 2.0 * 16 * iters * (double)grid.x * 256;
        printf(",\"dfma_tflops_bps%d\":%.2f", bps, flops / ms / 1e9);
    }
    printf(",\"err\":\"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
