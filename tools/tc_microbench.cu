// tc_microbench.cu -- measured tcgen05 tensor-core peaks on the B200 (roofline
// denominators for K2 and for INT8 Ozaki planning).  One CTA (or CTA pair)
// per SM issues back-to-back tcgen05.mma from zero-filled shared memory into
// TMEM (no global traffic), CUDA-event timed.
//   kind::tf32  M=128 N=256 K=8   (cta_group::1) and M=256 N=256 (cta_group::2)
//   kind::i8    M=128 N=256 K=32  (cta_group::1) and M=256 N=256 (cta_group::2)
//   kind::f16   M=256 N=256 K=16  BF16 operands (cta_group::2), and the tf32bf16 K2 mix
//               (per 4 instructions: 2 kind::f16 K=16 + 2 kind::tf32 K=8, cta_group::2),
//               reported as TF32-equivalent TFLOP/s (one f16 K=16 instruction = one
//               tf32 K=8 instruction's worth of time if BF16 runs at twice the TF32 rate)
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/tc_microbench tools/tc_microbench.cu
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint64_t desc_k_sw128(uint32_t saddr) {
    return (uint64_t)((saddr >> 4) & 0x3FFFu) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
           ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}

// kind: 0 = tf32 (a/b fmt 2, c F32), 1 = i8 (a/b fmt 1 signed, c S32), 2 = f16 with BF16 (a/b fmt 1, c F32)
__host__ __device__ constexpr uint32_t idesc(int kind, int M, int N) {
    return kind == 0 ? ((1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24))
           : kind == 1 ? ((2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24))
                       : ((1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24));
}

template <int KIND, int CG>
__global__ void __launch_bounds__(128, 1) tc_peak(int iters, int *flag) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = (uint8_t *)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
    __shared__ uint32_t tslot;
    __shared__ __align__(8) uint64_t bar;
    const int warp = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < 48 * 1024 / 4; i += blockDim.x) ((uint32_t *)smem)[i] = 0;
    uint32_t rank = 0;
    if (CG == 2) asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    if (warp == 0) {
        if (CG == 1) {
            asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(su32(&tslot)));
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
        } else {
            asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(su32(&tslot)));
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    if (CG == 2)
        asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    else
        __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = tslot;
    const uint32_t sa = su32(smem), sb = sa + 16384;
    constexpr int M = CG == 1 ? 128 : 256;
    constexpr uint32_t id = idesc(KIND == 3 ? 0 : KIND, M, 256);
    constexpr uint32_t id16 = idesc(2, M, 256);
    if (threadIdx.x == 0 && rank == 0) {
        for (int it = 0; it < iters; ++it) {
#pragma unroll
            for (int kk = 0; kk < 4; ++kk) {
                const uint64_t da = desc_k_sw128(sa + kk * 32), db = desc_k_sw128(sb + kk * 32);
                const uint32_t acc = (it | kk) ? 1u : 0u;
                if (KIND == 2 || (KIND == 3 && kk < 2))
                    asm volatile("{.reg .pred p; setp.ne.b32 p, %4, 0; tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;}"
                                 ::"r"(tmem), "l"(da), "l"(db), "r"(id16), "r"(acc));
                else if (KIND == 3)
                    asm volatile("{.reg .pred p; setp.ne.b32 p, %4, 0; tcgen05.mma.cta_group::2.kind::tf32 [%0], %1, %2, %3, p;}"
                                 ::"r"(tmem), "l"(da), "l"(db), "r"(id), "r"(acc));
                else if (KIND == 0 && CG == 1)
                    asm volatile("{.reg .pred p; setp.ne.b32 p, %4, 0; tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;}"
                                 ::"r"(tmem), "l"(da), "l"(db), "r"(id), "r"(acc));
                else if (KIND == 0)
                    asm volatile("{.reg .pred p; setp.ne.b32 p, %4, 0; tcgen05.mma.cta_group::2.kind::tf32 [%0], %1, %2, %3, p;}"
                                 ::"r"(tmem), "l"(da), "l"(db), "r"(id), "r"(acc));
                else if (CG == 1)
                    asm volatile("{.reg .pred p; setp.ne.b32 p, %4, 0; tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;}"
                                 ::"r"(tmem), "l"(da), "l"(db), "r"(id), "r"(acc));
                else
                    asm volatile("{.reg .pred p; setp.ne.b32 p, %4, 0; tcgen05.mma.cta_group::2.kind::i8 [%0], %1, %2, %3, p;}"
                                 ::"r"(tmem), "l"(da), "l"(db), "r"(id), "r"(acc));
            }
        }
        if (CG == 1)
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar))
                         : "memory");
        else
            asm volatile("{.reg .b16 m; mov.b16 m, 3; tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], m;}"
                         ::"r"(su32(&bar)) : "memory");
    }
    if (threadIdx.x == 0) {
        uint32_t ok = 0;
        while (!ok)
            asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0,1,0,p;}"
                         : "=r"(ok) : "r"(su32(&bar)) : "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    if (CG == 2)
        asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    else
        __syncthreads();
    if (warp == 0) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        if (CG == 1) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(tmem));
        else asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 256;" ::"r"(tmem));
    }
    if (threadIdx.x == 0 && iters < 0) flag[0] = 1;
}

template <int KIND, int CG>
double run(int sms, int iters) {
    auto k = tc_peak<KIND, CG>;
    const int smem = 48 * 1024 + 1024;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    int *flag;
    cudaMalloc(&flag, 4);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(sms);
    cfg.blockDim = dim3(128);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = CG;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaLaunchKernelEx(&cfg, k, 16, flag);
    cudaDeviceSynchronize();
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    cudaLaunchKernelEx(&cfg, k, iters, flag);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    const double K = (KIND == 0 || KIND == 3) ? 8 : KIND == 2 ? 16 : 32;   // KIND 3: TF32-equivalent
    const double per_instr = 2.0 * (CG == 1 ? 128 : 256) * 256 * K;
    const double issuers = CG == 1 ? sms : sms / 2;
    cudaFree(flag);
    return per_instr * 4.0 * iters * issuers / (ms * 1e-3) / 1e12;
}

int main() {
    cudaDeviceProp p;
    cudaGetDeviceProperties(&p, 0);
    int sms = p.multiProcessorCount;
    int iters = 20000;
    double tf1 = run<0, 1>(sms, iters);
    double tf2 = run<0, 2>(sms, iters);
    double i1 = run<1, 1>(sms, iters);
    double i2 = run<1, 2>(sms, iters);
    double b2 = run<2, 2>(sms, iters);
    double m2 = run<3, 2>(sms, iters);
    printf("{\"device\":\"%s\",\"sms\":%d,\"tf32_tflops_1sm_m128n256\":%.1f,\"tf32_tflops_2sm_m256n256\":%.1f,"
           "\"i8_tops_1sm_m128n256\":%.1f,\"i8_tops_2sm_m256n256\":%.1f,\"bf16_tflops_2sm_m256n256\":%.1f,"
           "\"tf32bf16_mix_tf32eq_tflops_2sm\":%.1f,\"err\":\"%s\"}\n",
           p.name, sms, tf1, tf2, i1, i2, b2, m2, cudaGetErrorString(cudaGetLastError()));
    return 0;
}
