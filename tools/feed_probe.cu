// feed_probe.cu -- how fast can TMA fill shared memory on this B200, and does multicast
// help?  (The measurement behind K2's feed analysis, profiles/r02_k2_measurements.md.)
//
// Every CTA runs K2's producer pattern without MMAs: a 3-stage ring of 64 KiB per CTA,
// per stage four 16 KiB TMA boxes (two "A" boxes of its own rows, two "B" boxes), a
// consumer thread that releases each stage as soon as it lands.  The operands are an
// L2-resident 64 MiB region (K2's loads are mostly L2 hits: 36.6 of 275 GB come from
// DRAM), so the rate measured is the L2 -> shared-memory delivery rate.
//   mode 0: clusters of 2, every box unicast (K2 today)
//   mode 1: clusters of 4, every box unicast
//   mode 2: clusters of 4, the B boxes multicast to the CTA pair that shares them
//           (ranks r and r ^ 2), so the B bytes are read from L2 once per two CTAs
// Reported: delivered bytes (landing in shared memory) per second, and the L2 read
// bytes per second they correspond to.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/feed_probe tools/feed_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <vector>

constexpr int BOX_ROWS = 128, BOX_BYTES = 128 * 128, STAGES = 3, STAGE_BYTES = 4 * BOX_BYTES;
constexpr int SMEM = STAGES * STAGE_BYTES + 1024 + 64;

__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint32_t ctarank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t mapa(uint32_t a, uint32_t r) {
    uint32_t o;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(o) : "r"(a), "r"(r));
    return o;
}
__device__ __forceinline__ void wait(uint32_t bar, uint32_t ph) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                     : "=r"(ok) : "r"(bar), "r"(ph) : "memory");
}

template <int MODE>
__global__ void __launch_bounds__(64, 1) feed(const __grid_constant__ CUtensorMap map, int nk, int rows_total) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    const uint32_t base = (su32(smem_raw) + 1023u) & ~1023u;
    const uint32_t full = base + STAGES * STAGE_BYTES, empty = full + 8 * STAGES;
    const uint32_t rank = ctarank();
    constexpr int CS = MODE == 0 ? 2 : 4;
    const uint32_t partner = rank ^ 2u;   // MODE 2: the CTA receiving the same B boxes
    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(full + 8 * s));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(empty + 8 * s), "r"(MODE == 2 ? 2 : 1));
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    const int cluster = blockIdx.x / CS;
    // A rows: distinct per CTA (within the L2-resident region); B rows: shared by the CTAs
    // of equal rank & 1 in a cluster (and, as in K2's raster, by neighbouring clusters)
    const int a_row = ((cluster * CS + (int)rank) * 2 * BOX_ROWS) % (rows_total / 2);
    const int b_row = rows_total / 2 + ((cluster % 8) * 4 + (int)(rank & 1u)) * 2 * BOX_ROWS % (rows_total / 2);
    if (threadIdx.x == 0) {   // producer
        for (int kb = 0; kb < nk; ++kb) {
            const int s = kb % STAGES;
            const uint32_t ph = (uint32_t)(kb / STAGES) & 1u;
            wait(empty + 8 * s, ph ^ 1u);
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(full + 8 * s),
                         "r"(STAGE_BYTES) : "memory");
            const uint32_t st = base + s * STAGE_BYTES;
            const int kc = (kb % 128) * 32;   // 128 columns of 4-byte elements = 128 B per box row
            for (int j = 0; j < 2; ++j)
                asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                             ::"r"(st + j * BOX_BYTES), "l"(&map), "r"(kc), "r"(a_row + j * BOX_ROWS), "r"(full + 8 * s)
                             : "memory");
            if (MODE == 2) {
                if (rank < 2) {   // issue the B boxes once, into this CTA and its partner
                    const uint16_t mask = (uint16_t)((1u << rank) | (1u << partner));
                    for (int j = 0; j < 2; ++j)
                        asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1, {%2, %3}], [%4], %5;"
                                     ::"r"(st + (2 + j) * BOX_BYTES), "l"(&map), "r"(kc), "r"(b_row + j * BOX_ROWS),
                                     "r"(full + 8 * s), "h"(mask) : "memory");
                }
            } else {
                for (int j = 0; j < 2; ++j)
                    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                                 ::"r"(st + (2 + j) * BOX_BYTES), "l"(&map), "r"(kc), "r"(b_row + j * BOX_ROWS),
                                 "r"(full + 8 * s) : "memory");
            }
        }
    } else if (threadIdx.x == 32) {   // consumer: release each stage as it lands
        for (int kb = 0; kb < nk; ++kb) {
            const int s = kb % STAGES;
            wait(full + 8 * s, (uint32_t)(kb / STAGES) & 1u);
            asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(empty + 8 * s) : "memory");
            if (MODE == 2)   // the B issuer of this stage (rank & 1) must see this CTA done too
                asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];"
                             ::"r"(mapa(empty + 8 * s, partner)) : "memory");
        }
    }
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

typedef CUresult (*EncFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                          const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                          CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

template <int MODE>
static double run(const CUtensorMap &map, int ctas, int nk, int rows_total) {
    constexpr int CS = MODE == 0 ? 2 : 4;
    auto k = feed<MODE>;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM);
    cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(ctas);
    cfg.blockDim = dim3(64);
    cfg.dynamicSmemBytes = SMEM;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = CS;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaLaunchKernelEx(&cfg, k, map, 8, rows_total);
    cudaDeviceSynchronize();
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    cudaLaunchKernelEx(&cfg, k, map, nk, rows_total);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    return ms;
}

int main() {
    cudaDeviceProp p;
    cudaGetDeviceProperties(&p, 0);
    const int rows_total = 4096;                       // x 16 KiB rows of 4 KiB? see below
    const uint64_t cols = 4096;                        // 4-byte elements per row: 16 KiB rows
    const size_t bytes = (size_t)rows_total * cols * 4;   // 64 MiB: L2-resident
    void *buf = nullptr;
    cudaMalloc(&buf, bytes);
    cudaMemset(buf, 0, bytes);
    EncFn enc = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void **)&enc, cudaEnableDefault, &q);
    CUtensorMap map;
    cuuint64_t dims[2] = {cols, (cuuint64_t)rows_total};
    cuuint64_t strides[1] = {cols * 4};
    cuuint32_t box[2] = {32, BOX_ROWS};
    cuuint32_t es[2] = {1, 1};
    enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, buf, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
        CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    const int nk = 4096;
    printf("{\"device\": \"%s\", \"sms\": %d", p.name, p.multiProcessorCount);
    struct M { int mode, ctas; const char *name; } modes[] = {{0, 148, "cluster2_unicast_148"},
                                                              {1, 132, "cluster4_unicast_132"},
                                                              {2, 132, "cluster4_multicastB_132"},
                                                              {0, 132, "cluster2_unicast_132"}};
    for (auto &m : modes) {
        double ms = m.mode == 0 ? run<0>(map, m.ctas, nk, rows_total)
                  : m.mode == 1 ? run<1>(map, m.ctas, nk, rows_total) : run<2>(map, m.ctas, nk, rows_total);
        const double delivered = (double)m.ctas * nk * STAGE_BYTES;
        const double l2 = m.mode == 2 ? delivered * 0.75 : delivered;
        printf(", \"%s\": {\"ms\": %.3f, \"delivered_TBps\": %.2f, \"l2_read_TBps\": %.2f}", m.name, ms,
               delivered / ms / 1e9, l2 / ms / 1e9);
    }
    printf(", \"err\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
