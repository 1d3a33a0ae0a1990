// cluster_probe.cu -- how many thread-block clusters of 2 / 4 / 8 CTAs (one CTA per SM:
// ~193 KB of dynamic shared memory, 576 threads, as K2) can be co-resident on this
// B200 (cudaOccupancyMaxActiveClusters): a cluster must fit in one GPC, so GPC sizes
// that are not multiples of the cluster size leave SMs idle.
#include <cuda_runtime.h>

#include <cstdio>

__global__ void dummy(int *p) {
    extern __shared__ int s[];
    if (p) p[0] = s[0];
}

int main() {
    cudaDeviceProp prop;
    cudaGetDeviceProperties(&prop, 0);
    const int smem = 3 * 65536 + 1024 + 256;
    cudaFuncSetAttribute(dummy, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(dummy, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    printf("{\"device\": \"%s\", \"sms\": %d", prop.name, prop.multiProcessorCount);
    for (int cs : {1, 2, 4, 8, 16}) {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(cs * 64);
        cfg.blockDim = dim3(576);
        cfg.dynamicSmemBytes = smem;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = cs;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        int n = -1;
        cudaError_t e = cudaOccupancyMaxActiveClusters(&n, dummy, &cfg);
        printf(", \"clusters_of_%d\": %d, \"sms_used_%d\": %d%s", cs, n, cs, n * cs, e ? " (error)" : "");
    }
    printf("}\n");
    return 0;
}
