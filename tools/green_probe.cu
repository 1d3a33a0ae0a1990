// Probe of green-context SM splits on this device (tools only): for each
// minCount, how many groups cuDevSmResourceSplitByCount yields and their sizes,
// and a sequential split (one group at a time from the remainder).
#include <cuda.h>
#include <cstdio>
#include <vector>
int main() {
    cuInit(0);
    CUdevice d;
    cuDeviceGet(&d, 0);
    CUcontext c;
    cuDevicePrimaryCtxRetain(&c, d);
    cuCtxSetCurrent(c);
    CUdevResource full;
    cuDeviceGetDevResource(d, &full, CU_DEV_RESOURCE_TYPE_SM);
    printf("{\"total\": %u, \"splits\": [", full.sm.smCount);
    int first = 1;
    for (unsigned mc : {8u, 16u, 24u, 32u, 40u, 48u, 64u, 72u, 80u, 96u}) {
        unsigned n = 64;
        std::vector<CUdevResource> r(64);
        CUdevResource rem;
        CUresult e = cuDevSmResourceSplitByCount(r.data(), &n, &full, &rem, 0, mc);
        printf("%s{\"min\": %u, \"rc\": %d, \"groups\": %u, \"sizes\": [", first ? "" : ", ", mc, (int)e, e ? 0 : n);
        first = 0;
        for (unsigned i = 0; !e && i < n; ++i) printf("%s%u", i ? ", " : "", r[i].sm.smCount);
        printf("], \"rem\": %u}", e ? 0 : rem.sm.smCount);
    }
    printf("], \"sequential\": [");
    for (auto seq : std::vector<std::vector<unsigned>>{{96, 48}, {80, 40, 24}, {48, 96}, {72, 72}, {64, 64, 16}}) {
        CUdevResource avail = full;
        printf("[");
        for (size_t i = 0; i < seq.size(); ++i) {
            CUdevResource part, rem;
            unsigned nb = 1;
            CUresult e = cuDevSmResourceSplitByCount(&part, &nb, &avail, &rem, 0, seq[i]);
            printf("%s{\"want\": %u, \"rc\": %d, \"nb\": %u, \"got\": %u, \"rem\": %u}", i ? ", " : "", seq[i], (int)e, nb,
                   e ? 0 : part.sm.smCount, e ? 0 : rem.sm.smCount);
            if (e || nb < 1) break;
            avail = rem;
        }
        printf("]%s", seq.size() == 3 && seq[2] == 16 ? "" : ", ");
    }
    printf("]}\n");
    return 0;
}
