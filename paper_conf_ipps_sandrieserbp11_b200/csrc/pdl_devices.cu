// pdl_devices.cu -- binding the descriptor's gpu Worker PUs to CUDA devices
// (PAPER.md SS III-A Worker PUs L505-511, unfixed properties instantiated by the
// runtime L737-747), SM partitions for heterogeneous-Worker emulation (green
// contexts, PDL property SM_LIMIT), and the Worker memory-region buffers.
#include "pdl_rt.hpp"

namespace pdlrt {

int get_encoder(pdlk::EncodeTiledFn *out) {
    if (g->encode) {
        *out = g->encode;
        return PDL_OK;
    }
    void *fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
    if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !fn)
        return set_err(PDL_ECUDA, "cuTensorMapEncodeTiled unavailable (%s)", cudaGetErrorString(e));
    g->encode = reinterpret_cast<pdlk::EncodeTiledFn>(fn);
    *out = g->encode;
    return PDL_OK;
}

const GreenApi *green_api() {
    static GreenApi a;
    static int state = 0;   // 0 untried, 1 ok, -1 unavailable
    if (state == 0) {
        auto get = [](const char *name, void **fn) {
            cudaDriverEntryPointQueryResult q;
            return cudaGetDriverEntryPoint(name, fn, cudaEnableDefault, &q) == cudaSuccess &&
                   q == cudaDriverEntryPointSuccess && *fn;
        };
        bool ok = get("cuDeviceGet", (void **)&a.dev_get) &&
                  get("cuDeviceGetDevResource", (void **)&a.get_resource) &&
                  get("cuDevSmResourceSplitByCount", (void **)&a.split) &&
                  get("cuDevResourceGenerateDesc", (void **)&a.gen_desc) &&
                  get("cuGreenCtxCreate", (void **)&a.create) &&
                  get("cuGreenCtxStreamCreate", (void **)&a.stream_create) &&
                  get("cuGreenCtxDestroy", (void **)&a.destroy);
        cudaGetLastError();
        state = ok ? 1 : -1;
    }
    return state == 1 ? &a : nullptr;
}

// A compute stream of the Worker: in its green context when it has an SM partition.
int worker_stream(const WorkerCtx &w, cudaStream_t *out, bool blocking) {
    if (w.gctx) {
        CUstream s = nullptr;
        if (green_api()->stream_create(&s, w.gctx, CU_STREAM_NON_BLOCKING, 0) != CUDA_SUCCESS)
            return set_err(PDL_ECUDA, "cuGreenCtxStreamCreate failed on device %d", w.device);
        *out = (cudaStream_t)s;
        return PDL_OK;
    }
    cudaError_t e = blocking ? cudaStreamCreate(out) : cudaStreamCreateWithFlags(out, cudaStreamNonBlocking);
    if (e != cudaSuccess) return set_err(PDL_ECUDA, "stream create failed: %s", cudaGetErrorString(e));
    return PDL_OK;
}

int gcd_int(int a, int b) { return b ? gcd_int(b, a % b) : a; }

// SM partitions (heterogeneous Workers emulated on one B200).
// Workers carrying the PDL property SM_LIMIT = n run on a green context of n
// SMs (rounded up to the partition granularity of 8 on sm_90+).  Workers that
// share a device get disjoint partitions: the device's SMs are split once into
// groups of u = gcd(n_i) SMs and Worker i takes n_i / u of them.  (A split's
// remainder cannot be split again -- CUDA_ERROR_INVALID_RESOURCE_CONFIGURATION
// on B200 -- and groups never straddle the GPC structure, so e.g. 8-SM groups
// cover only 120 of the 148 SMs; profiles/r01_green_probe.json.)
int make_partitions() {
    std::vector<int> devs;
    for (auto &w : g->workers)
        if (w.sm_limit > 0 && std::find(devs.begin(), devs.end(), w.device) == devs.end()) devs.push_back(w.device);
    for (int dev : devs) {
        const GreenApi *api = green_api();
        if (!api) return set_err(PDL_EUNSUPPORTED, "SM_LIMIT needs green contexts (driver API unavailable)");
        CUDA_TRY(cudaSetDevice(dev));
        CUDA_TRY(cudaFree(nullptr));   // primary context active before the green contexts retain it
        CUdevice cd;
        CUdevResource full;
        if (api->dev_get(&cd, dev) != CUDA_SUCCESS || api->get_resource(cd, &full, CU_DEV_RESOURCE_TYPE_SM) != CUDA_SUCCESS)
            return set_err(PDL_ECUDA, "cannot query the SM resource of device %d", dev);
        std::vector<WorkerCtx *> ws;
        int unit = 0, need = 0;
        for (auto &w : g->workers)
            if (w.device == dev && w.sm_limit > 0) {
                w.sm_limit = (w.sm_limit + 7) / 8 * 8;
                unit = gcd_int(unit, w.sm_limit);
                need += w.sm_limit;
                ws.push_back(&w);
            }
        if (need > (int)full.sm.smCount)
            return set_err(PDL_EINVAL, "SM_LIMIT of the Workers on device %d sums to %d SMs; the device has %u", dev, need,
                           full.sm.smCount);
        unsigned n = full.sm.smCount / unit;
        std::vector<CUdevResource> parts(n);
        CUdevResource rem;
        if (api->split(parts.data(), &n, &full, &rem, 0, unit) != CUDA_SUCCESS)
            return set_err(PDL_ECUDA, "cuDevSmResourceSplitByCount(%d) failed on device %d", unit, dev);
        if ((int)n * unit < need)
            return set_err(PDL_EINVAL,
                           "device %d yields only %u disjoint groups of %d SMs (gcd of the SM_LIMITs); %d SMs requested",
                           dev, n, unit, need);
        unsigned next = 0;
        for (WorkerCtx *w : ws) {
            const unsigned k = w->sm_limit / unit;
            CUdevResourceDesc desc;
            if (api->gen_desc(&desc, &parts[next], k) != CUDA_SUCCESS ||
                api->create(&w->gctx, desc, cd, CU_GREEN_CTX_DEFAULT_STREAM) != CUDA_SUCCESS)
                return set_err(PDL_ECUDA, "green context of %u SMs failed on device %d", k * unit, dev);
            unsigned sms = 0;
            for (unsigned i = 0; i < k; ++i) sms += parts[next + i].sm.smCount;
            next += k;
            w->sm_limit = (int)sms;
            if (w->own_stream && w->stream) cudaStreamDestroy(w->stream);
            int rc = worker_stream(*w, &w->stream, false);
            if (rc) return rc;
            w->own_stream = true;
            // runtime instantiation of the unfixed compute-unit property (L737-747)
            Property *q = g->model.prop_mut(w->pu, "MAX_COMPUTE_UNITS");
            if (q && !q->fixed) q->value = std::to_string(sms);
        }
    }
    return PDL_OK;
}

// Fill unfixed Worker properties from the bound device (L737-747 "Values for
// unfixed properties are marked to be editable by other tools ... later
// instantiation by a runtime"), adding the standard set when absent.
void fill_props(int pu, const cudaDeviceProp &p) {
    auto set = [&](const char *name, const std::string &val, const char *unit) {
        Property *q = g->model.prop_mut(pu, name);
        if (q) {
            if (!q->fixed) {
                q->value = val;
                q->unit = unit;
            }
            return;
        }
        Property np;
        np.name = name;
        np.key = norm_key(name);
        np.value = val;
        np.unit = unit;
        np.fixed = false;
        g->model.pus[pu].props.push_back(np);
    };
    set("DEVICE_NAME", p.name, "");
    set("MAX_COMPUTE_UNITS", std::to_string(p.multiProcessorCount), "");
    set("COMPUTE_CAPABILITY", std::to_string(p.major) + "." + std::to_string(p.minor), "");
    set("GLOBAL_MEM_SIZE", std::to_string((unsigned long long)p.totalGlobalMem), "B");
    set("LOCAL_MEM_SIZE", std::to_string((unsigned long long)p.sharedMemPerBlockOptin), "B");
    set("L2_CACHE_SIZE", std::to_string(p.l2CacheSize), "B");
    set("PCI_BUS_ID", std::to_string(p.pciBusID), "");
    // memory region of the Worker: HBM size
    auto &mrs = g->model.pus[pu].mrs;
    if (mrs.empty()) {
        MemoryRegion mr;
        mr.id = "hbm";
        mrs.push_back(mr);
    }
    bool found = false;
    for (auto &q : mrs[0].props)
        if (q.key == "SIZE") {
            found = true;
            if (!q.fixed) {
                q.value = std::to_string((unsigned long long)p.totalGlobalMem);
                q.unit = "B";
            }
        }
    if (!found) {
        Property np;
        np.name = "SIZE";
        np.key = "SIZE";
        np.value = std::to_string((unsigned long long)p.totalGlobalMem);
        np.unit = "B";
        np.fixed = false;
        mrs[0].props.push_back(np);
    }
}

int bind_devices() {
    std::vector<int> gw = g->model.all_gpu_workers();
    if (g->dry_run) {
        for (size_t i = 0; i < gw.size(); ++i) {
            if (g->nranks > 1 && (int)i != g->rank) continue;
            WorkerCtx w;
            w.pu = gw[i];
            w.gw = (int)i;
            w.device = -1;
            g->workers.push_back(w);
        }
        return PDL_OK;
    }
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess || ndev == 0)
        return set_err(PDL_ENOWORKER, "no CUDA device available (%s): no CPU fallback exists",
                       e == cudaSuccess ? "0 devices" : cudaGetErrorString(e));
    if (gw.empty()) return set_err(PDL_ENOWORKER, "descriptor has no Worker with ARCHITECTURE=gpu");
    int cur = 0;
    cudaGetDevice(&cur);
    std::vector<int> used(ndev, 0), limited(ndev, 0);
    for (size_t i = 0; i < gw.size(); ++i) {
        if (g->nranks > 1 && (int)i != g->rank) continue;
        int dev;
        const Property *ord = g->model.prop(gw[i], "DEVICE_ORDINAL");
        if (g->nranks > 1) dev = cur;   // rank mode: the process's current device
        else if (ord && !ord->value.empty()) dev = atoi(ord->value.c_str());
        else dev = (int)i;
        if (dev >= ndev) {
            if (!g->oversub)
                return set_err(PDL_ENOWORKER,
                               "descriptor names %zu gpu Workers but only %d CUDA device(s) exist "
                               "(set PDL_ALLOW_OVERSUBSCRIBE=1 to share devices)",
                               gw.size(), ndev);
            dev = dev % ndev;
        }
        // SM_LIMIT: the Worker owns a partition of the device's SMs (green context);
        // Workers that all carry it may share a device without oversubscription
        int sm_limit = 0;
        if (const Property *sl = g->model.prop(gw[i], "SM_LIMIT")) {
            char *end = nullptr;
            long v = std::strtol(sl->value.c_str(), &end, 10);
            if (!end || *end || v < 1)
                return set_err(PDL_EINVAL, "Worker %s: SM_LIMIT '%s' is not a positive integer",
                               g->model.pus[gw[i]].id.c_str(), sl->value.c_str());
            sm_limit = (int)v;
        }
        if (used[dev] && !g->oversub && !(sm_limit > 0 && limited[dev] == used[dev]))
            return set_err(PDL_ENOWORKER, "two Workers bound to device %d (set PDL_ALLOW_OVERSUBSCRIBE=1, "
                           "or give each an SM_LIMIT partition)", dev);
        used[dev]++;
        if (sm_limit > 0) limited[dev]++;
        cudaDeviceProp prop;
        CUDA_TRY(cudaGetDeviceProperties(&prop, dev));
        if (prop.major != 10)
            return set_err(PDL_ENOWORKER, "device %d is sm_%d%d; this build targets sm_100a (B200) only", dev,
                           prop.major, prop.minor);
        WorkerCtx w;
        w.pu = gw[i];
        w.gw = (int)i;
        w.device = dev;
        w.sm_limit = sm_limit;
        CUDA_TRY(cudaSetDevice(dev));
        // blocking stream: ordered with the legacy default stream callers often use
        CUDA_TRY(cudaStreamCreate(&w.stream));
        w.own_stream = true;
        CUDA_TRY(cudaEventCreate(&w.ev_k0));
        CUDA_TRY(cudaEventCreate(&w.ev_k1));
        g->model.pus[gw[i]].device = dev;
        fill_props(gw[i], prop);
        g->workers.push_back(w);
    }
    int rc = make_partitions();
    cudaSetDevice(cur);
    return rc;
}

void free_state() {
    if (!g) return;
    for (auto &w : g->workers) {
        if (w.device >= 0) cudaSetDevice(w.device);
        for (auto &b : w.buf)
            if (b.ptr) cudaFree(b.ptr);
        if (w.own_stream && w.stream) cudaStreamDestroy(w.stream);
        if (w.ev_k0) cudaEventDestroy(w.ev_k0);
        if (w.ev_k1) cudaEventDestroy(w.ev_k1);
        if (w.ev_legacy) cudaEventDestroy(w.ev_legacy);
        for (auto ev : w.kt_pool) cudaEventDestroy(ev);
        for (auto &ge : w.graphs) {
            if (ge.second.exec) cudaGraphExecDestroy(ge.second.exec);
            for (auto ev : ge.second.events) cudaEventDestroy(ev);
        }
        for (auto ev : w.ev_pool) cudaEventDestroy(ev);
        for (auto st : w.aux)
            if (st) cudaStreamDestroy(st);
        if (w.xs) cudaStreamDestroy(w.xs);
        for (auto ev : w.xev_pool) cudaEventDestroy(ev);
        for (cudaEvent_t ev : {w.ev_xdone, w.ev_bprep, w.ev_blast})
            if (ev) cudaEventDestroy(ev);
        if (w.gctx) green_api()->destroy(w.gctx);
    }
    if (g->dyn) {
        cudaSetDevice(g->dyn_dev);
        cudaFree(g->dyn);
    }
    delete g;
    g = nullptr;
}

int ensure_buf(WorkerCtx &w, int slot, size_t bytes, void **out) {
    DevBuf &b = w.buf[slot];
    if (b.bytes < bytes) {
        if (b.ptr) {
            cudaStreamSynchronize(w.stream);
            cudaFree(b.ptr);
            b.ptr = nullptr;
            b.bytes = 0;
        }
        cudaError_t e = cudaMalloc(&b.ptr, bytes);
        if (e != cudaSuccess) {
            cudaGetLastError();
            return set_err(PDL_ENOMEM, "cudaMalloc(%zu) on device %d failed: %s", bytes, w.device,
                           cudaGetErrorString(e));
        }
        b.bytes = bytes;
        ++w.buf_gen;   // captured graphs hold the old pointer
        if (slot == BUF_BHI || slot == BUF_BLO || slot == BUF_OZB || slot == BUF_OZE) w.bsig.valid = false;
    }
    *out = b.ptr;
    return PDL_OK;
}

// Where a pointer lives: -1 host (Master memory region), else device ordinal.
int locate(const void *p) {
    cudaPointerAttributes a;
    cudaError_t e = cudaPointerGetAttributes(&a, p);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return -1;
    }
    if (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) return a.device;
    return -1;
}

bool overlaps(const void *a, size_t an, const void *b, size_t bn) {
    uintptr_t x = (uintptr_t)a, y = (uintptr_t)b;
    return an && bn && x < y + bn && y < x + an;
}

}  // namespace pdlrt
