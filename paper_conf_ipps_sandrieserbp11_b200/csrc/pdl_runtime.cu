// pdl_runtime.cu -- the C ABI of libpdl.so (include/libpdl.h) and the task
// runtime behind it: descriptor loading, device binding, task queue, BLOCK
// mapping, operand staging along the interconnects, kernel launch, sync.
//
// PAPER.md SS IV-C step 3 "Output generation": "insertion of highly platform
// specific code for data-partitioning, transfer and task invocations.  The
// PDL allows us to derive data-transfer paths between memory-regions and
// communication between processing-units via the explicitly specified
// interconnect entity" (L1328-1341).  Here that step runs at run time:
// pdl_run partitions C (pdl_map.cpp), moves operand panels from the Master's
// memory region (host) to each Worker's memory region (HBM) over the Master->
// Worker interconnect (PCIe), and invokes the Worker's task variant (K1 for
// FP64, K3+K2 for FP32).  The Worker<->Worker exchange (NVLink) of the
// one-process-per-GPU mode runs in the Python runtime over torch.distributed.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <fstream>
#include <map>
#include <memory>
#include <sstream>
#include <string>
#include <vector>

#include <unistd.h>

#include "../../include/libpdl.h"
#include "kernels.h"
#include "pdl_model.hpp"
#include "pdl_xml.hpp"

using namespace pdl;

namespace {

thread_local std::string g_err;

int set_err(int code, const char *fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    if (getenv("PDL_LOG") && atoi(getenv("PDL_LOG")) > 0) fprintf(stderr, "[pdl] error %d: %s\n", code, buf);
    return code;
}

void logf(int level, const char *fmt, ...) {
    const char *e = getenv("PDL_LOG");
    if (!e || atoi(e) < level) return;
    va_list ap;
    va_start(ap, fmt);
    fprintf(stderr, "[pdl] ");
    vfprintf(stderr, fmt, ap);
    fprintf(stderr, "\n");
    va_end(ap);
}

bool env_on(const char *name) {
    const char *e = getenv(name);
    return e && *e && strcmp(e, "0") != 0;
}

// A library-owned device buffer in a Worker's memory region, reused across runs.
struct DevBuf {
    void *ptr = nullptr;
    size_t bytes = 0;
};

enum BufSlot { BUF_A = 0, BUF_B, BUF_C, BUF_AHI, BUF_ALO, BUF_BHI, BUF_BLO, BUF_OZA, BUF_OZB, BUF_OZE, BUF_OZR, BUF_COUNT };

struct WorkerCtx {
    int pu = -1;         // PU instance index in the model
    int gw = -1;         // index in the default group order
    int device = -1;
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    // SM partition (PDL Worker property SM_LIMIT): a green context owning
    // sm_limit SMs of the device; the Worker's compute streams belong to it
    int sm_limit = 0;
    CUgreenCtx gctx = nullptr;
    cudaEvent_t ev_legacy = nullptr;   // orders the non-blocking green stream with the legacy stream
    DevBuf buf[BUF_COUNT];
    cudaEvent_t ev_k0 = nullptr, ev_k1 = nullptr;   // around the dominant kernel of the last task
    int launches = 0;                               // kernels launched in the last run
    bool timed = false;
    // event pairs around every dominant-kernel launch since the last pdl_kernel_times():
    // kt_list holds the pairs in launch order; plain launches take events from kt_pool
    // (kt_used of them in use), graph replays append the events their graph records
    std::vector<cudaEvent_t> kt_pool;
    size_t kt_used = 0;
    std::vector<std::pair<cudaEvent_t, cudaEvent_t>> kt_list;
    cudaEvent_t kt_open = nullptr;   // start event of the launch being bracketed
    // CUDA graphs of repeated tasks (PDL_TASK_GRAPH / PDL_GRAPH=1): signature -> graph
    struct GraphEntry {
        cudaGraphExec_t exec = nullptr;
        std::vector<cudaEvent_t> events;                              // owned; recorded by the graph
        std::vector<std::pair<cudaEvent_t, cudaEvent_t>> kt_pairs;
        int launches = 0;
        bool timed = false;
    };
    std::map<std::string, GraphEntry> graphs;
    std::map<std::string, int> graph_seen;   // signatures run once (captured on the next run)
    int buf_gen = 0;                         // bumped when a buffer is reallocated (graphs go stale)
    bool capturing = false;
    long long graph_replays = 0;
    // pipelined staging: copy-in, copy-out, second compute stream; reusable events
    cudaStream_t aux[3] = {nullptr, nullptr, nullptr};
    std::vector<cudaEvent_t> ev_pool;
    // identity of the B operand whose prepared form (FP32 split / Ozaki slices)
    // sits in the B-side buffers (PDL_TASK_REUSE_B)
    struct BSig {
        bool valid = false;
        const void *B = nullptr;
        int64_t ldb = 0, K = 0, cols = 0;
        int dtype = -1, oz = 0, S = 0, rn = 0;
        bool operator==(const BSig &o) const {
            return valid && o.valid && B == o.B && ldb == o.ldb && K == o.K && cols == o.cols && dtype == o.dtype &&
                   oz == o.oz && S == o.S && rn == o.rn;
        }
    } bsig;
};

constexpr size_t kMaxKernelTimes = 4096;

// Record the start / end of a dominant-kernel launch on the worker's stream.  While a
// graph is being captured the records are external event-record nodes of the graph
// and the events move to its entry (they must not be reused by plain launches).
int kt_mark(WorkerCtx &w, bool start, cudaStream_t st) {
    auto record = [&](cudaEvent_t ev) {
        return w.capturing ? cudaEventRecordWithFlags(ev, st, cudaEventRecordExternal) : cudaEventRecord(ev, st);
    };
    cudaEvent_t &last = start ? w.ev_k0 : w.ev_k1;
    if (record(last) != cudaSuccess) return PDL_ECUDA;
    if (w.kt_list.size() >= kMaxKernelTimes) return PDL_OK;
    if (w.kt_used >= w.kt_pool.size()) {
        cudaEvent_t ev;
        if (cudaEventCreate(&ev) != cudaSuccess) return PDL_ECUDA;
        w.kt_pool.push_back(ev);
    }
    cudaEvent_t ev = w.kt_pool[w.kt_used++];
    if (record(ev) != cudaSuccess) return PDL_ECUDA;
    if (start) {
        w.kt_open = ev;
    } else {
        w.kt_list.emplace_back(w.kt_open, ev);
    }
    return PDL_OK;
}

struct Task {
    int dtype;
    const void *A;
    int64_t lda;
    const void *B;
    int64_t ldb;
    void *C;
    int64_t ldc;
    int64_t M, N, K, tile;
    bool has_group;
    std::string group;
    unsigned flags;
    DistSpec dist;
};

struct State {
    bool loaded = false;
    bool dry_run = false;
    bool oversub = false;
    int rank = 0, nranks = 1;
    Model model;
    std::vector<WorkerCtx> workers;   // one per bound gpu Worker (this process's)
    std::vector<Task> queue;
    std::string plan_json = "[]";
    pdlk::EncodeTiledFn encode = nullptr;
    int last_launches = 0;
    long long total_launches = 0;   // every kernel launched since pdl_load
    // DYNAMIC distribution: [0] next tile, [1 + i] tiles claimed by group Worker i
    int *dyn = nullptr;
    int dyn_dev = -1;
    int dyn_n = 0;                  // Workers of the last DYNAMIC task
    long long dyn_tiles = 0;        // its tile count
    std::string dyn_kernel;
};

State *g = nullptr;

const char *kVersion =
    "libpdl 0.2.0 (sm_100a: K1 FP64 DMMA+TMA, K2 3xTF32 tcgen05 CTA-pair, K4 FP64 Ozaki on INT8 tcgen05)";

std::string read_descriptor(const char *d, bool *ok) {
    *ok = true;
    const char *p = d;
    while (*p == ' ' || *p == '\t' || *p == '\n' || *p == '\r') ++p;
    if (*p == '<') return std::string(d);
    std::ifstream f(d, std::ios::binary);
    if (!f) {
        *ok = false;
        return "";
    }
    std::stringstream ss;
    ss << f.rdbuf();
    return ss.str();
}

#define CUDA_TRY(call)                                                                                   \
    do {                                                                                                 \
        cudaError_t _e = (call);                                                                         \
        if (_e != cudaSuccess) return set_err(PDL_ECUDA, "%s failed: %s", #call, cudaGetErrorString(_e)); \
    } while (0)

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

// Driver entry points for green contexts (SM partitions of one device), loaded
// through the runtime so libpdl does not link libcuda directly.
struct GreenApi {
    CUresult (*dev_get)(CUdevice *, int) = nullptr;
    CUresult (*get_resource)(CUdevice, CUdevResource *, CUdevResourceType) = nullptr;
    CUresult (*split)(CUdevResource *, unsigned *, const CUdevResource *, CUdevResource *, unsigned,
                      unsigned) = nullptr;
    CUresult (*gen_desc)(CUdevResourceDesc *, CUdevResource *, unsigned) = nullptr;
    CUresult (*create)(CUgreenCtx *, CUdevResourceDesc, CUdevice, unsigned) = nullptr;
    CUresult (*stream_create)(CUstream *, CUgreenCtx, unsigned, int) = nullptr;
    CUresult (*destroy)(CUgreenCtx) = nullptr;
};

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

int64_t round_up(int64_t x, int64_t m) { return (x + m - 1) / m * m; }

// ---- pipelined execution of one Worker rectangle -------------------------
//
// The rectangle is cut into RB row bands x CP column panels of whole task
// tiles.  Operands that live outside the Worker's memory region (host =
// Master MR, or another device) are moved per band / panel on a copy-in
// stream, each sub-rectangle's kernel waits only for its own A band and B
// panel, and results leave on a copy-out stream as soon as their kernel ends,
// so PCIe traffic overlaps the tile kernels (L1336-1341: "data-transfer paths
// between memory-regions ... via the explicitly specified interconnect").
// Sub-rectangle kernels alternate between two compute streams so one
// kernel's last wave overlaps the next.  Device-resident operands take a
// single launch (RB = CP = 1).  Every sub-kernel computes the same per-element
// K order, so C is bitwise identical for any cut (R14).

cudaEvent_t ev_get(WorkerCtx &w, size_t &next) {
    if (next >= w.ev_pool.size()) {
        cudaEvent_t e = nullptr;
        if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return nullptr;
        w.ev_pool.push_back(e);
    }
    return w.ev_pool[next++];
}

int ensure_aux(WorkerCtx &w) {
    // copy-in, copy-out: plain streams; aux[2] computes, so it joins the Worker's partition
    for (int i = 0; i < 2; ++i)
        if (!w.aux[i]) CUDA_TRY(cudaStreamCreateWithFlags(&w.aux[i], cudaStreamNonBlocking));
    if (!w.aux[2]) return worker_stream(w, &w.aux[2], false);
    return PDL_OK;
}

// Task variant of a Worker (task repository + static pre-selection, L1307-1326):
//   FP64: PDL property DGEMM_VARIANT ("dmma" default | "ozaki"), OZAKI_SLICES (default 6)
//   FP32: PDL property SGEMM_VARIANT ("3xtf32" default | "ozaki"), OZAKI_SLICES_F32 (default 3)
// OZAKI_ROUNDING ("nearest" default | "trunc") for both; env PDL_<NAME> overrides
// the descriptor (tests, bench).
bool worker_ozaki(const WorkerCtx &w, bool f64, int *slices, int *rn) {
    const char *vname = f64 ? "DGEMM_VARIANT" : "SGEMM_VARIANT";
    const char *sname = f64 ? "OZAKI_SLICES" : "OZAKI_SLICES_F32";
    std::string v;
    if (const char *e = getenv((std::string("PDL_") + vname).c_str())) v = e;
    else if (const Property *p = g->model.prop(w.pu, vname)) v = p->value;
    if (lower(trim(v)) != "ozaki") return false;
    // Defaults from the measured accuracy sweeps (profiles/r01_ozaki_accuracy*.txt):
    // FP64 -- round-to-nearest slices, S = 6 -> max scaled error 3.7e-14 at K = 16384
    // (truncation needs S = 7 for 3.0e-14; truncation S = 6 gives 1.6e-12);
    // FP32 -- S = 3 (8+7+7 bits) -> max 3.3e-7 (K = 256) .. 4.3e-8 (K = 16384), 1e-5 bar.
    int s = f64 ? 6 : 3;
    if (const char *e = getenv((std::string("PDL_") + sname).c_str())) s = atoi(e);
    else if (const Property *p = g->model.prop(w.pu, sname)) s = atoi(p->value.c_str());
    *slices = std::max(2, std::min(8, s));
    // OZAKI_ROUNDING: "nearest" (default) | "trunc"
    std::string r;
    if (const char *e = getenv("PDL_OZAKI_ROUNDING")) r = e;
    else if (const Property *p = g->model.prop(w.pu, "OZAKI_ROUNDING")) r = p->value;
    *rn = lower(trim(r)) == "trunc" ? 0 : 1;
    return true;
}

// FP64 variant "ozaki2" (Ozaki scheme II, K6/K7): DGEMM_VARIANT = "ozaki2";
// OZAKI2_MODULI (default 0 = the fewest giving OZAKI2_BITS), OZAKI2_BITS (default
// 43: |scaling error| <= 2^-44 of the row / column max; max scaled error at C4
// in profiles/r01_ozaki2_accuracy.txt).  env PDL_<NAME> overrides.
bool worker_ozaki2(const WorkerCtx &w, int *nmod, int *bits) {
    std::string v;
    if (const char *e = getenv("PDL_DGEMM_VARIANT")) v = e;
    else if (const Property *p = g->model.prop(w.pu, "DGEMM_VARIANT")) v = p->value;
    if (lower(trim(v)) != "ozaki2") return false;
    *nmod = 0;
    *bits = 43;
    if (const char *e = getenv("PDL_OZAKI2_MODULI")) *nmod = atoi(e);
    else if (const Property *p = g->model.prop(w.pu, "OZAKI2_MODULI")) *nmod = atoi(p->value.c_str());
    if (const char *e = getenv("PDL_OZAKI2_BITS")) *bits = atoi(e);
    else if (const Property *p = g->model.prop(w.pu, "OZAKI2_BITS")) *bits = atoi(p->value.c_str());
    *bits = std::max(8, std::min(52, *bits));
    return true;
}

bool worker_sgemm_ozaki2(const WorkerCtx &w) {
    std::string v;
    if (const char *e = getenv("PDL_SGEMM_VARIANT")) v = e;
    else if (const Property *p = g->model.prop(w.pu, "SGEMM_VARIANT")) v = p->value;
    return lower(trim(v)) == "ozaki2";
}

int run_rect(WorkerCtx &w, const Task &t, const void *A, const void *B, void *C, int64_t rows, int64_t cols) {
    if (rows <= 0 || cols <= 0) return PDL_OK;
    CUDA_TRY(cudaSetDevice(w.device));
    const int es = t.dtype == PDL_F64 ? 8 : 4;
    const bool f64 = t.dtype == PDL_F64;
    const int64_t K = t.K;
    const int64_t pe = 16 / es;   // elements per 16 bytes

    // Where the operands live and whether they must be staged into this Worker's MR.
    const bool a_st = K > 0 && (locate(A) != w.device || (f64 && (((uintptr_t)A % 16) || (t.lda * es) % 16)));
    const bool b_st = K > 0 && (locate(B) != w.device || (f64 && (((uintptr_t)B % 16) || (t.ldb * es) % 16)));
    const bool c_st = locate(C) != w.device;

    // Cut: row bands / column panels aligned to 128 (a K1/K2 tile edge).
    int RB = 1, CP = 1;
    const char *pe_env = getenv("PDL_PIPELINE");
    const bool force = pe_env && !strcmp(pe_env, "force");
    const bool off = pe_env && !strcmp(pe_env, "0");
    const double flops = 2.0 * rows * cols * (double)K;
    if (!off && (a_st || b_st || c_st) && K > 0 && (force || flops >= 2e11)) {
        // first sub-kernel waits for one A band + one B panel only: smaller
        // panels start compute sooner; >= 2048 x 4096 keeps each launch >= 1.7 waves
        RB = (int)std::min<int64_t>(8, std::max<int64_t>(1, rows / 2048));
        CP = (int)std::min<int64_t>(4, std::max<int64_t>(1, cols / 4096));
        if (force) {
            RB = (int)std::min<int64_t>(4, std::max<int64_t>(1, (rows + 127) / 128));
            CP = (int)std::min<int64_t>(2, std::max<int64_t>(1, (cols + 127) / 128));
        }
    }
    std::vector<int64_t> rb(RB + 1), cp(CP + 1);
    for (int i = 0; i <= RB; ++i) rb[i] = std::min<int64_t>(rows, round_up((int64_t)i * rows / RB, 128));
    for (int j = 0; j <= CP; ++j) cp[j] = std::min<int64_t>(cols, round_up((int64_t)j * cols / CP, 128));
    rb[RB] = rows;
    cp[CP] = cols;
    const bool piped = RB * CP > 1;
    int rc;
    if (piped && (rc = ensure_aux(w))) return rc;
    cudaStream_t s_in = piped ? w.aux[0] : w.stream, s_out = piped ? w.aux[1] : w.stream;
    cudaStream_t s_cmp[2] = {w.stream, piped ? w.aux[2] : w.stream};
    size_t evn = 0;
    cudaEvent_t ev_start = ev_get(w, evn);
    if (!ev_start) return set_err(PDL_ECUDA, "event create failed");
    if (piped) {
        // side streams start after everything already queued on the Worker stream
        CUDA_TRY(cudaEventRecord(ev_start, w.stream));
        for (int i = 0; i < 3; ++i) CUDA_TRY(cudaStreamWaitEvent(w.aux[i], ev_start, 0));
    }

    // Device views of the operands.
    const char *Ad = (const char *)A, *Bd = (const char *)B;
    char *Cd = (char *)C;
    int64_t lda = t.lda, ldb = t.ldb, ldcd = t.ldc;
    void *p;
    if (a_st) {
        lda = round_up(std::max<int64_t>(K, 1), pe);
        if ((rc = ensure_buf(w, BUF_A, (size_t)(lda * rows * es), &p))) return rc;
        Ad = (const char *)p;
    }
    if (b_st) {
        ldb = round_up(cols, pe);
        if ((rc = ensure_buf(w, BUF_B, (size_t)(ldb * K * es), &p))) return rc;
        Bd = (const char *)p;
    }
    if (c_st) {
        ldcd = round_up(cols, pe);
        if ((rc = ensure_buf(w, BUF_C, (size_t)(ldcd * rows * es), &p))) return rc;
        Cd = (char *)p;
    }
    // Task variant of this Worker, pre-selected from its PDL properties (task
    // repository + static pre-selection, L1307-1326): FP64 K1 (DMMA) or K4
    // (Ozaki), FP32 K3+K2 (3xTF32) or K4 (Ozaki).
    int oz_slices = 0;
    int oz_rn = 0;
    int oz2_nmod = 0, oz2_bits = 0;
    if (!f64 && K > 0 && worker_sgemm_ozaki2(w))
        return set_err(PDL_EUNSUPPORTED, "SGEMM_VARIANT ozaki2: Ozaki scheme II is an FP64 variant (use ozaki)");
    const bool ozaki2 = K > 0 && f64 && worker_ozaki2(w, &oz2_nmod, &oz2_bits);
    const bool ozaki = K > 0 && !ozaki2 && worker_ozaki(w, f64, &oz_slices, &oz_rn);
    // FP32 split buffers (K-major hi/lo of A rows and of B^T rows)
    const int64_t Kp = round_up(std::max<int64_t>(K, 1), pdlk::K2_BK);
    float *ahi = nullptr, *alo = nullptr, *bhi = nullptr, *blo = nullptr;
    if (!f64 && K > 0 && !ozaki) {
        if ((rc = ensure_buf(w, BUF_AHI, (size_t)(rows * Kp * 4), &p))) return rc;
        ahi = (float *)p;
        if ((rc = ensure_buf(w, BUF_ALO, (size_t)(rows * Kp * 4), &p))) return rc;
        alo = (float *)p;
        if ((rc = ensure_buf(w, BUF_BHI, (size_t)(cols * Kp * 4), &p))) return rc;
        bhi = (float *)p;
        if ((rc = ensure_buf(w, BUF_BLO, (size_t)(cols * Kp * 4), &p))) return rc;
        blo = (float *)p;
    }
    pdlk::EncodeTiledFn enc = nullptr;
    if (K > 0 && (rc = get_encoder(&enc))) return rc;
    const char *k2v = getenv("PDL_K2");
    const bool k2_1sm = k2v && !strcmp(k2v, "1sm");

    pdlk::OzakiLayout OL;
    int8_t *a8 = nullptr, *b8 = nullptr;
    int *oz_ea = nullptr, *oz_fb = nullptr;
    unsigned long long *oz_bmax = nullptr;
    if (ozaki) {
        OL = pdlk::ozaki_layout(rows, cols, K, oz_slices);
        OL.rn = oz_rn;
        if ((rc = ensure_buf(w, BUF_OZA, OL.a8_bytes, &p))) return rc;
        a8 = (int8_t *)p;
        if ((rc = ensure_buf(w, BUF_OZB, OL.b8_bytes, &p))) return rc;
        b8 = (int8_t *)p;
        const size_t eb = (size_t)round_up(rows, 2) * 4 + (size_t)round_up(cols, 2) * 4 + (size_t)cols * 8;
        if ((rc = ensure_buf(w, BUF_OZE, eb, &p))) return rc;
        // [bmax: cols u64][fb: cols int][ea: rows int] -- the B-side part does not
        // move with `rows`, so a prepared B survives row-chunk tasks (REUSE_B)
        oz_bmax = (unsigned long long *)p;
        oz_fb = (int *)(oz_bmax + cols);
        oz_ea = oz_fb + round_up(cols, 2);
    }

    pdlk::Ozaki2Plan P2;
    uint8_t *oz2_R = nullptr;
    int64_t oz2_ldr = 0, oz2_plane = 0;
    if (ozaki2) {
        P2 = pdlk::ozaki2_plan(rows, cols, K, oz2_nmod, oz2_bits);
        if ((rc = ensure_buf(w, BUF_OZA, P2.a8_bytes, &p))) return rc;
        a8 = (int8_t *)p;
        if ((rc = ensure_buf(w, BUF_OZB, P2.b8_bytes, &p))) return rc;
        b8 = (int8_t *)p;
        const size_t eb = (size_t)round_up(rows, 2) * 4 + (size_t)round_up(cols, 2) * 4 + (size_t)cols * 8;
        if ((rc = ensure_buf(w, BUF_OZE, eb, &p))) return rc;
        oz_bmax = (unsigned long long *)p;
        oz_fb = (int *)(oz_bmax + cols);
        oz_ea = oz_fb + round_up(cols, 2);
        oz2_ldr = round_up(cols, 16);
        oz2_plane = oz2_ldr * rows;
        if ((rc = ensure_buf(w, BUF_OZR, (size_t)(oz2_plane * P2.n * P2.nch), &p))) return rc;
        oz2_R = (uint8_t *)p;
    }

    // B prepared by a previous task of this Worker (PDL_TASK_REUSE_B)?
    WorkerCtx::BSig want;
    want.valid = true;
    want.B = B;
    want.ldb = t.ldb;
    want.K = K;
    want.cols = cols;
    want.dtype = t.dtype;
    want.oz = ozaki ? 1 : ozaki2 ? 2 : 0;
    want.S = ozaki ? OL.S : ozaki2 ? P2.n : 0;
    want.rn = ozaki ? OL.rn : ozaki2 ? P2.p : 0;
    const bool prep_b = K > 0 && (ozaki || ozaki2 || !f64);
    const bool b_ready = prep_b && (t.flags & PDL_TASK_REUSE_B) && !piped && !b_st && w.bsig == want;

    std::vector<cudaEvent_t> ev_a(RB, nullptr), ev_b(CP, nullptr), ev_sa(RB, nullptr), ev_sb(CP, nullptr);
    cudaEvent_t ev_last_out = nullptr, ev_last_cmp1 = nullptr;
    int launch_idx = 0;
    // Sub-rectangle order: the inner loop runs over the operand whose chunks are
    // smaller, so while the first outer chunk computes, the inner chunks stream in
    // at least as fast as the kernels consume them and only one A band + one B
    // panel precede the first kernel (C4 host-staged: A bands of 2048 x K = 268 MB
    // inner, B panels of K x 4096 = 537 MB outer).  Copies and the K3 / K5
    // operand preparation happen at a chunk's first use.
    const bool col_outer = piped && (rows / RB) * K <= K * (cols / CP);
    std::vector<char> a_in(RB, 0), b_in(CP, 0), a_prep(RB, 0), b_prep(CP, 0);
    const int n_outer = col_outer ? CP : RB, n_inner = col_outer ? RB : CP;
    for (int o = 0; o < n_outer; ++o) {
      for (int q = 0; q < n_inner; ++q) {
        const int i = col_outer ? q : o, j = col_outer ? o : q;
        const int64_t r0 = rb[i], nr = rb[i + 1] - rb[i];
        const int64_t c0 = cp[j], nc = cp[j + 1] - cp[j];
        if (nr <= 0 || nc <= 0) continue;
        if (a_st && !a_in[i]) {
            a_in[i] = 1;
            cudaError_t e = cudaMemcpy2DAsync(const_cast<char *>(Ad) + (size_t)(r0 * lda) * es, (size_t)(lda * es),
                                              (const char *)A + (size_t)(r0 * t.lda) * es, (size_t)(t.lda * es),
                                              (size_t)(K * es), (size_t)nr, cudaMemcpyDefault, s_in);
            if (e != cudaSuccess) return set_err(PDL_ECUDA, "A staging copy failed: %s", cudaGetErrorString(e));
            if (piped) {
                ev_a[i] = ev_get(w, evn);
                CUDA_TRY(cudaEventRecord(ev_a[i], s_in));
            }
        }
        {
            if (b_st && !b_in[j]) {
                b_in[j] = 1;
                cudaError_t e = cudaMemcpy2DAsync(const_cast<char *>(Bd) + (size_t)c0 * es, (size_t)(ldb * es),
                                                  (const char *)B + (size_t)c0 * es, (size_t)(t.ldb * es),
                                                  (size_t)(nc * es), (size_t)K, cudaMemcpyDefault, s_in);
                if (e != cudaSuccess) return set_err(PDL_ECUDA, "B staging copy failed: %s", cudaGetErrorString(e));
                if (piped) {
                    ev_b[j] = ev_get(w, evn);
                    CUDA_TRY(cudaEventRecord(ev_b[j], s_in));
                }
            }
            cudaStream_t cs = s_cmp[launch_idx & 1];
            if (piped) {
                if (ev_a[i]) CUDA_TRY(cudaStreamWaitEvent(cs, ev_a[i], 0));
                if (ev_b[j]) CUDA_TRY(cudaStreamWaitEvent(cs, ev_b[j], 0));
            }
            char *Cs = Cd + (size_t)(r0 * ldcd + c0) * es;
            cudaError_t e = cudaSuccess;
            if (K == 0) {
                e = cudaMemset2DAsync(Cs, (size_t)(ldcd * es), 0, (size_t)(nc * es), (size_t)nr, cs);
            } else if (ozaki2) {
                // K7 scaling + residues of this band / panel once, shared by both compute streams
                if (!a_prep[i]) {
                    a_prep[i] = 1;
                    e = pdlk::launch_ozaki2_split_a((const double *)(Ad + (size_t)(r0 * lda) * es), lda, nr, K, P2,
                                                    a8 + r0 * P2.ld8, oz_ea + r0, cs);
                    w.launches += 1;
                    if (piped) {
                        ev_sa[i] = ev_get(w, evn);
                        CUDA_TRY(cudaEventRecord(ev_sa[i], cs));
                    }
                } else if (ev_sa[i]) {
                    CUDA_TRY(cudaStreamWaitEvent(cs, ev_sa[i], 0));
                }
                if (e == cudaSuccess && !b_prep[j] && !b_ready) {
                    b_prep[j] = 1;
                    e = pdlk::launch_ozaki2_split_b((const double *)(Bd + (size_t)c0 * es), ldb, K, nc, P2,
                                                    b8 + c0 * P2.ld8, oz_fb + c0, oz_bmax + c0, cs);
                    w.launches += 2;
                    if (piped) {
                        ev_sb[j] = ev_get(w, evn);
                        CUDA_TRY(cudaEventRecord(ev_sb[j], cs));
                    }
                } else if (ev_sb[j]) {
                    CUDA_TRY(cudaStreamWaitEvent(cs, ev_sb[j], 0));
                }
                if (e != cudaSuccess) return set_err(PDL_ECUDA, "K7 residue launch failed: %s", cudaGetErrorString(e));
                if (kt_mark(w, true, cs)) return set_err(PDL_ECUDA, "event record failed");
                int nl = 0;
                uint8_t *Rs = oz2_R + r0 * oz2_ldr + c0;
                e = pdlk::launch_ozaki2_gemm(enc, a8 + r0 * P2.ld8, b8 + c0 * P2.ld8, P2, Rs, oz2_ldr, oz2_plane, nr,
                                             nc, cs, &nl);
                if (e == cudaSuccess)
                    e = pdlk::launch_ozaki2_reconstruct(Rs, oz2_ldr, oz2_plane, oz_ea + r0, oz_fb + c0, P2,
                                                        (double *)Cs, ldcd, nr, nc, cs);
                if (e == cudaSuccess && kt_mark(w, false, cs)) return set_err(PDL_ECUDA, "event record failed");
                w.launches += nl + 1;
            } else if (ozaki) {
                // K5 slicing of this band / panel once, shared by both compute streams
                if (!a_prep[i]) {
                    a_prep[i] = 1;
                    const char *Ab = Ad + (size_t)(r0 * lda) * es;
                    e = f64 ? pdlk::launch_ozaki_split_a((const double *)Ab, lda, nr, K, OL, a8 + r0 * OL.ld8,
                                                         oz_ea + r0, cs)
                            : pdlk::launch_ozaki_split_a((const float *)Ab, lda, nr, K, OL, a8 + r0 * OL.ld8,
                                                         oz_ea + r0, cs);
                    w.launches += 1;
                    if (piped) {
                        ev_sa[i] = ev_get(w, evn);
                        CUDA_TRY(cudaEventRecord(ev_sa[i], cs));
                    }
                } else if (ev_sa[i]) {
                    CUDA_TRY(cudaStreamWaitEvent(cs, ev_sa[i], 0));
                }
                if (e == cudaSuccess && !b_prep[j] && !b_ready) {
                    b_prep[j] = 1;
                    const char *Bp = Bd + (size_t)c0 * es;
                    e = f64 ? pdlk::launch_ozaki_split_b((const double *)Bp, ldb, K, nc, OL, b8 + c0 * OL.ld8,
                                                         oz_fb + c0, oz_bmax + c0, cs)
                            : pdlk::launch_ozaki_split_b((const float *)Bp, ldb, K, nc, OL, b8 + c0 * OL.ld8,
                                                         oz_fb + c0, oz_bmax + c0, cs);
                    w.launches += 2;
                    if (piped) {
                        ev_sb[j] = ev_get(w, evn);
                        CUDA_TRY(cudaEventRecord(ev_sb[j], cs));
                    }
                } else if (ev_sb[j]) {
                    CUDA_TRY(cudaStreamWaitEvent(cs, ev_sb[j], 0));
                }
                if (e != cudaSuccess) return set_err(PDL_ECUDA, "K5 slicing launch failed: %s", cudaGetErrorString(e));
                if (kt_mark(w, true, cs)) return set_err(PDL_ECUDA, "event record failed");
                int nl = 0;
                e = f64 ? pdlk::launch_ozaki_gemm(enc, a8 + r0 * OL.ld8, b8 + c0 * OL.ld8, oz_ea + r0, oz_fb + c0,
                                                  OL, (double *)Cs, ldcd, nr, nc, cs, &nl)
                        : pdlk::launch_ozaki_gemm(enc, a8 + r0 * OL.ld8, b8 + c0 * OL.ld8, oz_ea + r0, oz_fb + c0,
                                                  OL, (float *)Cs, ldcd, nr, nc, cs, &nl);
                if (e == cudaSuccess && kt_mark(w, false, cs)) return set_err(PDL_ECUDA, "event record failed");
                w.launches += nl;
            } else if (f64) {
                if (kt_mark(w, true, cs)) return set_err(PDL_ECUDA, "event record failed");
                e = pdlk::launch_dgemm_k1(enc, (const double *)(Ad + (size_t)(r0 * lda) * es), lda,
                                          (const double *)(Bd + (size_t)c0 * es), ldb, (double *)Cs, ldcd, nr, nc, K,
                                          cs);
                if (e == cudaSuccess && kt_mark(w, false, cs)) return set_err(PDL_ECUDA, "event record failed");
                w.launches += 1;
            } else {
                // K3 split of this band / panel once, shared by both compute streams
                if (!a_prep[i]) {
                    a_prep[i] = 1;
                    e = pdlk::launch_split_rows((const float *)(Ad + (size_t)(r0 * lda) * es), lda, nr, K,
                                                ahi + r0 * Kp, alo + r0 * Kp, Kp, cs);
                    w.launches += 1;
                    if (piped) {
                        ev_sa[i] = ev_get(w, evn);
                        CUDA_TRY(cudaEventRecord(ev_sa[i], cs));
                    }
                } else if (ev_sa[i]) {
                    CUDA_TRY(cudaStreamWaitEvent(cs, ev_sa[i], 0));
                }
                if (e == cudaSuccess && !b_prep[j] && !b_ready) {
                    b_prep[j] = 1;
                    e = pdlk::launch_split_cols_t((const float *)(Bd + (size_t)c0 * es), ldb, K, nc, bhi + c0 * Kp,
                                                  blo + c0 * Kp, Kp, cs);
                    w.launches += 1;
                    if (piped) {
                        ev_sb[j] = ev_get(w, evn);
                        CUDA_TRY(cudaEventRecord(ev_sb[j], cs));
                    }
                } else if (ev_sb[j]) {
                    CUDA_TRY(cudaStreamWaitEvent(cs, ev_sb[j], 0));
                }
                if (e != cudaSuccess) return set_err(PDL_ECUDA, "K3 split launch failed: %s", cudaGetErrorString(e));
                if (kt_mark(w, true, cs)) return set_err(PDL_ECUDA, "event record failed");
                if (k2_1sm)
                    e = pdlk::launch_gemm_3xtf32(enc, ahi + r0 * Kp, alo + r0 * Kp, bhi + c0 * Kp, blo + c0 * Kp, Kp,
                                                 (float *)Cs, ldcd, nr, nc, cs);
                else
                    e = pdlk::launch_gemm_3xtf32_2sm(enc, ahi + r0 * Kp, alo + r0 * Kp, bhi + c0 * Kp, blo + c0 * Kp,
                                                     Kp, (float *)Cs, ldcd, nr, nc, cs);
                if (e == cudaSuccess && kt_mark(w, false, cs)) return set_err(PDL_ECUDA, "event record failed");
                w.launches += 1;
            }
            if (e != cudaSuccess) return set_err(PDL_ECUDA, "tile kernel launch failed: %s", cudaGetErrorString(e));
            w.timed = true;
            if (piped && (launch_idx & 1)) {
                ev_last_cmp1 = ev_get(w, evn);
                CUDA_TRY(cudaEventRecord(ev_last_cmp1, cs));
            }
            if (c_st) {
                if (piped) {
                    cudaEvent_t ek = ev_get(w, evn);
                    CUDA_TRY(cudaEventRecord(ek, cs));
                    CUDA_TRY(cudaStreamWaitEvent(s_out, ek, 0));
                }
                e = cudaMemcpy2DAsync((char *)C + (size_t)(r0 * t.ldc + c0) * es, (size_t)(t.ldc * es), Cs,
                                      (size_t)(ldcd * es), (size_t)(nc * es), (size_t)nr, cudaMemcpyDefault, s_out);
                if (e != cudaSuccess) return set_err(PDL_ECUDA, "result gather copy failed: %s", cudaGetErrorString(e));
            }
            ++launch_idx;
        }
      }
    }
    if (prep_b) {
        // the B-side buffers now hold this task's prepared B (whole panel only when unpiped)
        w.bsig = want;
        w.bsig.valid = !piped && !b_st;
    }
    if (piped) {
        // join: the Worker stream completes after every side stream's work
        ev_last_out = ev_get(w, evn);
        CUDA_TRY(cudaEventRecord(ev_last_out, s_out));
        CUDA_TRY(cudaStreamWaitEvent(w.stream, ev_last_out, 0));
        if (ev_last_cmp1) CUDA_TRY(cudaStreamWaitEvent(w.stream, ev_last_cmp1, 0));
        cudaEvent_t ein = ev_get(w, evn);
        CUDA_TRY(cudaEventRecord(ein, s_in));
        CUDA_TRY(cudaStreamWaitEvent(w.stream, ein, 0));
    }
    return PDL_OK;
}

// ---- DYNAMIC distribution (dynamic schedulers, L1556-1562) ----
//
// Every Worker of the group launches the whole tile grid of its task variant
// (K1 128 x 128 tiles, K2 256 x 256 pair tiles); each CTA (pair) claims the next
// raster tile from one counter in the first Worker's memory region (system-scope
// atomics; NVLink peer memory for Workers on other devices), so a faster Worker
// (more SMs, higher clocks, less competing work) takes more tiles and all
// finish together, without a speed model.  A tile's computation is the static
// one, so C is bitwise the BLOCK result (R14).  Operands are used in place when
// resident on the Worker's device, else staged whole into its memory region.
// C is written in place by every Worker (peer access when it lives on another
// device) or, for a host C, into a staging buffer on the first Worker and copied
// out once every Worker is done.
constexpr int kMaxDynWorkers = 64;

int enable_peer(int from, int to) {
    if (from == to) return PDL_OK;
    int can = 0;
    CUDA_TRY(cudaDeviceCanAccessPeer(&can, from, to));
    if (!can) return set_err(PDL_EUNSUPPORTED, "DYNAMIC: device %d cannot access device %d's memory (no P2P)", from, to);
    CUDA_TRY(cudaSetDevice(from));
    cudaError_t e = cudaDeviceEnablePeerAccess(to, 0);
    if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
    else if (e != cudaSuccess) return set_err(PDL_ECUDA, "peer access %d -> %d: %s", from, to, cudaGetErrorString(e));
    return PDL_OK;
}

int run_dynamic(const Task &t, const std::vector<int> &gw) {
    std::vector<WorkerCtx *> ws;
    for (int pu : gw)
        for (auto &w : g->workers)
            if (w.pu == pu) ws.push_back(&w);
    if (ws.empty()) return set_err(PDL_ENOWORKER, "no Worker of the group is bound to this process");
    if ((int)ws.size() > kMaxDynWorkers) return set_err(PDL_EINVAL, "DYNAMIC supports %d Workers", kMaxDynWorkers);
    const bool f64 = t.dtype == PDL_F64;
    const int es = f64 ? 8 : 4;
    const int64_t M = t.M, N = t.N, K = t.K, pe = 16 / es;
    for (auto *w : ws) {
        int sl, rn;
        int n2, b2;
        if (K > 0 && (worker_ozaki(*w, f64, &sl, &rn) || (f64 && worker_ozaki2(*w, &n2, &b2))))
            return set_err(PDL_EUNSUPPORTED,
                           "DYNAMIC needs a single-launch task variant (dmma / 3xtf32); Worker %s runs Ozaki "
                           "(S diagonal launches updating C)",
                           g->model.pus[w->pu].id.c_str());
    }
    WorkerCtx &own = *ws[0];
    int rc;
    size_t evn_own = 0;
    // C destination
    const int cdev = locate(t.C);
    char *Cd = (char *)t.C;
    int64_t ldc = t.ldc;
    void *p;
    if (cdev < 0) {
        ldc = round_up(N, pe);
        if ((rc = ensure_buf(own, BUF_C, (size_t)(ldc * M * es), &p))) return rc;
        Cd = (char *)p;
    }
    const int c_home = cdev >= 0 ? cdev : own.device;
    if (K == 0) {
        CUDA_TRY(cudaSetDevice(c_home));
        CUDA_TRY(cudaMemset2DAsync(Cd, (size_t)(ldc * es), 0, (size_t)(N * es), (size_t)M, own.stream));
    } else {
        // shared claim counters in the first Worker's memory region
        if (g->dyn && g->dyn_dev != own.device) {
            CUDA_TRY(cudaSetDevice(g->dyn_dev));
            CUDA_TRY(cudaDeviceSynchronize());
            cudaFree(g->dyn);
            g->dyn = nullptr;
        }
        CUDA_TRY(cudaSetDevice(own.device));
        if (!g->dyn) {
            CUDA_TRY(cudaMalloc(&g->dyn, (1 + kMaxDynWorkers) * sizeof(int)));
            g->dyn_dev = own.device;
        }
        CUDA_TRY(cudaMemsetAsync(g->dyn, 0, (1 + kMaxDynWorkers) * sizeof(int), own.stream));
        cudaEvent_t ev_reset = ev_get(own, evn_own);
        if (!ev_reset) return set_err(PDL_ECUDA, "event create failed");
        CUDA_TRY(cudaEventRecord(ev_reset, own.stream));
        pdlk::EncodeTiledFn enc = nullptr;
        if ((rc = get_encoder(&enc))) return rc;
        const int64_t Kp = round_up(K, pdlk::K2_BK);
        for (size_t i = 0; i < ws.size(); ++i) {
            WorkerCtx &w = *ws[i];
            if ((rc = enable_peer(w.device, g->dyn_dev)) || (rc = enable_peer(w.device, c_home))) return rc;
            CUDA_TRY(cudaSetDevice(w.device));
            if (&w != &own) CUDA_TRY(cudaStreamWaitEvent(w.stream, ev_reset, 0));
            // operands readable by this Worker
            const char *Ad = (const char *)t.A, *Bd = (const char *)t.B;
            int64_t lda = t.lda, ldb = t.ldb;
            if (locate(t.A) != w.device || (f64 && (((uintptr_t)t.A % 16) || (t.lda * es) % 16))) {
                lda = round_up(K, pe);
                if ((rc = ensure_buf(w, BUF_A, (size_t)(lda * M * es), &p))) return rc;
                CUDA_TRY(cudaMemcpy2DAsync(p, (size_t)(lda * es), t.A, (size_t)(t.lda * es), (size_t)(K * es),
                                           (size_t)M, cudaMemcpyDefault, w.stream));
                Ad = (const char *)p;
            }
            if (locate(t.B) != w.device || (f64 && (((uintptr_t)t.B % 16) || (t.ldb * es) % 16))) {
                ldb = round_up(N, pe);
                if ((rc = ensure_buf(w, BUF_B, (size_t)(ldb * K * es), &p))) return rc;
                CUDA_TRY(cudaMemcpy2DAsync(p, (size_t)(ldb * es), t.B, (size_t)(t.ldb * es), (size_t)(N * es),
                                           (size_t)K, cudaMemcpyDefault, w.stream));
                Bd = (const char *)p;
            }
            int *mine = g->dyn + 1 + i;
            cudaError_t e;
            if (f64) {
                if (kt_mark(w, true, w.stream)) return set_err(PDL_ECUDA, "event record failed");
                e = pdlk::launch_dgemm_k1(enc, (const double *)Ad, lda, (const double *)Bd, ldb, (double *)Cd, ldc, M,
                                          N, K, w.stream, g->dyn, mine);
                w.launches += 1;
            } else {
                float *buf4[4];
                const int slots[4] = {BUF_AHI, BUF_ALO, BUF_BHI, BUF_BLO};
                for (int b = 0; b < 4; ++b) {
                    if ((rc = ensure_buf(w, slots[b], (size_t)((b < 2 ? M : N) * Kp * 4), &p))) return rc;
                    buf4[b] = (float *)p;
                }
                w.bsig.valid = false;
                e = pdlk::launch_split_rows((const float *)Ad, lda, M, K, buf4[0], buf4[1], Kp, w.stream);
                if (e == cudaSuccess)
                    e = pdlk::launch_split_cols_t((const float *)Bd, ldb, K, N, buf4[2], buf4[3], Kp, w.stream);
                if (e != cudaSuccess) return set_err(PDL_ECUDA, "K3 split launch failed: %s", cudaGetErrorString(e));
                if (kt_mark(w, true, w.stream)) return set_err(PDL_ECUDA, "event record failed");
                e = pdlk::launch_gemm_3xtf32_2sm(enc, buf4[0], buf4[1], buf4[2], buf4[3], Kp, (float *)Cd, ldc, M, N,
                                                 w.stream, g->dyn, mine);
                w.launches += 3;
            }
            if (e != cudaSuccess) return set_err(PDL_ECUDA, "tile kernel launch failed: %s", cudaGetErrorString(e));
            if (kt_mark(w, false, w.stream)) return set_err(PDL_ECUDA, "event record failed");
            w.timed = true;
            if (&w != &own) {
                size_t evn_w = 0;
                cudaEvent_t done = ev_get(w, evn_w);
                if (!done) return set_err(PDL_ECUDA, "event create failed");
                CUDA_TRY(cudaEventRecord(done, w.stream));
                CUDA_TRY(cudaStreamWaitEvent(own.stream, done, 0));   // join on the first Worker
            }
        }
        g->dyn_n = (int)ws.size();
        g->dyn_kernel = f64 ? "K1 dgemm_k1_kernel" : "K2 gemm_3xtf32_2sm_kernel";
    }
    if (cdev < 0) {
        CUDA_TRY(cudaSetDevice(own.device));
        CUDA_TRY(cudaMemcpy2DAsync(t.C, (size_t)(t.ldc * es), Cd, (size_t)(ldc * es), (size_t)(N * es), (size_t)M,
                                   cudaMemcpyDefault, own.stream));
    }
    return PDL_OK;
}

// ---- CUDA graphs of repeated tasks ----
//
// A Worker's launch sequence for one task (staging copies, split / slicing
// pre-passes, tile kernels, CRT pass, copy-out, across its side streams) depends
// only on the task's signature.  With PDL_TASK_GRAPH (or PDL_GRAPH=1) the first run
// of a signature executes normally (sizing the Worker's buffers), the second is
// captured from the Worker stream into a CUDA graph, and later runs replay it with
// one cudaGraphLaunch -- for launch-bound small tasks.  Anything the capture cannot
// hold (pageable host memory, a buffer reallocation) makes that signature run
// uncaptured from then on.  Not used with PDL_TASK_REUSE_B (its launches depend on
// state left by the previous task) or DYNAMIC.

constexpr size_t kMaxGraphs = 64;   // cached graphs per Worker

std::string graph_key(const WorkerCtx &w, const Task &t, const void *A, const void *B, void *C, int64_t rows,
                      int64_t cols) {
    std::ostringstream k;
    k << t.dtype << '|' << A << '|' << t.lda << '|' << B << '|' << t.ldb << '|' << C << '|' << t.ldc << '|' << t.M
      << '|' << t.N << '|' << t.K << '|' << t.tile << '|' << t.flags << '|' << rows << '|' << cols << '|'
      << (const void *)w.stream << '|' << w.buf_gen;
    for (char **e = environ; e && *e; ++e)   // library knobs change the launch sequence
        if (!strncmp(*e, "PDL_", 4)) k << '|' << *e;
    return k.str();
}

int run_rect_g(WorkerCtx &w, const Task &t, const void *A, const void *B, void *C, int64_t rows, int64_t cols) {
    const bool want = (t.flags & PDL_TASK_GRAPH) || env_on("PDL_GRAPH");
    if (!want || (t.flags & PDL_TASK_REUSE_B) || g->dry_run || rows <= 0 || cols <= 0)
        return run_rect(w, t, A, B, C, rows, cols);
    CUDA_TRY(cudaSetDevice(w.device));
    const std::string key = graph_key(w, t, A, B, C, rows, cols);
    auto replay = [&](WorkerCtx::GraphEntry &ge) -> int {
        CUDA_TRY(cudaGraphLaunch(ge.exec, w.stream));
        w.launches += ge.launches;
        w.timed |= ge.timed;
        for (auto &pr : ge.kt_pairs)
            if (w.kt_list.size() < kMaxKernelTimes) w.kt_list.push_back(pr);
        w.bsig.valid = false;
        ++w.graph_replays;
        return PDL_OK;
    };
    auto it = w.graphs.find(key);
    if (it != w.graphs.end()) return replay(it->second);
    if (w.graph_seen.size() >= 16 * kMaxGraphs) w.graph_seen.clear();
    int &seen = w.graph_seen[key];
    if (seen <= 0) {   // first run (or not capturable): plain
        const bool first = seen++ == 0;
        const int rc = run_rect(w, t, A, B, C, rows, cols);
        // the run may have sized the Worker's buffers: the next run has this key
        if (first && !rc) {
            int &s2 = w.graph_seen[graph_key(w, t, A, B, C, rows, cols)];
            if (s2 == 0) s2 = 1;
        }
        return rc;
    }
    const size_t used0 = w.kt_used, list0 = w.kt_list.size();
    const int launches0 = w.launches;
    const int gen0 = w.buf_gen;
    if (cudaStreamBeginCapture(w.stream, cudaStreamCaptureModeRelaxed) != cudaSuccess) {
        cudaGetLastError();
        seen = -1000000;
        return run_rect(w, t, A, B, C, rows, cols);
    }
    w.capturing = true;
    const int rc = run_rect(w, t, A, B, C, rows, cols);
    w.capturing = false;
    cudaGraph_t graph = nullptr;
    cudaError_t e = cudaStreamEndCapture(w.stream, &graph);
    cudaGraphExec_t exec = nullptr;
    if (!rc && e == cudaSuccess && graph && w.buf_gen == gen0) e = cudaGraphInstantiate(&exec, graph, 0);
    if (graph) cudaGraphDestroy(graph);
    if (rc || e != cudaSuccess || !exec || w.buf_gen != gen0) {
        // not capturable: drop what the capture recorded and run the task plainly
        cudaGetLastError();
        if (exec) cudaGraphExecDestroy(exec);
        w.kt_used = used0;
        w.kt_list.resize(list0);
        w.launches = launches0;
        seen = -1000000;
        logf(1, "task not capturable into a CUDA graph (%s); running it uncaptured", rc ? g_err.c_str() : "capture");
        return run_rect(w, t, A, B, C, rows, cols);
    }
    if (w.graphs.size() >= kMaxGraphs) {   // bounded cache: start over
        for (auto &kv : w.graphs) {
            cudaGraphExecDestroy(kv.second.exec);
            // the events may still be listed in kt_list: hand them back to the pool
            w.kt_pool.insert(w.kt_pool.end(), kv.second.events.begin(), kv.second.events.end());
        }
        w.graphs.clear();
    }
    WorkerCtx::GraphEntry ge;
    ge.exec = exec;
    ge.launches = w.launches - launches0;
    ge.timed = true;
    ge.events.assign(w.kt_pool.begin() + used0, w.kt_pool.begin() + w.kt_used);   // now recorded by the graph
    w.kt_pool.erase(w.kt_pool.begin() + used0, w.kt_pool.begin() + w.kt_used);
    w.kt_used = used0;
    ge.kt_pairs.assign(w.kt_list.begin() + list0, w.kt_list.end());
    w.kt_list.resize(list0);
    w.launches = launches0;
    return replay(w.graphs.emplace(key, std::move(ge)).first->second);
}

int check_loaded() {
    if (!g || !g->loaded) return set_err(PDL_ESTATE, "no platform loaded (call pdl_load first)");
    return PDL_OK;
}

int do_load(const char *descriptor, int rank, int nranks) {
    if (g && g->loaded) return set_err(PDL_ESTATE, "a platform is already loaded (call pdl_unload first)");
    if (!descriptor) return set_err(PDL_EINVAL, "descriptor is NULL");
    if (nranks < 1 || rank < 0 || rank >= nranks) return set_err(PDL_EINVAL, "bad rank %d of %d", rank, nranks);
    bool ok;
    std::string doc = read_descriptor(descriptor, &ok);
    if (!ok) return set_err(PDL_EINVAL, "cannot read descriptor file '%s'", descriptor);
    std::unique_ptr<State> st(new State());
    try {
        auto root = parse_xml(doc);
        st->model = build_model(*root);
    } catch (const XmlError &e) {
        return set_err(PDL_EPARSE, "XML error at line %d: %s", e.line, e.msg.c_str());
    } catch (const ModelError &e) {
        return set_err(PDL_EPARSE, "PDL error at line %d: %s", e.line, e.msg.c_str());
    }
    st->dry_run = env_on("PDL_DRY_RUN");
    st->oversub = env_on("PDL_ALLOW_OVERSUBSCRIBE");
    st->rank = rank;
    st->nranks = nranks;
    g = st.release();
    int rc = bind_devices();
    if (rc) {
        std::string msg = g_err;
        free_state();
        g_err = msg;
        return rc;
    }
    g->loaded = true;
    logf(1, "loaded: %zu PUs, %zu gpu Workers, rank %d/%d%s", g->model.pus.size(), g->model.all_gpu_workers().size(),
         rank, nranks, g->dry_run ? " (dry run)" : "");
    return PDL_OK;
}

int enqueue(int dtype, const void *A, int64_t lda, const void *B, int64_t ldb, void *C, int64_t ldc, int64_t M,
            int64_t N, int64_t K, int64_t tile, const char *group, const char *dist, unsigned flags) {
    int rc = check_loaded();
    if (rc) return rc;
    if (dtype != PDL_F64 && dtype != PDL_F32) return set_err(PDL_EINVAL, "unknown dtype %d", dtype);
    if (M < 0 || N < 0 || K < 0) return set_err(PDL_EINVAL, "negative size M=%lld N=%lld K=%lld", (long long)M,
                                                (long long)N, (long long)K);
    if (tile < 0) return set_err(PDL_EINVAL, "negative tile %lld", (long long)tile);
    if (flags & ~(PDL_TASK_PANELS | PDL_TASK_LOCAL | PDL_TASK_REUSE_B | PDL_TASK_GRAPH))
        return set_err(PDL_EINVAL, "unknown flags 0x%x", flags);
    if ((flags & PDL_TASK_PANELS) && (flags & PDL_TASK_LOCAL))
        return set_err(PDL_EINVAL, "PDL_TASK_PANELS and PDL_TASK_LOCAL are exclusive");
    DistSpec ds;
    if (!parse_dist(dist, &ds))
        return set_err(PDL_EINVAL, "unknown distribution '%s' (L1200-1206: BLOCK, CYCLIC, BLOCK-CYCLIC[:b])", dist);
    if (ds.kind != Dist::Block && ((flags & PDL_TASK_PANELS) || g->nranks > 1))
        return set_err(PDL_EUNSUPPORTED,
                       "distribution %s needs one process driving the Workers (the multi-rank panel exchange is BLOCK)",
                       dist);
    if (group && g->model.group_workers(group).empty())
        return set_err(PDL_EINVAL, "execution group '%s' names no gpu Worker (LogicGroupAttribute)", group);
    if (M == 0 || N == 0) return PDL_OK;   // nothing to write
    const int es = dtype == PDL_F64 ? 8 : 4;
    if (!C) return set_err(PDL_EINVAL, "C is NULL with M*N > 0");
    if (K > 0 && (!A || !B)) return set_err(PDL_EINVAL, "A or B is NULL with K > 0");
    // leading dimensions (0 = dense); in PANELS mode widths are the Worker's
    int64_t lda_ = lda ? lda : K, ldb_ = ldb, ldc_ = ldc;
    if (!(flags & PDL_TASK_PANELS)) {
        if (!ldb_) ldb_ = N;
        if (!ldc_) ldc_ = N;
        if (lda_ < K || ldb_ < N || ldc_ < N) return set_err(PDL_EINVAL, "leading dimension smaller than the row width");
        size_t an = (size_t)((M - 1) * lda_ + K) * es, bn = K ? (size_t)((K - 1) * ldb_ + N) * es : 0,
               cn = (size_t)((M - 1) * ldc_ + N) * es;
        if (K > 0 && (overlaps(C, cn, A, an) || overlaps(C, cn, B, bn)))
            return set_err(PDL_EINVAL, "C overlaps A or B (C has access mode write, A/B read, L1184-1186)");
    }
    Task t{dtype, A, lda_, B, ldb_, C, ldc_, M, N, K, tile, group != nullptr, group ? group : "", flags, ds};
    g->queue.push_back(t);
    return PDL_OK;
}

int execute(bool sync) {
    int rc = check_loaded();
    if (rc) return rc;
    std::vector<Task> q;
    q.swap(g->queue);   // the queue is cleared whatever happens
    std::ostringstream pj;
    pj << "[";
    for (auto &w : g->workers) {
        w.launches = 0;
        w.timed = false;
    }
    // Green-context streams are non-blocking: give them the ordering of the
    // blocking Worker streams (after the legacy default stream's prior work,
    // and the legacy stream after them -- see the end of this function).
    if (!g->dry_run)
        for (auto &w : g->workers)
            if (w.gctx && w.own_stream) {
                CUDA_TRY(cudaSetDevice(w.device));
                if (!w.ev_legacy) CUDA_TRY(cudaEventCreateWithFlags(&w.ev_legacy, cudaEventDisableTiming));
                CUDA_TRY(cudaEventRecord(w.ev_legacy, cudaStreamLegacy));
                CUDA_TRY(cudaStreamWaitEvent(w.stream, w.ev_legacy, 0));
            }
    for (size_t ti = 0; ti < q.size(); ++ti) {
        const Task &t = q[ti];
        if (t.flags & PDL_TASK_LOCAL) {
            // one tile task of this process's (first) Worker, no mapping
            if (ti) pj << ",";
            pj << "{\"local\":true,\"M\":" << t.M << ",\"N\":" << t.N << ",\"K\":" << t.K << "}";
            if (g->dry_run) continue;
            if (g->workers.empty()) return set_err(PDL_ENOWORKER, "no Worker bound to this process");
            rc = run_rect_g(g->workers[0], t, t.A, t.B, t.C, t.M, t.N);
            if (rc) return rc;
            continue;
        }
        std::vector<int> gw = g->model.group_workers(t.has_group ? t.group.c_str() : nullptr);
        const int G = (int)gw.size();
        if (G == 0) return set_err(PDL_ENOWORKER, "execution group has no gpu Worker");
        if (g->nranks > 1 && G != g->nranks)
            return set_err(PDL_ENOWORKER, "group has %d Workers but %d ranks co-exist: one process per Worker", G,
                           g->nranks);
        const std::vector<double> speeds = worker_speeds(g->model, gw);
        // one process driving the Workers maps through the PU hierarchy (Hybrid
        // subtrees, NEXT-4); the multi-rank panel exchange needs the flat grid
        Plan plan = g->nranks == 1 && !(t.flags & PDL_TASK_PANELS)
                        ? make_plan_tree(t.M, t.N, t.K, t.tile, g->model, gw, t.dist, speeds)
                        : make_plan(t.M, t.N, t.K, t.tile, G, t.dist, &speeds);
        std::vector<std::string> ids;
        for (int x : gw) ids.push_back(g->model.pus[x].id);
        if (ti) pj << ",";
        pj << plan.to_json(gw, ids);
        if (g->dry_run) continue;
        if (t.dist.kind == Dist::Dynamic) {
            rc = run_dynamic(t, gw);
            if (rc) return rc;
            continue;
        }
        const int es = t.dtype == PDL_F64 ? 8 : 4;
        for (auto &w : g->workers) {
            // group index of this bound Worker
            int gi = -1;
            for (int i = 0; i < G; ++i)
                if (gw[i] == w.pu) gi = i;
            if (gi < 0) continue;
            if (t.dist.kind != Dist::Block) {
                // CYCLIC / BLOCK-CYCLIC: the Worker's tasks form row segments x column
                // segments; each product is one sub-rectangle (same per-element K
                // order, so C is bitwise the BLOCK result, R14)
                for (const Seg &rs : plan.row_segs(gi / plan.Gc))
                    for (const Seg &cs : plan.col_segs(gi % plan.Gc)) {
                        const char *A = (const char *)t.A + (size_t)(rs.lo * t.lda) * es;
                        const char *B = (const char *)t.B + (size_t)cs.lo * es;
                        char *C = (char *)t.C + (size_t)(rs.lo * t.ldc + cs.lo) * es;
                        rc = run_rect_g(w, t, A, B, C, rs.hi - rs.lo, cs.hi - cs.lo);
                        if (rc) return rc;
                    }
                continue;
            }
            Rect R = plan.rect(gi);
            const int64_t rows = R.row1 - R.row0, cols = R.col1 - R.col0;
            const char *A = (const char *)t.A, *B = (const char *)t.B;
            char *C = (char *)t.C;
            int64_t lda = t.lda, ldb = t.ldb, ldc = t.ldc;
            if (t.flags & PDL_TASK_PANELS) {
                if (!lda) lda = t.K;
                if (!ldb) ldb = cols;
                if (!ldc) ldc = cols;
            } else {
                A += (size_t)(R.row0 * lda) * es;
                B += (size_t)R.col0 * es;
                C += (size_t)(R.row0 * ldc + R.col0) * es;
            }
            Task tt = t;
            tt.lda = lda;
            tt.ldb = ldb;
            tt.ldc = ldc;
            rc = run_rect_g(w, tt, A, B, C, rows, cols);
            if (rc) return rc;
        }
    }
    pj << "]";
    g->plan_json = pj.str();
    for (auto &w : g->workers) g->total_launches += w.launches;
    if (!g->dry_run)
        for (auto &w : g->workers)
            if (w.gctx && w.own_stream) {
                CUDA_TRY(cudaSetDevice(w.device));
                CUDA_TRY(cudaEventRecord(w.ev_legacy, w.stream));
                CUDA_TRY(cudaStreamWaitEvent(cudaStreamLegacy, w.ev_legacy, 0));
            }
    if (sync) return pdl_sync();
    return PDL_OK;
}

}  // namespace

extern "C" {

int pdl_load(const char *descriptor) { return do_load(descriptor, 0, 1); }

int pdl_load_rank(const char *descriptor, int rank, int nranks) { return do_load(descriptor, rank, nranks); }

int task_matmul(const double *A, const double *B, double *C, int64_t M, int64_t N, int64_t K, int64_t tile) {
    return enqueue(PDL_F64, A, 0, B, 0, C, 0, M, N, K, tile, nullptr, nullptr, 0);
}

int task_matmul_f32(const float *A, const float *B, float *C, int64_t M, int64_t N, int64_t K, int64_t tile) {
    return enqueue(PDL_F32, A, 0, B, 0, C, 0, M, N, K, tile, nullptr, nullptr, 0);
}

int task_matmul_ex(int dtype, const void *A, int64_t lda, const void *B, int64_t ldb, void *C, int64_t ldc, int64_t M,
                   int64_t N, int64_t K, int64_t tile, const char *group, const char *dist, unsigned flags) {
    if (lda < 0 || ldb < 0 || ldc < 0) return set_err(PDL_EINVAL, "negative leading dimension");
    return enqueue(dtype, A, lda, B, ldb, C, ldc, M, N, K, tile, group, dist, flags);
}

int pdl_run(void) { return execute(true); }

int pdl_run_async(void) { return execute(false); }

int pdl_sync(void) {
    int rc = check_loaded();
    if (rc) return rc;
    if (g->dry_run) return PDL_OK;
    int launches = 0;
    for (auto &w : g->workers) {
        CUDA_TRY(cudaSetDevice(w.device));
        cudaError_t e = cudaStreamSynchronize(w.stream);
        if (e != cudaSuccess) return set_err(PDL_ECUDA, "device work failed on device %d: %s", w.device,
                                             cudaGetErrorString(e));
        launches += w.launches;
    }
    g->last_launches = launches;
    return PDL_OK;
}

int pdl_set_stream(int worker, void *stream) {
    int rc = check_loaded();
    if (rc) return rc;
    if (worker < 0 || worker >= (int)g->workers.size()) return set_err(PDL_EINVAL, "no local Worker %d", worker);
    WorkerCtx &w = g->workers[worker];
    if (g->dry_run) return PDL_OK;
    CUDA_TRY(cudaSetDevice(w.device));
    if (stream) {
        if (w.own_stream && w.stream) {
            cudaStreamSynchronize(w.stream);
            cudaStreamDestroy(w.stream);
        }
        w.stream = (cudaStream_t)stream;
        w.own_stream = false;
    } else if (!w.own_stream) {
        int rc2 = worker_stream(w, &w.stream, true);
        if (rc2) return rc2;
        w.own_stream = true;
    }
    return PDL_OK;
}

int pdl_plan(int64_t M, int64_t N, int64_t K, int64_t tile, const char *group, int worker, int64_t *out, int nout) {
    int rc = check_loaded();
    if (rc) return rc;
    if (M < 0 || N < 0 || K < 0 || tile < 0) return set_err(PDL_EINVAL, "negative size");
    if (!out || nout < PDL_PLAN_LEN) return set_err(PDL_EINVAL, "out[] needs %d entries", PDL_PLAN_LEN);
    std::vector<int> gw = g->model.group_workers(group);
    if (gw.empty()) return set_err(PDL_ENOWORKER, "execution group has no gpu Worker");
    const int G = (int)gw.size();
    if (worker < 0 || worker >= G) return set_err(PDL_EINVAL, "worker %d outside the group of %d", worker, G);
    const std::vector<double> speeds = worker_speeds(g->model, gw);
    Plan p = g->nranks == 1 ? make_plan_tree(M, N, K, tile, g->model, gw, DistSpec(), speeds)
                            : make_plan(M, N, K, tile, G, DistSpec(), &speeds);
    Rect R = p.rect(worker);
    if (p.hierarchical()) {
        // explicit rectangle (Hybrid subtrees): no Worker grid, no panel exchange
        const int64_t e = p.tile > 0 ? p.tile : 1;
        int64_t v[PDL_PLAN_LEN] = {G, G, 1, worker, 0, R.row0, R.row1, R.col0, R.col1, R.row1 - R.row0, K,
                                   p.Tm, p.Tn, R.row0 / e, (R.row1 + e - 1) / e, R.col0 / e, (R.col1 + e - 1) / e,
                                   p.tile};
        for (int i = 0; i < PDL_PLAN_LEN; ++i) out[i] = v[i];
        return PDL_OK;
    }
    const int r = worker / p.Gc, c = worker % p.Gc;
    int64_t v[PDL_PLAN_LEN] = {G, p.Gr, p.Gc, r, c, R.row0, R.row1, R.col0, R.col1, p.qa(worker), p.qb(),
                               p.Tm, p.Tn, p.trow[r], p.trow[r + 1], p.tcol[c], p.tcol[c + 1], p.tile};
    for (int i = 0; i < PDL_PLAN_LEN; ++i) out[i] = v[i];
    return PDL_OK;
}

int pdl_query(const char *key, char *out, size_t len) {
    if (!key) return set_err(PDL_EINVAL, "key is NULL");
    std::string k(key), res;
    if (k == "version") {
        res = kVersion;
    } else if (k.rfind("ozaki2_plan/", 0) == 0) {
        // "ozaki2_plan/<K>[/<bits>[/<moduli>]]": the Ozaki-II parameters the FP64
        // variant ozaki2 uses for inner dimension K (host arithmetic, no device)
        long long K = 0;
        int bits = 43, nmod = 0;
        if (sscanf(k.c_str() + 12, "%lld/%d/%d", &K, &bits, &nmod) < 1 || K < 0)
            return set_err(PDL_EINVAL, "bad key '%s' (ozaki2_plan/<K>[/<bits>[/<moduli>]])", key);
        const pdlk::Ozaki2Plan P = pdlk::ozaki2_plan(1, 1, K, nmod, std::max(8, std::min(52, bits)));
        std::ostringstream o;
        o << "{\"n\":" << P.n << ",\"p\":" << P.p << ",\"nch\":" << P.nch << ",\"Kc\":" << P.Kc << ",\"moduli\":[";
        for (int t = 0; t < P.n; ++t) o << (t ? "," : "") << P.m[t];
        auto dec = [](unsigned long long lo, unsigned long long hi) {   // 128-bit value as decimal text
            unsigned __int128 v = ((unsigned __int128)hi << 64) | lo;
            std::string d;
            do {
                d.insert(d.begin(), (char)('0' + (int)(v % 10)));
                v /= 10;
            } while (v);
            return d;
        };
        o << "],\"W\":[";
        for (int t = 0; t < P.n; ++t) o << (t ? "," : "") << "\"" << dec(P.W[t][0], P.W[t][1]) << "\"";
        o << "],\"M\":\"" << dec(P.Mw[0], P.Mw[1]) << "\"}";
        res = o.str();
    } else {
        int rc = check_loaded();
        if (rc) return rc;
        const Model &m = g->model;
        if (k == "masters") res = std::to_string(m.masters.size());
        else if (k == "workers") res = std::to_string(m.all_gpu_workers().size());
        else if (k == "local_workers") res = std::to_string(g->workers.size());
        else if (k == "model") res = m.to_json();
        else if (k == "interconnects") res = m.ics_json();
        else if (k == "plan") res = g->plan_json;
        else if (k == "groups") {
            std::vector<std::string> gs;
            for (auto &p : m.pus)
                for (auto &x : p.groups)
                    if (std::find(gs.begin(), gs.end(), x) == gs.end()) gs.push_back(x);
            res = "[";
            for (size_t i = 0; i < gs.size(); ++i) res += (i ? ",\"" : "\"") + json_escape(gs[i]) + "\"";
            res += "]";
        } else if (k == "stats") {
            std::ostringstream o;
            o << "{\"launches\":" << g->last_launches << ",\"total_launches\":" << g->total_launches
              << ",\"workers\":[";
            bool first = true;
            for (auto &w : g->workers) {
                float ms = -1.f;
                if (w.timed && !g->dry_run) {
                    cudaSetDevice(w.device);
                    if (cudaEventElapsedTime(&ms, w.ev_k0, w.ev_k1) != cudaSuccess) {
                        cudaGetLastError();
                        ms = -1.f;
                    }
                }
                o << (first ? "" : ",") << "{\"id\":\"" << json_escape(m.pus[w.pu].id) << "\",\"device\":" << w.device
                  << ",\"kernel_ms\":" << ms << ",\"launches\":" << w.launches << ",\"sm_limit\":" << w.sm_limit
                  << ",\"graphs\":" << w.graphs.size() << ",\"graph_replays\":" << w.graph_replays << "}";
                first = false;
            }
            o << "]";
            // tiles each Worker claimed in the last DYNAMIC task (valid after pdl_sync)
            if (g->dyn_n > 0 && g->dyn && !g->dry_run) {
                std::vector<int> claims(g->dyn_n + 1, 0);
                cudaSetDevice(g->dyn_dev);
                if (cudaMemcpy(claims.data(), g->dyn, claims.size() * sizeof(int), cudaMemcpyDeviceToHost) != cudaSuccess)
                    cudaGetLastError();
                long long tot = 0;
                o << ",\"dynamic\":{\"kernel\":\"" << g->dyn_kernel << "\",\"tiles\":[";
                for (int i = 0; i < g->dyn_n; ++i) {
                    o << (i ? "," : "") << claims[1 + i];
                    tot += claims[1 + i];
                }
                o << "],\"total\":" << tot << "}";
            }
            o << "}";
            res = o.str();
        } else if (k.rfind("worker/", 0) == 0 || k.rfind("pu/", 0) == 0) {
            bool is_w = k[0] == 'w';
            size_t s1 = k.find('/'), s2 = k.find('/', s1 + 1);
            if (s2 == std::string::npos) return set_err(PDL_EINVAL, "bad key '%s'", key);
            std::string who = k.substr(s1 + 1, s2 - s1 - 1), what = k.substr(s2 + 1);
            int pu = -1;
            if (is_w) {
                std::vector<int> gw = m.all_gpu_workers();
                char *end;
                long i = strtol(who.c_str(), &end, 10);
                if (*end || i < 0 || i >= (long)gw.size()) return set_err(PDL_EINVAL, "no gpu Worker %s", who.c_str());
                pu = gw[i];
            } else {
                for (size_t i = 0; i < m.pus.size(); ++i)
                    if (m.pus[i].id == who) pu = (int)i;
                if (pu < 0) return set_err(PDL_EINVAL, "no PU with id '%s'", who.c_str());
            }
            if (what == "device") res = std::to_string(m.pus[pu].device);
            else if (what == "id") res = m.pus[pu].id;
            else if (what == "kind") res = kind_name(m.pus[pu].kind);
            else {
                const Property *p = m.prop(pu, what);
                if (!p) return set_err(PDL_EINVAL, "PU %s has no property %s", m.pus[pu].id.c_str(), what.c_str());
                res = p->value;
            }
        } else {
            return set_err(PDL_EINVAL, "unknown query key '%s'", key);
        }
    }
    if (out && len) {
        size_t n = std::min(len - 1, res.size());
        memcpy(out, res.data(), n);
        out[n] = '\0';
    }
    return (int)res.size();
}

int pdl_kernel_times(int worker, float *ms, int n) {
    int rc = check_loaded();
    if (rc) return rc;
    if (worker < 0 || worker >= (int)g->workers.size()) return set_err(PDL_EINVAL, "no local Worker %d", worker);
    if (n < 0 || (n > 0 && !ms)) return set_err(PDL_EINVAL, "bad output buffer");
    WorkerCtx &w = g->workers[worker];
    if (g->dry_run) return 0;
    CUDA_TRY(cudaSetDevice(w.device));
    const int cnt = (int)w.kt_list.size();
    for (int i = 0; i < cnt && i < n; ++i) {
        CUDA_TRY(cudaEventSynchronize(w.kt_list[i].second));
        CUDA_TRY(cudaEventElapsedTime(&ms[i], w.kt_list[i].first, w.kt_list[i].second));
    }
    w.kt_list.clear();
    w.kt_used = 0;
    return cnt;
}

int pdl_describe(char *out, size_t len) {
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        return set_err(PDL_ENOWORKER, "no CUDA device visible (%s)",
                       e == cudaSuccess ? "0 devices" : cudaGetErrorString(e));
    }
#if defined(__x86_64__)
    const char *arch = "x86";
#elif defined(__aarch64__)
    const char *arch = "arm";
#else
    const char *arch = "unknown";
#endif
    const long long host_bytes = (long long)sysconf(_SC_PHYS_PAGES) * (long long)sysconf(_SC_PAGE_SIZE);
    auto prop = [](std::ostringstream &o, const char *name, const std::string &val, const char *unit, bool fixed) {
        o << "      <Property fixed=\"" << (fixed ? "true" : "false") << "\"><name>" << name << "</name><value";
        if (unit && *unit) o << " unit=\"" << unit << "\"";
        std::string x;
        for (char ch : val) {
            switch (ch) {
                case '&': x += "&amp;"; break;
                case '<': x += "&lt;"; break;
                case '>': x += "&gt;"; break;
                default: x += ch;
            }
        }
        o << ">" << x << "</value></Property>\n";
    };
    std::ostringstream o;
    o << "<?xml version=\"1.0\"?>\n<!-- generated by pdl_describe (" << kVersion << ") -->\n";
    o << "<Master id=\"0\" quantity=\"1\">\n  <PUDescriptor>\n";
    prop(o, "ARCHITECTURE", arch, "", true);
    o << "  </PUDescriptor>\n  <MemoryRegion id=\"host\"><MRDescriptor>\n";
    prop(o, "SIZE", std::to_string(host_bytes), "B", false);
    o << "  </MRDescriptor></MemoryRegion>\n";
    for (int d = 0; d < ndev; ++d) {
        cudaDeviceProp p;
        if (cudaGetDeviceProperties(&p, d) != cudaSuccess) {
            cudaGetLastError();
            return set_err(PDL_ECUDA, "cudaGetDeviceProperties(%d) failed", d);
        }
        o << "  <Worker id=\"gpu" << d << "\" quantity=\"1\">\n    <PUDescriptor>\n";
        prop(o, "ARCHITECTURE", "gpu", "", true);
        prop(o, "DEVICE_ORDINAL", std::to_string(d), "", true);
        prop(o, "DEVICE_NAME", p.name, "", false);
        prop(o, "MAX_COMPUTE_UNITS", std::to_string(p.multiProcessorCount), "", false);
        prop(o, "COMPUTE_CAPABILITY", std::to_string(p.major) + "." + std::to_string(p.minor), "", false);
        prop(o, "GLOBAL_MEM_SIZE", std::to_string((unsigned long long)p.totalGlobalMem), "B", false);
        prop(o, "LOCAL_MEM_SIZE", std::to_string((unsigned long long)p.sharedMemPerBlockOptin), "B", false);
        prop(o, "L2_CACHE_SIZE", std::to_string(p.l2CacheSize), "B", false);
        int clk = 0;
        cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, d);
        prop(o, "CLOCK_RATE", std::to_string(clk), "kHz", false);
        prop(o, "PCI_BUS_ID", std::to_string(p.pciBusID), "", false);
        o << "    </PUDescriptor>\n    <MemoryRegion id=\"hbm\"><MRDescriptor>\n";
        prop(o, "SIZE", std::to_string((unsigned long long)p.totalGlobalMem), "B", false);
        o << "    </MRDescriptor></MemoryRegion>\n    <LogicGroupAttribute>gpus</LogicGroupAttribute>\n  </Worker>\n";
    }
    for (int d = 0; d < ndev; ++d) o << "  <Interconnect type=\"PCIe\" from=\"0\" to=\"gpu" << d << "\" scheme=\"\"/>\n";
    for (int a = 0; a < ndev; ++a)
        for (int b = a + 1; b < ndev; ++b) {
            int can = 0;
            if (cudaDeviceCanAccessPeer(&can, a, b) != cudaSuccess) {
                cudaGetLastError();
                can = 0;
            }
            if (can) o << "  <Interconnect type=\"NVLink\" from=\"gpu" << a << "\" to=\"gpu" << b << "\" scheme=\"p2p\"/>\n";
        }
    o << "</Master>\n";
    const std::string res = o.str();
    if (out && len) {
        size_t n = std::min(len - 1, res.size());
        memcpy(out, res.data(), n);
        out[n] = '\0';
    }
    return (int)res.size();
}

const char *pdl_last_error(void) { return g_err.c_str(); }

void pdl_unload(void) {
    free_state();
    g_err.clear();
}

}  // extern "C"
