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
#include "pdl_rt.hpp"

#include <chrono>

namespace pdlrt {


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
    if (flags & ~(PDL_TASK_PANELS | PDL_TASK_LOCAL | PDL_TASK_REUSE_B | PDL_TASK_GRAPH | PDL_TASK_SLOT(3) |
                  PDL_TASK_PREP_A | PDL_TASK_PREPARED_A))
        return set_err(PDL_EINVAL, "unknown flags 0x%x", flags);
    if ((flags & (PDL_TASK_PREP_A | PDL_TASK_PREPARED_A)) && !(flags & PDL_TASK_LOCAL))
        return set_err(PDL_EINVAL, "PDL_TASK_PREP_A / PDL_TASK_PREPARED_A need PDL_TASK_LOCAL");
    if ((flags & PDL_TASK_PREP_A) && (flags & PDL_TASK_PREPARED_A))
        return set_err(PDL_EINVAL, "PDL_TASK_PREP_A and PDL_TASK_PREPARED_A are exclusive");
    if (flags & PDL_TASK_PREP_A) {
        // A (M x K) -> prepared rows written to C; no product, no B
        if (M < 0 || K < 0) return set_err(PDL_EINVAL, "negative size");
        if (M == 0 || K == 0) return PDL_OK;
        if (!A || !C) return set_err(PDL_EINVAL, "A or the output C is NULL");
        const int64_t lda_ = lda ? lda : K;
        if (lda_ < K) return set_err(PDL_EINVAL, "leading dimension smaller than the row width");
        Task t{dtype, A, lda_, nullptr, 0, C, 0, M, 0, K, tile, group != nullptr, group ? group : "", flags, DistSpec()};
        g->queue.push_back(t);
        return PDL_OK;
    }
    if (((flags >> 4) & 3u) >= 3u) return set_err(PDL_EINVAL, "scratch slot %u out of range (0..2)", (flags >> 4) & 3u);
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

}  // namespace pdlrt

using namespace pdlrt;

namespace pdlrt {

// NVLink topology through NVML (dlopen'ed: the library must load where NVML is
// absent), for pdl_describe's Worker properties and NVLink ICDescriptors
// ("NVML NVLink topology").  links = active NVLink links of the
// device, version = NVLink generation, via_switch = a link ends at an NVSwitch.
struct NvLinkInfo {
    int links = -1, version = 0;
    bool via_switch = false;
};

std::vector<NvLinkInfo> nvlink_topology(int ndev) {
    std::vector<NvLinkInfo> info(ndev);
    void *h = dlopen("libnvidia-ml.so.1", RTLD_NOW | RTLD_LOCAL);
    if (!h) return info;
    typedef int (*init_t)();
    typedef int (*byid_t)(const char *, void **);
    typedef int (*state_t)(void *, unsigned, int *);
    typedef int (*ver_t)(void *, unsigned, unsigned *);
    typedef int (*rtype_t)(void *, unsigned, int *);
    auto init = (init_t)dlsym(h, "nvmlInit_v2");
    auto shutdown = (init_t)dlsym(h, "nvmlShutdown");
    auto byid = (byid_t)dlsym(h, "nvmlDeviceGetHandleByPciBusId_v2");
    auto state = (state_t)dlsym(h, "nvmlDeviceGetNvLinkState");
    auto ver = (ver_t)dlsym(h, "nvmlDeviceGetNvLinkVersion");
    auto rtype = (rtype_t)dlsym(h, "nvmlDeviceGetNvLinkRemoteDeviceType");
    if (init && byid && state && init() == 0) {
        for (int d = 0; d < ndev; ++d) {
            char bus[32];
            void *dev = nullptr;
            if (cudaDeviceGetPCIBusId(bus, sizeof bus, d) != cudaSuccess || byid(bus, &dev) != 0) {
                cudaGetLastError();
                continue;
            }
            info[d].links = 0;
            for (unsigned l = 0; l < 18; ++l) {   // NVML_NVLINK_MAX_LINKS
                int active = 0;
                if (state(dev, l, &active) != 0 || active != 1) continue;   // NVML_FEATURE_ENABLED
                ++info[d].links;
                unsigned v = 0;
                if (ver && ver(dev, l, &v) == 0 && (int)v > info[d].version) info[d].version = (int)v;
                int t = 0;
                if (rtype && rtype(dev, l, &t) == 0 && t == 2) info[d].via_switch = true;   // ..._TYPE_SWITCH
            }
        }
        if (shutdown) shutdown();
    }
    dlclose(h);
    return info;
}

// NVML NVLink version enum -> generation ("5.0" on B200) and per-link GB/s per direction
std::string nvlink_gen(int v) {
    static const char *g[] = {"", "1.0", "2.0", "2.2", "3.0", "3.1", "4.0", "5.0"};
    return v > 0 && v < 8 ? g[v] : std::to_string(v);
}
int nvlink_gbs(int v) { return v == 7 ? 50 : (v == 6 || v == 4 || v == 5) ? 25 : 0; }

}  // namespace pdlrt

// the C ABI is the only exported surface (built with -fvisibility=hidden)
#pragma GCC visibility push(default)
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

int task_matmul_prepared(int dtype, const void *Aprep, const void *Araw, int64_t lda_raw, void *raw_ready,
                         const void *B, int64_t ldb, void *C, int64_t ldc, int64_t M, int64_t N, int64_t K,
                         unsigned flags) {
    int rc = check_loaded();
    if (rc) return rc;
    if (dtype != PDL_F64 && dtype != PDL_F32) return set_err(PDL_EINVAL, "unknown dtype %d", dtype);
    if (M < 0 || N < 0 || K < 0 || lda_raw < 0 || ldb < 0 || ldc < 0) return set_err(PDL_EINVAL, "negative size");
    if (flags & ~(PDL_TASK_REUSE_B | PDL_TASK_GRAPH | PDL_TASK_SLOT(3)))
        return set_err(PDL_EINVAL, "task_matmul_prepared: flags may be PDL_TASK_REUSE_B | PDL_TASK_GRAPH | "
                                   "PDL_TASK_SLOT(s) (got 0x%x)", flags);
    if (((flags >> 4) & 3u) >= 3u) return set_err(PDL_EINVAL, "scratch slot %u out of range (0..2)", (flags >> 4) & 3u);
    if (M == 0 || N == 0) return PDL_OK;
    if (!C || (K > 0 && (!Aprep || !B))) return set_err(PDL_EINVAL, "Aprep, B or C is NULL with nonzero sizes");
    const int64_t ldb_ = ldb ? ldb : N, ldc_ = ldc ? ldc : N, ldr = lda_raw ? lda_raw : K;
    if (ldb_ < N || ldc_ < N || (Araw && ldr < K)) return set_err(PDL_EINVAL, "leading dimension smaller than the row width");
    Task t{dtype, Aprep, 0, B, ldb_, C, ldc_, M, N, K, 0, false, "", flags | PDL_TASK_LOCAL | PDL_TASK_PREPARED_A,
           DistSpec()};
    t.Araw = Araw;
    t.lda_raw = ldr;
    t.raw_ready = raw_ready;
    g->queue.push_back(t);
    return PDL_OK;
}

int pdl_run(void) { return execute(true); }

int pdl_run_async(void) { return execute(false); }

int pdl_sync(void) {
    int rc = check_loaded();
    if (rc) return rc;
    if (g->dry_run) return PDL_OK;
    int launches = 0;
    // PDL_SYNC_TIMEOUT_MS = t > 0: give up after t ms instead of blocking (a hung
    // Worker<->Worker transfer or kernel); the device work stays in flight and the
    // platform must be unloaded.  An unfinished exchange -> PDL_ENCCL.
    const char *te = getenv("PDL_SYNC_TIMEOUT_MS");
    const double tmo = te ? atof(te) : 0.0;
    const auto t0 = std::chrono::steady_clock::now();
    for (auto &w : g->workers) {
        CUDA_TRY(cudaSetDevice(w.device));
        cudaError_t e;
        if (tmo > 0) {
            while ((e = cudaStreamQuery(w.stream)) == cudaErrorNotReady) {
                const double ms =
                    std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
                if (ms > tmo) {
                    if (w.xpending && w.ev_xdone && cudaEventQuery(w.ev_xdone) == cudaErrorNotReady)
                        return set_err(PDL_ENCCL,
                                       "Worker<->Worker exchange into Worker %s (device %d) did not complete "
                                       "within %.0f ms",
                                       g->model.pus[w.pu].id.c_str(), w.device, tmo);
                    cudaGetLastError();
                    return set_err(PDL_ECUDA, "device work of Worker %s (device %d) did not complete within %.0f ms",
                                   g->model.pus[w.pu].id.c_str(), w.device, tmo);
                }
                usleep(50);
            }
        } else {
            e = cudaStreamSynchronize(w.stream);
        }
        if (e != cudaSuccess) {
            const bool xfail = w.xpending && w.ev_xdone && cudaEventQuery(w.ev_xdone) != cudaSuccess;
            return set_err(xfail ? PDL_ENCCL : PDL_ECUDA, "device work failed on device %d%s: %s", w.device,
                           xfail ? " (Worker<->Worker exchange)" : "", cudaGetErrorString(e));
        }
        w.xpending = false;
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
    if (w.gctx) {
        // an SM-partition Worker keeps its green-context stream (replacing it would
        // drop the partition); runs join the caller's stream on both sides instead
        w.join_stream = (cudaStream_t)stream;
        return PDL_OK;
    }
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
        o << "],\"M\":\"" << dec(P.Mw[0], P.Mw[1]) << "\",\"crt\":\"" << (pdlk::oz2_crt_fast_ok(P) ? "fp64" : "int")
          << "\"}";
        res = o.str();
    } else if (k.rfind("ozaki2_launches/", 0) == 0) {
        // "ozaki2_launches/<rows>/<cols>/<moduli>/<clusters>": persistent K6 launches
        // per K chunk and the moduli of each (host arithmetic, no device)
        long long rows = 0, cols = 0;
        int n = 0, cl = 0;
        if (sscanf(k.c_str() + 16, "%lld/%lld/%d/%d", &rows, &cols, &n, &cl) != 4 || rows < 0 || cols < 0 || n < 1 ||
            n > pdlk::OZ2_MAX_MODULI || cl < 1)
            return set_err(PDL_EINVAL, "bad key '%s' (ozaki2_launches/<rows>/<cols>/<moduli>/<clusters>)", key);
        const int nl = pdlk::oz2_launches_per_chunk(n, rows, cols, cl);
        std::ostringstream o;
        o << "[";
        for (int l = 0; l < nl; ++l) o << (l ? "," : "") << (l + 1) * n / nl - l * n / nl;
        o << "]";
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
        else if (k == "exchange_path" || k.rfind("exchange_path/", 0) == 0) {
            // the Worker<->Worker transfer path the descriptor allows for a group
            // (L1336-1341: paths are derived from the explicit interconnects):
            // "direct" when every pair of its gpu Workers is joined by an
            // Interconnect (NVLink on a B200 box), else "host" (through the
            // Master's memory region, over the Master<->Worker interconnects)
            const std::string grp = k.size() > 14 ? k.substr(14) : std::string();
            std::vector<int> gw = m.group_workers(grp.empty() ? nullptr : grp.c_str());
            bool direct = true;
            for (size_t i = 0; i < gw.size() && direct; ++i)
                for (size_t j = i + 1; j < gw.size() && direct; ++j) direct = m.ic_between(gw[i], gw[j], "");
            res = direct ? "direct" : "host";
        }
        else if (k == "concurrent_tasks/f64" || k == "concurrent_tasks/f32") {
            // whether two tasks on device-resident, 16-byte aligned operands may
            // run at once on different streams of a local Worker when they use
            // different scratch slots (PDL_TASK_SLOT): every task variant keeps its
            // per-task buffers per slot, and a REUSE_B task waits for the B
            // preparation on the other stream (a task re-preparing B there -- e.g.
            // after a graph replay of the first task -- waits for the last B-using
            // task).  SM-partition Workers keep their one green-context stream, so
            // their tasks serialise: "no"
            bool any_green = false;
            for (auto &w : g->workers) any_green |= w.gctx != nullptr;
            res = g->workers.empty() || any_green ? "no" : "yes";
        }
        else if (k.rfind("prepared_a/", 0) == 0) {
            // "prepared_a/<f64|f32>/<K>": bytes per prepared A row (PDL_TASK_PREP_A) of
            // local Worker 0's task variant, 0 when it exchanges raw rows
            char dts[8] = {0};
            long long K = -1;
            if (sscanf(k.c_str() + 11, "%3[^/]/%lld", dts, &K) != 2 || K < 0 ||
                (strcmp(dts, "f64") && strcmp(dts, "f32")))
                return set_err(PDL_EINVAL, "bad key '%s' (prepared_a/<f64|f32>/<K>)", key);
            std::vector<int> gw = m.group_workers(nullptr);
            if (gw.empty()) return set_err(PDL_ENOWORKER, "no gpu Worker");
            const int pu = g->workers.empty() ? gw[0] : g->workers[0].pu;
            bool raw = false;
            const int64_t pr = prepared_a_row_bytes(pu, strcmp(dts, "f64") ? PDL_F32 : PDL_F64, K, &raw);
            // "<bytes>" or "<bytes>+raw" (the prepared task also reads the raw rows)
            res = std::to_string(pr) + (raw ? "+raw" : "");
        }
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
            // bytes moved along the interconnects in the last run, by path (the
            // descriptor's IC types: Master<->Worker, Worker<->Worker)
            std::string mw_ic, ww_ic;
            const std::vector<int> gws = m.all_gpu_workers();
            if (!gws.empty() && !m.masters.empty()) mw_ic = m.ic_type_between(m.masters[0], gws[0]);
            if (gws.size() > 1) ww_ic = m.ic_type_between(gws[0], gws[1]);
            o << ",\"transfers\":{\"master_to_worker\":" << g->xfer.m2w << ",\"worker_to_master\":" << g->xfer.w2m
              << ",\"worker_to_worker\":" << g->xfer.w2w << ",\"exchange_tasks\":" << g->xfer.exchange_tasks
              << ",\"master_worker_ic\":\"" << json_escape(mw_ic) << "\",\"worker_worker_ic\":\""
              << json_escape(ww_ic) << "\"}";
            // Ozaki-II certificate of the last run (valid after pdl_sync): 128 x 128 tiles
            // checked per Worker and those recomputed by K1 (R21)
            bool any_guard = false;
            for (auto &w : g->workers) any_guard |= w.guard_epoch == g->run_epoch;
            if (any_guard && !g->dry_run) {
                o << ",\"ozaki_guard\":[";
                bool f1 = true;
                for (auto &w : g->workers) {
                    if (w.guard_epoch != g->run_epoch) continue;
                    unsigned cnt[4] = {0, 0, 0, 0};
                    cudaSetDevice(w.device);
                    if (cudaMemcpy(cnt, w.buf[BUF_OZG].ptr, sizeof cnt, cudaMemcpyDeviceToHost) != cudaSuccess)
                        cudaGetLastError();
                    // certified_in_crt: CRT launches that certify sign-uniform rows / columns;
                    // certificate_gemms_skipped: certificate GEMM launches skipped because no
                    // row or column of theirs mixes signs (R23)
                    o << (f1 ? "" : ",") << "{\"id\":\"" << json_escape(m.pus[w.pu].id)
                      << "\",\"tiles_checked\":" << w.guard_tiles << ",\"tiles_recomputed\":" << cnt[0]
                      << ",\"elements_recomputed\":" << cnt[1] << ",\"certified_in_crt\":" << cnt[2]
                      << ",\"certificate_gemms_skipped\":" << cnt[3] << "}";
                    f1 = false;
                }
                o << "]";
            }
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
    const std::vector<NvLinkInfo> nvl = nvlink_topology(ndev);
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
        if (nvl[d].links >= 0) {
            prop(o, "NVLINK_LINKS", std::to_string(nvl[d].links), "", false);
            if (nvl[d].version) prop(o, "NVLINK_VERSION", nvlink_gen(nvl[d].version), "", false);
        }
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
            if (!can) continue;
            const bool sw = nvl[a].via_switch && nvl[b].via_switch;
            o << "  <Interconnect type=\"NVLink\" from=\"gpu" << a << "\" to=\"gpu" << b << "\" scheme=\""
              << (sw ? "switch" : "p2p") << "\"";
            const int links = std::min(nvl[a].links, nvl[b].links);
            if (links > 0) {
                // NVLink 5 (B200): 50 GB/s per direction per link
                o << ">\n    <ICDescriptor>\n";
                prop(o, "LINKS", std::to_string(links), "", false);
                const int per_link = nvlink_gbs(std::min(nvl[a].version, nvl[b].version));
                if (per_link) prop(o, "BANDWIDTH", std::to_string(per_link * links), "GB/s", false);
                o << "    </ICDescriptor>\n  </Interconnect>\n";
            } else {
                o << "/>\n";
            }
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
#pragma GCC visibility pop
