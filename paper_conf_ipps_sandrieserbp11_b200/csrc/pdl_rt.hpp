// pdl_rt.hpp -- internal state and interfaces of the libpdl task runtime
// (pdl_runtime.cu: C ABI, loading, task queue; pdl_devices.cu: device binding,
// SM partitions, Worker memory regions; pdl_exec.cu: mapping execution, staging
// pipeline, task variants, DYNAMIC, CUDA graphs).  Not part of the public ABI.
#pragma once
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

#include <dlfcn.h>
#include <unistd.h>

#include <nvtx3/nvToolsExt.h>

#include "../../include/libpdl.h"
#include "kernels.h"
#include "pdl_model.hpp"
#include "pdl_xml.hpp"

namespace pdlrt {

using namespace pdl;

// NVTX range for profilers (nsys / ncu --nvtx): header-only NVTX v3, a no-op unless a
// tool injects itself (SURVEY.md SS5 tracing).  Ranges: pdl_run, each task, each
// Worker rectangle, the Worker<->Worker exchange, DYNAMIC, A preparation.
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    NvtxRange(const char *fmt, long long a, long long b, long long c) {
        char buf[96];
        snprintf(buf, sizeof buf, fmt, a, b, c);
        nvtxRangePushA(buf);
    }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange &) = delete;
    NvtxRange &operator=(const NvtxRange &) = delete;
};

extern thread_local std::string g_err;
int set_err(int code, const char *fmt, ...);
void logf(int level, const char *fmt, ...);
bool env_on(const char *name);

// A library-owned device buffer in a Worker's memory region, reused across runs.
struct DevBuf {
    void *ptr = nullptr;
    size_t bytes = 0;
};

enum BufSlot { BUF_A = 0, BUF_B, BUF_C, BUF_AHI, BUF_ALO, BUF_BHI, BUF_BLO, BUF_OZA, BUF_OZB, BUF_OZE, BUF_OZR,
               BUF_XA, BUF_XB,   // A row-panel / B column-panel gathered by the Worker<->Worker exchange
               BUF_OZF, BUF_OZM, BUF_OZG,   // Ozaki-II certificate: tile flags, element mask (per slot), counters
               BUF_COUNT };
// Scratch slots (PDL_TASK_SLOT): the per-task buffers (A staging, C staging, A
// split / slices / residues, A exponents, residue planes) exist once per slot, so
// tasks of different slots may run at once on different streams of the Worker;
// the B-side buffers (the prepared B of PDL_TASK_REUSE_B) are shared.
constexpr int kTaskSlots = 3;
inline int slot_buf(int buf, int slot) {
    return (buf == BUF_B || buf == BUF_BHI || buf == BUF_BLO || buf == BUF_OZB) ? buf : buf + slot * BUF_COUNT;
}

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
    DevBuf buf[BUF_COUNT * kTaskSlots];
    cudaEvent_t ev_bprep = nullptr;   // after the last B preparation (REUSE_B tasks on other streams wait)
    cudaEvent_t ev_blast = nullptr;   // after the last task that used the shared B-side buffers (a task
                                      // re-preparing B on another stream waits for it)
    // the caller's stream (pdl_set_stream) of a green-context Worker: the Worker
    // keeps its partition's stream and joins this one around every run
    cudaStream_t join_stream = nullptr;   // nullptr = cudaStreamLegacy
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
    };
    BSig bsig;
    long long bsig_gen = 0;   // bumped whenever a task writes the B-side buffers
    // CUDA graphs of repeated tasks (PDL_TASK_GRAPH / PDL_GRAPH=1): signature -> graph
    struct GraphEntry {
        cudaGraphExec_t exec = nullptr;
        std::vector<cudaEvent_t> events;                              // owned; recorded by the graph
        std::vector<std::pair<cudaEvent_t, cudaEvent_t>> kt_pairs;
        int launches = 0;
        bool timed = false;
        BSig bsig;            // the prepared B the captured task leaves in the B-side buffers
        bool uses_b = false;  // the captured task writes the B-side buffers
    };
    std::map<std::string, GraphEntry> graphs;
    std::map<std::string, int> graph_seen;   // signatures run once (captured on the next run)
    int buf_gen = 0;                         // bumped when a buffer is reallocated (graphs go stale)
    bool capturing = false;
    long long graph_replays = 0;
    // pipelined staging: copy-in, copy-out, second compute stream; reusable events
    cudaStream_t aux[3] = {nullptr, nullptr, nullptr};
    std::vector<cudaEvent_t> ev_pool;
    // Worker<->Worker exchange (pdl_xchg.cu): its copy stream, events, and the
    // event after the last exchange copy of the last run (sync timeouts)
    cudaStream_t xs = nullptr;
    std::vector<cudaEvent_t> xev_pool;
    cudaEvent_t ev_xdone = nullptr;
    bool xpending = false;
    // Ozaki-II certificate of the current run: tiles checked (host) and the device
    // counter of tiles recomputed by K1 (BUF_OZG), reset at the first use in a run
    long long guard_epoch = -1, guard_tiles = 0;
};

constexpr size_t kMaxKernelTimes = 4096;

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
    // task_matmul_prepared: the raw A rows a prepared task still reads (the
    // Ozaki-II certificate's K1 recompute) and the event that makes them ready
    const void *Araw = nullptr;
    int64_t lda_raw = 0;
    void *raw_ready = nullptr;
};

// Bytes moved along the descriptor's interconnects in the last run (pdl_query
// "stats"): Master MR <-> Worker MR (host staging, gather) and Worker MR <->
// Worker MR (the exchange, and device operands read by another device's Worker).
struct XferStats {
    long long m2w = 0, w2m = 0, w2w = 0;
    int exchange_tasks = 0;   // tasks that ran the Worker<->Worker exchange
    void count(int src_dev, int dst_dev, long long bytes) {
        if (src_dev < 0 && dst_dev >= 0) m2w += bytes;
        else if (src_dev >= 0 && dst_dev < 0) w2m += bytes;
        else if (src_dev >= 0 && dst_dev >= 0) w2w += bytes;
    }
};

struct State {
    bool loaded = false;
    XferStats xfer;
    long long run_epoch = 0;   // pdl_run / pdl_run_async calls since pdl_load
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

extern State *g;
extern const char *kVersion;

#define CUDA_TRY(call)                                                                                   \
    do {                                                                                                 \
        cudaError_t _e = (call);                                                                         \
        if (_e != cudaSuccess) return set_err(PDL_ECUDA, "%s failed: %s", #call, cudaGetErrorString(_e)); \
    } while (0)

inline int64_t round_up(int64_t x, int64_t m) { return (x + m - 1) / m * m; }

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

// pdl_runtime.cu
std::string read_descriptor(const char *d, bool *ok);
int check_loaded();
// pdl_devices.cu
int get_encoder(pdlk::EncodeTiledFn *out);
const GreenApi *green_api();
int worker_stream(const WorkerCtx &w, cudaStream_t *out, bool blocking);
int make_partitions();
void fill_props(int pu, const cudaDeviceProp &p);
int bind_devices();
void free_state();
int ensure_buf(WorkerCtx &w, int slot, size_t bytes, void **out);
int locate(const void *p);
bool overlaps(const void *a, size_t an, const void *b, size_t bn);
// pdl_exec.cu
int kt_mark(WorkerCtx &w, bool start, cudaStream_t st);
cudaEvent_t ev_get(WorkerCtx &w, size_t &next);
int ensure_aux(WorkerCtx &w);
bool worker_ozaki(const WorkerCtx &w, bool f64, int *slices, int *rn);
bool worker_ozaki2(const WorkerCtx &w, int *nmod, int *bits);
bool worker_sgemm_ozaki2(const WorkerCtx &w);
int worker_sgemm_mix(const WorkerCtx &w);
int run_rect(WorkerCtx &w, const Task &t, const void *A, const void *B, void *C, int64_t rows, int64_t cols);
int run_dynamic(const Task &t, const std::vector<int> &gw);
int run_rect_g(WorkerCtx &w, const Task &t, const void *A, const void *B, void *C, int64_t rows, int64_t cols);
int execute(bool sync);
int enable_peer(int from, int to);
int64_t prepared_a_row_bytes(int pu, int dtype, int64_t K, bool *needs_raw = nullptr);
int run_prep_a(WorkerCtx &w, const Task &t);
// pdl_xchg.cu
bool exchange_applies(const Task &t, const Plan &plan, const std::vector<int> &gw);
int run_exchange(const Task &t, const Plan &plan, const std::vector<int> &gw);

}  // namespace pdlrt
