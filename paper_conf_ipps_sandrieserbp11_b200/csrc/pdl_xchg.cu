// pdl_xchg.cu -- the Worker<->Worker exchange of one process driving several
// Workers.
//
// PAPER.md SS IV-C step 3: "The PDL allows us to derive data-transfer paths
// between memory-regions and communication between processing-units via the
// explicitly specified interconnect entity" (L1336-1341); Interconnects are the
// explicit communication facilities between PUs (SS III-A, L591-603).  When the
// descriptor joins every pair of the group's Workers by an Interconnect (the
// shipped B200 descriptors: NVLink with from == to on the replicated Worker,
// reading R8), the operands in the Master's memory region cross the
// Master->Worker interconnect (PCIe) ONCE: Worker (r, c) of the Gr x Gc BLOCK
// grid receives only its unique chunk -- chunk c (qa rows) of A's row-panel r
// and chunk r (qb K-rows) of B's column-panel c -- and the Workers then pull the
// other chunks of their panels from each other over the Worker<->Worker
// interconnect (cudaMemcpyPeerAsync: copy engines over NVLink, no SMs taken
// from the tile kernels).  Compute overlaps the exchange: the B panel first,
// then the Worker's own A chunk computes at once and the chunks before / after
// it as they land (three launches, the order of runtime.exchange_overlapped).
// Without such an interconnect every Worker stages its whole panels from the
// Master's memory region (run_rect), the path through the Master.
//
// PCIe bytes (Master -> Workers) = (M K + K N) s in total, each operand byte
// once; NVLink bytes per Worker = (Gc - 1) qa K s + (Gr - 1) qb cols s.  Every
// C element is computed by one kernel over the full K in the kernel's fixed
// order, so C is bitwise the G = 1 result (R14).
#include "pdl_rt.hpp"

namespace pdlrt {

static cudaEvent_t xev(WorkerCtx &w, size_t &next) {
    if (next >= w.xev_pool.size()) {
        cudaEvent_t e = nullptr;
        if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return nullptr;
        w.xev_pool.push_back(e);
    }
    return w.xev_pool[next++];
}

bool exchange_applies(const Task &t, const Plan &plan, const std::vector<int> &gw) {
    const char *e = getenv("PDL_EXCHANGE");
    if (e && !strcmp(e, "0")) return false;
    if (g->nranks != 1 || (t.flags & (PDL_TASK_PANELS | PDL_TASK_LOCAL)) || t.dist.kind != Dist::Block) return false;
    if (plan.hierarchical() || plan.G < 2 || (plan.Gr == 1 && plan.Gc == 1) || t.K <= 0) return false;
    // operands in the Master's memory region (device operands are read in place)
    if (locate(t.A) >= 0 || locate(t.B) >= 0) return false;
    // a Worker<->Worker interconnect joins every pair of the group
    for (size_t i = 0; i < gw.size(); ++i)
        for (size_t j = i + 1; j < gw.size(); ++j)
            if (!g->model.ic_between(gw[i], gw[j], "")) return false;
    // every group Worker is driven by this process
    for (int pu : gw) {
        bool bound = false;
        for (auto &w : g->workers) bound |= w.pu == pu;
        if (!bound) return false;
    }
    return true;
}

namespace {
struct XW {
    WorkerCtx *w = nullptr;
    int r = 0, c = 0;
    Rect R;
    int64_t rows = 0, cols = 0, qa = 0, qb = 0, ldk = 0, ldn = 0;
    char *xa = nullptr, *xb = nullptr;
    cudaEvent_t own = nullptr, bdone = nullptr;
    std::vector<cudaEvent_t> a_ev;   // per A chunk of the row-panel: landed here
    size_t evn = 0;
};
}  // namespace

int run_exchange(const Task &t, const Plan &plan, const std::vector<int> &gw) {
    NvtxRange nv("worker<->worker exchange");
    const int G = (int)gw.size();
    const int es = t.dtype == PDL_F64 ? 8 : 4, pe = 16 / es;
    const int64_t K = t.K;
    std::vector<XW> X(G);
    for (int gi = 0; gi < G; ++gi) {
        for (auto &w : g->workers)
            if (w.pu == gw[gi]) X[gi].w = &w;
        XW &x = X[gi];
        x.r = gi / plan.Gc;
        x.c = gi % plan.Gc;
        x.R = plan.rect(gi);
        x.rows = x.R.row1 - x.R.row0;
        x.cols = x.R.col1 - x.R.col0;
        x.qa = plan.qa(gi);
        x.qb = plan.qb();
        x.ldk = round_up(K, pe);
        x.ldn = round_up(std::max<int64_t>(x.cols, 1), pe);
    }
    // Panel buffers in each Worker's memory region.  A buffer that must grow may
    // still be read by a peer's copy of the previous run: wait for every Worker.
    bool grow = false;
    for (auto &x : X)
        grow |= x.w->buf[BUF_XA].bytes < (size_t)(plan.Gc * x.qa * x.ldk * es) ||
                x.w->buf[BUF_XB].bytes < (size_t)(plan.Gr * x.qb * x.ldn * es);
    if (grow)
        for (auto &x : X) {
            CUDA_TRY(cudaSetDevice(x.w->device));
            CUDA_TRY(cudaDeviceSynchronize());
        }
    for (auto &x : X) {
        WorkerCtx &w = *x.w;
        CUDA_TRY(cudaSetDevice(w.device));
        void *p = nullptr;
        int rc;
        if ((rc = ensure_buf(w, BUF_XA, (size_t)(std::max<int64_t>(1, plan.Gc * x.qa) * x.ldk * es), &p))) return rc;
        x.xa = (char *)p;
        if ((rc = ensure_buf(w, BUF_XB, (size_t)(std::max<int64_t>(1, plan.Gr * x.qb) * x.ldn * es), &p))) return rc;
        x.xb = (char *)p;
        if (!w.xs) CUDA_TRY(cudaStreamCreateWithFlags(&w.xs, cudaStreamNonBlocking));
        x.own = xev(w, x.evn);
        x.bdone = xev(w, x.evn);
        if (!w.ev_xdone) CUDA_TRY(cudaEventCreateWithFlags(&w.ev_xdone, cudaEventDisableTiming));
        x.a_ev.assign(plan.Gc, nullptr);
        for (int j = 0; j < plan.Gc; ++j)
            if (!(x.a_ev[j] = xev(w, x.evn))) return set_err(PDL_ECUDA, "event create failed");
        if (!x.own || !x.bdone) return set_err(PDL_ECUDA, "event create failed");
        // the copy stream starts after the Worker's earlier work (which may read the panels)
        cudaEvent_t start = xev(w, x.evn);
        if (!start) return set_err(PDL_ECUDA, "event create failed");
        CUDA_TRY(cudaEventRecord(start, w.stream));
        CUDA_TRY(cudaStreamWaitEvent(w.xs, start, 0));
    }
    // Peer access between the devices of the group (direct copies over NVLink);
    // a pair without it still copies, staged by the driver.
    for (auto &a : X)
        for (auto &b : X)
            if (a.w->device != b.w->device && enable_peer(a.w->device, b.w->device) != PDL_OK) g_err.clear();

    // (1) unique chunks: Master MR -> Worker MR over the Master->Worker interconnect
    for (auto &x : X) {
        WorkerCtx &w = *x.w;
        CUDA_TRY(cudaSetDevice(w.device));
        const int64_t a0 = std::min(x.c * x.qa, x.rows), a1 = std::min(a0 + x.qa, x.rows);
        const int64_t b0 = std::min(x.r * x.qb, K), b1 = std::min(b0 + x.qb, K);
        if (a1 > a0) {
            cudaError_t e = cudaMemcpy2DAsync(x.xa + (size_t)(a0 * x.ldk) * es, (size_t)(x.ldk * es),
                                              (const char *)t.A + (size_t)((x.R.row0 + a0) * t.lda) * es,
                                              (size_t)(t.lda * es), (size_t)(K * es), (size_t)(a1 - a0),
                                              cudaMemcpyDefault, w.xs);
            if (e != cudaSuccess) return set_err(PDL_ECUDA, "A chunk staging failed: %s", cudaGetErrorString(e));
            g->xfer.count(-1, w.device, (a1 - a0) * K * es);
        }
        if (b1 > b0 && x.cols > 0) {
            cudaError_t e = cudaMemcpy2DAsync(x.xb + (size_t)(b0 * x.ldn) * es, (size_t)(x.ldn * es),
                                              (const char *)t.B + (size_t)(b0 * t.ldb + x.R.col0) * es,
                                              (size_t)(t.ldb * es), (size_t)(x.cols * es), (size_t)(b1 - b0),
                                              cudaMemcpyDefault, w.xs);
            if (e != cudaSuccess) return set_err(PDL_ECUDA, "B chunk staging failed: %s", cudaGetErrorString(e));
            g->xfer.count(-1, w.device, (b1 - b0) * x.cols * es);
        }
        CUDA_TRY(cudaEventRecord(x.own, w.xs));
    }

    // (2) panels: Worker MR <- peer Worker MRs over the Worker<->Worker interconnect
    for (auto &x : X) {
        WorkerCtx &w = *x.w;
        CUDA_TRY(cudaSetDevice(w.device));
        // B chunks of the column-panel from the grid column (every C row needs them)
        for (int r2 = 0; r2 < plan.Gr; ++r2) {
            if (r2 == x.r) continue;
            XW &s = X[r2 * plan.Gc + x.c];
            const int64_t b0 = std::min(r2 * x.qb, K), b1 = std::min(b0 + x.qb, K);
            if (b1 <= b0 || x.cols <= 0) continue;
            CUDA_TRY(cudaStreamWaitEvent(w.xs, s.own, 0));
            const size_t off = (size_t)(b0 * x.ldn) * es, bytes = (size_t)((b1 - b0) * x.ldn) * es;
            cudaError_t e = cudaMemcpyPeerAsync(x.xb + off, w.device, s.xb + off, s.w->device, bytes, w.xs);
            if (e != cudaSuccess)
                return set_err(PDL_ENCCL, "exchange: B chunk %d -> Worker %s failed: %s", r2,
                               g->model.pus[w.pu].id.c_str(), cudaGetErrorString(e));
            g->xfer.count(s.w->device, w.device, (b1 - b0) * x.cols * es);
        }
        CUDA_TRY(cudaEventRecord(x.bdone, w.xs));
        // A chunks of the row-panel from the grid row: the chunks before this
        // Worker's, then the ones after it (the order they are computed in)
        for (int pass = 0; pass < 2; ++pass)
            for (int j = pass ? x.c + 1 : 0; j < (pass ? plan.Gc : x.c); ++j) {
                XW &s = X[x.r * plan.Gc + j];
                const int64_t a0 = std::min(j * x.qa, x.rows), a1 = std::min(a0 + x.qa, x.rows);
                if (a1 > a0) {
                    CUDA_TRY(cudaStreamWaitEvent(w.xs, s.own, 0));
                    const size_t off = (size_t)(a0 * x.ldk) * es, bytes = (size_t)((a1 - a0) * x.ldk) * es;
                    cudaError_t e = cudaMemcpyPeerAsync(x.xa + off, w.device, s.xa + off, s.w->device, bytes, w.xs);
                    if (e != cudaSuccess)
                        return set_err(PDL_ENCCL, "exchange: A chunk %d -> Worker %s failed: %s", j,
                                       g->model.pus[w.pu].id.c_str(), cudaGetErrorString(e));
                    g->xfer.count(s.w->device, w.device, (a1 - a0) * K * es);
                }
                CUDA_TRY(cudaEventRecord(x.a_ev[j], w.xs));
            }
        CUDA_TRY(cudaEventRecord(w.ev_xdone, w.xs));
        w.xpending = true;
    }

    // (3) tile tasks: own chunk at once, then the chunks before / after it as they land
    for (auto &x : X) {
        WorkerCtx &w = *x.w;
        CUDA_TRY(cudaSetDevice(w.device));
        CUDA_TRY(cudaStreamWaitEvent(w.stream, x.own, 0));
        CUDA_TRY(cudaStreamWaitEvent(w.stream, x.bdone, 0));
        const int groups[3][2] = {{x.c, x.c + 1}, {0, x.c}, {x.c + 1, plan.Gc}};
        bool first = true;
        for (auto &gr : groups) {
            const int64_t lo = std::min(gr[0] * x.qa, x.rows), hi = std::min(gr[1] * x.qa, x.rows);
            if (hi <= lo || x.cols <= 0) continue;
            for (int j = gr[0]; j < gr[1]; ++j)
                if (j != x.c) CUDA_TRY(cudaStreamWaitEvent(w.stream, x.a_ev[j], 0));
            Task tl = t;
            tl.lda = x.ldk;
            tl.ldb = x.ldn;
            tl.flags = t.flags | (first ? 0u : PDL_TASK_REUSE_B);
            char *Cw = (char *)t.C + (size_t)((x.R.row0 + lo) * t.ldc + x.R.col0) * es;
            int rc = run_rect_g(w, tl, x.xa + (size_t)(lo * x.ldk) * es, x.xb, Cw, hi - lo, x.cols);
            if (rc) return rc;
            first = false;
        }
        // the Worker stream completes after every exchange copy of this Worker
        CUDA_TRY(cudaStreamWaitEvent(w.stream, w.ev_xdone, 0));
    }
    g->xfer.exchange_tasks += 1;
    return PDL_OK;
}

}  // namespace pdlrt
