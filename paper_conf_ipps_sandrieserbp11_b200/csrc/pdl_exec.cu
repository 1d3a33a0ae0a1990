// pdl_exec.cu -- executing a mapped task on the Workers: the pipelined
// Master MR -> Worker MR staging of each Worker rectangle (PAPER.md SS IV-C step
// 3, L1328-1341), the PDL-selected task variants (task repository and static
// pre-selection, L1307-1326), the DYNAMIC distribution (dynamic schedulers,
// L1556-1562), CUDA-graph replay of repeated tasks, and the task loop of pdl_run.
#include "pdl_rt.hpp"

namespace pdlrt {

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

// The retired task variant "ozaki" (Ozaki scheme I, round 1's K4/K5): true when the
// Worker's PDL property DGEMM_VARIANT (FP64) / SGEMM_VARIANT (FP32), or env
// PDL_<NAME>, names it -- run_rect then reports PDL_EUNSUPPORTED.
bool worker_ozaki(const WorkerCtx &w, bool f64, int *slices, int *rn) {
    const char *vname = f64 ? "DGEMM_VARIANT" : "SGEMM_VARIANT";
    std::string v;
    if (const char *e = getenv((std::string("PDL_") + vname).c_str())) v = e;
    else if (const Property *p = g->model.prop(w.pu, vname)) v = p->value;
    *slices = 0;
    *rn = 1;
    return lower(trim(v)) == "ozaki";
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

// FP32 task variant of the Worker (PDL property SGEMM_VARIANT, env PDL_SGEMM_VARIANT):
// "tf32bf16" (default; R22: a_hi*b_hi in TF32 plus the two correction
// products in BF16 -- two TF32-equivalent tensor passes per K block) or "3xtf32"
// (three TF32 products, the round-1 default; split error ~2^-21 instead of <= 2^-17
// of |A||B|).  Returns 1 for tf32bf16, 0 for 3xtf32, -1 for a name this build does
// not know ("ozaki" / "ozaki2" are reported by their own checks).
int worker_sgemm_mix(const WorkerCtx &w) {
    std::string v;
    if (const char *e = getenv("PDL_SGEMM_VARIANT")) v = e;
    else if (const Property *p = g->model.prop(w.pu, "SGEMM_VARIANT")) v = p->value;
    v = lower(trim(v));
    if (v.empty() || v == "tf32bf16" || v == "default") return 1;
    if (v == "3xtf32" || v == "ozaki" || v == "ozaki2") return 0;
    return -1;
}

// Ozaki-II per-column arrays of a task: [bmax: cols u64][sb: cols u64][sbd: cols double]
// [fb: cols int][csign: cols u32][sbu: cols double] in the shared BUF_OZE (it does not move with `rows`, so
// a prepared B survives row-chunk tasks, REUSE_B).  The A side (residues, e_i, sa_i)
// lives in the packed prepared-A rows (pdlk::oz2_prep_row_bytes).  sb: the certificate's
// column sums; csign: each column's sign bits, sbu: the CRT certificate's column term (R23).
static int oz_b_arrays(WorkerCtx &w, int64_t cols, unsigned long long **bmax, int **fb, unsigned long long **sb,
                       double **sbd, unsigned **csign, double **sbu) {
    void *p = nullptr;
    int rc = ensure_buf(w, BUF_OZE, (size_t)cols * 32 + (size_t)round_up(cols, 2) * 8, &p);
    if (rc) return rc;
    *bmax = (unsigned long long *)p;
    *sb = *bmax + cols;
    *sbd = (double *)(*sb + cols);
    *fb = (int *)(*sbd + cols);
    *csign = (unsigned *)(*fb + round_up(cols, 2));
    *sbu = (double *)(*csign + round_up(cols, 2));
    return PDL_OK;
}

// R23: the certificate of sign-uniform rows and columns runs in the CRT pass when the
// plan reconstructs on the FP64-pipe pass (a property of the plan and the environment,
// never of the data, so the per-element decision is the same for any Worker count, tile
// and staging cut); PDL_OZ2_CERT_UNIFORM=0 turns it off.
static bool oz2_uniform_shortcut(const pdlk::Ozaki2Plan &P) {
    if (!P.check || !pdlk::oz2_crt_fast_ok(P)) return false;
    const char *crt = getenv("PDL_OZ2_CRT");
    if (crt && !strcmp(crt, "int")) return false;
    const char *e = getenv("PDL_OZ2_CERT_UNIFORM");
    return !(e && !strcmp(e, "0"));
}

// Certificate of the Ozaki-II variant (R21): PDL property OZAKI2_GUARD =
// "on" (default) | "off", OZAKI2_GUARD_TOL = tau (default 5e-13: the certified
// componentwise bound |C - AB| <= tau |A||B|, half the 1e-12 bar); env PDL_<NAME>.
static bool worker_oz2_guard(const WorkerCtx &w, double *tau) {
    std::string v;
    if (const char *e = getenv("PDL_OZAKI2_GUARD")) v = e;
    else if (const Property *p = g->model.prop(w.pu, "OZAKI2_GUARD")) v = p->value;
    *tau = 5e-13;
    if (const char *e = getenv("PDL_OZAKI2_GUARD_TOL")) *tau = atof(e);
    else if (const Property *p = g->model.prop(w.pu, "OZAKI2_GUARD_TOL")) *tau = atof(p->value.c_str());
    if (!(*tau > 0.0)) *tau = 5e-13;
    v = lower(trim(v));
    return !(v == "off" || v == "0" || v == "false");
}

// K2 shape for an nr x nc launch: the 1-SM 128 x 128 kernel when the CTA-pair
// grid of 256 x 256 tiles leaves TPCs idle, from a wave model with W = one pair
// tile's time: pairs ceil(p / (sms/2)) W, 1-SM ceil(t1 / sms) W / (2 e), e = the
// 1-SM kernel's per-SM rate relative to the pair's (0.8 measured at 4096^3 --
// 8192^3, tools/k1_shape_sweep.py f32; profiles/r01_k2_shape_sweep.jsonl).  Both
// give bitwise the same C (same K chunks and MMA order).
static bool k2_pick_1sm(int64_t nr, int64_t nc, int sms) {
    if (sms < 2) return false;
    const int64_t p = ((nr + 255) / 256) * ((nc + 255) / 256), t1 = ((nr + 127) / 128) * ((nc + 127) / 128);
    const double w2 = (double)((p + sms / 2 - 1) / (sms / 2));
    const double w1 = (double)((t1 + sms - 1) / sms) / (2 * 0.8);
    return w1 < w2;
}

int run_rect(WorkerCtx &w, const Task &t, const void *A, const void *B, void *C, int64_t rows, int64_t cols) {
    if (rows <= 0 || cols <= 0) return PDL_OK;
    CUDA_TRY(cudaSetDevice(w.device));
    const int slot = (int)((t.flags >> 4) & 3u) % kTaskSlots;   // PDL_TASK_SLOT
    auto ensure = [&](int buf, size_t bytes, void **out) { return ensure_buf(w, slot_buf(buf, slot), bytes, out); };
    const int es = t.dtype == PDL_F64 ? 8 : 4;
    const bool f64 = t.dtype == PDL_F64;
    const int64_t K = t.K;
    const int64_t pe = 16 / es;   // elements per 16 bytes

    // Where the operands live and whether they must be staged into this Worker's MR.
    // PDL_TASK_PREPARED_A: A is a panel of prepared rows (PDL_TASK_PREP_A) in this
    // Worker's memory region, read in place
    const bool prepared = (t.flags & PDL_TASK_PREPARED_A) != 0;
    if (prepared && K > 0 && (locate(A) != w.device || ((uintptr_t)A % 16)))
        return set_err(PDL_EINVAL, "PDL_TASK_PREPARED_A: A must be 16-byte aligned memory of the Worker's device");
    const bool a_st = K > 0 && !prepared &&
                      (locate(A) != w.device || (f64 && (((uintptr_t)A % 16) || (t.lda * es) % 16)));
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
    // tuning overrides of the cut counts (PDL_PIPE_RB / PDL_PIPE_CP)
    if (RB * CP > 1 || force) {
        if (const char *e = getenv("PDL_PIPE_RB")) RB = std::max(1, atoi(e));
        if (const char *e = getenv("PDL_PIPE_CP")) CP = std::max(1, atoi(e));
    }
    std::vector<int64_t> rb(RB + 1), cp(CP + 1);
    for (int i = 0; i <= RB; ++i) rb[i] = std::min<int64_t>(rows, round_up((int64_t)i * rows / RB, 128));
    for (int j = 0; j <= CP; ++j) cp[j] = std::min<int64_t>(cols, round_up((int64_t)j * cols / CP, 128));
    rb[RB] = rows;
    cp[CP] = cols;
    // PDL_PIPE_FIRST=f / PDL_PIPE_FIRST_COL=f: the first row band / column panel is 1/f of
    // the others (the first kernel waits for less staging; the rest spreads over the
    // remaining bands / panels)
    auto shrink_first = [](std::vector<int64_t> &cut, int n, int64_t len, const char *name) {
        const char *e = getenv(name);
        if (n <= 1 || !e) return;
        const int f = std::max(1, atoi(e));
        const int64_t first = std::max<int64_t>(128, round_up(len / n / f, 128));
        cut[1] = std::min<int64_t>(len, first);
        for (int i = 2; i < n; ++i)
            cut[i] = std::min<int64_t>(len, round_up(first + (int64_t)(i - 1) * (len - first) / (n - 1), 128));
    };
    shrink_first(rb, RB, rows, "PDL_PIPE_FIRST");
    shrink_first(cp, CP, cols, "PDL_PIPE_FIRST_COL");
    const bool piped = RB * CP > 1;
    // Task variant of this Worker, pre-selected from its PDL properties (task
    // repository + static pre-selection, L1307-1326): FP64 K1 (DMMA) or K6/K7
    // (Ozaki scheme II with its certificate), FP32 K3+K2 (TF32+BF16 or 3xTF32).
    int oz2_nmod = 0, oz2_bits = 0;
    if (K > 0 && (f64 ? false : worker_sgemm_ozaki2(w)))
        return set_err(PDL_EUNSUPPORTED, "SGEMM_VARIANT ozaki2: Ozaki scheme II is an FP64 variant");
    {
        int sl = 0, rn = 0;
        if (K > 0 && worker_ozaki(w, f64, &sl, &rn))
            return set_err(PDL_EUNSUPPORTED,
                           "%s_VARIANT ozaki (Ozaki scheme I) is retired: its dropped slice products bound the "
                           "error only by %s of K max|a| max|b|, which cannot certify the componentwise bar; use %s",
                           f64 ? "DGEMM" : "SGEMM", f64 ? "~2^-42" : "~2^-21",
                           f64 ? "DGEMM_VARIANT=ozaki2 (certified, DESIGN.md R21) or dmma" : "tf32bf16 (default) or 3xtf32");
    }
    const int mix = (K > 0 && !f64) ? worker_sgemm_mix(w) : 0;
    if (mix < 0) return set_err(PDL_EINVAL, "SGEMM_VARIANT: unknown FP32 task variant (3xtf32 | tf32bf16)");
    bool ozaki2 = K > 0 && f64 && worker_ozaki2(w, &oz2_nmod, &oz2_bits);
    double oz2_tau = 0.0;
    const bool oz2_guard = ozaki2 && worker_oz2_guard(w, &oz2_tau);
    pdlk::Ozaki2Plan P2;
    if (ozaki2) {
        P2 = pdlk::ozaki2_plan(rows, cols, K, oz2_nmod, oz2_bits, oz2_guard);
        // the certificate needs one K chunk (K <= 65536): longer tasks run K1 (IEEE FP64)
        if (oz2_guard && !P2.check) ozaki2 = false;
    }
    // the prepared-B signature of this task (PDL_TASK_REUSE_B)
    WorkerCtx::BSig want;
    want.valid = true;
    want.B = B;
    want.ldb = t.ldb;
    want.K = K;
    want.cols = cols;
    want.dtype = t.dtype;
    want.oz = ozaki2 ? 2 + P2.check : 0;
    want.S = ozaki2 ? P2.n : 0;
    want.rn = ozaki2 ? P2.p : mix;
    const bool prep_b = K > 0 && (ozaki2 || !f64);
    // A task that re-prepares B while another task of this Worker may still read
    // the shared B-side buffers on another stream (a side-stream chunk task, slot
    // != 0, after the main task was replayed from a graph or ran on other
    // operands) waits for the last B-using task first (piped tasks here, before
    // their side streams fork; unpiped ones below, once b_ready is known).
    if (piped && prep_b && slot != 0 && w.ev_blast) CUDA_TRY(cudaStreamWaitEvent(w.stream, w.ev_blast, 0));
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
        if ((rc = ensure(BUF_A, (size_t)(lda * rows * es), &p))) return rc;
        Ad = (const char *)p;
    }
    if (b_st) {
        ldb = round_up(cols, pe);
        if ((rc = ensure_buf(w, BUF_B, (size_t)(ldb * K * es), &p))) return rc;
        Bd = (const char *)p;
    }
    if (c_st) {
        ldcd = round_up(cols, pe);
        if ((rc = ensure(BUF_C, (size_t)(ldcd * rows * es), &p))) return rc;
        Cd = (char *)p;
    }
    // FP32 split buffers (K-major hi/lo of A rows and of B^T rows)
    const int64_t Kp = round_up(std::max<int64_t>(K, 1), pdlk::K2_BK);
    float *ahi = nullptr, *alo = nullptr, *bhi = nullptr, *blo = nullptr;
    const int64_t lda_s = 2 * Kp;   // prepared A rows [hi: Kp][lo: Kp] (PDL_TASK_PREP_A layout)
    if (!f64 && K > 0) {
        if (prepared) {
            p = const_cast<void *>(A);
        } else if ((rc = ensure(BUF_AHI, (size_t)(rows * lda_s * 4), &p))) {
            return rc;
        }
        ahi = (float *)p;
        alo = ahi + Kp;
        if ((rc = ensure_buf(w, BUF_BHI, (size_t)(cols * Kp * 4), &p))) return rc;
        bhi = (float *)p;
        if ((rc = ensure_buf(w, BUF_BLO, (size_t)(cols * Kp * 4), &p))) return rc;
        blo = (float *)p;
    }
    pdlk::EncodeTiledFn enc = nullptr;
    if (K > 0 && (rc = get_encoder(&enc))) return rc;
    const char *k2v = getenv("PDL_K2");   // measurement knob: force "1sm" or "2sm"
    // wave models of the shape pickers see this Worker's SMs (its partition)
    pdlk::set_worker_sms(w.sm_limit);
    const int sms = pdlk::worker_sms();

    int8_t *a8 = nullptr, *b8 = nullptr;
    int *oz_ea = nullptr, *oz_fb = nullptr;
    unsigned long long *oz_bmax = nullptr, *oz_sa = nullptr, *oz_sb = nullptr;
    unsigned *oz_csign = nullptr, *oz_sign_words = nullptr;
    double *oz_sbu = nullptr, *oz_rowT = nullptr;
    double *oz_sbd = nullptr;
    uint8_t *oz2_R = nullptr;
    int64_t oz2_ldr = 0, oz2_plane = 0;
    pdlk::Oz2Guard G2;
    int64_t oz_pr = 0, oz_ea_ld = 1, oz_sa_ld = 1;
    if (ozaki2 && prepared && P2.check && !(t.Araw && locate(t.Araw) == w.device))
        return set_err(PDL_EINVAL, "prepared A with DGEMM_VARIANT=ozaki2: the certificate's K1 recompute reads "
                                   "the raw A rows -- pass them (task_matmul_prepared Araw, this Worker's device)");
    if (ozaki2) {
        // packed prepared-A rows: [residues: ld8][e_i: int][sign bits: u32 (R23)][sa_i: u64]
        oz_pr = pdlk::oz2_prep_row_bytes(P2);
        if (prepared) {
            p = const_cast<void *>(A);
        } else if ((rc = ensure(BUF_OZA, (size_t)(rows * oz_pr), &p))) {
            return rc;
        }
        a8 = (int8_t *)p;
        oz_ea = (int *)(a8 + P2.ld8);
        oz_sa = (unsigned long long *)(a8 + P2.ld8 + 8);
        oz_ea_ld = oz_pr / 4;
        oz_sa_ld = oz_pr / 8;
        if ((rc = ensure_buf(w, BUF_OZB, P2.b8_bytes, &p))) return rc;
        b8 = (int8_t *)p;
        if ((rc = oz_b_arrays(w, cols, &oz_bmax, &oz_fb, &oz_sb, &oz_sbd, &oz_csign, &oz_sbu))) return rc;
        oz2_ldr = round_up(cols, 16);
        oz2_plane = oz2_ldr * rows;
        if ((rc = ensure(BUF_OZR, (size_t)(oz2_plane * P2.n * P2.nch), &p))) return rc;
        oz2_R = (uint8_t *)p;
        if (P2.check) {
            // recompute flags of the rectangle's 128 x 128 tiles, and the Worker's
            // count of flagged tiles in this run (pdl_query "stats")
            G2.ldf = (cols + 127) / 128;
            const size_t fbytes = (size_t)round_up((int64_t)(((rows + 127) / 128) * G2.ldf * 4), 16);
            // + 16 bytes per band x panel launch (R23), after the tile flags: the "mixed signs"
            // word and the largest uniform column term
            // and the rows' bounds T_i (8 bytes per row)
            if ((rc = ensure(BUF_OZF, fbytes + (size_t)RB * CP * 16 + (size_t)rows * 8, &p))) return rc;
            G2.flags = (uint32_t *)p;
            if (oz2_uniform_shortcut(P2)) {
                oz_sign_words = (unsigned *)((char *)p + fbytes);
                oz_rowT = (double *)((char *)p + fbytes + (size_t)RB * CP * 16);
                G2.rsign = (const unsigned *)(oz_ea + 1);   // the packed rows' pad words
                G2.rsign_ld = oz_ea_ld;
                G2.csign = oz_csign;
            }
            G2.ldw = (cols + 31) / 32;
            if ((rc = ensure(BUF_OZM, (size_t)(rows * G2.ldw * 4), &p))) return rc;
            G2.emask = (uint32_t *)p;
            if ((rc = ensure_buf(w, BUF_OZG, 16, &p))) return rc;
            G2.fallback = (unsigned *)p;
            if (w.guard_epoch != g->run_epoch) {
                CUDA_TRY(cudaMemsetAsync(G2.fallback, 0, 16, w.stream));
                w.guard_epoch = g->run_epoch;
                w.guard_tiles = 0;
            }
            w.guard_tiles += ((rows + 127) / 128) * G2.ldf;
            G2.tau = oz2_tau;
        }
    }

    // B prepared by a previous task of this Worker (PDL_TASK_REUSE_B)?  Decided after
    // the buffers above are sized: a reallocated B-side buffer invalidates it.
    const bool b_ready = prep_b && (t.flags & PDL_TASK_REUSE_B) && !piped && !b_st && w.bsig == want;
    if (!piped && prep_b && !b_ready && slot != 0 && w.ev_blast)
        CUDA_TRY(cudaStreamWaitEvent(w.stream, w.ev_blast, 0));
    // a B prepared on another stream (a task of another slot): wait for it
    if (b_ready && w.ev_bprep) CUDA_TRY(cudaStreamWaitEvent(w.stream, w.ev_bprep, 0));
    auto mark_bprep = [&](cudaStream_t st) -> int {
        if (piped) return PDL_OK;
        if (!w.ev_bprep && cudaEventCreateWithFlags(&w.ev_bprep, cudaEventDisableTiming) != cudaSuccess)
            return PDL_ECUDA;
        return cudaEventRecord(w.ev_bprep, st) == cudaSuccess ? PDL_OK : PDL_ECUDA;
    };

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
            g->xfer.count(locate(A), w.device, nr * K * es);
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
                g->xfer.count(locate(B), w.device, nc * K * es);
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
                if (!a_prep[i] && prepared) {
                    a_prep[i] = 1;
                } else if (!a_prep[i]) {
                    a_prep[i] = 1;
                    e = pdlk::launch_ozaki2_split_a((const double *)(Ad + (size_t)(r0 * lda) * es), lda, nr, K, P2,
                                                    a8 + r0 * oz_pr, oz_ea + r0 * oz_ea_ld, cs, &w.launches,
                                                    oz_sa + r0 * oz_sa_ld, oz_pr, oz_ea_ld, oz_sa_ld,
                                                    (unsigned *)(oz_ea + r0 * oz_ea_ld) + 1);
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
                                                    b8 + c0 * P2.ld8, oz_fb + c0, oz_bmax + c0, cs, oz_sb + c0,
                                                    oz_csign + c0);
                    w.launches += 2;
                    if (e == cudaSuccess && mark_bprep(cs)) return set_err(PDL_ECUDA, "event record failed");
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
                // the certificate of this band / panel (r0, c0: multiples of 128)
                pdlk::Oz2Guard gs = G2;
                if (P2.check) {
                    gs.sa = oz_sa + r0 * oz_sa_ld;
                    gs.sa_ld = oz_sa_ld;
                    gs.sb = oz_sb + c0;
                    gs.sbd = oz_sbd + c0;
                    if (G2.rsign) {   // R23: this band's rows, this panel's columns, this launch's word
                        gs.rsign = G2.rsign + r0 * G2.rsign_ld;
                        gs.csign = G2.csign + c0;
                        gs.sign_word = oz_sign_words + 4 * (i * CP + j);
                        gs.sbmax = (unsigned long long *)(gs.sign_word + 2);
                        gs.rowT = oz_rowT + r0;
                        gs.sbu = oz_sbu + c0;
                    }
                    gs.flags = G2.flags + (r0 / 128) * G2.ldf + c0 / 128;
                    gs.emask = G2.emask + r0 * G2.ldw + c0 / 32;
                    e = cudaMemset2DAsync(gs.flags, (size_t)(G2.ldf * 4), 0, (size_t)((nc + 127) / 128) * 4,
                                          (size_t)((nr + 127) / 128), cs);
                    if (e == cudaSuccess)
                        e = cudaMemset2DAsync(gs.emask, (size_t)(G2.ldw * 4), 0, (size_t)((nc + 31) / 32) * 4,
                                              (size_t)nr, cs);
                }
                if (e == cudaSuccess)
                    e = pdlk::launch_ozaki2_gemm(enc, a8 + r0 * oz_pr, b8 + c0 * P2.ld8, P2, Rs, oz2_ldr, oz2_plane,
                                                 nr, nc, cs, &nl, P2.check ? &gs : nullptr, oz_pr);
                if (e == cudaSuccess)
                    e = pdlk::launch_ozaki2_reconstruct(Rs, oz2_ldr, oz2_plane, oz_ea + r0 * oz_ea_ld, oz_fb + c0, P2,
                                                        (double *)Cs, ldcd, nr, nc, cs, oz_ea_ld,
                                                        gs.rsign ? &gs : nullptr);
                // flagged tiles: recomputed by K1 over the same operands (IEEE FP64); a
                // prepared task reads the raw rows it was given, once they are ready
                const char *Ar = prepared ? (const char *)t.Araw : Ad;
                const int64_t ldr_raw = prepared ? t.lda_raw : lda;
                if (e == cudaSuccess && P2.check && prepared && t.raw_ready)
                    e = cudaStreamWaitEvent(cs, (cudaEvent_t)t.raw_ready, 0);
                if (e == cudaSuccess && P2.check) {
                    e = pdlk::launch_dgemm_k1(enc, (const double *)(Ar + (size_t)(r0 * ldr_raw) * es), ldr_raw,
                                              (const double *)(Bd + (size_t)c0 * es), ldb, (double *)Cs, ldcd, nr, nc,
                                              K, cs, nullptr, nullptr, gs.flags, G2.ldf, gs.emask, G2.ldw);
                    ++nl;
                }
                if (e == cudaSuccess && kt_mark(w, false, cs)) return set_err(PDL_ECUDA, "event record failed");
                w.launches += nl + 1;
            } else if (f64) {
                if (kt_mark(w, true, cs)) return set_err(PDL_ECUDA, "event record failed");
                e = pdlk::launch_dgemm_k1(enc, (const double *)(Ad + (size_t)(r0 * lda) * es), lda,
                                          (const double *)(Bd + (size_t)c0 * es), ldb, (double *)Cs, ldcd, nr, nc, K,
                                          cs);
                if (e == cudaSuccess && kt_mark(w, false, cs)) return set_err(PDL_ECUDA, "event record failed");
                w.launches += 1;
            } else {
                // K3 split of this band / panel once, shared by both compute streams
                if (!a_prep[i] && prepared) {
                    a_prep[i] = 1;
                } else if (!a_prep[i]) {
                    a_prep[i] = 1;
                    e = pdlk::launch_split_rows((const float *)(Ad + (size_t)(r0 * lda) * es), lda, nr, K,
                                                ahi + r0 * lda_s, alo + r0 * lda_s, Kp, cs, lda_s, mix);
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
                                                  blo + c0 * Kp, Kp, cs, mix);
                    w.launches += 1;
                    if (e == cudaSuccess && mark_bprep(cs)) return set_err(PDL_ECUDA, "event record failed");
                    if (piped) {
                        ev_sb[j] = ev_get(w, evn);
                        CUDA_TRY(cudaEventRecord(ev_sb[j], cs));
                    }
                } else if (ev_sb[j]) {
                    CUDA_TRY(cudaStreamWaitEvent(cs, ev_sb[j], 0));
                }
                if (e != cudaSuccess) return set_err(PDL_ECUDA, "K3 split launch failed: %s", cudaGetErrorString(e));
                if (kt_mark(w, true, cs)) return set_err(PDL_ECUDA, "event record failed");
                if (k2v ? !strcmp(k2v, "1sm") : k2_pick_1sm(nr, nc, sms))
                    e = pdlk::launch_gemm_3xtf32(enc, ahi + r0 * lda_s, alo + r0 * lda_s, bhi + c0 * Kp, blo + c0 * Kp,
                                                 Kp, (float *)Cs, ldcd, nr, nc, cs, lda_s, mix);
                else
                    e = pdlk::launch_gemm_3xtf32_2sm(enc, ahi + r0 * lda_s, alo + r0 * lda_s, bhi + c0 * Kp,
                                                     blo + c0 * Kp, Kp, (float *)Cs, ldcd, nr, nc, cs, nullptr, nullptr,
                                                     lda_s, mix);
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
                g->xfer.count(w.device, locate(C), nr * nc * es);
            }
            ++launch_idx;
        }
      }
    }
    if (prep_b) {
        // the B-side buffers now hold this task's prepared B (whole panel only when unpiped)
        w.bsig = want;
        w.bsig.valid = !piped && !b_st;
        ++w.bsig_gen;
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
    // end of this task's use of the B-side buffers (a graph replay records it
    // after the launch instead: an event recorded inside a capture is a graph node)
    if (prep_b && !w.capturing) {
        if (!w.ev_blast) CUDA_TRY(cudaEventCreateWithFlags(&w.ev_blast, cudaEventDisableTiming));
        CUDA_TRY(cudaEventRecord(w.ev_blast, w.stream));
    }
    return PDL_OK;
}

// Bytes per prepared A row (PDL_TASK_PREP_A) of the task variant of PU `pu` for
// inner dimension K, 0 when the variant exchanges raw rows: FP32 -> [TF32 hi: Kp
// floats][second plane: Kp floats (tf32bf16: BF16 [hi' | lo'] per 16-wide K block; 3xtf32:
// TF32 lo)]; FP64 ozaki2 -> [residues: ld8 bytes][e_i][sign bits][sa_i]
// (pdlk::oz2_prep_row_bytes), and its prepared tasks still read the raw rows
// (needs_raw: the certificate's K1 recompute); FP64 dmma -> 0.
int64_t prepared_a_row_bytes(int pu, int dtype, int64_t K, bool *needs_raw) {
    if (needs_raw) *needs_raw = false;
    if (K <= 0) return 0;
    WorkerCtx w;
    w.pu = pu;
    int sl, rn;
    if (worker_ozaki(w, dtype == PDL_F64, &sl, &rn)) return 0;
    if (dtype == PDL_F32) return worker_sgemm_ozaki2(w) ? 0 : 2 * round_up(K, pdlk::K2_BK) * 4;
    int nmod = 0, bits = 0;
    if (!worker_ozaki2(w, &nmod, &bits)) return 0;
    double tau = 0.0;
    const bool guard = worker_oz2_guard(w, &tau);
    const pdlk::Ozaki2Plan P = pdlk::ozaki2_plan(1, 1, K, nmod, bits, guard);
    if (guard && !P.check) return 0;   // runs K1: raw rows
    if (needs_raw) *needs_raw = P.check != 0;
    return pdlk::oz2_prep_row_bytes(P);
}

// PDL_TASK_PREP_A: the A preparation of the Worker's task variant for the task's M
// rows, written as packed prepared rows to C (this Worker's memory region, 16-byte
// aligned) -- the unit the multi-rank runtime exchanges instead of raw A chunks.
int run_prep_a(WorkerCtx &w, const Task &t) {
    NvtxRange nv("prepare A");
    CUDA_TRY(cudaSetDevice(w.device));
    const int64_t pr = prepared_a_row_bytes(w.pu, t.dtype, t.K);
    if (pr == 0)
        return set_err(PDL_EUNSUPPORTED, "PDL_TASK_PREP_A: this Worker's %s task variant has no A preparation",
                       t.dtype == PDL_F64 ? "FP64" : "FP32");
    if (locate(t.C) != w.device || ((uintptr_t)t.C % 16))
        return set_err(PDL_EINVAL, "PDL_TASK_PREP_A: the output must be 16-byte aligned memory of the Worker's device");
    const int es = t.dtype == PDL_F64 ? 8 : 4;
    const char *A = (const char *)t.A;
    int64_t lda = t.lda;
    if (locate(t.A) != w.device || ((uintptr_t)A % 16) || (lda * es) % 16) {   // stage into the Worker's MR
        void *p = nullptr;
        lda = round_up(t.K, 16 / es);
        int rc = ensure_buf(w, BUF_A, (size_t)(t.M * lda * es), &p);
        if (rc) return rc;
        CUDA_TRY(cudaMemcpy2DAsync(p, (size_t)(lda * es), t.A, (size_t)(t.lda * es), (size_t)(t.K * es), (size_t)t.M,
                                   cudaMemcpyDefault, w.stream));
        g->xfer.count(locate(t.A), w.device, t.M * t.K * es);
        A = (const char *)p;
    }
    pdlk::set_worker_sms(w.sm_limit);
    cudaError_t e;
    if (t.dtype == PDL_F32) {
        const int64_t Kp = round_up(t.K, pdlk::K2_BK);
        float *hi = (float *)t.C;
        const int mix = worker_sgemm_mix(w);
        if (mix < 0) return set_err(PDL_EINVAL, "SGEMM_VARIANT: unknown FP32 task variant (3xtf32 | tf32bf16)");
        e = pdlk::launch_split_rows((const float *)A, lda, t.M, t.K, hi, hi + Kp, Kp, w.stream, 2 * Kp, mix);
        w.launches += 1;
    } else {
        int nmod = 0, bits = 0;
        double tau = 0.0;
        worker_ozaki2(w, &nmod, &bits);
        const pdlk::Ozaki2Plan P = pdlk::ozaki2_plan(t.M, 1, t.K, nmod, bits, worker_oz2_guard(w, &tau));
        int8_t *a8 = (int8_t *)t.C;
        // the rows' sign bits (R23) go into the pad word after e_i and travel with the rows
        e = pdlk::launch_ozaki2_split_a((const double *)A, lda, t.M, t.K, P, a8, (int *)(a8 + P.ld8), w.stream,
                                        &w.launches, (unsigned long long *)(a8 + P.ld8 + 8), pr, pr / 4, pr / 8,
                                        (unsigned *)(a8 + P.ld8 + 4));
    }
    if (e != cudaSuccess) return set_err(PDL_ECUDA, "A preparation launch failed: %s", cudaGetErrorString(e));
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
    NvtxRange nv("DYNAMIC");
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
                           "DYNAMIC needs a single-launch task variant (dmma / 3xtf32); Worker %s runs an Ozaki "
                           "variant (residue GEMMs, CRT pass and certificate recompute)",
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
            pdlk::set_worker_sms(w.sm_limit);
            // the shared counter lives in the first Worker's memory region: a Worker on
            // another device reaches it only over a Worker<->Worker interconnect of the
            // descriptor (L1336-1341)
            if (w.device != own.device && !g->model.ic_between(w.pu, own.pu, ""))
                return set_err(PDL_EUNSUPPORTED,
                               "DYNAMIC: the descriptor joins Workers %s and %s by no interconnect "
                               "(the tile counter sits in %s's memory region)",
                               g->model.pus[w.pu].id.c_str(), g->model.pus[own.pu].id.c_str(),
                               g->model.pus[own.pu].id.c_str());
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
                const int mix = worker_sgemm_mix(w);
                if (mix < 0) return set_err(PDL_EINVAL, "SGEMM_VARIANT: unknown FP32 task variant (3xtf32 | tf32bf16)");
                e = pdlk::launch_split_rows((const float *)Ad, lda, M, K, buf4[0], buf4[1], Kp, w.stream, 0, mix);
                if (e == cudaSuccess)
                    e = pdlk::launch_split_cols_t((const float *)Bd, ldb, K, N, buf4[2], buf4[3], Kp, w.stream, mix);
                if (e != cudaSuccess) return set_err(PDL_ECUDA, "K3 split launch failed: %s", cudaGetErrorString(e));
                if (kt_mark(w, true, w.stream)) return set_err(PDL_ECUDA, "event record failed");
                e = pdlk::launch_gemm_3xtf32_2sm(enc, buf4[0], buf4[1], buf4[2], buf4[3], Kp, (float *)Cd, ldc, M, N,
                                                 w.stream, g->dyn, mine, 0, mix);
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
    NvtxRange nv("worker rect %lldx%lld (pu %lld)", (long long)rows, (long long)cols, (long long)w.pu);
    const bool want = (t.flags & PDL_TASK_GRAPH) || env_on("PDL_GRAPH");
    if (!want || (t.flags & PDL_TASK_REUSE_B) || t.raw_ready || g->dry_run || rows <= 0 || cols <= 0)
        return run_rect(w, t, A, B, C, rows, cols);
    CUDA_TRY(cudaSetDevice(w.device));
    const std::string key = graph_key(w, t, A, B, C, rows, cols);
    auto replay = [&](WorkerCtx::GraphEntry &ge) -> int {
        CUDA_TRY(cudaGraphLaunch(ge.exec, w.stream));
        w.launches += ge.launches;
        w.timed |= ge.timed;
        for (auto &pr : ge.kt_pairs)
            if (w.kt_list.size() < kMaxKernelTimes) w.kt_list.push_back(pr);
        // the replay leaves the captured task's prepared B in the B-side buffers:
        // REUSE_B tasks may use it once the replay is done (ev_bprep), and a task
        // re-preparing B on another stream waits for it (ev_blast)
        w.bsig = ge.bsig;
        if (ge.bsig.valid || ge.uses_b) {
            for (cudaEvent_t *ev : {&w.ev_bprep, &w.ev_blast}) {
                if (!*ev) CUDA_TRY(cudaEventCreateWithFlags(ev, cudaEventDisableTiming));
                CUDA_TRY(cudaEventRecord(*ev, w.stream));
            }
        }
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
    const long long bsig_gen0 = w.bsig_gen;
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
    ge.bsig = w.bsig;
    ge.uses_b = w.bsig.dtype >= 0 && w.bsig_gen != bsig_gen0;
    w.kt_list.resize(list0);
    w.launches = launches0;
    return replay(w.graphs.emplace(key, std::move(ge)).first->second);
}

int execute(bool sync) {
    NvtxRange nv_run(sync ? "pdl_run" : "pdl_run_async");
    int rc = check_loaded();
    if (rc) return rc;
    std::vector<Task> q;
    q.swap(g->queue);   // the queue is cleared whatever happens
    std::ostringstream pj;
    pj << "[";
    for (auto &w : g->workers) {
        w.launches = 0;
        w.timed = false;
        w.xpending = false;
    }
    g->xfer = XferStats();
    ++g->run_epoch;
    // Green-context streams are non-blocking: give them the ordering of the
    // blocking Worker streams (after the prior work of the legacy default stream,
    // or of the caller's stream given to pdl_set_stream, and that stream after
    // them -- see the end of this function).
    if (!g->dry_run)
        for (auto &w : g->workers)
            if (w.gctx && w.own_stream) {
                CUDA_TRY(cudaSetDevice(w.device));
                if (!w.ev_legacy) CUDA_TRY(cudaEventCreateWithFlags(&w.ev_legacy, cudaEventDisableTiming));
                CUDA_TRY(cudaEventRecord(w.ev_legacy, w.join_stream ? w.join_stream : cudaStreamLegacy));
                CUDA_TRY(cudaStreamWaitEvent(w.stream, w.ev_legacy, 0));
            }
    for (size_t ti = 0; ti < q.size(); ++ti) {
        const Task &t = q[ti];
        NvtxRange nv_task("task %lldx%lldx%lld", (long long)t.M, (long long)t.N, (long long)t.K);
        if (t.flags & PDL_TASK_LOCAL) {
            // one tile task of this process's (first) Worker, no mapping
            if (ti) pj << ",";
            pj << "{\"local\":true,\"M\":" << t.M << ",\"N\":" << t.N << ",\"K\":" << t.K << "}";
            if (g->dry_run) continue;
            if (g->workers.empty()) return set_err(PDL_ENOWORKER, "no Worker bound to this process");
            rc = (t.flags & PDL_TASK_PREP_A) ? run_prep_a(g->workers[0], t)
                                              : run_rect_g(g->workers[0], t, t.A, t.B, t.C, t.M, t.N);
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
        if (exchange_applies(t, plan, gw)) {
            // operands in the Master's memory region cross PCIe once, then move
            // Worker <-> Worker over the descriptor's interconnect (pdl_xchg.cu)
            rc = run_exchange(t, plan, gw);
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
                CUDA_TRY(cudaStreamWaitEvent(w.join_stream ? w.join_stream : cudaStreamLegacy, w.ev_legacy, 0));
            }
    if (sync) return pdl_sync();
    return PDL_OK;
}

}  // namespace pdlrt
