/*
 * libpdl.h -- C ABI of the B200-native PDL-mapped blocked matmul.
 *
 * Paper: Sandrieser, Benkner, Pllana, "Explicit Platform Descriptions for
 * Heterogeneous Many-Core Architectures", IPDPS 2011.  Citations "L<n>" are
 * lines of /root/reference/PAPER.md (section in parentheses).
 *
 * The library is the run-time counterpart of the paper's PDL-parameterised,
 * task-annotated program (SS IV): a PDL descriptor (SS III-B/C) is parsed into
 * the hierarchical machine model (Master / Hybrid / Worker PUs, memory
 * regions, interconnects, SS III-A L472-603); a `task` call records one
 * DGEMM task C = A*B (the case-study kernel, SS IV-D L1402-1406); `pdl_run`
 * maps the task's tile tasks onto the execution group's Worker PUs with a
 * BLOCK distribution (SS IV-A L1199-1208, SS IV-B L1254-1281), stages operands
 * along the interconnects (SS IV-C step 3, L1336-1341) and runs the sm_100a
 * tile kernels.
 *
 * Conventions (readings R1-R6):
 *  - C = A*B with alpha = 1, beta = 0: C has access mode `write` and is
 *    overwritten (L1184-1186); A and B have access mode `read`.
 *  - Row-major storage.  A is M x K, B is K x N, C is M x N.  Leading
 *    dimensions are the number of columns unless given explicitly (_ex).
 *    Column-major callers compute C^T = B^T A^T by swapping A<->B and M<->N.
 *  - Pointers may be host memory (pageable or pinned; the Master's memory
 *    region) or CUDA device memory (a Worker's memory region).
 *  - Calls are not thread-safe: one Master thread drives the library
 *    (Master PU = "starting point for execution of a program", L495-503).
 *  - No CPU fallback exists.  If no usable B200 Worker is bound, pdl_run
 *    fails with PDL_ENOWORKER / PDL_ECUDA.
 *
 * Ownership: the caller owns A, B, C.  They must stay valid (A, B unchanged,
 * C untouched) from the task call until pdl_run/pdl_sync returns.  The
 * library never frees or retains them.  Library-owned device buffers (Worker
 * memory-region staging buffers, padded/split operand panels) are cached
 * across runs and freed by pdl_unload.
 *
 * Errors: every entry point returns PDL_OK (0) or a negative code and sets a
 * thread-local message readable with pdl_last_error().  After an error inside
 * pdl_run the queue is cleared and C's contents are unspecified.
 */
#ifndef LIBPDL_H
#define LIBPDL_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Return codes. */
#define PDL_OK            0
#define PDL_EINVAL       -1  /* bad argument (null pointer with nonzero size, negative dim, overlap, unknown group/dist) */
#define PDL_EPARSE       -2  /* malformed XML, or a structural rule of the machine model is broken */
#define PDL_ENOWORKER    -3  /* no gpu Worker in the execution group, or more Workers than devices */
#define PDL_ENOMEM       -4  /* device or host allocation failed */
#define PDL_ECUDA        -5  /* a CUDA runtime/driver call failed */
#define PDL_ENCCL        -6  /* Worker<->Worker exchange failed: a peer copy of pdl_run's exchange
                                failed or had not completed within PDL_SYNC_TIMEOUT_MS (pdl_sync);
                                the multi-rank Python runtime maps NCCL / gloo collective
                                failures and timeouts to the same code */
#define PDL_ESTATE       -7  /* call out of order (task before load, load twice, ...) */
#define PDL_EUNSUPPORTED -8  /* valid request this build does not implement */

/* Element types of task_matmul_ex. */
#define PDL_F64 0            /* the paper's precision: DGEMM (L1402-1406); FP64 DMMA tensor cores */
#define PDL_F32 1            /* FP32 in/out; TF32 split on tcgen05 tensor cores (north star (2)):
                                TF32 main product + BF16 corrections (default) or 3xTF32 */

/* task_matmul_ex flags. */
#define PDL_TASK_PANELS 1u   /* operands are this process's Worker panels (after the exchange):
                                A = rows_w x K, B = K x cols_w, C = rows_w x cols_w block at
                                the Worker's rectangle; see pdl_plan */
#define PDL_TASK_LOCAL 2u    /* the whole M x N x K task is one tile task of this process's
                                (first) Worker: no mapping over the group.  The multi-rank
                                runtime uses it to compute a Worker rectangle chunk by chunk
                                while the exchange of the next chunk is in flight */
#define PDL_TASK_GRAPH 8u    /* replay this task's launch sequence from a CUDA graph: the first
                                run of a task signature (dtype, pointers, sizes, leading dims,
                                tile, flags, stream) runs normally, the second is captured, later
                                runs are one cudaGraphLaunch per Worker (launch-bound small
                                tasks).  Env PDL_GRAPH=1 sets it for every task.  Ignored with
                                PDL_TASK_REUSE_B and DYNAMIC; uncapturable work (pageable host
                                memory) runs uncaptured */
#define PDL_TASK_REUSE_B 4u  /* B (same pointer, ldb, K, N) is unchanged since the previous task
                                of this Worker: reuse its prepared form (FP32 split / Ozaki
                                slices) instead of recomputing it; ignored when no matching
                                prepared B exists */
#define PDL_TASK_PREP_A 64u  /* with PDL_TASK_LOCAL: only prepare A -- write the task variant's
                                prepared form of A's M rows (K wide) to C as packed rows of
                                pdl_query("prepared_a/<dtype>/<K>") bytes (FP32: [TF32 hi: Kp
                                floats][second plane: Kp floats -- tf32bf16: per 16-wide K block
                                16 BF16 hi' then 16 BF16 lo'; 3xtf32: TF32 lo], Kp = K rounded up
                                to 32; FP64 ozaki2: [residues: ld8 bytes][e_i: int32][sign bits: u32]
                                [certificate row sum: u64]); B and N are ignored.  C: 16-byte
                                aligned memory of the Worker's device.  PDL_EUNSUPPORTED for
                                variants that exchange raw rows (query answers 0: FP64 dmma) */
#define PDL_TASK_PREPARED_A 128u
                             /* with PDL_TASK_LOCAL: A holds M prepared rows (PDL_TASK_PREP_A
                                on a Worker with the same variant and K) in this Worker's
                                memory region; lda is ignored; the task skips A's preparation.
                                The multi-rank runtime exchanges prepared A chunks so each
                                Worker prepares only its own chunk.  Variants that also read
                                the raw rows (ozaki2) need task_matmul_prepared */
#define PDL_TASK_SLOT(s) (((unsigned)(s) & 3u) << 4)
                             /* scratch slot s in 0..2 of the Worker: a task's own buffers (A
                                split / slices / residues and exponents, residue planes,
                                staging) exist once per slot, so tasks of different slots with
                                device-resident, 16-byte aligned operands may run at once on
                                different streams (pdl_set_stream between them); the prepared
                                B (PDL_TASK_REUSE_B) is shared and a reusing task on another
                                stream waits for its preparation.  Slot 3 -> PDL_EINVAL.
                                pdl_query("concurrent_tasks/f64"|"concurrent_tasks/f32") says
                                whether the loaded Workers support it ("yes") */

/*
 * pdl_load -- parse a PDL descriptor and build the machine model.
 * descriptor: path to an XML file, or XML text if its first non-blank
 *   character is '<'.  Entities: Master/Hybrid/Worker with PUDescriptor,
 *   MemoryRegion(MRDescriptor), Interconnect(ICDescriptor),
 *   LogicGroupAttribute; Descriptor -> Property(name, value) (L668-680);
 *   prefixed tags (ocl:name) match by local name (L876-909).
 * Rules checked (L495-531): >= 1 Master, Masters only at top level, Workers
 *   are leaves controlled by a Master or Hybrid, Hybrids are controlled by a
 *   Master or Hybrid, Interconnect endpoints exist, quantity >= 1, ids unique.
 * Worker PUs with ARCHITECTURE (alias ARCH, value case-insensitive) = gpu are
 *   bound to CUDA devices (DEVICE_ORDINAL property, else in document order)
 *   and their unfixed properties are filled from the device (L737-747).
 *   A Worker property SM_LIMIT = n (n >= 1, rounded up to a multiple of 8)
 *   runs the Worker on a green context of n SMs; Workers that all carry it may
 *   share a device, and get disjoint partitions (the device is split into groups
 *   of gcd(n_i) SMs; PDL_EINVAL when the device cannot supply enough groups or
 *   the sum exceeds its SMs).  This emulates heterogeneous Workers on one GPU.
 * Task variants (one task interface, several implementations pre-selected per
 *   Worker from its properties): DGEMM_VARIANT = dmma
 *   (default: K1, IEEE FP64 on DMMA) | ozaki2 (K6/K7: Ozaki scheme II on the
 *   INT8 tensor cores, OZAKI2_MODULI, default the fewest giving OZAKI2_BITS =
 *   43 scaling bits, finite inputs only).  ozaki2 carries a certificate
 *   (OZAKI2_GUARD = on | off, default on; OZAKI2_GUARD_TOL = tau, default
 *   5e-13): one more INT8 GEMM bounds every element's error against a lower
 *   bound of |A||B|, and K1 recomputes each element whose bound exceeds
 *   tau |A||B| -- so |C - AB| <= tau |A||B| holds element by element for any
 *   finite input (R20, R21); tasks with K > 65536 run K1.
 *   SGEMM_VARIANT = tf32bf16 (default: K3 + K2, a_hi*b_hi in TF32 plus the
 *   two correction products in BF16, split error <= 7.9e-6 |A||B|, DESIGN.md
 *   R22) | 3xtf32 (three TF32 products); another name is PDL_EINVAL at
 *   pdl_run.  The round-1 variant "ozaki" (Ozaki scheme I) is retired:
 *   PDL_EUNSUPPORTED at pdl_run.
 *   RELATIVE_SPEED weights the BLOCK mapping.  Env PDL_<PROPERTY> overrides a
 *   property for every Worker.
 * This process is the single Master driving every Worker of the descriptor.
 * Env: PDL_DRY_RUN=1 skips device binding (plans only; no device work);
 *   PDL_ALLOW_OVERSUBSCRIBE=1 lets several Workers share a device.
 * Errors: PDL_ESTATE if already loaded; PDL_EPARSE; PDL_ENOWORKER; PDL_ECUDA.
 */
int pdl_load(const char *descriptor);

/*
 * pdl_load_rank -- as pdl_load, for one process per GPU: `nranks` Masters
 * co-exist ("Masters ... may co-exist with other Masters within the same
 * system", L495-503) and process `rank` controls exactly Worker instance
 * `rank` of the execution group, bound to the process's current CUDA device.
 * nranks must equal the group's Worker count (checked at pdl_run).
 * rank = 0, nranks = 1 is pdl_load.
 */
int pdl_load_rank(const char *descriptor, int rank, int nranks);

/*
 * task_matmul -- record one FP64 DGEMM task C = A*B (L1402-1406) with task
 * tile edge `tile` (> 0: tile x tile tile tasks, the last row/column of tasks
 * partial; 0: one task per Worker rectangle).  Access modes: A read, B read,
 * C write (L1184-1186).  No device work happens here.
 * Quick returns: M == 0 or N == 0 -> no-op; K == 0 -> C is zero-filled.
 * Errors: PDL_ESTATE before pdl_load; PDL_EINVAL for negative sizes, null
 *   pointers with nonzero sizes, C overlapping A or B.
 */
int task_matmul(const double *A, const double *B, double *C,
                int64_t M, int64_t N, int64_t K, int64_t tile);

/* task_matmul_f32 -- FP32 variant of the same task interface (TF32-split tcgen05;
 * SGEMM_VARIANT picks tf32bf16 or 3xtf32). */
int task_matmul_f32(const float *A, const float *B, float *C,
                    int64_t M, int64_t N, int64_t K, int64_t tile);

/*
 * task_matmul_ex -- general form.
 * dtype: PDL_F64 | PDL_F32.  lda/ldb/ldc: leading dimensions in elements
 *   (0 = dense: K, N, N; in PANELS mode 0 = K, cols_w, cols_w).
 * group: LogicGroupAttribute naming the execution group (L1193-1199,
 *   L1254-1261); NULL = every gpu Worker.
 * dist: data distribution of C's tile tasks over the group (L1200-1206:
 *   "block, cyclic, block-cyclic ... and optional sizes"): "BLOCK" (or NULL;
 *   "BLOCK:N" accepted, N implied), "CYCLIC", "BLOCK-CYCLIC:b" (b tasks per
 *   block, default 1), "DYNAMIC" (no static assignment: every Worker launches
 *   the whole tile grid and its CTAs claim tiles from one counter in the first
 *   Worker's memory -- the dynamic scheduling of the paper's future work,
 *   L1556-1562; operands must be device-resident on, or are staged whole to,
 *   every Worker; C must be host memory or reachable by peer access; the
 *   single-launch variants only: Ozaki Workers -> PDL_EUNSUPPORTED at pdl_run;
 *   tiles claimed per Worker in pdl_query("stats")["dynamic"]),
 *   case-insensitive.  Non-BLOCK distributions need one
 *   process driving the Workers (pdl_load): with PDL_TASK_PANELS or
 *   pdl_load_rank they return PDL_EUNSUPPORTED.  Unknown names -> PDL_EINVAL.
 *   Workers whose PDL property RELATIVE_SPEED differs get a speed-weighted
 *   1-D BLOCK split (heterogeneous platforms, L1398-1402).  With one process
 *   driving the Workers, BLOCK follows the PU hierarchy: a PU whose group
 *   Workers lie in several subtrees (Hybrid PUs, L513-531) gives each subtree a
 *   row band sized by its total RELATIVE_SPEED (pdl_plan then reports Gr = G,
 *   Gc = 1 and the Worker's explicit rectangle).
 * flags: 0 or PDL_TASK_PANELS.
 */
int task_matmul_ex(int dtype, const void *A, int64_t lda, const void *B, int64_t ldb,
                   void *C, int64_t ldc, int64_t M, int64_t N, int64_t K, int64_t tile,
                   const char *group, const char *dist, unsigned flags);

/*
 * task_matmul_prepared -- a one-Worker task (PDL_TASK_LOCAL semantics) whose A
 * is given as M prepared rows (PDL_TASK_PREP_A on a Worker with the same task
 * variant and K; Aprep in this Worker's memory region, 16-byte aligned).
 * Araw, lda_raw: the raw A rows (M x K, this Worker's device) for variants whose
 * prepared tasks still read them -- ozaki2: the certificate's K1 recompute of
 * uncertified elements, after the residue GEMMs (pdl_query("prepared_a/f64/<K>")
 * ends in "+raw") -- else NULL.  raw_ready: a cudaEvent_t (as void *) the Worker
 * stream waits on just before reading Araw, or NULL; so the raw rows may still be
 * in flight while the residue GEMMs run.  B (K x N, ldb), C (M x N, ldc) as in
 * task_matmul_ex.  flags: PDL_TASK_REUSE_B | PDL_TASK_GRAPH | PDL_TASK_SLOT(s).
 * Errors: PDL_EINVAL (arguments; at pdl_run: Aprep or Araw not on the Worker's
 * device), PDL_EUNSUPPORTED at pdl_run for variants without an A preparation.
 */
int task_matmul_prepared(int dtype, const void *Aprep, const void *Araw, int64_t lda_raw, void *raw_ready,
                         const void *B, int64_t ldb, void *C, int64_t ldc, int64_t M, int64_t N, int64_t K,
                         unsigned flags);

/*
 * pdl_run -- map and execute all queued tasks in program order (access-mode
 * dependencies reduce to queue order for one task type), then synchronise,
 * harvest errors and clear the queue.  Blocks until C is written.
 * Transfer paths follow the descriptor's interconnects (SS IV-C step 3,
 * L1336-1341): with A and B in the Master's memory region (host), a BLOCK
 * task over G > 1 Workers that an Interconnect joins pairwise (the shipped
 * descriptors' NVLink) moves each operand byte over the Master->Worker
 * interconnect once -- Worker (r, c) receives chunk c of its A row-panel and
 * chunk r of its B column-panel -- and the Workers pull the rest of their
 * panels from each other (peer copies, overlapped with the tile kernels: own
 * A chunk first).  Otherwise each Worker stages its whole panels from the
 * Master's memory region.  Bytes per path: pdl_query("stats")["transfers"].
 * Env PDL_EXCHANGE=0 disables the Worker<->Worker path; PDL_SYNC_TIMEOUT_MS
 * bounds the wait (then PDL_ENCCL if an exchange copy is unfinished, else
 * PDL_ECUDA; the work stays in flight: unload the platform).
 */
int pdl_run(void);

/* pdl_run_async -- as pdl_run without the final synchronisation; errors of
 * the device work surface at the next pdl_sync.  The queue is cleared. */
int pdl_run_async(void);

/* pdl_sync -- wait for all device work issued by pdl_run_async. */
int pdl_sync(void);

/*
 * pdl_set_stream -- launch this process's device work for Worker `worker`
 * (local index, 0 in rank mode) on the given cudaStream_t (NULL = the
 * library's own stream, which is a blocking stream, i.e. ordered with the
 * legacy default stream; pass cudaStreamLegacy = (void*)1 for the legacy
 * default stream itself).  Lets a caller order the library with its own
 * stream and time it with its own events.  A Worker on an SM partition
 * (SM_LIMIT, a green context) keeps its partition's stream: each run then
 * waits for the prior work of `stream` and `stream` waits for the run.
 */
int pdl_set_stream(int worker, void *stream);

/*
 * pdl_plan -- the BLOCK mapping of an M x N x K task with task edge `tile`
 * onto the execution group (L1200-1206; SS IV-B static mapping L1254-1281).
 * Writes PDL_PLAN_LEN int64 values to out[] (nout >= PDL_PLAN_LEN):
 *   [0] G        Workers in the group        [1] Gr, [2] Gc  worker grid
 *   [3] r, [4] c grid position of group Worker `worker` (w = r*Gc + c)
 *   [5] row0, [6] row1, [7] col0, [8] col1   the Worker's C rectangle
 *   [9] qa   rows per A chunk: the A row-panel (rows row0..row1) is split in
 *            Gc chunks of qa rows; this Worker holds chunk c
 *   [10] qb  K-rows per B chunk: the B column-panel (cols col0..col1) is
 *            split in Gr chunks of qb K-rows; this Worker holds chunk r
 *   [11] T_m, [12] T_n  task grid (ceil(M/tile) x ceil(N/tile))
 *   [13] tr0, [14] tr1, [15] tc0, [16] tc1  the Worker's task rows / cols
 *   [17] tile  effective task edge (0 in the request -> per-Worker blocks)
 * Errors: PDL_ESTATE before pdl_load; PDL_EINVAL; PDL_ENOWORKER.
 */
#define PDL_PLAN_LEN 18
int pdl_plan(int64_t M, int64_t N, int64_t K, int64_t tile, const char *group,
             int worker, int64_t *out, int nout);

/*
 * pdl_query -- the "simple query API" over the loaded PDL (L935-937).
 * Keys: "version", "masters", "workers", "groups", "model" (JSON),
 *   "plan" (JSON of the last run's mappings), "stats" (JSON: launches,
 *   kernel time and SM partition per Worker of the last run; "transfers":
 *   bytes moved Master->Worker, Worker->Master and Worker<->Worker in the
 *   last run, the tasks that ran the Worker<->Worker exchange, and the
 *   descriptor's interconnect types of those paths; "dynamic": tiles
 *   each Worker claimed in the last DYNAMIC task -- read after pdl_sync),
 *   "worker/<i>/<PROPERTY>",
 *   "worker/<i>/device", "worker/<i>/id", "pu/<id>/<PROPERTY>",
 *   "interconnects" (JSON), "exchange_path[/<group>]" ("direct" when every
 *   pair of the group's gpu Workers is joined by an Interconnect, else "host":
 *   the transfer path the multi-rank exchange takes, L1336-1341),
 *   "ozaki2_plan/<K>[/<bits>[/<moduli>]]" (JSON; no pdl_load needed: moduli,
 *   scaling bits p, K chunks, CRT weights W_t and M as decimal strings, and
 *   "crt": "fp64" when the FP64-pipe reconstruction applies, else "int"),
 *   "ozaki2_launches/<rows>/<cols>/<items>/<clusters>" (JSON list, no pdl_load
 *   needed: GEMM items -- moduli, plus 1 for the certificate -- per persistent
 *   launch of one K chunk), "ozaki_guard" inside "stats" (JSON: per Worker the
 *   128 x 128 tiles the Ozaki-II certificate checked in the last run and the
 *   tiles / elements K1 recomputed),
 *   "concurrent_tasks/f64" | "concurrent_tasks/f32" ("yes" when tasks of
 *   different PDL_TASK_SLOTs may overlap on different streams).
 * Writes a NUL-terminated string (truncated to len-1) and returns the full
 * length, or a negative code (PDL_EINVAL for an unknown key).
 */
int pdl_query(const char *key, char *out, size_t len);

/*
 * pdl_kernel_times -- device durations (ms, CUDA events on the launching
 * stream) of the dominant tile-kernel launches (K1, or K2 for FP32) issued
 * for local Worker `worker` since the previous call, in launch order.  Waits
 * for those launches, writes min(count, n) values to ms[], clears the record
 * and returns the count (at most 4096 are kept).
 */
int pdl_kernel_times(int worker, float *ms, int n);

/*
 * pdl_describe -- generate a PDL descriptor of this machine (
 * the analogue of Listing 2, "Generated from OpenCL run-time libraries",
 * L869-917): one Master PU for the host (ARCHITECTURE from the build target,
 * host memory region size), one Worker PU per CUDA device (ARCHITECTURE gpu,
 * DEVICE_ORDINAL fixed; DEVICE_NAME, MAX_COMPUTE_UNITS, COMPUTE_CAPABILITY,
 * GLOBAL_MEM_SIZE, LOCAL_MEM_SIZE, L2_CACHE_SIZE, CLOCK_RATE, PCI_BUS_ID as
 * unfixed properties; LogicGroupAttribute "gpus"), a PCIe
 * Interconnect Master -> each Worker, and an NVLink Interconnect between every
 * pair of Workers with peer access (cudaDeviceCanAccessPeer).  Needs no
 * pdl_load.  Writes NUL-terminated XML (truncated to len-1) and returns its
 * full length; PDL_ENOWORKER if no CUDA device is visible.
 */
int pdl_describe(char *out, size_t len);

/* Message of the last error of this thread ("" if none). */
const char *pdl_last_error(void);

/* Free library-owned buffers and the model; the library can be loaded again. */
void pdl_unload(void);

#ifdef __cplusplus
}
#endif
#endif /* LIBPDL_H */
