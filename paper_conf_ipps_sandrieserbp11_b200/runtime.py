"""One-process-per-GPU task runtime: the multi-Worker path of the DGEMM task.

Each process is one co-existing Master controlling one Worker PU ("Masters
... may co-exist with other Masters within the same system", PAPER.md
L495-503), bound with ``pdl_load_rank``.  The BLOCK mapping (which C
rectangle, which operand chunk each Worker holds) comes from libpdl's
``pdl_plan`` (L1200-1208); this module only moves data between Workers:

* initial ("unique chunk") layout -- Worker (r, c) of the Gr x Gc grid holds
  chunk c of A's row-panel r (qa rows) and chunk r of B's column-panel c
  (qb K-rows), so every operand byte lives on exactly one Worker;
* exchange -- all-gather of the A chunks inside each grid row and of the B
  chunks inside each grid column over torch.distributed (NCCL over NVLink 5 /
  NVSwitch on the GPU box, gloo in the CPU tests).  This is the "derive
  data-transfer paths ... via the explicitly specified interconnect entity"
  step (L1336-1341) for the Worker<->Worker NVLink interconnect; a descriptor
  that joins the Workers by no interconnect sends the exchange through the
  Master's memory region instead (host-staged gloo groups, ``exchange_path``);
* local task -- ``task_matmul_ex(..., PDL_TASK_PANELS)`` + ``pdl_run`` on the
  gathered panels (libpdl, sm_100a kernels).

There is no split-K, hence no reduction: each C element is produced by one
Worker, and the result is bitwise identical for any Worker count (pin P7).
"""
from __future__ import annotations

from dataclasses import dataclass

import torch
import torch.distributed as dist

from . import pdl


@dataclass
class WorkerPlan:
    G: int
    Gr: int
    Gc: int
    r: int
    c: int
    row0: int
    row1: int
    col0: int
    col1: int
    qa: int
    qb: int
    M: int
    N: int
    K: int

    @property
    def rows(self):
        return self.row1 - self.row0

    @property
    def cols(self):
        return self.col1 - self.col0

    # this Worker's chunk of its A row-panel: panel rows [a0, a1)
    @property
    def a_span(self):
        a0 = min(self.c * self.qa, self.rows)
        return a0, min(a0 + self.qa, self.rows)

    # this Worker's chunk of its B column-panel: K rows [b0, b1)
    @property
    def b_span(self):
        b0 = min(self.r * self.qb, self.K)
        return b0, min(b0 + self.qb, self.K)


def worker_plan(M, N, K, tile, rank, group=None) -> WorkerPlan:
    p = pdl.plan(M, N, K, tile, group=group, worker=rank)
    return WorkerPlan(p["G"], p["Gr"], p["Gc"], p["r"], p["c"], p["row0"], p["row1"], p["col0"],
                      p["col1"], p["qa"], p["qb"], M, N, K)


def exchange_path(group=None) -> str:
    """The Worker<->Worker path the loaded descriptor allows (libpdl query
    "exchange_path"): "direct" when every pair of the group's Workers is joined
    by an Interconnect (NVLink on a B200 box), else "host" -- the exchange then
    stages through the Master's memory region ("derive data-transfer paths ...
    via the explicitly specified interconnect entity")."""
    return pdl.query("exchange_path" + (f"/{group}" if group else ""))


class Grid:
    """Row / column process groups of the Gr x Gc Worker grid (created
    collectively: every rank creates every group in the same order).
    via_host: exchange through host memory (gloo groups) because the
    descriptor has no Worker<->Worker interconnect."""

    def __init__(self, Gr, Gc, rank, via_host=False):
        self.Gr, self.Gc, self.rank = Gr, Gc, rank
        self.via_host = via_host
        self.row_group = self.col_group = None
        self.row_ranks = [rank // Gc * Gc + c for c in range(Gc)]   # global ranks of my grid row
        kw = {"backend": "gloo"} if via_host else {"pg_options": _nccl_high_priority()}
        for r in range(Gr):
            ranks = [r * Gc + c for c in range(Gc)]
            g = dist.new_group(ranks, **kw) if Gc > 1 else None
            if rank in ranks:
                self.row_group = g
        for c in range(Gc):
            ranks = [r * Gc + c for r in range(Gr)]
            g = dist.new_group(ranks, **kw) if Gr > 1 else None
            if rank in ranks:
                self.col_group = g


def _nccl_high_priority():
    """NCCL process-group options with high-priority streams, so the exchange
    kernels get SMs ahead of queued tile-kernel CTAs when both are pending (the
    A broadcasts must progress while the own-chunk kernel runs); None under gloo."""
    if dist.get_backend() != "nccl":
        return None
    Options = getattr(dist, "ProcessGroupNCCL", None)
    if Options is None or not hasattr(Options, "Options"):
        return None
    opts = Options.Options()
    opts.is_high_priority_stream = True
    return opts


def chunk_from_full(A, B, wp: WorkerPlan):
    """Slice this Worker's unique chunks out of full A (M x K) and B (K x N),
    zero-padded to qa x K and qb x cols (equal sizes for the all-gather)."""
    a0, a1 = wp.a_span
    b0, b1 = wp.b_span
    Ach = torch.zeros((wp.qa, wp.K), dtype=A.dtype, device=A.device)
    Bch = torch.zeros((wp.qb, wp.cols), dtype=B.dtype, device=B.device)
    if a1 > a0:
        Ach[: a1 - a0].copy_(A[wp.row0 + a0: wp.row0 + a1])
    if b1 > b0 and wp.cols:
        Bch[: b1 - b0].copy_(B[b0:b1, wp.col0: wp.col1])
    return Ach, Bch


class PanelBuffers:
    """The Worker's panels: B column-panel (Gr chunks of qb K-rows) and A
    row-panel (Gc chunks of qa rows).  prep_bytes > 0 (the task variant prepares
    A, pdl.prepared_a_row_bytes): the A panel holds PREPARED rows (bytes), so each
    Worker prepares only its own chunk and the exchange moves prepared chunks
    (FP32 3xTF32: TF32 hi/lo, 2x the raw bytes, instead of every Worker of a grid
    row splitting the whole panel again)."""

    def __init__(self, wp: WorkerPlan, dtype, device, prep_bytes: int = 0, keep_raw: bool = False):
        self.prepared = prep_bytes > 0
        # raw A rows beside the prepared ones: variants whose prepared tasks still
        # read them (ozaki2: the certificate's K1 recompute); they travel after the
        # prepared chunks and are needed only at the end of each chunk task
        self.Araw = None
        if self.prepared:
            self.A = torch.empty((wp.Gc * wp.qa, prep_bytes), dtype=torch.uint8, device=device)
            if keep_raw:
                self.Araw = torch.empty((wp.Gc * wp.qa, wp.K), dtype=dtype, device=device)
        else:
            self.A = torch.empty((wp.Gc * wp.qa, wp.K), dtype=dtype, device=device)
        self.B = torch.empty((wp.Gr * wp.qb, wp.cols), dtype=dtype, device=device)
        if _test_delay_cycles():
            # fault injection (tests): panels start as NaN, so a compute that does
            # not wait for its chunk's landing produces NaN rows of C
            self.A.fill_(255 if self.prepared else float("nan"))
            self.B.fill_(float("nan"))
            if self.Araw is not None:
                self.Araw.fill_(float("nan"))


def prepared_info(dtype, K, device):
    """(prepared-A row bytes, prepared tasks read raw rows too) of this Worker's
    task variant for device panels; (0, False): exchange raw rows."""
    if device is None or torch.device(device).type != "cuda":
        return 0, False
    return pdl.prepared_a_info(dtype, K)


def prepared_bytes(dtype, K, device) -> int:
    return prepared_info(dtype, K, device)[0]


def panel_buffers(wp: WorkerPlan, dtype, device, prepared: bool = True) -> PanelBuffers:
    """PanelBuffers in the exchange format of this Worker's task variant."""
    pb, raw = prepared_info(dtype, wp.K, device) if prepared else (0, False)
    return PanelBuffers(wp, dtype, device, pb, raw)


def exchange(Ach, Bch, wp: WorkerPlan, grid: Grid, bufs: PanelBuffers):
    """All-gather the operand chunks: afterwards bufs.A[:rows] is the A
    row-panel (rows x K) and bufs.B[:K] the B column-panel (K x cols)."""
    if wp.Gc > 1:
        _all_gather(bufs.A, Ach, grid.row_group)
    else:
        bufs.A.copy_(Ach)
    if wp.Gr > 1:
        _all_gather(bufs.B, Bch, grid.col_group)
    else:
        bufs.B.copy_(Bch)
    return bufs.A[: wp.rows], bufs.B[: wp.K]


# ---- collectives ------------------------------------------------------------
#
# NCCL (the B200 box): asynchronous work on NCCL's streams; Work.wait() makes the
# CURRENT stream wait for it, the host does not block.  gloo (CPU tests; several
# ranks sharing one GPU): gloo moves host tensors only, so device tensors are
# staged through pinned host memory, and _HostStaged gives the same stream
# semantics -- the landing copy runs on a comm stream and wait() makes the current
# stream wait for it -- so the ordering logic of compute_groups faces work that
# has not finished.  Fault injection for the tests: PDL_TEST_EXCHANGE_DELAY_US
# delays every landing on the comm stream (a spin kernel) and poisons the panel
# buffers with NaN; PDL_TEST_DROP_WAITS=1 drops the A-chunk waits (the test that
# the ordering matters must then see corrupt C).
# Failures of the collectives surface as pdl.PDLError(PDL_ENCCL); a hang is
# bounded by the process group's timeout (init_process_group(timeout=...)) and,
# for the broadcast handles, PDL_EXCHANGE_TIMEOUT_S.


def _test_delay_cycles():
    import os
    us = float(os.environ.get("PDL_TEST_EXCHANGE_DELAY_US", "0") or 0)
    return int(us * 2000)   # ~2 GHz SM clock


_comm_streams = {}


def _comm_stream():
    dev = torch.cuda.current_device()
    if dev not in _comm_streams:
        _comm_streams[dev] = torch.cuda.Stream(device=dev)
    return _comm_streams[dev]


def _exchange_error(what, e):
    return pdl.PDLError(pdl.PDL_ENCCL, f"{what} failed over {dist.get_backend()}: {e}")


class _HostStaged:
    """A gloo collective on pinned host memory whose result lands in a device
    tensor on the comm stream, with NCCL's wait() semantics (see above)."""

    def __init__(self, work, tmp, dst, drop_wait=False):
        self.work, self.tmp, self.dst = work, tmp, dst
        self.drop_wait = drop_wait
        self.issued = torch.cuda.Event()
        self.issued.record()   # the landing copy must not overtake earlier users of dst
        self.landed = None

    def _land(self):
        if self.landed is None:
            try:
                self.work.wait()   # the host copy is complete
            except RuntimeError as e:
                raise _exchange_error("host-staged collective", e) from e
            cs = _comm_stream()
            cs.wait_event(self.issued)
            with torch.cuda.stream(cs):
                cyc = _test_delay_cycles()
                if cyc:
                    torch.cuda._sleep(cyc)
                self.dst.copy_(self.tmp, non_blocking=True)
                self.landed = torch.cuda.Event()
                self.landed.record(cs)

    def wait(self):
        self._land()
        if not self.drop_wait:
            torch.cuda.current_stream().wait_event(self.landed)


class _Async:
    """Async work handle (NCCL: wait() = the current stream waits, no host block;
    gloo on host tensors: the host waits);
    errors (including the NCCL watchdog's async-error abort) -> PDL_ENCCL."""

    def __init__(self, work, what, drop_wait=False):
        self.work, self.what, self.drop_wait = work, what, drop_wait

    def wait(self):
        if self.drop_wait:
            return
        import os
        from datetime import timedelta
        try:
            t = os.environ.get("PDL_EXCHANGE_TIMEOUT_S")
            if t:
                self.work.wait(timeout=timedelta(seconds=float(t)))
            else:
                self.work.wait()
        except RuntimeError as e:
            raise _exchange_error(self.what, e) from e


def _staged(t, group):
    return t.is_cuda and dist.get_backend(group) == "gloo"


def _all_gather(out, chunk, group):
    """All-gather into a contiguous buffer (the current stream waits for it)."""
    try:
        if _staged(out, group):
            tmp = torch.empty(out.shape, dtype=out.dtype, pin_memory=True)
            w = dist.all_gather_into_tensor(tmp, chunk.contiguous().cpu(), group=group, async_op=True)
            _HostStaged(w, tmp, out).wait()
        else:
            dist.all_gather_into_tensor(out, chunk.contiguous(), group=group)
    except RuntimeError as e:
        if isinstance(e, pdl.PDLError):
            raise
        raise _exchange_error("all-gather", e) from e


def _broadcast(t, src, group):
    """Asynchronous broadcast of one A chunk inside the grid row; returns a
    handle whose wait() orders the current stream after the chunk's landing."""
    import os
    drop = os.environ.get("PDL_TEST_DROP_WAITS") == "1"
    try:
        if _staged(t, group):
            mine = dist.get_rank() == src
            tmp = t.cpu().pin_memory() if mine else torch.empty(t.shape, dtype=t.dtype, pin_memory=True)
            w = dist.broadcast(tmp, src=src, group=group, async_op=True)
            if mine:   # the source's chunk is already in place
                w.wait()
                return _Done()
            return _HostStaged(w, tmp, t, drop_wait=drop)
        return _Async(dist.broadcast(t, src=src, group=group, async_op=True), f"broadcast from rank {src}", drop)
    except RuntimeError as e:
        if isinstance(e, pdl.PDLError):
            raise
        raise _exchange_error("broadcast", e) from e


class _Done:
    def wait(self):
        pass


def chunk_rows(wp: WorkerPlan, j):
    """Rows [lo, hi) of the A row-panel (and of the C block) held by chunk j."""
    lo = min(j * wp.qa, wp.rows)
    return lo, min(lo + wp.qa, wp.rows)


# NVLink 5 peer bandwidth per direction -- an ESTIMATE: the B200 peer-copy figure
# quoted in /opt/skills/guides/B200_PROFILING.md, not re-measured on this pool (one GPU
# per gpurun call) -- and the A exchange below which one launch
# over the whole Worker rectangle beats the chunked overlap: tools/worker_emulate.py
# (profiles/r01_worker_emulate_single_*.jsonl) measured the chunk launches 0.41-0.46
# ms slower than one launch for C3 at G = 4 / 8 (host issue of three short tasks
# outlasts their kernels) against 0.13 / 0.07 ms of A transfer, and 0.03 ms slower
# for C0 / C5 at G = 8 and C0 at G = 2 against 0.12-0.35 ms.
NVLINK_BPS = 770e9
SINGLE_LAUNCH_BELOW_S = 2e-4


def a_exchange_seconds(wp: WorkerPlan, elem_bytes: int) -> float:
    """Time the other Gc - 1 A chunks take over NVLink (what a single launch
    over the whole rectangle leaves exposed)."""
    return (wp.Gc - 1) * wp.qa * wp.K * elem_bytes / NVLINK_BPS


def overlap_pays(wp: WorkerPlan, elem_bytes: int) -> bool:
    """Chunked overlap (True) or one launch after the A exchange (False);
    env PDL_OVERLAP_A = 1 / 0 forces either."""
    import os
    f = os.environ.get("PDL_OVERLAP_A")
    if f in ("0", "1"):
        return f == "1"
    return a_exchange_seconds(wp, elem_bytes) >= SINGLE_LAUNCH_BELOW_S


def exchange_overlapped(Ach, Bch, wp: WorkerPlan, grid: Grid, bufs: PanelBuffers, compute, concurrent=None,
                        overlap_a=None):
    """Exchange with the A transfer overlapped by compute.

    The B column-panel is all-gathered first (every C row needs it).  The A
    row-panel then arrives as Gc asynchronous broadcasts inside the grid row,
    one per owner; `compute(j, lo, hi, Apanel_rows, Bpanel, first)` runs on
    the Worker's own chunk first (no wait), then on the chunks before it and
    the chunks after it, each group as one launch once its broadcasts have
    landed (the stream waits on the NCCL work, the host does not), so the
    other (Gc-1)/Gc of the A traffic hides behind the own-chunk kernel.
    Results are bitwise identical to the non-overlapped path (R14).
    concurrent: see compute_groups (None = ask libpdl).  overlap_a: False =
    wait for every A chunk, then one compute over the whole rectangle (None =
    overlap_pays for device panels; host panels always chunk)."""
    if wp.Gr > 1:
        _all_gather(bufs.B, Bch, grid.col_group)
    else:
        bufs.B.copy_(Bch)
    Bp = bufs.B[: wp.K]
    qa, c = wp.qa, wp.c
    if bufs.prepared:
        # the own chunk's prepared rows (TF32 hi/lo, Ozaki-II residues ...), straight
        # into the panel: each Worker prepares only its own chunk
        pdl.prepare_a(Ach, bufs.A[c * qa:(c + 1) * qa])
        pdl.run_async()
        if bufs.Araw is not None:
            bufs.Araw[c * qa:(c + 1) * qa].copy_(Ach)
    else:
        bufs.A[c * qa:(c + 1) * qa].copy_(Ach)
    works, raw_works = {}, {}
    if wp.Gc > 1:
        for j in range(wp.Gc):   # same order on every rank of the row
            works[j] = _broadcast(bufs.A[j * qa:(j + 1) * qa], grid.row_ranks[j], grid.row_group)
        if bufs.Araw is not None:   # after every prepared chunk: needed only by the recompute
            for j in range(wp.Gc):
                raw_works[j] = _broadcast(bufs.Araw[j * qa:(j + 1) * qa], grid.row_ranks[j], grid.row_group)
    if overlap_a is None:
        overlap_a = wp.Gc == 1 or not bufs.A.is_cuda or \
            overlap_pays(wp, bufs.A.shape[1] * bufs.A.element_size() / max(1, wp.K))
    if overlap_a:
        compute_groups(wp, bufs, Bp, compute, works, concurrent, raw_works)
    else:
        for w in list(works.values()) + list(raw_works.values()):
            w.wait()
        if wp.rows > 0 and wp.cols > 0:
            kw = {} if bufs.Araw is None else {"raw": (bufs.Araw[: wp.rows], None)}
            compute(wp.c, 0, wp.rows, bufs.A[: wp.rows], Bp, True, **kw)
    for w in list(works.values()) + list(raw_works.values()):
        w.wait()
    return bufs.A[: wp.rows], Bp


_side_streams = {}


def _side_stream(i):
    dev = torch.cuda.current_device()
    if (dev, i) not in _side_streams:
        _side_streams[(dev, i)] = torch.cuda.Stream(device=dev)
    return _side_streams[(dev, i)]


def tasks_may_overlap(*panels) -> bool:
    """Whether tasks on these device panels may run on different streams of the
    Worker at once: libpdl keeps every task variant's own buffers per scratch
    slot (PDL_TASK_SLOT; query "concurrent_tasks/<dtype>"), and stages nothing
    when every operand is on the Worker's device, 16-byte aligned, with 16-byte
    row pitches."""
    dt = panels[-1].dtype   # the B panel: raw operand dtype (A may be prepared bytes)
    key = "concurrent_tasks/" + ("f64" if dt == torch.float64 else "f32")
    if not all(t.is_cuda for t in panels):
        return False
    dev = torch.cuda.current_device()
    for t in panels:
        es = t.element_size()
        if not t.is_cuda or t.device.index != dev or t.data_ptr() % 16 or (t.stride(0) * es) % 16:
            return False
    return pdl.query(key) == "yes"


def chunk_groups(wp: WorkerPlan):
    """The Worker's chunk launches, in order: its own chunk (computes at once), then
    two groups of contiguous chunks.  The broadcasts arrive in chunk order, so the
    second group is the chunk that lands first when the own chunk sits at an end of
    the row (c = 0: [1], then [2..]; c = Gc-1: [0], then [1..Gc-2]) -- it computes
    while the rest lands -- and otherwise the chunks before / after the own one
    (whose earlier chunks already landed while the own chunk computed)."""
    c, G = wp.c, wp.Gc
    if G >= 3 and c == 0:
        return [[0], [1], list(range(2, G))]
    if G >= 3 and c == G - 1:
        return [[c], [0], list(range(1, c))]
    return [[c], list(range(0, c)), list(range(c + 1, G))]


_raw_streams = {}


def _raw_ready(grp, raw_works):
    """An event after the landing of the raw chunks of `grp` (None: all local),
    recorded on a helper stream so no compute stream waits for them early."""
    pending = [raw_works[j] for j in grp if j in raw_works]
    if not pending:
        return None
    dev = torch.cuda.current_device()
    if dev not in _raw_streams:
        _raw_streams[dev] = torch.cuda.Stream(device=dev)
    s = _raw_streams[dev]
    ev = torch.cuda.Event()
    with torch.cuda.stream(s):
        for w in pending:
            w.wait()
        ev.record(s)
    return ev


def compute_groups(wp: WorkerPlan, bufs: PanelBuffers, Bp, compute, works, concurrent=None, raw_works=None):
    """The chunk computations of exchange_overlapped, in at most three launches
    so each stays wave-efficient: the own chunk at once, then the chunks before
    it (broadcast first, so they land first), then the chunks after it.
    works: chunk -> broadcast handle (absent = already resident).

    concurrent (default: tasks_may_overlap(A panel, B panel)): the
    later groups go on side streams, each with its own scratch slot, that wait
    only for their own broadcasts (and the B panel libpdl prepared), so
    their CTAs fill the SMs the previous launch leaves idle in its last wave
    (three serial launches each round up to whole waves); the Worker stream
    joins them before returning.  C regions are disjoint, so C is bitwise the
    serial result."""
    c = wp.c
    if concurrent is None:
        concurrent = tasks_may_overlap(bufs.A, Bp)
    main = torch.cuda.current_stream() if concurrent else None
    groups = chunk_groups(wp)
    first = True
    joins = []
    if concurrent:
        ready = torch.cuda.Event()
        ready.record(main)   # everything the chunks need (B panel, own chunk) is enqueued
    for grp in groups:
        if not grp:
            continue
        lo, hi = chunk_rows(wp, grp[0])[0], chunk_rows(wp, grp[-1])[1]
        if hi <= lo or wp.cols <= 0:
            continue
        kw = {}   # raw A rows only for variants that read them (compute callbacks may not take them)
        if bufs.Araw is not None:
            kw["raw"] = (bufs.Araw[lo:hi], _raw_ready(grp, raw_works or {}))
        if first or not concurrent:
            for j in grp:
                if j != c and j in works:
                    works[j].wait()
            compute(grp[0], lo, hi, bufs.A[lo:hi], Bp, first, **kw)
        else:
            side = _side_stream(len(joins))
            side.wait_event(ready)
            with torch.cuda.stream(side):
                for j in grp:
                    if j in works:
                        works[j].wait()
                pdl.set_stream(side)
                try:
                    compute(grp[0], lo, hi, bufs.A[lo:hi], Bp, first, slot=len(joins) + 1, **kw)
                finally:
                    pdl.set_stream(main)
                done = torch.cuda.Event()
                done.record(side)
            joins.append(done)
        first = False
    for ev in joins:
        main.wait_event(ev)


def chunk_task(Cblock, wp: WorkerPlan, tile=0):
    """compute() for exchange_overlapped: one PDL_TASK_LOCAL task per A chunk
    on this process's Worker; the prepared B panel is reused after the first;
    `slot` is the task's scratch slot (compute_groups gives each concurrent
    launch group its own)."""
    def compute(j, lo, hi, Arows, Bp, first, slot=0, raw=None):
        Cv = Cblock[lo:hi]
        if Arows.dtype == torch.uint8:   # prepared A rows (PanelBuffers prep_bytes)
            Araw, ev = raw if raw is not None else (None, None)
            pdl.task_matmul_prepared(Arows, Bp, Cv, M=hi - lo, N=wp.cols, K=wp.K, Araw=Araw,
                                     lda_raw=0 if Araw is None else Araw.stride(0), raw_ready=ev,
                                     ldb=Bp.stride(0), ldc=Cv.stride(0), reuse_b=not first, slot=slot)
        else:
            pdl.task_matmul(Arows, Bp, Cv, M=hi - lo, N=wp.cols, K=wp.K, tile=tile, lda=Arows.stride(0),
                            ldb=Bp.stride(0), ldc=Cv.stride(0), local=True, reuse_b=not first, slot=slot)
        pdl.run_async()
    return compute


def local_task(Apanel, Bpanel, Cblock, wp: WorkerPlan, tile=0, run=True):
    """Run this Worker's rectangle through libpdl on the gathered panels."""
    if wp.rows == 0 or wp.cols == 0:
        return
    pdl.task_matmul(Apanel, Bpanel, Cblock, M=wp.M, N=wp.N, K=wp.K, tile=tile,
                    lda=Apanel.stride(0), ldb=Bpanel.stride(0), ldc=Cblock.stride(0), panels=True)
    if run:
        pdl.run_async()


def distributed_matmul(A_full, B_full, C_full, tile=0, group=None, overlap=True):
    """Public multi-Worker API: every rank passes the full (host or device)
    A, B and its own C; rank r writes its rectangle of C.  Host operands are
    copied chunk-wise to the Worker (PCIe), exchanged over NVLink (overlapped
    with the tile kernels unless overlap=False) -- or through host memory when
    the descriptor joins the Workers by no interconnect -- computed, and the C
    block copied back (PCIe)."""
    rank = dist.get_rank()
    if not (A_full.dtype == B_full.dtype == C_full.dtype):
        raise TypeError(f"A, B, C must have one dtype (got {A_full.dtype}, {B_full.dtype}, {C_full.dtype})")
    M, K = A_full.shape
    N = B_full.shape[1]
    if B_full.shape[0] != K or tuple(C_full.shape) != (M, N):
        raise ValueError(f"shapes do not chain: A {tuple(A_full.shape)} @ B {tuple(B_full.shape)} -> "
                         f"C {tuple(C_full.shape)}")
    wp = worker_plan(M, N, K, tile, rank, group)
    grid = Grid(wp.Gr, wp.Gc, rank, via_host=exchange_path(group) == "host")
    dev = torch.device("cuda", torch.cuda.current_device())
    Ach, Bch = chunk_from_full(A_full, B_full, wp)
    Ach, Bch = Ach.to(dev, non_blocking=True), Bch.to(dev, non_blocking=True)
    bufs = panel_buffers(wp, A_full.dtype, dev, prepared=overlap)
    Cb = torch.empty((wp.rows, wp.cols), dtype=C_full.dtype, device=dev)
    pdl.set_stream(torch.cuda.current_stream())
    if overlap:
        exchange_overlapped(Ach, Bch, wp, grid, bufs, chunk_task(Cb, wp, tile))
    else:
        Ap, Bp = exchange(Ach, Bch, wp, grid, bufs)
        local_task(Ap, Bp, Cb, wp, tile)
    pdl.sync()
    C_full[wp.row0: wp.row1, wp.col0: wp.col1].copy_(Cb)
    return wp
