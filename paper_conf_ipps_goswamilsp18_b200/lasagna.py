"""Thin Python binding of liblasagna.so (include/lasagna.h) — argument marshalling only.

Every step of the hot path runs in the library's sm_100a kernels; torch only supplies device
memory (workspaces, outputs), pinned host buffers and the current CUDA stream.  There is no
CPU fallback: if the shared library cannot be loaded, every call raises.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import torch

from . import build as _build

OK, EINVAL, ERANGE, ENOSPC, ECUDA = 0, 1, 2, 3, 4
NONE = 0xFFFFFFFF
_NAMES = {0: "OK", 1: "EINVAL", 2: "ERANGE", 3: "ENOSPC", 4: "ECUDA"}


class LasagnaError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"lasagna {_NAMES.get(status, status)}: {msg}")
        self.status = status


class _Stats(ctypes.Structure):
    _fields_ = [("n_pairs", ctypes.c_uint64), ("n_greedy", ctypes.c_uint64),
                ("fp_false_matches", ctypes.c_uint64), ("kernel_launches", ctypes.c_uint64),
                ("rounds_max", ctypes.c_uint32), ("passes", ctypes.c_uint32),
                ("lengths_per_pass", ctypes.c_uint32), ("key_sort_bits", ctypes.c_uint32),
                ("sort_launches", ctypes.c_uint32), ("search_launches", ctypes.c_uint32),
                ("bucketed", ctypes.c_uint32),
                ("ms_table", ctypes.c_float), ("ms_sort", ctypes.c_float),
                ("ms_search", ctypes.c_float),
                ("ms_greedy", ctypes.c_float),
                ("greedy_pair_rounds", ctypes.c_uint64), ("pruned_entries", ctypes.c_uint64),
                ("partition_levels", ctypes.c_uint32),
                ("hash_subpasses", ctypes.c_uint32)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


class ShardGeom(ctypes.Structure):
    """lasagna_shard_geom (include/lasagna.h): sizes of the sharded fast path."""
    _fields_ = [("levels", ctypes.c_uint32), ("last_bits", ctypes.c_uint32),
                ("nb_pad", ctypes.c_uint32), ("vbits", ctypes.c_uint32),
                ("n_pad", ctypes.c_uint64), ("slice", ctypes.c_uint64), ("cap1", ctypes.c_uint64),
                ("send_entries", ctypes.c_uint64), ("fill_words", ctypes.c_uint64),
                ("part_bytes", ctypes.c_uint64), ("buckets", ctypes.c_uint64)]


class GreedyRank(ctypes.Structure):
    """lasagna_greedy_rank: one rank's buffers, as device pointers valid in this process."""
    _fields_ = [(k, ctypes.c_void_p) for k in
                ("pool", "pool2", "pool_count", "ctr", "best", "claimed", "succ", "olen", "tail")]


_lib = None


def lib() -> ctypes.CDLL:
    """Load the in-tree liblasagna.so (building it first if sources are newer and nvcc exists)."""
    global _lib
    if _lib is not None:
        return _lib
    checked = os.environ.get("LASAGNA_CHECKED", "") == "1"  # bounds-checked build (tests)
    path = _build.SO_CHECKED if checked else _build.SO
    try:
        if _build.stale(checked):
            _build.build(checked=checked)
    except RuntimeError:
        if not os.path.exists(path):
            raise
    if not os.path.exists(path):
        raise LasagnaError(ECUDA, f"{path} missing: run __graft_entry__.build()")
    L = ctypes.CDLL(path)
    vp, u64, u32, sz = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_size_t
    psz = ctypes.POINTER(ctypes.c_size_t)
    pu64 = ctypes.POINTER(ctypes.c_uint64)
    pu32 = ctypes.POINTER(ctypes.c_uint32)
    L.lasagna_last_error.restype = ctypes.c_char_p
    L.lasagna_kernel_launches.restype = u64
    L.lasagna_words_per_read.argtypes = [u32]
    L.lasagna_words_per_read.restype = u32
    sigs = {
        "lasagna_load_reads": [vp, u64, u32, vp, vp, vp],
        "lasagna_fingerprints": [vp, u64, u32, u32, vp, vp, vp],
        "lasagna_overlaps": [vp, u64, u32, u32, vp, psz, vp, vp, vp, u64, pu64, vp],
        "lasagna_overlaps_approx": [vp, u64, u32, u32, vp, psz, vp, vp, vp, u64, pu64, vp],
        "lasagna_greedy_graph": [vp, u64, u32, u32, u32, vp, psz, vp, vp,
                                 ctypes.POINTER(_Stats), vp],
        "lasagna_greedy_graph_ascii": [vp, u64, u32, u32, u32, vp, psz, vp, vp, vp, vp,
                                       ctypes.POINTER(_Stats), vp],
        "lasagna_plan": [u64, u32, u32, sz, pu32, psz],
        "lasagna_sort_u64": [vp, vp, u64, u32, u32, vp, psz, vp],
        "lasagna_greedy_pairs": [u64, vp, vp, vp, u64, vp, psz, vp, vp, pu32, vp],
        "lasagna_compress": [vp, u64, u32, vp, vp, vp, psz, vp, u64, vp, vp, u64, pu64, pu64,
                             vp],
        "lasagna_shard_geometry": [u64, u32, u32, u32, ctypes.POINTER(ShardGeom)],
        "lasagna_shard_part_bytes": [u64, u32, u32, u32, u32, psz],
        "lasagna_shard_scatter": [vp, u64, u64, u64, u32, u32, u32, u32, u32, vp, vp, vp, vp, vp],
        "lasagna_shard_partition": [vp, vp, u64, u32, u32, u32, u32, u32, vp, vp, vp],
        "lasagna_shard_join": [vp, u64, u32, u32, u32, u32, u32, u32, vp, vp, u64, vp, vp, vp],
        "lasagna_greedy_shard_length": [ctypes.POINTER(GreedyRank), u32, ctypes.c_int32, u64,
                                        u64, u32, vp],
        "lasagna_peer_alloc": [sz, ctypes.POINTER(ctypes.c_void_p), vp],
        "lasagna_peer_free": [vp],
        "lasagna_peer_open": [vp, ctypes.POINTER(ctypes.c_void_p)],
        "lasagna_peer_close": [vp],
    }
    for name, args in sigs.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = ctypes.c_int
    _lib = L
    return L


def _check(status: int) -> None:
    if status != OK:
        raise LasagnaError(status, lib().lasagna_last_error().decode(errors="replace"))


def _stream(device=None) -> int:
    return torch.cuda.current_stream(device).cuda_stream


def _ptr(t: torch.Tensor | None):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def kernel_launches() -> int:
    """Process-wide number of kernels liblasagna.so has launched."""
    return int(lib().lasagna_kernel_launches())


def words_per_read(L: int) -> int:
    return int(lib().lasagna_words_per_read(L))


def _workspace(nbytes: int, device) -> torch.Tensor:
    return torch.empty(max(int(nbytes), 256), dtype=torch.uint8, device=device)


# ---------------------------------------------------------------------------- a1
def load_reads(ascii, device: str | torch.device = "cuda", check: bool = True):
    """2-bit pack reads on the GPU.  ``ascii``: (n, L) uint8 tensor on the device or in
    page-locked host memory (read in place by the kernel), or a numpy array (copied into a
    pinned staging tensor first).  Returns the packed u64 rows as an int64 tensor [n, W]."""
    if not isinstance(ascii, torch.Tensor):
        ascii = torch.from_numpy(ascii).pin_memory()
    if ascii.dtype != torch.uint8 or ascii.dim() != 2:
        raise ValueError("ascii must be a (n, L) uint8 tensor")
    ascii = ascii.contiguous()
    if not ascii.is_cuda and not ascii.is_pinned():
        ascii = ascii.pin_memory()
    n, L = ascii.shape
    dev = ascii.device if ascii.is_cuda else torch.device(device)
    packed = torch.empty((n, words_per_read(L)), dtype=torch.int64, device=dev)
    bad = torch.empty(1, dtype=torch.int64, device=dev)
    with torch.cuda.device(dev):
        _check(lib().lasagna_load_reads(_ptr(ascii), n, L, _ptr(packed), _ptr(bad), _stream(dev)))
    if check:
        b = int(bad.item()) & 0xFFFFFFFFFFFFFFFF
        if b != 0xFFFFFFFFFFFFFFFF:
            raise LasagnaError(EINVAL, f"read {b} holds a byte outside ACGTacgt")
    return packed


# ---------------------------------------------------------------------------- a2
def fingerprints(packed: torch.Tensor, n: int, L: int, l_min: int):
    """(pfx, sfx) int64 tensors [L - l_min + 1, 2n] holding the u64 fingerprints."""
    V = 2 * n
    pfx = torch.empty((L - l_min + 1, V), dtype=torch.int64, device=packed.device)
    sfx = torch.empty_like(pfx)
    with torch.cuda.device(packed.device):
        _check(lib().lasagna_fingerprints(_ptr(packed), n, L, l_min, _ptr(pfx), _ptr(sfx),
                                          _stream(packed.device)))
    return pfx, sfx


# ---------------------------------------------------------------------------- a2..a5
def overlaps(packed: torch.Tensor, n: int, L: int, l_min: int, capacity: int | None = None,
             approx: bool = False):
    """All read-end pairs sorted by (l desc, a, b): (pl uint8, pa int32, pb int32) tensors
    (pa/pb hold u32 vertex ids).  approx: the paper's 128-bit fingerprint acceptance
    (lasagna_overlaps_approx) instead of the exact base comparison."""
    dev = packed.device
    fn = lib().lasagna_overlaps_approx if approx else lib().lasagna_overlaps
    ws_bytes = ctypes.c_size_t(0)
    npairs = ctypes.c_uint64(0)
    with torch.cuda.device(dev):
        _check(fn(_ptr(packed), n, L, l_min, None, ctypes.byref(ws_bytes), None, None, None, 0,
                  ctypes.byref(npairs), _stream(dev)))
        for _ in range(4):
            ws = _workspace(ws_bytes.value, dev)
            cap = max(1, int(capacity if capacity is not None else max(1, n)))
            pa = torch.empty(cap, dtype=torch.int32, device=dev)
            pb = torch.empty(cap, dtype=torch.int32, device=dev)
            pl = torch.empty(cap, dtype=torch.uint8, device=dev)
            st = fn(_ptr(packed), n, L, l_min, _ptr(ws), ctypes.byref(ws_bytes), _ptr(pa),
                    _ptr(pb), _ptr(pl), cap, ctypes.byref(npairs), _stream(dev))
            if st == ENOSPC:
                if npairs.value > cap:
                    capacity = npairs.value
                continue
            _check(st)
            m = int(npairs.value)
            return pl[:m], pa[:m], pb[:m]
    raise LasagnaError(ENOSPC, "overlaps: could not size workspace/capacity")


# ---------------------------------------------------------------------------- a1..a7
@dataclass
class GraphResult:
    succ: torch.Tensor   # int32 [2n] (u32 ids; NONE = -1)
    olen: torch.Tensor   # uint8 [2n]
    stats: dict


def plan(n: int, L: int, l_min: int, budget_bytes: int):
    lp = ctypes.c_uint32(0)
    ws = ctypes.c_size_t(0)
    st = lib().lasagna_plan(n, L, l_min, budget_bytes, ctypes.byref(lp), ctypes.byref(ws))
    if st == ENOSPC:
        return 0, int(ws.value)
    _check(st)
    return int(lp.value), int(ws.value)


class GreedyGraph:
    """Reusable greedy-graph runner: owns the workspace (sized once, kept across calls)."""

    def __init__(self, n: int, L: int, l_min: int, device="cuda", lengths_per_pass: int = 0,
                 budget_bytes: int | None = None):
        """budget_bytes: device memory for the WORKSPACE (lengths_per_pass = 0 lets the a8
        planner pick the largest length group that fits it).  Default: 92 % of the free
        memory less what the runner allocates besides the workspace (the outputs and the
        packed rows from_ascii writes)."""
        self.n, self.L, self.l_min = n, L, l_min
        self.device = torch.device(device)
        if self.device.type == "cuda" and self.device.index is None:
            self.device = torch.device("cuda", torch.cuda.current_device())
        planned = None
        if lengths_per_pass == 0:
            if budget_bytes is None:
                free, _ = torch.cuda.mem_get_info(self.device)
                budget_bytes = int(free * 0.92) - self.side_bytes(n, L)
            lp, need = plan(n, L, l_min, max(0, budget_bytes))
            if lp == 0:
                raise LasagnaError(ENOSPC, f"needs {need} bytes of workspace, budget {budget_bytes}")
            lengths_per_pass, planned = lp, need
        self.lengths_per_pass = lengths_per_pass
        ws = ctypes.c_size_t(0)
        _check(lib().lasagna_greedy_graph(None, n, L, l_min, lengths_per_pass, None,
                                          ctypes.byref(ws), None, None, None, None))
        # below one whole length the planner's workspace runs hash-range sub-passes (smaller
        # than the one-length query)
        self.ws_bytes = int(ws.value) if planned is None else min(int(ws.value), planned)
        self.ws = _workspace(self.ws_bytes, self.device)
        self.succ = torch.empty(2 * n, dtype=torch.int32, device=self.device)
        self.olen = torch.empty(2 * n, dtype=torch.uint8, device=self.device)

    @staticmethod
    def side_bytes(n: int, L: int) -> int:
        """Device bytes a runner holds besides its workspace: succ u32[2n], olen u8[2n], the
        packed rows u64[n][W] and first_bad (from_ascii)."""
        return 2 * n * 5 + n * 8 * words_per_read(L) + 4096

    def _check_input(self, t: torch.Tensor, kind: str) -> None:
        if kind == "packed":
            shape, dtype = (self.n, words_per_read(self.L)), torch.int64
        else:
            shape, dtype = (self.n, self.L), torch.uint8
        if t.dtype != dtype or tuple(t.shape) != shape:
            raise ValueError(f"{kind} input must be a {dtype} tensor of shape {shape}, "
                             f"got {t.dtype} {tuple(t.shape)}")
        if not t.is_contiguous():
            raise ValueError(f"{kind} input must be contiguous")
        if t.is_cuda and t.device != self.device:
            raise ValueError(f"{kind} input on {t.device}, runner on {self.device}")

    def __call__(self, packed: torch.Tensor, stats: bool = True) -> GraphResult:
        """a1-a7 on already packed reads (lasagna_greedy_graph)."""
        self._check_input(packed, "packed")
        if not packed.is_cuda:
            raise ValueError("packed rows must be device memory")
        return self._run(lambda ws, st: lib().lasagna_greedy_graph(
            _ptr(packed), self.n, self.L, self.l_min, self.lengths_per_pass, _ptr(self.ws),
            ctypes.byref(ws), _ptr(self.succ), _ptr(self.olen), st, _stream(self.device)), stats)

    def from_ascii(self, ascii: torch.Tensor, stats: bool = True) -> GraphResult:
        """a1-a7 from (n, L) uint8 ASCII reads on the device or in page-locked host memory
        (lasagna_greedy_graph_ascii: staging fused into the first table pass)."""
        # device memory or page-locked host memory (torch-pinned or cudaHostRegister'ed): the
        # library checks the pointer and rejects pageable memory with EINVAL
        ascii = ascii.contiguous()
        self._check_input(ascii, "ascii")
        if getattr(self, "packed", None) is None:
            self.packed = torch.empty((self.n, words_per_read(self.L)), dtype=torch.int64,
                                      device=self.device)
            self.first_bad = torch.empty(1, dtype=torch.int64, device=self.device)
        return self._run(lambda ws, st: lib().lasagna_greedy_graph_ascii(
            _ptr(ascii), self.n, self.L, self.l_min, self.lengths_per_pass, _ptr(self.ws),
            ctypes.byref(ws), _ptr(self.packed), _ptr(self.first_bad), _ptr(self.succ),
            _ptr(self.olen), st, _stream(self.device)), stats)

    def _run(self, call, stats: bool) -> GraphResult:
        st = _Stats()
        for _ in range(4):
            ws = ctypes.c_size_t(self.ws_bytes)
            with torch.cuda.device(self.device):
                rc = call(ws, ctypes.byref(st) if stats else None)
            if rc == ENOSPC and ws.value > self.ws_bytes:
                self.ws_bytes = int(ws.value)
                self.ws = None
                self.ws = _workspace(self.ws_bytes, self.device)
                continue
            _check(rc)
            return GraphResult(self.succ, self.olen, st.as_dict() if stats else {})
        raise LasagnaError(ENOSPC, "greedy_graph: could not size the workspace")


class GraphPipeline:
    """Greedy graphs of a stream of read batches with two batches in flight (a8 level 2 across
    batches): batch k+1's host -> device copy (one copy stream, so the copies run back to back
    at the link's rate) overlaps batch k's device work and its result read-back.  Two
    GreedyGraph runners with their own workspaces and device input buffers, one compute stream
    and one host thread each (a call blocks its thread until its stream is done); batch k goes
    to runner k % 2, whose buffer is refilled only after its previous call returned.
    Plumbing only: every step of the path runs in liblasagna.so (lasagna_greedy_graph_ascii on
    the device copy of the batch)."""

    def __init__(self, n: int, L: int, l_min: int, device="cuda", lengths_per_pass: int = 0,
                 stream_input: bool = False):
        """stream_input: each runner reads its batch straight from page-locked host memory
        (lasagna_greedy_graph_ascii's chunked DMA, the scatter of chunk c running while chunk
        c+1 lands), so a batch's fingerprint/partition pass overlaps its own copy and no device
        input buffers are held; otherwise the batch is first copied whole to a device buffer.
        The whole-batch copy is the faster default at cfg3 (80.0 vs 97.5 ms per batch, r02o):
        two lanes streaming at once interleave their chunk copies and event-ordered scatters."""
        dev = torch.device(device)
        if dev.index is None:  # the worker threads select the device by index
            dev = torch.device(dev.type, torch.cuda.current_device())
        self.n, self.L, self.device = n, L, dev
        self.stream_input = stream_input
        self.bufs = [] if stream_input else [
            torch.empty((n, L), dtype=torch.uint8, device=self.device) for _ in range(2)]
        # the two runners share what is free after the input buffers: half each, less what a
        # runner holds besides its workspace
        free, _ = torch.cuda.mem_get_info(self.device)
        budget = int(free * 0.92) // 2 - GreedyGraph.side_bytes(n, L)
        self.runners = [GreedyGraph(n, L, l_min, self.device, lengths_per_pass,
                                    budget_bytes=budget) for _ in range(2)]
        self.copy = torch.cuda.Stream(self.device)
        self.lanes = [torch.cuda.Stream(self.device) for _ in range(2)]

    def run(self, batches, outs) -> None:
        """batches[k]: (n, L) uint8 page-locked host tensor; outs[k]: (succ, olen) page-locked
        host tensors receiving batch k's result.  Returns when every result is on the host."""
        import queue
        import threading
        q = [queue.Queue(), queue.Queue()]
        free = [threading.Semaphore(1), threading.Semaphore(1)]
        errors = []

        def lane(j: int) -> None:
            try:
                torch.cuda.set_device(self.device)
                with torch.cuda.stream(self.lanes[j]):
                    while True:
                        item = q[j].get()
                        if item is None:
                            return
                        ev, k = item
                        if self.stream_input:  # chunked DMA from the host batch inside the call
                            r = self.runners[j].from_ascii(batches[k], stats=False)
                        else:
                            # wait on the host, not in-stream: a stream parked on an event wait
                            # can hold a hardware queue that the other lane's kernels share
                            ev.synchronize()
                            r = self.runners[j].from_ascii(self.bufs[j], stats=False)
                        outs[k][0].copy_(r.succ, non_blocking=True)
                        outs[k][1].copy_(r.olen, non_blocking=True)
                        self.lanes[j].synchronize()
                        free[j].release()
            except BaseException as e:  # re-raised by the caller's thread
                errors.append(e)
                free[j].release()

        th = [threading.Thread(target=lane, args=(j,)) for j in range(2)]
        for t in th:
            t.start()
        try:
            for k, b in enumerate(batches):
                j = k % 2
                free[j].acquire()  # runner j's previous batch has returned
                if errors:
                    break
                if self.stream_input:
                    q[j].put((None, k))
                    continue
                self.copy.wait_stream(self.lanes[j])
                with torch.cuda.stream(self.copy):
                    self.bufs[j].copy_(b, non_blocking=True)
                    ev = torch.cuda.Event()
                    ev.record(self.copy)
                q[j].put((ev, k))
        finally:
            for j in range(2):
                q[j].put(None)
            for t in th:
                t.join()
        if errors:
            raise errors[0]


def greedy_graph(packed: torch.Tensor, n: int, L: int, l_min: int, lengths_per_pass: int = 0,
                 stats: bool = True) -> GraphResult:
    g = GreedyGraph(n, L, l_min, packed.device, lengths_per_pass)
    r = g(packed, stats)
    return GraphResult(r.succ.clone(), r.olen.clone(), r.stats)


# ---------------------------------------------------------------------------- Compress
@dataclass
class Contigs:
    bases: torch.Tensor    # uint8 [total]: ASCII contigs back to back
    offsets: torch.Tensor  # int64 [c + 1]: contig k = bases[offsets[k]:offsets[k+1]]
    seeds: torch.Tensor    # int32 [c]: seed vertex of each contig (u32 ids)


def compress(packed: torch.Tensor, n: int, L: int, succ: torch.Tensor, olen: torch.Tensor,
             workspace: torch.Tensor | None = None) -> Contigs:
    """Paths and contigs of a greedy string graph (lasagna_compress; Fig. 7)."""
    dev = packed.device
    ws_bytes = ctypes.c_size_t(0)
    nc, tot = ctypes.c_uint64(0), ctypes.c_uint64(0)
    f = lib().lasagna_compress
    with torch.cuda.device(dev):
        _check(f(None, n, L, None, None, None, ctypes.byref(ws_bytes), None, 0, None, None, 0,
                 ctypes.byref(nc), ctypes.byref(tot), _stream(dev)))
        if workspace is None or workspace.numel() < ws_bytes.value:
            workspace = _workspace(ws_bytes.value, dev)
        ws_bytes = ctypes.c_size_t(workspace.numel())
        args = (_ptr(packed), n, L, _ptr(succ), _ptr(olen), _ptr(workspace), ctypes.byref(ws_bytes))
        st = f(*args, None, 0, None, None, 0, ctypes.byref(nc), ctypes.byref(tot), _stream(dev))
        if st != ENOSPC:
            _check(st)
        bases = torch.empty(max(1, tot.value), dtype=torch.uint8, device=dev)
        offs = torch.empty(nc.value + 1, dtype=torch.int64, device=dev)
        seeds = torch.empty(max(1, nc.value), dtype=torch.int32, device=dev)
        _check(f(*args, _ptr(bases), tot.value, _ptr(offs), _ptr(seeds), nc.value + 1,
                 ctypes.byref(nc), ctypes.byref(tot), _stream(dev)))
    return Contigs(bases[:tot.value], offs, seeds[:nc.value])


# ---------------------------------------------------------------------------- phase entry points
def sort_u64(keys: torch.Tensor, bit_lo: int = 0, bit_hi: int = 64) -> torch.Tensor:
    """Stable LSD sort (in place) of an int64 tensor holding u64 keys, by bits [lo, hi)."""
    keys = keys.contiguous()
    dev = keys.device
    scratch = torch.empty_like(keys)
    ws_bytes = ctypes.c_size_t(0)
    with torch.cuda.device(dev):
        _check(lib().lasagna_sort_u64(_ptr(keys), _ptr(scratch), keys.numel(), bit_lo, bit_hi,
                                      None, ctypes.byref(ws_bytes), _stream(dev)))
        ws = _workspace(ws_bytes.value, dev)
        _check(lib().lasagna_sort_u64(_ptr(keys), _ptr(scratch), keys.numel(), bit_lo, bit_hi,
                                      _ptr(ws), ctypes.byref(ws_bytes), _stream(dev)))
    return keys


def greedy_pairs(n: int, pl: torch.Tensor, pa: torch.Tensor, pb: torch.Tensor):
    """Greedy claim on a given candidate list -> (succ int32 [2n], olen uint8 [2n], rounds)."""
    dev = pa.device
    count = pa.numel()
    succ = torch.empty(2 * n, dtype=torch.int32, device=dev)
    olen = torch.empty(2 * n, dtype=torch.uint8, device=dev)
    ws_bytes = ctypes.c_size_t(0)
    rounds = ctypes.c_uint32(0)
    with torch.cuda.device(dev):
        _check(lib().lasagna_greedy_pairs(n, None, None, None, count, None, ctypes.byref(ws_bytes),
                                          None, None, None, _stream(dev)))
        ws = _workspace(ws_bytes.value, dev)
        _check(lib().lasagna_greedy_pairs(n, _ptr(pl.contiguous()), _ptr(pa.contiguous()),
                                          _ptr(pb.contiguous()), count, _ptr(ws),
                                          ctypes.byref(ws_bytes), _ptr(succ), _ptr(olen),
                                          ctypes.byref(rounds), _stream(dev)))
    return succ, olen, int(rounds.value)
