"""Multi-GPU greedy string graph: one process per GPU, tables partitioned by hash range.

SURVEY §8(e); paper: distributed map/shuffle/reduce and its stated future work
"partitioning the suffixes/prefixes based on their fingerprints rather than on lengths"
(P:L333).  Every rank holds a contiguous slice of the reads; per length group:

  1. all-gather of the 2-bit packed reads (every rank can verify any candidate)   [NCCL]
  2. table keys of the LOCAL reads (global vertex ids)                           [table_kernel]
  3. partition by hash range: one 8-bit radix pass on the top key bits; bucket b
     (256 buckets) belongs to rank  b * g // 256  (contiguous ranges, any g <= 256) [onesweep]
  4. per length: all-to-all of the key shards (split sizes from the bucket counts) [NCCL]
  5. per length: radix sort of the received shard + join (search + verify)     [onesweep, join]
  6. all-gather of the candidate pairs; every rank runs the same deterministic
     greedy on the same pair set -> identical succ/olen on every rank          [NCCL, greedy]

The greedy result depends only on the pair SET (the greedy visits it in (l desc, a, b)
order), so the output equals the single-GPU result bit for bit.

Compute goes through a backend object: `CudaBackend` calls liblasagna.so (the product);
tests drive the same orchestration over gloo with a CPU backend of their own.
"""
from __future__ import annotations

import ctypes
import json
import math
import os
import time

import torch
import torch.distributed as dist

from . import lasagna as lz

DEST_BITS = 8  # hash-range buckets for the partition (256; rank(b) = b * g // 256)


# ------------------------------------------------------------------------------ backend
class CudaBackend:
    """Phase calls into liblasagna.so (argument marshalling only)."""

    def __init__(self, device):
        self.device = torch.device(device)
        self.L = lz.lib()

    def _s(self):
        return lz._stream(self.device)

    def pack(self, ascii_local: torch.Tensor) -> torch.Tensor:
        return lz.load_reads(ascii_local, device=self.device)

    def vertex_bits(self, n_total: int) -> int:
        self.L.lasagna_vertex_bits.restype = ctypes.c_uint32
        self.L.lasagna_vertex_bits.argtypes = [ctypes.c_uint64]
        return int(self.L.lasagna_vertex_bits(n_total))

    def sort_bits(self, n_total: int) -> int:
        self.L.lasagna_key_sort_bits.restype = ctypes.c_uint32
        self.L.lasagna_key_sort_bits.argtypes = [ctypes.c_uint64]
        return int(self.L.lasagna_key_sort_bits(n_total))

    def table_keys(self, packed_local, n_local, read_offset, n_total, L, l_lo, l_hi):
        G = l_hi - l_lo + 1
        tab = torch.empty((G, 2 * n_local), dtype=torch.int64, device=self.device)
        f = self.L.lasagna_table_keys
        f.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64,
                      ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p,
                      ctypes.c_void_p]
        f.restype = ctypes.c_int
        lz._check(f(lz._ptr(packed_local), n_local, read_offset, n_total, L, l_lo, l_hi,
                    lz._ptr(tab), self._s()))
        return tab

    def sort_segments(self, keys: torch.Tensor, seg_len: int, n_seg: int, lo: int, hi: int):
        if seg_len == 0 or n_seg == 0:
            return keys
        f = self.L.lasagna_sort_segments
        f.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32,
                      ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p,
                      ctypes.POINTER(ctypes.c_size_t), ctypes.c_void_p]
        f.restype = ctypes.c_int
        scratch = torch.empty_like(keys)
        ws_bytes = ctypes.c_size_t(0)
        lz._check(f(lz._ptr(keys), lz._ptr(scratch), seg_len, n_seg, lo, hi, None,
                    ctypes.byref(ws_bytes), self._s()))
        ws = lz._workspace(ws_bytes.value, self.device)
        lz._check(f(lz._ptr(keys), lz._ptr(scratch), seg_len, n_seg, lo, hi, lz._ptr(ws),
                    ctypes.byref(ws_bytes), self._s()))
        return keys

    def digit_counts(self, keys, seg_len, n_seg, shift, bits) -> torch.Tensor:
        counts = torch.empty((n_seg, 256), dtype=torch.int32, device=self.device)
        f = self.L.lasagna_digit_counts
        f.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32,
                      ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p]
        f.restype = ctypes.c_int
        lz._check(f(lz._ptr(keys), seg_len, n_seg, shift, bits, lz._ptr(counts), self._s()))
        return counts[:, : 1 << bits].to(torch.int64).cpu()

    def new_pairs(self, capacity: int):
        return (torch.empty(max(1, capacity), dtype=torch.int64, device=self.device),
                torch.zeros(2, dtype=torch.int64, device=self.device))

    def join(self, keys, count, packed_all, n_total, L, l, pairs, counters):
        f = self.L.lasagna_join
        f.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_uint64,
                      ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_uint64,
                      ctypes.c_void_p, ctypes.c_void_p]
        f.restype = ctypes.c_int
        lz._check(f(lz._ptr(keys), count, lz._ptr(packed_all), n_total, L, l, lz._ptr(pairs),
                    pairs.numel(), lz._ptr(counters), self._s()))

    def greedy_pairs(self, n_total, pl, pa, pb):
        return lz.greedy_pairs(n_total, pl, pa, pb)[:2]


# ------------------------------------------------------------------------------ orchestration
def shard_range(n_total: int, world: int, rank: int):
    """Reads [lo, hi) of `rank`: equal slices of ceil(n/g) rows (the all-gather layout)."""
    n_pad = -(-n_total // world) if n_total else 0
    lo = min(n_total, rank * n_pad)
    return lo, min(n_total, lo + n_pad), n_pad


def owner_of_buckets(world: int) -> list[int]:
    """Hash-range ownership: bucket b of the top DEST_BITS key bits -> rank b * g // 256."""
    return [b * world // (1 << DEST_BITS) for b in range(1 << DEST_BITS)]


class _Coll:
    """Collectives of one process group.  NCCL moves device tensors directly over NVLink;
    a gloo group (CPU tests, or several ranks sharing one GPU) stages through host memory."""

    def __init__(self, group, device):
        self.g = group
        self.host = dist.get_backend(group) == "gloo"
        self.device = device

    def _in(self, t):
        return t.cpu() if self.host else t

    def all_gather_into_tensor(self, out, inp):
        if self.host and out.device.type != "cpu":
            o = torch.empty(out.shape, dtype=out.dtype)
            dist.all_gather_into_tensor(o, inp.cpu(), group=self.g)
            out.copy_(o)
        else:
            dist.all_gather_into_tensor(out, inp, group=self.g)

    def all_to_all_single(self, out, inp, outs=None, ins=None):
        if self.host and out.device.type != "cpu":
            o = torch.empty(out.shape, dtype=out.dtype)
            dist.all_to_all_single(o, inp.cpu(), outs, ins, group=self.g)
            out.copy_(o)
        else:
            dist.all_to_all_single(out, inp, outs, ins, group=self.g)

    def all_reduce(self, t, op=dist.ReduceOp.SUM):
        if self.host and t.device.type != "cpu":
            h = t.cpu()
            dist.all_reduce(h, op=op, group=self.g)
            t.copy_(h)
        else:
            dist.all_reduce(t, op=op, group=self.g)

    def all_gather(self, outs, inp):
        if self.host and inp.device.type != "cpu":
            h = [torch.empty_like(o, device="cpu") for o in outs]
            dist.all_gather(h, inp.cpu(), group=self.g)
            for o, x in zip(outs, h):
                o.copy_(x)
        else:
            dist.all_gather(outs, inp, group=self.g)


def greedy_graph(ascii_local: torch.Tensor, n_total: int, L: int, l_min: int, backend=None,
                 group=None, lengths_per_pass: int = 0, pair_capacity: int | None = None):
    """Greedy string graph of the n_total reads spread over the ranks of `group` (rank r holds
    reads shard_range(n_total, g, r)).  Returns (succ, olen, stats) — identical on all ranks."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    be = backend or CudaBackend(ascii_local.device if ascii_local.is_cuda else "cuda")
    lo, hi, n_pad = shard_range(n_total, world, rank)
    n_local = hi - lo
    assert ascii_local.shape[0] == n_local, (ascii_local.shape, n_local)

    # 1. packed reads: local pack, all-gather (padded slices) -> every rank has all reads
    packed_local = be.pack(ascii_local)
    C = _Coll(group, packed_local.device)
    W = packed_local.shape[1] if packed_local.dim() == 2 else lz_words(L)
    buf = torch.zeros((n_pad, W), dtype=torch.int64, device=packed_local.device)
    buf[:n_local] = packed_local
    packed_all = torch.empty(world * n_pad * W, dtype=torch.int64, device=packed_local.device)
    C.all_gather_into_tensor(packed_all, buf.reshape(-1))
    packed_all = packed_all.view(world * n_pad, W)[:n_total]

    T = be.sort_bits(n_total)
    owner = torch.tensor(owner_of_buckets(world), dtype=torch.int64)
    n_len = L - l_min
    G = n_len if lengths_per_pass <= 0 else min(lengths_per_pass, n_len)
    # local pair buffer for all lengths (expected |P| ~ 3n at 40x coverage; grown on overflow)
    cap = pair_capacity if pair_capacity is not None else max(1 << 16, (6 * n_total) // world)
    pairs, counters = be.new_pairs(cap)
    bounds = []  # (l, end position in the local pair buffer) after each length
    for l_hi in range(L - 1, l_min - 1, -G):
        l_lo = max(l_min, l_hi - G + 1)
        Gc = l_hi - l_lo + 1
        # 2-3. local table, partitioned by destination hash range
        tab = be.table_keys(packed_local, n_local, lo, n_total, L, l_lo, l_hi)
        seg = 2 * n_local
        be.sort_segments(tab, seg, Gc, 64 - DEST_BITS, 64)
        cnt = be.digit_counts(tab, seg, Gc, 64 - DEST_BITS, DEST_BITS)          # [Gc, 256]
        send_counts = torch.zeros((Gc, world), dtype=torch.int64)
        send_counts.index_add_(1, owner, cnt)                                   # [Gc, g]
        # every rank learns what it receives: all-to-all of the count matrix
        sc = send_counts.t().contiguous().to(packed_all.device)                 # [g, Gc]
        rc = torch.empty_like(sc)
        C.all_to_all_single(rc, sc)
        recv_counts = rc.cpu().t().contiguous()                                 # [Gc, g]
        for l in range(l_hi, l_lo - 1, -1):
            s = l - l_lo
            ins = send_counts[s].tolist()
            outs = recv_counts[s].tolist()
            recv = torch.empty(sum(outs), dtype=torch.int64, device=packed_all.device)
            # 4. the key shard of my hash range from every rank
            C.all_to_all_single(recv, tab[s].contiguous(), outs, ins)
            # 5. sort + join (search + exact verification) of my shard of length l
            be.sort_segments(recv, recv.numel(), 1, 64 - T, 64)
            be.join(recv, recv.numel(), packed_all, n_total, L, l, pairs, counters)
            bounds.append((l, counters[0].clone()))
        del tab
    # 6. all-gather the candidate pairs of every length, then the replicated greedy
    found = int(counters[0].item())
    over = torch.tensor([1 if found > pairs.numel() else 0], dtype=torch.int64,
                        device=packed_all.device)
    C.all_reduce(over)
    if int(over.item()):
        need = torch.tensor([found], dtype=torch.int64, device=packed_all.device)
        C.all_reduce(need, op=dist.ReduceOp.MAX)
        return greedy_graph(ascii_local, n_total, L, l_min, be, group, lengths_per_pass,
                            int(need.item()) * 5 // 4 + 1)
    ends = torch.stack([b for _, b in bounds]).cpu().tolist() if bounds else []
    lengths = [l for l, _ in bounds]
    starts = [0] + ends[:-1]
    per_len = torch.tensor([e - s for s, e in zip(starts, ends)], dtype=torch.int64)
    all_per_len = [torch.empty_like(per_len) for _ in range(world)]
    C.all_gather(all_per_len, per_len)
    totals = [int(x.sum()) for x in all_per_len]
    mx = max(totals) if totals else 0
    mine = torch.zeros(max(1, mx), dtype=torch.int64, device=pairs.device)
    mine[:found] = pairs[:found]
    gathered = torch.empty(world * max(1, mx), dtype=torch.int64, device=pairs.device)
    C.all_gather_into_tensor(gathered, mine)
    gathered = gathered.view(world, max(1, mx))
    recs, ls = [], []
    for r in range(world):
        pos = 0
        for l, c in zip(lengths, all_per_len[r].tolist()):
            if c:
                recs.append(gathered[r, pos:pos + c])
                ls.append(torch.full((c,), l, dtype=torch.uint8, device=pairs.device))
            pos += c
    if recs:
        rec = torch.cat(recs)
        pl = torch.cat(ls)
    else:
        rec = torch.empty(0, dtype=torch.int64, device=pairs.device)
        pl = torch.empty(0, dtype=torch.uint8, device=pairs.device)
    pa = (rec >> 32).to(torch.int32)
    pb = (rec & 0xFFFFFFFF).to(torch.int64).to(torch.int32)
    succ, olen = be.greedy_pairs(n_total, pl, pa, pb)
    stats = {"n_pairs": int(rec.numel()), "fp_false_matches_local": int(counters[1].item()),
             "lengths_per_pass": G, "key_sort_bits": T}
    return succ, olen, stats


# ------------------------------------------------------------------------------ fast path
class _DevView:
    """A raw device buffer seen by torch (``__cuda_array_interface__``, zero copy): the
    library-allocated peer arena is initialised and gathered with ordinary tensor ops."""

    def __init__(self, ptr: int, nbytes: int):
        self.__cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1",
                                         "data": (ptr, False), "version": 3}


def _arena_layout(slice_: int) -> dict:
    """Byte offsets of one rank's peer arena: best u64[slice], claimed u32[slice/32],
    succ u32[slice], olen u8[slice], ctr u64[16], tail u64[4096] (256-byte aligned)."""
    off, lay = 0, {}
    for name, nbytes in (("best", 8 * slice_), ("claimed", slice_ // 8), ("succ", 4 * slice_),
                         ("olen", slice_), ("ctr", 16 * 8), ("tail", 4096 * 8)):
        lay[name] = off
        off += -(-max(nbytes, 1) // 256) * 256
    lay["total"] = off
    return lay


class PeerArena:
    """This rank's IPC-shareable greedy state and the peers' arenas opened in this process."""

    def __init__(self, slice_: int, device, group):
        self.L = lz.lib()
        self.lay = _arena_layout(slice_)
        self.slice = slice_
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.group = group
        ptr = ctypes.c_void_p()
        handle = ctypes.create_string_buffer(64)
        lz._check(self.L.lasagna_peer_alloc(self.lay["total"], ctypes.byref(ptr), handle))
        self.base = ptr.value
        self.view = torch.as_tensor(_DevView(self.base, self.lay["total"]), device=device)
        self.view.zero_()
        self.tensor("succ", torch.int32).fill_(-1)  # LASAGNA_NONE
        self.bases = [0] * self.world
        self.opened = []
        if self.world > 1:
            handles = [None] * self.world
            dist.all_gather_object(handles, handle.raw, group=group)
            for q, h in enumerate(handles):
                if q == self.rank:
                    self.bases[q] = self.base
                    continue
                pq = ctypes.c_void_p()
                lz._check(self.L.lasagna_peer_open(ctypes.create_string_buffer(h, 64),
                                                   ctypes.byref(pq)))
                self.bases[q] = pq.value
                self.opened.append(pq.value)
        else:
            self.bases[0] = self.base

    def tensor(self, name: str, dtype) -> torch.Tensor:
        n = {"best": 8 * self.slice, "claimed": self.slice // 8, "succ": 4 * self.slice,
             "olen": self.slice, "ctr": 128, "tail": 4096 * 8}[name]
        return self.view[self.lay[name]:self.lay[name] + n].view(dtype)

    def ptr(self, q: int, name: str) -> int:
        return self.bases[q] + self.lay[name]

    def close(self):
        torch.cuda.synchronize()
        if self.world > 1:
            dist.barrier(group=self.group)  # no peer still reads or writes my arena
        for p in self.opened:
            self.L.lasagna_peer_close(ctypes.c_void_p(p))
        self.opened = []
        if self.base:
            self.view = None
            self.L.lasagna_peer_free(ctypes.c_void_p(self.base))
            self.base = 0


def shard_geometry(n_total: int, world: int, L: int, l_min: int) -> "lz.ShardGeom":
    geo = lz.ShardGeom()
    lz._check(lz.lib().lasagna_shard_geometry(n_total, world, L, l_min, ctypes.byref(geo)))
    return geo


def fast_shard_range(n_total: int, world: int, rank: int):
    """Reads [lo, hi) of `rank` on the fast path: slices of n_pad = ceil(n/g) rounded up to
    16 rows (a rank's 2 n_pad read ends fill whole words of the claimed bitmap)."""
    n_pad = ((-(-n_total // world) if n_total else 0) + 15) // 16 * 16
    lo = min(n_total, rank * n_pad)
    return lo, min(n_total, lo + n_pad), n_pad


class RegionOverflow(RuntimeError):
    """A slack region of the sharded partition overflowed: rerun on the exact path."""


class _Phases:
    """CUDA-event pairs per phase on the call's stream, read once at the end (no host sync
    inside the call)."""

    def __init__(self, on: bool):
        self.on = on
        self.recs: list[tuple[str, torch.cuda.Event, torch.cuda.Event]] = []
        self.launches = {"scatter": 0, "refine": 0, "join": 0, "greedy_lengths": 0}

    def start(self, name):
        if not self.on:
            return None
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        self.recs.append((name, a, b))
        return b

    @staticmethod
    def stop(b):
        if b is not None:
            b.record()

    def totals(self) -> dict:
        out: dict[str, float] = {}
        for name, a, b in self.recs:
            out[name] = out.get(name, 0.0) + a.elapsed_time(b)
        return out


class ShardedGraph:
    """Reusable runner of the sharded fast path (include/lasagna.h "Sharded FAST path"): the
    peer arena (opened by every rank once), the pair pools, the packed-read buffer and the
    exchange / partition buffers are allocated once and kept across calls.  Per call: one fused
    scatter of the local reads per length group, two equal-split all-to-alls, the multi-source
    refine, then per length the join and the sharded greedy over peer memory — no host
    synchronisation until the end of the call.  Rank r holds reads fast_shard_range(n, g, r)."""

    def __init__(self, n_total: int, L: int, l_min: int, group=None, device=None,
                 lengths_per_pass: int = 0, pair_capacity: int | None = None):
        self.n, self.L, self.l_min, self.group = n_total, L, l_min, group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.dev = torch.device(device) if device is not None else \
            torch.device("cuda", torch.cuda.current_device())
        self.Lb = lz.lib()
        self.geo = shard_geometry(n_total, self.world, L, l_min)
        self.lo, self.hi, n_pad = fast_shard_range(n_total, self.world, self.rank)
        assert n_pad == self.geo.n_pad, (n_pad, self.geo.n_pad)
        self.n_local = self.hi - self.lo
        n_len = L - l_min
        G = n_len if lengths_per_pass <= 0 else min(lengths_per_pass, n_len)
        self.G = min(G, 64)
        self.W = lz.words_per_read(L)
        self.cap = pair_capacity if pair_capacity is not None else max(1 << 20, (2 * n_total) // 8)
        dev = self.dev
        self.coll = _Coll(group, dev)
        self.packed_all = torch.zeros((self.world * n_pad, self.W), dtype=torch.int64, device=dev)
        self.pool = torch.empty(self.cap, dtype=torch.int64, device=dev)
        self.pool2 = torch.empty(self.cap, dtype=torch.int64, device=dev)
        self.pool_count = torch.zeros(1, dtype=torch.int64, device=dev)
        self.counters = torch.zeros(4, dtype=torch.int64, device=dev)
        self.send = torch.empty(self.G * self.geo.send_entries, dtype=torch.int64, device=dev)
        self.send_fill = torch.empty(self.G * self.geo.fill_words, dtype=torch.int32, device=dev)
        # one rank: the exchange is the identity (no copy)
        self.recv = torch.empty_like(self.send) if self.world > 1 else self.send
        self.recv_fill = torch.empty_like(self.send_fill) if self.world > 1 else self.send_fill
        nbytes = ctypes.c_size_t(0)
        lz._check(self.Lb.lasagna_shard_part_bytes(n_total, self.world, L, l_min, self.G,
                                                   ctypes.byref(nbytes)))
        self.part = lz._workspace(nbytes.value, dev)
        self.arena = PeerArena(int(self.geo.slice), dev, group)
        ranks = (lz.GreedyRank * self.world)()
        for q in range(self.world):
            for f in ("ctr", "best", "claimed", "succ", "olen", "tail"):
                setattr(ranks[q], f, self.arena.ptr(q, f))
        ranks[self.rank].pool = self.pool.data_ptr()
        ranks[self.rank].pool2 = self.pool2.data_ptr()
        ranks[self.rank].pool_count = self.pool_count.data_ptr()
        self.ranks = ranks
        self.succ_all = torch.empty(self.world * int(self.geo.slice), dtype=torch.int32, device=dev)
        self.olen_all = torch.empty(self.world * int(self.geo.slice), dtype=torch.uint8, device=dev)

    def close(self):
        if self.arena is not None:
            self.arena.close()
            self.arena = None

    def __call__(self, ascii_local: torch.Tensor, timing: bool = False):
        """(succ int32 [2n], olen uint8 [2n], stats) of the whole read set, identical on every
        rank; ascii_local: this rank's (n_local, L) uint8 reads (device, or host: copied in)."""
        n_total, L, l_min, world, rank = self.n, self.L, self.l_min, self.world, self.rank
        geo, Lb, dev, C = self.geo, self.Lb, self.dev, self.coll
        assert ascii_local.shape[0] == self.n_local, (ascii_local.shape, self.n_local)
        s = lz._stream(dev)
        ph = _Phases(timing)
        n_pad, lo, n_local, cap = int(geo.n_pad), self.lo, self.n_local, self.cap
        # per call: fresh greedy state in the arena, zeroed counters
        self.arena.view.zero_()
        self.arena.tensor("succ", torch.int32).fill_(-1)
        self.counters.zero_()
        # 1. packed reads: local pack into my slice, all-gather -> every rank verifies any hit
        mine = self.packed_all[rank * n_pad:(rank + 1) * n_pad]
        if n_local:  # device ASCII, or page-locked host ASCII read in place by the pack kernel
            mine[:n_local] = lz.load_reads(ascii_local, device=dev)
        if world > 1:
            C.all_gather_into_tensor(self.packed_all.view(-1), mine.reshape(-1).clone())
        packed_all = self.packed_all
        packed_local = mine
        claimed_mine = self.arena.ptr(rank, "claimed")
        G = self.G
        first = True
        for l_hi in range(L - 1, l_min - 1, -G):
            l_lo = max(l_min, l_hi - G + 1)
            Gc = l_hi - l_lo + 1
            send = self.send[:Gc * geo.send_entries]
            send_fill = self.send_fill[:Gc * geo.fill_words]
            # 2. a1..a3 + level 1 of my reads, regions in shard order (pruned after group 1)
            t = ph.start("scatter")
            lz._check(Lb.lasagna_shard_scatter(
                lz._ptr(packed_local), n_local, lo, n_total, world, L, l_min, l_lo, l_hi,
                None if first else ctypes.c_void_p(claimed_mine), lz._ptr(send),
                lz._ptr(send_fill), lz._ptr(self.counters), s))
            ph.stop(t)
            ph.launches["scatter"] += 1
            first = False
            # 3. the hash-range shuffle: equal split sizes, nothing to count or synchronise
            recv = self.recv[:Gc * geo.send_entries]
            recv_fill = self.recv_fill[:Gc * geo.fill_words]
            if world > 1:
                t = ph.start("exchange")
                C.all_to_all_single(recv, send)
                C.all_to_all_single(recv_fill, send_fill)
                ph.stop(t)
            t = ph.start("refine")
            lz._check(Lb.lasagna_shard_partition(lz._ptr(recv), lz._ptr(recv_fill), n_total, world,
                                                 L, l_min, l_lo, l_hi, lz._ptr(self.part),
                                                 lz._ptr(self.counters), s))
            ph.stop(t)
            ph.launches["refine"] += int(geo.levels) - 1
            # 4. per length: join (my buckets) and the sharded greedy (everyone's pairs)
            for l in range(l_hi, l_lo - 1, -1):
                t = ph.start("join")
                lz._check(Lb.lasagna_shard_join(lz._ptr(self.part), n_total, world, L, l_min, l_lo,
                                                l_hi, l, lz._ptr(packed_all), lz._ptr(self.pool),
                                                cap, lz._ptr(self.pool_count),
                                                lz._ptr(self.counters), s))
                ph.stop(t)
                t = ph.start("greedy")
                lz._check(Lb.lasagna_greedy_shard_length(self.ranks, world, rank, int(geo.slice),
                                                         cap, l, s))
                ph.stop(t)
                ph.launches["join"] += 1
                ph.launches["greedy_lengths"] += 1
        # 5. outcome: region or pool overflow anywhere -> every rank reruns
        ctr = self.arena.tensor("ctr", torch.int64)
        flags = torch.stack([self.counters[0].clamp(max=1), ctr[5]]).to(torch.int64)
        C.all_reduce(flags, op=dist.ReduceOp.MAX)
        ovf, max_pl = (int(x) for x in flags.tolist())
        if ovf:
            raise RegionOverflow("a slack region overflowed")
        if max_pl > cap:
            raise PoolOverflow(max_pl)
        # the graph: every rank's slices of succ/olen, all-gathered
        if world > 1:
            C.all_gather_into_tensor(self.succ_all, self.arena.tensor("succ", torch.int32).clone())
            C.all_gather_into_tensor(self.olen_all, self.arena.tensor("olen", torch.uint8).clone())
        else:
            self.succ_all.copy_(self.arena.tensor("succ", torch.int32))
            self.olen_all.copy_(self.arena.tensor("olen", torch.uint8))
        tot = torch.stack([ctr[4], ctr[3], self.counters[1], self.counters[3]]).clone()
        C.all_reduce(tot)
        mx = ctr[6:7].clone()
        C.all_reduce(mx, op=dist.ReduceOp.MAX)
        n_pairs, n_greedy, pruned, false_m = (int(x) for x in tot.tolist())
        stats = {"n_pairs": n_pairs, "n_greedy": n_greedy, "pruned_entries": pruned,
                 "fp_false_matches": false_m, "rounds_max": int(mx.item()),
                 "lengths_per_pass": G, "partition_levels": int(geo.levels), "path": "fast",
                 "greedy_pair_rounds": int(ctr[7].item()), "n_local": n_local,
                 "launches": dict(ph.launches)}
        if timing:
            torch.cuda.synchronize()
            stats["ms"] = ph.totals()
        return self.succ_all[:2 * n_total], self.olen_all[:2 * n_total], stats


class PoolOverflow(RuntimeError):
    """A length produced more candidate pairs than the pool holds (rerun with a larger one)."""

    def __init__(self, need: int):
        super().__init__(f"a length produced {need} pairs")
        self.need = need


def greedy_graph_fast(ascii_local: torch.Tensor, n_total: int, L: int, l_min: int, group=None,
                      lengths_per_pass: int = 0, pair_capacity: int | None = None,
                      timing: bool = False):
    """One call of the sharded fast path (a ShardedGraph built, run and closed); a pool
    overflow reruns with a pool 1.25x the largest length.  Returns (succ, olen, stats)."""
    dev = ascii_local.device if ascii_local.is_cuda else None
    for _ in range(2):
        g = ShardedGraph(n_total, L, l_min, group, dev, lengths_per_pass, pair_capacity)
        try:
            succ, olen, st = g(ascii_local, timing)
            return succ.clone(), olen.clone(), st
        except PoolOverflow as e:
            pair_capacity = e.need * 5 // 4 + 1
        finally:
            g.close()
    raise RuntimeError("sharded fast path: pool overflow after a resize")


def lz_words(L: int) -> int:
    w = (L + 31) // 32
    return 1 if w <= 1 else 2 if w <= 2 else 4 if w <= 4 else 8


# ------------------------------------------------------------------------------ bench (N > 1)
def _fast_roofline(st: dict, n_total: int, L: int, l_min: int, world: int, peak: dict,
                   ms_step: float, steps: int) -> dict:
    """Algorithmic bytes per launch of this rank's phases over their
    CUDA-event times: scatter 8 B per key written (+ packed rows read), refine 16 B per key
    and level, join 8 B per key read + 64 B per verified candidate, greedy 64 B per pair-round.
    Exchange: the bytes this rank sends over NVLink (all-to-all of its level-1 regions)."""
    ms = {k: v / steps for k, v in st.get("ms", {}).items()}
    la = {k: v / steps for k, v in st["launches"].items()}
    n_len = L - l_min
    N_rank = 2 * n_total / world                 # keys per length per rank after the exchange
    W = lz_words(L)
    per_len_keys = 2 * st["n_local"]
    bytes_ = {
        "scatter_table_kernel": 8.0 * per_len_keys * n_len + 8.0 * W * st["n_local"],
        "refine_kernel": 16.0 * N_rank * n_len * max(1, st["partition_levels"] - 1),
        "bucket_join_kernel": 8.0 * N_rank * n_len + 64.0 * (st["n_pairs"] + st["fp_false_matches"]) / world,
        "greedy": 64.0 * st["greedy_pair_rounds"] / steps,
        "exchange": 8.0 * per_len_keys * n_len * 1.02,
    }
    keymap = {"scatter_table_kernel": "scatter", "refine_kernel": "refine",
              "bucket_join_kernel": "join", "greedy": "greedy", "exchange": "exchange"}
    phases = {}
    for k, b in bytes_.items():
        t = ms.get(keymap[k], 0.0)
        phases[k] = {"ms_per_step": t, "bytes_per_step": b,
                     "gbs": b / (t / 1e3) / 1e9 if t > 0 else None}
    hbm = {k: v for k, v in phases.items() if k not in ("exchange", "greedy")}
    name = max(hbm, key=lambda k: hbm[k]["ms_per_step"])
    ach = hbm[name]["gbs"] or 0.0
    step_bytes = sum(v["bytes_per_step"] for k, v in phases.items() if k != "exchange")
    step_gbs = step_bytes / (ms_step / 1e3) / 1e9
    return {"bound": "hbm", "kernel": name, "achieved": round(ach, 1), "peak": peak["hbm_gbs"],
            "peak_source": peak["source"], "unit": "GB/s", "frac": round(ach / peak["hbm_gbs"], 4),
            "traffic": None, "per_rank": True,
            "step": {"bytes": step_bytes, "achieved": round(step_gbs, 1),
                     "frac": round(step_gbs / peak["hbm_gbs"], 4)},
            "phases": phases}


def bench_main(args, cfg, metric, peak, ClockSampler, bus_id, cpu_baseline) -> None:
    """`bench.py` under torchrun: strong scaling at fixed n (every rank holds 1/g of the reads),
    barrier + synchronize around exactly K steps, time = max over ranks.  Default path: the
    sharded fast path (greedy_graph_fast); --dist-path exact runs the round-1 exact path."""
    import readgen
    for k, v in (("RANK", "0"), ("WORLD_SIZE", "1"), ("MASTER_ADDR", "127.0.0.1"),
                 ("MASTER_PORT", "29517")):
        os.environ.setdefault(k, v)  # --force-dist without torchrun: a one-rank group
    os.environ.setdefault("NCCL_DEBUG", "INFO")  # the communicator's rank count in the log
    os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    local = int(os.environ.get("LOCAL_RANK", "0")) % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if getattr(args, "dist_backend", "nccl") == "nccl":
        dist.init_process_group("nccl", device_id=dev)
    else:
        dist.init_process_group("gloo")
    world, rank = dist.get_world_size(), dist.get_rank()
    fast = getattr(args, "dist_path", "fast") == "fast"
    n, L, l_min = cfg.n, cfg.L, cfg.l_min
    lo, hi, _ = fast_shard_range(n, world, rank) if fast else shard_range(n, world, rank)
    host = torch.empty((hi - lo, L), dtype=torch.uint8).pin_memory()
    readgen.reads_into(host.data_ptr(), cfg.seed, cfg.G, L, cfg.p_err, lo, hi)
    dev_ascii = host.to(dev)
    be = CudaBackend(dev)
    stream = torch.cuda.current_stream(dev)

    runner = ShardedGraph(n, L, l_min, None, dev, args.lengths_per_pass) if fast else None

    h_succ = torch.empty(2 * n, dtype=torch.int32).pin_memory()
    h_olen = torch.empty(2 * n, dtype=torch.uint8).pin_memory()

    def step(src, d2h: bool, timing: bool = False):
        if fast:
            succ, olen, st = runner(src, timing=timing)
        else:
            succ, olen, st = greedy_graph(src, n, L, l_min, be,
                                          lengths_per_pass=args.lengths_per_pass)
        if d2h:
            h_succ.copy_(succ, non_blocking=True)
            h_olen.copy_(olen, non_blocking=True)
        return st

    for _ in range(args.warmup):
        st = step(dev_ascii, False)
    torch.cuda.synchronize()
    sampler = ClockSampler(bus_id(torch, local))
    sampler.start()
    dist.barrier()
    torch.cuda.synchronize()
    launches0 = lz.kernel_launches()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.steps):
        st = step(dev_ascii, False)
    e1.record(stream)
    torch.cuda.synchronize()
    dist.barrier()
    launches = lz.kernel_launches() - launches0
    clocks = sampler.stop()
    ms = torch.tensor([e0.elapsed_time(e1) / args.steps], device=dev)
    dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    # one more step with phase events (outside the timed region) for the roofline
    st_t = step(dev_ascii, False, timing=True) if fast else None
    # end to end from pinned host ASCII
    dist.barrier()
    torch.cuda.synchronize()
    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    f0.record(stream)
    for _ in range(args.steps):
        step(host, True)
    f1.record(stream)
    torch.cuda.synchronize()
    ems = torch.tensor([f0.elapsed_time(f1) / args.steps], device=dev)
    dist.all_reduce(ems, op=dist.ReduceOp.MAX)
    ms_step, e2e_ms = float(ms.item()), float(ems.item())
    if rank == 0:
        out = {
            "metric": metric, "value": n / (ms_step / 1e3), "unit": "reads/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u64",
            "data": "synthetic",
            "config": {"workload": f"{cfg.name}: {cfg.note}", "n": n, "L": L, "l_min": l_min,
                       "G": cfg.G, "p_err": cfg.p_err, "seed": cfg.seed,
                       "parallelism": f"hash-range x{world}",
                       "dist_path": "fast (scatter -> equal-split all-to-all -> refine -> join -> "
                                    "sharded greedy over peer memory)" if fast else "exact",
                       "l2": "inputs larger than L2"},
            "overlap_edges_per_s": st["n_pairs"] / (ms_step / 1e3),
            "read_end_pairs": st["n_pairs"], "greedy_pairs": st.get("n_greedy"),
            "e2e": {"value": n / (e2e_ms / 1e3), "unit": "reads/s", "ms_per_step": e2e_ms,
                    "h2d_bytes_per_step": n * L, "d2h_bytes_per_step": 2 * n * 5},
            "roofline": (_fast_roofline(st_t, n, L, l_min, world, peak, ms_step, 1)
                         if st_t else None),
            "clocks": clocks,
            "gpu_launches": launches,
        }
        if world == 1 and not getattr(args, "no_cpu_baseline", False):
            out["cpu_baseline"] = cpu_baseline(cfg, host.numpy())
        print(json.dumps(out), flush=True)
    if runner is not None:
        runner.close()
    dist.barrier()
    dist.destroy_process_group()
