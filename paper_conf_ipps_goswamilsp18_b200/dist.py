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


def lz_words(L: int) -> int:
    w = (L + 31) // 32
    return 1 if w <= 1 else 2 if w <= 2 else 4 if w <= 4 else 8


# ------------------------------------------------------------------------------ bench (N > 1)
def bench_main(args, cfg, metric, peak, ClockSampler, bus_id, cpu_baseline) -> None:
    """`bench.py` under torchrun: strong scaling at fixed n (every rank holds 1/g of the reads),
    barrier + synchronize around exactly K steps, time = max over ranks."""
    import readgen
    for k, v in (("RANK", "0"), ("WORLD_SIZE", "1"), ("MASTER_ADDR", "127.0.0.1"),
                 ("MASTER_PORT", "29517")):
        os.environ.setdefault(k, v)  # --force-dist without torchrun: a one-rank group
    local = int(os.environ.get("LOCAL_RANK", "0")) % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if getattr(args, "dist_backend", "nccl") == "nccl":
        dist.init_process_group("nccl", device_id=dev)
    else:
        dist.init_process_group("gloo")
    world, rank = dist.get_world_size(), dist.get_rank()
    n, L, l_min = cfg.n, cfg.L, cfg.l_min
    lo, hi, _ = shard_range(n, world, rank)
    host = torch.empty((hi - lo, L), dtype=torch.uint8).pin_memory()
    readgen.reads_into(host.data_ptr(), cfg.seed, cfg.G, L, cfg.p_err, lo, hi)
    dev_ascii = host.to(dev)
    be = CudaBackend(dev)
    stream = torch.cuda.current_stream(dev)

    def step(src, d2h: bool):
        succ, olen, st = greedy_graph(src, n, L, l_min, be, lengths_per_pass=args.lengths_per_pass)
        if d2h:
            succ.cpu(), olen.cpu()
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
                       "l2": "inputs larger than L2"},
            "overlap_edges_per_s": 2 * st["n_pairs"] / (ms_step / 1e3),
            "read_end_pairs": st["n_pairs"],
            "e2e": {"value": n / (e2e_ms / 1e3), "unit": "reads/s", "ms_per_step": e2e_ms,
                    "h2d_bytes_per_step": n * L, "d2h_bytes_per_step": 2 * n * 5},
            "roofline": None,
            "clocks": clocks,
            "gpu_launches": launches,
        }
        print(json.dumps(out), flush=True)
    dist.barrier()
    dist.destroy_process_group()
