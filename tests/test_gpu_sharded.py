"""The multi-GPU fast path on one B200.

* The sharded greedy's device protocol (greedy_rounds.cu): `world` ranks in ONE launch
  (lasagna_greedy_shard_length with rank = -1: plain device pointers stand in for the NVLink
  peer pointers, the cross-rank barriers are the same code) against the oracle's sequential
  greedy, on real overlap sets and on adversarial chains that need many rounds.
* dist.greedy_graph_fast end to end: world 1 in-process, and world 2 over gloo with both ranks
  sharing cuda:0 (CUDA IPC between the two processes, equal-split all-to-alls staged through
  the host) — against the oracle bit for bit.
"""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest

import oracle
import readgen

gpu = pytest.mark.gpu


def _free_port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _sharded_greedy(n: int, pl, pa, pb, world: int, assign_seed: int = 0):
    """Run the sharded greedy over `world` in-process ranks: every pair goes to a pseudo-random
    rank (as a hash-range join would spread them), lengths descending."""
    import torch
    from paper_conf_ipps_goswamilsp18_b200 import lasagna as lz
    L = lz.lib()
    dev = torch.device("cuda")
    V = 2 * n
    slice_ = -(-V // world)
    slice_ = (slice_ + 31) // 32 * 32
    pl = np.asarray(pl, dtype=np.int64)
    pa = np.asarray(pa, dtype=np.int64)
    pb = np.asarray(pb, dtype=np.int64)
    rng = np.random.default_rng(assign_seed)
    owner = rng.integers(0, world, size=len(pl))
    cap = max(4096, len(pl))
    bufs = []
    ranks = (lz.GreedyRank * world)()
    for q in range(world):
        b = {"pool": torch.empty(cap, dtype=torch.int64, device=dev),
             "pool2": torch.empty(cap, dtype=torch.int64, device=dev),
             "count": torch.zeros(1, dtype=torch.int64, device=dev),
             "ctr": torch.zeros(16, dtype=torch.int64, device=dev),
             "best": torch.zeros(slice_, dtype=torch.int64, device=dev),
             "claimed": torch.zeros(slice_ // 32, dtype=torch.int32, device=dev),
             "succ": torch.full((slice_,), -1, dtype=torch.int32, device=dev),
             "olen": torch.zeros(slice_, dtype=torch.uint8, device=dev),
             "tail": torch.zeros(4096, dtype=torch.int64, device=dev)}
        bufs.append(b)
        r = ranks[q]
        r.pool, r.pool2, r.pool_count = (b["pool"].data_ptr(), b["pool2"].data_ptr(),
                                         b["count"].data_ptr())
        r.ctr, r.best, r.claimed = b["ctr"].data_ptr(), b["best"].data_ptr(), b["claimed"].data_ptr()
        r.succ, r.olen, r.tail = b["succ"].data_ptr(), b["olen"].data_ptr(), b["tail"].data_ptr()
    stream = torch.cuda.current_stream().cuda_stream
    for l in sorted(set(pl.tolist()), reverse=True):
        sel = pl == l
        for q in range(world):
            m = sel & (owner == q)
            rec = (pa[m] << 32) | pb[m]
            k = len(rec)
            if k:
                bufs[q]["pool"][:k] = torch.from_numpy(rec).to(dev)
            bufs[q]["count"].fill_(k)
        lz._check(L.lasagna_greedy_shard_length(ranks, world, -1, slice_, cap, int(l), stream))
    torch.cuda.synchronize()
    succ = torch.cat([b["succ"] for b in bufs])[:V].cpu().numpy().view(np.uint32)
    olen = torch.cat([b["olen"] for b in bufs])[:V].cpu().numpy()
    acc = sum(int(b["ctr"][3].item()) for b in bufs)
    return succ, olen, acc


@gpu
@pytest.mark.parametrize("world", [1, 2, 3, 4])
def test_sharded_greedy_protocol_on_overlaps(world):
    """cfg1-shaped reads: the oracle's overlap set, split across ranks, greedy == sequential."""
    reads = readgen.reads(11, 60_000, 12_000, 100, 0.01)
    n = reads.shape[0]
    pl, pa, pb = oracle.overlaps(reads, 40)
    esucc, eolen, eacc = oracle.greedy(n, pl, pa, pb)
    succ, olen, acc = _sharded_greedy(n, pl, pa, pb, world, assign_seed=world)
    assert np.array_equal(succ, esucc) and np.array_equal(olen, eolen)
    assert acc == eacc


@gpu
@pytest.mark.parametrize("world,chain", [(1, 20_000), (2, 20_000), (4, 9000), (3, 150)])
def test_sharded_greedy_protocol_on_chains(world, chain):
    """An adversarial chain {2i, 2i+2} of one length plus a random overlay: a round accepts
    only the pairs that are minimal at both ends (about one per remaining chain segment), so
    thousands of survivors reach the tail (distributed block-local rounds, the gather, rank 0's
    rounds, the sequential scan)."""
    n = chain + 10
    rng = np.random.default_rng(5)
    d = {}
    for i in range(chain - 1):  # the chain {2i, 2i+2}: reads i and i+1 share end 2i+2
        d[(2 * i, 2 * i + 2)] = 70
    ra = rng.integers(0, 2 * n, size=3 * chain)
    rb = rng.integers(0, 2 * n, size=3 * chain)
    rl = rng.integers(63, 80, size=3 * chain)
    for x, y, l_ in zip(ra.tolist(), rb.tolist(), rl.tolist()):
        if (x >> 1) != (y >> 1):
            d.setdefault((min(x, y), max(x, y)), l_)
    items = sorted(d.items(), key=lambda kv: (-kv[1], kv[0]))  # the greedy's (l desc, a, b)
    A = np.array([k[0] for k, _ in items], dtype=np.int64)
    B = np.array([k[1] for k, _ in items], dtype=np.int64)
    Lh = np.array([v for _, v in items], dtype=np.int64)
    esucc, eolen, eacc = oracle.greedy(n, Lh.astype(np.uint8), A.astype(np.uint32), B.astype(np.uint32))
    succ, olen, acc = _sharded_greedy(n, Lh, A, B, world, assign_seed=7)
    assert np.array_equal(succ, esucc) and np.array_equal(olen, eolen)
    assert acc == eacc


def _fast_worker(rank, world, port, n, L, l_min, G_len, out_dir):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        from paper_conf_ipps_goswamilsp18_b200 import dist as ldist
        reads = readgen.config_reads("cfg1", n=n)
        lo, hi, _ = ldist.fast_shard_range(n, world, rank)
        succ, olen, st = ldist.greedy_graph_fast(torch.from_numpy(reads[lo:hi].copy()).cuda(), n, L,
                                                 l_min, lengths_per_pass=G_len)
        np.save(os.path.join(out_dir, f"succ{rank}.npy"), succ.cpu().numpy().view(np.uint32))
        np.save(os.path.join(out_dir, f"olen{rank}.npy"), olen.cpu().numpy())
        np.save(os.path.join(out_dir, f"st{rank}.npy"),
                np.array([st["n_greedy"], st["pruned_entries"], st["partition_levels"]]))
    finally:
        dist.destroy_process_group()


@gpu
@pytest.mark.parametrize("world,G_len,levels", [(1, 0, ""), (1, 5, "3"), (2, 0, ""), (2, 7, "3")])
def test_fast_dist_matches_oracle(tmp_path, monkeypatch, world, G_len, levels):
    """dist.greedy_graph_fast on cfg1 reads == the oracle's greedy graph, bit for bit (world 2:
    two processes on one GPU, peer memory through CUDA IPC); forced three-level partitions and
    several length groups (claimed-end pruning from the sharded greedy's bitmap slices)."""
    import torch.multiprocessing as mp
    if levels:
        monkeypatch.setenv("LASAGNA_TEST_LEVELS", levels)
        monkeypatch.setenv("LASAGNA_TEST_LAST_BITS", "2")
    n, L, l_min = 20_000, 100, 63
    ctx = mp.start_processes(_fast_worker, args=(world, _free_port(), n, L, l_min, G_len, str(tmp_path)),
                             nprocs=world, join=False, start_method="spawn")
    import time
    deadline = time.time() + 600
    while not ctx.join(timeout=5):
        if time.time() > deadline:  # still running: kill and fail
            for p in ctx.processes:
                if p.is_alive():
                    p.kill()
            pytest.fail("sharded fast path did not finish in 600 s")
    reads = readgen.config_reads("cfg1", n=n)
    esucc, eolen, m, acc = oracle.greedy_graph(reads, l_min)
    for r in range(world):
        assert np.array_equal(np.load(tmp_path / f"succ{r}.npy"), esucc), r
        assert np.array_equal(np.load(tmp_path / f"olen{r}.npy"), eolen), r
        st = np.load(tmp_path / f"st{r}.npy")
        assert int(st[0]) == acc
        assert int(st[2]) == (3 if levels else 2)
