"""Multi-process (gloo, CPU) test of the multi-GPU driver's exchange logic: world sizes 2 and
3 over a CPU stand-in backend must give the oracle's greedy graph bit for bit."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import readgen


def _free_port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n, L, l_min, G_len, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ipps_goswamilsp18_b200 import dist as ldist
        from tests._cpu_backend import CpuBackend
        reads = readgen.reads(7, 3000, n, L, 0.01)
        be = CpuBackend(reads)
        lo, hi, _ = ldist.shard_range(n, world, rank)
        succ, olen, st = ldist.greedy_graph(torch.from_numpy(reads[lo:hi].copy()), n, L, l_min,
                                            be, lengths_per_pass=G_len)
        np.save(os.path.join(out_dir, f"succ{rank}.npy"), succ.numpy().view(np.uint32))
        np.save(os.path.join(out_dir, f"olen{rank}.npy"), olen.numpy())
        np.save(os.path.join(out_dir, f"np{rank}.npy"), np.array([st["n_pairs"]]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,G_len", [(2, 0), (3, 4), (2, 1)])
def test_dist_greedy_graph_matches_oracle(tmp_path, world, G_len):
    import oracle
    n, L, l_min = 240, 40, 24
    mp.spawn(_worker, args=(world, _free_port(), n, L, l_min, G_len, str(tmp_path)),
             nprocs=world, join=True)
    reads = readgen.reads(7, 3000, n, L, 0.01)
    esucc, eolen, m, _ = oracle.greedy_graph(reads, l_min)
    assert m > 50  # the instance has overlaps to exchange
    for r in range(world):
        assert np.array_equal(np.load(tmp_path / f"succ{r}.npy"), esucc), r
        assert np.array_equal(np.load(tmp_path / f"olen{r}.npy"), eolen), r
        assert int(np.load(tmp_path / f"np{r}.npy")[0]) == m


def test_shard_ranges_cover_reads():
    from paper_conf_ipps_goswamilsp18_b200 import dist as ldist
    for n in [0, 1, 7, 1000]:
        for g in [1, 2, 3, 8]:
            rs = [ldist.shard_range(n, g, r) for r in range(g)]
            assert rs[0][0] == 0 and rs[-1][1] == n
            assert all(rs[i][1] == rs[i + 1][0] for i in range(g - 1))
    own = ldist.owner_of_buckets(3)
    assert own[0] == 0 and own[-1] == 2 and sorted(own) == own


def _gpu_worker(rank, world, port, n, L, l_min, G_len, out_dir):
    """Ranks sharing cuda:0 over gloo: the real CUDA phase calls, host-staged collectives."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        from paper_conf_ipps_goswamilsp18_b200 import dist as ldist
        reads = readgen.config_reads("cfg1", n=n)
        lo, hi, _ = ldist.shard_range(n, world, rank)
        succ, olen, st = ldist.greedy_graph(torch.from_numpy(reads[lo:hi].copy()).cuda(), n, L,
                                            l_min, lengths_per_pass=G_len)
        np.save(os.path.join(out_dir, f"succ{rank}.npy"), succ.cpu().numpy().view(np.uint32))
        np.save(os.path.join(out_dir, f"olen{rank}.npy"), olen.cpu().numpy())
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.parametrize("world,G_len", [(2, 0), (4, 7)])
def test_dist_cuda_shards_match_oracle(tmp_path, world, G_len):
    """Hash-range sharded CUDA path (table_keys, partition sort, all-to-all, shard sort, join,
    gathered greedy) on cfg1 reads == the oracle, bit for bit."""
    import oracle
    n, L, l_min = 20_000, 100, 63
    ctx = mp.get_context("spawn")
    mp.start_processes(_gpu_worker, args=(world, _free_port(), n, L, l_min, G_len, str(tmp_path)),
                       nprocs=world, join=True, start_method="spawn")
    reads = readgen.config_reads("cfg1", n=n)
    esucc, eolen, m, _ = oracle.greedy_graph(reads, l_min)
    for r in range(world):
        assert np.array_equal(np.load(tmp_path / f"succ{r}.npy"), esucc), r
        assert np.array_equal(np.load(tmp_path / f"olen{r}.npy"), eolen), r
    del ctx
