"""Small invocations of every kernel family for compute-sanitizer (memcheck, racecheck,
synccheck, initcheck): cfg1-sized inputs, each result checked against the oracle so a run that
silently computes garbage under the tool is caught too.  Used by scripts/gpu_sanitize.sh."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import readgen  # noqa: E402
import paper_conf_ipps_goswamilsp18_b200 as lz  # noqa: E402


def main():
    n, L, l_min = 6000, 100, 63
    reads = readgen.reads(20181, 60_000, n, L, 0.01)
    esucc, eolen, m, acc = oracle.greedy_graph(reads, l_min)
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    quick = bool(os.environ.get("SANITIZE_QUICK"))  # racecheck: one geometry, fewer calls
    envs = ({"LASAGNA_TEST_LEVELS": "2"},) if quick else (
        {}, {"LASAGNA_TEST_LEVELS": "2"}, {"LASAGNA_TEST_LEVELS": "3", "LASAGNA_TEST_LAST_BITS": "2"},
        {"LASAGNA_PATH": "exact"})
    # bucketed one level (T = 8), forced two and three levels, the exact path
    for env in envs:
        os.environ.update(env)
        r = lz.greedy_graph(packed, n, L, l_min, lengths_per_pass=5)
        assert np.array_equal(r.succ.cpu().numpy().view(np.uint32), esucc), env
        assert np.array_equal(r.olen.cpu().numpy(), eolen), env
        for k in env:
            del os.environ[k]
    if quick:
        from tests.test_gpu_sharded import _sharded_greedy
        pl, pa, pb = lz.overlaps(packed, n, L, l_min)
        ssucc, solen, _ = _sharded_greedy(n, pl.cpu().numpy(), pa.cpu().numpy().view(np.uint32),
                                          pb.cpu().numpy().view(np.uint32), 2)
        assert np.array_equal(ssucc, esucc) and np.array_equal(solen, eolen)
        print("sanitize driver ok (quick)")
        return
    # fused a1 from device and pinned ASCII (two levels)
    os.environ["LASAGNA_TEST_LEVELS"] = "2"
    g = lz.GreedyGraph(n, L, l_min, "cuda", lengths_per_pass=7)
    for src in (torch.from_numpy(reads).cuda(), torch.from_numpy(reads).pin_memory()):
        r = g.from_ascii(src)
        assert np.array_equal(r.succ.cpu().numpy().view(np.uint32), esucc)
    del os.environ["LASAGNA_TEST_LEVELS"]
    pl, pa, pb = lz.overlaps(packed, n, L, l_min)
    assert len(pl) == m
    succ, olen, _ = lz.greedy_pairs(n, pl, pa, pb)
    assert np.array_equal(succ.cpu().numpy().view(np.uint32), esucc)
    pfx, sfx = lz.fingerprints(packed, n, L, l_min)
    c = lz.compress(packed, n, L, r.succ, r.olen)
    eb, _, _ = oracle.compress(reads, esucc, eolen)
    assert c.bases.cpu().numpy().tobytes() == eb
    # hash-range sub-passes (f4): a workspace below one whole length
    import ctypes
    ws = ctypes.c_size_t(0)
    lz.lasagna._check(lz.lib().lasagna_greedy_graph(None, n, L, l_min, 1, None, ctypes.byref(ws),
                                                    None, None, None, None))
    os.environ["LASAGNA_TEST_LEVELS"] = "2"
    _, least = lz.plan(n, L, l_min, 1)
    sub = lz.GreedyGraph(n, L, l_min, "cuda", budget_bytes=least + (int(ws.value) - least) // 4)
    r = sub(packed)
    assert r.stats["hash_subpasses"] > 1, r.stats
    assert np.array_equal(r.succ.cpu().numpy().view(np.uint32), esucc)
    del os.environ["LASAGNA_TEST_LEVELS"]
    # the sharded greedy's cross-rank protocol: three ranks in one launch
    from tests.test_gpu_sharded import _sharded_greedy
    ssucc, solen, _ = _sharded_greedy(n, pl.cpu().numpy(), pa.cpu().numpy().view(np.uint32),
                                      pb.cpu().numpy().view(np.uint32), 3)
    assert np.array_equal(ssucc, esucc) and np.array_equal(solen, eolen)
    keys = torch.randint(0, 2**62, (100_003,), dtype=torch.int64, device="cuda")
    lz.sort_u64(keys)
    torch.cuda.synchronize()
    print("sanitize driver ok")


if __name__ == "__main__":
    main()
