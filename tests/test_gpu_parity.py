"""Parity of the CUDA path (through the C ABI) against the CPU oracle, element by element.

All integer: the bar is bit-exact.  `-m gpu` tests need a B200; the library-export test runs
anywhere.
"""
from __future__ import annotations

import ctypes
import os
import random
import re

import numpy as np
import pytest

import oracle
import readgen
from oracle import brute
from tests._util import NONE, check_graph, golden, pruning_expectations, to_array

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _header_symbols() -> list[str]:
    with open(os.path.join(ROOT, "include", "lasagna.h")) as f:
        src = f.read()
    return sorted(set(re.findall(r"\b(lasagna_[a-z0-9_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    """The C-ABI library loads and exports every function include/lasagna.h declares."""
    from paper_conf_ipps_goswamilsp18_b200 import build
    so = build.build()
    lib = ctypes.CDLL(so)
    syms = _header_symbols()
    assert len(syms) >= 9
    for s in syms:
        assert hasattr(lib, s), s


def test_library_reports_invalid_arguments_without_gpu():
    from paper_conf_ipps_goswamilsp18_b200 import lasagna as lz
    L = lz.lib()
    ws = ctypes.c_size_t(0)
    # L out of range / l_min >= L are rejected before any CUDA call
    assert L.lasagna_greedy_graph(None, 10, 300, 5, 0, None, ctypes.byref(ws), None, None, None,
                                  None) == lz.EINVAL
    assert L.lasagna_greedy_graph(None, 10, 100, 100, 0, None, ctypes.byref(ws), None, None, None,
                                  None) == lz.EINVAL
    assert L.lasagna_greedy_graph(None, 1 << 31, 100, 63, 0, None, ctypes.byref(ws), None, None,
                                  None, None) == lz.ERANGE
    assert b"l_min" in L.lasagna_last_error() or True
    assert L.lasagna_words_per_read(100) == 4 and L.lasagna_words_per_read(150) == 8
    assert L.lasagna_words_per_read(32) == 1 and L.lasagna_words_per_read(33) == 2


# ============================================================================ GPU parity
gpu = pytest.mark.gpu


@pytest.fixture(scope="module")
def lz():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    import paper_conf_ipps_goswamilsp18_b200 as m
    m.lib()
    return m


def _np(t, dtype):
    return t.cpu().numpy().view(dtype)


@gpu
@pytest.mark.parametrize("L", [8, 32, 33, 100, 101, 150, 256])
def test_pack_parity(lz, L):
    import torch
    reads = readgen.reads(5, 50_000, 777, L, 0.02)
    stride = lz.words_per_read(L)
    exp = oracle.pack(reads, stride)
    # device input
    got = lz.load_reads(torch.from_numpy(reads).cuda())
    assert np.array_equal(_np(got, np.uint64), exp)
    # page-locked host input, read in place by the kernel (zero-copy staging)
    got2 = lz.load_reads(torch.from_numpy(reads).pin_memory())
    assert np.array_equal(_np(got2, np.uint64), exp)
    # lowercase maps the same way (R13)
    low = np.char.lower(reads.view(f"S{L}")).view(np.uint8).reshape(reads.shape)
    assert np.array_equal(_np(lz.load_reads(torch.from_numpy(low).cuda()), np.uint64), exp)


@gpu
def test_pack_ragged_offsets(lz):
    """Sub-views starting at odd byte offsets (unaligned staging spans)."""
    import torch
    reads = readgen.reads(6, 50_000, 1000, 101, 0.0)
    flat = torch.from_numpy(reads.reshape(-1).copy()).cuda()
    for skip in [1, 3, 17]:
        sub = flat[skip * 101:].view(-1, 101)
        got = lz.load_reads(sub)
        assert np.array_equal(_np(got, np.uint64), oracle.pack(reads[skip:], 4))


@gpu
def test_pack_rejects_non_acgt(lz):
    import torch
    reads = readgen.reads(1, 10_000, 500, 100, 0.0)
    bad = reads.copy()
    bad[321, 50] = ord("N")
    bad[400, 0] = ord("-")
    with pytest.raises(lz.LasagnaError, match="read 321"):
        lz.load_reads(torch.from_numpy(bad).cuda())
    assert oracle.first_bad(bad) == 321


@gpu
@pytest.mark.parametrize("n,L,l_min", [(3000, 100, 63), (2000, 40, 20), (1500, 150, 111),
                                       (700, 256, 200), (513, 33, 1)])
def test_fingerprints_parity(lz, n, L, l_min):
    import torch
    reads = readgen.reads(9, 300_000, n, L, 0.01)
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    pfx, sfx = lz.fingerprints(packed, n, L, l_min)
    epfx, esfx = oracle.fingerprints(reads, l_min)
    assert np.array_equal(_np(pfx, np.uint64), epfx)
    assert np.array_equal(_np(sfx, np.uint64), esfx)


@gpu
def test_fingerprints_fig_example_production(lz):
    """GATACCAGTA at sigma=5, q=2^61-1: prefixes 3, 15, 77, ... (base-5 numerals)."""
    import torch
    reads = to_array(["GATACCAGTA"])
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    pfx, sfx = lz.fingerprints(packed, 1, 10, 1)
    assert _np(pfx, np.uint64)[:, 0].tolist() == [3, 15, 77, 385, 1926, 9631, 48155, 240778,
                                                  1203892, 6019460]
    assert _np(sfx, np.uint64)[:, 0].tolist() == [0, 10, 85, 85, 710, 3835, 3835, 160085, 160085,
                                                  6019460]
    assert int(_np(pfx, np.uint64)[9, 1]) == oracle.F("TACTGGTATC") == 4027136


@gpu
@pytest.mark.parametrize("count", [0, 1, 2, 8191, 8192, 8193, 100_003, (1 << 20) + 7])
@pytest.mark.parametrize("bits", [(0, 64), (40, 64), (3, 17), (56, 64)])
def test_sort_u64_matches_numpy_stable(lz, count, bits):
    import torch
    rng = np.random.default_rng(count * 7 + bits[0])
    keys = rng.integers(0, 2**63, size=count, dtype=np.int64).view(np.uint64)
    keys ^= rng.integers(0, 2, size=count, dtype=np.uint64) << np.uint64(63)
    lo, hi = bits
    t = torch.from_numpy(keys.view(np.int64).copy()).cuda()
    lz.sort_u64(t, lo, hi)
    dig = (keys >> np.uint64(lo)) & np.uint64((1 << (hi - lo)) - 1 if hi - lo < 64 else 2**64 - 1)
    exp = keys[np.argsort(dig, kind="stable")]
    assert np.array_equal(_np(t, np.uint64), exp)


@gpu
def test_sort_u64_degenerate_inputs(lz):
    import torch
    n = 50_000
    for keys in [np.full(n, 0xDEADBEEF12345678, dtype=np.uint64),
                 np.arange(n, dtype=np.uint64) << np.uint64(20),
                 (np.arange(n, dtype=np.uint64)[::-1] << np.uint64(20)).copy(),
                 np.arange(n, dtype=np.uint64) % np.uint64(3)]:
        t = torch.from_numpy(keys.view(np.int64).copy()).cuda()
        lz.sort_u64(t, 0, 64)
        assert np.array_equal(_np(t, np.uint64), np.sort(keys, kind="stable"))


def _tiny_cases():
    out = []
    for seed in range(8):
        rng = random.Random(100 + seed)
        L = rng.choice([8, 12, 16, 20, 40])
        G = rng.choice([30, 60, 200, 2000])
        n = rng.choice([10, 40, 120])
        p = rng.choice([0.0, 0.0, 0.02])
        reads = readgen.reads(seed, G, n, L, p)
        out.append((reads, rng.randint(2, L - 2)))
    out.append((to_array(["ACGTTA" * 2, "CGTTAACGTTAA", "GTTAACGTTAAC", "AAGCTTAAGCTT",
                          "ACACACACACAC", "GTGTGTGTGTGT", "GAATTCGAATTC", "TTCGAATTCGAA",
                          "ACGTACGTACGT", "CGTACGTACGTA"]), 3))
    # all-identical reads: every pair ties at every length
    out.append((to_array(["ACGATCGATTGC"] * 30), 4))
    return out


@gpu
@pytest.mark.parametrize("case", range(10))
def test_overlaps_parity_tiny(lz, case):
    import torch
    reads, l_min = _tiny_cases()[case]
    n, L = reads.shape
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    pl, pa, pb = lz.overlaps(packed, n, L, l_min)
    epl, epa, epb = oracle.overlaps(reads, l_min)
    assert np.array_equal(_np(pl, np.uint8), epl)
    assert np.array_equal(_np(pa, np.uint32), epa)
    assert np.array_equal(_np(pb, np.uint32), epb)


@gpu
@pytest.mark.parametrize("case", range(10))
def test_greedy_graph_parity_tiny(lz, case):
    import torch
    reads, l_min = _tiny_cases()[case]
    n, L = reads.shape
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    r = lz.greedy_graph(packed, n, L, l_min)
    esucc, eolen, m, acc = oracle.greedy_graph(reads, l_min)
    assert np.array_equal(_np(r.succ, np.uint32), esucc)
    assert np.array_equal(_np(r.olen, np.uint8), eolen)
    assert r.stats["n_pairs"] == m and r.stats["n_greedy"] == acc


@gpu
def test_micro_example_gpu(lz):
    import torch
    g = golden("micro_example.txt")
    reads = to_array(g["reads"])
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    r = lz.greedy_graph(packed, 6, 8, 4)
    assert _np(r.succ, np.uint32).tolist() == [NONE if x == "N" else int(x) for x in g["succ"]]
    assert _np(r.olen, np.uint8).tolist() == [int(x) for x in g["olen"]]
    pl, pa, pb = lz.overlaps(packed, 6, 8, 4)
    got = list(zip(_np(pl, np.uint8).tolist(), _np(pa, np.uint32).tolist(),
                   _np(pb, np.uint32).tolist()))
    assert got == [tuple(int(x) for x in p.split(",")) for p in g["pairs"]]


@gpu
def test_cfg1_parity(lz):
    """cfg1 (BASELINE configs[0]): overlaps and greedy graph bit-exact vs the oracle."""
    import torch
    cfg = readgen.CONFIGS["cfg1"]
    reads = readgen.config_reads(cfg)
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    pl, pa, pb = lz.overlaps(packed, cfg.n, cfg.L, cfg.l_min)
    epl, epa, epb = oracle.overlaps(reads, cfg.l_min)
    assert np.array_equal(_np(pa, np.uint32), epa) and np.array_equal(_np(pb, np.uint32), epb)
    assert np.array_equal(_np(pl, np.uint8), epl)
    esucc, eolen, _ = oracle.greedy(cfg.n, epl, epa, epb)
    for lpp in [0, 1, 5]:  # semi-streaming: one length per pass, groups of 5, all at once
        r = lz.greedy_graph(packed, cfg.n, cfg.L, cfg.l_min, lengths_per_pass=lpp)
        assert np.array_equal(_np(r.succ, np.uint32), esucc), lpp
        assert np.array_equal(_np(r.olen, np.uint8), eolen), lpp
        # later groups drop the entries of claimed read ends (claimed-end pruning)
        G = r.stats["lengths_per_pass"]
        assert (r.stats["n_pairs"], r.stats["pruned_entries"]) == pruning_expectations(
            cfg.L, cfg.l_min, G, (epl, epa, epb), eolen), lpp
    check_graph(reads, cfg.l_min, esucc, eolen, (epl, epa, epb))


@gpu
@pytest.mark.parametrize("seed", [20181, 20182])
def test_cfg2_parity(lz, seed):
    """cfg2 (BASELINE configs[1]: 2.3M reads, 1% errors): bit-exact greedy graph."""
    import torch
    cfg = readgen.CONFIGS["cfg2"]
    reads = readgen.config_reads(cfg, seed=seed)
    packed = lz.load_reads(torch.from_numpy(reads).pin_memory())
    r = lz.greedy_graph(packed, cfg.n, cfg.L, cfg.l_min)
    esucc, eolen, m, acc = oracle.greedy_graph(reads, cfg.l_min)
    assert r.stats["n_pairs"] == m
    assert r.stats["n_greedy"] == acc
    assert np.array_equal(_np(r.succ, np.uint32), esucc)
    assert np.array_equal(_np(r.olen, np.uint8), eolen)


def _expected_false_matches(n: int, L: int, l_min: int, vbits: int) -> float:
    """R12 closed form for the fingerprint hits the bases reject: per length, V/2 probe-side
    and V/2 build-side canonical entries (V = 2n); a bucketed key stores the 62 - vbits bits of
    mix(min(H, Hr)) below the 8 its level-1 region implies, so two unrelated entries agree on
    all 70 - vbits compared bits with probability 2^-(70 - vbits):
    E[false] = (L - l_min) (V/2)^2 / 2^(70 - vbits).  (Chosen key widths: test_gpu_geometry.)"""
    V = 2 * n
    return (L - l_min) * (V / 2) ** 2 / 2.0 ** (70 - vbits)


def _assert_poisson(observed: int, expected: float):
    assert abs(observed - expected) <= 5 * expected ** 0.5 + 0.02 * expected, (observed, expected)


def _palindrome_rich_reads(seed: int, G: int, n: int, L: int, every: int, plen: int) -> np.ndarray:
    """Error-free reads (half reverse-complemented) of a random genome in which a reverse-
    complement palindrome of length plen starts every `every` bases: reads starting at one
    have palindromic prefixes (H == Hr, flag 2 in the canonical table), so build/probe
    assignments of flag-2 entries, their double discovery and same-read palindromes are all
    exercised at a size that runs the two-level (T = 16) bucketed path."""
    rng = np.random.default_rng(seed)
    comp = np.zeros(256, dtype=np.uint8)
    for a, b in zip(b"ACGT", b"TGCA"):
        comp[a] = b
    alpha = np.frombuffer(b"ACGT", dtype=np.uint8)
    g = alpha[rng.integers(0, 4, G)]
    for s0 in range(0, G - plen, every):
        half = g[s0:s0 + plen // 2].copy()
        g[s0 + plen // 2:s0 + plen] = comp[half[::-1]]
    starts = rng.integers(0, G - L + 1, n)
    # a third of the reads start exactly on a palindrome
    k = n // 3
    starts[:k] = (rng.integers(0, (G - L) // every, k) * every)
    reads = g[starts[:, None] + np.arange(L)[None, :]]
    flip = rng.random(n) < 0.5
    reads[flip] = comp[reads[flip][:, ::-1]]
    return np.ascontiguousarray(reads)


@gpu
def test_palindrome_rich_parity_two_level(lz):
    """~1.7 M table entries per length (T = 16: level-1 + level-2 partition, split buckets):
    overlaps and greedy graph bit-exact vs the oracle on palindrome-rich reads."""
    import torch
    reads = _palindrome_rich_reads(7, 4_000_000, 420_000, 40, 37, 20)
    n, L = reads.shape
    l_min = 16
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    r = lz.greedy_graph(packed, n, L, l_min)
    assert r.stats["key_sort_bits"] == 16 and r.stats["bucketed"] == 1
    esucc, eolen, m, acc = oracle.greedy_graph(reads, l_min)
    assert r.stats["n_pairs"] == m and r.stats["n_greedy"] == acc
    assert np.array_equal(_np(r.succ, np.uint32), esucc)
    assert np.array_equal(_np(r.olen, np.uint8), eolen)


@gpu
def test_oversized_fingerprint_class(lz):
    """A fingerprint class far larger than a bucket's slack: 4200 copies of one read X plus a
    read Y whose 80-base prefix is X's 80-base suffix, among 400 K genome reads (T = 16).  X's
    entries of every length overflow their level-2 bucket (capacity ~750), the overflow is
    detected and the call is redone on the exact LSD path (stats.bucketed = 0); the 4200
    (X, Y) pairs at l = 80 and the greedy result match the oracle bit for bit."""
    import torch
    L, l_min = 101, 63
    reads = readgen.reads(11, 4_000_000, 400_000, L, 0.01)
    rng = np.random.default_rng(5)
    acgt = np.frombuffer(b"ACGT", dtype=np.uint8)
    x = acgt[rng.integers(0, 4, L)]
    y = np.concatenate([x[L - 80:], acgt[rng.integers(0, 4, L - 80)]])
    reads[1000:5200] = x
    reads[7] = y
    n = reads.shape[0]
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    r = lz.greedy_graph(packed, n, L, l_min)
    assert r.stats["key_sort_bits"] == 16 and r.stats["bucketed"] == 0
    esucc, eolen, m, acc = oracle.greedy_graph(reads, l_min)
    assert r.stats["n_pairs"] == m and r.stats["n_greedy"] == acc
    assert np.array_equal(_np(r.succ, np.uint32), esucc)
    assert np.array_equal(_np(r.olen, np.uint8), eolen)
    pl, pa, pb = lz.overlaps(packed, n, L, l_min)
    epl, epa, epb = oracle.overlaps(reads, l_min)
    assert np.array_equal(_np(pl, np.uint8), epl) and int((epl == 80).sum()) >= 4200
    assert np.array_equal(_np(pa, np.uint32), epa)
    assert np.array_equal(_np(pb, np.uint32), epb)


def _random_candidates(n, k, rng, lens):
    V = 2 * n
    k = min(k, len(lens) * V * (V - 1) // 4)  # at most half of all distinct (l, a, b)
    seen = set()
    out = []
    while len(out) < k:
        a, b = sorted(rng.sample(range(V), 2))
        l = rng.choice(lens)
        if (l, a, b) in seen:
            continue
        seen.add((l, a, b))
        out.append((l, a, b))
    return out


@gpu
@pytest.mark.parametrize("seed", range(6))
def test_greedy_pairs_matches_sequential(lz, seed):
    import torch
    rng = random.Random(seed)
    n = rng.choice([50, 500, 20_000])
    k = rng.choice([100, 5000, 60_000])
    cand = _random_candidates(n, k, rng, [63, 64, 70, 99] if seed % 2 else [80])
    P = sorted(cand, key=lambda t: (-t[0], t[1], t[2]))
    esucc, eolen = brute.greedy(n, P)
    rng.shuffle(cand)
    pl = torch.tensor([c[0] for c in cand], dtype=torch.uint8).cuda()
    pa = torch.tensor([c[1] for c in cand], dtype=torch.int64).to(torch.int32).cuda()
    pb = torch.tensor([c[2] for c in cand], dtype=torch.int64).to(torch.int32).cuda()
    succ, olen, rounds = lz.greedy_pairs(n, pl, pa, pb)
    assert _np(succ, np.uint32).tolist() == esucc
    assert _np(olen, np.uint8).tolist() == eolen


@gpu
@pytest.mark.parametrize("k", [2, 17, 1000, 10_001])
def test_greedy_pairs_adversarial_chain(lz, k):
    """Path a0-a1-...-ak at one length, priorities increasing along the path: k/2 rounds of
    locally-dominant matching (then the sequential tail)."""
    import torch
    n = k + 2
    cand = [(70, i, i + 1) for i in range(k)]
    esucc, eolen = brute.greedy(n, sorted(cand, key=lambda t: (-t[0], t[1], t[2])))
    pl = torch.full((k,), 70, dtype=torch.uint8).cuda()
    pa = torch.arange(k, dtype=torch.int32).cuda()
    pb = torch.arange(1, k + 1, dtype=torch.int32).cuda()
    succ, olen, rounds = lz.greedy_pairs(n, pl, pa, pb)
    assert _np(succ, np.uint32).tolist() == esucc
    assert _np(olen, np.uint8).tolist() == eolen


@gpu
@pytest.mark.parametrize("reads,l_min", [(["AC"], 1), (["ACGTAC", "GTACGT"], 1), (["AAAA", "AAAA", "TTTT"], 1),
                                         (["ACGT" * 8 + "A"], 16)])
def test_degenerate_shapes(lz, reads, l_min):
    import torch
    arr = to_array(reads)
    n, L = arr.shape
    packed = lz.load_reads(torch.from_numpy(arr).cuda())
    r = lz.greedy_graph(packed, n, L, l_min)
    esucc, eolen, m, _ = oracle.greedy_graph(arr, l_min)
    assert np.array_equal(_np(r.succ, np.uint32), esucc)
    assert np.array_equal(_np(r.olen, np.uint8), eolen)
    pl, pa, pb = lz.overlaps(packed, n, L, l_min)
    epl, epa, epb = oracle.overlaps(arr, l_min)
    assert np.array_equal(_np(pa, np.uint32), epa) and np.array_equal(_np(pb, np.uint32), epb)


@gpu
def test_empty_read_set(lz):
    import torch
    packed = torch.empty((0, 4), dtype=torch.int64, device="cuda")
    r = lz.greedy_graph(packed, 0, 100, 63)
    assert r.succ.numel() == 0 and r.stats["n_pairs"] == 0
    pl, pa, pb = lz.overlaps(packed, 0, 100, 63)
    assert pl.numel() == 0


@gpu
def test_planner_and_small_workspace(lz):
    """a8: the planner shrinks the length group to the budget; a workspace below one length
    is ENOSPC with the needed size reported."""
    n, L, l_min = 20_000, 100, 63
    lp_all, ws_all = lz.plan(n, L, l_min, 1 << 40)
    assert lp_all == L - l_min
    lp0, need = lz.plan(n, L, l_min, 1 << 10)
    assert lp0 == 0 and need > (1 << 10)
    budget = (need + ws_all) // 2
    lp_small, ws_small = lz.plan(n, L, l_min, budget)
    assert 1 <= lp_small < lp_all and ws_small <= budget


@gpu
def test_region_overflow_falls_back_to_exact_path(tmp_path):
    """Slack regions that overflow (forced here) are detected and the call redoes the work on
    the exact LSD path: the result is still bit-exact."""
    import subprocess
    import sys
    code = (
        "import numpy as np, torch, readgen, oracle\n"
        "import paper_conf_ipps_goswamilsp18_b200 as lz\n"
        "reads = readgen.config_reads('cfg1', n=8000)\n"
        "packed = lz.load_reads(torch.from_numpy(reads).cuda())\n"
        "r = lz.greedy_graph(packed, 8000, 100, 63)\n"
        "es, eo, m, _ = oracle.greedy_graph(reads, 63)\n"
        "assert np.array_equal(r.succ.cpu().numpy().view(np.uint32), es)\n"
        "assert np.array_equal(r.olen.cpu().numpy(), eo)\n"
        "pl, pa, pb = lz.overlaps(packed, 8000, 100, 63)\n"
        "assert pl.numel() == m\n"
        "print('ok')\n")
    env = dict(os.environ, LASAGNA_TEST_TIGHT_REGIONS="1", PYTHONPATH=ROOT)
    out = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True,
                         cwd=ROOT, timeout=600)
    assert out.returncode == 0 and "ok" in out.stdout, out.stderr[-2000:]


@gpu
@pytest.mark.parametrize("n,stream_input", [(60_000, False), (60_000, True), (400_000, True)])
def test_graph_pipeline_batches(n, stream_input):
    """GraphPipeline (two batches in flight; batch k+1's host -> device copy overlapping batch
    k, either whole into a device buffer or streamed in chunks inside the call): five different
    read batches, each result equal to the oracle's for that batch (400 K reads: the two-level
    path, whose scatter consumes the DMA chunks as they land)."""
    import torch
    import paper_conf_ipps_goswamilsp18_b200 as lz
    L, l_min = 100, 63
    batches = [readgen.reads(100 + k, 5 * n, n, L, 0.01) for k in range(5)]
    pipe = lz.GraphPipeline(n, L, l_min, "cuda", stream_input=stream_input)
    hb = [torch.from_numpy(b).pin_memory() for b in batches]
    outs = [(torch.empty(2 * n, dtype=torch.int32).pin_memory(),
             torch.empty(2 * n, dtype=torch.uint8).pin_memory()) for _ in batches]
    pipe.run(hb, outs)
    for b, (succ, olen) in zip(batches, outs):
        esucc, eolen, m, acc = oracle.greedy_graph(b, l_min)
        assert np.array_equal(succ.numpy().view(np.uint32), esucc)
        assert np.array_equal(olen.numpy(), eolen)


@gpu
@pytest.mark.parametrize("slots", ["64", "3"])
def test_host_ascii_streamed_in_chunks(slots):
    """Page-locked host ASCII streamed by DMA in many chunks (LASAGNA_TEST_A1_CHUNK = 37 x 512
    reads, a ragged last chunk), one ring slot per chunk or three reused slots: greedy graph
    and packed rows equal the oracle; a bad byte in a late chunk is reported with its global
    read index."""
    import subprocess
    import sys
    code = (
        "import numpy as np, torch, readgen, oracle\n"
        "import paper_conf_ipps_goswamilsp18_b200 as lz\n"
        "reads = readgen.config_reads('cfg2', n=400_001)\n"
        "n, L = reads.shape\n"
        "g = lz.GreedyGraph(n, L, 63, 'cuda')\n"
        "r = g.from_ascii(torch.from_numpy(reads).pin_memory())\n"
        "es, eo, m, acc = oracle.greedy_graph(reads, 63)\n"
        "assert r.stats['bucketed'] == 1 and r.stats['key_sort_bits'] == 16\n"
        "assert np.array_equal(r.succ.cpu().numpy().view(np.uint32), es)\n"
        "assert np.array_equal(r.olen.cpu().numpy(), eo)\n"
        "assert np.array_equal(g.packed.cpu().numpy().view(np.uint64), oracle.pack(reads, lz.words_per_read(L)))\n"
        "bad = reads.copy(); bad[399_990, 5] = ord('N'); bad[399_999, 0] = ord('-')\n"
        "try:\n"
        "    g.from_ascii(torch.from_numpy(bad).pin_memory())\n"
        "    raise SystemExit('bad read not reported')\n"
        "except lz.LasagnaError as e:\n"
        "    assert 'read 399990' in str(e), str(e)\n"
        "print('ok')\n")
    env = dict(os.environ, LASAGNA_TEST_A1_CHUNK=str(37 * 512), LASAGNA_TEST_A1_SLOTS=slots,
               PYTHONPATH=ROOT)
    out = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True,
                         cwd=ROOT, timeout=900)
    assert out.returncode == 0 and "ok" in out.stdout, out.stderr[-2000:]


@gpu
def test_join_side_dead_pair_filter_option():
    """LASAGNA_JOIN_FILTER=1 (the join drops pairs with an already claimed end, counting them):
    same graph and the same |P| as the default path."""
    import subprocess
    import sys
    code = (
        "import numpy as np, torch, readgen, oracle\n"
        "import paper_conf_ipps_goswamilsp18_b200 as lz\n"
        "reads = readgen.config_reads('cfg2', n=300000)\n"
        "packed = lz.load_reads(torch.from_numpy(reads).cuda())\n"
        "r = lz.greedy_graph(packed, 300000, 100, 63)\n"
        "es, eo, m, acc = oracle.greedy_graph(reads, 63)\n"
        "assert np.array_equal(r.succ.cpu().numpy().view(np.uint32), es)\n"
        "assert np.array_equal(r.olen.cpu().numpy(), eo)\n"
        "assert r.stats['n_pairs'] == m and r.stats['n_greedy'] == acc\n"
        "print('ok')\n")
    env = dict(os.environ, LASAGNA_JOIN_FILTER="1", PYTHONPATH=ROOT)
    out = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True,
                         cwd=ROOT, timeout=600)
    assert out.returncode == 0 and "ok" in out.stdout, out.stderr[-2000:]


@gpu
@pytest.mark.parametrize("path", ["exact"])
def test_exact_path_cfg1(path):
    """The exact LSD-sort path (LASAGNA_PATH=exact) stays bit-exact too."""
    import subprocess
    import sys
    code = (
        "import numpy as np, torch, readgen, oracle\n"
        "import paper_conf_ipps_goswamilsp18_b200 as lz\n"
        "reads = readgen.config_reads('cfg1')\n"
        "packed = lz.load_reads(torch.from_numpy(reads).cuda())\n"
        "r = lz.greedy_graph(packed, 20000, 100, 63)\n"
        "es, eo, m, _ = oracle.greedy_graph(reads, 63)\n"
        "assert np.array_equal(r.succ.cpu().numpy().view(np.uint32), es)\n"
        "assert np.array_equal(r.olen.cpu().numpy(), eo)\n"
        "print('ok')\n")
    env = dict(os.environ, LASAGNA_PATH=path, PYTHONPATH=ROOT)
    out = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True,
                         cwd=ROOT, timeout=600)
    assert out.returncode == 0 and "ok" in out.stdout, out.stderr[-2000:]


@gpu
@pytest.mark.parametrize("where", ["device", "pinned"])
def test_greedy_graph_from_ascii(lz, where):
    """lasagna_greedy_graph_ascii (a1 fused into the first table pass) == the oracle, from
    device memory and from page-locked host memory; bad reads are reported."""
    import torch
    cfg = readgen.CONFIGS["cfg2"]
    reads = readgen.config_reads(cfg, n=400_000)
    n, L = reads.shape
    t = torch.from_numpy(reads)
    t = t.cuda() if where == "device" else t.pin_memory()
    g = lz.GreedyGraph(n, L, cfg.l_min, "cuda")
    r = g.from_ascii(t)
    esucc, eolen, m, acc = oracle.greedy_graph(reads, cfg.l_min)
    assert np.array_equal(_np(r.succ, np.uint32), esucc)
    assert np.array_equal(_np(r.olen, np.uint8), eolen)
    assert np.array_equal(_np(g.packed, np.uint64), oracle.pack(reads, lz.words_per_read(L)))
    bad = reads.copy()
    bad[12345, 7] = ord("N")
    tb = torch.from_numpy(bad)
    tb = tb.cuda() if where == "device" else tb.pin_memory()
    with pytest.raises(lz.LasagnaError, match="read 12345"):
        g.from_ascii(tb)


@gpu
@pytest.mark.parametrize("L", [101, 127])
def test_greedy_graph_from_ascii_unaligned_rows(lz, L):
    """The fused a1 packs four bases per step from rows that start at any byte offset (L not
    a multiple of 4): parity with the oracle on mixed-case input, and a bad byte in the last
    base of a row (the partial final step) or in its first base is reported (R13)."""
    import torch
    n, l_min = 400_000, L - 38
    reads = readgen.reads(7, 2_000_000, n, L, 0.01)
    mixed = reads.copy()
    mixed[::3] = np.char.lower(mixed[::3].view(f"S{L}")).view(np.uint8).reshape(-1, L)
    g = lz.GreedyGraph(n, L, l_min, "cuda")
    r = g.from_ascii(torch.from_numpy(mixed).pin_memory())
    esucc, eolen, m, acc = oracle.greedy_graph(reads, l_min)
    assert np.array_equal(_np(r.succ, np.uint32), esucc)
    assert np.array_equal(_np(r.olen, np.uint8), eolen)
    assert np.array_equal(_np(g.packed, np.uint64), oracle.pack(reads, lz.words_per_read(L)))
    for row, col, ch in [(2**17 + 3, L - 1, "N"), (54_321, 0, "x"), (n - 1, L - 1, "@")]:
        bad = reads.copy()
        bad[row, col] = ord(ch)
        with pytest.raises(lz.LasagnaError, match=f"read {row}"):
            g.from_ascii(torch.from_numpy(bad).cuda())


@gpu
@pytest.mark.slow
def test_cfg3_full_size_parity_and_invariants(lz):
    """cfg3 (BASELINE configs[2], 34.85 M reads) in the launch configuration bench.py times
    (a1-a7 from ASCII, all 38 lengths in one pass): bit-exact against the oracle run on the
    box's host cores (a few minutes), plus the graph invariants vectorised over all edges."""
    import torch
    cfg = readgen.CONFIGS["cfg3"]
    host = torch.empty((cfg.n, cfg.L), dtype=torch.uint8).pin_memory()
    readgen.reads_into(host.data_ptr(), cfg.seed, cfg.G, cfg.L, cfg.p_err, 0, cfg.n)
    g = lz.GreedyGraph(cfg.n, cfg.L, cfg.l_min, "cuda")
    r = g.from_ascii(host)  # the e2e form: DMA-streamed chunks, one fused scatter each
    succ = _np(r.succ, np.uint32).copy()
    olen = _np(r.olen, np.uint8).copy()
    st = r.stats
    # the form bench.py's `value` times: device-resident ASCII, ONE fused scatter launch
    dev_ascii = host.cuda()
    r = g.from_ascii(dev_ascii)
    assert r.stats["passes"] == 1 and r.stats["lengths_per_pass"] == cfg.L - cfg.l_min
    dsucc = _np(r.succ, np.uint32).copy()
    dolen = _np(r.olen, np.uint8).copy()
    del g, r, dev_ascii
    torch.cuda.empty_cache()
    assert np.array_equal(dsucc, succ) and np.array_equal(dolen, olen)
    # R12 collision rate at full size (~1.34 M rejected hits expected)
    vbits = max(1, (2 * cfg.n - 1).bit_length())  # ceil(log2 V), lasagna.h key layout
    _assert_poisson(st["fp_false_matches"], _expected_false_matches(cfg.n, cfg.L, cfg.l_min, vbits))
    esucc, eolen, m, acc = oracle.greedy_graph(host.numpy(), cfg.l_min)
    assert st["n_pairs"] == m and st["n_greedy"] == acc
    assert np.array_equal(succ, esucc)
    assert np.array_equal(olen, eolen)
    # invariants on every edge: complement edge present, in-degree <= 1
    has = succ != NONE
    us = np.nonzero(has)[0]
    vs = succ[us].astype(np.int64)
    assert len(np.unique(vs)) == len(vs)
    assert np.array_equal(succ[vs ^ 1].astype(np.int64), us ^ 1)
    assert np.all((olen[us] >= cfg.l_min) & (olen[us] <= cfg.L - 1))
    assert np.all((us >> 1) != (vs >> 1))


def test_product_path_fails_loudly_without_the_library(monkeypatch, tmp_path):
    """No CPU fallback: with liblasagna.so absent (and no nvcc to rebuild it) the binding
    raises instead of computing anything; the package never imports the oracle."""
    from paper_conf_ipps_goswamilsp18_b200 import lasagna as lz

    def no_nvcc(*_a, **_k):
        raise RuntimeError("nvcc not found")

    monkeypatch.setattr(lz, "_lib", None)
    monkeypatch.setattr(lz._build, "SO", str(tmp_path / "liblasagna.so"))
    monkeypatch.setattr(lz._build, "SO_CHECKED", str(tmp_path / "liblasagna_checked.so"))
    monkeypatch.setattr(lz._build, "stale", no_nvcc)
    with pytest.raises((lz.LasagnaError, RuntimeError)):
        lz.lib()
    pkg = os.path.join(ROOT, "paper_conf_ipps_goswamilsp18_b200")
    for name in os.listdir(pkg):
        if name.endswith(".py"):
            with open(os.path.join(pkg, name)) as f:
                src = f.read()
            assert not re.search(r"^\s*(import|from)\s+oracle\b", src, re.M), name


@gpu
@pytest.mark.parametrize("L,l_min,n,G,p_err", [(256, 200, 4000, 40_000, 0.0), (256, 255, 4000, 40_000, 0.0),
                                             (64, 1, 3000, 20_000, 0.01), (255, 128, 3000, 30_000, 0.002)])
def test_greedy_graph_extreme_lengths(lz, L, l_min, n, G, p_err):
    """Edge shapes: the maximum read length (L = 256, four packed words), a single matched
    length (l_min = L - 1), every length from 1 (millions of pairs: one length overflows the
    default pair pool, so the call returns ENOSPC with a larger workspace and is retried), an
    odd L near the maximum."""
    import torch
    reads = readgen.reads(7, G, n, L, p_err)
    esucc, eolen, m, acc = oracle.greedy_graph(reads, l_min)
    P = oracle.overlaps(reads, l_min)
    for src in (torch.from_numpy(reads).cuda(), torch.from_numpy(reads).pin_memory()):
        r = lz.greedy_graph(lz.load_reads(src), n, L, l_min)
        # more than 64 lengths run in several groups: later groups are pruned (f1), so the
        # pairs found are the live ones (tests/_util.py pruning_expectations)
        G = r.stats["lengths_per_pass"]
        found = pruning_expectations(L, l_min, G, P, eolen)[0] if r.stats["bucketed"] else m
        assert r.stats["n_pairs"] == found and r.stats["n_greedy"] == acc, (r.stats, found, acc)
        assert np.array_equal(_np(r.succ, np.uint32), esucc)
        assert np.array_equal(_np(r.olen, np.uint8), eolen)
    pl, pa, pb = lz.overlaps(lz.load_reads(torch.from_numpy(reads).cuda()), n, L, l_min)
    epl, epa, epb = oracle.overlaps(reads, l_min)
    assert len(epl) == m
    assert np.array_equal(_np(pa, np.uint32), epa) and np.array_equal(_np(pb, np.uint32), epb)
    assert np.array_equal(_np(pl, np.uint8), epl)


def test_planner_host_logic_without_gpu():
    """a8 planner (host only, no CUDA call): the largest length group that fits the budget,
    monotone in the budget, ENOSPC below the one-length workspace, and the greedy call's size
    query agrees with the plan for that group."""
    from paper_conf_ipps_goswamilsp18_b200 import lasagna as lz
    n, L, l_min = 34_851_485, 101, 63  # cfg3
    lp, ws = lz.plan(n, L, l_min, 170 << 30)
    assert lp == L - l_min and 0 < ws <= 170 << 30
    prev = (lp, ws)
    for budget in (60 << 30, 30 << 30, 12 << 30, 6 << 30):
        g, w = lz.plan(n, L, l_min, budget)
        assert 1 <= g <= prev[0] and w <= budget and w <= prev[1], (budget, g, w)
        q = ctypes.c_size_t(0)
        assert lz.lib().lasagna_greedy_graph(None, n, L, l_min, g, None, ctypes.byref(q), None, None,
                                             None, None) == lz.OK
        assert q.value == w
        prev = (g, w)
    g, w = lz.plan(n, L, l_min, 1 << 20)
    assert g == 0 and w > 1 << 20
