"""GPU parity of the a8 semi-streaming paths and of every table geometry, against the oracle.

The configs of BASELINE.json take three geometries of the bucketed (radix-partition) path:
one level (T = 8, cfg1-sized), two levels (T = 16: cfg2, cfg3) and three levels (T = 20:
cfg4, cfg5 with 2n ~ 2.5e9).  cfg4/cfg5 are too large for the oracle, so their geometry is
forced here at cfg1/cfg2 sizes through test hooks (LASAGNA_TEST_LEVELS, LASAGNA_TEST_LAST_BITS;
read by the library on every call).  Each test crosses a geometry with the semi-streaming
driver's length groups (lengths_per_pass, a8: P:L61-67), the input form (packed
rows, device ASCII, page-locked host ASCII streamed by DMA) and the exact LSD fallback path;
every result must equal the oracle bit for bit (succ, olen, |P|, accepted pairs).
"""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import readgen
from tests._util import pruning_expectations

gpu = pytest.mark.gpu


@pytest.fixture(scope="module")
def lz():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    import paper_conf_ipps_goswamilsp18_b200 as m
    m.lib()
    return m


_P2 = {}


@pytest.fixture(scope="module")
def cfg2():
    """cfg2 (BASELINE configs[1]: 2.3 M reads of 100 bp, 1 % errors) and its oracle graph."""
    cfg = readgen.CONFIGS["cfg2"]
    reads = readgen.config_reads(cfg)
    P = oracle.overlaps(reads, cfg.l_min)
    esucc, eolen, acc = oracle.greedy(cfg.n, *P)
    _P2["P"] = P
    return cfg, reads, esucc, eolen, len(P[0]), acc


@pytest.fixture(scope="module")
def cfg1():
    cfg = readgen.CONFIGS["cfg1"]
    reads = readgen.config_reads(cfg)
    epl, epa, epb = oracle.overlaps(reads, cfg.l_min)
    esucc, eolen, _ = oracle.greedy(cfg.n, epl, epa, epb)
    return cfg, reads, (epl, epa, epb), esucc, eolen


def _u32(t):
    return t.cpu().numpy().view(np.uint32)


def _u8(t):
    return t.cpu().numpy().view(np.uint8)


def _same(r, esucc, eolen, m, acc, L=100, l_min=63):
    """Bit-exact graph; |P| exact on one pass, or the claimed-end pruning counts of several
    (tests/_util.pruning_expectations, from the oracle's pairs and claim lengths)."""
    st = r.stats
    assert st["n_greedy"] == acc, (st, acc)
    assert np.array_equal(_u32(r.succ), esucc)
    assert np.array_equal(_u8(r.olen), eolen)
    if st["passes"] > 1 and st["bucketed"]:
        found, pruned = pruning_expectations(L, l_min, st["lengths_per_pass"], _P2["P"], eolen)
        assert (st["n_pairs"], st["pruned_entries"]) == (found, pruned), (st, found, pruned)
        assert found < m and pruned > 0
    else:
        assert st["n_pairs"] == m and st["pruned_entries"] == 0, (st, m)


@gpu
@pytest.mark.parametrize("lpp", [1, 5])
def test_two_level_multipass_from_packed(lz, cfg2, lpp):
    """T = 16 (level-1 scatter + level-2 refine), lengths_per_pass 1 and 5: 37 and 8 device
    passes over the resident packed reads."""
    import torch
    cfg, reads, esucc, eolen, m, acc = cfg2
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    r = lz.greedy_graph(packed, cfg.n, cfg.L, cfg.l_min, lengths_per_pass=lpp)
    assert r.stats["key_sort_bits"] == 16 and r.stats["bucketed"] == 1
    assert r.stats["passes"] == -(-(cfg.L - cfg.l_min) // lpp)
    _same(r, esucc, eolen, m, acc)


@gpu
@pytest.mark.parametrize("where", ["device", "pinned"])
def test_two_level_multipass_from_ascii(lz, cfg2, where):
    """a1 fused into the FIRST group's scatter (device ASCII, or page-locked host ASCII streamed
    in by DMA chunks), later groups reading the packed rows that first pass wrote."""
    import torch
    cfg, reads, esucc, eolen, m, acc = cfg2
    t = torch.from_numpy(reads)
    t = t.cuda() if where == "device" else t.pin_memory()
    g = lz.GreedyGraph(cfg.n, cfg.L, cfg.l_min, "cuda", lengths_per_pass=5)
    r = g.from_ascii(t)
    assert r.stats["passes"] == 8
    _same(r, esucc, eolen, m, acc)
    assert np.array_equal(g.packed.cpu().numpy().view(np.uint64),
                          oracle.pack(reads, lz.words_per_read(cfg.L)))


@gpu
def test_exact_path_multipass(lz, cfg2, monkeypatch):
    """The exact LSD path (table + onesweep passes + contiguous join) with several length
    groups, from packed rows and from ASCII (a separate pack launch on that path)."""
    import torch
    cfg, reads, esucc, eolen, m, acc = cfg2
    monkeypatch.setenv("LASAGNA_PATH", "exact")
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    r = lz.greedy_graph(packed, cfg.n, cfg.L, cfg.l_min, lengths_per_pass=5)
    assert r.stats["bucketed"] == 0 and r.stats["passes"] == 8
    _same(r, esucc, eolen, m, acc)
    g = lz.GreedyGraph(cfg.n, cfg.L, cfg.l_min, "cuda", lengths_per_pass=7)
    r = g.from_ascii(torch.from_numpy(reads).pin_memory())
    assert r.stats["bucketed"] == 0
    _same(r, esucc, eolen, m, acc)


@gpu
@pytest.mark.parametrize("path,lpp,levels", [("", 0, ""), ("", 5, ""), ("", 5, "3"), ("exact", 5, "")])
def test_verification_in_the_greedy(lz, cfg2, monkeypatch, path, lpp, levels):
    """R27: with LASAGNA_VERIFY=greedy the join stores its fingerprint hits unverified and the
    greedy's first round of each length checks them on the bases; the graph, |P| (counted
    there) and the accepted pairs must equal the oracle on the two- and three-level and exact
    paths, one and several length groups."""
    import torch
    cfg, reads, esucc, eolen, m, acc = cfg2
    monkeypatch.setenv("LASAGNA_VERIFY", "greedy")
    if path:
        monkeypatch.setenv("LASAGNA_PATH", path)
    if levels:
        monkeypatch.setenv("LASAGNA_TEST_LEVELS", levels)
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    r = lz.greedy_graph(packed, cfg.n, cfg.L, cfg.l_min, lengths_per_pass=lpp)
    assert r.stats["bucketed"] == (0 if path else 1)
    _same(r, esucc, eolen, m, acc)


@gpu
@pytest.mark.parametrize("lpp,src", [(0, "packed"), (5, "packed"), (5, "pinned"), (3, "device")])
def test_three_level_geometry(lz, cfg2, monkeypatch, lpp, src):
    """The cfg4/cfg5 geometry (three partition levels of 8, 8 and 4 bits: T = 20, 2^20 split
    buckets per length) forced at cfg2 size: one pass and several, from packed rows, from
    page-locked host ASCII (the DMA ring in the level-2 buffer) and from device ASCII."""
    import torch
    cfg, reads, esucc, eolen, m, acc = cfg2
    monkeypatch.setenv("LASAGNA_TEST_LEVELS", "3")
    monkeypatch.setenv("LASAGNA_TEST_LAST_BITS", "4")
    if src == "packed":
        packed = lz.load_reads(torch.from_numpy(reads).cuda())
        r = lz.greedy_graph(packed, cfg.n, cfg.L, cfg.l_min, lengths_per_pass=lpp)
    else:
        t = torch.from_numpy(reads)
        t = t.cuda() if src == "device" else t.pin_memory()
        g = lz.GreedyGraph(cfg.n, cfg.L, cfg.l_min, "cuda", lengths_per_pass=lpp)
        r = g.from_ascii(t)
    assert r.stats["key_sort_bits"] == 20 and r.stats["bucketed"] == 1, r.stats
    assert r.stats["sort_launches"] == 2 * r.stats["passes"]
    _same(r, esucc, eolen, m, acc)


@gpu
@pytest.mark.parametrize("levels,last", [("1", "8"), ("2", "8"), ("3", "4"), ("3", "1")])
def test_forced_geometries_overlaps_cfg1(lz, cfg1, monkeypatch, levels, last):
    """lasagna_overlaps and the greedy graph under every partition depth at cfg1 (T = 8, 16,
    20 and 17): the full read-end pair list, element by element."""
    import torch
    cfg, reads, (epl, epa, epb), esucc, eolen = cfg1
    monkeypatch.setenv("LASAGNA_TEST_LEVELS", levels)
    monkeypatch.setenv("LASAGNA_TEST_LAST_BITS", last)
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    pl, pa, pb = lz.overlaps(packed, cfg.n, cfg.L, cfg.l_min)
    assert np.array_equal(_u32(pa), epa) and np.array_equal(_u32(pb), epb)
    assert np.array_equal(_u8(pl), epl)
    r = lz.greedy_graph(packed, cfg.n, cfg.L, cfg.l_min, lengths_per_pass=4)
    T = {"1": 8, "2": 16, "3": 16 + int(last)}[levels]
    assert r.stats["key_sort_bits"] == T and r.stats["bucketed"] == 1
    assert np.array_equal(_u32(r.succ), esucc) and np.array_equal(_u8(r.olen), eolen)


@gpu
def test_pool_growth_retry_with_length_groups(lz, monkeypatch):
    """A length with more verified pairs than the default pair pool (every length from 1, all
    reads of a 20 kbp genome) under lengths_per_pass = 5: ENOSPC, the binding regrows the
    workspace and retries; the graph equals the oracle."""
    import torch
    reads = readgen.reads(7, 20_000, 3000, 64, 0.01)
    P = oracle.overlaps(reads, 1)
    esucc, eolen, acc = oracle.greedy(3000, *P)
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    r = lz.greedy_graph(packed, 3000, 64, 1, lengths_per_pass=5)
    assert np.array_equal(_u32(r.succ), esucc) and np.array_equal(_u8(r.olen), eolen)
    if r.stats["bucketed"]:
        found, pruned = pruning_expectations(64, 1, r.stats["lengths_per_pass"], P, eolen)
    else:  # the 1-base lengths overflow a slack region: the exact path (no pruning)
        found, pruned = len(P[0]), 0
    assert (r.stats["n_pairs"], r.stats["pruned_entries"]) == (found, pruned)


def _expected_false_matches(n: int, n_len: int, bits: float) -> float:
    """R12 closed form: per length V/2 probe-side and V/2 build-side canonical entries agree
    on `bits` bits of mix(min(H, Hr)) with probability 2^-bits."""
    V = 2 * n
    return n_len * (V / 2) ** 2 / 2.0 ** bits


@gpu
@pytest.mark.parametrize("fp_bits", [26, 30])
def test_false_match_rate_at_chosen_key_width(lz, cfg2, monkeypatch, fp_bits):
    """Hash-collision rate (north star: "checked on hash-collision rates").  A bucketed key
    compares 8 implied bits (its level-1 region) plus its stored fingerprint bits; keeping only
    the top `fp_bits` stored bits (test hook), the rejected hits at cfg2 must follow the R12
    closed form with 8 + fp_bits bits (Poisson, 5 sigma) and the graph must stay exact."""
    import torch
    cfg, reads, esucc, eolen, m, acc = cfg2
    monkeypatch.setenv("LASAGNA_TEST_FP_BITS", str(fp_bits))
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    r = lz.greedy_graph(packed, cfg.n, cfg.L, cfg.l_min)
    exp = _expected_false_matches(cfg.n, cfg.L - cfg.l_min, 8 + fp_bits)
    assert exp > 100
    obs = r.stats["fp_false_matches"]
    assert abs(obs - exp) <= 5 * exp ** 0.5 + 0.02 * exp, (obs, exp)
    _same(r, esucc, eolen, m, acc)


def test_false_match_rate_vertex_bits_32_closed_form():
    """at cfg4/cfg5 (vbits = 32) a key stores 62 - 32 = 30 fingerprint bits.  The
    bucketed key stores the 30 bits BELOW the level-1 digit, which its region implies, so a
    comparison covers 38 bits: (V/2)^2 / 2^38 ~ 5.7e6 rejected hits per length at cfg5 (~5 %
    of the true pairs), against 1.45e9 (~15x the true pairs) if the region digit were stored."""
    cfg = readgen.CONFIGS["cfg5"]
    V = 2 * cfg.n
    vbits = (V - 1).bit_length()
    assert vbits == 32
    per_len = _expected_false_matches(cfg.n, 1, (62 - vbits) + 8)
    assert 3e6 < per_len < 1e7
    true_per_len = 3.86e9 / (cfg.L - cfg.l_min)  # SURVEY 8(d) expected |P|
    assert per_len < 0.1 * true_per_len
    assert _expected_false_matches(cfg.n, 1, 62 - vbits) > 10 * true_per_len


@gpu
def test_pruning_off_gives_full_pair_count(lz, cfg2, monkeypatch):
    """LASAGNA_NO_PRUNE=1: several passes, nothing pruned, |P| exact, same graph."""
    import torch
    cfg, reads, esucc, eolen, m, acc = cfg2
    monkeypatch.setenv("LASAGNA_NO_PRUNE", "1")
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    r = lz.greedy_graph(packed, cfg.n, cfg.L, cfg.l_min, lengths_per_pass=5)
    assert r.stats["passes"] == 8 and r.stats["pruned_entries"] == 0
    assert r.stats["n_pairs"] == m and r.stats["n_greedy"] == acc
    assert np.array_equal(_u32(r.succ), esucc) and np.array_equal(_u8(r.olen), eolen)


def _one_length_workspace(lz, n, L, l_min) -> int:
    import ctypes
    ws = ctypes.c_size_t(0)
    lz.lasagna._check(lz.lib().lasagna_greedy_graph(None, n, L, l_min, 1, None, ctypes.byref(ws),
                                                    None, None, None, None))
    return int(ws.value)


@gpu
@pytest.mark.parametrize("frac,levels", [(0.6, ""), (0.12, ""), (0.0, ""), (0.3, "3")])
def test_hash_range_subpasses_cfg2(lz, cfg2, monkeypatch, frac, levels):
    """f4: a workspace below one whole length's tables makes every length run
    in K hash-range sub-passes (the replacement of the paper's external merge, Alg. 1): the
    graph, |P| (live pairs under pruning) and the pruned-entry count equal the oracle's."""
    import torch
    if levels:
        monkeypatch.setenv("LASAGNA_TEST_LEVELS", levels)
        monkeypatch.setenv("LASAGNA_TEST_LAST_BITS", "4")
    cfg, reads, esucc, eolen, m, acc = cfg2
    one = _one_length_workspace(lz, cfg.n, cfg.L, cfg.l_min)
    _, least = lz.plan(cfg.n, cfg.L, cfg.l_min, 1)  # 256 sub-passes: the fixed parts remain
    budget = least + int((one - least) * frac)
    lp, need = lz.plan(cfg.n, cfg.L, cfg.l_min, budget)
    assert lp == 1 and need <= budget
    runner = lz.GreedyGraph(cfg.n, cfg.L, cfg.l_min, "cuda", budget_bytes=budget)
    assert runner.ws_bytes <= budget
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    r = runner(packed)
    K = r.stats["hash_subpasses"]
    assert K > 1 and K & (K - 1) == 0, r.stats
    assert r.stats["passes"] == K * (cfg.L - cfg.l_min)
    assert r.stats["partition_levels"] == (3 if levels else 2)
    assert np.array_equal(_u32(r.succ), esucc) and np.array_equal(r.olen.cpu().numpy(), eolen)
    found, pruned = pruning_expectations(cfg.L, cfg.l_min, 1, _P2["P"], eolen)
    assert (r.stats["n_pairs"], r.stats["pruned_entries"], r.stats["n_greedy"]) == (found, pruned, acc)
    # the same from device ASCII (a1 fused into the first sub-pass of the first length)
    r2 = runner.from_ascii(torch.from_numpy(reads).cuda())
    assert np.array_equal(_u32(r2.succ), esucc) and np.array_equal(r2.olen.cpu().numpy(), eolen)


@gpu
def test_plan_subpasses_monotone(lz):
    """The planner: one whole length at its exact size, then the fewest sub-passes that fit,
    K doubling as the budget shrinks; ENOSPC only below 256 sub-passes."""
    n, L, l_min = 2_000_000, 100, 63
    one = _one_length_workspace(lz, n, L, l_min)
    lp, need = lz.plan(n, L, l_min, one)
    assert lp == 1 and need == one
    lp, least = lz.plan(n, L, l_min, 1 << 20)
    assert lp == 0 and least > 1 << 20 and least < one
    prev = one
    for frac in (0.7, 0.4, 0.2, 0.1, 0.05):
        b = least + int((one - least) * frac)
        lp, need = lz.plan(n, L, l_min, b)
        assert lp == 1 and least <= need <= b and need <= prev
        prev = need
    assert prev < one
