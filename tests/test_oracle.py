"""Pins for the CPU oracle (`-m "not gpu"`): the oracle against what the paper and the
mathematics fix — never against itself.  See oracle/oracle.c's header for the map."""
from __future__ import annotations

import itertools
import random

import numpy as np
import pytest

import oracle
import readgen
from oracle import brute
from tests._util import NONE, check_graph, golden, to_array

Q61 = (1 << 61) - 1


# ---------------------------------------------------------------- Fig. 5 / Fig. 6
def _fig():
    g = golden("fig5_fig6.txt")
    return (g["read"][0], int(g["sigma"][0]), int(g["q"][0]),
            [int(x) for x in g["P"]], [int(x) for x in g["S"]],
            [int(x) for x in g["Pprime_raw"]], [int(x) for x in g["Pprime_mod"]])


def test_fig5_hillis_steele_prefix_scan():
    read, sigma, q, P, _, _, _ = _fig()
    assert oracle.scan_prefix(read, sigma, q).tolist() == P


def test_fig5_definition_matches_printed_prefixes():
    read, sigma, q, P, _, _, _ = _fig()
    assert [oracle.F(read[: i + 1], sigma, q) for i in range(len(read))] == P


def test_fig6_suffix_from_prefix():
    read, sigma, q, P, S, raw, mod = _fig()
    S_got, Pp = oracle.suffix_from_prefix(np.array(P, dtype=np.uint64), sigma, q)
    assert S_got.tolist() == S
    assert Pp[1:].tolist() == mod
    # the raw row is P[i-1] * M[L-i] before the reduction
    M = oracle.place_values(sigma, q, len(read))
    L = len(read)
    assert [P[i - 1] * int(M[L - i]) for i in range(1, L)] == raw


def test_fig6_definition_matches_printed_suffixes():
    read, sigma, q, _, S, _, _ = _fig()
    assert [oracle.F(read[i:], sigma, q) for i in range(len(read))] == S


def test_encoding_is_the_unique_one_reproducing_fig5():
    """Reading R1: of the 24 code assignments only A0 C1 T2 G3 reproduces Fig. 5's P."""
    read, sigma, q, P, _, _, _ = _fig()
    hits = []
    for perm in itertools.permutations(range(4)):
        enc = dict(zip("ACGT", perm))
        f, vals = 0, []
        for ch in read:
            f = (f * sigma + enc[ch]) % q
            vals.append(f)
        if vals == P:
            hits.append(enc)
    assert hits == [{"A": 0, "C": 1, "G": 3, "T": 2}]
    assert [oracle.code(c) for c in "ACGTacgt"] == [0, 1, 3, 2, 0, 1, 3, 2]
    assert oracle.code("N") == -1


# ---------------------------------------------------------------- production parameters
def _base5(s: str) -> int:
    digits = "".join(str({"A": 0, "C": 1, "T": 2, "G": 3}[c]) for c in s)
    return int(digits, 5)


@pytest.mark.parametrize("seed", range(5))
def test_F_equals_base5_integer_mod_q(seed):
    """F(s) = (value of s read as a base-sigma numeral) mod q — closed form via Python's
    own int(., 5) parser (R2, R4)."""
    rng = random.Random(seed)
    for m in [1, 2, 10, 26, 27, 40, 63, 100, 150, 256]:
        s = "".join(rng.choice("ACGT") for _ in range(m))
        assert oracle.F(s) == _base5(s) % Q61
        if m <= 26:  # injective range: 5^26 < 2^61 - 1, no reduction at all
            assert oracle.F(s) == _base5(s)


def test_F_small_prime_agrees_with_scan():
    rng = random.Random(7)
    for q in [13, 101, 65521, Q61]:
        for sigma in [4, 5, 7]:
            s = "".join(rng.choice("ACGT") for _ in range(37))
            P = oracle.scan_prefix(s, sigma, q).tolist()
            assert P == [_base_sigma(s[: i + 1], sigma) % q for i in range(len(s))]


def _base_sigma(s, sigma):
    v = 0
    for c in s:
        v = v * sigma + {"A": 0, "C": 1, "T": 2, "G": 3}[c]
    return v


def test_fingerprints_table_layout_and_rc():
    reads = readgen.reads(3, 5000, 12, 40, 0.0)
    l_min = 30
    pfx, sfx = oracle.fingerprints(reads, l_min)
    n, L = reads.shape
    assert pfx.shape == (L - l_min + 1, 2 * n)
    comp = {"A": "T", "C": "G", "G": "C", "T": "A"}
    for i in range(n):
        r = bytes(reads[i]).decode()
        rc = "".join(comp[c] for c in reversed(r))
        for l in range(l_min, L + 1):
            k = l - l_min
            assert int(pfx[k, 2 * i]) == _base5(r[:l]) % Q61
            assert int(sfx[k, 2 * i]) == _base5(r[L - l:]) % Q61
            assert int(pfx[k, 2 * i + 1]) == _base5(rc[:l]) % Q61
            assert int(sfx[k, 2 * i + 1]) == _base5(rc[L - l:]) % Q61


# ---------------------------------------------------------------- packing
@pytest.mark.parametrize("L,stride", [(8, 1), (32, 1), (33, 2), (100, 4), (101, 4), (150, 8)])
def test_pack_unpack_roundtrip(L, stride):
    reads = readgen.reads(11, 10_000, 50, L, 0.05)
    packed = oracle.pack(reads, stride)
    for i in range(reads.shape[0]):
        for k in range(L):
            c = (int(packed[i, k // 32]) >> (2 * (k % 32))) & 3
            assert c == "ACTG".index(chr(reads[i, k])), (i, k)
        # unused bits and padding words are zero
        total_bits = 64 * stride
        val = sum(int(packed[i, w]) << (64 * w) for w in range(stride))
        assert val >> (2 * L) == 0 or 2 * L >= total_bits


def test_first_bad():
    reads = readgen.reads(1, 1000, 20, 30, 0.0)
    assert oracle.first_bad(reads) == -1
    bad = reads.copy()
    bad[7, 3] = ord("N")
    bad[12, 0] = ord("x")
    assert oracle.first_bad(bad) == 7
    low = np.char.lower(reads.view("S30")).view(np.uint8).reshape(reads.shape)
    assert oracle.first_bad(low) == -1
    with pytest.raises(ValueError):
        oracle.overlaps(bad, 10)


# ---------------------------------------------------------------- overlaps & greedy
def test_micro_example():
    g = golden("micro_example.txt")
    reads = to_array(g["reads"])
    l_min = int(g["l_min"][0])
    exp_pairs = [tuple(int(x) for x in p.split(",")) for p in g["pairs"]]
    pl, pa, pb = oracle.overlaps(reads, l_min)
    assert list(zip(pl.tolist(), pa.tolist(), pb.tolist())) == exp_pairs
    succ, olen, m, acc = oracle.greedy_graph(reads, l_min)
    exp_succ = [NONE if x == "N" else int(x) for x in g["succ"]]
    assert succ.tolist() == exp_succ
    assert olen.tolist() == [int(x) for x in g["olen"]]
    assert m == 3 and acc == 2
    # brute force agrees too
    assert brute.pairs(g["reads"], l_min) == exp_pairs


def _tiny_instances():
    """Repeat-rich tiny inputs: small genomes (many ties and duplicates), tandem repeats,
    reverse-complement palindromes and periodic reads (reading R9's cases)."""
    out = []
    for seed in range(8):
        rng = random.Random(seed)
        L = rng.choice([8, 12, 16, 20])
        G = rng.choice([30, 60, 200])
        n = rng.choice([10, 25, 40])
        p = rng.choice([0.0, 0.0, 0.02])
        reads = [bytes(r).decode() for r in readgen.reads(seed, G, n, L, p)]
        l_min = rng.randint(2, L - 2)
        out.append((reads, l_min))
    # tandem repeat + palindrome + periodic
    L = 12
    reads = ["ACGTTA" * 2, "CGTTAACGTTAA", "GTTAACGTTAAC", "AAGCTTAAGCTT", "ACACACACACAC",
             "GTGTGTGTGTGT", "GAATTCGAATTC", "TTCGAATTCGAA", "ACGTACGTACGT", "CGTACGTACGTA"]
    out.append((reads, 3))
    return out


@pytest.mark.parametrize("case", range(9))
def test_overlaps_match_brute_force(case):
    reads, l_min = _tiny_instances()[case]
    arr = to_array(reads)
    pl, pa, pb = oracle.overlaps(arr, l_min)
    got = list(zip(pl.tolist(), pa.tolist(), pb.tolist()))
    assert got == brute.pairs(reads, l_min)


@pytest.mark.parametrize("case", range(9))
def test_greedy_matches_brute_force_and_invariants(case):
    reads, l_min = _tiny_instances()[case]
    arr = to_array(reads)
    P = brute.pairs(reads, l_min)
    exp_succ, exp_olen = brute.greedy(len(reads), P)
    succ, olen, m, acc = oracle.greedy_graph(arr, l_min)
    assert succ.tolist() == exp_succ
    assert olen.tolist() == exp_olen
    assert m == len(P)
    pairs = tuple(np.array(x) for x in zip(*P)) if P else None
    check_graph(arr, l_min, succ, olen, pairs)


def test_twin_symmetry_of_directed_overlaps():
    """Every directed overlap has its complementary edge: |O| = 2|P|."""
    reads, l_min = _tiny_instances()[8]
    O = brute.directed_overlaps(reads, l_min)
    for (u, v, l) in O:
        assert (v ^ 1, u ^ 1, l) in O
    assert len(O) == 2 * len(brute.pairs(reads, l_min))


def test_cfg1_invariants_and_expected_count():
    """cfg1 (20k error-free reads): invariants, and |P| against the closed form
    E|P_l| = n(n-1) (G-L+1-d) / (G-L+1)^2 (1-p)^(2l), d = L - l (reads offset by exactly
    d on the genome overlap by l; both overlapping stretches must be error-free)."""
    cfg = readgen.CONFIGS["cfg1"]
    reads = readgen.config_reads(cfg)
    pl, pa, pb = oracle.overlaps(reads, cfg.l_min)
    succ, olen, acc = oracle.greedy(cfg.n, pl, pa, pb)
    n, G, L, p = cfg.n, cfg.G, cfg.L, cfg.p_err
    Gp = G - L + 1
    exp = sum(n * (n - 1) * (Gp - (L - l)) / Gp ** 2 * (1 - p) ** (2 * l)
              for l in range(cfg.l_min, L))
    assert abs(len(pl) / exp - 1) < 0.03, (len(pl), exp)
    # order: l descending, then (a, b)
    key = (255 - pl.astype(np.int64)) * (1 << 40) + pa.astype(np.int64) * (1 << 20) + pb
    assert np.all(np.diff(key) > 0)
    assert np.all(pa < pb)
    # invariants on a sample of edges (checking all 40k takes a few seconds; do all)
    check_graph(reads, cfg.l_min, succ, olen, (pl, pa, pb))
    # the greedy keeps every read end's longest overlap when it is free: the first pair of
    # each read end in order is accepted unless its partner was taken earlier
    assert acc > 0.9 * n


def test_error_reads_expected_count():
    """1% substitution errors: the (1-p)^(2l) factor of the closed form."""
    G, n, L, l_min, p = 300_000, 30_000, 100, 63, 0.01
    reads = readgen.reads(99, G, n, L, p)
    pl, _, _ = oracle.overlaps(reads, l_min)
    Gp = G - L + 1
    exp = sum(n * (n - 1) * (Gp - (L - l)) / Gp ** 2 * (1 - p) ** (2 * l)
              for l in range(l_min, L))
    assert abs(len(pl) / exp - 1) < 0.04, (len(pl), exp)


def test_fingerprint_collision_rate_small_modulus():
    """Hash-collision rate of the oracle's Rabin-Karp F with a small prime
    modulus: N distinct 40-mers that share their last 24 bases and differ only in the first 16
    collide in pairs as a uniform hash would (Poisson, mean C(N, 2) / q), i.e. the leading
    bases reach the fingerprint through their place values.  Negative control: radix 4 modulo
    2^13, whose place values vanish beyond 7 bases, maps every one of them to one value."""
    rng = np.random.default_rng(11)
    q, N = 8191, 20_000
    tail = "".join("ACGT"[i] for i in rng.integers(0, 4, 24))
    heads = np.unique(rng.integers(0, 4 ** 16, N + 100, dtype=np.int64))[:N]
    assert len(heads) == N
    strs = ["".join("ACGT"[(int(h) >> (2 * k)) & 3] for k in range(16)) + tail for h in heads]
    vals = np.array([oracle.F(x, 5, q) for x in strs], dtype=np.int64)
    assert vals.min() >= 0 and vals.max() < q
    c = np.bincount(vals, minlength=q)
    pairs = int((c * (c - 1) // 2).sum())
    exp = N * (N - 1) / 2 / q
    assert abs(pairs - exp) <= 5 * exp ** 0.5, (pairs, exp)
    bad = {oracle.F(x, 4, 8192) for x in strs}
    assert len(bad) == 1


# ---------------------------------------------------------------- approximate mode
_CODE = {"A": 0, "C": 1, "T": 2, "G": 3}
_COMPL = {"A": "T", "C": "G", "G": "C", "T": "A"}


def _oriented_str(r: str, o: int) -> str:
    return r if o == 0 else "".join(_COMPL[c] for c in reversed(r))


def _fp_bigint(s: str, sigma: int, q: int) -> int:
    """F(s) = sum_k c(s_k) sigma^(|s|-1-k) mod q as one Python big integer, reduced once."""
    return sum(_CODE[c] * sigma ** (len(s) - 1 - k) for k, c in enumerate(s)) % q


def _approx_brute(reads: list[str], l_min: int, s1, q1, s2, q2):
    """The definition over every ordered pair of oriented reads: (l, u, v^1) for u < v^1, other
    reads, when the suffix_l of seq(u) and the prefix_l of seq(v) have equal fingerprint pairs."""
    L = len(reads[0])
    seqs = [_oriented_str(reads[v >> 1], v & 1) for v in range(2 * len(reads))]
    out = []
    for l in range(L - 1, l_min - 1, -1):
        pref = [(_fp_bigint(s[:l], s1, q1), _fp_bigint(s[:l], s2, q2)) for s in seqs]
        for u, su in enumerate(seqs):
            f = (_fp_bigint(su[L - l:], s1, q1), _fp_bigint(su[L - l:], s2, q2))
            for v in range(len(seqs)):
                if (u >> 1) != (v >> 1) and u < (v ^ 1) and pref[v] == f:
                    out.append((l, u, v ^ 1))
    return sorted(out, key=lambda t: (-t[0], t[1], t[2]))


@pytest.mark.parametrize("case", range(9))
def test_approx_overlaps_equal_exact_with_128bit_fingerprints(case):
    """With the paper's two 64-bit-class fingerprints (radix 5 mod 2^61-1, radix 7 mod
    2^64-59) the approximate pair list is the exact overlap set (brute force of strings)."""
    reads, l_min = _tiny_instances()[case]
    got = list(zip(*(t.tolist() for t in oracle.overlaps_approx(to_array(reads), l_min))))
    assert got == brute.pairs(reads, l_min)


@pytest.mark.parametrize("case,q1,q2", [(0, 11, 13), (3, 7, 5), (6, 31, 29), (8, 3, 2)])
def test_approx_overlaps_tiny_moduli_match_definition(case, q1, q2):
    """Deliberately tiny primes: fingerprints collide, the approximate list grows past the
    exact one, and equals a big-integer brute force of its definition; every exact overlap is
    in it (equal strings have equal fingerprints)."""
    reads, l_min = _tiny_instances()[case]
    got = list(zip(*(t.tolist() for t in oracle.overlaps_approx(to_array(reads), l_min, 7, q2, 5, q1))))
    assert got == _approx_brute(reads, l_min, 5, q1, 7, q2)
    exact = set(brute.pairs(reads, l_min))
    assert exact <= set(got)
    assert len(got) > len(exact)  # the tiny moduli do produce false pairs


def test_approx_overlaps_cfg1_equal_exact():
    """cfg1 reads (20 k reads, 10x): the 128-bit approximate mode finds no false pair."""
    cfg = readgen.CONFIGS["cfg1"]
    reads = readgen.config_reads(cfg)
    e = oracle.overlaps(reads, cfg.l_min)
    a = oracle.overlaps_approx(reads, cfg.l_min)
    assert all(np.array_equal(x, y) for x, y in zip(e, a))
