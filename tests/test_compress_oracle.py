"""Pins of the Compress oracle (oracle_compress; PAPER §III-D, Fig. 7; readings
R20, R21 in DESIGN.md), CPU only.

* the hand-derived micro example (tests/golden/micro_compress.txt);
* error-free reads of a random genome: every contig is a substring of the genome or of its
  reverse complement (the contigs re-assemble the sequence the reads came from);
* every read of a path lies in its contig at its offset (an exact overlap chain);
* the pure-Python transcription of the paper's text (oracle/brute.py) on tiny inputs;
* a circular genome: every vertex has in- and out-degree 1, no seed, no contig (R21).
"""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import readgen
from oracle import brute
from tests._util import NONE, golden, to_array

_COMP = bytes.maketrans(b"ACGT", b"TGCA")


def _graph(reads, l_min):
    succ, olen, _, _ = oracle.greedy_graph(reads, l_min)
    return succ, olen


def _contig_list(c, offs):
    return [c[int(offs[k]):int(offs[k + 1])] for k in range(len(offs) - 1)]


def test_micro_example_contig():
    g = golden("micro_example.txt")
    reads = to_array(g["reads"])
    succ = np.array([NONE if x == "N" else int(x) for x in g["succ"]], dtype=np.uint32)
    olen = np.array([int(x) for x in g["olen"]], dtype=np.uint8)
    c, offs, seeds = oracle.compress(reads, succ, olen)
    exp = golden("micro_compress.txt")
    assert [int(s) for s in seeds] == [int(x) for x in exp["seeds"]]
    assert [x.decode() for x in _contig_list(c, offs)] == exp["contigs"]


def test_error_free_contigs_are_genome_substrings():
    cfg = readgen.CONFIGS["cfg1"]  # 200 kbp genome, 20 k error-free reads (10x)
    reads = readgen.config_reads(cfg)
    genome = readgen.genome(cfg.seed, cfg.G).tobytes()
    rc = genome[::-1].translate(_COMP)
    succ, olen = _graph(reads, cfg.l_min)
    c, offs, seeds = oracle.compress(reads, succ, olen)
    contigs = _contig_list(c, offs)
    assert len(contigs) > 100
    for t in contigs:
        assert len(t) > cfg.L
        assert t in genome or t in rc
    # total = sum of the overhangs of the path vertices (Fig. 7's scans)
    assert int(offs[-1]) == len(c) == sum(len(t) for t in contigs)


def _oriented(reads, v):
    r = bytes(reads[v >> 1])
    return r[::-1].translate(_COMP) if v & 1 else r


@pytest.mark.parametrize("p_err", [0.0, 0.01])
def test_every_path_read_sits_in_its_contig(p_err):
    """Walking each emitted path: read v_j starts at offset sum_{i<j} (L - olen(v_i)) of its
    contig and all L of its bases are there (consecutive reads overlap exactly)."""
    reads = readgen.reads(3, 60_000, 6000, 100, p_err)
    n, L = reads.shape
    succ, olen = _graph(reads, 63)
    c, offs, seeds = oracle.compress(reads, succ, olen)
    assert len(seeds) > 50
    for k, s in enumerate(seeds.tolist()):
        pos, v = int(offs[k]), s
        while True:
            assert c[pos:pos + L] == _oriented(reads, v)
            if succ[v] == NONE:
                assert pos + L == int(offs[k + 1])
                break
            pos += L - int(olen[v])
            v = int(succ[v])


@pytest.mark.parametrize("seed", range(6))
def test_matches_transcription_of_the_text(seed):
    rng = np.random.default_rng(seed)
    G = int(rng.integers(200, 800))
    reads = readgen.reads(seed, G, int(rng.integers(20, 120)), 24, float(rng.choice([0, 0.02])))
    succ, olen = _graph(reads, 10)
    c, offs, seeds = oracle.compress(reads, succ, olen)
    exp = brute.contigs([bytes(r).decode() for r in reads], succ.tolist(), olen.tolist())
    assert [int(s) for s in seeds] == [s for s, _ in exp]
    assert [x.decode() for x in _contig_list(c, offs)] == [t for _, t in exp]


def _circular_reads(G: int, L: int, step: int, seed: int = 9) -> np.ndarray:
    rng = np.random.default_rng(seed)
    g = np.frombuffer(b"ACGT", dtype=np.uint8)[rng.integers(0, 4, G)]
    gg = np.concatenate([g, g[:L]])
    return np.ascontiguousarray(np.stack([gg[s:s + L] for s in range(0, G, step)]))


def test_circular_genome_has_no_seed():
    """Reads tiling a circular genome: the greedy graph is one cycle and its complement,
    every vertex with in- and out-degree 1, so no seed and no contig (R21)."""
    reads = _circular_reads(300, 40, 10)
    succ, olen = _graph(reads, 20)
    assert np.all(succ != NONE)
    c, offs, seeds = oracle.compress(reads, succ, olen)
    assert len(seeds) == 0 and len(c) == 0 and offs.tolist() == [0]
    assert brute.contigs([bytes(r).decode() for r in reads], succ.tolist(), olen.tolist()) == []
