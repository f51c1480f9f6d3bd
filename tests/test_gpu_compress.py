"""GPU parity of Compress (lasagna_compress: paths by list ranking, contigs by two scans and a
placement; Fig. 7) against oracle_compress, byte for byte: the contig bases, the
offsets and the seed of every contig."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import readgen
from tests._util import NONE, golden, to_array
from tests.test_compress_oracle import _circular_reads

gpu = pytest.mark.gpu


@pytest.fixture(scope="module")
def lz():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    import paper_conf_ipps_goswamilsp18_b200 as m
    m.lib()
    return m


def _check(lz, reads, succ, olen):
    import torch
    n, L = reads.shape
    packed = lz.load_reads(torch.from_numpy(reads).cuda())
    c = lz.compress(packed, n, L, torch.from_numpy(succ.view(np.int32)).cuda(),
                    torch.from_numpy(olen).cuda())
    eb, eo, es = oracle.compress(reads, succ, olen)
    assert c.bases.cpu().numpy().tobytes() == eb
    assert np.array_equal(c.offsets.cpu().numpy().astype(np.uint64), eo)
    assert np.array_equal(c.seeds.cpu().numpy().view(np.uint32), es)
    return len(es)


@gpu
def test_micro_example(lz):
    g = golden("micro_example.txt")
    reads = to_array(g["reads"])
    succ = np.array([NONE if x == "N" else int(x) for x in g["succ"]], dtype=np.uint32)
    olen = np.array([int(x) for x in g["olen"]], dtype=np.uint8)
    assert _check(lz, reads, succ, olen) == 1


@gpu
@pytest.mark.parametrize("cfg", ["cfg1", "cfg2"])
def test_config_contigs(lz, cfg):
    c = readgen.CONFIGS[cfg]
    reads = readgen.config_reads(c)
    succ, olen, _, _ = oracle.greedy_graph(reads, c.l_min)
    assert _check(lz, reads, succ, olen) > 100


@gpu
@pytest.mark.parametrize("L,l_min,p", [(40, 20, 0.0), (150, 111, 0.01), (256, 200, 0.0), (33, 5, 0.02)])
def test_shapes(lz, L, l_min, p):
    reads = readgen.reads(5, 30_000, 4000, L, p)
    succ, olen, _, _ = oracle.greedy_graph(reads, l_min)
    _check(lz, reads, succ, olen)


@gpu
def test_cycles_and_paths_together(lz):
    """A circular genome's reads (one cycle and its complement: no seed, R21) next to a linear
    genome's reads: only the linear contigs come out."""
    circ = _circular_reads(300, 40, 10)
    lin = readgen.reads(2, 3000, 400, 40, 0.0)
    reads = np.ascontiguousarray(np.concatenate([circ, lin]))
    succ, olen, _, _ = oracle.greedy_graph(reads, 20)
    assert np.all(succ[: 2 * len(circ)] != NONE)
    _check(lz, reads, succ, olen)


@gpu
def test_graph_without_edges(lz):
    reads = readgen.reads(1, 10_000, 50, 100, 0.0)
    succ = np.full(100, NONE, dtype=np.uint32)
    olen = np.zeros(100, dtype=np.uint8)
    assert _check(lz, reads, succ, olen) == 0
