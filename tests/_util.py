"""Shared test helpers: golden-file parsing and the string-graph invariant checker.

The invariant checker follows the definitions only (P:L37 edge + complementary edge,
P:L168 at most one in/out edge per vertex, P:L105 length range) and is used on both the
oracle's and the CUDA path's outputs.
"""
from __future__ import annotations

import os

import numpy as np

NONE = 0xFFFFFFFF
_COMP = bytes.maketrans(b"ACGTacgt", b"TGCAtgca")


def read_golden(path: str) -> dict[str, list[str]]:
    out: dict[str, list[str]] = {}
    with open(path) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            key, *vals = line.split()
            out[key] = vals
    return out


def golden(name: str) -> dict[str, list[str]]:
    here = os.path.dirname(os.path.abspath(__file__))
    return read_golden(os.path.join(here, "golden", name))


def to_array(reads: list[str]) -> np.ndarray:
    return np.array([[ord(c) for c in r] for r in reads], dtype=np.uint8)


def oriented(reads: np.ndarray, v: int) -> bytes:
    r = bytes(reads[v >> 1]).upper()
    if v & 1:
        return r[::-1].translate(_COMP)
    return r


def check_graph(reads: np.ndarray, l_min: int, succ: np.ndarray, olen: np.ndarray,
                pairs=None) -> int:
    """Assert the greedy string-graph invariants; return the number of directed edges.

    * every edge (u, succ[u], olen[u]) is a true overlap with l in [l_min, L-1] between
      different reads (reading R9);
    * its complementary edge (v', u', l) is present: succ[succ[u]^1] == u^1;
    * in-degree <= 1 (out-degree <= 1 holds by construction of succ);
    * maximality, when the candidate pair list is given: no pair (l, a, b) has both read
      ends free (the greedy would have taken it).
    """
    n, L = reads.shape
    V = 2 * n
    succ = np.asarray(succ, dtype=np.int64)
    olen = np.asarray(olen, dtype=np.int64)
    has = succ != NONE
    assert np.all((olen == 0) == ~has), "olen must be 0 exactly where succ is NONE"
    us = np.nonzero(has)[0]
    vs = succ[us]
    assert np.all(vs < V)
    # in-degree <= 1
    assert len(np.unique(vs)) == len(vs), "a vertex has two incoming edges"
    # complementary edges
    tw = succ[vs ^ 1]
    assert np.all(tw == (us ^ 1)), "missing complementary edge"
    assert np.all(olen[vs ^ 1] == olen[us])
    for u, v in zip(us.tolist(), vs.tolist()):
        l = int(olen[u])
        assert l_min <= l <= L - 1
        assert (u >> 1) != (v >> 1)
        su, sv = oriented(reads, u), oriented(reads, v)
        assert su[L - l:] == sv[:l], f"edge {u}->{v} l={l} is not an overlap"
    if pairs is not None:
        pl, pa, pb = pairs
        free_a = ~has[np.asarray(pa, dtype=np.int64)]
        free_b = ~has[np.asarray(pb, dtype=np.int64)]
        assert not np.any(free_a & free_b), "greedy result is not maximal"
    return len(us)


def pruning_expectations(L: int, l_min: int, G: int, pairs, olen) -> tuple[int, int]:
    """What claimed-end pruning must report for length groups of G lengths
    (L-1 down to l_min): a read end x is claimed at length olen[x] (the greedy claims every end
    at most once), so when the group whose top length is l_hi is built, exactly the ends with
    olen[x] > l_hi are claimed.  The entry of vertex x^1 at each length of that group is then
    dropped (pruned entries), and a pair (l, a, b) is still found iff neither a nor b was
    claimed before its group.  Returns (pairs found, entries pruned)."""
    pl, pa, pb = (np.asarray(t) for t in pairs)
    olen = np.asarray(olen, dtype=np.int64)
    top = L - 1 - ((L - 1 - pl.astype(np.int64)) // G) * G  # l_hi of each pair's group
    found = int(np.count_nonzero((olen[pa] <= top) & (olen[pb] <= top)))
    counts = np.bincount(olen, minlength=256)  # ends claimed at each length (0: never)
    pruned = 0
    for l_hi in range(L - 1 - G, l_min - 1, -G):
        g = min(G, l_hi - l_min + 1)
        pruned += g * int(counts[l_hi + 1:].sum())
    return found, pruned
