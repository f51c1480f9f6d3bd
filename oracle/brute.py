"""Pure-Python brute force for tiny inputs — TEST INFRASTRUCTURE ONLY.

Cross-checks oracle.c: every ordered pair of oriented reads at every
length, compared character by character, straight from the string-graph definition
 with the length range of P:L105 and readings R5, R7-R10.  It shares no
code with oracle.c (own complement table, own loops) and none with the CUDA path.
"""
from __future__ import annotations

_COMP = {"A": "T", "C": "G", "G": "C", "T": "A"}


def oriented_reads(reads: list[str]) -> list[str]:
    """seq(2i) = r_i, seq(2i+1) = WC complement of r_i (reading R8)."""
    out = []
    for r in reads:
        r = r.upper()
        out.append(r)
        out.append("".join(_COMP[c] for c in reversed(r)))
    return out


def directed_overlaps(reads: list[str], l_min: int) -> set[tuple[int, int, int]]:
    """O = {(u, v, l)}: l-suffix of seq(u) == l-prefix of seq(v), l in [l_min, L-1],
    u and v from different reads (reading R9)."""
    seq = oriented_reads(reads)
    L = len(seq[0])
    out = set()
    for u in range(len(seq)):
        for v in range(len(seq)):
            if u // 2 == v // 2:
                continue
            for l in range(l_min, L):
                if all(seq[u][L - l + k] == seq[v][k] for k in range(l)):
                    out.add((u, v, l))
    return out


def pairs(reads: list[str], l_min: int) -> list[tuple[int, int, int]]:
    """P = [(l, a, b)] with a = u, b = v^1, a < b; sorted by (l desc, a, b) (reading R7)."""
    O = directed_overlaps(reads, l_min)
    P = {(l, u, v ^ 1) for (u, v, l) in O if u < (v ^ 1)}
    return sorted(P, key=lambda t: (-t[0], t[1], t[2]))


def greedy(n_reads: int, P: list[tuple[int, int, int]]):
    """Sequential greedy: accept in order iff neither read end has an edge."""
    V = 2 * n_reads
    succ = [0xFFFFFFFF] * V
    olen = [0] * V
    used = [False] * V
    for (l, a, b) in P:
        if used[a] or used[b]:
            continue
        used[a] = used[b] = True
        succ[a] = b ^ 1
        succ[b] = a ^ 1
        olen[a] = olen[b] = l
    return succ, olen


def contigs(reads: list[str], succ: list[int], olen: list[int]) -> list[tuple[int, str]]:
    """Compress straight from the text: seeds have in-degree 0 and out-degree 1;
    a path follows succ to a vertex without an out-edge; each read contributes its first
    overhang bases (L - olen, or L for the last); a path and its complementary path spell
    reverse-complementary contigs, the one with the smaller seed is kept (R20).  Returns
    [(seed, contig)] in seed order."""
    seq = oriented_reads(reads)
    L = len(seq[0])
    V = len(seq)
    has_in = [False] * V
    for u in range(V):
        if succ[u] != 0xFFFFFFFF:
            has_in[succ[u]] = True
    out = []
    for s in range(V):
        if has_in[s] or succ[s] == 0xFFFFFFFF:
            continue
        path = [s]
        while succ[path[-1]] != 0xFFFFFFFF:
            path.append(succ[path[-1]])
        if not s < (path[-1] ^ 1):
            continue
        text = "".join(seq[v][: L - olen[v]] for v in path[:-1]) + seq[path[-1]]
        out.append((s, text))
    return out
