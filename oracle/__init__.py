"""CPU oracle for the LaSAGNA hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_ipps_goswamilsp18_b200``) never imports it, and the two share no code:
the only common dependency is the seeded input generator ``readgen``.

* ``oracle.c`` — plain C (gcc), fp64-free integer definitions, each function citing its
  PAPER.md passage.  Loaded here through ctypes.
* ``brute.py`` — pure-Python brute force for tiny inputs (cross-checks ``oracle.c``).

Pins: see the header of oracle.c.  Parity of the tie-break / self-overlap conventions
(readings R7-R9) is pinned only by the written definition implemented twice (brute.py and
oracle.c): "parity unpinned by the paper" for those conventions.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_SO = os.path.join(_HERE, "liboracle.so")

NONE = 0xFFFFFFFF
#: production fingerprint parameters (reading R4): radix 5, Mersenne prime 2^61 - 1
SIGMA = 5
Q = (1 << 61) - 1

_u64p = ctypes.POINTER(ctypes.c_uint64)


def build() -> str:
    subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-o", _SO, _SRC])
    return _SO


_lib = None


def lib():
    global _lib
    if _lib is None:
        if (not os.path.exists(_SO)) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
            build()
        L = ctypes.CDLL(_SO)
        vp, u64, u32, i32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
        L.oracle_code.argtypes = [i32]
        L.oracle_code.restype = i32
        L.oracle_place_values.argtypes = [u64, u64, i32, vp]
        L.oracle_F.argtypes = [vp, i32, u64, u64]
        L.oracle_F.restype = u64
        L.oracle_scan_prefix.argtypes = [vp, i32, u64, u64, vp]
        L.oracle_suffix_from_prefix.argtypes = [vp, i32, u64, u64, vp, vp]
        L.oracle_first_bad.argtypes = [vp, u64, u32]
        L.oracle_first_bad.restype = u64
        L.oracle_fingerprints.argtypes = [vp, u64, u32, u32, u64, u64, vp, vp]
        L.oracle_pack.argtypes = [vp, u64, u32, u32, vp]
        L.oracle_overlaps.argtypes = [vp, u64, u32, u32, u64, vp, vp, vp]
        L.oracle_overlaps.restype = u64
        L.oracle_overlaps_approx.argtypes = [vp, u64, u32, u32, u64, u64, u64, u64, u64, vp, vp, vp]
        L.oracle_overlaps_approx.restype = u64
        L.oracle_greedy.argtypes = [u64, u64, vp, vp, vp, vp, vp]
        L.oracle_greedy.restype = u64
        L.oracle_greedy_graph.argtypes = [vp, u64, u32, u32, vp, vp, vp]
        L.oracle_greedy_graph.restype = u64
        L.oracle_compress.argtypes = [vp, u64, u32, vp, vp, vp, vp, vp, vp]
        L.oracle_compress.restype = u64
        _lib = L
    return _lib


def _ascii(reads) -> np.ndarray:
    a = np.ascontiguousarray(reads)
    if a.dtype != np.uint8:
        raise TypeError("reads must be a uint8 (n, L) ASCII array")
    if a.ndim != 2:
        raise ValueError("reads must be 2-D (n, L)")
    return a


def code(ch: str) -> int:
    return lib().oracle_code(ord(ch))


def codes(s: str) -> np.ndarray:
    return np.array([code(c) for c in s], dtype=np.uint8)


def place_values(sigma: int, q: int, m: int) -> np.ndarray:
    M = np.empty(m + 1, dtype=np.uint64)
    lib().oracle_place_values(sigma, q, m, M.ctypes.data)
    return M


def F(s: str | np.ndarray, sigma: int = SIGMA, q: int = Q) -> int:
    c = codes(s) if isinstance(s, str) else np.ascontiguousarray(s, dtype=np.uint8)
    return int(lib().oracle_F(c.ctypes.data, len(c), sigma, q))


def scan_prefix(s: str, sigma: int, q: int) -> np.ndarray:
    E = codes(s)
    P = np.empty(len(E), dtype=np.uint64)
    lib().oracle_scan_prefix(E.ctypes.data, len(E), sigma, q, P.ctypes.data)
    return P


def suffix_from_prefix(P: np.ndarray, sigma: int, q: int):
    P = np.ascontiguousarray(P, dtype=np.uint64)
    S = np.empty(len(P), dtype=np.uint64)
    Pp = np.empty(len(P), dtype=np.uint64)
    lib().oracle_suffix_from_prefix(P.ctypes.data, len(P), sigma, q, S.ctypes.data,
                                    Pp.ctypes.data)
    return S, Pp


def first_bad(reads) -> int:
    a = _ascii(reads)
    r = int(lib().oracle_first_bad(a.ctypes.data, a.shape[0], a.shape[1]))
    return -1 if r == 0xFFFFFFFFFFFFFFFF else r


def fingerprints(reads, l_min: int, sigma: int = SIGMA, q: int = Q):
    """(pfx, sfx), each uint64 [L - l_min + 1, 2n] (row k = length l_min + k)."""
    a = _ascii(reads)
    n, L = a.shape
    pfx = np.empty((L - l_min + 1, 2 * n), dtype=np.uint64)
    sfx = np.empty_like(pfx)
    lib().oracle_fingerprints(a.ctypes.data, n, L, l_min, sigma, q, pfx.ctypes.data,
                              sfx.ctypes.data)
    return pfx, sfx


def pack(reads, stride: int) -> np.ndarray:
    a = _ascii(reads)
    n, L = a.shape
    out = np.empty((n, stride), dtype=np.uint64)
    lib().oracle_pack(a.ctypes.data, n, L, stride, out.ctypes.data)
    return out


def overlaps(reads, l_min: int):
    """Read-end pair list P sorted by (l desc, a, b): (l uint8[], a uint32[], b uint32[])."""
    a = _ascii(reads)
    n, L = a.shape
    m = int(lib().oracle_overlaps(a.ctypes.data, n, L, l_min, 0, None, None, None))
    if m == 0xFFFFFFFFFFFFFFFF:
        raise ValueError("oracle: invalid reads or parameters")
    pl = np.empty(m, dtype=np.uint8)
    pa = np.empty(m, dtype=np.uint32)
    pb = np.empty(m, dtype=np.uint32)
    lib().oracle_overlaps(a.ctypes.data, n, L, l_min, m, pl.ctypes.data, pa.ctypes.data,
                          pb.ctypes.data)
    return pl, pa, pb


SIGMA2 = 7                   # the approximate mode's second fingerprint: radix 7,
Q2 = (1 << 64) - 59          # the largest prime below 2^64 (reading R22)


def overlaps_approx(reads, l_min: int, sigma2: int = SIGMA2, q2: int = Q2, sigma1: int = SIGMA,
                    q1: int = Q):
    """Approximate mode: pairs whose (F(sigma1, q1), F(sigma2, q2)) fingerprints of
    suffix and prefix agree, by Algorithm 2 on the P_l / S_l lists; (l, a, b) as overlaps()."""
    a = _ascii(reads)
    n, L = a.shape
    args = (a.ctypes.data, n, L, l_min, sigma1, q1, sigma2, q2)
    m = int(lib().oracle_overlaps_approx(*args, 0, None, None, None))
    if m == 0xFFFFFFFFFFFFFFFF:
        raise ValueError("oracle: invalid reads or parameters")
    pl = np.empty(m, dtype=np.uint8)
    pa = np.empty(m, dtype=np.uint32)
    pb = np.empty(m, dtype=np.uint32)
    lib().oracle_overlaps_approx(*args, m, pl.ctypes.data, pa.ctypes.data, pb.ctypes.data)
    return pl, pa, pb


def greedy(n: int, pl, pa, pb):
    pl = np.ascontiguousarray(pl, dtype=np.uint8)
    pa = np.ascontiguousarray(pa, dtype=np.uint32)
    pb = np.ascontiguousarray(pb, dtype=np.uint32)
    succ = np.empty(2 * n, dtype=np.uint32)
    olen = np.empty(2 * n, dtype=np.uint8)
    g = lib().oracle_greedy(n, len(pl), pl.ctypes.data, pa.ctypes.data, pb.ctypes.data,
                            succ.ctypes.data, olen.ctypes.data)
    return succ, olen, int(g)


def greedy_graph(reads, l_min: int):
    """(succ uint32[2n], olen uint8[2n], |P|, accepted pairs)."""
    a = _ascii(reads)
    n, L = a.shape
    succ = np.empty(2 * n, dtype=np.uint32)
    olen = np.empty(2 * n, dtype=np.uint8)
    ng = ctypes.c_uint64(0)
    m = int(lib().oracle_greedy_graph(a.ctypes.data, n, L, l_min, succ.ctypes.data,
                                      olen.ctypes.data, ctypes.byref(ng)))
    if m == 0xFFFFFFFFFFFFFFFF:
        raise ValueError("oracle: invalid reads or parameters")
    return succ, olen, m, int(ng.value)


def compress(reads, succ, olen):
    """Contigs of the greedy graph: (contigs bytes, offsets uint64[c+1],
    seeds uint32[c]); contig k = contigs[offsets[k]:offsets[k+1]]."""
    a = _ascii(reads)
    n, L = a.shape
    succ = np.ascontiguousarray(succ, dtype=np.uint32)
    olen = np.ascontiguousarray(olen, dtype=np.uint8)
    nc = ctypes.c_uint64(0)
    tot = int(lib().oracle_compress(a.ctypes.data, n, L, succ.ctypes.data, olen.ctypes.data,
                                    None, None, None, ctypes.byref(nc)))
    c = int(nc.value)
    buf = ctypes.create_string_buffer(max(1, tot))
    offs = np.empty(c + 1, dtype=np.uint64)
    seeds = np.empty(max(1, c), dtype=np.uint32)
    lib().oracle_compress(a.ctypes.data, n, L, succ.ctypes.data, olen.ctypes.data, buf,
                          offs.ctypes.data, seeds.ctypes.data, ctypes.byref(nc))
    return buf.raw[:tot], offs, seeds[:c]
