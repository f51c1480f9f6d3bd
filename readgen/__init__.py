"""Seeded synthetic read generator (shared input infrastructure).

Both the CUDA path's tests/bench and the CPU oracle draw their inputs from here.
This module holds none of the method's arithmetic: it only produces ASCII reads
(recipe in readgen.c and DESIGN.md "Input recipe"; configs from BASELINE.json
``configs`` with the sizes fixed in SURVEY §8(d)).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "readgen.c")
_SO = os.path.join(_HERE, "libreadgen.so")


@dataclass(frozen=True)
class ReadConfig:
    name: str
    G: int          # genome length
    n: int          # number of reads
    L: int          # read length
    l_min: int      # minimum overlap length
    p_err: float    # substitution rate
    seed: int = 20181
    note: str = ""


# BASELINE.json configs[0..4]; l_min per P:L218 (63 for 100/101 bp, 111 for 150 bp).
CONFIGS = {
    "cfg1": ReadConfig("cfg1", 200_000, 20_000, 100, 63, 0.0,
                       note="200 kbp random genome, 20k error-free 100 bp reads (10x)"),
    "cfg2": ReadConfig("cfg2", 4_600_000, 2_300_000, 100, 63, 0.01,
                       note="E. coli-sized 4.6 Mbp genome, 50x 100 bp reads, 1% substitutions"),
    "cfg3": ReadConfig("cfg3", 88_000_000, 34_851_485, 101, 63, 0.01,
                       note="chr14-sized 88 Mbp genome, 40x 101 bp reads, 1% substitutions"),
    "cfg4": ReadConfig("cfg4", 3_000_000_000, 1_200_000_000, 150, 111, 0.01,
                       note="3 Gbp genome, 1.2B 150 bp reads (60x)"),
    "cfg5": ReadConfig("cfg5", 3_000_000_000, 1_247_518_392, 100, 63, 0.01,
                       note="3 Gbp genome, H.Genome read count (41.6x), semi-streamed"),
}


def _build() -> None:
    cmd = ["gcc", "-O3", "-fopenmp", "-fPIC", "-shared", "-o", _SO, _SRC]
    subprocess.check_call(cmd)


_lib = None


def lib():
    global _lib
    if _lib is None:
        if (not os.path.exists(_SO)) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
            _build()
        L = ctypes.CDLL(_SO)
        L.readgen_genome.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p]
        L.readgen_genome.restype = None
        L.readgen_reads.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint32,
                                    ctypes.c_double, ctypes.c_uint64, ctypes.c_uint64,
                                    ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
        L.readgen_reads.restype = ctypes.c_int
        L.readgen_starts.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint32,
                                     ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p]
        L.readgen_starts.restype = ctypes.c_int
        _lib = L
    return _lib


def genome(seed: int, G: int) -> np.ndarray:
    out = np.empty(G, dtype=np.uint8)
    lib().readgen_genome(seed, G, out.ctypes.data)
    return out


def reads_into(ptr: int, seed: int, G: int, L: int, p_err: float, i0: int, i1: int,
               starts_ptr: int = 0, strands_ptr: int = 0) -> None:
    """Write reads [i0, i1) as ASCII rows of L bytes to the host address ``ptr``."""
    rc = lib().readgen_reads(seed, G, L, p_err, i0, i1, ptr, starts_ptr or None,
                             strands_ptr or None)
    if rc != 0:
        raise ValueError("readgen: invalid parameters")


def reads(seed: int, G: int, n: int, L: int, p_err: float, i0: int = 0,
          with_truth: bool = False):
    """Reads [i0, i0+n) as an (n, L) uint8 ASCII array (optionally with start/strand)."""
    out = np.empty((n, L), dtype=np.uint8)
    starts = np.empty(n, dtype=np.uint64) if with_truth else None
    strands = np.empty(n, dtype=np.uint8) if with_truth else None
    reads_into(out.ctypes.data, seed, G, L, p_err, i0, i0 + n,
               starts.ctypes.data if with_truth else 0,
               strands.ctypes.data if with_truth else 0)
    if with_truth:
        return out, starts, strands
    return out


def config_reads(cfg: ReadConfig | str, n: int | None = None, seed: int | None = None):
    """The first ``n`` reads (default: all) of a named config."""
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg]
    return reads(cfg.seed if seed is None else seed, cfg.G, cfg.n if n is None else n,
                 cfg.L, cfg.p_err)


def starts(seed: int, G: int, L: int, i0: int, i1: int) -> np.ndarray:
    """Start positions of reads [i0, i1) (uint64), without generating their bases."""
    out = np.empty(i1 - i0, dtype=np.uint64)
    if lib().readgen_starts(seed, G, L, i0, i1, out.ctypes.data) != 0:
        raise ValueError("readgen: invalid parameters")
    return out


def window_sample(cfg: ReadConfig | str, n_target: int) -> np.ndarray:
    """Indices of the reads of a config that start in the genome window [0, f (G - L + 1)),
    f = n_target / n: a sample of the SAME read set at the same coverage and error rate
    (a prefix of the read list would have ~f times the coverage instead)."""
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg]
    st = starts(cfg.seed, cfg.G, cfg.L, 0, cfg.n)
    lim = int(min(1.0, n_target / cfg.n) * (cfg.G - cfg.L + 1))
    return np.nonzero(st < lim)[0]
