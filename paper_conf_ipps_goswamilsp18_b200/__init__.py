"""B200-native LaSAGNA hot path: all-pair suffix-prefix overlaps and the greedy string graph.

The compute path is liblasagna.so (hand-written sm_100a CUDA kernels behind the C ABI of
include/lasagna.h); this package is its thin Python binding plus the multi-GPU driver.
There is no CPU fallback.
"""
from .lasagna import (  # noqa: F401
    NONE, Contigs, GraphPipeline, GraphResult, GreedyGraph, LasagnaError, compress, fingerprints,
    greedy_graph, greedy_pairs, kernel_launches, lib, load_reads, overlaps, plan, sort_u64,
    words_per_read,
)

__all__ = ["NONE", "Contigs", "GraphPipeline", "GraphResult", "GreedyGraph", "LasagnaError",
           "compress", "fingerprints", "greedy_graph", "greedy_pairs", "kernel_launches", "lib",
           "load_reads", "overlaps", "plan", "sort_u64", "words_per_read"]
