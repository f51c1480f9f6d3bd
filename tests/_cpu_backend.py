"""CPU stand-in for the sharded phase calls of the multi-GPU driver — TEST ONLY.

Lets tests drive paper_conf_ipps_goswamilsp18_b200.dist's exchange logic (hash-range
partition, all-to-all split sizes, pair all-gather, replicated greedy) over the gloo backend
on CPU.  The key layout mirrors include/lasagna.h's description; fingerprints, string checks
and the greedy come from the oracle.
"""
from __future__ import annotations

import math

import numpy as np
import torch

import oracle

MIX = np.uint64(0x9E3779B97F4A7C15)


class CpuBackend:
    def __init__(self, reads_all: np.ndarray):
        self.reads = reads_all  # (n_total, L) ASCII, the whole read set

    def pack(self, ascii_local):
        a = ascii_local.numpy() if isinstance(ascii_local, torch.Tensor) else ascii_local
        L = a.shape[1] if a.ndim == 2 else 1
        w = (L + 31) // 32
        stride = 1 if w <= 1 else 2 if w <= 2 else 4 if w <= 4 else 8
        return torch.from_numpy(oracle.pack(a, stride).view(np.int64).copy())

    def vertex_bits(self, n_total):
        return max(1, math.ceil(math.log2(2 * n_total))) if n_total > 0 else 1

    def sort_bits(self, n_total):
        vb = self.vertex_bits(n_total)
        N = 2 * n_total  # one canonical entry per vertex and length
        P = math.ceil((math.log2(N) - 11.5) / 8) if N > 1 else 1
        return min(8 * max(1, min(P, 4)), 62 - vb)

    def table_keys(self, packed_local, n_local, read_offset, n_total, L, l_lo, l_hi):
        """Canonical entries (include/lasagna.h): per vertex v and length l, with
        H = F(prefix_l(v)) and Hr = F(RC(prefix_l(v))) = F(suffix_l(v ^ 1)):
        key = mix(min(H, Hr)) top bits | flag << vbits | v, flag 0 (H < Hr) / 1 (>) / 2 (=)."""
        vb = self.vertex_bits(n_total)
        keep = np.uint64(~((4 << vb) - 1) & 0xFFFFFFFFFFFFFFFF)
        G = l_hi - l_lo + 1
        out = np.zeros((G, 2 * n_local), dtype=np.uint64)
        if n_local:
            pfx, sfx = oracle.fingerprints(self.reads[read_offset:read_offset + n_local], l_lo)
            v = (2 * (read_offset + np.arange(n_local, dtype=np.uint64)))
            for s in range(G):
                for o in (0, 1):
                    H = pfx[s, o::2]
                    Hr = sfx[s, (o ^ 1)::2]  # RC of the prefix of r (r') is the suffix of r' (r)
                    c = np.minimum(H, Hr)
                    f = np.where(H < Hr, 0, np.where(H > Hr, 1, 2)).astype(np.uint64)
                    out[s, o::2] = ((c * MIX) & keep) | (f << np.uint64(vb)) | (v + np.uint64(o))
        return torch.from_numpy(out.view(np.int64))

    def sort_segments(self, keys, seg_len, n_seg, lo, hi):
        k = keys.numpy().view(np.uint64).reshape(n_seg, seg_len) if seg_len else None
        if k is None:
            return keys
        mask = np.uint64((1 << (hi - lo)) - 1 if hi - lo < 64 else 0xFFFFFFFFFFFFFFFF)
        for s in range(n_seg):
            d = (k[s] >> np.uint64(lo)) & mask
            k[s] = k[s][np.argsort(d, kind="stable")]
        return keys

    def digit_counts(self, keys, seg_len, n_seg, shift, bits):
        k = keys.numpy().view(np.uint64).reshape(n_seg, seg_len)
        out = np.zeros((n_seg, 1 << bits), dtype=np.int64)
        for s in range(n_seg):
            d = ((k[s] >> np.uint64(shift)) & np.uint64((1 << bits) - 1)).astype(np.int64)
            out[s] = np.bincount(d, minlength=1 << bits)
        return torch.from_numpy(out)

    def new_pairs(self, capacity):
        return torch.zeros(max(1, capacity), dtype=torch.int64), torch.zeros(2, dtype=torch.int64)

    def join(self, keys, count, packed_all, n_total, L, l, pairs, counters):
        """Build side: flags 0/2; probe side: flags 1/2; a match (probe w, build v) is the
        read-end pair {w^1, v^1} if suffix_l(seq(w^1)) == prefix_l(seq(v))."""
        vb = self.vertex_bits(n_total)
        k = keys.numpy().view(np.uint64)[:count]
        kb = (k >> np.uint64(vb + 2)).tolist()
        flag = ((k >> np.uint64(vb)) & np.uint64(3)).tolist()
        vid = (k & np.uint64((1 << vb) - 1)).astype(np.int64).tolist()
        byk: dict[int, list[tuple[int, int]]] = {}
        for key, f, v in zip(kb, flag, vid):
            if f != 1:
                byk.setdefault(key, []).append((v, f))
        comp = bytes.maketrans(b"ACGT", b"TGCA")

        def seq(v):
            r = bytes(self.reads[v >> 1])
            return r[::-1].translate(comp) if v & 1 else r
        pos = int(counters[0])
        nf = 0
        for key, fw, w in zip(kb, flag, vid):
            if fw == 0:
                continue
            for v, fv in byk.get(key, []):
                if (w >> 1) == (v >> 1) or (fw == 2 and fv == 2 and w > v):
                    continue
                a, b = sorted((w ^ 1, v ^ 1))
                if seq(w ^ 1)[L - l:] != seq(v)[:l]:
                    nf += 1
                    continue
                if pos < pairs.numel():
                    pairs[pos] = (a << 32) | b
                pos += 1
        counters[0] = pos
        counters[1] += nf

    def greedy_pairs(self, n_total, pl, pa, pb):
        pl = pl.numpy().astype(np.int64)
        pa = pa.numpy().view(np.uint32).astype(np.int64)
        pb = pb.numpy().view(np.uint32).astype(np.int64)
        order = np.lexsort((pb, pa, -pl))
        succ, olen, _ = oracle.greedy(n_total, pl[order], pa[order], pb[order])
        return torch.from_numpy(succ.view(np.int32).copy()), torch.from_numpy(olen.copy())
