// pack.cuh — a1 device helpers: stage a contiguous span of ASCII reads into shared memory
// (16-byte vector loads from HBM or, zero-copy, from page-locked host memory over PCIe) and
// pack one read into 2-bit words (encoding R1: (ascii >> 1) & 3; validation R13).
#pragma once

#include "kernels.cuh"

namespace lsg {

// Copy bytes [b0, b1) of `ascii` into smem so that smem offset = absolute address - sbase,
// sbase = (ascii + b0) & ~15.  Returns the smem offset of byte b0.  All `nthreads` threads of
// the block must call it; the caller synchronises afterwards.
__device__ __forceinline__ uint32_t stage_ascii(const unsigned char *ascii, uint64_t b0, uint64_t b1,
                                                unsigned char *sbuf, uint32_t nthreads)
{
    const uint64_t base = (uint64_t)(uintptr_t)ascii;
    const uint64_t sbase = (base + b0) & ~15ull;
    const uint64_t a0 = min64((base + b0 + 15) & ~15ull, base + b1), a1 = (base + b1) & ~15ull;
    if (a0 < a1) {
        const uint64_t nv = (a1 - a0) / 16;
        const uint4 *src = reinterpret_cast<const uint4 *>((uintptr_t)a0);
        for (uint64_t t = threadIdx.x; t < nv; t += nthreads)
            *reinterpret_cast<uint4 *>(sbuf + (a0 - sbase) + 16 * t) = src[t];
        for (uint64_t t = base + b0 + threadIdx.x; t < a0; t += nthreads)
            sbuf[t - sbase] = *reinterpret_cast<const unsigned char *>((uintptr_t)t);
        for (uint64_t t = a1 + threadIdx.x; t < base + b1; t += nthreads)
            sbuf[t - sbase] = *reinterpret_cast<const unsigned char *>((uintptr_t)t);
    } else {
        for (uint64_t t = base + b0 + threadIdx.x; t < base + b1; t += nthreads)
            sbuf[t - sbase] = *reinterpret_cast<const unsigned char *>((uintptr_t)t);
    }
    return (uint32_t)(base + b0 - sbase);
}

// pack one L-base ASCII row into `stride` words (unused bits 0); returns false on a byte
// outside ACGTacgt
__device__ __forceinline__ bool pack_row(const unsigned char *row, uint32_t L, uint32_t stride,
                                         uint64_t *out)
{
    bool bad = false;
    for (uint32_t w = 0; w < stride; ++w) {
        uint64_t word = 0;
        const uint32_t kend = min(L, 32u * (w + 1));
        for (uint32_t k = 32u * w; k < kend; ++k) {
            const unsigned ch = row[k];
            const unsigned lc = ch | 0x20u;
            bad |= !(lc == 'a' || lc == 'c' || lc == 'g' || lc == 't');
            word |= (uint64_t)((ch >> 1) & 3u) << (2 * (k & 31));
        }
        out[w] = word;
    }
    return !bad;
}

// the same into registers (W = ceil(L/32) words)
template <int W>
__device__ __forceinline__ bool pack_row_regs(const unsigned char *row, uint32_t L, uint64_t (&x)[W])
{
    bool bad = false;
#pragma unroll
    for (int w = 0; w < W; ++w) {
        uint64_t word = 0;
        const uint32_t kend = min(L, 32u * (w + 1));
        for (uint32_t k = 32u * w; k < kend; ++k) {
            const unsigned ch = row[k];
            const unsigned lc = ch | 0x20u;
            bad |= !(lc == 'a' || lc == 'c' || lc == 'g' || lc == 't');
            word |= (uint64_t)((ch >> 1) & 3u) << (2 * (k & 31));
        }
        x[w] = word;
    }
    return !bad;
}

// The same, four bases per step (SWAR), for a row in shared memory staged by stage_ascii with
// at least 8 readable bytes after the row end: each step funnel-shifts 4 bytes out of two
// aligned words; the codes are (byte >> 1) & 3 in every byte lane, and a byte is valid iff
// (byte | 0x20) equals the lowercase letter its own code names ("a", "c", "t", "g" for codes
// 0..3), looked up for all four lanes at once with one byte permute.
template <int W>
__device__ __forceinline__ bool pack_row_regs_swar(const unsigned char *row, uint32_t L,
                                                   uint64_t (&x)[W])
{
    const uint32_t *p = reinterpret_cast<const uint32_t *>((uintptr_t)row & ~(uintptr_t)3);
    const uint32_t sh = ((uint32_t)(uintptr_t)row & 3u) * 8u;
    uint32_t bad = 0, lo = p[0];
#pragma unroll
    for (int w = 0; w < W; ++w) x[w] = 0;
#pragma unroll
    for (int g = 0; g < 8 * W; ++g) {
        if (4u * g >= L) break;
        const uint32_t hi = p[g + 1];
        const uint32_t c4 = __funnelshift_r(lo, hi, sh); // bytes row[4g .. 4g+3]
        lo = hi;
        const uint32_t rem = L - 4u * g;                 // >= 1
        const uint32_t cx = (c4 >> 1) & 0x03030303u;     // codes, one per byte lane
        const uint32_t nib = cx | (cx >> 4);             // codes in nibbles 0, 1, 4, 5
        const uint32_t sel = (nib & 0xFFu) | ((nib >> 8) & 0xFF00u);
        const uint32_t expect = __byte_perm(0x67746361u, 0u, sel); // 'a' 'c' 't' 'g' by code
        const uint32_t t = cx | (cx >> 6);               // codes at bits 0-3 and 16-19
        uint32_t b8 = (t & 0xFu) | ((t >> 12) & 0xF0u);
        uint32_t diff = (c4 | 0x20202020u) ^ expect;
        if (rem < 4) {
            diff &= 0xFFFFFFFFu >> (8u * (4u - rem));
            b8 &= (1u << (2u * rem)) - 1u;
        }
        bad |= diff;
        x[g >> 3] |= (uint64_t)b8 << (8 * (g & 7));
    }
    return bad == 0;
}

} // namespace lsg
