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

} // namespace lsg
