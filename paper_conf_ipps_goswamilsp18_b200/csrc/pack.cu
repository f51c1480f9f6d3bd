// pack.cu — a1: stage + 2-bit pack ("batches of reads are loaded in the GPU";
// two-level streaming model P:L61-67; encoding R1 = Fig. 5's A0 C1 T2 G3).
//
// One CTA stages READS_PER_CTA consecutive reads: their n*L-byte ASCII span is contiguous,
// so the CTA copies it into shared memory with 16-byte vector loads (from HBM, or straight
// from page-locked host memory over PCIe: zero-copy staging), validates every byte, and
// each thread packs one read (32 bases per u64, base 0 in the low bits).
#include "kernels.cuh"

namespace lsg {

constexpr int PACK_THREADS = 128;
constexpr int READS_PER_CTA = 128;

__global__ void __launch_bounds__(PACK_THREADS)
pack_kernel(const unsigned char *__restrict__ ascii, uint64_t n, uint32_t L, uint32_t stride,
            uint64_t *__restrict__ packed, unsigned long long *__restrict__ first_bad)
{
    extern __shared__ __align__(16) unsigned char sbuf[];
    const uint64_t r0 = (uint64_t)blockIdx.x * READS_PER_CTA;
    if (r0 >= n) return;
    const uint64_t r1 = min64(n, r0 + READS_PER_CTA);
    const uint64_t b0 = r0 * L, b1 = r1 * L; // byte span [b0, b1)
    // Shared-memory image of the span, laid out so that smem offset = absolute address - sbase
    // with sbase 16-byte aligned: the aligned interior moves with 16 B vector loads/stores
    // (from HBM, or straight from page-locked host memory), the ragged ends byte by byte.
    const uint64_t base = (uint64_t)(uintptr_t)ascii;
    const uint64_t sbase = (base + b0) & ~15ull;
    const uint64_t a0 = min64((base + b0 + 15) & ~15ull, base + b1), a1 = (base + b1) & ~15ull;
    if (a0 < a1) {
        const uint64_t nv = (a1 - a0) / 16;
        const uint4 *src = reinterpret_cast<const uint4 *>((uintptr_t)a0);
        for (uint64_t t = threadIdx.x; t < nv; t += PACK_THREADS)
            *reinterpret_cast<uint4 *>(sbuf + (a0 - sbase) + 16 * t) = src[t];
        for (uint64_t t = base + b0 + threadIdx.x; t < a0; t += PACK_THREADS)
            sbuf[t - sbase] = *reinterpret_cast<const unsigned char *>((uintptr_t)t);
        for (uint64_t t = a1 + threadIdx.x; t < base + b1; t += PACK_THREADS)
            sbuf[t - sbase] = *reinterpret_cast<const unsigned char *>((uintptr_t)t);
    } else {
        for (uint64_t t = base + b0 + threadIdx.x; t < base + b1; t += PACK_THREADS)
            sbuf[t - sbase] = *reinterpret_cast<const unsigned char *>((uintptr_t)t);
    }
    __syncthreads();

    const uint64_t i = r0 + threadIdx.x;
    if (i >= r1) return;
    const unsigned char *row = sbuf + (base + b0 - sbase) + (uint64_t)threadIdx.x * L;
    bool bad = false;
    uint64_t *out = packed + i * stride;
    for (uint32_t w = 0; w < stride; ++w) {
        uint64_t word = 0;
        uint32_t kend = min(L, 32u * (w + 1));
        for (uint32_t k = 32u * w; k < kend; ++k) {
            unsigned ch = row[k];
            unsigned lc = ch | 0x20u;
            bad |= !(lc == 'a' || lc == 'c' || lc == 'g' || lc == 't');
            word |= (uint64_t)((ch >> 1) & 3u) << (2 * (k & 31));
        }
        out[w] = word;
    }
    if (bad && first_bad) atomicMin(first_bad, (unsigned long long)i);
}

__global__ void set_u64(unsigned long long *p, unsigned long long v) { *p = v; }

lasagna_status launch_pack(const char *ascii, uint64_t n, uint32_t L, uint64_t *packed,
                           uint64_t *first_bad, cudaStream_t s)
{
    const uint32_t stride = stride_for(L);
    if (first_bad) {
        set_u64<<<1, 1, 0, s>>>(reinterpret_cast<unsigned long long *>(first_bad), ~0ull);
        LSG_LAUNCHED("set_u64");
    }
    if (n == 0) return LASAGNA_OK;
    const size_t smem = (size_t)READS_PER_CTA * L + 16;
    if (smem > 48 * 1024)
        LSG_CUDA(cudaFuncSetAttribute(pack_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      (int)smem));
    const uint64_t blocks = ceil_div(n, READS_PER_CTA);
    pack_kernel<<<(unsigned)blocks, PACK_THREADS, smem, s>>>(
        reinterpret_cast<const unsigned char *>(ascii), n, L, stride, packed,
        reinterpret_cast<unsigned long long *>(first_bad));
    LSG_LAUNCHED("pack_kernel");
    return LASAGNA_OK;
}

} // namespace lsg
