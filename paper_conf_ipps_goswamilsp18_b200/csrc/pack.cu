// pack.cu — a1: stage + 2-bit pack ("batches of reads are loaded in the GPU";
// two-level streaming model P:L61-67; encoding R1 = Fig. 5's A0 C1 T2 G3).
//
// One CTA stages READS_PER_CTA consecutive reads: their n*L-byte ASCII span is contiguous,
// so the CTA copies it into shared memory with 16-byte vector loads (from HBM, or straight
// from page-locked host memory over PCIe: zero-copy staging), validates every byte, and
// each thread packs one read (32 bases per u64, base 0 in the low bits).
#include "pack.cuh"

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
    const uint32_t off = stage_ascii(ascii, r0 * L, r1 * L, sbuf, PACK_THREADS);
    __syncthreads();
    const uint64_t i = r0 + threadIdx.x;
    if (i >= r1) return;
    const bool ok = pack_row(sbuf + off + (uint64_t)threadIdx.x * L, L, stride, packed + i * stride);
    if (!ok && first_bad) atomicMin(first_bad, (unsigned long long)i);
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
