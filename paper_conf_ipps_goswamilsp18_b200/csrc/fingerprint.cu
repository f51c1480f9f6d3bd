// fingerprint.cu — a2/a3: Rabin-Karp prefix/suffix fingerprints of every read and its
// reverse complement (Fig. 5/6) and the length-partitioned key tables.
//
// Thread per read, four rolling streams in ONE forward pass (no explicit RC in memory):
//   stream over r   (x_j = r_j):   pfx_l(r)  = Horner over x_0..x_{l-1}
//                                  sfx_l(r') = sum_{j<l} (x_j ^ 2) 5^j   (ascending powers)
//   stream over r'  (y_j = r'_j, r' = RC(r) reversed in registers):
//                                  pfx_l(r') = Horner over y_0..y_{l-1}
//                                  sfx_l(r)  = sum_{j<l} (y_j ^ 2) 5^j
// After base j all four values for length l = j+1 are available together, so the thread
// stores the pair (vertex 2i, vertex 2i+1) as one 16-byte word: a warp writes 512
// contiguous bytes per length (fully coalesced), unlike the paper's Hillis-Steele scan
// (one CTA per read) that was shaped for Kepler's shared memory.
#include "fingerprint.cuh"

namespace lsg {

// ---------------------------------------------------------------- API: raw fingerprints
template <int W>
__global__ void __launch_bounds__(256)
fp_values_kernel(const uint64_t *__restrict__ packed, uint64_t n, uint32_t L, uint32_t l_min,
                 uint32_t stride, uint64_t *__restrict__ pfx, uint64_t *__restrict__ sfx)
{
    const uint64_t V = 2 * n;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
         i += (uint64_t)gridDim.x * blockDim.x) {
        uint64_t x[W], y[W];
        load_read<W>(packed, stride, i, x);
        rc_words<W>(x, L, y);
        roll_read<W>(x, y, l_min, L, [&](uint32_t l, const FpStreams &st) {
            const uint64_t off = (uint64_t)(l - l_min) * V + 2 * i;
            if (pfx)
                *reinterpret_cast<ulonglong2 *>(pfx + off) =
                    make_ulonglong2(exact61(st.P0), exact61(st.P1));
            if (sfx)
                *reinterpret_cast<ulonglong2 *>(sfx + off) =
                    make_ulonglong2(exact61(st.S0), exact61(st.S1));
        });
    }
}

lasagna_status launch_fp_values(const uint64_t *packed, uint64_t n, uint32_t L, uint32_t l_min,
                                uint64_t *pfx, uint64_t *sfx, cudaStream_t s)
{
    if (n == 0) return LASAGNA_OK;
    const uint32_t stride = stride_for(L);
    return dispatch_W(L, [&](auto wc) -> lasagna_status {
        constexpr int W = decltype(wc)::value;
        uint64_t blocks = std::min<uint64_t>(ceil_div(n, 256), (uint64_t)num_sms() * 16);
        fp_values_kernel<W><<<(unsigned)blocks, 256, 0, s>>>(packed, n, L, l_min, stride, pfx, sfx);
        LSG_LAUNCHED("fp_values_kernel");
        return LASAGNA_OK;
    });
}

// ---------------------------------------------------------------- key tables (a2 + a3)
// For each length l in the group [l_lo, l_hi] (segment s = l - l_lo) and every vertex v the
// canonical entry (common.cuh): one list of V entries per length whose build side plays the
// paper's prefix list P_l and whose probe side plays its suffix list S_l:
//   tab[s*V + 2i]     = canon(pfx_l(r_i),  sfx_l(r_i'))  of vertex 2i
//   tab[s*V + 2i + 1] = canon(pfx_l(r_i'), sfx_l(r_i))   of vertex 2i+1
// (RC of the l-prefix of r is the l-suffix of r' and vice versa), i.e. 16 contiguous bytes per
// read per length, plus the histogram of the first LSD digit per segment (onesweep's upfront
// histogram), accumulated in shared memory and flushed once per CTA.
template <int W>
__global__ void __launch_bounds__(256)
table_kernel(TableArgs a)
{
    extern __shared__ uint32_t shist[]; // [G][256]
    const uint32_t G = a.l_hi - a.l_lo + 1;
    const bool with_hist = a.hist != nullptr;
    if (with_hist)
        for (uint32_t t = threadIdx.x; t < G * 256; t += blockDim.x) shist[t] = 0;
    __syncthreads();
    const uint64_t N = 2 * a.n; // V entries per length (of this read range)
    const uint64_t keep = key_keep(a.vbits);
    const uint32_t dmask = (1u << a.d_bits) - 1;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < a.n;
         i += (uint64_t)gridDim.x * blockDim.x) {
        uint64_t x[W], y[W];
        load_read<W>(a.packed, a.stride, i, x);
        rc_words<W>(x, a.L, y);
        roll_read<W>(x, y, a.l_lo, a.l_hi, [&](uint32_t l, const FpStreams &st) {
            const uint32_t s = l - a.l_lo;
            const uint64_t v0 = 2 * (a.read_offset + i); // global vertex ids
            const uint64_t e0 = canon_key(st.P0, st.S1, keep, a.vbits, v0);
            const uint64_t e1 = canon_key(st.P1, st.S0, keep, a.vbits, v0 + 1);
            *reinterpret_cast<ulonglong2 *>(a.tab + (uint64_t)s * N + 2 * i) = make_ulonglong2(e0, e1);
            if (with_hist) {
                uint32_t *h = shist + s * 256;
                atomicAdd(&h[(uint32_t)((e0 >> a.d_shift) & dmask)], 1u);
                atomicAdd(&h[(uint32_t)((e1 >> a.d_shift) & dmask)], 1u);
            }
        });
    }
    __syncthreads();
    if (with_hist)
        for (uint32_t t = threadIdx.x; t < G * 256; t += blockDim.x)
            if (shist[t]) atomicAdd(&a.hist[t], shist[t]);
}

lasagna_status launch_table(const TableArgs &args, cudaStream_t s)
{
    if (args.n == 0) return LASAGNA_OK;
    const uint32_t G = args.l_hi - args.l_lo + 1;
    const size_t smem = args.hist ? (size_t)G * 256 * sizeof(uint32_t) : 0;
    return dispatch_W(args.L, [&](auto wc) -> lasagna_status {
        constexpr int W = decltype(wc)::value;
        if (smem > 48 * 1024)
            LSG_CUDA(cudaFuncSetAttribute(table_kernel<W>,
                                          cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        int per_sm = 0;
        LSG_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, table_kernel<W>, 256, smem));
        if (per_sm < 1) per_sm = 1;
        uint64_t blocks = std::min<uint64_t>(ceil_div(args.n, 256), (uint64_t)num_sms() * per_sm);
        table_kernel<W><<<(unsigned)blocks, 256, smem, s>>>(args);
        LSG_LAUNCHED("table_kernel");
        return LASAGNA_OK;
    });
}

} // namespace lsg
