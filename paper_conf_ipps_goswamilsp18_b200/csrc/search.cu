// search.cu — a5: batched sorted-table lookup of suffix fingerprints + exact verification
// (Algorithm 2: lower bound L, upper bound U, count C = U - L of each suffix
// key in the sorted prefix list; an edge per match; R12 exact check).
//
// The table of one length is sorted by its top D key bits (a4), so the run of entries of
// directory bucket d = key >> (64-D) is [dir[d], dir[d+1]).  For a query q = sfx key of u:
//   L_u = dir[q >> (64-D)], U_u = dir[(q >> (64-D)) + 1]   (bucket bounds, ~4-8 entries)
// and within the bucket the entries whose stored key bits equal q's are the fingerprint
// matches (the lower/upper-bound interval of P:L164 restricted to equal keys).  Each match
// v from a different read with u < v^1 is verified on the 2-bit bases and emitted as the
// read-end pair (a = u, b = v^1): every pair exactly once (its twin has a > b).
#include "kernels.cuh"

namespace lsg {

// dir[d] = first index whose key has top-D bits >= d, d = 0..2^D (dir[2^D] = V)
__global__ void dir_kernel(const uint64_t *__restrict__ tab, uint64_t V, uint32_t D,
                           uint32_t *__restrict__ dir)
{
    const uint32_t s = blockIdx.y;
    const uint64_t nd = 1ull << D;
    const uint64_t *t = tab + (uint64_t)s * V;
    uint32_t *dr = dir + (uint64_t)s * (nd + 1);
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < V;
         i += (uint64_t)gridDim.x * blockDim.x) {
        const int64_t k = (int64_t)(t[i] >> (64 - D));
        const int64_t kp = i ? (int64_t)(t[i - 1] >> (64 - D)) : -1;
        for (int64_t d = kp + 1; d <= k; ++d) dr[d] = (uint32_t)i;
        if (i == V - 1)
            for (uint64_t d = (uint64_t)k + 1; d <= nd; ++d) dr[d] = (uint32_t)V;
    }
    if (V == 0 && blockIdx.x == 0)
        for (uint64_t d = threadIdx.x; d <= nd; d += blockDim.x) dr[d] = 0;
}

constexpr int SEARCH_THREADS = 256;
constexpr int SEARCH_BUF = 4096; // staged pairs per CTA


template <int W>
__global__ void __launch_bounds__(SEARCH_THREADS)
search_kernel(SearchArgs a)
{
    __shared__ unsigned long long buf[SEARCH_BUF];
    __shared__ uint32_t bcount;
    __shared__ unsigned long long gbase;
    if (threadIdx.x == 0) bcount = 0;
    __syncthreads();
    const uint64_t vmask = (1ull << a.vbits) - 1;
    const uint32_t dshift = 64 - a.D;
    unsigned long long nfalse = 0;
    for (uint64_t base = (uint64_t)blockIdx.x * SEARCH_THREADS; base < a.V;
         base += (uint64_t)gridDim.x * SEARCH_THREADS) {
        const uint64_t u = base + threadIdx.x;
        if (u < a.V && !(a.claimed && a.claimed[u])) {
            const uint64_t q = a.sfxk[u];
            const uint64_t d = q >> dshift;
            const uint32_t lo = a.dir[d], hi = a.dir[d + 1];
            for (uint32_t j = lo; j < hi; ++j) {
                const uint64_t e = a.tab[j];
                if ((e ^ q) > vmask) continue; // key bits differ
                const uint32_t v = (uint32_t)(e & vmask);
                const uint32_t b = v ^ 1u;
                if ((u >> 1) == (v >> 1) || u >= b) continue; // R9; emit each pair once
                if (a.claimed && a.claimed[b]) continue;
                if (!verify_overlap<W>(a.packed, a.stride, a.L, (uint32_t)u, v, a.l)) {
                    ++nfalse;
                    continue;
                }
                const unsigned long long rec = ((unsigned long long)u << 32) | b;
                uint32_t slot = atomicAdd(&bcount, 1u);
                if (slot < SEARCH_BUF) buf[slot] = rec;
                else {
                    unsigned long long gs = atomicAdd(a.count, 1ull);
                    if (gs < a.cap) a.pairs[gs] = rec;
                }
            }
        }
        __syncthreads();
        const uint32_t c = bcount;
        if (c >= SEARCH_BUF / 2) {
            const uint32_t m = min(c, (uint32_t)SEARCH_BUF);
            if (threadIdx.x == 0) gbase = atomicAdd(a.count, (unsigned long long)m);
            __syncthreads();
            for (uint32_t t = threadIdx.x; t < m; t += SEARCH_THREADS)
                if (gbase + t < a.cap) a.pairs[gbase + t] = buf[t];
            __syncthreads();
            if (threadIdx.x == 0) bcount = 0;
            __syncthreads();
        }
    }
    __syncthreads();
    const uint32_t m = min(bcount, (uint32_t)SEARCH_BUF);
    if (m) {
        if (threadIdx.x == 0) gbase = atomicAdd(a.count, (unsigned long long)m);
        __syncthreads();
        for (uint32_t t = threadIdx.x; t < m; t += SEARCH_THREADS)
            if (gbase + t < a.cap) a.pairs[gbase + t] = buf[t];
    }
    // false-match count: warp reduce then one atomic per warp
    for (int o = 16; o; o >>= 1) nfalse += __shfl_xor_sync(0xffffffffu, nfalse, o);
    if ((threadIdx.x & 31) == 0 && nfalse) atomicAdd(a.false_matches, nfalse);
}

lasagna_status launch_dir(const uint64_t *tab, uint64_t V, uint32_t n_seg, uint32_t D,
                          uint32_t *dir, cudaStream_t s)
{
    dim3 grid((unsigned)std::max<uint64_t>(1, std::min<uint64_t>(ceil_div(V, 256), 65535)), n_seg);
    dir_kernel<<<grid, 256, 0, s>>>(tab, V, D, dir);
    LSG_LAUNCHED("dir_kernel");
    return LASAGNA_OK;
}

lasagna_status launch_search(const SearchArgs &args, cudaStream_t s)
{
    if (args.V == 0) return LASAGNA_OK;
    return dispatch_W(args.L, [&](auto wc) -> lasagna_status {
        constexpr int W = decltype(wc)::value;
        int per_sm = 0;
        LSG_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, search_kernel<W>,
                                                               SEARCH_THREADS, 0));
        if (per_sm < 1) per_sm = 1;
        uint64_t blocks = std::min<uint64_t>(ceil_div(args.V, SEARCH_THREADS),
                                             (uint64_t)num_sms() * per_sm * 4);
        search_kernel<W><<<(unsigned)blocks, SEARCH_THREADS, 0, s>>>(args);
        LSG_LAUNCHED("search_kernel");
        return LASAGNA_OK;
    });
}

// pool record (a << 32 | b) -> compact sort key (a << vbits | b)
__global__ void pairs_to_keys(const unsigned long long *pool, const unsigned long long *count,
                              unsigned long long cap, uint32_t vbits, uint64_t *keys)
{
    const unsigned long long m = min(*count, cap);
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m;
         i += (uint64_t)gridDim.x * blockDim.x) {
        unsigned long long r = pool[i];
        keys[i] = ((r >> 32) << vbits) | (r & 0xFFFFFFFFull);
    }
}

// sorted compact keys -> (pair_a, pair_b, pair_l) at output offset
__global__ void keys_to_output(const uint64_t *keys, uint64_t m, uint32_t vbits, uint8_t l,
                               uint32_t *pa, uint32_t *pb, uint8_t *pl)
{
    const uint64_t vmask = (1ull << vbits) - 1;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m;
         i += (uint64_t)gridDim.x * blockDim.x) {
        uint64_t k = keys[i];
        if (pa) pa[i] = (uint32_t)(k >> vbits);
        if (pb) pb[i] = (uint32_t)(k & vmask);
        if (pl) pl[i] = l;
    }
}

lasagna_status launch_pairs_to_keys(const unsigned long long *pool, const unsigned long long *count,
                                    uint64_t m, unsigned long long cap, uint32_t vbits,
                                    uint64_t *keys, cudaStream_t s)
{
    if (m == 0) return LASAGNA_OK;
    pairs_to_keys<<<(unsigned)std::min<uint64_t>(ceil_div(m, 256), 4096), 256, 0, s>>>(
        pool, count, cap, vbits, keys);
    LSG_LAUNCHED("pairs_to_keys");
    return LASAGNA_OK;
}

lasagna_status launch_keys_to_output(const uint64_t *keys, uint64_t m, uint32_t vbits, uint8_t l,
                                     uint32_t *pa, uint32_t *pb, uint8_t *pl, cudaStream_t s)
{
    if (m == 0) return LASAGNA_OK;
    keys_to_output<<<(unsigned)std::min<uint64_t>(ceil_div(m, 256), 4096), 256, 0, s>>>(
        keys, m, vbits, l, pa, pb, pl);
    LSG_LAUNCHED("keys_to_output");
    return LASAGNA_OK;
}

} // namespace lsg
