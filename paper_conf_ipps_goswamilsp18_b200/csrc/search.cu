// search.cu — a5: batched sorted-table lookup of suffix fingerprints against prefix
// fingerprints + exact verification (Algorithm 2; R12).
//
// Per length l the table holds BOTH lists of the paper — the prefix list P_l (tag 0) and
// the suffix list S_l (tag 1) — as one array of 2V keys
//     key = mix(F) top bits | tag << vbits | vertex id,
// radix-sorted by the top T key bits (a4).  After the sort, equal fingerprints sit in the
// same T-bit bucket, so Algorithm 2's windows W_S / W_P "such that a fingerprint present in
// W_S cannot be present in any window except W_P" are exactly runs of whole
// buckets.  Each CTA owns the buckets that START inside its chunk of the sorted array,
// stages their entries in shared memory, builds a small hash table over the prefix entries
// and looks every suffix entry up in it (the vectorised lower/upper bound of P:L164-166,
// done as a shared-memory probe: all matches of a key are found, C = U - L of them).
// Each fingerprint match v of a suffix u from a different read with u < v^1 is verified
// on the 2-bit bases and emitted as the read-end pair (a = u, b = v^1), so every pair is
// emitted exactly once (its twin has a > b).
//
// Traffic: the sorted array is streamed once (8 B per entry, 16 B per vertex); random
// accesses are limited to the verification loads of fingerprint matches.
#include "joinwin.cuh"

namespace lsg {

// first index i in [lo, hi) with (A[i] >> shift) >= b (lower bound of bucket b), by one
// warp: each round the 32 lanes probe 32 evenly spaced positions (32-ary search).
__device__ __forceinline__ uint64_t warp_lower_bound(const uint64_t *A, uint64_t lo, uint64_t hi,
                                                     uint32_t shift, uint64_t b)
{
    const int lane = threadIdx.x & 31;
    while (hi - lo > 32) {
        const uint64_t step = (hi - lo) / 33;
        const uint64_t p = lo + (uint64_t)(lane + 1) * step;
        const bool below = (A[p] >> shift) < b;
        const uint32_t m = __ballot_sync(0xffffffffu, below);
        const int k = 32 - __clz((int)m); // number of probes below b (they are a prefix)
        const uint64_t nlo = k ? lo + (uint64_t)k * step + 1 : lo;
        const uint64_t nhi = k < 32 ? lo + (uint64_t)(k + 1) * step : hi;
        lo = nlo;
        hi = nhi;
    }
    const uint64_t p = lo + lane;
    const bool below = p < hi && (A[p] >> shift) < b;
    return lo + __popc(__ballot_sync(0xffffffffu, below));
}

// Persistent join: CTA c owns the buckets [c*B/grid, (c+1)*B/grid) of the 2^T buckets and
// streams their (contiguous) entries through shared memory in windows of whole buckets.
template <int W>
__global__ void __launch_bounds__(JOIN_THREADS, 2)
join_kernel(JoinArgs a)
{
    extern __shared__ __align__(16) unsigned char jsm[];
    uint64_t *ent = reinterpret_cast<uint64_t *>(jsm);                                   // [CAP]
    unsigned long long *buf = reinterpret_cast<unsigned long long *>(jsm + JOIN_CAP * 8); // [BUF]
    uint32_t *slot = reinterpret_cast<uint32_t *>(jsm + (JOIN_CAP + JOIN_BUF) * 8);     // [SLOTS]
    unsigned short *next =
        reinterpret_cast<unsigned short *>(jsm + (JOIN_CAP + JOIN_BUF) * 8 + JOIN_SLOTS * 4); // [CAP]
    __shared__ uint32_t bcount, vdone;
    __shared__ unsigned long long s_r[2], s_cut, s_end;

    const uint64_t N = a.N;
    const uint32_t bshift = 64 - a.T;
    const uint64_t *A = a.keys;
    const int warp = threadIdx.x >> 5;

    if (threadIdx.x == 0) bcount = 0, vdone = 0;
    // CTA c owns the buckets that start in [c N/grid, (c+1) N/grid): its range starts at the
    // first entry of the bucket holding entry c N/grid (balanced by entries, whatever the
    // key distribution — e.g. one hash range of a multi-GPU shard)
    if (warp < 2) {
        const uint64_t q = (N * (blockIdx.x + warp)) / gridDim.x;
        uint64_t r = N;
        if (q < N) r = warp_lower_bound(A, 0, q + 1, bshift, A[q] >> bshift);
        if ((threadIdx.x & 31) == 0) s_r[warp] = r;
    }
    __syncthreads();
    const uint64_t r0 = s_r[0], r1 = s_r[1];
    Stager em{buf, &bcount, a.pairs, a.cap, a.count};
    unsigned long long nfalse = 0;

    // hash slots hold (window epoch << 16) | entry index: a slot written in an earlier window
    // reads as empty, so the table is never cleared
    for (uint32_t t = threadIdx.x; t < JOIN_SLOTS; t += JOIN_THREADS) slot[t] = 0;
    uint32_t epoch = 0;
    uint64_t t0 = r0;
    while (t0 < r1) {
        if (++epoch == 0x10000u) { // 16-bit tags wrapped: clear once and restart the epochs
            __syncthreads();
            for (uint32_t t = threadIdx.x; t < JOIN_SLOTS; t += JOIN_THREADS) slot[t] = 0;
            epoch = 1;
        }
        const uint32_t cnt = (uint32_t)min64(JOIN_CAP, r1 - t0);
        for (uint32_t k = threadIdx.x; k < cnt; k += JOIN_THREADS) ent[k] = A[t0 + k];
        __syncthreads();
        uint64_t t1;
        if (t0 + cnt == r1) {
            t1 = r1;
        } else {
            // the window is cut at the start of its last bucket (binary search: the staged
            // entries are sorted by bucket)
            if (threadIdx.x == 0) {
                const uint64_t bl = ent[cnt - 1] >> bshift;
                uint32_t lo = 0, hi = cnt - 1;
                while (lo < hi) {
                    const uint32_t mid = (lo + hi) >> 1;
                    if ((ent[mid] >> bshift) < bl) lo = mid + 1;
                    else hi = mid;
                }
                s_cut = lo;
            }
            __syncthreads();
            t1 = t0 + s_cut;
        }
        if (t1 == t0) {
            // ---- one bucket larger than a window (massively repeated fingerprints): find its
            // end in global memory, then every suffix entry scans the bucket there.
            const uint64_t bk = ent[0] >> bshift;
            if (threadIdx.x == 0) s_end = r1;
            __syncthreads();
            for (uint64_t i0 = t0 + cnt; i0 < r1; i0 += JOIN_THREADS) {
                const uint64_t i = i0 + threadIdx.x;
                if (i < r1 && (A[i] >> bshift) != bk) atomicMin(&s_end, (unsigned long long)i);
                __syncthreads();
                if (s_end != r1) break;
                __syncthreads();
            }
            __syncthreads();
            const uint64_t be = s_end;
            oversized_join<W>(a, A, t0, be, em, nfalse);
            t1 = be;
        } else {
            hash_join_window<W>(a, ent, (uint32_t)(t1 - t0), slot, next, epoch, em, nfalse);
        }
        __syncthreads();
        window_epilogue<W>(a, buf, &bcount, &vdone, nfalse);
        __syncthreads();
        t0 = t1;
    }
    final_flush<W>(a, buf, &bcount, nfalse);
    for (int o = 16; o; o >>= 1) nfalse += __shfl_xor_sync(0xffffffffu, nfalse, o);
    if ((threadIdx.x & 31) == 0 && nfalse) atomicAdd(a.false_matches, nfalse);
}

lasagna_status launch_join(const JoinArgs &args, cudaStream_t s)
{
    if (args.N == 0) return LASAGNA_OK;
    return dispatch_W(args.L, [&](auto wc) -> lasagna_status {
        constexpr int W = decltype(wc)::value;
        const size_t smem =
            (size_t)(JOIN_CAP + JOIN_BUF) * 8 + (size_t)JOIN_SLOTS * 4 + (size_t)JOIN_CAP * 2;
        LSG_CUDA(cudaFuncSetAttribute(join_kernel<W>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      (int)smem));
        int per_sm = 0;
        LSG_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, join_kernel<W>,
                                                               JOIN_THREADS, smem));
        per_sm = std::max(per_sm, 1);
        // persistent grid, but never more CTAs than ~one window of entries each
        uint64_t blocks = std::min<uint64_t>((uint64_t)num_sms() * per_sm,
                                             std::max<uint64_t>(1, args.N / JOIN_CHUNK));
        join_kernel<W><<<(unsigned)blocks, JOIN_THREADS, smem, s>>>(args);
        LSG_LAUNCHED("join_kernel");
        return LASAGNA_OK;
    });
}

// pool record (a << 32 | b) -> compact sort key (a << vbits | b)
__global__ void pairs_to_keys(const unsigned long long *pool, const unsigned long long *count,
                              unsigned long long cap, uint32_t vbits, uint64_t *keys)
{
    const unsigned long long c = *count;
    const unsigned long long m = c < cap ? c : cap;
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
