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
#include "kernels.cuh"

namespace lsg {

constexpr int JOIN_THREADS = 512;
constexpr int JOIN_CHUNK = 2048;   // nominal entries per CTA
constexpr int JOIN_CAP = 6144;     // staged entries per CTA (chunk + the bucket straddling its end)
constexpr int JOIN_SLOTS = 8192;   // u16 hash slots (load <= 0.75 even when all staged are P)
constexpr int JOIN_BUF = 1024;     // staged output pairs
constexpr unsigned short SLOT_EMPTY = 0xFFFF;

struct Emitter {
    unsigned long long *buf;  // shared
    uint32_t *bcount;         // shared
    unsigned long long *pairs, cap, *count;
    __device__ __forceinline__ void emit(unsigned long long rec)
    {
        uint32_t slot = atomicAdd(bcount, 1u);
        if (slot < JOIN_BUF) buf[slot] = rec;
        else {
            unsigned long long gs = atomicAdd(count, 1ull);
            if (gs < cap) pairs[gs] = rec;
        }
    }
};

template <int W>
__device__ __forceinline__ void candidate(const JoinArgs &a, uint64_t s_ent, uint64_t p_ent,
                                          uint64_t vmask, Emitter &em, unsigned long long &nfalse)
{
    const uint32_t u = (uint32_t)(s_ent & vmask), v = (uint32_t)(p_ent & vmask);
    const uint32_t b = v ^ 1u;
    if ((u >> 1) == (v >> 1) || u >= b) return; // R9: no same-read edge; each pair once
    if (!verify_overlap<W>(a.packed, a.stride, a.L, u, v, a.l)) {
        ++nfalse;
        return;
    }
    em.emit(((unsigned long long)u << 32) | b);
}

template <int W>
__global__ void __launch_bounds__(JOIN_THREADS)
join_kernel(JoinArgs a)
{
    extern __shared__ __align__(16) unsigned char jsm[];
    uint64_t *ent = reinterpret_cast<uint64_t *>(jsm);                                   // [CAP]
    unsigned long long *buf = reinterpret_cast<unsigned long long *>(jsm + JOIN_CAP * 8); // [BUF]
    unsigned short *slot = reinterpret_cast<unsigned short *>(jsm + (JOIN_CAP + JOIN_BUF) * 8);
    __shared__ uint32_t bcount;
    __shared__ unsigned long long gbase;
    __shared__ unsigned long long s_lo, s_hi;

    const uint64_t N = a.N;
    const uint64_t base = (uint64_t)blockIdx.x * JOIN_CHUNK;
    if (base >= N) return;
    const uint32_t bshift = 64 - a.T;
    const uint32_t kshift = a.vbits + 1; // key bits above tag + vid
    const uint64_t vmask = (1ull << a.vbits) - 1;
    const uint64_t *A = a.keys;

    if (threadIdx.x == 0) {
        bcount = 0;
        s_lo = ~0ull;
        s_hi = ~0ull;
    }
    for (int t = threadIdx.x; t < JOIN_SLOTS; t += JOIN_THREADS) slot[t] = SLOT_EMPTY;
    __syncthreads();

    // bucket starts: i is a start if i == 0 or bucket(A[i]) != bucket(A[i-1]).
    // lo = first start in [base, base+CHUNK); hi = first start >= base+CHUNK (or N).
    const uint64_t cend = min64(N, base + JOIN_CHUNK);
    for (uint64_t i = base + threadIdx.x; i < cend; i += JOIN_THREADS) {
        bool st = (i == 0) || ((A[i] >> bshift) != (A[i - 1] >> bshift));
        if (st) atomicMin(&s_lo, (unsigned long long)i);
    }
    __syncthreads();
    const uint64_t lo = s_lo;
    if (lo == ~0ull) return; // no bucket starts here: the chunk is inside an earlier bucket
    for (uint64_t i0 = cend; i0 < N; i0 += JOIN_THREADS) {
        uint64_t i = i0 + threadIdx.x;
        if (i < N && (A[i] >> bshift) != (A[i - 1] >> bshift))
            atomicMin(&s_hi, (unsigned long long)i);
        __syncthreads();
        if (s_hi != ~0ull) break;
        __syncthreads();
    }
    __syncthreads();
    const uint64_t hi = (s_hi == ~0ull) ? N : (uint64_t)s_hi;
    const uint64_t cnt = hi - lo;

    Emitter em{buf, &bcount, a.pairs, a.cap, a.count};
    unsigned long long nfalse = 0;

    if (cnt <= JOIN_CAP) {
        // ---- stage, build the hash of prefix entries, probe with suffix entries
        for (uint32_t k = threadIdx.x; k < cnt; k += JOIN_THREADS) ent[k] = A[lo + k];
        __syncthreads();
        for (uint32_t k = threadIdx.x; k < cnt; k += JOIN_THREADS) {
            uint64_t e = ent[k];
            if ((e >> a.vbits) & 1) continue; // suffix entry
            uint32_t h = (uint32_t)(e >> kshift) & (JOIN_SLOTS - 1);
            while (atomicCAS(&slot[h], SLOT_EMPTY, (unsigned short)k) != SLOT_EMPTY)
                h = (h + 1) & (JOIN_SLOTS - 1);
        }
        __syncthreads();
        for (uint32_t k = threadIdx.x; k < cnt; k += JOIN_THREADS) {
            uint64_t e = ent[k];
            if (!((e >> a.vbits) & 1)) continue; // prefix entry
            uint32_t h = (uint32_t)(e >> kshift) & (JOIN_SLOTS - 1);
            while (true) {
                unsigned short s = slot[h];
                if (s == SLOT_EMPTY) break;
                uint64_t p = ent[s];
                if (((p ^ e) >> kshift) == 0) candidate<W>(a, e, p, vmask, em, nfalse);
                h = (h + 1) & (JOIN_SLOTS - 1);
            }
        }
    } else {
        // ---- oversized run of buckets (only with massively repeated fingerprints): every
        // suffix entry scans its own bucket in global memory.
        for (uint64_t i = lo + threadIdx.x; i < hi; i += JOIN_THREADS) {
            uint64_t e = A[i];
            if (!((e >> a.vbits) & 1)) continue;
            const uint64_t bk = e >> bshift;
            uint64_t j0 = i;
            while (j0 > lo && (A[j0 - 1] >> bshift) == bk) --j0;
            for (uint64_t j = j0; j < hi && (A[j] >> bshift) == bk; ++j) {
                uint64_t p = A[j];
                if (((p >> a.vbits) & 1) == 0 && ((p ^ e) >> kshift) == 0)
                    candidate<W>(a, e, p, vmask, em, nfalse);
            }
        }
    }
    __syncthreads();
    const uint32_t m = min(bcount, (uint32_t)JOIN_BUF);
    if (m) {
        if (threadIdx.x == 0) gbase = atomicAdd(a.count, (unsigned long long)m);
        __syncthreads();
        for (uint32_t t = threadIdx.x; t < m; t += JOIN_THREADS)
            if (gbase + t < a.cap) a.pairs[gbase + t] = buf[t];
    }
    for (int o = 16; o; o >>= 1) nfalse += __shfl_xor_sync(0xffffffffu, nfalse, o);
    if ((threadIdx.x & 31) == 0 && nfalse) atomicAdd(a.false_matches, nfalse);
}

lasagna_status launch_join(const JoinArgs &args, cudaStream_t s)
{
    if (args.N == 0) return LASAGNA_OK;
    return dispatch_W(args.L, [&](auto wc) -> lasagna_status {
        constexpr int W = decltype(wc)::value;
        const uint64_t blocks = ceil_div(args.N, JOIN_CHUNK);
        const size_t smem = (size_t)(JOIN_CAP + JOIN_BUF) * 8 + (size_t)JOIN_SLOTS * 2;
        LSG_CUDA(cudaFuncSetAttribute(join_kernel<W>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      (int)smem));
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
