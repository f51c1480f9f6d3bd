// warpjoin.cu — a5 over the final buckets of the bucketed path, one WARP per bucket
// (Algorithm 2: "a fingerprint present in W_S cannot be present in any window
// except W_P" — a bucket is such a window pair: its build half plays W_P, its probe half W_S).
//
// The block-wide window join (partition.cu bucket_join_kernel) pays two block barriers, a
// window plan and a filter clear per ~7 K entries: ~105 instructions per entry at cfg3.  A
// bucket holds ~1 K entries (cfg3: ~531 per half), small enough for one warp:
//   1. the warp copies its bucket's build half (flags 0/2) into its own shared-memory slice
//      and hashes it (epoch-tagged chain heads: never cleared, only re-tagged);
//   2. it streams the probe half (flag 1) from global memory, four loads per lane in flight,
//      and walks the chain of each probe's slot; flag-2 build entries probe too (they play
//      both lists; a pair of two flag-2 entries is found twice and kept once, w < v);
//   3. candidates (equal stored key bits, different reads) go to a per-warp buffer; when it
//      fills, the warp verifies them on the 2-bit bases, one per lane (R12), and appends the
//      verified read-end pairs (a << 32) | b with ONE global atomic per flush.
// No block barrier anywhere: the warps of a CTA drift independently, so one warp's loads
// overlap another's hashing.  A bucket with more build entries than a slice holds is joined
// chunk by chunk (every chunk against the whole probe list).
#include "kernels.cuh"

namespace lsg {

constexpr int WJ_WARPS = 16;   // warps per CTA (one CTA per SM)
constexpr int WJ_SB = 768;     // build entries per slice (cfg3 half capacity: 747)
constexpr int WJ_HS = 1024;    // chain heads per slice
constexpr int WJ_CAND = 128;   // staged candidates per warp
constexpr int WJ_FLUSH = 96;   // flush when this many are staged at a warp-uniform point
constexpr int WJ_U = 4;        // probe loads in flight per lane

struct WarpSlice {
    unsigned long long key[WJ_SB];
    uint32_t head[WJ_HS];   // (epoch << 16) | index
    unsigned short next[WJ_SB];
    unsigned long long cand[WJ_CAND];
    uint32_t ncand;
    uint32_t pad[3];
};

// verify and append the staged candidates (warp-uniform call)
template <int W>
__device__ __forceinline__ void wj_flush(const JoinArgs &a, WarpSlice &S, unsigned long long &nfalse)
{
    __syncwarp();
    const int lane = threadIdx.x & 31;
    const uint32_t n = min(S.ncand, (uint32_t)WJ_CAND);
    for (uint32_t t0 = 0; t0 < n; t0 += 32) {
        const uint32_t t = t0 + lane;
        unsigned long long rec = ~0ull;
        bool keep = false;
        if (t < n) {
            rec = S.cand[t];
            const uint32_t u = (uint32_t)(rec >> 32), b = (uint32_t)rec;
            if (verify_overlap<W>(a.packed, a.stride, a.L, u, b ^ 1u, a.l)) {
                keep = true;
                if (a.found) atomicAdd(a.found, 1ull);
                if (a.claimed && (((a.claimed[u >> 5] >> (u & 31u)) | (a.claimed[b >> 5] >> (b & 31u))) & 1u))
                    keep = false;
            } else {
                ++nfalse;
            }
        }
        const uint32_t m = __ballot_sync(0xffffffffu, keep);
        unsigned long long base = 0;
        if (lane == 0 && m) base = atomicAdd(a.count, (unsigned long long)__popc(m));
        base = __shfl_sync(0xffffffffu, base, 0);
        if (keep) {
            const unsigned long long pos = base + __popc(m & ((1u << lane) - 1u));
            if (pos < a.cap) a.pairs[pos] = rec;
        }
    }
    __syncwarp();
    if (lane == 0) S.ncand = 0;
    __syncwarp();
}

// probe entry e (vertex w, flag 1 or 2) against the slice's hash table
template <int W>
__device__ __forceinline__ void wj_probe(const JoinArgs &a, WarpSlice &S, uint64_t e, uint32_t epoch,
                                         uint32_t kshift, uint64_t vmask, unsigned long long &nfalse)
{
    const uint32_t hv = S.head[(uint32_t)(e >> kshift) & (WJ_HS - 1)];
    uint32_t s = (hv >> 16) == epoch ? (hv & 0xFFFFu) : 0xFFFFu;
    while (s != 0xFFFFu) {
        const uint64_t p = S.key[s];
        if (((p ^ e) >> kshift) == 0) {
            const uint32_t w = (uint32_t)(e & vmask), v = (uint32_t)(p & vmask);
            // R9 (different reads); two flag-2 entries find each other twice: keep w < v
            if ((w >> 1) != (v >> 1) && !(w > v && key_flag(e, a.vbits) == 2 && key_flag(p, a.vbits) == 2)) {
                const uint32_t x = w ^ 1u, y = v ^ 1u;
                const unsigned long long rec =
                    ((unsigned long long)min(x, y) << 32) | (unsigned long long)max(x, y);
                const uint32_t slot = atomicAdd(&S.ncand, 1u);
                if (slot < (uint32_t)WJ_CAND) {
                    S.cand[slot] = rec;
                } else if (!verify_overlap<W>(a.packed, a.stride, a.L, min(x, y), max(x, y) ^ 1u, a.l)) {
                    ++nfalse; // buffer full (rare): verify inline, emit straight to the pool
                } else {
                    if (a.found) atomicAdd(a.found, 1ull);
                    const uint32_t lo = min(x, y), hi = max(x, y);
                    if (!(a.claimed && (((a.claimed[lo >> 5] >> (lo & 31u)) | (a.claimed[hi >> 5] >> (hi & 31u))) & 1u))) {
                        const unsigned long long pos = atomicAdd(a.count, 1ull);
                        if (pos < a.cap) a.pairs[pos] = rec;
                    }
                }
            }
        }
        s = S.next[s];
    }
}

template <int W>
__global__ void __launch_bounds__(WJ_WARPS * 32, 1)
warp_join_kernel(BucketJoinArgs b)
{
    extern __shared__ __align__(16) unsigned char wjsm[];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    WarpSlice &S = reinterpret_cast<WarpSlice *>(wjsm)[wid];
    const JoinArgs &a = b.j;
    const uint32_t kshift = a.vbits + FLAG_BITS;
    const uint64_t vmask = (1ull << a.vbits) - 1;
    const uint64_t flag2bit = 2ull << a.vbits;
    for (uint32_t t = lane; t < (uint32_t)WJ_HS; t += 32) S.head[t] = 0;
    if (lane == 0) S.ncand = 0;
    __syncwarp();
    uint32_t epoch = 0;
    unsigned long long nfalse = 0;
    const uint64_t nw = (uint64_t)gridDim.x * WJ_WARPS;
    // the fills of the warp's next bucket are loaded one bucket ahead, and once they are in,
    // lane 0 prefetches that bucket's two halves into L2 (cp.async.bulk.prefetch) while the
    // warp still works on the current one
    uint64_t bk = (uint64_t)blockIdx.x * WJ_WARPS + wid;
    uint32_t nfP = 0, nfS = 0;
    if (bk < b.n_buckets) nfP = b.fills[2 * bk], nfS = b.fills[2 * bk + 1];
    for (; bk < b.n_buckets; bk += nw) {
        uint32_t fP = nfP, fS = nfS;
        const uint64_t bn = bk + nw;
        if (bn < b.n_buckets) nfP = b.fills[2 * bn], nfS = b.fills[2 * bn + 1];
        if (fP > b.half_cap || fS > b.half_cap) {
            if (lane == 0) *b.overflow = 1u; // the call is redone on the exact path
            fP = (uint32_t)min64(fP, b.half_cap);
            fS = (uint32_t)min64(fS, b.half_cap);
        }
        const uint64_t *P = b.buckets + bk * 2 * b.half_cap;
        const uint64_t *Q = P + b.half_cap;
        // flag-2 build entries also probe; with several chunks every chunk must see all of them
        bool has2 = false;
        if (fP > (uint32_t)WJ_SB) {
            for (uint32_t j = lane; j < fP; j += 32) has2 |= (P[j] & flag2bit) != 0;
            has2 = __any_sync(0xffffffffu, has2);
        }
        for (uint32_t c0 = 0; c0 < fP; c0 += WJ_SB) {
            const uint32_t nb = min((uint32_t)WJ_SB, fP - c0);
            if (++epoch == 0x10000u) {
                __syncwarp();
                for (uint32_t t = lane; t < (uint32_t)WJ_HS; t += 32) S.head[t] = 0;
                epoch = 1;
            }
            __syncwarp();
            // 1. copy + hash the build chunk, WJ_U loads per lane in flight
            bool h2 = false;
            for (uint32_t j0 = 0; j0 < nb; j0 += 32 * WJ_U) {
                uint64_t be[WJ_U];
#pragma unroll
                for (int u = 0; u < WJ_U; ++u) {
                    const uint32_t j = j0 + u * 32 + lane;
                    be[u] = j < nb ? P[c0 + j] : 0ull;
                }
#pragma unroll
                for (int u = 0; u < WJ_U; ++u) {
                    const uint32_t j = j0 + u * 32 + lane;
                    if (j < nb) {
                        const uint64_t e = be[u];
                        S.key[j] = e;
                        h2 |= (e & flag2bit) != 0;
                        const uint32_t old =
                            atomicExch(&S.head[(uint32_t)(e >> kshift) & (WJ_HS - 1)], (epoch << 16) | j);
                        S.next[j] = (old >> 16) == epoch ? (unsigned short)(old & 0xFFFFu)
                                                         : (unsigned short)0xFFFFu;
                    }
                }
            }
            if (fP <= (uint32_t)WJ_SB) has2 = __any_sync(0xffffffffu, h2);
            if (c0 == 0 && lane == 0 && bn < b.n_buckets) {
                const uint64_t *Pn = b.buckets + bn * 2 * b.half_cap;
                const uint32_t bp = (uint32_t)min64(nfP, b.half_cap) * 8u, bs = (uint32_t)min64(nfS, b.half_cap) * 8u;
                if (bp >= 16)
                    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(Pn), "r"(bp & ~15u) : "memory");
                if (bs >= 16)
                    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(Pn + b.half_cap), "r"(bs & ~15u)
                                 : "memory");
            }
            __syncwarp();
            // 2. the probe half, WJ_U loads per lane in flight
            for (uint32_t t0 = 0; t0 < fS; t0 += 32 * WJ_U) {
                uint64_t pe[WJ_U];
#pragma unroll
                for (int u = 0; u < WJ_U; ++u) {
                    const uint32_t t = t0 + u * 32 + lane;
                    pe[u] = t < fS ? Q[t] : 0ull;
                }
#pragma unroll
                for (int u = 0; u < WJ_U; ++u)
                    if (t0 + u * 32 + lane < fS) wj_probe<W>(a, S, pe[u], epoch, kshift, vmask, nfalse);
                __syncwarp();
                if (S.ncand >= (uint32_t)WJ_FLUSH) wj_flush<W>(a, S, nfalse);
            }
            // flag-2 build entries as probes (palindromic prefixes or H == Hr: rare)
            if (has2) {
                for (uint32_t j = lane; j < fP; j += 32) {
                    const uint64_t e = P[j];
                    if (e & flag2bit) wj_probe<W>(a, S, e, epoch, kshift, vmask, nfalse);
                }
                __syncwarp();
                if (S.ncand >= (uint32_t)WJ_FLUSH) wj_flush<W>(a, S, nfalse);
            }
        }
    }
    __syncwarp();
    wj_flush<W>(a, S, nfalse);
    for (int o = 16; o; o >>= 1) nfalse += __shfl_xor_sync(0xffffffffu, nfalse, o);
    if (lane == 0 && nfalse) atomicAdd(a.false_matches, nfalse);
}

lasagna_status launch_warp_join(const BucketJoinArgs &args, cudaStream_t s)
{
    if (args.n_buckets == 0) return LASAGNA_OK;
    return dispatch_W(args.j.L, [&](auto wc) -> lasagna_status {
        constexpr int W = decltype(wc)::value;
        const size_t smem = sizeof(WarpSlice) * WJ_WARPS;
        LSG_CUDA(cudaFuncSetAttribute(warp_join_kernel<W>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                      (int)smem));
        int per_sm = 0;
        LSG_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, warp_join_kernel<W>,
                                                               WJ_WARPS * 32, smem));
        per_sm = std::max(per_sm, 1);
        const uint64_t blocks = std::max<uint64_t>(
            1, std::min<uint64_t>((uint64_t)num_sms() * per_sm, ceil_div(args.n_buckets, WJ_WARPS)));
        warp_join_kernel<W><<<(unsigned)blocks, WJ_WARPS * 32, smem, s>>>(args);
        LSG_LAUNCHED("warp_join_kernel");
        return LASAGNA_OK;
    });
}

} // namespace lsg
