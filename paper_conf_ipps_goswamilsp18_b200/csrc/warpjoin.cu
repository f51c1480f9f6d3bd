// warpjoin.cu — a5 over the final buckets of the bucketed path, one WARP per bucket
// (Algorithm 2: "a fingerprint present in W_S cannot be present in any window
// except W_P" — a bucket is such a window pair: its build half plays W_P, its probe half W_S).
//
// The block-wide window join (partition_join.cu bucket_join_kernel) pays two block barriers, a
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
// No block barrier anywhere: the warps of a CTA drift independently.  Each warp double-
// buffers its buckets: while it joins bucket k out of shared memory, the copy engine brings
// bucket k + 1's two halves in (cp.async.bulk issued by lane 0, one mbarrier per buffer), so
// the warp never waits on a global load.  Used when a half fits a slice (half capacity <=
// WJ_SB: cfg1-cfg4 geometries); larger halves take the block-window join.
#include "kernels.cuh"

namespace lsg {

constexpr int WJ_WARPS = 7;    // warps per CTA (one CTA per SM; the slices fill shared memory)
constexpr int WJ_SB = 768;     // entries per staged half (cfg3 half capacity: 747)
constexpr int WJ_HS = 1024;    // chain heads per slice
constexpr int WJ_CAND = 128;   // staged candidates per warp
constexpr int WJ_FLUSH = 96;   // flush when this many are staged at a warp-uniform point

struct alignas(128) WarpSlice {
    unsigned long long buf[2][2][WJ_SB]; // [buffer][build, probe half][entry]
    uint32_t head[WJ_HS];                // (epoch << 16) | index
    unsigned short next[WJ_SB];
    unsigned long long cand[WJ_CAND];
    unsigned long long mbar[2];
    uint32_t ncand;
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
            if (verify_pair<W>(a, u, b ^ 1u)) {
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
__device__ __forceinline__ void wj_probe(const JoinArgs &a, WarpSlice &S, const unsigned long long *key,
                                         uint64_t e, uint32_t epoch, uint32_t kshift, uint64_t vmask,
                                         unsigned long long &nfalse)
{
    const uint32_t hv = S.head[(uint32_t)(e >> kshift) & (WJ_HS - 1)];
    uint32_t s = (hv >> 16) == epoch ? (hv & 0xFFFFu) : 0xFFFFu;
    while (s != 0xFFFFu) {
        const uint64_t p = key[s];
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
                } else if (!verify_pair<W>(a, min(x, y), max(x, y) ^ 1u)) {
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

// lane 0: start the copies of bucket bk's halves (fills fP, fS) into buffer c
__device__ __forceinline__ void wj_issue(const BucketJoinArgs &b, WarpSlice &S, int c, uint64_t bk,
                                         uint32_t fP, uint32_t fS)
{
    const uint32_t bp = ((fP + 1u) & ~1u) * 8u, bs = ((fS + 1u) & ~1u) * 8u; // 16-byte units
    const uint32_t bar = smem_u32(&S.mbar[c]);
    fence_proxy_async(); // the buffer was last read by the generic proxy
    if (bp + bs == 0) {
        asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
        return;
    }
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bp + bs)
                 : "memory");
    const uint64_t *P = b.buckets + bk * 2 * b.half_cap;
    if (bp)
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     ::"r"(smem_u32(S.buf[c][0])), "l"(P), "r"(bp), "r"(bar) : "memory");
    if (bs)
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     ::"r"(smem_u32(S.buf[c][1])), "l"(P + b.half_cap), "r"(bs), "r"(bar) : "memory");
}

template <int W>
__global__ void __launch_bounds__(WJ_WARPS * 32, 1)
warp_join_kernel(BucketJoinArgs b)
{
    extern __shared__ __align__(128) unsigned char wjsm[];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    WarpSlice &S = reinterpret_cast<WarpSlice *>(wjsm)[wid];
    const JoinArgs &a = b.j;
    const uint32_t kshift = a.vbits + FLAG_BITS;
    const uint64_t vmask = (1ull << a.vbits) - 1;
    const uint64_t flag2bit = 2ull << a.vbits;
    for (uint32_t t = lane; t < (uint32_t)WJ_HS; t += 32) S.head[t] = 0;
    if (lane == 0) {
        S.ncand = 0;
        mbar_init(&S.mbar[0], 1);
        mbar_init(&S.mbar[1], 1);
        fence_mbar_init();
    }
    __syncwarp();
    uint32_t epoch = 0, phases = 0; // bit c: parity of the next completion of mbar[c]
    unsigned long long nfalse = 0;
    const uint64_t nw = (uint64_t)gridDim.x * WJ_WARPS;
    uint64_t bk = (uint64_t)blockIdx.x * WJ_WARPS + wid;
    auto fills = [&](uint64_t k, uint32_t &fP, uint32_t &fS) {
        fP = b.fills[2 * k];
        fS = b.fills[2 * k + 1];
        if (fP > b.half_cap || fS > b.half_cap) {
            if (lane == 0) *b.overflow = 1u; // the call is redone on the exact path
            fP = fS = 0; // unwritten slots: join nothing from an overflowed bucket
        }
    };
    uint32_t fP = 0, fS = 0;
    if (bk < b.n_buckets) {
        fills(bk, fP, fS);
        if (lane == 0) wj_issue(b, S, 0, bk, fP, fS);
    }
    for (int c = 0; bk < b.n_buckets; bk += nw, c ^= 1) {
        // start the next bucket's copies into the other buffer (free: its last bucket is done)
        const uint64_t bn = bk + nw;
        uint32_t nP = 0, nS = 0;
        if (bn < b.n_buckets) {
            fills(bn, nP, nS);
            __syncwarp();
            if (lane == 0) wj_issue(b, S, c ^ 1, bn, nP, nS);
        }
        mbar_wait(&S.mbar[c], (phases >> c) & 1u);
        phases ^= 1u << c;
        const unsigned long long *Pb = S.buf[c][0], *Qb = S.buf[c][1];
        if (++epoch == 0x10000u) {
            for (uint32_t t = lane; t < (uint32_t)WJ_HS; t += 32) S.head[t] = 0;
            epoch = 1;
            __syncwarp();
        }
        // 1. hash the build half
        bool h2 = false;
        for (uint32_t j = lane; j < fP; j += 32) {
            const uint64_t e = Pb[j];
            h2 |= (e & flag2bit) != 0;
            const uint32_t old = atomicExch(&S.head[(uint32_t)(e >> kshift) & (WJ_HS - 1)], (epoch << 16) | j);
            S.next[j] = (old >> 16) == epoch ? (unsigned short)(old & 0xFFFFu) : (unsigned short)0xFFFFu;
        }
        const bool has2 = __any_sync(0xffffffffu, h2);
        __syncwarp();
        // 2. the probe half (and flag-2 build entries, rare)
        for (uint32_t t0 = 0; t0 < fS; t0 += 32) {
            if (t0 + lane < fS) wj_probe<W>(a, S, Pb, Qb[t0 + lane], epoch, kshift, vmask, nfalse);
            __syncwarp();
            if (S.ncand >= (uint32_t)WJ_FLUSH) wj_flush<W>(a, S, nfalse);
        }
        if (has2) {
            for (uint32_t j0 = 0; j0 < fP; j0 += 32) {
                const uint32_t j = j0 + lane;
                if (j < fP && (Pb[j] & flag2bit)) wj_probe<W>(a, S, Pb, Pb[j], epoch, kshift, vmask, nfalse);
                __syncwarp();
                if (S.ncand >= (uint32_t)WJ_FLUSH) wj_flush<W>(a, S, nfalse);
            }
        }
        __syncwarp(); // buffer c is read: the next issue may overwrite it
        fP = nP;
        fS = nS;
    }
    __syncwarp();
    wj_flush<W>(a, S, nfalse);
    for (int o = 16; o; o >>= 1) nfalse += __shfl_xor_sync(0xffffffffu, nfalse, o);
    if (lane == 0 && nfalse) atomicAdd(a.false_matches, nfalse);
}

bool warp_join_fits(const BucketJoinArgs &args) { return args.half_cap <= (uint64_t)WJ_SB; }

lasagna_status launch_warp_join(const BucketJoinArgs &args, cudaStream_t s)
{
    if (args.n_buckets == 0) return LASAGNA_OK;
    if (!warp_join_fits(args) || (args.half_cap & 1)) return LASAGNA_EINVAL;
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
