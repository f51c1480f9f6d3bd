// partition_join.cu — a5 over the final buckets: bucket_join_kernel (the bucketed fast path; overview in partition.cuh)
#include "partition.cuh"

namespace lsg {

// ------------------------------------------------------------------ a5 over the buckets
// Buckets are stored split: prefix entries [b][0][0..fillP), suffix entries [b][1][0..fillS).
// A window = consecutive whole buckets whose prefix halves and suffix halves each fit a
// staging buffer.  The copy engine (cp.async.bulk, one mbarrier per buffer pair) stages both
// halves of window w+1 while window w is joined: its prefix entries are hashed in shared
// memory (chained, epoch-tagged heads: never cleared) and its suffix entries probe the table.
// A half's copy is rounded up to 16 bytes: an odd fill drags one more slot along, which the
// CTA overwrote beforehand (in global memory) with a sentinel of the wrong tag — ~0 (tag 1)
// in a prefix half, ~0 ^ (1 << vbits) (tag 0) in a suffix half — so the insert and probe
// loops skip it by its tag bit alone.  Two barriers per window.
// CTA geometry (BjCfg): threads, staged entries per half per window, chain heads (u32
// epoch-tagged), filter words (u32) per buffer.  Default 1024 / 4096 / 4096 / 2048 (one CTA
// per SM, a 64 Ki-bit filter); smaller CTAs run several per SM (a block barrier then stalls
// one of them, not the SM).
template <int NT, int HALF, int SLOTS, int BLOOMW>
struct BjCfg {
    static constexpr int THREADS = NT, HALF_ = HALF, SLOTS_ = SLOTS, BLOOM = BLOOMW;
};
constexpr int BJ_MAXB = 64;     // buckets per window
constexpr int BJ_FILLS = 256;   // buckets whose fills are staged at once
constexpr int BJ_QCAP = 64;     // per-warp queue of probes that passed the filter

struct WinDesc {
    uint32_t nb, nP, nS;             // buckets (0: one oversized bucket), staged slots
    uint32_t first;                  // first bucket (index within the chunk)
};

// one bucket with a half larger than a staging buffer (massively repeated fingerprints),
// joined in global memory: every probe entry (the probe half, plus flag-2 entries of the build
// half) scans the build half
template <int W, int BJ_THREADS>
__device__ __forceinline__ void oversized_join_split(const JoinArgs &a, const uint64_t *P,
                                                     uint32_t nP, const uint64_t *S, uint32_t nS,
                                                     Stager &em, unsigned long long &nfalse)
{
    const uint32_t kshift = a.vbits + FLAG_BITS;
    const uint64_t vmask = (1ull << a.vbits) - 1;
    for (uint32_t i = threadIdx.x; i < nS + nP; i += BJ_THREADS) {
        const uint64_t e = i < nS ? S[i] : P[i - nS];
        if (i >= nS && key_flag(e, a.vbits) != 2) continue;
        for (uint32_t j = 0; j < nP; ++j) {
            const uint64_t p = P[j];
            if (((p ^ e) >> kshift) == 0) candidate<W>(a, e, p, vmask, em, nfalse);
        }
    }
}

template <int W, class C>
__global__ void __launch_bounds__(C::THREADS, 1024 / C::THREADS)
bucket_join_kernel(BucketJoinArgs b)
{
    constexpr int BJ_THREADS = C::THREADS, BJ_HALF = C::HALF_, BJ_SLOTS = C::SLOTS_;
    constexpr int BJ_BLOOM = C::BLOOM, BJ_BUF = 2 * BJ_THREADS;
    static_assert((BJ_BLOOM & (BJ_BLOOM - 1)) == 0 && (BJ_SLOTS & (BJ_SLOTS - 1)) == 0, "powers of two");
    constexpr uint32_t FMASK = BJ_BLOOM * 32u - 1u; // filter bit index mask
    extern __shared__ __align__(128) unsigned char jsm[];
    uint64_t *pst = reinterpret_cast<uint64_t *>(jsm);                    // [2][BJ_HALF]
    uint64_t *sst = pst + 2 * BJ_HALF;                                    // [2][BJ_HALF]
    unsigned long long *buf = reinterpret_cast<unsigned long long *>(sst + 2 * BJ_HALF); // [BUF]
    uint32_t *slot = reinterpret_cast<uint32_t *>(buf + BJ_BUF);       // [BJ_SLOTS]
    uint32_t *bloom = slot + BJ_SLOTS;                                    // [2][BJ_BLOOM]
    unsigned short *queue = reinterpret_cast<unsigned short *>(bloom + 2 * BJ_BLOOM); // [16][QCAP]
    unsigned short *next = queue + (BJ_THREADS / 32) * BJ_QCAP;         // [BJ_HALF]
    uint32_t *sfill = reinterpret_cast<uint32_t *>(next + BJ_HALF);       // [2 * BJ_FILLS]
    __shared__ WinDesc wd[2];
    __shared__ __align__(8) unsigned long long mbar[2];
    __shared__ uint32_t bcount, vdone, s_k[2], s_has2[2];
    const JoinArgs &a = b.j;
    const uint64_t nbk = b.n_buckets;
    const uint64_t b0 = nbk * blockIdx.x / gridDim.x, b1 = nbk * (blockIdx.x + 1) / gridDim.x;
    const uint32_t kshift = a.vbits + FLAG_BITS;
    const uint64_t vmask = (1ull << a.vbits) - 1;
    const uint64_t tagbit = 1ull << a.vbits;      // half bit: 0 build side, 1 probe side
    const uint64_t flag2bit = 2ull << a.vbits;
    if (threadIdx.x == 0) {
        bcount = 0, vdone = 0, s_has2[0] = 0, s_has2[1] = 0;
        mbar_init(&mbar[0], 1);
        mbar_init(&mbar[1], 1);
        fence_mbar_init();
    }
    for (uint32_t t = threadIdx.x; t < BJ_SLOTS; t += BJ_THREADS) slot[t] = 0;
    for (uint32_t t = threadIdx.x; t < 2 * BJ_BLOOM; t += BJ_THREADS) bloom[t] = 0;
    Stager em{buf, &bcount, a.pairs, a.cap, a.count, BJ_BUF};
    unsigned long long nfalse = 0;
    uint32_t epoch = 0, phases = 0; // bit w: parity of the next phase of mbar[w]
    const int lane = threadIdx.x & 31;
    unsigned short *wq = queue + (threadIdx.x >> 5) * BJ_QCAP; // this warp's probe queue

    for (uint64_t c0 = b0; c0 < b1; c0 += BJ_FILLS) {
        const uint32_t nc = (uint32_t)min64(BJ_FILLS, b1 - c0);
        __syncthreads();
        for (uint32_t t = threadIdx.x; t < 2 * nc; t += BJ_THREADS) {
            const uint32_t f = b.fills[2 * c0 + t];
            if (f > b.half_cap) *b.overflow = 1u;
            // an overflowed half lost keys and holds slots this call never wrote: the call is
            // redone on the exact path, so join nothing from it (no stale vertex ids)
            const uint32_t fc = f > b.half_cap ? 0u : f;
            sfill[t] = fc;
            if (fc & 1) // half_cap is even: the slot after an odd fill is inside the half
                b.buckets[(c0 + t / 2) * 2 * b.half_cap + (t & 1) * b.half_cap + fc] =
                    (t & 1) ? ~tagbit : ~0ull;
        }
        // the sentinels are read by the async proxy (bulk copies)
        asm volatile("fence.proxy.async.global;" ::: "memory");
        __syncthreads();
        // plan the window starting at chunk bucket k into descriptor w and start its copies
        // (thread 0).  A bucket with a half larger than a staging buffer is a window of its
        // own with nb = 0, joined in global memory.
        // plan the window starting at chunk bucket k into descriptor w and start its copies.
        // Run by all 32 lanes of the planning warp: lane j sizes bucket k + j, a warp scan
        // finds how many whole buckets fit both staging halves, and each lane issues its
        // bucket's two bulk copies (a serial plan on one thread made its warp the last to
        // reach the next block barrier).  A bucket with a half larger than a staging buffer is
        // a window of its own with nb = 0, joined in global memory.
        auto plan = [&](uint32_t k, int w) -> uint32_t {
            const uint32_t j = k + lane;
            const bool in = lane < BJ_MAXB && j < nc;
            const uint32_t pp = in ? (sfill[2 * j] + 1) & ~1u : 0u;
            const uint32_t ps = in ? (sfill[2 * j + 1] + 1) & ~1u : 0u;
            WinDesc &d = wd[w];
            const uint32_t bar = smem_u32(&mbar[w]);
            if (sfill[2 * k] > (uint32_t)BJ_HALF || sfill[2 * k + 1] > (uint32_t)BJ_HALF) {
                if (lane == 0) d.first = k, d.nb = 0;
                __syncwarp();
                return k + 1;
            }
            uint32_t sp = pp, ss = ps; // inclusive scans
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t yp = __shfl_up_sync(0xffffffffu, sp, o);
                const uint32_t ys = __shfl_up_sync(0xffffffffu, ss, o);
                if (lane >= o) sp += yp, ss += ys;
            }
            const bool fits = in && sp <= (uint32_t)BJ_HALF && ss <= (uint32_t)BJ_HALF;
            const uint32_t nb = __popc(__ballot_sync(0xffffffffu, fits)); // fits is a lane prefix
            const uint32_t nP = __shfl_sync(0xffffffffu, sp, nb - 1);
            const uint32_t nS = __shfl_sync(0xffffffffu, ss, nb - 1);
            if (lane == 0) {
                d.first = k, d.nb = nb, d.nP = nP, d.nS = nS;
                if (nP + nS)
                    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar),
                                 "r"((nP + nS) * 8)
                                 : "memory");
                else
                    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
            }
            __syncwarp();
            if ((uint32_t)lane < nb) {
                LSG_DCHECK(c0 + j < b.n_buckets);
                const uint64_t *gb = b.buckets + (c0 + j) * 2 * b.half_cap;
                if (pp)
                    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::"
                                 "bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(pst + w * BJ_HALF + sp - pp)),
                                 "l"(gb), "r"(pp * 8), "r"(bar)
                                 : "memory");
                if (ps)
                    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::"
                                 "bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(sst + w * BJ_HALF + ss - ps)),
                                 "l"(gb + b.half_cap), "r"(ps * 8), "r"(bar)
                                 : "memory");
            }
            return k + nb;
        };
        constexpr int PLAN_WARP = BJ_THREADS / 32 - 1;
        const bool planner = (threadIdx.x >> 5) == PLAN_WARP;
        if (planner) {
            fence_proxy_async();
            const uint32_t kn = plan(0, 0);
            if (lane == 0) s_k[0] = kn;
        }
        __syncthreads();
        int w = 0;
        uint32_t kcur = 0;
        while (kcur < nc) {
            const uint32_t knext = s_k[w];
            if (planner && knext < nc) {
                fence_proxy_async();
                const uint32_t kn = plan(knext, w ^ 1);
                if (lane == 0) s_k[w ^ 1] = kn;
            }
            const WinDesc &d = wd[w];
            // the other filter buffer was last read by window w-1 and is next written by
            // window w+1 (both across an end-of-window barrier): clear it now
            for (uint32_t t = threadIdx.x; t < BJ_BLOOM / 4; t += BJ_THREADS)
                reinterpret_cast<uint4 *>(bloom + (w ^ 1) * BJ_BLOOM)[t] = make_uint4(0, 0, 0, 0);
            if (d.nb == 0) {
                const uint64_t bk = c0 + d.first;
                const uint64_t *gb = b.buckets + bk * 2 * b.half_cap;
                oversized_join_split<W, BJ_THREADS>(a, gb, sfill[2 * d.first], gb + b.half_cap,
                                        sfill[2 * d.first + 1], em, nfalse);
            } else {
                mbar_wait(&mbar[w], (phases >> w) & 1u);
                phases ^= 1u << w;
                if (++epoch == 0x10000u) { // block-uniform
                    for (uint32_t t = threadIdx.x; t < BJ_SLOTS; t += BJ_THREADS) slot[t] = 0;
                    epoch = 1;
                    __syncthreads();
                }
                const uint64_t *P = pst + w * BJ_HALF, *S = sst + w * BJ_HALF;
                uint32_t *bl = bloom + w * BJ_BLOOM;
                const uint32_t tag = epoch << 16;
                const uint32_t nP = d.nP, nS = d.nS;
                // ---- build: chained hash of the build entries + the 64 Ki-bit filter
                // the planner warp (which planned the next window just before) sits the build
                // out unless LASAGNA_BJ_PLANNER_BUILDS: its share would make every other warp wait
                // at the barrier below
                const uint32_t nbuild = b.planner_builds ? BJ_THREADS : BJ_THREADS - 32;
                const uint32_t kb0 = (b.planner_builds || !planner) ? threadIdx.x : nP;
#pragma unroll 2
                for (uint32_t k2 = kb0; k2 < nP; k2 += nbuild) {
                    const uint64_t e = P[k2];
                    if (e & tagbit) continue; // sentinel
                    if (e & flag2bit) s_has2[w] = 1u; // a flag-2 entry also probes (rare)
                    const uint32_t hk = (uint32_t)(e >> kshift);
                    atomicOr(&bl[(hk & FMASK) >> 5], 1u << (hk & 31u));
                    const uint32_t old = atomicExch(&slot[hk & (BJ_SLOTS - 1)], tag | k2);
                    next[k2] = (old >> 16) == epoch ? (unsigned short)(old & 0xFFFFu) : 0xFFFFu;
                }
                __syncthreads();
                if (threadIdx.x == 0) s_has2[w ^ 1] = 0u; // the other window's flag is stale
                // ---- probe: ~95 % of the probe keys miss the filter; the rest are queued per
                // warp and their chains walked 32 at a time (full warps, no per-lane divergence
                // between a probe that has a chain and one that has none)
                auto walk = [&](uint64_t e) {
                    const uint32_t hv = slot[(uint32_t)(e >> kshift) & (BJ_SLOTS - 1)];
                    uint32_t sl = (hv >> 16) == epoch ? (hv & 0xFFFFu) : 0xFFFFu;
                    while (sl != 0xFFFFu) {
                        const uint64_t p = P[sl];
                        if (((p ^ e) >> kshift) == 0) candidate<W>(a, e, p, vmask, em, nfalse);
                        sl = next[sl];
                    }
                };
                auto drain = [&](uint32_t from, uint32_t cnt) { // lanes < cnt walk wq[from + lane]
                    __syncwarp();
                    const bool act = (uint32_t)lane < cnt;
                    const uint32_t qi = act ? wq[from + lane] : 0u;
                    __syncwarp();
                    if (act) walk((qi & 0x8000u) ? P[qi & 0x7FFFu] : S[qi]);
                };
                uint32_t qn = 0; // warp-uniform
                auto push = [&](bool pass, uint32_t qi) {
                    const uint32_t m = __ballot_sync(0xffffffffu, pass);
                    if (pass) wq[qn + __popc(m & ((1u << lane) - 1u))] = (unsigned short)qi;
                    qn += __popc(m);
                    if (qn >= 32) {
                        drain(qn - 32, 32);
                        qn -= 32;
                    }
                };
                auto passes = [&](uint64_t e) {
                    const uint32_t hk = (uint32_t)(e >> kshift) & FMASK;
                    return ((bl[hk >> 5] >> (hk & 31u)) & 1u) != 0;
                };
#pragma unroll 2
                for (uint32_t t0 = 0; t0 < nS; t0 += BJ_THREADS) { // block-uniform trip count
                    const uint32_t t = t0 + threadIdx.x;
                    bool pass = false;
                    if (t < nS) {
                        const uint64_t e = S[t];
                        pass = (e & tagbit) && passes(e); // !tagbit: sentinel
                    }
                    push(pass, t);
                }
                if (s_has2[w]) { // block-uniform
                    for (uint32_t t0 = 0; t0 < nP; t0 += BJ_THREADS) {
                        const uint32_t k2 = t0 + threadIdx.x;
                        const bool pass = k2 < nP && (P[k2] & (tagbit | flag2bit)) == flag2bit;
                        push(pass, 0x8000u | k2);
                    }
                }
                if (qn) drain(0, qn);
            }
            __syncthreads(); // window w done: its buffers may be refilled
            window_epilogue<W, BJ_THREADS>(a, buf, &bcount, &vdone, nfalse);
            kcur = knext;
            w ^= 1;
        }
    }
    final_flush<W, BJ_THREADS>(a, buf, &bcount, nfalse);
    for (int o = 16; o; o >>= 1) nfalse += __shfl_xor_sync(0xffffffffu, nfalse, o);
    if ((threadIdx.x & 31) == 0 && nfalse) atomicAdd(a.false_matches, nfalse);
}

template <int W, class C>
static lasagna_status launch_bucket_join_cfg(const BucketJoinArgs &args, cudaStream_t s)
{
    constexpr int NT = C::THREADS, HALF = C::HALF_;
    const size_t smem = (size_t)4 * HALF * 8 + (size_t)2 * NT * 8 + (size_t)C::SLOTS_ * 4 +
                        (size_t)2 * C::BLOOM * 4 + (size_t)(NT / 32) * BJ_QCAP * 2 +
                        (size_t)HALF * 2 + (size_t)2 * BJ_FILLS * 4;
    LSG_CUDA(cudaFuncSetAttribute(bucket_join_kernel<W, C>,
                                  cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0;
    LSG_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, bucket_join_kernel<W, C>, NT,
                                                           smem));
    per_sm = std::max(per_sm, 1);
    const uint64_t blocks =
        std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)num_sms() * per_sm, args.n_buckets));
    bucket_join_kernel<W, C><<<(unsigned)blocks, NT, smem, s>>>(args);
    LSG_LAUNCHED("bucket_join_kernel");
    return LASAGNA_OK;
}

lasagna_status launch_bucket_join(const BucketJoinArgs &args, cudaStream_t s)
{
    if (args.n_buckets == 0) return LASAGNA_OK;
    if (args.half_cap & 1) return LASAGNA_EINVAL; // sentinels need an even half capacity
    // CTA geometry: one 1024-thread CTA per SM (512 x 2 and 256 x 4 per SM with proportionally
    // smaller windows measured the same at cfg3: DESIGN.md 6.1)
    static const bool planner_builds = [] {
        const char *e = getenv("LASAGNA_BJ_PLANNER_BUILDS");
        return e && e[0] == '1';
    }();
    BucketJoinArgs a = args;
    a.planner_builds = planner_builds;
    return dispatch_W(args.j.L, [&](auto wc) -> lasagna_status {
        constexpr int W = decltype(wc)::value;
        return launch_bucket_join_cfg<W, BjCfg<1024, 4096, 4096, 2048>>(a, s);
    });
}


} // namespace lsg
