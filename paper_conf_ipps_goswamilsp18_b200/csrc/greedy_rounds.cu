// greedy_rounds.cu — a6/a7 per length: FAST_ROUNDS grid-wide locally-dominant rounds
// (greedy.cu's rule: propose the partner to both ends with an epoch-tagged atomicMax, accept
// the pairs chosen at both ends, drop pairs with a claimed end), then one CTA finishes the
// survivors (block-local rounds, then the sequential definition).
//
// The same kernels run the sharded greedy of the multi-GPU driver (the paper's
// reduce step P:L206-210 without its token): read end x is OWNED by rank x / slice, which
// holds best[], claimed[], succ[] and olen[] of its slice; every rank runs the rounds over the
// candidate pairs ITS join found and reaches the other ranks' slices through peer pointers
// (NVLink loads, stores and system-scope atomics).  A one-thread kernel per rank is the
// cross-rank barrier between the propose and accept phases (stream-ordered, no host
// synchronisation).  The survivors of every rank are gathered into rank 0's tail buffer and
// rank 0 finishes them.  The result equals the single-GPU greedy bit for bit: each round's
// accepted set depends only on the global live set, and every rank runs the same rounds with
// the same epochs.
//
// One launch may also run SEVERAL ranks (GreedyPeers::nranks_here > 1: blocks grouped by rank)
// so that the cross-rank protocol is tested on one GPU with plain device pointers.
#include <cstdio>
#include <utility>

#include "kernels.cuh"

namespace lsg {

namespace {

constexpr int GR_THREADS = 256;
constexpr int GR_K = 4;                // pairs per thread per trip (independent random loads)
constexpr uint32_t GR_TAIL_MAX = GR_TAIL_CAP; // live pairs (all ranks) handed to the one-CTA tail
constexpr int TL_THREADS = 1024;
constexpr uint32_t TL_SEQ_MAX = 64;    // the tail's sequential scan takes at most this many

__device__ __forceinline__ unsigned long long proposal(uint32_t epoch, uint32_t partner)
{
    return ((unsigned long long)epoch << 32) | (unsigned long long)(~partner);
}

// device-scope atomics on one GPU, system scope (peer memory over NVLink) across ranks
__device__ __forceinline__ void amax(unsigned long long *x, unsigned long long v, bool sys)
{
    if (sys) atomicMax_system(x, v);
    else atomicMax(x, v);
}
__device__ __forceinline__ void aor(uint32_t *x, uint32_t v, bool sys)
{
    if (sys) atomicOr_system(x, v);
    else atomicOr(x, v);
}

// MULTI: peer memory (system-scope atomics, uncached loads of state other ranks write);
// single GPU: device-scope atomics and ordinary (L1-cacheable) loads in the round kernels
template <bool MULTI>
struct Owner {
    const GreedyPeers *p;
    __device__ __forceinline__ uint32_t rank(uint32_t x) const
    {
        return MULTI ? (uint32_t)(x / p->slice) : 0u;
    }
    __device__ __forceinline__ uint64_t local(uint32_t x) const
    {
        return MULTI ? x % p->slice : x;
    }
    __device__ __forceinline__ bool claimed(uint32_t x) const
    {
        LSG_DCHECK(p->slice == 0 || x < p->slice * p->g);
        const uint64_t i = local(x);
        const uint32_t *w = p->r[rank(x)].claimed + (i >> 5);
        const uint32_t v = MULTI ? *(volatile const uint32_t *)w : *w;
        return (v >> (i & 31u)) & 1u;
    }
    __device__ __forceinline__ unsigned long long best_val(uint32_t x) const
    {
        const unsigned long long *b = best(x);
        return MULTI ? *(volatile const unsigned long long *)b : *b;
    }
    __device__ __forceinline__ unsigned long long *best(uint32_t x) const
    {
        LSG_DCHECK(p->slice == 0 || x < p->slice * p->g);
        return p->r[rank(x)].best + local(x);
    }
    __device__ __forceinline__ void propose(uint32_t a, uint32_t b, uint32_t epoch) const
    {
        amax(best(a), proposal(epoch, b), MULTI);
        amax(best(b), proposal(epoch, a), MULTI);
    }
    __device__ __forceinline__ void accept(uint32_t a, uint32_t b, uint8_t l) const
    {
        const uint32_t ra = rank(a), rb = rank(b);
        const uint64_t ia = local(a), ib = local(b);
        aor(p->r[ra].claimed + (ia >> 5), 1u << (ia & 31u), MULTI);
        aor(p->r[rb].claimed + (ib >> 5), 1u << (ib & 31u), MULTI);
        p->r[ra].succ[ia] = b ^ 1u, p->r[rb].succ[ib] = a ^ 1u; // a -> b^1, b -> a^1
        p->r[ra].olen[ia] = l, p->r[rb].olen[ib] = l;
    }
};

__device__ __forceinline__ unsigned long long vload(const unsigned long long *x)
{
    return *(volatile const unsigned long long *)x;
}

// Cross-rank barrier, thread 0 of one block per rank: every rank's writes to any slice (system
// fence) happen before every rank's reads after it.  Arrivals are counted on each rank's own
// word; its k-th barrier completes when g * k arrivals have landed.
__device__ __forceinline__ void xrank_sync(const GreedyPeers &p, uint32_t me)
{
    if (p.g == 1) return;
    __threadfence_system();
    for (uint32_t q = 0; q < p.g; ++q) atomicAdd_system(&p.r[q].ctr[PC_XARRIVE], 1ull);
    unsigned long long *mine = p.r[me].ctr;
    const unsigned long long target = (unsigned long long)p.g * (mine[PC_XCOUNT] + 1);
    while (vload(&mine[PC_XARRIVE]) < target) __nanosleep(64);
    mine[PC_XCOUNT] += 1;
    __threadfence_system();
}

// append the pairs r[k] with bit k of keepm set: one global atomic per block and trip
__device__ __forceinline__ void block_append(const unsigned long long (&r)[GR_K], uint32_t keepm,
                                             unsigned long long *out, unsigned long long *out_count,
                                             uint32_t *wsum, unsigned long long *sbase)
{
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const uint32_t nk = __popc(keepm);
    uint32_t x = nk;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) wsum[wid] = x;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t tot = 0;
        for (int w = 0; w < GR_THREADS / 32; ++w) {
            const uint32_t v = wsum[w];
            wsum[w] = tot;
            tot += v;
        }
        *sbase = tot ? atomicAdd(out_count, (unsigned long long)tot) : 0ull;
    }
    __syncthreads();
    unsigned long long pos = *sbase + wsum[wid] + x - nk;
#pragma unroll
    for (int k = 0; k < GR_K; ++k)
        if (keepm & (1u << k)) out[pos++] = r[k];
    __syncthreads();
}

// Round kernels (greedy.cu's rule and counter rotation), blocks grouped by rank.  Phase j
// (propose = even j, accept = odd j; FAST_ROUNDS rounds) reads list j % 2 == 0 ? pool : pool2
// with count slot j % 3, appends to the other list with count slot (j + 1) % 3, and block 0
// zeroes slot (j + 2) % 3 (written by phase j + 1, last read by phase j - 1: stream order).
// Slot 0 is the join's pool counter (in_count), slots 1 and 2 are ctr[PC_RING + 1, 2]; after
// three rounds (six phases) the survivors are in pool with their count in slot 0.
constexpr uint32_t FAST_ROUNDS = 3;

__device__ __forceinline__ unsigned long long *ring_slot(const PeerRank &R, uint32_t k)
{
    return k == 0 ? R.in_count : R.ctr + PC_RING + k;
}

// VW > 0 (first round with deferred verification): candidates are checked on the bases
// (read width VW words) before they propose; a rejected hit is dropped and counted
template <bool MULTI, int VW = 0>
__global__ void __launch_bounds__(GR_THREADS)
greedy_propose_kernel(GreedyPeers p, uint32_t j, uint8_t l)
{
    pdl_wait(); // launched with PDL after the previous round / the join
    pdl_trigger();
    __shared__ uint32_t wsum[GR_THREADS / 32];
    __shared__ unsigned long long sbase;
    const uint32_t me = p.rank0 + blockIdx.x / p.bpr;
    const uint32_t bl = blockIdx.x % p.bpr;
    const PeerRank &R = p.r[me];
    const Owner<MULTI> own{&p};
    const unsigned long long c = *ring_slot(R, j % 3);
    const unsigned long long m = c < p.cap ? c : p.cap;
    // the epoch of this round: every rank counts the same rounds
    const uint32_t epoch = (uint32_t)R.ctr[PC_EPOCH] + 1u + j / 2;
    if (bl == 0 && threadIdx.x == 0) {
        *ring_slot(R, (j + 2) % 3) = 0;
        atomicAdd(&R.ctr[PC_WORK], m);
        if (j == 0) { // first round of a length: |P_l| bookkeeping (VW > 0: counted below)
            if (VW == 0) atomicAdd(&R.ctr[PC_BOOK + 1], c);
            atomicMax(&R.ctr[PC_BOOK + 2], c);
        }
    }
    const unsigned long long *X = R.pool;
    unsigned long long *outc = ring_slot(R, (j + 1) % 3);
    uint32_t ntrue = 0, nbad = 0; // VW > 0
    const uint64_t stride = (uint64_t)p.bpr * GR_THREADS * GR_K;
    for (uint64_t i0 = (uint64_t)bl * GR_THREADS * GR_K + threadIdx.x; i0 - threadIdx.x < m;
         i0 += stride) { // block-uniform trip count
        unsigned long long r[GR_K];
        bool dead[GR_K];
#pragma unroll
        for (int k = 0; k < GR_K; ++k) {
            const uint64_t i = i0 + (uint64_t)k * GR_THREADS;
            r[k] = i < m ? X[i] : ~0ull;
        }
        if constexpr (VW > 0) {
            // the bases decide (as the join's verify_staged would): a pair (u, b) of read ends
            // is the directed overlap (u, b ^ 1, l)
#pragma unroll
            for (int k = 0; k < GR_K; ++k)
                if (r[k] != ~0ull) {
                    if (verify_overlap<VW>(p.vpacked, p.vstride, p.vL, (uint32_t)(r[k] >> 32),
                                           (uint32_t)r[k] ^ 1u, l))
                        ++ntrue;
                    else
                        ++nbad, r[k] = ~0ull;
                }
        }
#pragma unroll
        for (int k = 0; k < GR_K; ++k)
            dead[k] = r[k] == ~0ull || own.claimed((uint32_t)(r[k] >> 32)) ||
                      own.claimed((uint32_t)r[k]);
        uint32_t keepm = 0;
#pragma unroll
        for (int k = 0; k < GR_K; ++k) {
            if (dead[k]) continue;
            own.propose((uint32_t)(r[k] >> 32), (uint32_t)r[k], epoch);
            keepm |= 1u << k;
        }
        block_append(r, keepm, R.pool2, outc, wsum, &sbase);
    }
    if constexpr (VW > 0) {
        for (int o = 16; o; o >>= 1) {
            ntrue += __shfl_xor_sync(0xffffffffu, ntrue, o);
            nbad += __shfl_xor_sync(0xffffffffu, nbad, o);
        }
        if ((threadIdx.x & 31) == 0) {
            if (ntrue) atomicAdd(&R.ctr[PC_BOOK + 1], (unsigned long long)ntrue);
            if (nbad) atomicAdd(p.vfalse, (unsigned long long)nbad);
        }
    }
    if (MULTI) __threadfence_system(); // proposals to peers' best[] before the barrier kernel
}

template <bool MULTI>
__global__ void __launch_bounds__(GR_THREADS)
greedy_accept_kernel(GreedyPeers p, uint32_t j, uint8_t l)
{
    pdl_wait(); // launched with PDL after the previous round / the join
    pdl_trigger();
    __shared__ uint32_t wsum[GR_THREADS / 32];
    __shared__ unsigned long long sbase;
    const uint32_t me = p.rank0 + blockIdx.x / p.bpr;
    const uint32_t bl = blockIdx.x % p.bpr;
    const PeerRank &R = p.r[me];
    const Owner<MULTI> own{&p};
    const unsigned long long c = *ring_slot(R, j % 3);
    const unsigned long long m = c < p.cap ? c : p.cap;
    const uint32_t epoch = (uint32_t)R.ctr[PC_EPOCH] + 1u + j / 2;
    if (bl == 0 && threadIdx.x == 0) *ring_slot(R, (j + 2) % 3) = 0;
    unsigned long long *outc = ring_slot(R, (j + 1) % 3);
    uint32_t acc = 0;
    const uint64_t stride = (uint64_t)p.bpr * GR_THREADS * GR_K;
    for (uint64_t i0 = (uint64_t)bl * GR_THREADS * GR_K + threadIdx.x; i0 - threadIdx.x < m;
         i0 += stride) {
        unsigned long long r[GR_K], ba[GR_K], bb[GR_K];
#pragma unroll
        for (int k = 0; k < GR_K; ++k) {
            const uint64_t i = i0 + (uint64_t)k * GR_THREADS;
            r[k] = i < m ? R.pool2[i] : ~0ull;
        }
#pragma unroll
        for (int k = 0; k < GR_K; ++k)
            if (r[k] != ~0ull)
                ba[k] = own.best_val((uint32_t)(r[k] >> 32)), bb[k] = own.best_val((uint32_t)r[k]);
        uint32_t keepm = 0;
#pragma unroll
        for (int k = 0; k < GR_K; ++k) {
            if (r[k] == ~0ull) continue;
            const uint32_t a = (uint32_t)(r[k] >> 32), b = (uint32_t)r[k];
            if (ba[k] == proposal(epoch, b) && bb[k] == proposal(epoch, a)) {
                own.accept(a, b, l);
                ++acc;
            } else {
                keepm |= 1u << k;
            }
        }
        block_append(r, keepm, R.pool, outc, wsum, &sbase);
    }
    for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if ((threadIdx.x & 31) == 0 && acc) atomicAdd(&R.ctr[PC_BOOK + 0], (unsigned long long)acc);
    if (MULTI) __threadfence_system(); // claims / edges on peers before the barrier kernel
}

// one thread per rank: the cross-rank barrier between phases (g > 1)
__global__ void greedy_xbar_kernel(GreedyPeers p)
{
    xrank_sync(p, p.rank0 + blockIdx.x);
}

// One block-local locally-dominant round over cur[0..live) (claimed pairs dropped, accepted
// pairs claimed, survivors appended to other); returns the survivor count.  With MULTI, the
// ranks' tail blocks run their rounds in lockstep: a cross-rank barrier between the propose
// and accept halves and after the accept half.
template <bool MULTI>
__device__ uint32_t tail_round(const GreedyPeers &p, uint32_t me, const Owner<MULTI> &own,
                               const unsigned long long *cur, uint32_t live,
                               unsigned long long *other, uint32_t epoch, uint8_t l,
                               uint32_t *s_live, uint32_t *s_acc, bool xsync)
{
    for (uint32_t i = threadIdx.x; i < live; i += TL_THREADS) {
        const unsigned long long r = cur[i];
        const uint32_t a = (uint32_t)(r >> 32), b = (uint32_t)r;
        if (own.claimed(a) || own.claimed(b)) continue;
        own.propose(a, b, epoch);
    }
    if (threadIdx.x == 0) *s_live = 0;
    if (MULTI) __threadfence_system();
    __syncthreads();
    if (MULTI && xsync && threadIdx.x == 0) xrank_sync(p, me);
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < live; i += TL_THREADS) {
        const unsigned long long r = cur[i];
        const uint32_t a = (uint32_t)(r >> 32), b = (uint32_t)r;
        if (own.claimed(a) || own.claimed(b)) continue;
        if (vload(own.best(a)) == proposal(epoch, b) && vload(own.best(b)) == proposal(epoch, a)) {
            own.accept(a, b, l);
            atomicAdd(s_acc, 1u);
        } else {
            other[atomicAdd(s_live, 1u)] = r;
        }
    }
    if (MULTI) __threadfence_system();
    __syncthreads();
    if (MULTI && xsync && threadIdx.x == 0) xrank_sync(p, me);
    __syncthreads();
    return *s_live;
}

// The tail (one CTA per rank).  MULTI: while more than GR_TAIL_MAX pairs are live over all
// ranks, every rank's block runs block-local rounds on its own survivors (in lockstep); then
// the survivors are gathered into rank 0's tail buffer.  Rank 0 (or the single GPU) then runs
// block-local rounds while more than TL_SEQ_MAX pairs are live, and finally the sequential
// definition (bitonic sort by (a, b); thread 0 visits them in order).
template <bool MULTI>
__global__ void __launch_bounds__(TL_THREADS)
greedy_tail_kernel(GreedyPeers p, uint8_t l)
{
    pdl_wait(); // launched with PDL after the previous round / the join
    pdl_trigger();
    __shared__ unsigned long long s[TL_SEQ_MAX];
    __shared__ unsigned long long offs[MAX_PEERS + 1];
    __shared__ uint32_t s_live, s_acc;
    const uint32_t me = p.rank0 + blockIdx.x;
    const PeerRank &R = p.r[me];
    const Owner<MULTI> own{&p};
    uint32_t epoch = (uint32_t)R.ctr[PC_EPOCH] + 1u + FAST_ROUNDS;
    uint32_t rounds = FAST_ROUNDS;
    const unsigned long long c0 = *R.in_count;
    uint32_t live = (uint32_t)(c0 < p.cap ? c0 : p.cap); // my survivors of the fast rounds
    unsigned long long *cur = R.pool, *other = R.pool2;
    if (threadIdx.x == 0) {
        s_acc = 0;
        if (live) atomicAdd(&R.ctr[PC_WORK], (unsigned long long)live);
    }
    if (MULTI) {
        for (;;) {
            // every rank's live count, visible to all
            if (threadIdx.x == 0) {
                R.ctr[PC_TAILIN] = live;
                xrank_sync(p, me);
                unsigned long long o = 0;
                for (uint32_t q = 0; q < p.g; ++q) {
                    offs[q] = o;
                    o += vload(&p.r[q].ctr[PC_TAILIN]);
                }
                offs[p.g] = o;
            }
            __syncthreads();
            if (offs[p.g] <= GR_TAIL_MAX) break;
            live = tail_round<MULTI>(p, me, own, cur, live, other, epoch, l, &s_live, &s_acc, true);
            unsigned long long *t = cur;
            cur = other;
            other = t;
            ++epoch;
            ++rounds;
            if (threadIdx.x == 0 && live) atomicAdd(&R.ctr[PC_WORK], (unsigned long long)live);
            // (every rank read the counts before the barriers inside tail_round)
        }
        // survivors of every rank -> rank 0's tail buffer (remote stores)
        unsigned long long *gathered = p.r[0].tail;
        for (uint32_t i = threadIdx.x; i < live; i += TL_THREADS) gathered[offs[me] + i] = cur[i];
        __threadfence_system();
        __syncthreads();
        if (threadIdx.x == 0) xrank_sync(p, me);
        __syncthreads();
        if (me == 0) {
            cur = gathered;
            other = R.pool2;
            live = (uint32_t)offs[p.g];
        }
    }
    if (me == 0 && live) {
        while (live > TL_SEQ_MAX) {
            // rank 0 alone: no cross-rank barriers inside (the others wait at the final one)
            live = tail_round<MULTI>(p, me, own, cur, live, other, epoch, l, &s_live, &s_acc, false);
            unsigned long long *t = cur;
            cur = other;
            other = t;
            ++epoch;
            ++rounds;
            if (threadIdx.x == 0 && live) atomicAdd(&R.ctr[PC_WORK], (unsigned long long)live);
        }
        if (live) {
            // the sequential definition over <= TL_SEQ_MAX pairs in (a, b) order
            uint32_t P = 1;
            while (P < live) P <<= 1;
            for (uint32_t i = threadIdx.x; i < P; i += TL_THREADS) s[i] = i < live ? cur[i] : ~0ull;
            __syncthreads();
            for (uint32_t k = 2; k <= P; k <<= 1)
                for (uint32_t j = k >> 1; j > 0; j >>= 1) {
                    for (uint32_t i = threadIdx.x; i < P; i += TL_THREADS) {
                        const uint32_t ixj = i ^ j;
                        if (ixj > i) {
                            const bool up = (i & k) == 0;
                            const unsigned long long x = s[i], y = s[ixj];
                            if ((x > y) == up) s[i] = y, s[ixj] = x;
                        }
                    }
                    __syncthreads();
                }
            // claimed state of every end before the scan, read in parallel
            __shared__ uint8_t cl[2 * TL_SEQ_MAX];
            for (uint32_t i = threadIdx.x; i < 2 * live; i += TL_THREADS) {
                const unsigned long long r = s[i >> 1];
                cl[i] = own.claimed((i & 1) ? (uint32_t)r : (uint32_t)(r >> 32)) ? 1 : 0;
            }
            __syncthreads();
            if (threadIdx.x == 0) {
                uint32_t acc = 0;
                uint32_t taken[2 * TL_SEQ_MAX];
                uint32_t nt = 0;
                for (uint32_t i = 0; i < live; ++i) {
                    const uint32_t a = (uint32_t)(s[i] >> 32), b = (uint32_t)s[i];
                    bool busy = cl[2 * i] || cl[2 * i + 1];
                    for (uint32_t t = 0; t < nt && !busy; ++t) busy = taken[t] == a || taken[t] == b;
                    if (busy) continue;
                    own.accept(a, b, l);
                    taken[nt++] = a;
                    taken[nt++] = b;
                    ++acc;
                }
                s_acc += acc;
            }
            ++rounds;
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        if (s_acc) atomicAdd(&R.ctr[PC_BOOK + 0], (unsigned long long)s_acc);
        atomicMax(&R.ctr[PC_BOOK + 3], (unsigned long long)rounds);
        // the next length starts after the last epoch any rank used (rank 0's rounds are a
        // superset of the others'): the same on every rank
        if (me == 0) R.ctr[PC_TAILEPOCH] = epoch - 1u;
        if (MULTI) {
            __threadfence_system();
            xrank_sync(p, me);
        }
        R.ctr[PC_EPOCH] = vload(&p.r[0].ctr[PC_TAILEPOCH]);
    }
}

} // namespace

lasagna_status greedy_length_peers(const GreedyPeers &p, uint8_t l, cudaStream_t s)
{
    if (p.g < 1 || p.g > MAX_PEERS || p.nranks_here < 1 || p.rank0 + p.nranks_here > p.g) {
        set_error("greedy: bad rank layout (g=%u)", p.g);
        return LASAGNA_EINVAL;
    }
    GreedyPeers q = p;
    // blocks per SM of the first round (the whole pool) and of the later rounds (survivors);
    // LASAGNA_GREEDY_BPS=a,b overrides (A/B only)
    static const std::pair<uint32_t, uint32_t> bps = [] {
        uint32_t a0 = 8, a1 = 4; // first round: 8 blocks per SM, later rounds 4 (r02t A/B)
        if (const char *e = getenv("LASAGNA_GREEDY_BPS")) sscanf(e, "%u,%u", &a0, &a1);
        return std::make_pair(std::max(1u, a0), std::max(1u, a1));
    }();
    auto per_rank = [&](uint32_t per_sm) {
        const uint64_t want = std::max<uint64_t>(
            1, std::min<uint64_t>(ceil_div(q.cap, GR_THREADS * GR_K), (uint64_t)num_sms() * per_sm));
        return (uint32_t)std::max<uint64_t>(1, want / q.nranks_here);
    };
    const uint32_t bpr0 = q.bpr ? q.bpr : per_rank(bps.first);
    const uint32_t bpr1 = q.bpr ? q.bpr : per_rank(bps.second);
    // PDL between the single-GPU rounds (LASAGNA_PDL=0: plain launches, A/B only)
    static const bool use_pdl = [] {
        const char *e = getenv("LASAGNA_PDL");
        return !(e && e[0] == '0');
    }();
    auto run = [&](auto multi) -> lasagna_status {
        constexpr bool M = decltype(multi)::value;
        for (uint32_t r = 0; r < FAST_ROUNDS; ++r) {
            q.bpr = r == 0 ? bpr0 : bpr1;
            const dim3 grid(q.bpr * q.nranks_here);
            if (!M && r == 0 && q.vpacked) {
                // first round with deferred verification: the kernel for the read width
                lasagna_status rc = dispatch_W(q.vL, [&](auto wc) -> lasagna_status {
                    constexpr int VW = decltype(wc)::value;
                    if (!use_pdl) greedy_propose_kernel<false, VW><<<grid, GR_THREADS, 0, s>>>(q, 0, l);
                    else LSG_CUDA(launch_pdl(greedy_propose_kernel<false, VW>, grid, dim3(GR_THREADS),
                                             0, s, q, 0u, l));
                    return LASAGNA_OK;
                });
                if (rc != LASAGNA_OK) return rc;
            } else if (M || !use_pdl) {
                greedy_propose_kernel<M><<<grid, GR_THREADS, 0, s>>>(q, 2 * r, l);
            } else {
                LSG_CUDA(launch_pdl(greedy_propose_kernel<M>, grid, dim3(GR_THREADS), 0, s, q, 2 * r, l));
            }
            LSG_LAUNCHED("greedy_propose_kernel");
            if (M) {
                greedy_xbar_kernel<<<q.nranks_here, 1, 0, s>>>(q);
                LSG_LAUNCHED("greedy_xbar_kernel");
            }
            q.bpr = bpr1;
            const dim3 grid2(q.bpr * q.nranks_here);
            if (M || !use_pdl) greedy_accept_kernel<M><<<grid2, GR_THREADS, 0, s>>>(q, 2 * r + 1, l);
            else LSG_CUDA(launch_pdl(greedy_accept_kernel<M>, grid2, dim3(GR_THREADS), 0, s, q,
                                     2 * r + 1, l));
            LSG_LAUNCHED("greedy_accept_kernel");
            if (M) {
                greedy_xbar_kernel<<<q.nranks_here, 1, 0, s>>>(q);
                LSG_LAUNCHED("greedy_xbar_kernel");
            }
        }
        if (M || !use_pdl) greedy_tail_kernel<M><<<q.nranks_here, TL_THREADS, 0, s>>>(q, l);
        else LSG_CUDA(launch_pdl(greedy_tail_kernel<M>, dim3(q.nranks_here), dim3(TL_THREADS), 0, s,
                                 q, l));
        LSG_LAUNCHED("greedy_tail_kernel");
        return LASAGNA_OK;
    };
    return q.g > 1 ? run(std::true_type{}) : run(std::false_type{});
    return LASAGNA_OK;
}

} // namespace lsg
