// greedy_rounds.cu — a6/a7 as TWO launches per length: one persistent cooperative kernel runs
// the locally-dominant rounds (greedy.cu's rule) grid-wide until at most TAIL_MAX pairs are
// live, then one CTA finishes them (block-local rounds, then the sequential definition).
//
// The same kernels run the sharded greedy of the multi-GPU driver (the paper's
// reduce step P:L206-210 without its token): read end x is OWNED by rank x / slice, which
// holds best[], claimed[], succ[] and olen[] of its slice; every rank runs the rounds over the
// candidate pairs ITS join found and reaches the other ranks' slices through peer pointers
// (NVLink loads, stores and atomics).  Ranks meet at a cross-rank barrier between the propose
// and accept phases; the round count and the tail decision use the sum of every rank's live
// count, so all ranks run the same rounds with the same epochs.  The survivors of every rank
// are gathered into rank 0's tail buffer, and rank 0 finishes them.  The result equals the
// single-GPU greedy bit for bit: a round's accepted set depends only on the global live set.
//
// One launch may also run SEVERAL ranks (GreedyPeers::nranks_here > 1: blocks grouped by rank)
// so that the cross-rank protocol is tested on one GPU with plain device pointers.
#include <cooperative_groups.h>

#include "kernels.cuh"

namespace lsg {

namespace {

constexpr int GR_THREADS = 512;
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

struct Owner {
    const GreedyPeers *p;
    __device__ __forceinline__ uint32_t rank(uint32_t x) const
    {
        return p->g == 1 ? 0u : (uint32_t)(x / p->slice);
    }
    __device__ __forceinline__ uint64_t local(uint32_t x) const
    {
        return p->g == 1 ? x : x % p->slice;
    }
    __device__ __forceinline__ bool claimed(uint32_t x) const
    {
        const uint64_t i = local(x);
        const uint32_t w = *((volatile const uint32_t *)p->r[rank(x)].claimed + (i >> 5));
        return (w >> (i & 31u)) & 1u;
    }
    __device__ __forceinline__ unsigned long long *best(uint32_t x) const
    {
        return p->r[rank(x)].best + local(x);
    }
    __device__ __forceinline__ void propose(uint32_t a, uint32_t b, uint32_t epoch) const
    {
        amax(best(a), proposal(epoch, b), p->g > 1);
        amax(best(b), proposal(epoch, a), p->g > 1);
    }
    __device__ __forceinline__ void accept(uint32_t a, uint32_t b, uint8_t l) const
    {
        const uint32_t ra = rank(a), rb = rank(b);
        const uint64_t ia = local(a), ib = local(b);
        aor(p->r[ra].claimed + (ia >> 5), 1u << (ia & 31u), p->g > 1);
        aor(p->r[rb].claimed + (ib >> 5), 1u << (ib & 31u), p->g > 1);
        p->r[ra].succ[ia] = b ^ 1u, p->r[rb].succ[ib] = a ^ 1u; // a -> b^1, b -> a^1
        p->r[ra].olen[ia] = l, p->r[rb].olen[ib] = l;
    }
};

__device__ __forceinline__ unsigned long long vload(const unsigned long long *x)
{
    return *(volatile const unsigned long long *)x;
}

// Barrier of the `nb` blocks of one rank (co-resident: cooperative launch).
__device__ __forceinline__ void group_sync(unsigned long long *ctr, uint32_t nb)
{
    __syncthreads();
    if (threadIdx.x == 0) {
        const unsigned long long gen = vload(&ctr[PC_GEN]);
        __threadfence();
        if (atomicAdd(&ctr[PC_ARRIVE], 1ull) == nb - 1) {
            ctr[PC_ARRIVE] = 0;
            __threadfence();
            atomicAdd(&ctr[PC_GEN], 1ull);
        } else {
            while (vload(&ctr[PC_GEN]) == gen) __nanosleep(32);
        }
        __threadfence();
    }
    __syncthreads();
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

// all ranks: group barrier, cross-rank barrier by block 0, group barrier
__device__ __forceinline__ void all_sync(const GreedyPeers &p, uint32_t me, uint32_t bl)
{
    unsigned long long *ctr = p.r[me].ctr;
    group_sync(ctr, p.bpr);
    if (p.g > 1) {
        if (bl == 0 && threadIdx.x == 0) xrank_sync(p, me);
        group_sync(ctr, p.bpr);
    }
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

// Rounds of one length.  Phase j (propose = even j, accept = odd j) reads the count its
// predecessor wrote and appends to ring slot j mod 3; during phase j block 0 zeroes slot
// (j + 1) mod 3, whose last reader was phase j - 1 (ordered by the barrier in between).
// Phase 0 reads the join's pool count (in_count).
__global__ void __launch_bounds__(GR_THREADS)
greedy_rounds_kernel(GreedyPeers p, uint8_t l)
{
    __shared__ uint32_t wsum[GR_THREADS / 32];
    __shared__ unsigned long long sbase;
    const uint32_t me = p.rank0 + blockIdx.x / p.bpr;
    const uint32_t bl = blockIdx.x % p.bpr;
    const PeerRank &R = p.r[me];
    unsigned long long *ctr = R.ctr;
    const Owner own{&p};
    // PC_EPOCH = the last epoch used (0: none yet); read by every block before any update
    const uint32_t epoch0 = (uint32_t)ctr[PC_EPOCH] + 1u;
    const unsigned long long c_in = *R.in_count;
    const unsigned long long m_in = c_in < p.cap ? c_in : p.cap;
    if (bl == 0 && threadIdx.x == 0) {
        atomicAdd(&ctr[PC_BOOK + 1], c_in);
        atomicMax(&ctr[PC_BOOK + 2], c_in);
    }
    const uint64_t stride = (uint64_t)p.bpr * GR_THREADS * GR_K;
    uint32_t round = 0;
    for (uint32_t j = 0;; j += 2, ++round) {
        const uint32_t epoch = epoch0 + round;
        // ---- propose: X (input) -> Y (pool2), dropping pairs with a claimed end
        {
            const unsigned long long *X = R.pool;
            const unsigned long long m = j == 0 ? m_in : vload(&ctr[PC_RING + (j + 2) % 3]);
            unsigned long long *outc = &ctr[PC_RING + j % 3];
            if (bl == 0 && threadIdx.x == 0) {
                ctr[PC_RING + (j + 1) % 3] = 0;
                atomicAdd(&ctr[PC_WORK], m);
            }
            for (uint64_t i0 = (uint64_t)bl * GR_THREADS * GR_K + threadIdx.x; i0 - threadIdx.x < m;
                 i0 += stride) {
                unsigned long long r[GR_K];
                bool dead[GR_K];
#pragma unroll
                for (int k = 0; k < GR_K; ++k) {
                    const uint64_t i = i0 + (uint64_t)k * GR_THREADS;
                    r[k] = i < m ? X[i] : ~0ull;
                }
#pragma unroll
                for (int k = 0; k < GR_K; ++k)
                    dead[k] = r[k] == ~0ull || own.claimed((uint32_t)(r[k] >> 32)) ||
                              own.claimed((uint32_t)r[k]);
                uint32_t keepm = 0;
#pragma unroll
                for (int k = 0; k < GR_K; ++k) {
                    if (dead[k]) continue;
                    const uint32_t a = (uint32_t)(r[k] >> 32), b = (uint32_t)r[k];
                    own.propose(a, b, epoch);
                    keepm |= 1u << k;
                }
                block_append(r, keepm, R.pool2, outc, wsum, &sbase);
            }
        }
        all_sync(p, me, bl);
        // ---- accept: Y -> survivors back into X
        {
            const unsigned long long *Y = R.pool2;
            const unsigned long long m = vload(&ctr[PC_RING + j % 3]);
            unsigned long long *outc = &ctr[PC_RING + (j + 1) % 3];
            if (bl == 0 && threadIdx.x == 0) ctr[PC_RING + (j + 2) % 3] = 0;
            uint32_t acc = 0;
            for (uint64_t i0 = (uint64_t)bl * GR_THREADS * GR_K + threadIdx.x; i0 - threadIdx.x < m;
                 i0 += stride) {
                unsigned long long r[GR_K], ba[GR_K], bb[GR_K];
#pragma unroll
                for (int k = 0; k < GR_K; ++k) {
                    const uint64_t i = i0 + (uint64_t)k * GR_THREADS;
                    r[k] = i < m ? Y[i] : ~0ull;
                }
#pragma unroll
                for (int k = 0; k < GR_K; ++k)
                    if (r[k] != ~0ull)
                        ba[k] = vload(own.best((uint32_t)(r[k] >> 32))),
                        bb[k] = vload(own.best((uint32_t)r[k]));
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
            if ((threadIdx.x & 31) == 0 && acc) atomicAdd(&ctr[PC_BOOK + 0], (unsigned long long)acc);
        }
        all_sync(p, me, bl);
        // every rank sums the same counts: the same decision everywhere
        unsigned long long live = 0;
        for (uint32_t q = 0; q < p.g; ++q) live += vload(&p.r[q].ctr[PC_RING + (j + 1) % 3]);
        if (live <= GR_TAIL_MAX) {
            // the tail kernel reads the survivors' count from PC_TAILIN; the next length starts
            // with a zero ring
            // (peers may still read the ring: the tail kernel zeroes it after its first
            // cross-rank barrier)
            group_sync(ctr, p.bpr); // every block has read epoch0 and the counts
            if (bl == 0 && threadIdx.x == 0) {
                ctr[PC_TAILIN] = ctr[PC_RING + (j + 1) % 3];
                ctr[PC_EPOCH] = epoch0 + round;
                ctr[PC_ROUNDS] = round + 1;
            }
            return;
        }
    }
}

// The tail (one CTA per rank): ranks > 0 copy their survivors into rank 0's tail buffer;
// rank 0 runs block-local rounds while more than TL_SEQ_MAX pairs are live, then the
// sequential definition (bitonic sort by (a, b); thread 0 visits them in order, with the
// ends it claims kept in shared memory).
__global__ void __launch_bounds__(TL_THREADS)
greedy_tail_kernel(GreedyPeers p, uint8_t l)
{
    __shared__ unsigned long long s[GR_TAIL_MAX];
    __shared__ unsigned long long offs[MAX_PEERS + 1];
    __shared__ uint32_t s_live, s_acc;
    const uint32_t me = p.rank0 + blockIdx.x;
    const PeerRank &R = p.r[me];
    const Owner own{&p};
    if (threadIdx.x == 0) {
        xrank_sync(p, me); // every rank's rounds kernel has published its survivor count
        R.ctr[PC_RING + 0] = R.ctr[PC_RING + 1] = R.ctr[PC_RING + 2] = 0; // for the next length
        unsigned long long o = 0;
        for (uint32_t q = 0; q < p.g; ++q) {
            offs[q] = o;
            o += vload(&p.r[q].ctr[PC_TAILIN]);
        }
        offs[p.g] = o;
        s_acc = 0;
    }
    __syncthreads();
    const uint32_t total = (uint32_t)offs[p.g];
    unsigned long long *gathered = p.r[0].tail;
    if (p.g > 1) {
        // survivors of every rank -> rank 0's tail buffer (remote stores)
        const uint32_t mine = (uint32_t)(offs[me + 1] - offs[me]);
        for (uint32_t i = threadIdx.x; i < mine; i += TL_THREADS) gathered[offs[me] + i] = R.pool[i];
        __syncthreads();
        if (threadIdx.x == 0) xrank_sync(p, me);
        __syncthreads();
    } else {
        gathered = R.pool;
    }
    uint32_t rounds = 0;
    if (me == 0 && total) {
        unsigned long long *cur = gathered, *other = R.pool2;
        uint32_t live = total;
        uint32_t epoch = (uint32_t)R.ctr[PC_EPOCH] + 1u;
        if (threadIdx.x == 0) atomicAdd(&R.ctr[PC_WORK], (unsigned long long)live);
        while (live > TL_SEQ_MAX) {
            for (uint32_t i = threadIdx.x; i < live; i += TL_THREADS) {
                const unsigned long long r = cur[i];
                const uint32_t a = (uint32_t)(r >> 32), b = (uint32_t)r;
                if (own.claimed(a) || own.claimed(b)) continue;
                own.propose(a, b, epoch);
            }
            if (threadIdx.x == 0) s_live = 0;
            __threadfence_system();
            __syncthreads();
            for (uint32_t i = threadIdx.x; i < live; i += TL_THREADS) {
                const unsigned long long r = cur[i];
                const uint32_t a = (uint32_t)(r >> 32), b = (uint32_t)r;
                if (own.claimed(a) || own.claimed(b)) continue;
                if (vload(own.best(a)) == proposal(epoch, b) && vload(own.best(b)) == proposal(epoch, a)) {
                    own.accept(a, b, l);
                    atomicAdd(&s_acc, 1u);
                } else {
                    other[atomicAdd(&s_live, 1u)] = r;
                }
            }
            __threadfence_system();
            __syncthreads();
            live = s_live;
            if (threadIdx.x == 0 && live) atomicAdd(&R.ctr[PC_WORK], (unsigned long long)live);
            unsigned long long *t = cur;
            cur = other;
            other = t;
            ++epoch;
            ++rounds;
            __syncthreads();
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
            // claimed state of every end before the scan, read in parallel (remote reads)
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
        __syncthreads();
        if (threadIdx.x == 0) R.ctr[PC_EPOCH] = epoch - 1u;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        if (s_acc) atomicAdd(&R.ctr[PC_BOOK + 0], (unsigned long long)s_acc);
        atomicMax(&R.ctr[PC_BOOK + 3], R.ctr[PC_ROUNDS] + rounds);
        // every rank continues with the same epoch as rank 0
        if (p.g > 1) {
            __threadfence_system();
            xrank_sync(p, me);
            R.ctr[PC_EPOCH] = vload(&p.r[0].ctr[PC_EPOCH]);
        }
    }
}

} // namespace

int greedy_rounds_blocks_per_sm()
{
    static const int v = [] {
        int b = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, greedy_rounds_kernel, GR_THREADS, 0);
        return std::max(1, std::min(b, 2));
    }();
    return v;
}

lasagna_status greedy_length_peers(const GreedyPeers &p, uint8_t l, cudaStream_t s)
{
    if (p.g < 1 || p.g > MAX_PEERS || p.nranks_here < 1 || p.rank0 + p.nranks_here > p.g) {
        set_error("greedy: bad rank layout (g=%u)", p.g);
        return LASAGNA_EINVAL;
    }
    GreedyPeers q = p;
    if (q.bpr == 0) {
        // blocks per rank: every block of the launch co-resident (cooperative launch), and at
        // most half of the device, so that two such launches (pipelined batches on two
        // streams) always fit side by side and cannot deadlock on each other's barriers
        const int per = num_sms() * greedy_rounds_blocks_per_sm() / 2;
        q.bpr = (uint32_t)std::max(1, per / (int)q.nranks_here);
    }
    void *args[] = {(void *)&q, (void *)&l};
    LSG_CUDA(cudaLaunchCooperativeKernel((const void *)greedy_rounds_kernel,
                                         dim3(q.bpr * q.nranks_here), dim3(GR_THREADS), args, 0, s));
    LSG_LAUNCHED("greedy_rounds_kernel");
    greedy_tail_kernel<<<q.nranks_here, TL_THREADS, 0, s>>>(q, l);
    LSG_LAUNCHED("greedy_tail_kernel");
    return LASAGNA_OK;
}

} // namespace lsg
