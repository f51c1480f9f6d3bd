// greedy.cu — a6/a7: the greedy edge claim ("longest overlap" P:L39; lengths in
// descending order P:L152) on the GPU with atomics, instead of the paper's host loop
// (P:L170-172 — on B200 the 5-byte-per-vertex graph fits in HBM).
//
// Sequential definition (R7, R10): visit the read-end pairs of one length in (a, b) order
// and accept a pair iff both read ends are free.  GPU version: locally-dominant rounds.
// Per round every live pair {a, b} proposes its partner id to both ends with 64-bit-free
// 32-bit atomicMin; a pair whose two ends both chose each other is the minimum live pair at
// both ends (ordering pairs at a fixed end by partner id == the (min, max) order), so the
// sequential greedy accepts it too; accept those, drop pairs with a claimed end, repeat.
// The minimum live pair is always accepted, so every round makes progress; when few pairs
// remain the tail runs the sequential definition on one CTA (bitonic sort + scan).
#include "kernels.cuh"

namespace lsg {

// Proposals are epoch-tagged 64-bit words best[x] = (epoch << 32) | ~partner combined with
// atomicMax: within a round the largest word is the smallest partner, and words of earlier
// rounds (smaller epochs) lose automatically, so best[] is never reset between rounds or
// lengths (it is zeroed once per call).  No host synchronisation anywhere: every kernel
// reads its pair count from device memory.
__device__ __forceinline__ unsigned long long proposal(uint32_t epoch, uint32_t partner)
{
    return ((unsigned long long)epoch << 32) | (unsigned long long)(~partner);
}

// Both round kernels are bound by the latency of random accesses (claimed[], best[] over
// 2n read ends): each thread handles GK pairs per trip and issues all their loads before
// using any, so a warp keeps 4x more random requests in flight.
constexpr int GREEDY_THREADS = 256;
constexpr int GK = 4;

// claimed read ends: a bitmap of 2n bits (8.7 MB at cfg3: L2-resident, unlike a byte per end)
__device__ __forceinline__ bool is_claimed(const uint32_t *cl, uint32_t x)
{
    return (cl[x >> 5] >> (x & 31u)) & 1u;
}
__device__ __forceinline__ void set_claimed(uint32_t *cl, uint32_t x)
{
    atomicOr(&cl[x >> 5], 1u << (x & 31u));
}

// Append the pairs r[k] with bit k of keepm set to out[]: one global atomic per block and
// loop trip (a per-thread or per-warp atomic on the single counter serialises at L2).  Called
// by every thread of the block (block-uniform trip counts).
__device__ __forceinline__ void block_append(const unsigned long long (&r)[GK], uint32_t keepm,
                                             unsigned long long *out, unsigned long long *out_count)
{
    __shared__ uint32_t wsum[GREEDY_THREADS / 32];
    __shared__ unsigned long long sbase;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const uint32_t nk = __popc(keepm);
    uint32_t x = nk; // warp inclusive scan of the counts
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) wsum[wid] = x;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t tot = 0;
        for (int w = 0; w < GREEDY_THREADS / 32; ++w) {
            const uint32_t v = wsum[w];
            wsum[w] = tot;
            tot += v;
        }
        sbase = tot ? atomicAdd(out_count, (unsigned long long)tot) : 0ull;
    }
    __syncthreads();
    unsigned long long pos = sbase + wsum[wid] + x - nk;
#pragma unroll
    for (int k = 0; k < GK; ++k)
        if (keepm & (1u << k)) out[pos++] = r[k];
    __syncthreads(); // wsum / sbase reuse
}

// Round part 1: every pair with both ends free proposes its partner to both ends and is
// appended to the round's live list (dead pairs — an end claimed by a longer length or an
// earlier round — are dropped here, once).  *reset is the counter two kernels ahead.
__global__ void __launch_bounds__(GREEDY_THREADS)
greedy_propose(const unsigned long long *pairs, const unsigned long long *count,
               unsigned long long cap, const uint32_t *claimed, unsigned long long *best,
               uint32_t epoch, unsigned long long *live, unsigned long long *live_count,
               unsigned long long *reset, unsigned long long *book, unsigned long long *work)
{
    const unsigned long long c = *count;
    const unsigned long long m = c < cap ? c : cap;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        *reset = 0;
        atomicAdd(work, m);
        if (book) { // first round of a length: |P_l| bookkeeping
            atomicAdd(&book[1], c);
            atomicMax(&book[2], c);
        }
    }
    const uint64_t stride = (uint64_t)gridDim.x * GREEDY_THREADS * GK;
    for (uint64_t i0 = (uint64_t)blockIdx.x * GREEDY_THREADS * GK + threadIdx.x;
         i0 - threadIdx.x < m; i0 += stride) { // block-uniform trip count
        unsigned long long r[GK];
        bool ca[GK], cb[GK];
#pragma unroll
        for (int k = 0; k < GK; ++k) {
            const uint64_t i = i0 + (uint64_t)k * GREEDY_THREADS;
            r[k] = i < m ? pairs[i] : ~0ull;
        }
#pragma unroll
        for (int k = 0; k < GK; ++k)
            if (r[k] != ~0ull)
                ca[k] = is_claimed(claimed, (uint32_t)(r[k] >> 32)), cb[k] = is_claimed(claimed, (uint32_t)r[k]);
        uint32_t keepm = 0;
#pragma unroll
        for (int k = 0; k < GK; ++k) {
            if (r[k] == ~0ull || (ca[k] | cb[k])) continue;
            const uint32_t a = (uint32_t)(r[k] >> 32), b = (uint32_t)r[k];
            atomicMax(&best[a], proposal(epoch, b));
            atomicMax(&best[b], proposal(epoch, a));
            keepm |= 1u << k;
        }
        block_append(r, keepm, live, live_count);
    }
}

__device__ __forceinline__ void accept_pair(uint32_t a, uint32_t b, uint32_t *claimed, uint32_t *succ,
                                            uint8_t *olen, uint8_t l)
{
    set_claimed(claimed, a), set_claimed(claimed, b);
    succ[a] = b ^ 1u, succ[b] = a ^ 1u; // edges a -> b^1 and (complement) b -> a^1
    olen[a] = l, olen[b] = l;
}

// Round part 2 over the live list: a pair whose two ends both chose each other is accepted;
// the others survive to the next round (some of them now have an end claimed by a pair
// accepted in this round: the next propose drops them).  No claimed-bit reads: every listed
// pair was live when the proposals were made, and acceptance is decided by best[] alone.
__global__ void __launch_bounds__(GREEDY_THREADS)
greedy_accept(const unsigned long long *pairs, const unsigned long long *count,
              unsigned long long cap, uint32_t *claimed, const unsigned long long *best,
              uint32_t epoch, uint32_t *succ, uint8_t *olen, uint8_t l, unsigned long long *out,
              unsigned long long *out_count, unsigned long long *reset, unsigned long long *book)
{
    const unsigned long long c = *count;
    const unsigned long long m = c < cap ? c : cap;
    if (blockIdx.x == 0 && threadIdx.x == 0) *reset = 0;
    const int lane = threadIdx.x & 31;
    uint32_t acc = 0;
    const uint64_t stride = (uint64_t)gridDim.x * GREEDY_THREADS * GK;
    for (uint64_t i0 = (uint64_t)blockIdx.x * GREEDY_THREADS * GK + threadIdx.x;
         i0 - threadIdx.x < m; i0 += stride) { // block-uniform trip count
        unsigned long long r[GK], ba[GK], bb[GK];
#pragma unroll
        for (int k = 0; k < GK; ++k) {
            const uint64_t i = i0 + (uint64_t)k * GREEDY_THREADS;
            r[k] = i < m ? pairs[i] : ~0ull;
        }
        // best[] of both ends (random 32 B sectors in an 8 B/end array: the traffic that bounds
        // the round)
#pragma unroll
        for (int k = 0; k < GK; ++k)
            if (r[k] != ~0ull) ba[k] = best[(uint32_t)(r[k] >> 32)], bb[k] = best[(uint32_t)r[k]];
        uint32_t keepm = 0;
#pragma unroll
        for (int k = 0; k < GK; ++k) {
            if (r[k] == ~0ull) continue;
            const uint32_t a = (uint32_t)(r[k] >> 32), b = (uint32_t)r[k];
            if (ba[k] == proposal(epoch, b) && bb[k] == proposal(epoch, a)) {
                accept_pair(a, b, claimed, succ, olen, l);
                ++acc;
            } else {
                keepm |= 1u << k;
            }
        }
        block_append(r, keepm, out, out_count);
    }
    for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0 && acc) atomicAdd(&book[0], (unsigned long long)acc);
}

constexpr int TAIL_MAX = 4096;
constexpr int FINISH_THREADS = 1024;

// Finishes one length on a single CTA: locally-dominant rounds with block barriers while more
// than TAIL_MAX pairs are live, then the sequential definition itself (bitonic sort by
// (a, b) in shared memory, one thread visits the pairs in order).
__global__ void __launch_bounds__(FINISH_THREADS)
greedy_finish(unsigned long long *cur, const unsigned long long *cur_count,
              unsigned long long *other, unsigned long long *other_count, uint32_t *claimed,
              unsigned long long *best, uint32_t epoch, uint32_t fast_rounds, uint32_t *succ,
              uint8_t *olen, uint8_t l, unsigned long long *book, unsigned long long *work)
{
    __shared__ unsigned long long s[TAIL_MAX];
    __shared__ uint32_t s_live, s_acc;
    uint32_t live = (uint32_t)*cur_count;
    uint32_t rounds = fast_rounds;
    if (threadIdx.x == 0) s_acc = 0;
    if (threadIdx.x == 0 && live) atomicAdd(work, (unsigned long long)live);
    while (live > (uint32_t)TAIL_MAX) {
        for (uint32_t i = threadIdx.x; i < live; i += FINISH_THREADS) {
            const unsigned long long r = cur[i];
            const uint32_t a = (uint32_t)(r >> 32), b = (uint32_t)r;
            if (is_claimed(claimed, a) || is_claimed(claimed, b)) continue;
            atomicMax(&best[a], proposal(epoch, b));
            atomicMax(&best[b], proposal(epoch, a));
        }
        if (threadIdx.x == 0) s_live = 0;
        __syncthreads();
        for (uint32_t i = threadIdx.x; i < live; i += FINISH_THREADS) {
            const unsigned long long r = cur[i];
            const uint32_t a = (uint32_t)(r >> 32), b = (uint32_t)r;
            if (is_claimed(claimed, a) || is_claimed(claimed, b)) continue;
            if (best[a] == proposal(epoch, b) && best[b] == proposal(epoch, a)) {
                accept_pair(a, b, claimed, succ, olen, l);
                atomicAdd(&s_acc, 1u);
            } else {
                other[atomicAdd(&s_live, 1u)] = r;
            }
        }
        __syncthreads();
        live = s_live;
        if (threadIdx.x == 0 && live) atomicAdd(work, (unsigned long long)live);
        unsigned long long *t = cur;
        cur = other;
        other = t;
        ++epoch;
        ++rounds;
        __syncthreads();
    }
    if (live) {
        uint32_t P = 1;
        while (P < live) P <<= 1;
        for (uint32_t i = threadIdx.x; i < P; i += FINISH_THREADS) s[i] = i < live ? cur[i] : ~0ull;
        __syncthreads();
        for (uint32_t k = 2; k <= P; k <<= 1)
            for (uint32_t j = k >> 1; j > 0; j >>= 1) {
                for (uint32_t i = threadIdx.x; i < P; i += FINISH_THREADS) {
                    const uint32_t ixj = i ^ j;
                    if (ixj > i) {
                        const bool up = (i & k) == 0;
                        const unsigned long long x = s[i], y = s[ixj];
                        if ((x > y) == up) s[i] = y, s[ixj] = x;
                    }
                }
                __syncthreads();
            }
        if (threadIdx.x == 0) {
            uint32_t acc = 0;
            for (uint32_t i = 0; i < live; ++i) {
                const uint32_t a = (uint32_t)(s[i] >> 32), b = (uint32_t)s[i];
                if (is_claimed(claimed, a) || is_claimed(claimed, b)) continue;
                accept_pair(a, b, claimed, succ, olen, l);
                ++acc;
            }
            s_acc += acc;
            ++rounds;
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        if (s_acc) atomicAdd(&book[0], (unsigned long long)s_acc);
        atomicMax(&book[3], (unsigned long long)rounds);
    }
    (void)other_count;
}

constexpr uint32_t FAST_ROUNDS = 3;
constexpr uint32_t EPOCHS_PER_LENGTH = 1u << 22; // fast rounds + at most ~4M finishing rounds

// Greedy over the pairs of length l in g.pool (count in *g.cnt, device).  Fully
// asynchronous: FAST_ROUNDS grid-wide rounds, then one CTA finishes the (few) survivors.
lasagna_status greedy_length(GreedyBufs &g, uint8_t l, uint32_t *succ, uint8_t *olen,
                             cudaStream_t s)
{
    const int sms = num_sms();
    const unsigned blocks = (unsigned)std::max<uint64_t>(
        1, std::min<uint64_t>(ceil_div(g.cap, GREEDY_THREADS * GK), (uint64_t)sms * 16));
    // Round r: propose reads X (count ctr[2r % 3]) and lists the live pairs in Y
    // (ctr[(2r+1) % 3]); accept reads Y and writes the survivors back to X (ctr[(2r+2) % 3]).
    // A kernel never resets a counter another block of the same launch may still read: each
    // one zeroes the counter two launches ahead.  With three rounds the survivors end in
    // ctr[0], and the last reset (ctr[1]) is the first append target of the next length.
    static_assert(FAST_ROUNDS == 3, "counter rotation");
    unsigned long long *X = g.pool, *Y = g.pool2;
    unsigned long long *ctr[3] = {g.cnt, g.cnt2, g.cnt3};
    const uint32_t e0 = g.epoch;
    g.epoch += EPOCHS_PER_LENGTH;
    for (uint32_t r = 0; r < FAST_ROUNDS; ++r) {
        greedy_propose<<<blocks, GREEDY_THREADS, 0, s>>>(X, ctr[(2 * r) % 3], g.cap, g.claimed, g.best,
                                                         e0 + r, Y, ctr[(2 * r + 1) % 3],
                                                         ctr[(2 * r + 2) % 3], r == 0 ? g.book : nullptr,
                                                         g.work);
        LSG_LAUNCHED("greedy_propose");
        greedy_accept<<<blocks, GREEDY_THREADS, 0, s>>>(Y, ctr[(2 * r + 1) % 3], g.cap, g.claimed, g.best,
                                                        e0 + r, succ, olen, l, X, ctr[(2 * r + 2) % 3],
                                                        ctr[(2 * r) % 3], g.book);
        LSG_LAUNCHED("greedy_accept");
    }
    greedy_finish<<<1, FINISH_THREADS, 0, s>>>(X, ctr[0], Y, ctr[1], g.claimed, g.best,
                                               e0 + FAST_ROUNDS, FAST_ROUNDS, succ, olen, l, g.book,
                                               g.work);
    LSG_LAUNCHED("greedy_finish");
    return LASAGNA_OK;
}

// lasagna_greedy_pairs helpers: key (255 - l) << 56 | i groups a caller's list by length
__global__ void lkeys_kernel(const uint8_t *pl, uint64_t count, uint64_t *keys)
{
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count;
         i += (uint64_t)gridDim.x * blockDim.x)
        keys[i] = ((uint64_t)(255u - pl[i]) << 56) | i;
}

__global__ void gather_pairs_kernel(const uint64_t *order, uint64_t off, uint64_t m,
                                    const uint32_t *pa, const uint32_t *pb,
                                    unsigned long long *pool, unsigned long long *cnt)
{
    const uint64_t mask = (1ull << 56) - 1;
    for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < m;
         j += (uint64_t)gridDim.x * blockDim.x) {
        uint64_t i = order[off + j] & mask;
        pool[j] = ((unsigned long long)pa[i] << 32) | pb[i];
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) *cnt = m;
}

lasagna_status launch_lkeys(const uint8_t *pl, uint64_t count, uint64_t *keys, cudaStream_t s)
{
    if (!count) return LASAGNA_OK;
    lkeys_kernel<<<(unsigned)std::min<uint64_t>(ceil_div(count, 256), 4096), 256, 0, s>>>(pl, count, keys);
    LSG_LAUNCHED("lkeys_kernel");
    return LASAGNA_OK;
}

lasagna_status launch_gather_pairs(const uint64_t *order, uint64_t off, uint64_t m,
                                   const uint32_t *pa, const uint32_t *pb,
                                   unsigned long long *pool, unsigned long long *cnt,
                                   cudaStream_t s)
{
    gather_pairs_kernel<<<(unsigned)std::max<uint64_t>(1, std::min<uint64_t>(ceil_div(m, 256), 4096)), 256, 0, s>>>(
        order, off, m, pa, pb, pool, cnt);
    LSG_LAUNCHED("gather_pairs_kernel");
    return LASAGNA_OK;
}

} // namespace lsg
