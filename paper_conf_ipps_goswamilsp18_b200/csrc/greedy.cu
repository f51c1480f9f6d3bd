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

__global__ void greedy_init(const unsigned long long *pairs, const unsigned long long *count,
                            uint32_t *best0, uint32_t *best1)
{
    const unsigned long long m = *count;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m;
         i += (uint64_t)gridDim.x * blockDim.x) {
        unsigned long long r = pairs[i];
        uint32_t a = (uint32_t)(r >> 32), b = (uint32_t)r;
        best0[a] = NONE, best0[b] = NONE, best1[a] = NONE, best1[b] = NONE;
    }
}

__global__ void greedy_propose(const unsigned long long *pairs, const unsigned long long *count,
                               const uint8_t *claimed, uint32_t *best)
{
    const unsigned long long m = *count;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m;
         i += (uint64_t)gridDim.x * blockDim.x) {
        unsigned long long r = pairs[i];
        uint32_t a = (uint32_t)(r >> 32), b = (uint32_t)r;
        if (claimed[a] | claimed[b]) continue;
        atomicMin(&best[a], b);
        atomicMin(&best[b], a);
    }
}

__global__ void greedy_accept(const unsigned long long *pairs, const unsigned long long *count,
                              uint8_t *claimed, const uint32_t *best, uint32_t *best_next,
                              uint32_t *succ, uint8_t *olen, uint8_t l,
                              unsigned long long *out, unsigned long long *out_count,
                              unsigned long long *accepted)
{
    const unsigned long long m = *count;
    uint32_t acc = 0;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m;
         i += (uint64_t)gridDim.x * blockDim.x) {
        unsigned long long r = pairs[i];
        uint32_t a = (uint32_t)(r >> 32), b = (uint32_t)r;
        if (claimed[a] | claimed[b]) continue; // dead: an end was taken in an earlier round
        if (best[a] == b && best[b] == a) {
            claimed[a] = 1, claimed[b] = 1;
            succ[a] = b ^ 1u, succ[b] = a ^ 1u;
            olen[a] = l, olen[b] = l;
            ++acc;
        } else {
            best_next[a] = NONE, best_next[b] = NONE;
            out[atomicAdd(out_count, 1ull)] = r;
        }
    }
    for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if ((threadIdx.x & 31) == 0 && acc) atomicAdd(accepted, (unsigned long long)acc);
}

constexpr int TAIL_MAX = 4096;

// Sequential definition on the remaining pairs: bitonic sort by (a, b) in shared memory,
// then one thread visits them in order.
__global__ void __launch_bounds__(1024)
greedy_tail(const unsigned long long *pairs, const unsigned long long *count, uint8_t *claimed,
            uint32_t *succ, uint8_t *olen, uint8_t l, unsigned long long *accepted)
{
    __shared__ unsigned long long s[TAIL_MAX];
    const unsigned long long cnt_ = *count;
    const uint32_t m = (uint32_t)(cnt_ < (unsigned long long)TAIL_MAX ? cnt_ : (unsigned long long)TAIL_MAX);
    uint32_t P = 1;
    while (P < m) P <<= 1;
    for (uint32_t i = threadIdx.x; i < P; i += blockDim.x) s[i] = i < m ? pairs[i] : ~0ull;
    __syncthreads();
    for (uint32_t k = 2; k <= P; k <<= 1)
        for (uint32_t j = k >> 1; j > 0; j >>= 1) {
            for (uint32_t i = threadIdx.x; i < P; i += blockDim.x) {
                uint32_t ixj = i ^ j;
                if (ixj > i) {
                    bool up = (i & k) == 0;
                    unsigned long long x = s[i], y = s[ixj];
                    if ((x > y) == up) s[i] = y, s[ixj] = x;
                }
            }
            __syncthreads();
        }
    if (threadIdx.x == 0) {
        unsigned long long acc = 0;
        for (uint32_t i = 0; i < m; ++i) {
            uint32_t a = (uint32_t)(s[i] >> 32), b = (uint32_t)s[i];
            if (claimed[a] | claimed[b]) continue;
            claimed[a] = 1, claimed[b] = 1;
            succ[a] = b ^ 1u, succ[b] = a ^ 1u;
            olen[a] = l, olen[b] = l;
            ++acc;
        }
        if (acc) atomicAdd(accepted, acc);
    }
}


// Greedy over the m pairs of length l in bufs.pool (count in *bufs.cnt, device; m its host
// copy).  Synchronises the stream once per round.
lasagna_status greedy_length(GreedyBufs &g, uint64_t m, uint8_t l, uint32_t *succ, uint8_t *olen,
                             cudaStream_t s, uint32_t *rounds_out)
{
    *rounds_out = 0;
    if (m == 0) return LASAGNA_OK;
    const int sms = num_sms();
    auto blocks_for = [&](uint64_t k) {
        return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(ceil_div(k, 256), (uint64_t)sms * 8));
    };
    unsigned long long *in = g.pool, *out = g.pool2, *cin = g.cnt, *cout = g.cnt2;
    uint32_t *best = g.best0, *bnext = g.best1;
    greedy_init<<<blocks_for(m), 256, 0, s>>>(in, cin, g.best0, g.best1);
    LSG_LAUNCHED("greedy_init");
    uint32_t rounds = 0;
    uint64_t live = m;
    while (live > 0) {
        if (rounds >= 4 && live <= (uint64_t)TAIL_MAX) {
            greedy_tail<<<1, 1024, 0, s>>>(in, cin, g.claimed, succ, olen, l, g.accepted);
            LSG_LAUNCHED("greedy_tail");
            ++rounds;
            break;
        }
        LSG_CUDA(cudaMemsetAsync(cout, 0, sizeof(unsigned long long), s));
        greedy_propose<<<blocks_for(live), 256, 0, s>>>(in, cin, g.claimed, best);
        LSG_LAUNCHED("greedy_propose");
        greedy_accept<<<blocks_for(live), 256, 0, s>>>(in, cin, g.claimed, best, bnext, succ, olen,
                                                       l, out, cout, g.accepted);
        LSG_LAUNCHED("greedy_accept");
        ++rounds;
        unsigned long long h = 0;
        LSG_CUDA(cudaMemcpyAsync(&h, cout, sizeof(h), cudaMemcpyDeviceToHost, s));
        LSG_CUDA(cudaStreamSynchronize(s));
        live = h;
        std::swap(in, out);
        std::swap(cin, cout);
        std::swap(best, bnext);
    }
    *rounds_out = rounds;
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
