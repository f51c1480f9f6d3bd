// sort.cu — a4: stable LSD radix sort of u64 keys ("sort read-IDs by their
// fingerprints"; the paper used Thrust's radix sort, ref. [38] P:L144 — prior art).
//
// One launch per 8-bit digit, "onesweep" style: every CTA takes the next tile of 8192 keys
// (atomic tile counter => tiles are processed in acquisition order), ranks them stably
// with warp-level multi-split (__match_any_sync) into a shared-memory tile, obtains each
// digit's global offset by decoupled look-back over the preceding tiles' published
// counts, and writes the tile out digit run by digit run (coalesced).  Reads 8 B + writes
// 8 B per key per pass.  The histogram of the NEXT pass's digit is accumulated in the same
// pass (shared-memory counts, one global atomic per digit per CTA), so no separate
// histogram sweep is needed after the first.
//
// Segmented: n_seg independent arrays of seg_len keys each (one per overlap length) are
// sorted by one launch.
#include <cstdlib>

#include "kernels.cuh"

namespace lsg {

constexpr int SORT_THREADS = 512;
constexpr int SORT_KPT = 16;
constexpr int SORT_WARPS = SORT_THREADS / 32;
constexpr int SORT_TILE = SORT_THREADS * SORT_KPT; // 8192 keys

// look-back status word: [63:48] epoch, [47] inclusive-prefix flag, [46:0] count
constexpr unsigned long long ST_PREFIX = 1ull << 47;
constexpr unsigned long long ST_VALUE = (1ull << 47) - 1;

struct SortPassArgs {
    const uint64_t *in;
    uint64_t *out;
    uint64_t seg_len;
    uint32_t n_seg, tiles_per_seg;
    uint32_t shift, bits;          // this pass's digit
    const uint32_t *hist;          // [n_seg][256] counts of this digit
    uint32_t *hist_next;           // [n_seg][256] counts of the next digit (or null)
    uint32_t next_shift, next_bits;
    unsigned long long *status;    // [n_seg * tiles_per_seg][256]
    uint32_t *tile_ctr;
    uint32_t epoch;
};

// look-back words are single 64-bit values (flag and count together): relaxed GPU-scope
// accesses suffice (no other data is published through them)
__device__ __forceinline__ void st_relaxed(unsigned long long *p, unsigned long long v)
{
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_relaxed(const unsigned long long *p)
{
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ uint32_t lanemask_lt()
{
    uint32_t m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// exclusive scan of v over the 256 threads 0..255 (8 warps); returns the exclusive prefix;
// *total (shared) receives the sum.  Must be called by all SORT_THREADS threads.
__device__ __forceinline__ uint32_t scan256(uint32_t v, uint32_t *wsum /* [8] shared */)
{
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (threadIdx.x < 256 && lane == 31) wsum[warp] = x;
    __syncthreads();
    uint32_t add = 0;
    if (threadIdx.x < 256)
        for (int w = 0; w < warp; ++w) add += wsum[w];
    __syncthreads();
    return x - v + add;
}

// RANK = 0: bit-sliced multi-split (8 ballots); RANK = 1: match.any
template <int RANK>
__global__ void __launch_bounds__(SORT_THREADS, 2)
onesweep_kernel(SortPassArgs a)
{
    extern __shared__ __align__(16) unsigned char smem_raw[];
    uint64_t *skeys = reinterpret_cast<uint64_t *>(smem_raw);                       // [TILE]
    uint32_t *wcnt = reinterpret_cast<uint32_t *>(smem_raw + SORT_TILE * 8);        // [WARPS][256]
    __shared__ uint32_t lstart[256], gbase[256], dofs[256], nhist[256], wsum[8];
    __shared__ uint32_t s_tile;

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) s_tile = atomicAdd(a.tile_ctr, 1u);
    for (int t = tid; t < SORT_WARPS * 256 / 4; t += SORT_THREADS)
        reinterpret_cast<uint4 *>(wcnt)[t] = make_uint4(0, 0, 0, 0);
    if (tid < 256) nhist[tid] = 0;
    __syncthreads();
    const uint32_t g = s_tile;
    const uint32_t seg = g / a.tiles_per_seg, t = g % a.tiles_per_seg;
    const uint64_t seg_base = (uint64_t)seg * a.seg_len;
    const uint64_t tile_lo = (uint64_t)t * SORT_TILE;
    const uint32_t cnt = (uint32_t)min64(SORT_TILE, a.seg_len - tile_lo);
    const uint32_t dmask = (1u << a.bits) - 1;

    // digit offsets of this segment: exclusive scan of the pass histogram
    {
        uint32_t h = tid < 256 ? a.hist[(uint64_t)seg * 256 + tid] : 0;
        uint32_t ex = scan256(h, wsum);
        if (tid < 256) dofs[tid] = ex;
    }

    // load (warp-blocked: warp w owns keys [w*512, w*512+512), lane-strided)
    uint64_t key[SORT_KPT];
    const uint64_t *src = a.in + seg_base + tile_lo;
#pragma unroll
    for (int i = 0; i < SORT_KPT; ++i) {
        uint32_t idx = warp * (32 * SORT_KPT) + i * 32 + lane;
        key[i] = idx < cnt ? src[idx] : 0ull;
    }
    // early counts: per-warp digit histograms (order-free atomics)
    uint32_t *mycnt = wcnt + warp * 256;
#pragma unroll
    for (int i = 0; i < SORT_KPT; ++i) {
        uint32_t idx = warp * (32 * SORT_KPT) + i * 32 + lane;
        if (idx < cnt) atomicAdd(&mycnt[(uint32_t)((key[i] >> a.shift) & dmask)], 1u);
    }
    __syncthreads();

    // per digit: totals, exclusive over digits (local tile offsets), then each warp's start
    uint32_t total = 0;
    if (tid < 256) {
        for (int w = 0; w < SORT_WARPS; ++w) total += wcnt[w * 256 + tid];
    }
    {
        uint32_t ex = scan256(total, wsum);
        if (tid < 256) {
            lstart[tid] = ex;
            uint32_t run = ex;
            for (int w = 0; w < SORT_WARPS; ++w) {
                uint32_t c = wcnt[w * 256 + tid];
                wcnt[w * 256 + tid] = run;
                run += c;
            }
        }
    }

    // decoupled look-back on the early counts: global offset of each digit's run of this tile
    if (tid < 256) {
        unsigned long long *my = a.status + (uint64_t)g * 256 + tid;
        const unsigned long long ep = (unsigned long long)a.epoch << 48;
        if (t == 0) {
            st_relaxed(my, ep | ST_PREFIX | total);
            gbase[tid] = dofs[tid];
        } else {
            st_relaxed(my, ep | total);
            unsigned long long excl = 0;
            uint64_t p = (uint64_t)g - 1;
            while (true) {
                unsigned long long w;
                do {
                    w = ld_relaxed(a.status + p * 256 + tid);
                } while ((w >> 48) != (unsigned long long)a.epoch);
                excl += w & ST_VALUE;
                if (w & ST_PREFIX) break;
                --p;
            }
            st_relaxed(my, ep | ST_PREFIX | (excl + total));
            gbase[tid] = dofs[tid] + (uint32_t)excl;
        }
    }
    __syncthreads();

    // stable ranking straight into the tile's sorted position: keys are visited in their
    // original order (i, lane); the group leader reserves popc(peers) slots of the warp's
    // run of the digit with one shared atomic (issued in program order within the warp)
#pragma unroll
    for (int i = 0; i < SORT_KPT; ++i) {
        uint32_t idx = warp * (32 * SORT_KPT) + i * 32 + lane;
        bool valid = idx < cnt;
        uint32_t d = valid ? (uint32_t)((key[i] >> a.shift) & dmask) : 0u;
        // peers with the same digit: bit-sliced multi-split with 8 ballots (cheaper than
        // match.any on this part), restricted to valid lanes
        uint32_t peers;
        if constexpr (RANK == 0) {
            peers = __ballot_sync(0xffffffffu, valid);
#pragma unroll
            for (int bb = 0; bb < 8; ++bb) {
                const bool bit = (d >> bb) & 1u;
                const uint32_t m = __ballot_sync(0xffffffffu, bit);
                peers &= bit ? m : ~m;
            }
            if (!valid) peers = 1u << lane;
        } else {
            peers = __match_any_sync(0xffffffffu, valid ? d : 256u + lane);
        }
        int leader = 31 - __clz((int)peers);
        uint32_t lower = __popc(peers & lanemask_lt());
        uint32_t base_pos = 0;
        if (valid && lane == leader) base_pos = atomicAdd(&mycnt[d], __popc(peers));
        base_pos = __shfl_sync(0xffffffffu, base_pos, leader);
        if (valid) skeys[base_pos + lower] = key[i];
    }
    __syncthreads();

    // write out digit runs; count the next digit
    uint64_t *dst = a.out + seg_base;
    const uint32_t nmask = (1u << a.next_bits) - 1;
    for (uint32_t j = tid; j < cnt; j += SORT_THREADS) {
        uint64_t k = skeys[j];
        uint32_t d = (uint32_t)((k >> a.shift) & dmask);
        dst[gbase[d] + (j - lstart[d])] = k;
        if (a.hist_next) atomicAdd(&nhist[(uint32_t)((k >> a.next_shift) & nmask)], 1u);
    }
    if (a.hist_next) {
        __syncthreads();
        if (tid < 256 && nhist[tid]) atomicAdd(&a.hist_next[(uint64_t)seg * 256 + tid], nhist[tid]);
    }
}

// histogram of one digit over segmented keys (first pass of a generic sort)
__global__ void hist_kernel(const uint64_t *__restrict__ in, uint64_t seg_len, uint32_t shift,
                            uint32_t bits, uint32_t *__restrict__ hist)
{
    __shared__ uint32_t h[256];
    const uint32_t seg = blockIdx.y;
    for (int t = threadIdx.x; t < 256; t += blockDim.x) h[t] = 0;
    __syncthreads();
    const uint32_t mask = (1u << bits) - 1;
    const uint64_t *p = in + (uint64_t)seg * seg_len;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < seg_len;
         i += (uint64_t)gridDim.x * blockDim.x)
        atomicAdd(&h[(uint32_t)((p[i] >> shift) & mask)], 1u);
    __syncthreads();
    for (int t = threadIdx.x; t < 256; t += blockDim.x)
        if (h[t]) atomicAdd(&hist[(uint64_t)seg * 256 + t], h[t]);
}

lasagna_status launch_hist(const uint64_t *keys, uint64_t seg_len, uint32_t n_seg, uint32_t shift,
                           uint32_t bits, uint32_t *hist, cudaStream_t s)
{
    if (seg_len == 0 || n_seg == 0) return LASAGNA_OK;
    dim3 grid((unsigned)std::min<uint64_t>(ceil_div(seg_len, 256 * 16), 1024), n_seg);
    hist_kernel<<<grid, 256, 0, s>>>(keys, seg_len, shift, bits, hist);
    LSG_LAUNCHED("hist_kernel");
    return LASAGNA_OK;
}

// ---------------------------------------------------------------- host side
size_t sort_status_bytes(uint64_t seg_len, uint32_t n_seg)
{
    return (size_t)n_seg * ceil_div(seg_len, SORT_TILE) * 256 * sizeof(unsigned long long);
}



lasagna_status sort_ctx_reset(SortCtx &c, cudaStream_t s)
{
    LSG_CUDA(cudaMemsetAsync(c.status, 0, c.status_bytes, s));
    LSG_CUDA(cudaMemsetAsync(c.tile_ctrs, 0, SORT_CTRS * sizeof(uint32_t), s));
    c.epoch = 0;
    return LASAGNA_OK;
}

// digit plan for bits [lo, hi): P passes of <= 8 bits, as even as possible
void digit_plan(uint32_t lo, uint32_t hi, uint32_t *P, uint32_t *shifts, uint32_t *bits)
{
    uint32_t span = hi - lo;
    uint32_t p = (span + 7) / 8;
    uint32_t b = (span + p - 1) / p;
    for (uint32_t i = 0; i < p; ++i) {
        shifts[i] = lo + i * b;
        bits[i] = std::min(b, hi - shifts[i]);
    }
    *P = p;
}

// Sort n_seg segments of seg_len keys by bits [lo, hi).  The keys start in bufs[0]; on
// return *which tells which of bufs[0], bufs[1] holds the result.  hist: [P][n_seg][256]
// u32, zeroed here; if hist0_ready, hist[0] was already filled by the caller (the table
// kernel produces it while writing the keys).
lasagna_status sort_segments(uint64_t *bufs[2], uint64_t seg_len, uint32_t n_seg, uint32_t lo,
                             uint32_t hi, uint32_t *hist, bool hist0_ready, SortCtx &ctx,
                             cudaStream_t s, int *which)
{
    uint32_t P, shifts[8], bits[8];
    digit_plan(lo, hi, &P, shifts, bits);
    *which = 0;
    if (seg_len == 0 || n_seg == 0) return LASAGNA_OK;
    const size_t hseg = (size_t)n_seg * 256;
    if (hist0_ready)
        LSG_CUDA(cudaMemsetAsync(hist + hseg, 0, (P - 1) * hseg * sizeof(uint32_t), s));
    else {
        LSG_CUDA(cudaMemsetAsync(hist, 0, P * hseg * sizeof(uint32_t), s));
        dim3 grid((unsigned)std::min<uint64_t>(ceil_div(seg_len, 256 * 16), 1024), n_seg);
        hist_kernel<<<grid, 256, 0, s>>>(bufs[0], seg_len, shifts[0], bits[0], hist);
        LSG_LAUNCHED("hist_kernel");
    }
    const size_t smem = (size_t)SORT_TILE * 8 + (size_t)SORT_WARPS * 256 * 4;
    static const int rank_mode = [] {
        const char *e = getenv("LASAGNA_SORT_RANK");
        return (e && e[0] == 'm') ? 1 : 0;
    }();
    auto kern = rank_mode ? onesweep_kernel<1> : onesweep_kernel<0>;
    LSG_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const uint32_t tps = (uint32_t)ceil_div(seg_len, SORT_TILE);
    if (sort_status_bytes(seg_len, n_seg) > ctx.status_bytes) {
        set_error("sort status buffer too small");
        return LASAGNA_ENOSPC;
    }
    int cur = 0;
    for (uint32_t p = 0; p < P; ++p) {
        if (ctx.epoch + 1 >= SORT_CTRS || ctx.epoch + 1 >= 65535) {
            lasagna_status st = sort_ctx_reset(ctx, s);
            if (st != LASAGNA_OK) return st;
        }
        ++ctx.epoch;
        SortPassArgs a;
        a.in = bufs[cur];
        a.out = bufs[cur ^ 1];
        a.seg_len = seg_len;
        a.n_seg = n_seg;
        a.tiles_per_seg = tps;
        a.shift = shifts[p];
        a.bits = bits[p];
        a.hist = hist + p * hseg;
        a.hist_next = (p + 1 < P) ? hist + (p + 1) * hseg : nullptr;
        a.next_shift = (p + 1 < P) ? shifts[p + 1] : 0;
        a.next_bits = (p + 1 < P) ? bits[p + 1] : 1;
        a.status = ctx.status;
        a.tile_ctr = ctx.tile_ctrs + ctx.epoch;
        a.epoch = ctx.epoch;
        uint64_t grid = (uint64_t)tps * n_seg;
        kern<<<(unsigned)grid, SORT_THREADS, smem, s>>>(a);
        LSG_LAUNCHED("onesweep_kernel");
        cur ^= 1;
    }
    *which = cur;
    return LASAGNA_OK;
}

} // namespace lsg
