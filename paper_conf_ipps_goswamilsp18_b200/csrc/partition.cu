// partition.cu — the bucketed (MSD radix-partition) form of a3/a4/a5, the fast path of
// lasagna_greedy_graph / lasagna_overlaps.
//
// The join only needs the keys of one length GROUPED by their top T bits (a bucket holds
// every prefix and suffix entry that can match); it never needs them in sorted
// order.  So instead of a stable LSD sort, the table is radix-PARTITIONED most-significant
// digit first into regions with slack (capacity = mean + 8 sigma + 32 of the multinomial
// occupancy, overflow detected and answered by the exact LSD path):
//
//   scatter_table_kernel  fingerprints (a2) + level-1 partition by the top 8 key bits, fused:
//                         each CTA computes the keys of 512 reads for one length at a time,
//                         ranks them by digit in shared memory and reserves space in the 256
//                         regions of that length with one atomic per (CTA, digit); no
//                         histogram pass, no look-back (order inside a region is irrelevant)
//   refine_kernel         level k -> k+1: one CTA owns one region and streams it in tiles,
//                         splitting it by the next 8 bits into 256 sub-regions it alone
//                         writes (CTA-local running offsets: no atomics, no look-back)
//   bucket_join_kernel    a5 over the final regions (= buckets, fills known): windows of
//                         whole buckets go through the shared-memory hash join (joinwin.cuh)
//
// Traffic per entry: 8 B written by the scatter, 8 + 8 B per refine level, 8 B read by the
// join (T = 16: 32 B, against 48 B for table + 2 LSD passes + join).
#include "fingerprint.cuh"
#include "joinwin.cuh"

namespace lsg {

constexpr int SC_THREADS = 512; // reads per scatter CTA (one per thread)
constexpr int RF_THREADS = 512;
constexpr int RF_KPT = 8;
constexpr int RF_TILE = RF_THREADS * RF_KPT;

// exclusive scan over the first 256 threads of a block of >= 256 threads (8 warps used);
// every thread of the block must call it.  wsum: 8 shared words.
__device__ __forceinline__ uint32_t block_scan256(uint32_t v, uint32_t *wsum)
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

// ------------------------------------------------------------------ level 1: fused with a2
template <int W>
__global__ void __launch_bounds__(SC_THREADS, 2)
scatter_table_kernel(ScatterArgs a)
{
    __shared__ uint64_t stage[SC_THREADS * 4];
    __shared__ uint32_t cnt[256], lstart[256], base[256], wsum[8];
    __shared__ uint32_t s_total;

    const uint64_t i = (uint64_t)blockIdx.x * SC_THREADS + threadIdx.x;
    const bool valid = i < a.n;
    uint64_t x[W], y[W];
    if (valid) {
        load_read<W>(a.packed, a.stride, i, x);
        rc_words<W>(x, a.L, y);
    } else {
#pragma unroll
        for (int j = 0; j < W; ++j) x[j] = y[j] = 0;
    }
    if (threadIdx.x < 256) cnt[threadIdx.x] = 0;
    __syncthreads();
    const uint64_t keep = ~((2ull << a.vbits) - 1);
    const uint64_t tagS = 1ull << a.vbits;
    const uint64_t v0 = 2 * (a.read_offset + i);
    FpStreams st;
    st.init();
#pragma unroll
    for (int w = 0; w < W; ++w) {
        uint64_t xa = x[w], yb = y[w];
        const uint32_t k0 = 32u * w;
        if (k0 >= a.l_hi) break;
        const uint32_t kn = min(32u, a.l_hi - k0);
        for (uint32_t j = 0; j < kn; ++j) {
            st.step((uint32_t)(xa & 3u), (uint32_t)(yb & 3u), k0 + j);
            xa >>= 2;
            yb >>= 2;
            const uint32_t l = k0 + j + 1;
            if (l < a.l_lo) continue; // uniform across the block
            // ---- one partition round for length l: 4 keys per read
            uint64_t kk[4];
            uint32_t dd[4], rk[4];
            if (valid) {
                kk[0] = (mix(exact61(st.P0)) & keep) | v0;
                kk[1] = (mix(exact61(st.S0)) & keep) | tagS | v0;
                kk[2] = (mix(exact61(st.P1)) & keep) | (v0 + 1);
                kk[3] = (mix(exact61(st.S1)) & keep) | tagS | (v0 + 1);
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    dd[q] = (uint32_t)(kk[q] >> 56);
                    rk[q] = atomicAdd(&cnt[dd[q]], 1u);
                }
            }
            __syncthreads();
            const uint32_t seg = l - a.l_lo;
            uint32_t c = 0;
            if (threadIdx.x < 256) {
                c = cnt[threadIdx.x];
                cnt[threadIdx.x] = 0;
                base[threadIdx.x] =
                    c ? atomicAdd(&a.fill[(uint64_t)seg * 256 + threadIdx.x], c) : 0u;
            }
            const uint32_t ex = block_scan256(c, wsum);
            if (threadIdx.x < 256) {
                lstart[threadIdx.x] = ex;
                if (threadIdx.x == 255) s_total = ex + c;
            }
            __syncthreads();
            if (valid) {
#pragma unroll
                for (int q = 0; q < 4; ++q) stage[lstart[dd[q]] + rk[q]] = kk[q];
            }
            __syncthreads();
            const uint32_t total = s_total;
            uint64_t *dst = a.out + (uint64_t)seg * 256 * a.cap;
            for (uint32_t t = threadIdx.x; t < total; t += SC_THREADS) {
                const uint64_t key = stage[t];
                const uint32_t d = (uint32_t)(key >> 56);
                const uint64_t pos = (uint64_t)base[d] + (t - lstart[d]);
                if (pos < a.cap) dst[(uint64_t)d * a.cap + pos] = key;
                else *a.overflow = 1u;
            }
            // the next round's first barrier orders these reads before stage/lstart reuse
        }
    }
}

lasagna_status launch_scatter_table(const ScatterArgs &args, cudaStream_t s)
{
    if (args.n == 0) return LASAGNA_OK;
    return dispatch_W(args.L, [&](auto wc) -> lasagna_status {
        constexpr int W = decltype(wc)::value;
        const uint64_t blocks = ceil_div(args.n, SC_THREADS);
        scatter_table_kernel<W><<<(unsigned)blocks, SC_THREADS, 0, s>>>(args);
        LSG_LAUNCHED("scatter_table_kernel");
        return LASAGNA_OK;
    });
}

// ------------------------------------------------------------------ level k -> k+1
// One CTA owns one region and streams it: the bulk-copy engine prefetches tile t+1 into the
// other half of a double buffer while tile t is ranked (shared atomics: order inside a
// sub-region is irrelevant), staged by digit and written out in digit runs.
__global__ void __launch_bounds__(RF_THREADS, 2)
refine_kernel(RefineArgs a)
{
    extern __shared__ __align__(128) uint64_t rsm[];
    uint64_t *inb = rsm;                 // [2][RF_TILE]
    uint64_t *rstage = rsm + 2 * RF_TILE; // [RF_TILE]
    __shared__ __align__(8) unsigned long long mbar[2];
    __shared__ uint32_t cnt[256], lstart[256], running[256], wsum[8];
    const uint64_t r = blockIdx.x;
    const uint32_t fill = a.fill_in[r];
    const uint64_t count = min64(fill, a.cap_in);
    const uint64_t *src = a.in + r * a.cap_in;
    uint64_t *dst = a.out + r * 256 * a.cap_out;
    const uint32_t ntiles = (uint32_t)ceil_div(count, RF_TILE);
    if (threadIdx.x < 256) cnt[threadIdx.x] = 0, running[threadIdx.x] = 0;
    if (threadIdx.x == 0) {
        mbar_init(&mbar[0], 1);
        mbar_init(&mbar[1], 1);
        fence_mbar_init();
    }
    __syncthreads();
    // bytes of tile t (rounded up to 16: the region capacity is even, so the rounding stays
    // inside the region)
    auto tile_bytes = [&](uint32_t t) {
        const uint64_t m = min64(RF_TILE, count - (uint64_t)t * RF_TILE);
        return (uint32_t)(((m * 8) + 15) & ~15ull);
    };
    if (threadIdx.x == 0 && ntiles) bulk_load(inb, src, tile_bytes(0), &mbar[0]);
    for (uint32_t t = 0; t < ntiles; ++t) {
        const uint32_t bsel = t & 1;
        const uint64_t t0 = (uint64_t)t * RF_TILE;
        const uint32_t m = (uint32_t)min64(RF_TILE, count - t0);
        if (threadIdx.x == 0 && t + 1 < ntiles) {
            fence_proxy_async();
            bulk_load(inb + (bsel ^ 1) * RF_TILE, src + t0 + RF_TILE, tile_bytes(t + 1),
                      &mbar[bsel ^ 1]);
        }
        mbar_wait(&mbar[bsel], (t >> 1) & 1);
        const uint64_t *tin = inb + bsel * RF_TILE;
        uint32_t rk[RF_KPT];
#pragma unroll
        for (int q = 0; q < RF_KPT; ++q) {
            const uint32_t idx = q * RF_THREADS + threadIdx.x;
            if (idx < m) rk[q] = atomicAdd(&cnt[(uint32_t)(tin[idx] >> a.dshift) & 255u], 1u);
        }
        __syncthreads();
        uint32_t c = 0;
        if (threadIdx.x < 256) {
            c = cnt[threadIdx.x];
            cnt[threadIdx.x] = 0;
        }
        const uint32_t ex = block_scan256(c, wsum);
        if (threadIdx.x < 256) lstart[threadIdx.x] = ex;
        __syncthreads();
#pragma unroll
        for (int q = 0; q < RF_KPT; ++q) {
            const uint32_t idx = q * RF_THREADS + threadIdx.x;
            if (idx < m) {
                const uint64_t k = tin[idx];
                rstage[lstart[(uint32_t)(k >> a.dshift) & 255u] + rk[q]] = k;
            }
        }
        __syncthreads();
        for (uint32_t u = threadIdx.x; u < m; u += RF_THREADS) {
            const uint64_t k = rstage[u];
            const uint32_t d = (uint32_t)(k >> a.dshift) & 255u;
            const uint64_t pos = (uint64_t)running[d] + (u - lstart[d]);
            if (pos < a.cap_out) dst[(uint64_t)d * a.cap_out + pos] = k;
            else *a.overflow = 1u;
        }
        __syncthreads();
        if (threadIdx.x < 256) running[threadIdx.x] += c;
        __syncthreads();
    }
    if (threadIdx.x < 256) {
        a.fill_out[r * 256 + threadIdx.x] = running[threadIdx.x];
        if (running[threadIdx.x] > a.cap_out) *a.overflow = 1u;
    }
    if (threadIdx.x == 0 && fill > a.cap_in) *a.overflow = 1u;
}

lasagna_status launch_refine(const RefineArgs &args, uint64_t n_regions, cudaStream_t s)
{
    if (n_regions == 0) return LASAGNA_OK;
    const size_t smem = (size_t)3 * RF_TILE * 8;
    LSG_CUDA(cudaFuncSetAttribute(refine_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  (int)smem));
    refine_kernel<<<(unsigned)n_regions, RF_THREADS, smem, s>>>(args);
    LSG_LAUNCHED("refine_kernel");
    return LASAGNA_OK;
}

// ------------------------------------------------------------------ a5 over the buckets
constexpr int BJ_FILLS = 2048; // bucket fills staged per chunk

template <int W>
__global__ void __launch_bounds__(JOIN_THREADS, 2)
bucket_join_kernel(BucketJoinArgs b)
{
    extern __shared__ __align__(16) unsigned char jsm[];
    uint64_t *ent = reinterpret_cast<uint64_t *>(jsm);                                   // [CAP]
    unsigned long long *buf = reinterpret_cast<unsigned long long *>(jsm + JOIN_CAP * 8); // [BUF]
    uint32_t *slot = reinterpret_cast<uint32_t *>(jsm + (JOIN_CAP + JOIN_BUF) * 8);     // [SLOTS]
    unsigned short *next =
        reinterpret_cast<unsigned short *>(jsm + (JOIN_CAP + JOIN_BUF) * 8 + JOIN_SLOTS * 4);
    uint32_t *sfill =
        reinterpret_cast<uint32_t *>(jsm + (JOIN_CAP + JOIN_BUF) * 8 + JOIN_SLOTS * 4 + JOIN_CAP * 2);
    __shared__ uint32_t bcount, vdone, s_nb, s_total, s_np, s_ns;
    const JoinArgs &a = b.j;
    const uint64_t nb = b.n_buckets;
    const uint64_t b0 = nb * blockIdx.x / gridDim.x, b1 = nb * (blockIdx.x + 1) / gridDim.x;
    if (threadIdx.x == 0) bcount = 0, vdone = 0;
    for (uint32_t t = threadIdx.x; t < JOIN_SLOTS; t += JOIN_THREADS) slot[t] = 0;
    Stager em{buf, &bcount, a.pairs, a.cap, a.count};
    unsigned long long nfalse = 0;
    uint32_t epoch = 0;
    for (uint64_t c0 = b0; c0 < b1; c0 += BJ_FILLS) {
        const uint32_t nc = (uint32_t)min64(BJ_FILLS, b1 - c0);
        __syncthreads();
        for (uint32_t t = threadIdx.x; t < nc; t += JOIN_THREADS) {
            const uint32_t f = b.fills[c0 + t];
            if (f > b.bucket_cap) *b.overflow = 1u;
            sfill[t] = (uint32_t)min64(f, b.bucket_cap);
        }
        __syncthreads();
        uint32_t k = 0;
        while (k < nc) {
            // window: buckets [k, k + nb_w) with total <= JOIN_CAP (at least one bucket)
            if (threadIdx.x == 0) {
                uint32_t tot = sfill[k], e = k + 1;
                while (e < nc && tot + sfill[e] <= (uint32_t)JOIN_CAP) tot += sfill[e++];
                s_nb = e - k;
                s_total = tot;
            }
            __syncthreads();
            const uint32_t nbw = s_nb, total = s_total;
            if (++epoch == 0x10000u) {
                for (uint32_t t = threadIdx.x; t < JOIN_SLOTS; t += JOIN_THREADS) slot[t] = 0;
                epoch = 1;
                __syncthreads();
            }
            if (total > (uint32_t)JOIN_CAP) {
                const uint64_t bk = c0 + k;
                oversized_join<W>(a, b.buckets + bk * b.bucket_cap, 0, total, em, nfalse);
            } else {
                // stage the window split by list: prefix entries from the front, suffix
                // entries from the back (warp-aggregated slots)
                if (threadIdx.x == 0) s_np = 0, s_ns = 0;
                __syncthreads();
                const int lane = threadIdx.x & 31;
                for (uint32_t q = 0; q < nbw; ++q) {
                    const uint32_t f = sfill[k + q];
                    const uint64_t *srcb = b.buckets + (c0 + k + q) * b.bucket_cap;
                    for (uint32_t t0 = 0; t0 < f; t0 += JOIN_THREADS) {
                        const uint32_t t = t0 + threadIdx.x;
                        const bool ok = t < f;
                        const uint64_t e = ok ? srcb[t] : 0;
                        const bool isS = ok && ((e >> a.vbits) & 1);
                        const uint32_t bS = __ballot_sync(0xffffffffu, isS);
                        const uint32_t bP = __ballot_sync(0xffffffffu, ok && !isS);
                        uint32_t baseP = 0, baseS = 0;
                        if (lane == 0) {
                            if (bP) baseP = atomicAdd(&s_np, (uint32_t)__popc(bP));
                            if (bS) baseS = atomicAdd(&s_ns, (uint32_t)__popc(bS));
                        }
                        baseP = __shfl_sync(0xffffffffu, baseP, 0);
                        baseS = __shfl_sync(0xffffffffu, baseS, 0);
                        const uint32_t lt = (1u << lane) - 1;
                        if (ok) {
                            if (isS) ent[JOIN_CAP - 1 - (baseS + __popc(bS & lt))] = e;
                            else ent[baseP + __popc(bP & lt)] = e;
                        }
                    }
                }
                __syncthreads();
                const uint32_t nP = s_np, nS = s_ns;
                hash_join_split<W>(a, ent, nP, JOIN_CAP - nS, nS, slot, next, epoch, em, nfalse);
            }
            __syncthreads();
            window_epilogue<W>(a, buf, &bcount, &vdone, nfalse);
            __syncthreads();
            k += nbw;
        }
    }
    __syncthreads();
    flush_staged(buf, min(bcount, (uint32_t)JOIN_BUF), a.pairs, a.cap, a.count);
    for (int o = 16; o; o >>= 1) nfalse += __shfl_xor_sync(0xffffffffu, nfalse, o);
    if ((threadIdx.x & 31) == 0 && nfalse) atomicAdd(a.false_matches, nfalse);
}

lasagna_status launch_bucket_join(const BucketJoinArgs &args, cudaStream_t s)
{
    if (args.n_buckets == 0) return LASAGNA_OK;
    return dispatch_W(args.j.L, [&](auto wc) -> lasagna_status {
        constexpr int W = decltype(wc)::value;
        const size_t smem = (size_t)(JOIN_CAP + JOIN_BUF) * 8 + (size_t)JOIN_SLOTS * 4 +
                            (size_t)JOIN_CAP * 2 + (size_t)BJ_FILLS * 4;
        LSG_CUDA(cudaFuncSetAttribute(bucket_join_kernel<W>,
                                      cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        int per_sm = 0;
        LSG_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, bucket_join_kernel<W>,
                                                               JOIN_THREADS, smem));
        per_sm = std::max(per_sm, 1);
        const uint64_t blocks =
            std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)num_sms() * per_sm, args.n_buckets));
        bucket_join_kernel<W><<<(unsigned)blocks, JOIN_THREADS, smem, s>>>(args);
        LSG_LAUNCHED("bucket_join_kernel");
        return LASAGNA_OK;
    });
}

} // namespace lsg
