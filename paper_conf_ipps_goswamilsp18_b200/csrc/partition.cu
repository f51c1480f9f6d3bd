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
//                         splitting it by the next dbits (<= 8) bits into 2^dbits sub-regions
//                         it alone writes (CTA-local running offsets: no atomics, no
//                         look-back).  T = 16 (cfg3): one refine; T = 16 + d (cfg4/cfg5, 2n
//                         ~ 2.5e9): two, the second by d = 4 bits, so a final bucket holds
//                         ~2.4 K entries like cfg3's ~1.1 K (one shared-memory join window)
//   bucket_join_kernel    a5 over the final regions (= buckets, fills known): windows of
//                         whole buckets go through the shared-memory hash join (joinwin.cuh)
//
// Traffic per entry: 8 B written by the scatter, 8 + 8 B per refine level, 8 B read by the
// join (T = 16: 32 B, against 48 B for table + 2 LSD passes + join).
#include <cstdlib>

#include "fingerprint.cuh"
#include "pack.cuh"
#include "joinwin.cuh"

namespace lsg {

constexpr int SC_THREADS = 512; // reads per scatter CTA (one per thread)
constexpr int RF_THREADS = 512;


// exclusive scan of v over the first NB threads (NB a multiple of 32, <= 512); every thread of
// the block must call it.  wsum: 16 shared words.
template <int NB>
__device__ __forceinline__ uint32_t block_scan(uint32_t v, uint32_t *wsum)
{
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (threadIdx.x < NB && lane == 31) wsum[warp] = x;
    __syncthreads();
    uint32_t add = 0;
    if (threadIdx.x < NB)
        for (int w = 0; w < warp; ++w) add += wsum[w];
    __syncthreads();
    return x - v + add;
}

// ------------------------------------------------------------------ level 1: fused with a2
// One thread per read, LPR lengths per partition round: the rolling streams (a2) produce the
// two canonical keys of the read (vertex 2i and 2i+1, common.cuh) for each length; a round
// ranks its 2 * LPR keys per thread by bin in shared memory (atomics: order inside a region is
// irrelevant), reserves space in the regions of its lengths with one global atomic per
// (CTA, bin), stages the keys by bin and writes them out in bin runs.  Bins are
// q * NBL + d1 (split: q * NBL + 2 d1 + flag bit) for the round's q-th length, d1 = the top 8
// bits of the mixed canonical fingerprint, which the stored key no longer carries.
template <int W, bool ASCII, bool SPLIT, int LPR>
__global__ void __launch_bounds__(SC_THREADS, 2)
scatter_table_kernel_v1(ScatterArgs a)
{
    constexpr int NBL = SPLIT ? 512 : 256; // bins per length
    constexpr int NBIN = LPR * NBL;
    constexpr int BPT = NBIN / SC_THREADS; // bins per thread in the round's scan
    constexpr int KPT = 2 * LPR;           // keys per thread per round
    static_assert(NBIN % SC_THREADS == 0 && BPT >= 1 && BPT <= 4, "bins per thread");
    // dynamic: stage[SC_THREADS * KPT] keys, sbin[SC_THREADS * KPT] their bins, then (ASCII)
    // the CTA's staged read bytes
    extern __shared__ __align__(16) uint64_t stage[];
    unsigned short *sbin = reinterpret_cast<unsigned short *>(stage + SC_THREADS * KPT);
    __shared__ uint32_t cnt[NBIN], lstart[NBIN + 1], wsum[16];
    __shared__ long long gofs[NBIN]; // per bin: element offset of stage slot 0's destination, -1 = overflow

    const uint64_t i = (uint64_t)blockIdx.x * SC_THREADS + threadIdx.x;
    const bool valid = i < a.n;
    uint64_t x[W], y[W];
    if constexpr (ASCII) {
        // a1 fused: stage this CTA's ASCII span (zero-copy from host memory over PCIe when
        // the caller passed page-locked host memory), pack, validate, keep the packed rows
        unsigned char *sascii = reinterpret_cast<unsigned char *>(sbin + SC_THREADS * KPT);
        const uint64_t r0 = (uint64_t)blockIdx.x * SC_THREADS;
        const uint64_t r1 = min64(a.n, r0 + SC_THREADS);
        const uint32_t off = stage_ascii(a.ascii, r0 * a.L, r1 * a.L, sascii, SC_THREADS);
        __syncthreads();
        if (valid) {
            const bool ok = pack_row_regs_swar<W>(sascii + off + (uint64_t)threadIdx.x * a.L, a.L, x);
            uint64_t *po = a.packed_out + i * a.stride;
#pragma unroll
            for (int j = 0; j < W; ++j) po[j] = x[j];
            for (uint32_t j = W; j < a.stride; ++j) po[j] = 0;
            if (!ok) atomicMin(a.first_bad, (unsigned long long)(a.read_offset + i));
            rc_words<W>(x, a.L, y);
        } else {
#pragma unroll
            for (int j = 0; j < W; ++j) x[j] = y[j] = 0;
        }
    } else if (valid) {
        load_read<W>(a.packed, a.stride, i, x);
        rc_words<W>(x, a.L, y);
    } else {
#pragma unroll
        for (int j = 0; j < W; ++j) x[j] = y[j] = 0;
    }
    for (uint32_t t = threadIdx.x; t < NBIN; t += SC_THREADS) cnt[t] = 0;
    __syncthreads();
    const uint64_t v0 = 2 * (a.read_offset + i);
    FpStreams st;
    const uint32_t nh = min(skip_halves(a.l_lo), 2u * W); // leading bases absorbed in chunks
    fp_skip<W>(x, y, nh, st);
    const uint32_t kskip = 16u * nh;
    uint64_t kk[KPT];
    uint32_t rk[KPT]; // bin << 16 | rank within the bin
    uint32_t kc = 0, lfirst = 0; // lengths buffered this round (block-uniform)
#pragma unroll
    for (int w = 0; w < W; ++w) {
        const uint32_t kb = 32u * w;
        if (kb >= a.l_hi) break;
        if (kb + 32u <= kskip) continue;
        const uint32_t j0 = kskip > kb ? kskip - kb : 0u; // 0 or 16
        uint64_t xa = x[w] >> (2 * j0), yb = y[w] >> (2 * j0);
        const uint32_t kn = min(32u, a.l_hi - kb);
        for (uint32_t j = j0; j < kn; ++j) {
            st.step((uint32_t)(xa & 3u), (uint32_t)(yb & 3u), kb + j);
            xa >>= 2;
            yb >>= 2;
            const uint32_t l = kb + j + 1;
            if (l < a.l_lo) continue; // uniform across the block
            if (kc == 0) lfirst = l;
            if (valid) {
                uint32_t d0, d1; // level-1 digits (implied by the region, not stored)
                const uint64_t e0 = canon_key_d1(st.P0, st.S1, a.keep, a.vbits, v0, &d0);
                const uint64_t e1 = canon_key_d1(st.P1, st.S0, a.keep, a.vbits, v0 + 1, &d1);
                if constexpr (SPLIT) {
                    d0 = (d0 << 1) | (uint32_t)((e0 >> a.vbits) & 1);
                    d1 = (d1 << 1) | (uint32_t)((e1 >> a.vbits) & 1);
                }
#pragma unroll
                for (int q = 0; q < LPR; ++q)
                    if ((uint32_t)q == kc) { // constant register indices after unrolling
                        kk[2 * q] = e0;
                        kk[2 * q + 1] = e1;
                        const uint32_t b0 = q * NBL + d0, b1 = q * NBL + d1;
                        rk[2 * q] = (b0 << 16) | atomicAdd(&cnt[b0], 1u);
                        rk[2 * q + 1] = (b1 << 16) | atomicAdd(&cnt[b1], 1u);
                    }
            }
            ++kc;
            if (kc < (uint32_t)LPR && l < a.l_hi) continue;
            // ---- partition round for lengths lfirst .. lfirst + kc - 1
            __syncthreads();
            uint32_t c[BPT], bs[BPT], sum = 0;
#pragma unroll
            for (int b = 0; b < BPT; ++b) {
                const uint32_t bin = threadIdx.x * BPT + b;
                c[b] = cnt[bin];
                cnt[bin] = 0;
                const uint32_t q = bin / NBL;
                bs[b] = (c[b] && q < kc)
                            ? atomicAdd(&a.fill[(uint64_t)(lfirst - a.l_lo + q) * NBL + bin % NBL], c[b])
                            : 0u;
                sum += c[b];
            }
            uint32_t run = block_scan<SC_THREADS>(sum, wsum);
#pragma unroll
            for (int b = 0; b < BPT; ++b) {
                const uint32_t bin = threadIdx.x * BPT + b;
                const uint32_t q = bin / NBL;
                lstart[bin] = run;
                if ((uint64_t)bs[b] + c[b] > a.cap) {
                    gofs[bin] = -1;
                    *a.overflow = 1u;
                } else {
                    gofs[bin] = (long long)(((uint64_t)(lfirst - a.l_lo + q) * NBL + bin % NBL) * a.cap +
                                            bs[b]) - (long long)run;
                }
                run += c[b];
            }
            if (threadIdx.x == SC_THREADS - 1) lstart[NBIN] = run;
            __syncthreads();
            if (valid) {
#pragma unroll
                for (int q = 0; q < 2 * LPR; ++q)
                    if ((uint32_t)q < 2 * kc) {
                        const uint32_t b = rk[q] >> 16;
                        const uint32_t u = lstart[b] + (rk[q] & 0xFFFFu);
                        stage[u] = kk[q];
                        sbin[u] = (unsigned short)b;
                    }
            }
            __syncthreads();
            const uint32_t total = lstart[NBIN];
            for (uint32_t u = threadIdx.x; u < total; u += SC_THREADS) {
                const long long go = gofs[sbin[u]];
                if (go >= 0) a.out[go + u] = stage[u];
            }
            kc = 0;
            // the next round's first barrier orders these reads before stage/lstart reuse
        }
    }
}

template <int W, bool ASCII, bool SPLIT, int LPR>
__global__ void __launch_bounds__(SC_THREADS, 2)
scatter_table_kernel(ScatterArgs a)
{
    constexpr int NBL = SPLIT ? 512 : 256; // bins per length
    constexpr int NBIN = LPR * NBL;
    constexpr int BPT = NBIN / SC_THREADS; // bins per thread in the round's scan
    constexpr int KPT = 2 * LPR;           // keys per thread per round
    static_assert(NBIN % SC_THREADS == 0 && BPT >= 1 && BPT <= 4, "bins per thread");
    // dynamic: stage[SC_THREADS * KPT] keys, sbin[SC_THREADS * KPT] their bins, then (ASCII)
    // the CTA's staged read bytes
    extern __shared__ __align__(16) uint64_t stage[];
    unsigned short *sbin = reinterpret_cast<unsigned short *>(stage + SC_THREADS * KPT);
    __shared__ uint32_t cnt[NBIN], lstart[NBIN + 1], wsum[16];
    __shared__ uint32_t rbase[SPLIT ? 1 : 256]; // region of (segment 0, digit d); + s * nb_pad
    __shared__ long long gofs[NBIN]; // per bin: element offset of stage slot 0's destination, -1 = overflow

    const uint64_t i = (uint64_t)blockIdx.x * SC_THREADS + threadIdx.x;
    const bool valid = i < a.n;
    uint64_t x[W], y[W];
    if constexpr (ASCII) {
        // a1 fused: stage this CTA's ASCII span (zero-copy from host memory over PCIe when
        // the caller passed page-locked host memory), pack, validate, keep the packed rows
        unsigned char *sascii = reinterpret_cast<unsigned char *>(sbin + SC_THREADS * KPT);
        const uint64_t r0 = (uint64_t)blockIdx.x * SC_THREADS;
        const uint64_t r1 = min64(a.n, r0 + SC_THREADS);
        const uint32_t off = stage_ascii(a.ascii, r0 * a.L, r1 * a.L, sascii, SC_THREADS);
        __syncthreads();
        if (valid) {
            const bool ok = pack_row_regs_swar<W>(sascii + off + (uint64_t)threadIdx.x * a.L, a.L, x);
            uint64_t *po = a.packed_out + i * a.stride;
#pragma unroll
            for (int j = 0; j < W; ++j) po[j] = x[j];
            for (uint32_t j = W; j < a.stride; ++j) po[j] = 0;
            if (!ok) atomicMin(a.first_bad, (unsigned long long)(a.read_offset + i));
            rc_words<W>(x, a.L, y);
        } else {
#pragma unroll
            for (int j = 0; j < W; ++j) x[j] = y[j] = 0;
        }
    } else if (valid) {
        load_read<W>(a.packed, a.stride, i, x);
        rc_words<W>(x, a.L, y);
    } else {
#pragma unroll
        for (int j = 0; j < W; ++j) x[j] = y[j] = 0;
    }
    for (uint32_t t = threadIdx.x; t < NBIN; t += SC_THREADS) cnt[t] = 0;
    if (!SPLIT)
        for (uint32_t d = threadIdx.x; d < 256; d += SC_THREADS)
            rbase[d] = (uint32_t)(shard_region(0, a.l_hi - a.l_lo + 1u, d, a.dest_g, a.nb_pad) -
                                  (a.keep_owner < 0 ? 0ull
                                                    : (uint64_t)a.keep_owner *
                                                          (a.l_hi - a.l_lo + 1u) * a.nb_pad));
    __syncthreads();
    const uint64_t v0 = 2 * (a.read_offset + i);
    Fp64Streams st; // key streams modulo 2^64 (R26)
    // the l_lo - 1 bases before the first emitted length, absorbed in 8-base chunks
    fp64_absorb<W>(x, y, a.l_lo - 1u, st);
    // Base cursors over x (y is dead from here): tx holds base k of r in its low bits; ty
    // holds base L-1-k of r in its top bits, i.e. base k of r' = RC(r) complemented.  A word
    // boundary reloads a cursor from x with a register select (block-uniform branch).
    const uint32_t k = a.l_lo - 1u; // next base to consume (block-uniform)
    uint64_t tx = wsel<W>(x, k >> 5) >> (2u * (k & 31u));
    uint64_t ty;
    {
        const uint32_t m = a.L - 1u - k;
        ty = wsel<W>(x, m >> 5) << (62u - 2u * (m & 31u));
    }
    auto step_base = [&](uint32_t kb) {
        st.step((uint32_t)tx & 3u, (uint32_t)(ty >> 62) ^ 2u, kb);
        tx >>= 2;
        ty <<= 2;
        if (((kb + 1u) & 31u) == 0u) tx = wsel<W>(x, (kb + 1u) >> 5);
        const uint32_t m = a.L - 1u - kb;
        if ((m & 31u) == 0u && m) ty = wsel<W>(x, (m >> 5) - 1u);
    };
    // claimed-end pruning: entry of v0 = 2i needs read end 2i+1 free, entry of 2i+1 needs 2i
    bool live0 = valid, live1 = valid;
    if (a.claimed) { // block-uniform
        if (valid) {
            const uint32_t cw = a.claimed[v0 >> 5] >> (uint32_t)(v0 & 31u);
            live0 = ((cw >> 1) & 1u) == 0u;
            live1 = (cw & 1u) == 0u;
        }
        uint32_t np = valid ? ((uint32_t)!live0 + (uint32_t)!live1) * (a.l_hi - a.l_lo + 1u) : 0u;
        for (int o = 16; o; o >>= 1) np += __shfl_xor_sync(0xffffffffu, np, o);
        if ((threadIdx.x & 31) == 0 && np && a.pruned) atomicAdd(a.pruned, (unsigned long long)np);
    }
    uint64_t kk[KPT];
    uint32_t rk[KPT]; // bin << 16 | rank within the bin
    for (uint32_t lfirst = a.l_lo; lfirst <= a.l_hi; lfirst += LPR) {
        const uint32_t kc = min((uint32_t)LPR, a.l_hi - lfirst + 1u); // lengths this round
#pragma unroll
        for (int q = 0; q < LPR; ++q) {
            if ((uint32_t)q >= kc) break; // block-uniform
            step_base(lfirst + q - 1u);    // the streams now hold length lfirst + q
            rk[2 * q] = rk[2 * q + 1] = ~0u; // no key (pruned or no read)
            if (live0 | live1) {
                uint32_t d0, d1; // level-1 digits (implied by the region, not stored)
                const uint64_t e0 = canon_key64_d1(st.P0, st.S1, a.keep, a.vbits, v0, &d0);
                const uint64_t e1 = canon_key64_d1(st.P1, st.S0, a.keep, a.vbits, v0 + 1, &d1);
                if constexpr (SPLIT) {
                    d0 = (d0 << 1) | (uint32_t)((e0 >> a.vbits) & 1);
                    d1 = (d1 << 1) | (uint32_t)((e1 >> a.vbits) & 1);
                }
                kk[2 * q] = e0;
                kk[2 * q + 1] = e1;
                const uint32_t b0 = q * NBL + d0, b1 = q * NBL + d1;
                bool k0 = live0, k1 = live1;
                if (!SPLIT && a.keep_owner >= 0) { // block-uniform: this sub-pass's digits only
                    k0 = k0 && (int32_t)((d0 * a.dest_g) >> 8) == a.keep_owner;
                    k1 = k1 && (int32_t)((d1 * a.dest_g) >> 8) == a.keep_owner;
                }
                if (k0) rk[2 * q] = (b0 << 16) | atomicAdd(&cnt[b0], 1u);
                if (k1) rk[2 * q + 1] = (b1 << 16) | atomicAdd(&cnt[b1], 1u);
            }
        }
        {
            // ---- partition round for lengths lfirst .. lfirst + kc - 1
            __syncthreads();
            uint32_t c[BPT], bs[BPT], sum = 0;
            uint64_t rg[BPT];
#pragma unroll
            for (int b = 0; b < BPT; ++b) {
                const uint32_t bin = threadIdx.x * BPT + b;
                c[b] = cnt[bin];
                cnt[bin] = 0;
                const uint32_t q = bin / NBL;
                rg[b] = SPLIT ? (uint64_t)(lfirst - a.l_lo + q) * NBL + bin % NBL
                              : (uint64_t)rbase[bin % NBL] + (uint64_t)(lfirst - a.l_lo + q) * a.nb_pad;
                bs[b] = (c[b] && q < kc) ? atomicAdd(&a.fill[rg[b]], c[b]) : 0u;
                sum += c[b];
            }
            uint32_t run = block_scan<SC_THREADS>(sum, wsum);
#pragma unroll
            for (int b = 0; b < BPT; ++b) {
                const uint32_t bin = threadIdx.x * BPT + b;
                lstart[bin] = run;
                if ((uint64_t)bs[b] + c[b] > a.cap) {
                    gofs[bin] = -1;
                    *a.overflow = 1u;
                } else {
                    gofs[bin] = (long long)(rg[b] * a.cap + bs[b]) - (long long)run;
                }
                run += c[b];
            }
            if (threadIdx.x == SC_THREADS - 1) lstart[NBIN] = run;
            __syncthreads();
            if (live0 | live1) {
#pragma unroll
                for (int q = 0; q < 2 * LPR; ++q)
                    if ((uint32_t)q < 2 * kc && rk[q] != ~0u) {
                        const uint32_t b = rk[q] >> 16;
                        const uint32_t u = lstart[b] + (rk[q] & 0xFFFFu);
                        stage[u] = kk[q];
                        sbin[u] = (unsigned short)b;
                    }
            }
            __syncthreads();
            const uint32_t total = lstart[NBIN];
            for (uint32_t u = threadIdx.x; u < total; u += SC_THREADS) {
                const long long go = gofs[sbin[u]];
                if (go >= 0) a.out[go + u] = stage[u];
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
        const unsigned blocks = (unsigned)ceil_div(args.n, SC_THREADS);
        const size_t ascii_b = args.ascii ? (size_t)SC_THREADS * args.L + 32 : 0; // + SWAR overread
        auto run = [&](auto kern, int lpr) -> lasagna_status {
            const size_t smem = (size_t)SC_THREADS * 2 * lpr * (8 + 2) + ascii_b;
            LSG_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                          (int)smem));
            kern<<<blocks, SC_THREADS, smem, s>>>(args);
            LSG_LAUNCHED("scatter_table_kernel");
            return LASAGNA_OK;
        };
        // LASAGNA_SCATTER=1 (A/B measurements only): round-1 form of the kernel
        const char *ev = getenv("LASAGNA_SCATTER");
        if (ev && ev[0] == '1') {
            if (args.split)
                return args.ascii ? run(scatter_table_kernel_v1<W, true, true, 1>, 1)
                                  : run(scatter_table_kernel_v1<W, false, true, 1>, 1);
            return args.ascii ? run(scatter_table_kernel_v1<W, true, false, 4>, 4)
                              : run(scatter_table_kernel_v1<W, false, false, 4>, 4);
        }
        if (args.split)
            return args.ascii ? run(scatter_table_kernel<W, true, true, 1>, 1)
                              : run(scatter_table_kernel<W, false, true, 1>, 1);
        return args.ascii ? run(scatter_table_kernel<W, true, false, 4>, 4)
                          : run(scatter_table_kernel<W, false, false, 4>, 4);
    });
}

// ------------------------------------------------------------------ level k -> k+1
// One CTA owns one region and streams it: the bulk-copy engine prefetches tile t+1 into the
// other half of a double buffer while tile t is ranked (shared atomics: order inside a
// sub-region is irrelevant), staged by digit and written out in digit runs.
template <bool SPLIT, int RF_KPT>
__global__ void __launch_bounds__(RF_THREADS, 1)
refine_kernel(RefineArgs a)
{
    constexpr int RF_TILE = RF_THREADS * RF_KPT;
    constexpr int NBMAX = 512; // 2^dbits bins (x 2 when split), dbits <= 8
    extern __shared__ __align__(128) uint64_t rsm[];
    uint64_t *inb = rsm;                 // [2][RF_TILE]
    uint64_t *rstage = rsm + 2 * RF_TILE; // [RF_TILE]
    __shared__ __align__(8) unsigned long long mbar[2];
    __shared__ uint32_t cnt[NBMAX], lstart[NBMAX], running[NBMAX], wsum[16];
    __shared__ long long gofs[NBMAX];
    const uint32_t nb = (1u << a.dbits) << (SPLIT ? 1 : 0);
    const uint32_t dmask = (1u << a.dbits) - 1u;
    auto binof = [&](uint64_t k) -> uint32_t {
        const uint32_t d = (uint32_t)(k >> a.dshift) & dmask;
        if constexpr (SPLIT) return (d << 1) | (uint32_t)((k >> a.vbits) & 1);
        else return d;
    };
    const uint64_t r = blockIdx.x;
    // the region's entries: n_src source segments (multi-GPU: one per sending rank), region
    // k * src_stride + r of `in`, streamed as one sequence of tiles
    __shared__ uint32_t stile[MAX_REFINE_SRC + 1];
    __shared__ uint64_t scount[MAX_REFINE_SRC];
    if (threadIdx.x == 0) {
        uint32_t acc = 0;
        for (uint32_t k = 0; k < a.n_src; ++k) {
            const uint32_t f = a.fill_in[k * a.src_stride + r];
            if (f > a.cap_in) *a.overflow = 1u;
            scount[k] = min64(f, a.cap_in);
            stile[k] = acc;
            acc += (uint32_t)ceil_div(scount[k], RF_TILE);
        }
        stile[a.n_src] = acc;
    }
    if (threadIdx.x < NBMAX) cnt[threadIdx.x] = 0, running[threadIdx.x] = 0;
    if (threadIdx.x == 0) {
        mbar_init(&mbar[0], 1);
        mbar_init(&mbar[1], 1);
        fence_mbar_init();
    }
    __syncthreads();
    const uint32_t ntiles = stile[a.n_src];
    // source segment of tile t, and its first entry / length inside that segment
    auto tile_src = [&](uint32_t t, const uint64_t **p, uint32_t *m) {
        uint32_t k = 0;
        while (t >= stile[k + 1]) ++k;
        const uint64_t t0 = (uint64_t)(t - stile[k]) * RF_TILE;
        *p = a.in + ((uint64_t)k * a.src_stride + r) * a.cap_in + t0;
        *m = (uint32_t)min64(RF_TILE, scount[k] - t0);
    };
    // bytes of a tile of m entries (rounded up to 16: the region capacity is even, so the
    // rounding stays inside the region)
    auto tile_bytes = [](uint32_t m) { return (uint32_t)((((uint64_t)m * 8) + 15) & ~15ull); };
    if (threadIdx.x == 0 && ntiles) {
        const uint64_t *p;
        uint32_t m;
        tile_src(0, &p, &m);
        bulk_load(inb, p, tile_bytes(m), &mbar[0]);
    }
    for (uint32_t t = 0; t < ntiles; ++t) {
        const uint32_t bsel = t & 1;
        const uint64_t *pcur;
        uint32_t m;
        tile_src(t, &pcur, &m);
        if (threadIdx.x == 0 && t + 1 < ntiles) {
            const uint64_t *p;
            uint32_t mn;
            tile_src(t + 1, &p, &mn);
            fence_proxy_async();
            bulk_load(inb + (bsel ^ 1) * RF_TILE, p, tile_bytes(mn), &mbar[bsel ^ 1]);
        }
        mbar_wait(&mbar[bsel], (t >> 1) & 1);
        const uint64_t *tin = inb + bsel * RF_TILE;
        uint32_t rk[RF_KPT];
#pragma unroll
        for (int q = 0; q < RF_KPT; ++q) {
            const uint32_t idx = q * RF_THREADS + threadIdx.x;
            if (idx < m) rk[q] = atomicAdd(&cnt[binof(tin[idx])], 1u);
        }
        __syncthreads();
        uint32_t c = 0;
        if (threadIdx.x < nb) {
            c = cnt[threadIdx.x];
            cnt[threadIdx.x] = 0;
        }
        const uint32_t ex = block_scan<RF_THREADS>(c, wsum);
        if (threadIdx.x < nb) {
            lstart[threadIdx.x] = ex;
            const uint32_t run = running[threadIdx.x];
            if ((uint64_t)run + c > a.cap_out) {
                gofs[threadIdx.x] = -1;
                *a.overflow = 1u;
            } else {
                gofs[threadIdx.x] =
                    (long long)((r * nb + threadIdx.x) * a.cap_out + run) - (long long)ex;
            }
        }
        __syncthreads();
#pragma unroll
        for (int q = 0; q < RF_KPT; ++q) {
            const uint32_t idx = q * RF_THREADS + threadIdx.x;
            if (idx < m) {
                const uint64_t k = tin[idx];
                rstage[lstart[binof(k)] + rk[q]] = k;
            }
        }
        __syncthreads();
#pragma unroll 4
        for (uint32_t u = threadIdx.x; u < m; u += RF_THREADS) {
            const uint64_t k = rstage[u];
            const long long go = gofs[binof(k)];
            if (go >= 0) a.out[go + u] = k;
        }
        __syncthreads();
        if (threadIdx.x < nb) running[threadIdx.x] += c;
        __syncthreads();
    }
    if (threadIdx.x < nb) {
        a.fill_out[r * nb + threadIdx.x] = running[threadIdx.x];
        if (running[threadIdx.x] > a.cap_out) *a.overflow = 1u;
    }
}

lasagna_status launch_refine(const RefineArgs &args, uint64_t n_regions, cudaStream_t s)
{
    if (n_regions == 0) return LASAGNA_OK;
    if (args.dbits < 1 || args.dbits > 8) return LASAGNA_EINVAL;
    if (args.n_src < 1 || args.n_src > MAX_REFINE_SRC) return LASAGNA_EINVAL;
    // tile of 16 keys per thread (one 512-thread CTA per SM, measured faster than 8 keys at
    // two CTAs per SM: 22 vs 30 ms at cfg3); LASAGNA_RF_KPT=8 selects the smaller tile
    static const int kpt = [] {
        const char *e = getenv("LASAGNA_RF_KPT");
        return (e && atoi(e) == 8) ? 8 : 16;
    }();
    const size_t smem = (size_t)3 * RF_THREADS * kpt * 8;
    auto kern = kpt == 16 ? (args.split ? refine_kernel<true, 16> : refine_kernel<false, 16>)
                          : (args.split ? refine_kernel<true, 8> : refine_kernel<false, 8>);
    LSG_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    kern<<<(unsigned)n_regions, RF_THREADS, smem, s>>>(args);
    LSG_LAUNCHED("refine_kernel");
    return LASAGNA_OK;
}

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
            const uint32_t fc = (uint32_t)min64(f, b.half_cap);
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
#pragma unroll 2
                for (uint32_t k2 = threadIdx.x; k2 < nP; k2 += BJ_THREADS) {
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
    // CTA geometry: LASAGNA_BJ=1 (A/B): 512 threads, 2048-entry halves, two CTAs per SM;
    // LASAGNA_BJ=2: 256 threads, 1024-entry halves, four per SM.  A geometry is only used when
    // a whole bucket half fits its staging buffer twice over.
    int v = 0;
    if (const char *e = getenv("LASAGNA_BJ")) v = atoi(e);
    if (v == 2 && 2 * args.half_cap > 1024) v = 1;
    if (v == 1 && 2 * args.half_cap > 2048) v = 0;
    return dispatch_W(args.j.L, [&](auto wc) -> lasagna_status {
        constexpr int W = decltype(wc)::value;
        if (v == 2) return launch_bucket_join_cfg<W, BjCfg<256, 1024, 1024, 512>>(args, s);
        if (v == 1) return launch_bucket_join_cfg<W, BjCfg<512, 2048, 2048, 1024>>(args, s);
        return launch_bucket_join_cfg<W, BjCfg<1024, 4096, 4096, 2048>>(args, s);
    });
}

} // namespace lsg
