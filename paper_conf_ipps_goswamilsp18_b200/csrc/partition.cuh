// partition.cuh — shared pieces of the bucketed (MSD radix-partition) form of a3/a4/a5, the fast path of
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
#pragma once

#include <cstdlib>

#include "fingerprint.cuh"
#include "pack.cuh"
#include "joinwin.cuh"

namespace lsg {

constexpr int SC_THREADS = 512; // reads per scatter CTA (one per thread)
constexpr int RF_THREADS = 512;


// exclusive scan of v over the first NB threads (NB a multiple of 32, <= 512); every thread of
// the block must call it.  wsum: 16 shared words.  The caller must pass a block barrier before
// the next call (both callers do: their offsets are published with one right after).
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
    return x - v + add;
}

} // namespace lsg
