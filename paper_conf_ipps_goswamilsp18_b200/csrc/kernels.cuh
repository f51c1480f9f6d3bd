// kernels.cuh — argument structs and host launchers shared between the translation units
// of liblasagna.so (pack.cu, fingerprint.cu, sort.cu, search.cu, greedy.cu, lasagna.cu).
#pragma once

#include "common.cuh"

namespace lsg {

// ---- a1 (pack.cu)
lasagna_status launch_pack(const char *ascii, uint64_t n, uint32_t L, uint64_t *packed,
                           uint64_t *first_bad, cudaStream_t s);

// ---- a2/a3 (fingerprint.cu)
lasagna_status launch_fp_values(const uint64_t *packed, uint64_t n, uint32_t L, uint32_t l_min,
                                uint64_t *pfx, uint64_t *sfx, cudaStream_t s);

struct TableArgs {
    const uint64_t *packed;
    uint64_t n;               // reads in this range
    uint64_t read_offset;     // global id of the first read (vertex ids are global)
    uint32_t L, stride;
    uint32_t l_lo, l_hi;      // group of lengths (segment s = l - l_lo)
    uint32_t vbits;           // b_v: vertex-id bits at the bottom of a key
    uint32_t d_shift, d_bits; // first LSD digit (histogram produced on the fly)
    uint64_t *tab;            // [G][V]: entry v = canonical key of vertex v (common.cuh)
    uint32_t *hist;           // [G][256] first-digit histogram, or null
};
lasagna_status launch_table(const TableArgs &a, cudaStream_t s);

// ---- a4 (sort.cu)
struct SortCtx {
    unsigned long long *status; // look-back words
    size_t status_bytes;
    uint32_t *tile_ctrs;        // [SORT_CTRS]
    uint32_t epoch;             // last used
};
constexpr uint32_t SORT_CTRS = 4096;
size_t sort_status_bytes(uint64_t seg_len, uint32_t n_seg);
lasagna_status sort_ctx_reset(SortCtx &c, cudaStream_t s);
void digit_plan(uint32_t lo, uint32_t hi, uint32_t *P, uint32_t *shifts, uint32_t *bits);
lasagna_status sort_segments(uint64_t *bufs[2], uint64_t seg_len, uint32_t n_seg, uint32_t lo,
                             uint32_t hi, uint32_t *hist, bool hist0_ready, SortCtx &ctx,
                             cudaStream_t s, int *which);
lasagna_status launch_hist(const uint64_t *keys, uint64_t seg_len, uint32_t n_seg, uint32_t shift,
                           uint32_t bits, uint32_t *hist, cudaStream_t s);

// ---- a5 (search.cu)
struct JoinArgs {
    const uint64_t *packed;
    const uint64_t *keys;      // sorted canonical table of this length (N = V entries)
    uint64_t N;
    uint32_t L, stride, l, vbits, T; // T: sorted (bucket) bits
    unsigned long long *pairs; // out pool: (a << 32) | b
    unsigned long long cap;
    unsigned long long *count; // pool fill (may exceed cap: overflow)
    unsigned long long *false_matches;
    // greedy mode (may be null): pairs with a read end already claimed by a longer length
    // (bitmap) are counted in *found but not stored — they can never be accepted
    const uint32_t *claimed = nullptr;
    unsigned long long *found = nullptr;
};
lasagna_status launch_join(const JoinArgs &a, cudaStream_t s);
lasagna_status launch_pairs_to_keys(const unsigned long long *pool, const unsigned long long *count,
                                    uint64_t m, unsigned long long cap, uint32_t vbits,
                                    uint64_t *keys, cudaStream_t s);
lasagna_status launch_keys_to_output(const uint64_t *keys, uint64_t m, uint32_t vbits, uint8_t l,
                                     uint32_t *pa, uint32_t *pb, uint8_t *pl, cudaStream_t s);

// ---- bucketed a3/a4/a5 (partition.cu)
struct ScatterArgs {
    const uint64_t *packed;
    uint64_t n, read_offset;
    uint32_t L, stride, l_lo, l_hi, vbits;
    uint64_t keep;      // stored fingerprint bits (key_keep(vbits); tests may clear low ones)
    uint64_t *out;      // [G][256][cap] level-1 regions (top 8 bits of mix(min(H, Hr)), not
                        // stored: common.cuh canon_key_d1); split: [G][256][2][cap]
                        // (half 0: flags 0/2 = build side, half 1: flag 1 = probe side)
    uint32_t *fill;     // [G][256] (split: [G][256][2])
    uint64_t cap;
    uint32_t *overflow;
    bool split;         // final level: prefix and suffix entries in separate halves
    // a1 fused in (optional): read ASCII (device or page-locked host memory) instead of
    // `packed`, write the packed rows to packed_out and report bad reads in first_bad
    const unsigned char *ascii;
    uint64_t *packed_out;
    unsigned long long *first_bad;
    // claimed-end pruning (may be null): the entry of vertex v is dropped when
    // read end v^1 is already claimed (bitmap of 2n bits) — every pair it could produce
    // contains v^1, which the greedy would reject; pruned entries are counted
    const uint32_t *claimed = nullptr;
    unsigned long long *pruned = nullptr;
};
lasagna_status launch_scatter_table(const ScatterArgs &a, cudaStream_t s);
struct RefineArgs {
    const uint64_t *in;
    const uint32_t *fill_in;
    uint64_t cap_in;
    uint32_t dshift;    // this level's digit: key bits [dshift, dshift + dbits)
    uint32_t dbits;     // 1..8
    uint64_t *out;      // [regions][2^dbits][cap_out] (split: [regions][2^dbits][2][cap_out])
    uint32_t *fill_out; // [regions][2^dbits] (split: [regions][2^dbits][2])
    uint64_t cap_out;
    uint32_t vbits;
    uint32_t *overflow;
    bool split;
};
lasagna_status launch_refine(const RefineArgs &a, uint64_t n_regions, cudaStream_t s);
struct BucketJoinArgs {
    JoinArgs j;               // packed, L, stride, l, vbits, pairs, cap, count, false_matches
    uint64_t *buckets;        // [n_buckets][2][half_cap]: prefix half, suffix half (the join
                              // writes sentinels after odd fills)
    const uint32_t *fills;    // [n_buckets][2]
    uint64_t half_cap, n_buckets;
    uint32_t *overflow;
};
lasagna_status launch_bucket_join(const BucketJoinArgs &a, cudaStream_t s); // block windows
lasagna_status launch_warp_join(const BucketJoinArgs &a, cudaStream_t s);   // warp per bucket
bool warp_join_fits(const BucketJoinArgs &a); // a bucket half fits a warp's staging slice

// ---- a6/a7 (greedy.cu)
struct GreedyBufs {
    unsigned long long *pool, *pool2; // pair lists (ping-pong)
    unsigned long long *cnt, *cnt2;   // their fills (device); cnt: the input count
    unsigned long long *cnt3;         // third round counter (zero, like cnt2, on the first call)
    unsigned long long *book;         // device: [0] accepted, [1] sum |P_l|, [2] max |P_l|, [3] max rounds
    unsigned long long *work;         // device: sum over rounds of the pairs a round visits
    unsigned long long *best;         // u64 [V]: epoch-tagged proposals, zeroed once per call
    uint32_t *claimed;                // bitmap of claimed read ends (2n bits)
    unsigned long long cap;
    uint32_t epoch;                   // next free epoch (host side)
};
lasagna_status greedy_length(GreedyBufs &g, uint8_t l, uint32_t *succ, uint8_t *olen,
                             cudaStream_t s);
lasagna_status launch_gather_pairs(const uint64_t *order, uint64_t off, uint64_t m,
                                   const uint32_t *pa, const uint32_t *pb,
                                   unsigned long long *pool, unsigned long long *cnt,
                                   cudaStream_t s);
lasagna_status launch_lkeys(const uint8_t *pl, uint64_t count, uint64_t *keys, cudaStream_t s);

// ---- Compress (compress.cu)
lasagna_status compress_impl(const uint64_t *packed, uint64_t n, uint32_t L, const uint32_t *succ,
                             const uint8_t *olen, void *workspace, size_t *workspace_bytes,
                             char *contigs, uint64_t contig_capacity, uint64_t *contig_offsets,
                             uint32_t *contig_seed, uint64_t count_capacity, uint64_t *n_contigs,
                             uint64_t *total_bases, cudaStream_t s);

} // namespace lsg
