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
    // approximate mode: hits are accepted by the 128-bit fingerprint
    // pair (common.cuh verify_fp128) instead of the bases
    bool approx = false;
    uint64_t V = 0; // vertex ids in the pairs are < V (checked build; 0: not checked)
    // greedy mode, single GPU: store the fingerprint hits unverified; the greedy's first round
    // verifies them on the bases (greedy_rounds.cu), in parallel with its random proposals
    bool defer_verify = false;
};
// the check a hit passes: bases (exact) or the fingerprint pair (approximate mode)
template <int W>
__device__ __forceinline__ bool verify_pair(const JoinArgs &a, uint32_t u, uint32_t v)
{
    return a.approx ? verify_fp128<W>(a.packed, a.stride, a.L, u, v, a.l)
                    : verify_overlap<W>(a.packed, a.stride, a.L, u, v, a.l);
}
lasagna_status launch_join(const JoinArgs &a, cudaStream_t s);
lasagna_status launch_pairs_to_keys(const unsigned long long *pool, const unsigned long long *count,
                                    uint64_t m, unsigned long long cap, uint32_t vbits,
                                    uint64_t *keys, cudaStream_t s);
lasagna_status launch_keys_to_output(const uint64_t *keys, uint64_t m, uint32_t vbits, uint8_t l,
                                     uint32_t *pa, uint32_t *pb, uint8_t *pl, cudaStream_t s);

// ---- bucketed a3/a4/a5 (partition_*.cu)
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
    // hash-range shards (multi-GPU, not split): level-1 digit d belongs to rank
    // o = d * dest_g >> 8, whose digits start at first(o) = ceil(256 o / dest_g); region of
    // (length s, digit d) = (o * G + s) * nb_pad + d - first(o), nb_pad = ceil(256 / dest_g),
    // so every rank's regions of all G lengths are one contiguous slice of out/fill (equal
    // split sizes for the all-to-all).  dest_g = 1, nb_pad = 256: the single-GPU [G][256].
    uint32_t dest_g = 1, nb_pad = 256;
    // hash-range sub-pass (single GPU, tables larger than the workspace): keep only the keys
    // whose level-1 digit belongs to range keep_owner of dest_g, regions numbered from 0
    int32_t keep_owner = -1;
};
// region index of (segment s of G, level-1 digit d) under ScatterArgs' shard layout
__host__ __device__ __forceinline__ uint64_t shard_region(uint32_t s, uint32_t G, uint32_t d,
                                                          uint32_t dest_g, uint32_t nb_pad)
{
    const uint32_t o = (d * dest_g) >> 8;
    const uint32_t first = (o * 256u + dest_g - 1u) / dest_g;
    return ((uint64_t)o * G + s) * nb_pad + (d - first);
}
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
    // multi-GPU: region r of the output gathers the input regions k * src_stride + r of
    // n_src senders (1 <= n_src <= MAX_REFINE_SRC); single GPU: n_src = 1
    uint32_t n_src = 1;
    uint64_t src_stride = 0;
};
constexpr uint32_t MAX_REFINE_SRC = 64;
lasagna_status launch_refine(const RefineArgs &a, uint64_t n_regions, cudaStream_t s);
struct BucketJoinArgs {
    JoinArgs j;               // packed, L, stride, l, vbits, pairs, cap, count, false_matches
    uint64_t *buckets;        // [n_buckets][2][half_cap]: prefix half, suffix half (the join
                              // writes sentinels after odd fills)
    const uint32_t *fills;    // [n_buckets][2]
    uint64_t half_cap, n_buckets;
    uint32_t *overflow;
    bool planner_builds = false; // A/B: the planning warp takes a build share too
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

// ---- a6/a7, two launches per length (greedy_rounds.cu), single GPU or sharded over ranks
constexpr uint32_t MAX_PEERS = 8;
// per-rank u64 counters (PeerRank::ctr, PC_N words, zeroed once per call)
enum { PC_RING = 0,    // [3] live-list counts of the round phases
       PC_BOOK = 3,    // [4] accepted, sum |P_l|, max |P_l|, max rounds (as GreedyBufs::book)
       PC_WORK = 7,    // sum over rounds of the pairs visited
       PC_EPOCH = 8,   // last proposal epoch used (0: none)
       PC_ARRIVE = 9, PC_GEN = 10,   // barrier of one rank's blocks
       PC_XARRIVE = 11, PC_XCOUNT = 12, // cross-rank barrier: arrivals, barriers completed
       PC_TAILEPOCH = 13, PC_TAILIN = 14, PC_N = 16 }; // rank 0's last tail epoch; survivors
struct PeerRank {
    unsigned long long *pool, *pool2; // this rank's candidate pairs (pool) and scratch list
    unsigned long long *in_count;     // device: pairs in pool (the join's counter; ring slot 0)
    unsigned long long *ctr;          // PC_N words
    unsigned long long *best;         // owned slice of the epoch-tagged proposals
    uint32_t *claimed;                // owned slice of the claimed bitmap
    uint32_t *succ;                   // owned slices of the outputs
    uint8_t *olen;
    unsigned long long *tail;         // rank 0: gathered survivors (GR_TAIL_MAX pairs)
};
struct GreedyPeers {
    PeerRank r[MAX_PEERS];
    uint32_t g = 1;           // ranks
    uint64_t slice = 0;       // read ends per rank (multiple of 32): end x on rank x / slice
    unsigned long long cap = 0; // pool capacity
    uint32_t rank0 = 0;       // first rank this launch runs (multi-GPU: my rank)
    uint32_t nranks_here = 1; // ranks this launch runs (> 1: one-GPU test of the protocol)
    uint32_t bpr = 0;         // blocks per rank (0: sized from cap)
    // deferred verification (single GPU, JoinArgs::defer_verify): the first round checks every
    // candidate on the bases (R12) before proposing; true pairs are counted in
    // ctr[PC_BOOK + 1] (|P_l|), rejected hits in *vfalse.  vpacked = nullptr: verified by the join
    const uint64_t *vpacked = nullptr;
    uint32_t vL = 0, vstride = 0;
    unsigned long long *vfalse = nullptr;
};
constexpr uint32_t GR_TAIL_CAP = 4096;
lasagna_status greedy_length_peers(const GreedyPeers &p, uint8_t l, cudaStream_t s);
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
