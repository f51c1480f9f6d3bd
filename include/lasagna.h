/*
 * lasagna.h — C ABI of the B200-native LaSAGNA hot path (all-pair suffix-prefix overlaps
 * and the greedy string graph; Goswami et al., IPDPS 2018 = PAPER.md).
 *
 * Citations: "P:L<n>" is PAPER.md line n; R<k> is reading k in DESIGN.md.
 *
 * Conventions (every entry point):
 *   - extern "C"; plain pointers and sizes only.  `stream` is a cudaStream_t (NULL = legacy
 *     default stream) on the CURRENT device; all device work is stream-ordered on it.
 *   - The caller owns every buffer.  The library allocates no device memory (except
 *     lasagna_peer_alloc, the IPC-shareable buffers of the multi-GPU greedy): scratch comes
 *     from a caller-provided workspace whose size the caller obtains first (workspace == NULL
 *     -> *workspace_bytes is set and nothing runs).  Device pointers must be 256-byte aligned
 *     (any torch CUDA tensor's data_ptr() is).
 *   - Arguments are validated before any launch; on error nothing has been launched (except
 *     LASAGNA_ECUDA / LASAGNA_ENOSPC, after which outputs are unspecified).
 *   - Calls that produce host-side outputs (n_pairs, stats, first_bad on the host) synchronise
 *     `stream` before returning; all others are asynchronous.
 *   - Errors are returned, never thrown or aborted; lasagna_last_error() gives the text
 *     (thread-local; valid until this thread's next lasagna_* call).
 *   - Reentrant across streams and devices (no global mutable state besides the thread-local
 *     error text).
 *
 * Terms:
 *   reads r_0..r_{n-1}, each exactly L bases (R14); oriented vertex v = 2i+o with
 *   seq(2i) = r_i and seq(2i+1) = reverse complement of r_i (R8); V = 2n.
 *   Base code c = (ascii >> 1) & 3: A=0 C=1 T=2 G=3 (R1, Fig. 5); complement c^2.
 *   Fingerprint F(s) = sum_k c(s_k) * 5^(|s|-1-k) mod (2^61 - 1) (R2, R4).
 *   Read-end pair (l, a, b), a < b: suffix_l(seq(a)) == prefix_l(seq(b^1)), different reads,
 *   l in [l_min, L-1] (R5, R9); its directed edges are a -> b^1 and its
 *   complement b -> a^1.
 */
#ifndef LASAGNA_H
#define LASAGNA_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define LASAGNA_API __attribute__((visibility("default")))
#else
#define LASAGNA_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    LASAGNA_OK = 0,
    LASAGNA_EINVAL = 1, /* NULL/misaligned pointer, L < 2 or L > 256, l_min < 1 or >= L,
                           host pointer that is not page-locked, unsupported bit range    */
    LASAGNA_ERANGE = 2, /* 2n > 0xFFFFFFFE: vertex ids must fit u32 with NONE reserved
                           ("4-byte vertex-ID")                               */
    LASAGNA_ENOSPC = 3, /* workspace or output capacity too small; the needed size is
                           reported through the size argument                           */
    LASAGNA_ECUDA = 4   /* a CUDA call failed; see lasagna_last_error()                   */
} lasagna_status;

#define LASAGNA_NONE 0xFFFFFFFFu /* succ[] value of a read end without an edge */

LASAGNA_API const char *lasagna_last_error(void);

/* Process-wide count of CUDA kernels launched by this library (monotonic). */
LASAGNA_API uint64_t lasagna_kernel_launches(void);

/* u64 words per packed read (the row stride of `packed`): ceil(L/32) rounded up to 1, 2, 4
 * or 8 so that a read is one aligned 8/16/32/64-byte unit (L <= 128: one 32 B sector). */
LASAGNA_API uint32_t lasagna_words_per_read(uint32_t L);

/* ---------------------------------------------------------------------------------------
 * a1 — stage + 2-bit pack ("batches of reads are loaded in the GPU"; P:L61-67 the
 * host->device level of the two-level streaming model; encoding R1).
 *   ascii     n*L bytes, read i at ascii + i*L, no separators; bytes in ACGTacgt.  Device
 *             memory, or PAGE-LOCKED host memory (read in place over PCIe by the kernel:
 *             zero-copy staging).  Pageable host memory -> LASAGNA_EINVAL.
 *   packed    device u64 [n][lasagna_words_per_read(L)]: base k of read i in bits
 *             [2(k mod 32), 2(k mod 32)+2) of word k/32; unused bits and padding words 0.
 *   first_bad device u64 (one word), written asynchronously: UINT64_MAX if every byte is in
 *             ACGTacgt, else the smallest index of a read holding another byte (R13).  May be
 *             NULL (no report; packed rows of bad reads are then unspecified).
 */
LASAGNA_API lasagna_status lasagna_load_reads(const char *ascii, uint64_t n, uint32_t L, uint64_t *packed,
                                  uint64_t *first_bad, void *stream);

/* ---------------------------------------------------------------------------------------
 * a2 — prefix and suffix fingerprints of every oriented read for every length l in
 * [l_min, L] (Fig. 5/6; both orientations P:L77).  Row k is length l_min + k,
 * column is the vertex v:
 *   pfx[k*2n + v] = F(seq(v)[0..l)),  sfx[k*2n + v] = F(seq(v)[L-l..L))   (device u64).
 * Either output may be NULL.  No reverse complement is materialised: one pass over r gives
 * F of r's prefixes (Horner) and of r''s suffixes (ascending powers), and the same pass over
 * the register-reversed read gives the other two.
 */
LASAGNA_API lasagna_status lasagna_fingerprints(const uint64_t *packed, uint64_t n, uint32_t L,
                                    uint32_t l_min, uint64_t *pfx, uint64_t *sfx, void *stream);

/* ---------------------------------------------------------------------------------------
 * a2-a5 — every read-end pair (the overlap set; Algorithm 2), exact:
 * fingerprint hits are verified on the packed bases (R12), so the result equals the
 * definition.  Output sorted by (l descending, a, b) (R6, R7), a < b:
 *   pair_a, pair_b  device u32[capacity];  pair_l  device u8[capacity]   (any may be NULL
 *   when capacity == 0: count only).
 *   *n_pairs        host out: |P|.  If |P| > capacity -> LASAGNA_ENOSPC (first capacity
 *                   pairs written).
 * workspace: device scratch of *workspace_bytes bytes; workspace == NULL -> query.
 */
LASAGNA_API lasagna_status lasagna_overlaps(const uint64_t *packed, uint64_t n, uint32_t L, uint32_t l_min,
                                void *workspace, size_t *workspace_bytes, uint32_t *pair_a,
                                uint32_t *pair_b, uint8_t *pair_l, uint64_t capacity,
                                uint64_t *n_pairs, void *stream);

/* Approximate mode: as lasagna_overlaps, but a fingerprint hit is
 * accepted when the 128-bit fingerprint pair of the suffix and the prefix agree — F (radix 5
 * mod 2^61 - 1) and F2 (radix 7 mod 2^64 - 59, R22) — instead of the bases.  Equal
 * strings have equal fingerprints, so every exact pair is in the result; a pair whose strings
 * differ appears only if both fingerprints collide (none observed; the oracle's
 * oracle_overlaps_approx is the reference, R23). */
LASAGNA_API lasagna_status lasagna_overlaps_approx(const uint64_t *packed, uint64_t n, uint32_t L,
                                                   uint32_t l_min, void *workspace,
                                                   size_t *workspace_bytes, uint32_t *pair_a,
                                                   uint32_t *pair_b, uint8_t *pair_l,
                                                   uint64_t capacity, uint64_t *n_pairs,
                                                   void *stream);

typedef struct {
    uint64_t n_pairs;          /* |P|: read-end pairs found (overlap edges / 2)             */
    uint64_t n_greedy;         /* pairs accepted by the greedy (directed edges / 2)         */
    uint64_t fp_false_matches; /* table hits whose key bits matched but bases did not (R12) */
    uint64_t kernel_launches;  /* CUDA kernels this call launched                           */
    uint32_t rounds_max;       /* most greedy rounds any length needed                      */
    uint32_t passes;           /* device passes over the packed reads (length groups, a8)   */
    uint32_t lengths_per_pass; /* length-group size the planner chose                       */
    uint32_t key_sort_bits;    /* key bits T the tables are radix-sorted by (bucket bits)   */
    uint32_t sort_launches;    /* onesweep passes launched (each sorts a whole group)       */
    uint32_t search_launches;  /* search (join) launches, one per length                    */
    uint32_t bucketed;         /* 1: radix-partition path (partition_*.cu), 0: exact LSD path */
    /* device time per phase, CUDA events on `stream` (ms).  ms_table covers a1 (when the
     * staging is fused into the first pass), a2 and the level-1 partition: one kernel */
    float ms_table, ms_sort, ms_search, ms_greedy;
    uint64_t greedy_pair_rounds; /* sum over greedy rounds of the candidate pairs visited    */
    uint64_t pruned_entries;     /* table entries dropped by claimed-end pruning (groups after
                                    the first; then n_pairs counts only pairs of entries that
                                    were live when their group was built, not the full |P|) */
    uint32_t partition_levels;   /* bucketed path: MSD partition levels (1..3); 0: exact path */
    uint32_t hash_subpasses;     /* K > 1: each length built and joined in K hash-range
                                    sub-passes (the workspace holds no whole length; f4) */
} lasagna_stats;

/* ---------------------------------------------------------------------------------------
 * a1-a7 — the greedy string graph ("each vertex ... at most one incoming edge and at
 * most one outgoing edge"; lengths in descending order P:L152; ties to the smaller
 * read-end id R7).  Equal, byte for byte, to visiting P in (l desc, a, b) order and
 * accepting a pair iff neither read end is taken:
 *   succ  device u32[2n]: succ[a] = b^1 and succ[b] = a^1 for each accepted (l, a, b),
 *         LASAGNA_NONE elsewhere (the edge a -> b^1 and its complement b -> a^1).
 *   olen  device u8[2n]:  l for both ends of an accepted pair, 0 elsewhere.
 *   stats host out, may be NULL (when non-NULL the call synchronises and times phases).
 * lengths_per_pass: lengths whose tables are built per device pass (a8 semi-streaming);
 *   0 = all of [l_min, L-1] in one pass.  The call uses the largest group <= this that fits
 *   *workspace_bytes; the query (workspace == NULL) reports the size for lengths_per_pass.
 *   When not even one length's tables fit, each length is built and joined in K hash-range
 *   sub-passes (K a power of two <= 256, the smallest that fits; stats->hash_subpasses): the
 *   B200 replacement of the paper's external merge (Alg. 1).
 * Returns LASAGNA_ENOSPC with *workspace_bytes raised when a length produced more candidate
 * pairs than the workspace's pair pool holds (call again with the larger workspace).
 */
LASAGNA_API lasagna_status lasagna_greedy_graph(const uint64_t *packed, uint64_t n, uint32_t L,
                                    uint32_t l_min, uint32_t lengths_per_pass, void *workspace,
                                    size_t *workspace_bytes, uint32_t *succ, uint8_t *olen,
                                    lasagna_stats *stats, void *stream);

/* a1-a7 from the ASCII reads: as lasagna_greedy_graph, with the 2-bit staging (a1) fused into
 * the first table pass when the fast path runs (the packed rows are written to packed_out,
 * device u64 [n][lasagna_words_per_read(L)], for the verification step), so the read-in of
 * host reads over PCIe overlaps the fingerprint computation.
 *   ascii      n*L bytes, device memory or PAGE-LOCKED host memory.  Host input is streamed in
 *              by the DMA engine (a8 level 2): chunks of 512 Ki reads on an internal
 *              copy stream into a ring of up to 64 chunk buffers inside the workspace, each chunk's table
 *              pass launched on `stream` as soon as it lands (event-ordered); off the fast
 *              path, or when the workspace has no room for the ring, it is read in place
 *              (zero-copy).  The host buffer must stay valid until the call returns.
 *   first_bad  device u64: UINT64_MAX, or the smallest index of a read holding a byte outside
 *              ACGTacgt -> the call returns LASAGNA_EINVAL (outputs unspecified).
 * Synchronises `stream` once at the end. */
LASAGNA_API lasagna_status lasagna_greedy_graph_ascii(const char *ascii, uint64_t n, uint32_t L,
                                                      uint32_t l_min, uint32_t lengths_per_pass,
                                                      void *workspace, size_t *workspace_bytes,
                                                      uint64_t *packed_out, uint64_t *first_bad,
                                                      uint32_t *succ, uint8_t *olen,
                                                      lasagna_stats *stats, void *stream);

/* Planner for the semi-streaming driver (a8): the largest
 * lengths_per_pass whose workspace fits `budget_bytes`, and that workspace size; below one
 * whole length, lengths_per_pass = 1 and the workspace of the fewest hash-range sub-passes
 * that fit.  Returns LASAGNA_ENOSPC when not even 256 sub-passes fit (*workspace_bytes =
 * minimum). */
LASAGNA_API lasagna_status lasagna_plan(uint64_t n, uint32_t L, uint32_t l_min, size_t budget_bytes,
                            uint32_t *lengths_per_pass, size_t *workspace_bytes);

/* ---------------------------------------------------------------------------------------
 * Compress (PAPER §III-D, Fig. 7): paths and contigs of the
 * greedy string graph (succ/olen as lasagna_greedy_graph writes them; packed rows as a1).
 *   A path starts at a seed — a vertex with in-degree 0 and out-degree 1 — and
 *   follows succ until a vertex without an out-edge.  The overhang of a vertex is L - olen
 *   with an out-edge, L without.  The contig of a path is the concatenation of
 *   seq(v)[0 .. overhang(v)) over its vertices, ASCII ACGT.  Every path has a
 *   complementary path (seed = its tail ^ 1) spelling the reverse complement; only the one
 *   with the smaller seed id is emitted (R20).  Cycles (no seed) and edgeless reads give no
 *   contig (R21).  Contigs are ordered by seed id.
 *   contigs         device char[contig_capacity]: the contigs back to back
 *   contig_offsets  device u64[count_capacity]: contig c = contigs[off[c] .. off[c+1])
 *   contig_seed     device u32[count_capacity - 1] or NULL: the seed vertex of contig c
 *   *n_contigs, *total_bases  host out.  A capacity below total_bases bases or n_contigs + 1
 *                   offsets -> LASAGNA_ENOSPC (sizes reported, nothing written).
 * workspace: device scratch (28 B per vertex); workspace == NULL -> query.  Synchronises. */
LASAGNA_API lasagna_status lasagna_compress(const uint64_t *packed, uint64_t n, uint32_t L,
                                            const uint32_t *succ, const uint8_t *olen,
                                            void *workspace, size_t *workspace_bytes,
                                            char *contigs, uint64_t contig_capacity,
                                            uint64_t *contig_offsets, uint32_t *contig_seed,
                                            uint64_t count_capacity, uint64_t *n_contigs,
                                            uint64_t *total_bases, void *stream);

/* ---------------------------------------------------------------------------------------
 * Phase entry points (exported for tests and the multi-GPU driver).
 *
 * a4 — stable LSD radix sort (K4 P:L144) of `count` u64 keys by bits
 * [bit_lo, bit_hi) (0 <= bit_lo < bit_hi <= 64), 8-bit digits, one onesweep pass per digit.
 * keys: device in/out; the sorted keys end in `keys`.  scratch: device u64[count].
 */
LASAGNA_API lasagna_status lasagna_sort_u64(uint64_t *keys, uint64_t *scratch, uint64_t count,
                                uint32_t bit_lo, uint32_t bit_hi, void *workspace,
                                size_t *workspace_bytes, void *stream);

/* a6 — the greedy claim alone, on a caller-given candidate list: pairs
 * (pl[i], pa[i], pb[i]) with pa < pb < 2n, no duplicates, any order.  Result equals the
 * sequential greedy over the list sorted by (l desc, a, b).  succ/olen as above, fully
 * written.  *rounds (host out, may be NULL) = total locally-dominant rounds used. */
LASAGNA_API lasagna_status lasagna_greedy_pairs(uint64_t n, const uint8_t *pl, const uint32_t *pa,
                                    const uint32_t *pb, uint64_t count, void *workspace,
                                    size_t *workspace_bytes, uint32_t *succ, uint8_t *olen,
                                    uint32_t *rounds, void *stream);

/* ---------------------------------------------------------------------------------------
 * Sharded phases: the building blocks of the multi-GPU driver (one process per GPU, tables
 * partitioned by hash range; paper_conf_ipps_goswamilsp18_b200/dist.py).  The key layout is
 * the one lasagna_greedy_graph uses internally for a read set of n_total reads: ONE canonical
 * entry per oriented read v and length l.  With
 * x = prefix_l(seq(v)), H = F(x) and Hr = F(RC(x)) (= F(suffix_l(seq(v^1)))):
 *   key  = mix(min(H, Hr)) top (62 - vbits) bits | flag << vbits | global vertex id
 *   flag = 0 if H < Hr, 1 if H > Hr, 2 if H == Hr;  mix(f) = f * 0x9E3779B97F4A7C15 mod 2^64;
 *   vbits = lasagna_vertex_bits(n_total).
 * The paper's prefix list P_l is the build side (flags 0 and 2), its suffix list S_l
 * the probe side (flags 1 and 2): suffix_l(seq(u)) == prefix_l(seq(v)) iff the prefixes of
 * u^1 and v are reverse complements, i.e. equal canonical fingerprints with opposite flags
 * (or both 2).  The join needs the keys of one length sorted by their top
 * lasagna_key_sort_bits(n_total) bits.  A hash-range shard is any set of keys sharing their
 * top bits.
 */
LASAGNA_API uint32_t lasagna_vertex_bits(uint64_t n_total);
LASAGNA_API uint32_t lasagna_key_sort_bits(uint64_t n_total);

/* a2/a3 for the reads [read_offset, read_offset + n_local) of an n_total-read set whose packed
 * rows start at `packed`: tab[(l - l_lo) * 2 n_local + 2i + o] = the canonical key of vertex
 * 2(read_offset + i) + o at length l, for l in [l_lo, l_hi] (at most 64 lengths), i local read,
 * o orientation.  Asynchronous. */
LASAGNA_API lasagna_status lasagna_table_keys(const uint64_t *packed, uint64_t n_local,
                                              uint64_t read_offset, uint64_t n_total, uint32_t L,
                                              uint32_t l_lo, uint32_t l_hi, uint64_t *tab,
                                              void *stream);

/* counts[s*256 + d] = number of keys of segment s (n_seg segments of seg_len keys) whose
 * bits [shift, shift+bits) equal d (bits <= 8).  counts is zeroed by the call.  Async. */
LASAGNA_API lasagna_status lasagna_digit_counts(const uint64_t *keys, uint64_t seg_len,
                                                uint32_t n_seg, uint32_t shift, uint32_t bits,
                                                uint32_t *counts, void *stream);

/* a4, segmented: n_seg independent arrays of seg_len keys (contiguous), each sorted stably
 * by bits [bit_lo, bit_hi); result in keys.  Workspace query as usual.  Async. */
LASAGNA_API lasagna_status lasagna_sort_segments(uint64_t *keys, uint64_t *scratch,
                                                 uint64_t seg_len, uint32_t n_seg, uint32_t bit_lo,
                                                 uint32_t bit_hi, void *workspace,
                                                 size_t *workspace_bytes, void *stream);

/* a5 on one length l: `keys` (count entries, any hash-range shard of length l's table, sorted
 * by the top lasagna_key_sort_bits(n_total) bits); packed_all = the packed rows of ALL n_total
 * reads (verification).  Appends the verified read-end pairs (a << 32) | b, a < b, to pairs
 * (at most capacity are stored); counters (device u64[2]) accumulate [0] pairs found (may
 * exceed capacity: overflow) and [1] rejected fingerprint matches.  Async. */
LASAGNA_API lasagna_status lasagna_join(const uint64_t *keys, uint64_t count,
                                        const uint64_t *packed_all, uint64_t n_total, uint32_t L,
                                        uint32_t l, uint64_t *pairs, uint64_t capacity,
                                        uint64_t *counters, void *stream);

/* ---------------------------------------------------------------------------------------
 * Sharded FAST path (the multi-GPU driver's default).  g = world ranks,
 * one process per GPU.  Rank r holds the reads [r n_pad, min(n_total, (r+1) n_pad)) with
 * n_pad = lasagna_shard_geom.n_pad (ceil(n_total / g) rounded up to 16), and OWNS the read ends
 * [r slice, (r+1) slice), slice = 2 n_pad, for the greedy.  The level-1 digit d (top 8 bits of
 * the mixed canonical fingerprint) belongs to rank o = floor(d g / 256): the hash-range
 * partition of P:L333 (the paper's shuffle P:L204, re-keyed by fingerprint).  Per length group
 * [l_lo, l_hi] (G <= 64 lengths):
 *   1. lasagna_shard_scatter: keys of the rank's reads into `send`, [g][G][nb_pad][cap1] u64
 *      (+ fills [g][G][nb_pad] u32): the slice for rank o is contiguous and equally sized;
 *   2. the caller exchanges send -> recv and send_fill -> recv_fill with two all-to-alls of
 *      EQUAL split sizes (G nb_pad cap1 keys, G nb_pad fills per rank pair): no count
 *      exchange, no host synchronisation;
 *   3. lasagna_shard_partition: the remaining radix levels over the g received slices;
 *   4. per length l (descending): lasagna_shard_join into the rank's pair pool, then
 *      lasagna_greedy_shard_length.
 * counters: device u64[4], zeroed by the caller once per call: [0] nonzero = a slack region
 * overflowed (the result is incomplete: rerun on the exact path), [1] entries pruned (claimed
 * ends, f1), [2] reserved, [3] rejected fingerprint matches.  All calls are asynchronous.
 */
typedef struct {
    uint32_t levels;       /* MSD partition levels (2 or 3)                                  */
    uint32_t last_bits;    /* bits of the last level                                        */
    uint32_t nb_pad;       /* level-1 digits per rank, padded: ceil(256 / g)                 */
    uint32_t vbits;        /* vertex-id bits of a key                                        */
    uint64_t n_pad;        /* reads per rank                                                 */
    uint64_t slice;        /* read ends owned per rank (2 n_pad, a multiple of 32)           */
    uint64_t cap1;         /* level-1 region capacity (keys)                                 */
    uint64_t send_entries; /* keys of send (= of recv) PER LENGTH: g nb_pad cap1             */
    uint64_t fill_words;   /* u32 fills of send_fill (= of recv_fill) PER LENGTH: g nb_pad    */
    uint64_t part_bytes;   /* workspace of lasagna_shard_partition for ONE length            */
    uint64_t buckets;      /* final buckets per length on one rank                           */
} lasagna_shard_geom;

LASAGNA_API lasagna_status lasagna_shard_geometry(uint64_t n_total, uint32_t world, uint32_t L,
                                                  uint32_t l_min, lasagna_shard_geom *out);
/* workspace bytes of lasagna_shard_partition for a group of `lengths` lengths */
LASAGNA_API lasagna_status lasagna_shard_part_bytes(uint64_t n_total, uint32_t world, uint32_t L,
                                                    uint32_t l_min, uint32_t lengths, size_t *bytes);
/* packed_local: the rank's packed rows (device); read_offset = r n_pad; claimed: the rank's
 * slice of the claimed-end bitmap (device, slice/32 words) or NULL (no pruning). */
LASAGNA_API lasagna_status lasagna_shard_scatter(const uint64_t *packed_local, uint64_t n_local,
                                                 uint64_t read_offset, uint64_t n_total,
                                                 uint32_t world, uint32_t L, uint32_t l_min,
                                                 uint32_t l_lo, uint32_t l_hi,
                                                 const uint32_t *claimed, uint64_t *send,
                                                 uint32_t *send_fill, uint64_t *counters,
                                                 void *stream);
/* recv/recv_fill: the g received slices, sender-major; part: lasagna_shard_part_bytes bytes. */
LASAGNA_API lasagna_status lasagna_shard_partition(const uint64_t *recv, const uint32_t *recv_fill,
                                                   uint64_t n_total, uint32_t world, uint32_t L,
                                                   uint32_t l_min, uint32_t l_lo, uint32_t l_hi,
                                                   void *part, uint64_t *counters, void *stream);
/* a5 of length l over this rank's buckets: verified pairs (a << 32) | b, a < b, written to
 * pool (device u64[capacity]); *pool_count (device u64) is zeroed, then counts every pair found
 * (may exceed capacity: overflow).  packed_all: the packed rows of all n_total reads. */
LASAGNA_API lasagna_status lasagna_shard_join(const void *part, uint64_t n_total, uint32_t world,
                                              uint32_t L, uint32_t l_min, uint32_t l_lo,
                                              uint32_t l_hi, uint32_t l,
                                              const uint64_t *packed_all, uint64_t *pool,
                                              uint64_t capacity, uint64_t *pool_count,
                                              uint64_t *counters, void *stream);

/* a6/a7 sharded (the reduce step P:L206-210): the greedy of length l over the
 * pairs every rank's pool holds, each rank owning best/claimed/succ/olen of its slice of read
 * ends.  ranks[q] describes rank q with pointers VALID IN THIS PROCESS (peer memory opened with
 * lasagna_peer_open: NVLink loads, stores and atomics); the ranks meet at device-side barriers
 * in their ctr words, so every rank must make the same sequence of calls.  rank = -1 runs all
 * `world` ranks in one launch (one GPU: a test of the protocol).  Result: the single-GPU
 * greedy over the union of the pools, bit for bit.
 *   pool, pool2   device u64[capacity]: the rank's pairs (count *pool_count) and scratch
 *   ctr           device u64[16], zeroed before the call's first length: [3] pairs accepted,
 *                 [4] sum of |P_l|, [5] max |P_l|, [6] max rounds, [7] pairs visited
 *   best          device u64[slice], zeroed before the first length
 *   claimed       device u32[slice/32], zeroed before the first length (bit x: end x claimed)
 *   succ, olen    device u32[slice] (LASAGNA_NONE), u8[slice] (0) initialised by the caller
 *   tail          rank 0: device u64[4096] (the gathered survivors); others may be NULL
 * world = 1: slice is ignored (one rank owns every end). */
typedef struct {
    uint64_t *pool, *pool2;
    uint64_t *pool_count; /* the pair count; the rounds reuse it as a list counter */
    uint64_t *ctr;
    uint64_t *best;
    uint32_t *claimed;
    uint32_t *succ;
    uint8_t *olen;
    uint64_t *tail;
} lasagna_greedy_rank;
LASAGNA_API lasagna_status lasagna_greedy_shard_length(const lasagna_greedy_rank *ranks,
                                                       uint32_t world, int32_t rank,
                                                       uint64_t slice, uint64_t capacity,
                                                       uint32_t l, void *stream);

/* Peer memory (CUDA IPC): the one place the library allocates device memory.  alloc returns a
 * device buffer and its 64-byte IPC handle; another process opens it with peer_open (the
 * device pointer is valid there until peer_close); free releases the owner's buffer. */
LASAGNA_API lasagna_status lasagna_peer_alloc(size_t bytes, void **dev_ptr, void *handle);
LASAGNA_API lasagna_status lasagna_peer_free(void *dev_ptr);
LASAGNA_API lasagna_status lasagna_peer_open(const void *handle, void **dev_ptr);
LASAGNA_API lasagna_status lasagna_peer_close(void *dev_ptr);

#ifdef __cplusplus
}
#endif

#endif /* LASAGNA_H */
