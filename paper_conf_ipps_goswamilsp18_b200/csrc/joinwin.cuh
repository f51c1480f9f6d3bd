// joinwin.cuh — the shared-memory join of one window of whole buckets (a5), used by the
// contiguous-table join (search.cu) and the bucketed join (partition_join.cu).
//
// A window holds the entries of complete T-bit buckets, so every fingerprint match of a
// probe entry is a build entry of the same window ("a fingerprint present in W_S
// cannot be present in any window except W_P").  Entries are canonical (common.cuh): the
// build side (flags 0 and 2) plays the paper's prefix list, the probe side (flags 1 and 2)
// its suffix list.  The build entries are hashed (chained table in shared memory, one
// atomicExch per insert), every probe entry looks its key up (all matches of its key: the
// C = U - L matches of P:L164-166), and each candidate from a different read is staged, then
// verified on the 2-bit bases in a parallel pass (R12) and written to the global pool as the
// read-end pair (a << 32) | b, a < b.
#pragma once

#include "kernels.cuh"

namespace lsg {

constexpr int JOIN_THREADS = 512;
constexpr int JOIN_CHUNK = 2048;   // nominal entries per CTA
constexpr int JOIN_CAP = 6144;     // staged entries per CTA (chunk + the bucket straddling its end)
constexpr int JOIN_SLOTS = 8192;   // hash chain heads (u32); chains through next[] (u16)
constexpr int JOIN_BUF = 1024;     // staged output pairs (2 per thread of a JOIN_THREADS block)

// Candidates are staged in shared memory and verified in a separate, fully parallel pass
// (a fingerprint match is rare: verifying it inline would run the long verify path with one
// or two active lanes per warp).
struct Stager {
    unsigned long long *buf; // shared: staged (u << 32 | b) records, ~0 = rejected
    uint32_t *bcount;        // shared
    unsigned long long *pairs, cap, *count;
    uint32_t bufcap = JOIN_BUF; // records `buf` holds (2 per thread of the block)
};

// Fingerprint match of probe entry e (vertex w, flag 1 or 2) and build entry p (vertex v,
// flag 0 or 2): if the bases agree, the l-prefixes of w and v are reverse complements, i.e.
// suffix_l(seq(w^1)) == prefix_l(seq(v)): the directed overlap (w^1, v, l) and its read-end
// pair {w^1, v^1}.  Each pair has exactly one (build, probe) assignment, except when
// both entries carry flag 2 (each probes the other): then only w < v is kept.
template <int W>
__device__ __forceinline__ void candidate(const JoinArgs &a, uint64_t e, uint64_t p,
                                          uint64_t vmask, Stager &sg, unsigned long long &nfalse)
{
    const uint32_t w = (uint32_t)(e & vmask), v = (uint32_t)(p & vmask);
    LSG_DCHECK(a.V == 0 || (w < a.V && v < a.V));
    if ((w >> 1) == (v >> 1)) return; // R9: no same-read edge (also the entry itself)
    if (w > v && key_flag(e, a.vbits) == 2 && key_flag(p, a.vbits) == 2) return;
    const uint32_t x = w ^ 1u, y = v ^ 1u;
    const uint32_t lo = min(x, y), hi = max(x, y);
    const unsigned long long rec = ((unsigned long long)lo << 32) | hi;
    const uint32_t slot = atomicAdd(sg.bcount, 1u);
    if (slot < sg.bufcap) {
        sg.buf[slot] = rec;
        return;
    }
    // staging full: verify inline (unless the greedy verifies) and emit straight to global memory
    if (!a.defer_verify && !verify_pair<W>(a, lo, hi ^ 1u)) {
        ++nfalse;
        return;
    }
    if (a.found) atomicAdd(a.found, 1ull);
    if (a.claimed && (((a.claimed[lo >> 5] >> (lo & 31u)) | (a.claimed[hi >> 5] >> (hi & 31u))) & 1u))
        return;
    const unsigned long long gs = atomicAdd(sg.count, 1ull);
    if (gs < sg.cap) sg.pairs[gs] = rec;
}

// verify staged records [from, to) in parallel; rejected ones become ~0.  In greedy mode a
// verified pair with a claimed read end becomes ~1 (counted as found, not stored).
template <int W, int NT = JOIN_THREADS>
__device__ __forceinline__ void verify_staged(const JoinArgs &a, unsigned long long *buf,
                                              uint32_t from, uint32_t to, unsigned long long &nfalse)
{
    uint32_t nfound = 0;
    for (uint32_t t = from + threadIdx.x; t < to; t += NT) {
        const unsigned long long rec = buf[t];
        const uint32_t u = (uint32_t)(rec >> 32), b = (uint32_t)rec;
        LSG_DCHECK(a.V == 0 || (u < a.V && b < a.V));
        if (!verify_pair<W>(a, u, b ^ 1u)) {
            buf[t] = ~0ull;
            ++nfalse;
            continue;
        }
        ++nfound;
        if (a.claimed && (((a.claimed[u >> 5] >> (u & 31u)) | (a.claimed[b >> 5] >> (b & 31u))) & 1u))
            buf[t] = ~1ull;
    }
    if (a.found) {
        for (int o = 16; o; o >>= 1) nfound += __shfl_xor_sync(0xffffffffu, nfound, o);
        if ((threadIdx.x & 31) == 0 && nfound) atomicAdd(a.found, (unsigned long long)nfound);
    }
}

// write the accepted staged records [0, m) to the global pool: one global atomic per block
// reserves the block's range (a per-record or per-warp atomic on the single pool counter
// serialises at L2 — ~86 K warp atomics per length at cfg3).  Called by all threads.
template <int NT = JOIN_THREADS>
__device__ __forceinline__ void flush_staged(const unsigned long long *buf, uint32_t m,
                                             unsigned long long *pairs, unsigned long long cap,
                                             unsigned long long *count)
{
    __shared__ uint32_t fw[NT / 32];
    __shared__ unsigned long long fbase;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    uint32_t c = 0;
    for (uint32_t t = threadIdx.x; t < m; t += NT) c += buf[t] < ~1ull;
    uint32_t x = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) fw[wid] = x;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t tot = 0;
        for (int w = 0; w < NT / 32; ++w) {
            const uint32_t v = fw[w];
            fw[w] = tot;
            tot += v;
        }
        fbase = tot ? atomicAdd(count, (unsigned long long)tot) : 0ull;
    }
    __syncthreads();
    unsigned long long pos = fbase + fw[wid] + x - c;
    for (uint32_t t = threadIdx.x; t < m; t += NT) {
        const unsigned long long rec = buf[t];
        if (rec >= ~1ull) continue; // rejected (~0) or dead (~1)
        if (pos < cap) pairs[pos] = rec;
        ++pos;
    }
}

// hash-join the m staged entries ent[0..m) (whole buckets, both sides mixed); slot tags =
// (epoch << 16) | index
template <int W>
__device__ __forceinline__ void hash_join_window(const JoinArgs &a, const uint64_t *ent, uint32_t m,
                                                 uint32_t *slot, unsigned short *next,
                                                 uint32_t epoch, Stager &em,
                                                 unsigned long long &nfalse)
{
    const uint32_t kshift = a.vbits + FLAG_BITS;
    const uint64_t vmask = (1ull << a.vbits) - 1;
    const uint32_t tag = (epoch & 0xFFFFu) << 16;
    for (uint32_t k = threadIdx.x; k < m; k += JOIN_THREADS) {
        const uint64_t e = ent[k];
        if ((e >> a.vbits) & 1) continue; // flag 1: probe side only
        const uint32_t h = (uint32_t)(e >> kshift) & (JOIN_SLOTS - 1);
        const uint32_t old = atomicExch(&slot[h], tag | k);
        next[k] = (old >> 16) == (tag >> 16) ? (unsigned short)(old & 0xFFFFu) : 0xFFFFu;
    }
    __syncthreads();
    for (uint32_t k = threadIdx.x; k < m; k += JOIN_THREADS) {
        const uint64_t e = ent[k];
        if (key_flag(e, a.vbits) == 0) continue; // flag 0: build side only
        const uint32_t sv = slot[(uint32_t)(e >> kshift) & (JOIN_SLOTS - 1)];
        uint32_t sl = (sv >> 16) == (tag >> 16) ? (sv & 0xFFFFu) : 0xFFFFu;
        while (sl != 0xFFFFu) {
            const uint64_t p = ent[sl];
            if (((p ^ e) >> kshift) == 0) candidate<W>(a, e, p, vmask, em, nfalse);
            sl = next[sl];
        }
    }
}

// a run [lo, hi) of global entries too large for a window (massively repeated fingerprints):
// every probe entry scans the whole run in global memory
template <int W>
__device__ __forceinline__ void oversized_join(const JoinArgs &a, const uint64_t *A, uint64_t lo,
                                               uint64_t hi, Stager &em, unsigned long long &nfalse)
{
    const uint32_t kshift = a.vbits + FLAG_BITS;
    const uint64_t vmask = (1ull << a.vbits) - 1;
    for (uint64_t i = lo + threadIdx.x; i < hi; i += JOIN_THREADS) {
        const uint64_t e = A[i];
        if (key_flag(e, a.vbits) == 0) continue;
        for (uint64_t j = lo; j < hi; ++j) {
            const uint64_t p = A[j];
            if (((p >> a.vbits) & 1) == 0 && ((p ^ e) >> kshift) == 0)
                candidate<W>(a, e, p, vmask, em, nfalse);
        }
    }
}

// after a window (called by all threads after a __syncthreads()): once at least one candidate
// per thread is staged, verify them all in parallel (the long verify path runs with full
// warps) and flush the accepted ones.  Cheaper windows just leave the buffer as it is.
template <int W, int NT = JOIN_THREADS>
__device__ __forceinline__ void window_epilogue(const JoinArgs &a, unsigned long long *buf,
                                                uint32_t *bcount, uint32_t *vdone,
                                                unsigned long long &nfalse)
{
    const uint32_t to = min(*bcount, 2u * NT);
    if (to >= (uint32_t)NT) {
        if (!a.defer_verify) {
            verify_staged<W, NT>(a, buf, 0, to, nfalse);
            __syncthreads();
        }
        flush_staged<NT>(buf, to, a.pairs, a.cap, a.count);
        __syncthreads();
        if (threadIdx.x == 0) *bcount = 0;
        __syncthreads();
    }
    (void)vdone;
}

// end of a join kernel: verify and flush whatever is still staged
template <int W, int NT = JOIN_THREADS>
__device__ __forceinline__ void final_flush(const JoinArgs &a, unsigned long long *buf,
                                            uint32_t *bcount, unsigned long long &nfalse)
{
    __syncthreads();
    const uint32_t to = min(*bcount, 2u * NT);
    if (!a.defer_verify) {
        verify_staged<W, NT>(a, buf, 0, to, nfalse);
        __syncthreads();
    }
    flush_staged<NT>(buf, to, a.pairs, a.cap, a.count);
}

} // namespace lsg
