// lasagna.cu — the C ABI (include/lasagna.h): argument validation, the workspace planner of
// the semi-streaming driver (a8) and the per-length-group orchestration of a2..a7.
#include <algorithm>
#include <atomic>
#include <cmath>
#include <vector>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "kernels.cuh"

namespace lsg {

// ------------------------------------------------------------------ errors, launch counter
static thread_local char g_err[512] = "";
static std::atomic<unsigned long long> g_launches{0};

void count_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }
uint64_t launch_count() { return g_launches.load(std::memory_order_relaxed); }

void set_error(const char *fmt, ...)
{
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof g_err, fmt, ap);
    va_end(ap);
}

lasagna_status cuda_status(cudaError_t e, const char *what)
{
    set_error("%s: %s (%s)", what, cudaGetErrorString(e), cudaGetErrorName(e));
    return LASAGNA_ECUDA;
}

// Test hooks and tuning knobs come from the environment, read on every call (so a test can
// set one in-process, around one call).  Production runs set none of them.
static uint64_t env_u64(const char *name, uint64_t dflt)
{
    const char *e = getenv(name);
    return (e && *e) ? strtoull(e, nullptr, 10) : dflt;
}
static bool env_flag(const char *name, char first)
{
    const char *e = getenv(name);
    return e && e[0] == first;
}

// ------------------------------------------------------------------ planning
// Geometry of the key tables:
//   N = V entries per length (one canonical entry per vertex, common.cuh), V = 2n vertices
//   key = mix(min(H, Hr)) top (62 - vbits) bits | flag << vbits | vertex id,
//   vbits = ceil(log2 V)
//   grouped by the top T bits of mix(min(H, Hr)) so that a T-bit bucket holds
//   ~N / 2^T <= ~2.9K entries (one shared-memory join window):
//   P = ceil((log2 N - 11.5) / 8) levels; T = 8 (P - 1) + dlast, dlast = 8 for P <= 2 and
//   ceil(log2 N - 11.5) - 16 for P = 3 (cfg4/cfg5: 4)
struct Geometry {
    uint64_t n, V, N;
    uint32_t L, l_min, n_len, vbits, T;
    // bucketed path (partition_*.cu): P MSD levels (8, 8, dlast bits), capacities with slack
    uint32_t P, dlast;
    uint64_t cap1, cap2;    // unsplit region capacities of levels 1 and 2 (when not final)
    uint64_t half;          // half-bucket capacity of the final level
    uint64_t n_buckets;     // final-level buckets per length (2^T)
};

// capacity of a region expecting `mean` keys: mean + 8 sigma + 32 (multinomial occupancy;
// a region that still overflows makes the call fall back to the exact LSD path)
static uint64_t region_cap(double mean)
{
    // LASAGNA_TEST_TIGHT_REGIONS=1 (tests only): half-size regions force the overflow fallback
    if (getenv("LASAGNA_TEST_TIGHT_REGIONS")) return ((uint64_t)(mean / 2) + 2) & ~1ull;
    uint64_t c = (uint64_t)std::ceil(mean + 8.0 * std::sqrt(mean) + 32.0);
    return (c + 1) & ~1ull;
}

static uint32_t ceil_log2(uint64_t x)
{
    uint32_t b = 0;
    while ((1ull << b) < x) ++b;
    return b;
}

static Geometry geometry(uint64_t n, uint32_t L, uint32_t l_min)
{
    Geometry g;
    g.n = n;
    g.V = 2 * n;
    g.N = g.V;
    g.L = L;
    g.l_min = l_min;
    g.n_len = L - l_min; // lengths l_min .. L-1 (R5: the l = L partition is dropped)
    g.vbits = std::max<uint32_t>(1, ceil_log2(g.V));
    const double lg = g.N > 1 ? std::log2((double)g.N) : 0.0;
    int P = (int)std::ceil((lg - 11.5) / 8.0);
    P = std::max(1, std::min(P, 3)); // 2n < 2^32: log2 N - 11.5 < 20.5
    // LASAGNA_TEST_LEVELS / LASAGNA_TEST_LAST_BITS (tests only): force the cfg4/cfg5 geometry
    // (three levels, a short last digit) at sizes the oracle checks
    P = (int)std::max<uint64_t>(1, std::min<uint64_t>(3, env_u64("LASAGNA_TEST_LEVELS", P)));
    g.P = (uint32_t)P;
    g.dlast = 8;
    if (P == 3) {
        const int d = (int)std::ceil(lg - 11.5) - 16;
        g.dlast = (uint32_t)std::max(1, std::min(8, d));
        g.dlast = (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(8, env_u64("LASAGNA_TEST_LAST_BITS", g.dlast)));
    }
    g.T = 8u * (g.P - 1) + g.dlast;
    g.n_buckets = 1ull << g.T;
    g.cap1 = region_cap((double)g.N / 256.0);
    g.cap2 = region_cap((double)g.N / 65536.0);
    g.half = region_cap((double)g.N / (double)(2 * g.n_buckets));
    return g;
}

static size_t align256(size_t x) { return (x + 255) & ~(size_t)255; }

struct Layout {
    uint32_t G;          // lengths per group
    uint32_t K;          // hash-range sub-passes per length (1: whole tables)
    uint64_t pool_cap;   // pair pool capacity (pairs)
    size_t tabA, tabB, status, status_bytes, hist, ctrs, pool, pool2, best, claimed, fill1,
        fill2, fill3, total;
    size_t tabB_bytes;   // tabB's size (the level-2 regions; the a1 staging ring before them)
};

constexpr size_t CTR_BYTES = 4096 * 4 + 1024;
// u64 counters after the sort tile counters
enum { CTR_POOL = 0, CTR_FALSE = 1, CTR_POOL2 = 2, CTR_OVERFLOW = 3, CTR_BOOK = 4, CTR_FOUND = 8,
       CTR_POOL3 = 9, CTR_WORK = 10, CTR_PRUNED = 11, CTR_PEER = 16, CTR64_N = CTR_PEER + PC_N };

// The greedy: two launches per length (greedy_rounds.cu); LASAGNA_GREEDY=old (A/B only) runs
// the seven-launch form (greedy.cu)
static bool old_greedy() { return env_flag("LASAGNA_GREEDY", 'o'); }

// a one-rank GreedyPeers over a call's buffers
static GreedyPeers single_peers(const GreedyBufs &gb, unsigned long long *ctr_peer, uint32_t *succ,
                                uint8_t *olen, uint64_t V)
{
    GreedyPeers p;
    p.r[0].pool = gb.pool;
    p.r[0].pool2 = gb.pool2;
    p.r[0].in_count = gb.cnt;
    p.r[0].ctr = ctr_peer;
    p.r[0].best = gb.best;
    p.r[0].claimed = gb.claimed;
    p.r[0].succ = succ;
    p.r[0].olen = olen;
    p.r[0].tail = nullptr;
    p.g = 1;
    p.slice = V;
    p.cap = gb.cap;
    return p;
}

// K > 1 (hash-range sub-passes, one length per pass): the tables hold only the level-1 digits
// of one of K ranges at a time (nb = ceil(256 / K) digits, shard_region's layout with dest_g =
// K), and there is no exact-path fallback (it needs whole tables)
static Layout layout(const Geometry &g, uint32_t G, uint64_t pool_cap, bool greedy, uint32_t K = 1)
{
    Layout l;
    l.G = G;
    l.pool_cap = pool_cap;
    l.K = K;
    size_t off = 0;
    auto take = [&](size_t bytes) {
        size_t o = off;
        off += align256(bytes);
        return o;
    };
    // tabA/tabB: the exact path's LSD ping-pong buffers, or the bucketed path's levels with
    // slack: level 1 in tabA, level 2 in tabB, level 3 (P = 3) in tabA again
    const uint64_t nb = (256 + K - 1) / K; // level-1 digits per pass
    const size_t exact_b = K > 1 ? 0 : (size_t)G * g.N * 8;
    const size_t lvl1_b = (size_t)G * (g.P == 1 ? 512 * g.half : nb * g.cap1) * 8;
    const size_t lvl2_b = g.P == 2   ? (size_t)G * nb * 512 * g.half * 8
                          : g.P == 3 ? (size_t)G * nb * 256 * g.cap2 * 8
                                     : 0;
    const size_t lvl3_b = g.P == 3 ? (size_t)G * 2 * (g.n_buckets / 256 * nb) * g.half * 8 : 0;
    l.tabA = take(std::max({exact_b, lvl1_b, lvl3_b}));
    l.tabB_bytes = std::max(exact_b, lvl2_b);
    l.tabB = take(l.tabB_bytes);
    l.fill1 = take((size_t)G * 512 * 4);
    l.fill2 = take(g.P == 2 ? (size_t)G * nb * 512 * 4 : g.P == 3 ? (size_t)G * nb * 256 * 4 : 4);
    l.fill3 = take(g.P == 3 ? (size_t)G * 2 * (g.n_buckets / 256 * nb) * 4 : 4);
    l.status_bytes = std::max(K > 1 ? (size_t)0 : sort_status_bytes(g.N, G),
                              sort_status_bytes(pool_cap, 1));
    l.status = take(l.status_bytes);
    l.hist = take((size_t)8 * std::max<uint32_t>(G, 1) * 256 * 4);
    l.ctrs = take(CTR_BYTES);
    l.pool = take(pool_cap * 8);
    l.pool2 = take(pool_cap * 8);
    if (greedy) {
        l.best = take(g.V * 8);
        l.claimed = take(ceil_div(g.V, 32) * 4);
    } else {
        l.best = l.claimed = 0; // overlaps: pairs sorted in pool/pool2
    }
    l.total = off;
    return l;
}

// The bucketed path (partition_*.cu) serves every geometry (P <= 3); LASAGNA_PATH=exact forces
// the exact LSD-sort path (also the fallback when a slack region overflows).
static bool use_bucketed(const Geometry &g)
{
    return !env_flag("LASAGNA_PATH", 'e') && g.P >= 1 && g.P <= 3;
}

static uint64_t default_pool_cap(const Geometry &g)
{
    return std::max<uint64_t>(g.V / 8, 1ull << 20);
}

// ------------------------------------------------------------------ validation
static bool is_device_ptr(const void *p)
{
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

static lasagna_status check_shape(uint64_t n, uint32_t L, uint32_t l_min)
{
    if (L < 2 || L > 256) {
        set_error("L=%u out of range [2, 256]", L);
        return LASAGNA_EINVAL;
    }
    if (l_min < 1 || l_min >= L) {
        set_error("l_min=%u out of range [1, L-1]", l_min);
        return LASAGNA_EINVAL;
    }
    if (n > 0x7FFFFFFFull) {
        set_error("2n=%llu exceeds 0xFFFFFFFE vertex ids", (unsigned long long)(2 * n));
        return LASAGNA_ERANGE;
    }
    return LASAGNA_OK;
}

static bool aligned(const void *p, size_t a) { return ((uintptr_t)p % a) == 0; }

// ------------------------------------------------------------------ the group pipeline
struct Run {
    Geometry g;
    Layout lay;
    char *ws;
    cudaStream_t s;
    SortCtx sctx;
    uint64_t *tab[2];
    uint32_t *hist;
    bool bucketed;              // partition_*.cu path (else exact LSD sort + contiguous join)
    const unsigned char *ascii = nullptr; // a1 still to do: the first group's scatter packs it
    const char *ascii_host = nullptr;     // ... from this page-locked host copy (chunked DMA)
    uint64_t *packed_out = nullptr;
    unsigned long long *first_bad = nullptr;
    uint32_t *fill1, *fill2, *fill3;
    unsigned long long *ctr64; // CTR_* counters
    unsigned long long *pool, *pool2;
    const uint32_t *claimed = nullptr; // greedy mode: the join drops pairs with a claimed end
    bool prune = false; // this group's scatter drops entries whose read end is claimed (f1)
    bool approx = false; // f4: hits accepted by the 128-bit fingerprint pair
    bool defer_verify = false; // greedy mode: the greedy's first round verifies the join's hits
    template <typename T> T *at(size_t off) { return reinterpret_cast<T *>(ws + off); }
    void bind(void *workspace)
    {
        ws = (char *)workspace;
        tab[0] = at<uint64_t>(lay.tabA);
        tab[1] = at<uint64_t>(lay.tabB);
        hist = at<uint32_t>(lay.hist);
        fill1 = at<uint32_t>(lay.fill1);
        fill2 = at<uint32_t>(lay.fill2);
        fill3 = at<uint32_t>(lay.fill3);
        sctx.status = at<unsigned long long>(lay.status);
        sctx.status_bytes = lay.status_bytes;
        sctx.tile_ctrs = at<uint32_t>(lay.ctrs);
        sctx.epoch = 0;
        ctr64 = reinterpret_cast<unsigned long long *>(ws + lay.ctrs + 4096 * 4);
        pool = at<unsigned long long>(lay.pool);
        pool2 = at<unsigned long long>(lay.pool2);
    }
};

// Phase timing without extra synchronisation: event pairs are recorded on the stream as the
// call proceeds and read once at the end of the call (which synchronises anyway for stats).
enum Phase { PH_TABLE, PH_SORT, PH_SEARCH, PH_GREEDY, PH_N };
struct PhaseTimer {
    bool on = false;
    cudaStream_t s = nullptr;
    struct Rec {
        int ph;
        cudaEvent_t a, b;
    };
    std::vector<Rec> recs;
    int open = -1;
    ~PhaseTimer()
    {
        for (auto &r : recs) cudaEventDestroy(r.a), cudaEventDestroy(r.b);
    }
    lasagna_status start(int ph)
    {
        if (!on) return LASAGNA_OK;
        Rec r;
        r.ph = ph;
        LSG_CUDA(cudaEventCreate(&r.a));
        LSG_CUDA(cudaEventCreate(&r.b));
        recs.push_back(r);
        LSG_CUDA(cudaEventRecord(r.a, s));
        return LASAGNA_OK;
    }
    lasagna_status stop()
    {
        if (!on) return LASAGNA_OK;
        LSG_CUDA(cudaEventRecord(recs.back().b, s));
        return LASAGNA_OK;
    }
    lasagna_status finish(lasagna_stats *st)
    {
        if (!on) return LASAGNA_OK;
        LSG_CUDA(cudaStreamSynchronize(s));
        float *acc[PH_N] = {&st->ms_table, &st->ms_sort, &st->ms_search, &st->ms_greedy};
        for (auto &r : recs) {
            float ms = 0;
            LSG_CUDA(cudaEventElapsedTime(&ms, r.a, r.b));
            *acc[r.ph] += ms;
        }
        return LASAGNA_OK;
    }
};

// a8 level 2: the host -> device leg of the semi-streaming driver.  The ASCII
// reads (page-locked host memory) are copied by the DMA engine in chunks into a ring of device
// buffers on a copy stream, and each chunk's fused a1 + a2 + level-1 partition launch runs on
// the call's stream as soon as its copy has landed, while the next chunks are in flight
// (events order copy k before scatter k, and scatter k before a copy that reuses its slot).  The ring lives in the level-2 region buffer, which nothing touches before the refine
// pass that follows.  Chunks are whole scatter CTAs (multiples of 512 reads); per-(CTA, bin)
// reservations accumulate across the launches exactly as within one.
static lasagna_status scatter_from_host(Run &r, const ScatterArgs &base, const char *host)
{
    const uint64_t n = base.n, L = base.L;
    // 512 Ki reads per chunk (~53 MB at L = 101); LASAGNA_TEST_A1_CHUNK (tests only) overrides
    const uint64_t want = env_u64("LASAGNA_TEST_A1_CHUNK", 0) ? env_u64("LASAGNA_TEST_A1_CHUNK", 0)
                                                               : (uint64_t)512 * 1024;
    const uint64_t chunk = std::max<uint64_t>(512, want / 512 * 512);
    const size_t slot_bytes = (size_t)chunk * L;
    const uint64_t nchunk = ceil_div(n, chunk);
    // as many ring slots as the region buffer holds, up to one per chunk (then the copy engine
    // never waits for a table pass, e.g. while another call's kernels hold the SMs), at most 64
    // LASAGNA_TEST_A1_SLOTS (tests only) lowers it
    const uint64_t ts = env_u64("LASAGNA_TEST_A1_SLOTS", 0);
    const uint64_t max_slots = ts >= 3 && ts < 64 ? ts : 64;
    const uint64_t nslot = std::min<uint64_t>({nchunk, max_slots, r.lay.tabB_bytes / slot_bytes});
    if (nslot < std::min<uint64_t>(nchunk, 3)) return launch_scatter_table(base, r.s); // zero-copy
    unsigned char *ring = reinterpret_cast<unsigned char *>(r.tab[1]);
    struct Res {
        cudaStream_t cs = nullptr;
        std::vector<cudaEvent_t> ev;
        ~Res()
        {
            for (auto e : ev)
                if (e) cudaEventDestroy(e);
            if (cs) cudaStreamDestroy(cs);
        }
    } res;
    LSG_CUDA(cudaStreamCreateWithFlags(&res.cs, cudaStreamNonBlocking));
    // copied: two alternating events (a wait snapshots the event's latest record); consumed:
    // one per ring slot, recorded after the table pass that read it
    const uint64_t nreuse = nchunk > nslot ? nslot : 0;
    res.ev.assign(3 + nreuse, nullptr);
    for (auto &e : res.ev) LSG_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    cudaEvent_t start = res.ev[0], *copied = &res.ev[1], *consumed = res.ev.data() + 3;
    LSG_CUDA(cudaEventRecord(start, r.s)); // the ring's previous users (an earlier call) are done
    LSG_CUDA(cudaStreamWaitEvent(res.cs, start, 0));
    for (uint64_t k = 0; k < nchunk; ++k) {
        const uint64_t slot = k % nslot, r0 = k * chunk, m = std::min(chunk, n - r0);
        if (k >= nslot) LSG_CUDA(cudaStreamWaitEvent(res.cs, consumed[slot], 0));
        LSG_CUDA(cudaMemcpyAsync(ring + slot * slot_bytes, host + r0 * L, m * L,
                                 cudaMemcpyHostToDevice, res.cs));
        LSG_CUDA(cudaEventRecord(copied[k & 1], res.cs));
        LSG_CUDA(cudaStreamWaitEvent(r.s, copied[k & 1], 0));
        ScatterArgs sa = base;
        sa.ascii = ring + slot * slot_bytes;
        sa.n = m;
        sa.read_offset = base.read_offset + r0;
        sa.packed_out = base.packed_out + r0 * base.stride;
        lasagna_status rc = launch_scatter_table(sa, r.s);
        if (rc != LASAGNA_OK) return rc;
        if (nreuse) LSG_CUDA(cudaEventRecord(consumed[slot], r.s));
    }
    return LASAGNA_OK;
}

// Stored fingerprint bits of a bucketed key: bits [vbits + 2, 64) (the top 8 bits of the mixed
// fingerprint are implied by the level-1 region).  LASAGNA_TEST_FP_BITS=b (tests only) keeps
// just the top b of them, to measure the collision rate at a chosen key width (R12).
static uint64_t stored_keep(const Geometry &g)
{
    uint64_t keep = ~((1ull << (g.vbits + FLAG_BITS)) - 1);
    const uint64_t b = env_u64("LASAGNA_TEST_FP_BITS", 64);
    if (b < 64 - g.vbits - FLAG_BITS) keep &= b ? ~0ull << (64 - b) : 0ull;
    return keep;
}

// Build + partition the key tables of lengths [l_lo, l_hi] (level 1 fused with a2, then the
// refine levels; the final buckets end in tabB for P = 2, tabA for P = 1 and P = 3).
static lasagna_status build_group_bucketed(Run &r, const uint64_t *packed, uint32_t l_lo,
                                           uint32_t l_hi, PhaseTimer &tm, lasagna_stats *st,
                                           uint32_t sub = 0)
{
    const Geometry &g = r.g;
    const uint32_t G = l_hi - l_lo + 1;
    const uint32_t K = r.lay.K, nb = (256 + K - 1) / K; // sub-pass `sub` of K: digit range
    unsigned int *ovf = reinterpret_cast<unsigned int *>(r.ctr64 + CTR_OVERFLOW);
    LSG_CUDA(cudaMemsetAsync(r.fill1, 0, (size_t)G * 512 * 4, r.s));
    ScatterArgs sa;
    sa.packed = packed;
    sa.n = g.n;
    sa.read_offset = 0;
    sa.L = g.L;
    sa.stride = stride_for(g.L);
    sa.l_lo = l_lo;
    sa.l_hi = l_hi;
    sa.vbits = g.vbits;
    sa.keep = stored_keep(g);
    sa.out = r.tab[0];
    sa.fill = r.fill1;
    sa.split = g.P == 1; // one level: the level-1 regions are the (split) buckets
    sa.cap = sa.split ? g.half : g.cap1;
    sa.overflow = ovf;
    sa.ascii = r.ascii; // fused a1 (first group only)
    sa.claimed = r.prune ? r.claimed : nullptr;
    sa.pruned = sub == 0 ? r.ctr64 + CTR_PRUNED : nullptr; // counted once per length
    sa.packed_out = r.packed_out;
    sa.first_bad = r.first_bad;
    sa.dest_g = K;
    sa.nb_pad = nb;
    sa.keep_owner = K > 1 ? (int32_t)sub : -1;
    const char *host = r.ascii_host;
    r.ascii = nullptr;
    r.ascii_host = nullptr;
    lasagna_status rc;
    if ((rc = tm.start(PH_TABLE)) != LASAGNA_OK) return rc;
    if (sa.ascii && host && g.P >= 2) {
        if ((rc = scatter_from_host(r, sa, host)) != LASAGNA_OK) return rc;
    } else if ((rc = launch_scatter_table(sa, r.s)) != LASAGNA_OK) {
        return rc;
    }
    if ((rc = tm.stop()) != LASAGNA_OK) return rc;
    if (g.P >= 2) {
        // level 2: the next 8 bits (the stored key's top byte)
        RefineArgs ra;
        ra.in = r.tab[0];
        ra.fill_in = r.fill1;
        ra.cap_in = g.cap1;
        ra.dshift = 56;
        ra.dbits = 8;
        ra.out = r.tab[1];
        ra.fill_out = r.fill2;
        ra.cap_out = g.P == 2 ? g.half : g.cap2;
        ra.vbits = g.vbits;
        ra.split = g.P == 2;
        ra.overflow = ovf;
        if ((rc = tm.start(PH_SORT)) != LASAGNA_OK) return rc;
        if ((rc = launch_refine(ra, (uint64_t)G * nb, r.s)) != LASAGNA_OK) return rc;
        if (g.P == 3) {
            // level 3: dlast more bits, split into build and probe halves
            ra.in = r.tab[1];
            ra.fill_in = r.fill2;
            ra.cap_in = g.cap2;
            ra.dshift = 56 - g.dlast;
            ra.dbits = g.dlast;
            ra.out = r.tab[0];
            ra.fill_out = r.fill3;
            ra.cap_out = g.half;
            ra.split = true;
            if ((rc = launch_refine(ra, (uint64_t)G * nb * 256, r.s)) != LASAGNA_OK) return rc;
        }
        if ((rc = tm.stop()) != LASAGNA_OK) return rc;
        if (st) st->sort_launches += g.P - 1;
    }
    return LASAGNA_OK;
}

static lasagna_status build_group(Run &r, const uint64_t *packed, uint32_t l_lo, uint32_t l_hi,
                                  int *which, PhaseTimer &tm, lasagna_stats *st)
{
    if (r.bucketed) {
        *which = 0;
        return build_group_bucketed(r, packed, l_lo, l_hi, tm, st);
    }
    const Geometry &g = r.g;
    const uint32_t G = l_hi - l_lo + 1;
    uint32_t P, shifts[8], bits[8];
    digit_plan(64 - g.T, 64, &P, shifts, bits);
    LSG_CUDA(cudaMemsetAsync(r.hist, 0, (size_t)G * 256 * 4, r.s));
    TableArgs ta;
    ta.packed = packed;
    ta.n = g.n;
    ta.read_offset = 0;
    ta.L = g.L;
    ta.stride = stride_for(g.L);
    ta.l_lo = l_lo;
    ta.l_hi = l_hi;
    ta.vbits = g.vbits;
    ta.d_shift = shifts[0];
    ta.d_bits = bits[0];
    ta.tab = r.tab[0];
    ta.hist = r.hist;
    lasagna_status rc;
    if ((rc = tm.start(PH_TABLE)) != LASAGNA_OK) return rc;
    if ((rc = launch_table(ta, r.s)) != LASAGNA_OK) return rc;
    if ((rc = tm.stop()) != LASAGNA_OK) return rc;
    if ((rc = tm.start(PH_SORT)) != LASAGNA_OK) return rc;
    if ((rc = sort_segments(r.tab, g.N, G, 64 - g.T, 64, r.hist, true, r.sctx, r.s, which)) !=
        LASAGNA_OK)
        return rc;
    if ((rc = tm.stop()) != LASAGNA_OK) return rc;
    if (st) st->sort_launches += P;
    return LASAGNA_OK;
}

// LASAGNA_JOIN_FILTER=1: the join drops pairs with an end claimed by a longer length (counted,
// not stored).  Off by default: measured at cfg3 the claimed-bit reads cost the join more
// (+2.5 ms) than the smaller pool saves the greedy (-1.2 ms); the greedy drops them instead.
static bool join_filter() { return env_flag("LASAGNA_JOIN_FILTER", '1'); }

// Join (search + verify) of length l into the pool; if m_out, synchronise and report the
// pair count.
static lasagna_status search_length(Run &r, const uint64_t *packed, uint32_t l, uint32_t l_lo,
                                    int which, uint64_t *m_out, bool reset_pool = true)
{
    const Geometry &g = r.g;
    const uint32_t s = l - l_lo;
    // buckets per length: all of them, or those of one hash-range sub-pass
    const uint64_t nbk = r.lay.K > 1 ? g.n_buckets / 256 * ((256 + r.lay.K - 1) / r.lay.K) : g.n_buckets;
    if (reset_pool)
        LSG_CUDA(cudaMemsetAsync(r.ctr64 + CTR_POOL, 0, sizeof(unsigned long long), r.s));
    JoinArgs ja;
    ja.packed = packed;
    ja.keys = r.tab[which] + (uint64_t)s * g.N;
    ja.N = g.N;
    ja.V = g.V;
    ja.L = g.L;
    ja.stride = stride_for(g.L);
    ja.l = l;
    ja.vbits = g.vbits;
    ja.T = g.T;
    ja.pairs = r.pool;
    ja.cap = r.lay.pool_cap;
    ja.count = r.ctr64 + CTR_POOL;
    ja.false_matches = r.ctr64 + CTR_FALSE;
    ja.claimed = join_filter() ? r.claimed : nullptr;
    ja.found = ja.claimed ? r.ctr64 + CTR_FOUND : nullptr;
    ja.approx = r.approx;
    ja.defer_verify = r.defer_verify;
    lasagna_status rc;
    if (r.bucketed) {
        BucketJoinArgs bj;
        bj.j = ja;
        bj.overflow = reinterpret_cast<unsigned int *>(r.ctr64 + CTR_OVERFLOW);
        // final level: [G][n_buckets][2][half] (tabB for P = 2, tabA for P = 1 and 3)
        bj.buckets = (g.P == 2 ? r.tab[1] : r.tab[0]) + (uint64_t)s * 2 * nbk * g.half;
        bj.fills = (g.P == 1 ? r.fill1 : g.P == 2 ? r.fill2 : r.fill3) + (uint64_t)s * 2 * nbk;
        bj.half_cap = g.half;
        bj.n_buckets = nbk;
        // block windows (partition_*.cu); LASAGNA_JOIN=warp (A/B only): one warp per bucket
        // (warpjoin.cu) when a half fits a warp's slice — measured slower at cfg3 (31.9 vs
        // 17.1 ms per step)
        rc = (env_flag("LASAGNA_JOIN", 'w') && warp_join_fits(bj)) ? launch_warp_join(bj, r.s)
                                                                   : launch_bucket_join(bj, r.s);
    } else {
        rc = launch_join(ja, r.s);
    }
    if (rc != LASAGNA_OK) return rc;
    if (m_out) {
        unsigned long long m = 0;
        LSG_CUDA(cudaMemcpyAsync(&m, r.ctr64 + CTR_POOL, sizeof(m), cudaMemcpyDeviceToHost, r.s));
        LSG_CUDA(cudaStreamSynchronize(r.s));
        *m_out = m;
    }
    return LASAGNA_OK;
}

// hash-range sub-passes needed when no whole length fits (G == 0): the smallest power of two
// K whose one-length layout fits `bytes` (bucketed path, two or three levels); 1 otherwise
static bool use_bucketed(const Geometry &g);
static Layout layout(const Geometry &g, uint32_t G, uint64_t pool_cap, bool greedy, uint32_t K);
static uint32_t subpasses_for(const Geometry &g, size_t bytes, uint64_t cap, uint32_t G)
{
    if (G > 0 || !use_bucketed(g) || g.P < 2) return 1;
    for (uint32_t K = 2; K <= 256; K *= 2)
        if (layout(g, 1, cap, true, K).total <= bytes) return K;
    return 1;
}

static uint32_t choose_G(const Geometry &g, uint32_t want, size_t bytes, uint64_t cap, bool greedy)
{
    uint32_t hi = want ? std::min(want, g.n_len) : g.n_len;
    hi = std::min<uint32_t>(hi, 64);
    for (uint32_t G = hi; G >= 1; --G)
        if (layout(g, G, cap, greedy).total <= bytes) return G;
    return 0;
}

} // namespace lsg

using namespace lsg;

// ==================================================================== exported
extern "C" {

const char *lasagna_last_error(void) { return g_err; }

uint64_t lasagna_kernel_launches(void) { return launch_count(); }

uint32_t lasagna_words_per_read(uint32_t L) { return stride_for(L); }

// Device address of an ASCII read buffer: device memory, or page-locked host memory mapped
// into the device address space (read in place over PCIe).  Pageable memory is rejected.
static lasagna_status resolve_ascii(const char *ascii, const char **dev, bool *is_host = nullptr)
{
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, ascii) != cudaSuccess) {
        cudaGetLastError();
        set_error("ascii: not a CUDA-visible pointer");
        return LASAGNA_EINVAL;
    }
    *dev = ascii;
    if (is_host) *is_host = at.type == cudaMemoryTypeHost;
    if (at.type == cudaMemoryTypeHost) {
        void *mapped = nullptr;
        if (!at.devicePointer && cudaHostGetDevicePointer(&mapped, (void *)ascii, 0) == cudaSuccess)
            at.devicePointer = mapped;
        cudaGetLastError();
        if (!at.devicePointer) {
            set_error("ascii: page-locked host memory is not mapped into the device");
            return LASAGNA_EINVAL;
        }
        *dev = (const char *)at.devicePointer;
    } else if (at.type != cudaMemoryTypeDevice && at.type != cudaMemoryTypeManaged) {
        set_error("ascii: pageable host memory; pass device or page-locked host memory");
        return LASAGNA_EINVAL;
    }
    return LASAGNA_OK;
}

lasagna_status lasagna_load_reads(const char *ascii, uint64_t n, uint32_t L, uint64_t *packed,
                                  uint64_t *first_bad, void *stream)
{
    g_err[0] = 0;
    if (L < 1 || L > 256) {
        set_error("L=%u out of range", L);
        return LASAGNA_EINVAL;
    }
    if (n > 0x7FFFFFFFull) {
        set_error("n too large");
        return LASAGNA_ERANGE;
    }
    if (n == 0) {
        if (first_bad) {
            cudaStream_t s = (cudaStream_t)stream;
            unsigned long long v = ~0ull;
            LSG_CUDA(cudaMemcpyAsync(first_bad, &v, 8, cudaMemcpyHostToDevice, s));
            LSG_CUDA(cudaStreamSynchronize(s));
        }
        return LASAGNA_OK;
    }
    if (!ascii || !packed || !aligned(packed, 16) || (first_bad && !aligned(first_bad, 8))) {
        set_error("NULL or misaligned pointer");
        return LASAGNA_EINVAL;
    }
    const char *src = nullptr;
    lasagna_status rs = resolve_ascii(ascii, &src);
    if (rs != LASAGNA_OK) return rs;
    if (!is_device_ptr(packed)) {
        set_error("packed must be device memory");
        return LASAGNA_EINVAL;
    }
    return launch_pack(src, n, L, packed, first_bad, (cudaStream_t)stream);
}

lasagna_status lasagna_fingerprints(const uint64_t *packed, uint64_t n, uint32_t L,
                                    uint32_t l_min, uint64_t *pfx, uint64_t *sfx, void *stream)
{
    g_err[0] = 0;
    lasagna_status rc = check_shape(n, L, l_min);
    if (rc != LASAGNA_OK) return rc;
    if (n == 0) return LASAGNA_OK;
    if (!packed || !aligned(packed, 16) || (pfx && !aligned(pfx, 16)) || (sfx && !aligned(sfx, 16))) {
        set_error("NULL or misaligned pointer (16-byte alignment required)");
        return LASAGNA_EINVAL;
    }
    return launch_fp_values(packed, n, L, l_min, pfx, sfx, (cudaStream_t)stream);
}

lasagna_status lasagna_plan(uint64_t n, uint32_t L, uint32_t l_min, size_t budget_bytes,
                            uint32_t *lengths_per_pass, size_t *workspace_bytes)
{
    g_err[0] = 0;
    lasagna_status rc = check_shape(n, L, l_min);
    if (rc != LASAGNA_OK) return rc;
    if (!lengths_per_pass || !workspace_bytes) {
        set_error("NULL output");
        return LASAGNA_EINVAL;
    }
    Geometry g = geometry(n, L, l_min);
    uint64_t cap = default_pool_cap(g);
    uint32_t G = choose_G(g, 0, budget_bytes, cap, true);
    const uint32_t K = subpasses_for(g, budget_bytes, cap, G);
    if (K > 1) G = 1;
    if (G == 0) {
        *lengths_per_pass = 0;
        *workspace_bytes = layout(g, 1, cap, true, use_bucketed(g) && g.P >= 2 ? 256 : 1).total;
        set_error("budget %zu below the smallest workspace %zu", budget_bytes, *workspace_bytes);
        return LASAGNA_ENOSPC;
    }
    *lengths_per_pass = G;
    *workspace_bytes = layout(g, G, cap, true, K).total;
    return LASAGNA_OK;
}

// a1-a7.  Either `packed` (already staged) or `ascii_dev` (device address of the ASCII reads:
// a1 is fused into the first group's table build, the packed rows land in packed_out, bad
// reads in *first_bad).
static lasagna_status greedy_graph_impl(const uint64_t *packed, const char *ascii_dev,
                                        const char *ascii_host,
                                        uint64_t *packed_out, uint64_t *first_bad, uint64_t n,
                                        uint32_t L, uint32_t l_min, uint32_t lengths_per_pass,
                                        void *workspace, size_t *workspace_bytes, uint32_t *succ,
                                        uint8_t *olen, lasagna_stats *stats, void *stream)
{
    lasagna_status rc = check_shape(n, L, l_min);
    if (rc != LASAGNA_OK) return rc;
    if (!workspace_bytes) {
        set_error("workspace_bytes is NULL");
        return LASAGNA_EINVAL;
    }
    Geometry g = geometry(n, L, l_min);
    // pool capacity: the default, or more when the caller grew the workspace after ENOSPC
    uint64_t cap = default_pool_cap(g);
    const uint32_t G_want = lengths_per_pass ? std::min(lengths_per_pass, g.n_len) : g.n_len;
    const uint32_t G_req = std::min<uint32_t>(G_want, 64);
    if (!workspace) {
        *workspace_bytes = layout(g, G_req, cap, true).total;
        return LASAGNA_OK;
    }
    if (n == 0) {
        if (stats) memset(stats, 0, sizeof *stats);
        return LASAGNA_OK;
    }
    if (ascii_dev) packed = packed_out;
    if (!packed || !succ || !olen || !aligned(packed, 16) || !aligned(succ, 4) ||
        !aligned(workspace, 256) || (ascii_dev && (!first_bad || !aligned(first_bad, 8)))) {
        set_error("NULL or misaligned pointer");
        return LASAGNA_EINVAL;
    }
    uint32_t G = choose_G(g, G_req, *workspace_bytes, cap, true);
    // f4: when even one length's tables exceed the workspace, each length is
    // built and joined in K hash-range sub-passes (level-1 digit ranges) — the B200 form of the
    // paper's external merge (Alg. 1): a range's tables are complete in HBM, so
    // nothing is merged; the fingerprints are recomputed per sub-pass instead of spilled
    uint32_t K = subpasses_for(g, *workspace_bytes, cap, G);
    if (K > 1) G = 1;
    if (G == 0) {
        *workspace_bytes = layout(g, 1, cap, true, use_bucketed(g) && g.P >= 2 ? 256 : 1).total;
        set_error("workspace too small");
        return LASAGNA_ENOSPC;
    }
    // spare bytes beyond the chosen layout enlarge the pair pool
    {
        size_t spare = *workspace_bytes - layout(g, G, cap, true, K).total;
        cap += spare / 16; // pool + pool2: 16 B per pair (the status words shrink it below)
        while (cap > default_pool_cap(g) && layout(g, G, cap, true, K).total > *workspace_bytes) cap -= cap / 256 + 1;
    }
    cudaStream_t s = (cudaStream_t)stream;
    Run r;
    r.g = g;
    r.lay = layout(g, G, cap, true, K);
    r.s = s;
    r.bind(workspace);
    uint32_t *claimed = r.at<uint32_t>(r.lay.claimed);
    r.claimed = claimed;
    if (ascii_dev) {
        // a1: fused into the first partition pass when the fast path runs (T >= 16, L <= 160),
        // otherwise a separate pack launch
        LSG_CUDA(cudaMemsetAsync(first_bad, 0xFF, 8, s));
        if (use_bucketed(g) && g.P >= 2 && L <= 160) {
            r.ascii = reinterpret_cast<const unsigned char *>(ascii_dev);
            r.ascii_host = ascii_host;
            r.packed_out = packed_out;
            r.first_bad = reinterpret_cast<unsigned long long *>(first_bad);
        } else {
            if ((rc = launch_pack(ascii_dev, n, L, packed_out, first_bad, s)) != LASAGNA_OK)
                return rc;
        }
    }
    GreedyBufs gb;
    gb.pool = r.pool;
    gb.pool2 = r.pool2;
    gb.cnt = r.ctr64 + CTR_POOL;
    gb.cnt2 = r.ctr64 + CTR_POOL2;
    gb.cnt3 = r.ctr64 + CTR_POOL3;
    gb.book = r.ctr64 + CTR_BOOK;
    gb.work = r.ctr64 + CTR_WORK;
    gb.best = r.at<unsigned long long>(r.lay.best);
    gb.claimed = claimed;
    gb.cap = cap;
    gb.epoch = 1;
    GreedyPeers peers = single_peers(gb, r.ctr64 + CTR_PEER, succ, olen, g.V);
    // LASAGNA_VERIFY=greedy (R27): the join stores its fingerprint hits unverified and the
    // greedy's first round checks them on the bases.  Measured the same at cfg3 (join 12.13 +
    // greedy 11.70 vs 17.34 + 6.37 ms: the ~5 ms of random base reads cost the same in either
    // kernel), so the default verifies inside the join, like the overlaps and multi-GPU paths.
    // (The round-1 greedy and the join-side claimed filter need verified pairs.)
    r.defer_verify = !old_greedy() && !join_filter() && env_flag("LASAGNA_VERIFY", 'g');
    if (r.defer_verify) {
        peers.vpacked = packed;
        peers.vL = L;
        peers.vstride = stride_for(L);
        peers.vfalse = r.ctr64 + CTR_FALSE;
    }

  for (int attempt = 0; attempt < 2; ++attempt) {
    r.bucketed = attempt == 0 && use_bucketed(g);
    if (r.lay.K > 1 && !r.bucketed) {
        set_error("hash-range sub-passes need the bucketed path");
        return LASAGNA_EINVAL;
    }
    gb.epoch = 1;
    lasagna_stats st;
    memset(&st, 0, sizeof st);
    st.lengths_per_pass = G;
    st.key_sort_bits = g.T;
    st.bucketed = r.bucketed ? 1u : 0u;
    PhaseTimer tm;
    tm.on = stats != nullptr;
    tm.s = s;
    const uint64_t launches0 = launch_count();

    if ((rc = sort_ctx_reset(r.sctx, s)) != LASAGNA_OK) return rc;
    LSG_CUDA(cudaMemsetAsync(r.ctr64, 0, CTR64_N * sizeof(unsigned long long), s));
    LSG_CUDA(cudaMemsetAsync(succ, 0xFF, g.V * 4, s));
    LSG_CUDA(cudaMemsetAsync(olen, 0, g.V, s));
    LSG_CUDA(cudaMemsetAsync(claimed, 0, ceil_div(g.V, 32) * 4, s));
    LSG_CUDA(cudaMemsetAsync(gb.best, 0, g.V * 8, s));

    // Everything below is stream-ordered with no host round trip: the join of length l and
    // its greedy claim read/write counts in device memory (one synchronisation at the end).
    for (int64_t l_hi = (int64_t)L - 1; l_hi >= (int64_t)l_min; l_hi -= G) {
        const uint32_t l_lo = (uint32_t)std::max<int64_t>(l_min, l_hi - (int64_t)G + 1);
        int which = 0;
        // f1: every group after the first is built after the greedy of all
        // longer lengths, so its scatter drops the entries of claimed read ends (P:L152,
        // a claimed end can never gain an edge).  LASAGNA_NO_PRUNE=1 keeps them (then
        // n_pairs is the full |P|).
        r.prune = l_hi != (int64_t)L - 1 && !env_flag("LASAGNA_NO_PRUNE", '1');
        if (r.lay.K > 1) {
            // one length in K hash-range sub-passes: each builds the tables of one digit range
            // and joins them into the length's pool; the greedy runs once all are in
            const uint32_t l = (uint32_t)l_hi;
            for (uint32_t sub = 0; sub < r.lay.K; ++sub) {
                if ((rc = build_group_bucketed(r, packed, l, l, tm, &st, sub)) != LASAGNA_OK)
                    return rc;
                ++st.passes;
                if ((rc = tm.start(PH_SEARCH)) != LASAGNA_OK) return rc;
                if ((rc = search_length(r, packed, l, l, 0, nullptr, sub == 0)) != LASAGNA_OK)
                    return rc;
                if ((rc = tm.stop()) != LASAGNA_OK) return rc;
                ++st.search_launches;
            }
            if ((rc = tm.start(PH_GREEDY)) != LASAGNA_OK) return rc;
            if ((rc = old_greedy() ? greedy_length(gb, (uint8_t)l, succ, olen, s)
                                   : greedy_length_peers(peers, (uint8_t)l, s)) != LASAGNA_OK)
                return rc;
            if ((rc = tm.stop()) != LASAGNA_OK) return rc;
            continue;
        }
        if ((rc = build_group(r, packed, l_lo, (uint32_t)l_hi, &which, tm, &st)) != LASAGNA_OK)
            return rc;
        ++st.passes;
        for (int64_t l = l_hi; l >= (int64_t)l_lo; --l) {
            if ((rc = tm.start(PH_SEARCH)) != LASAGNA_OK) return rc;
            // every length's full pair list is found and counted (|P| = overlap edges / 2);
            // pairs with an end claimed by a longer length are not stored for the greedy
            if ((rc = search_length(r, packed, (uint32_t)l, l_lo, which, nullptr)) != LASAGNA_OK)
                return rc;
            if ((rc = tm.stop()) != LASAGNA_OK) return rc;
            ++st.search_launches;
            if ((rc = tm.start(PH_GREEDY)) != LASAGNA_OK) return rc;
            if ((rc = old_greedy() ? greedy_length(gb, (uint8_t)l, succ, olen, s)
                                   : greedy_length_peers(peers, (uint8_t)l, s)) != LASAGNA_OK)
                return rc;
            if ((rc = tm.stop()) != LASAGNA_OK) return rc;
        }
    }
    unsigned long long h[CTR64_N];
    LSG_CUDA(cudaMemcpyAsync(h, r.ctr64, sizeof h, cudaMemcpyDeviceToHost, s));
    LSG_CUDA(cudaStreamSynchronize(s));
    if (ascii_dev) {
        unsigned long long fb = 0;
        LSG_CUDA(cudaMemcpyAsync(&fb, first_bad, 8, cudaMemcpyDeviceToHost, s));
        LSG_CUDA(cudaStreamSynchronize(s));
        if (fb != ~0ull) {
            set_error("read %llu holds a byte outside ACGTacgt", fb);
            return LASAGNA_EINVAL;
        }
    }
    if (r.bucketed && h[CTR_OVERFLOW]) {
        if (r.lay.K > 1) { // the exact path needs whole tables: not in a sub-pass workspace
            set_error("a slack region overflowed in a hash-range sub-pass: give the call a "
                      "workspace for one whole length (%zu bytes)", layout(g, 1, cap, true, 1).total);
            return LASAGNA_ENOSPC;
        }
        continue; // a slack region overflowed: exact path
    }
    const unsigned long long *book = old_greedy() ? h + CTR_BOOK : h + CTR_PEER + PC_BOOK;
    const unsigned long long work = old_greedy() ? h[CTR_WORK] : h[CTR_PEER + PC_WORK];
    if (book[2] > cap) {
        const uint64_t need = book[2] + book[2] / 4;
        *workspace_bytes = layout(g, G, need, true, r.lay.K).total;
        set_error("a length produced %llu pairs > pool %llu", book[2], (unsigned long long)cap);
        return LASAGNA_ENOSPC;
    }
    if (stats) {
        // every verified pair, including those the join dropped as dead
        st.n_pairs = join_filter() ? h[CTR_FOUND] : book[1];
        st.n_greedy = book[0];
        st.rounds_max = (uint32_t)book[3];
        st.fp_false_matches = h[CTR_FALSE];
        st.greedy_pair_rounds = work;
        st.pruned_entries = h[CTR_PRUNED];
        st.partition_levels = r.bucketed ? g.P : 0;
        st.hash_subpasses = r.lay.K;
        if ((rc = tm.finish(&st)) != LASAGNA_OK) return rc;
        st.kernel_launches = launch_count() - launches0;
        *stats = st;
    }
    return LASAGNA_OK;
  }
    set_error("internal: no path completed");
    return LASAGNA_ECUDA;
}

lasagna_status lasagna_greedy_graph(const uint64_t *packed, uint64_t n, uint32_t L,
                                    uint32_t l_min, uint32_t lengths_per_pass, void *workspace,
                                    size_t *workspace_bytes, uint32_t *succ, uint8_t *olen,
                                    lasagna_stats *stats, void *stream)
{
    g_err[0] = 0;
    return greedy_graph_impl(packed, nullptr, nullptr, nullptr, nullptr, n, L, l_min, lengths_per_pass,
                             workspace, workspace_bytes, succ, olen, stats, stream);
}

lasagna_status lasagna_greedy_graph_ascii(const char *ascii, uint64_t n, uint32_t L,
                                          uint32_t l_min, uint32_t lengths_per_pass,
                                          void *workspace, size_t *workspace_bytes,
                                          uint64_t *packed_out, uint64_t *first_bad,
                                          uint32_t *succ, uint8_t *olen, lasagna_stats *stats,
                                          void *stream)
{
    g_err[0] = 0;
    const char *dev = nullptr;
    bool is_host = false;
    if (workspace && n) {
        if (!ascii) {
            set_error("ascii is NULL");
            return LASAGNA_EINVAL;
        }
        lasagna_status rc = resolve_ascii(ascii, &dev, &is_host);
        if (rc != LASAGNA_OK) return rc;
    }
    // page-locked host input: the fast path streams it in by DMA (scatter_from_host)
    const char *host = is_host ? ascii : nullptr;
    return greedy_graph_impl(nullptr, dev ? dev : ascii, host, packed_out, first_bad, n, L, l_min,
                             lengths_per_pass, workspace, workspace_bytes, succ, olen, stats,
                             stream);
}

static lasagna_status overlaps_impl(const uint64_t *packed, uint64_t n, uint32_t L, uint32_t l_min,
                                    void *workspace, size_t *workspace_bytes, uint32_t *pair_a,
                                    uint32_t *pair_b, uint8_t *pair_l, uint64_t capacity,
                                    uint64_t *n_pairs, void *stream, bool approx);

lasagna_status lasagna_overlaps(const uint64_t *packed, uint64_t n, uint32_t L, uint32_t l_min,
                                void *workspace, size_t *workspace_bytes, uint32_t *pair_a,
                                uint32_t *pair_b, uint8_t *pair_l, uint64_t capacity,
                                uint64_t *n_pairs, void *stream)
{
    g_err[0] = 0;
    return overlaps_impl(packed, n, L, l_min, workspace, workspace_bytes, pair_a, pair_b, pair_l,
                         capacity, n_pairs, stream, false);
}

lasagna_status lasagna_overlaps_approx(const uint64_t *packed, uint64_t n, uint32_t L,
                                       uint32_t l_min, void *workspace, size_t *workspace_bytes,
                                       uint32_t *pair_a, uint32_t *pair_b, uint8_t *pair_l,
                                       uint64_t capacity, uint64_t *n_pairs, void *stream)
{
    g_err[0] = 0;
    return overlaps_impl(packed, n, L, l_min, workspace, workspace_bytes, pair_a, pair_b, pair_l,
                         capacity, n_pairs, stream, true);
}

static lasagna_status overlaps_impl(const uint64_t *packed, uint64_t n, uint32_t L, uint32_t l_min,
                                    void *workspace, size_t *workspace_bytes, uint32_t *pair_a,
                                    uint32_t *pair_b, uint8_t *pair_l, uint64_t capacity,
                                    uint64_t *n_pairs, void *stream, bool approx)
{
    lasagna_status rc = check_shape(n, L, l_min);
    if (rc != LASAGNA_OK) return rc;
    if (!workspace_bytes || !n_pairs) {
        set_error("NULL size/count pointer");
        return LASAGNA_EINVAL;
    }
    Geometry g = geometry(n, L, l_min);
    uint64_t cap = default_pool_cap(g);
    const uint32_t G_req = std::min<uint32_t>(g.n_len, 64);
    if (!workspace) {
        *workspace_bytes = layout(g, G_req, cap, false).total;
        return LASAGNA_OK;
    }
    *n_pairs = 0;
    if (n == 0) return LASAGNA_OK;
    if (!packed || !aligned(packed, 16) || !aligned(workspace, 256) ||
        (capacity && (!pair_a && !pair_b && !pair_l))) {
        set_error("NULL or misaligned pointer");
        return LASAGNA_EINVAL;
    }
    uint32_t G = choose_G(g, G_req, *workspace_bytes, cap, false);
    if (G == 0) {
        *workspace_bytes = layout(g, 1, cap, false).total;
        set_error("workspace too small");
        return LASAGNA_ENOSPC;
    }
    {
        size_t spare = *workspace_bytes - layout(g, G, cap, false).total;
        cap += spare / 16; // pool + pool2: 16 B per pair (the status words shrink it below)
        while (cap > default_pool_cap(g) && layout(g, G, cap, false).total > *workspace_bytes) cap -= cap / 256 + 1;
    }
    cudaStream_t s = (cudaStream_t)stream;
    Run r;
    r.g = g;
    r.lay = layout(g, G, cap, false);
    r.s = s;
    r.bind(workspace);
    r.approx = approx;
  for (int attempt = 0; attempt < 2; ++attempt) {
    r.bucketed = attempt == 0 && use_bucketed(g);
    PhaseTimer tm;
    tm.on = false;
    if ((rc = sort_ctx_reset(r.sctx, s)) != LASAGNA_OK) return rc;
    LSG_CUDA(cudaMemsetAsync(r.ctr64, 0, 8 * sizeof(unsigned long long), s));
    uint64_t total = 0;
    uint64_t worst = 0;
    for (int64_t l_hi = (int64_t)L - 1; l_hi >= (int64_t)l_min; l_hi -= G) {
        const uint32_t l_lo = (uint32_t)std::max<int64_t>(l_min, l_hi - (int64_t)G + 1);
        int which = 0;
        if ((rc = build_group(r, packed, l_lo, (uint32_t)l_hi, &which, tm, nullptr)) != LASAGNA_OK)
            return rc;
        for (int64_t l = l_hi; l >= (int64_t)l_lo; --l) {
            uint64_t m = 0;
            if ((rc = search_length(r, packed, (uint32_t)l, l_lo, which, &m)) != LASAGNA_OK)
                return rc;
            worst = std::max(worst, m);
            if (m > cap) { // count only from here on
                total += m;
                continue;
            }
            if (m && total < capacity) {
                // sort this length's pairs by (a, b): compact key a << vbits | b
                uint64_t *keys[2] = {reinterpret_cast<uint64_t *>(r.pool2),
                                     reinterpret_cast<uint64_t *>(r.pool)};
                if ((rc = launch_pairs_to_keys(r.pool, r.ctr64, m, cap, g.vbits, keys[0], s)) !=
                    LASAGNA_OK)
                    return rc;
                int which2 = 0;
                if ((rc = sort_segments(keys, m, 1, 0, 2 * g.vbits, r.hist, false, r.sctx, s,
                                        &which2)) != LASAGNA_OK)
                    return rc;
                const uint64_t take = std::min<uint64_t>(m, capacity - total);
                if ((rc = launch_keys_to_output(keys[which2], take, g.vbits, (uint8_t)l,
                                                pair_a ? pair_a + total : nullptr,
                                                pair_b ? pair_b + total : nullptr,
                                                pair_l ? pair_l + total : nullptr, s)) != LASAGNA_OK)
                    return rc;
            }
            total += m;
        }
    }
    unsigned long long ovf = 0;
    LSG_CUDA(cudaMemcpyAsync(&ovf, r.ctr64 + CTR_OVERFLOW, 8, cudaMemcpyDeviceToHost, s));
    LSG_CUDA(cudaStreamSynchronize(s));
    if (r.bucketed && ovf) continue; // a slack region overflowed: redo on the exact path
    *n_pairs = total;
    if (worst > cap) {
        *workspace_bytes = layout(g, G, worst + worst / 4, false).total;
        set_error("a length produced %llu pairs > pool %llu", (unsigned long long)worst,
                  (unsigned long long)cap);
        return LASAGNA_ENOSPC;
    }
    if (total > capacity) {
        set_error("|P| = %llu > capacity %llu", (unsigned long long)total,
                  (unsigned long long)capacity);
        return LASAGNA_ENOSPC;
    }
    return LASAGNA_OK;
  }
    set_error("internal: no path completed");
    return LASAGNA_ECUDA;
}

lasagna_status lasagna_compress(const uint64_t *packed, uint64_t n, uint32_t L,
                                const uint32_t *succ, const uint8_t *olen, void *workspace,
                                size_t *workspace_bytes, char *contigs, uint64_t contig_capacity,
                                uint64_t *contig_offsets, uint32_t *contig_seed,
                                uint64_t count_capacity, uint64_t *n_contigs,
                                uint64_t *total_bases, void *stream)
{
    g_err[0] = 0;
    if (L < 2 || L > 256) {
        set_error("L=%u out of range [2, 256]", L);
        return LASAGNA_EINVAL;
    }
    if (n > 0x7FFFFFFFull) {
        set_error("2n exceeds 0xFFFFFFFE vertex ids");
        return LASAGNA_ERANGE;
    }
    if (!workspace_bytes || (workspace && (!n_contigs || !total_bases))) {
        set_error("NULL size/count pointer");
        return LASAGNA_EINVAL;
    }
    if (workspace && n && (!packed || !succ || !olen || !aligned(packed, 16) ||
                           !aligned(succ, 4) || !aligned(workspace, 256) ||
                           (contig_offsets && !aligned(contig_offsets, 8)))) {
        set_error("NULL or misaligned pointer");
        return LASAGNA_EINVAL;
    }
    return compress_impl(packed, n, L, succ, olen, workspace, workspace_bytes, contigs,
                         contig_capacity, contig_offsets, contig_seed, count_capacity, n_contigs,
                         total_bases, (cudaStream_t)stream);
}

lasagna_status lasagna_sort_u64(uint64_t *keys, uint64_t *scratch, uint64_t count,
                                uint32_t bit_lo, uint32_t bit_hi, void *workspace,
                                size_t *workspace_bytes, void *stream)
{
    return lasagna_sort_segments(keys, scratch, count, 1, bit_lo, bit_hi, workspace,
                                 workspace_bytes, stream);
}

} // extern "C"

extern "C" lasagna_status lasagna_greedy_pairs(uint64_t n, const uint8_t *pl, const uint32_t *pa,
                                               const uint32_t *pb, uint64_t count, void *workspace,
                                               size_t *workspace_bytes, uint32_t *succ,
                                               uint8_t *olen, uint32_t *rounds, void *stream)
{
    g_err[0] = 0;
    if (!workspace_bytes) {
        set_error("workspace_bytes is NULL");
        return LASAGNA_EINVAL;
    }
    if (n > 0x7FFFFFFFull) {
        set_error("2n exceeds 0xFFFFFFFE vertex ids");
        return LASAGNA_ERANGE;
    }
    const uint64_t V = 2 * n;
    const uint64_t c1 = std::max<uint64_t>(count, 1);
    // keys, keys2 | pool, pool2 | status | ctrs | hist | best | claimed
    size_t off = 0;
    auto take = [&](size_t b) {
        size_t o = off;
        off += align256(b);
        return o;
    };
    const size_t o_keys = take(c1 * 8), o_keys2 = take(c1 * 8), o_pool = take(c1 * 8),
                 o_pool2 = take(c1 * 8), o_status = take(sort_status_bytes(c1, 1)),
                 o_ctrs = take(CTR_BYTES), o_hist = take(8 * 256 * 4), o_best = take(V * 8 + 8),
                 o_claimed = take(ceil_div(V, 32) * 4 + 4);
    if (!workspace) {
        *workspace_bytes = off;
        return LASAGNA_OK;
    }
    if (*workspace_bytes < off) {
        *workspace_bytes = off;
        set_error("workspace too small");
        return LASAGNA_ENOSPC;
    }
    if (!succ || !olen || !aligned(workspace, 256) || (count && (!pl || !pa || !pb))) {
        set_error("NULL or misaligned pointer");
        return LASAGNA_EINVAL;
    }
    cudaStream_t s = (cudaStream_t)stream;
    char *ws = (char *)workspace;
    LSG_CUDA(cudaMemsetAsync(succ, 0xFF, V * 4, s));
    LSG_CUDA(cudaMemsetAsync(olen, 0, V, s));
    if (rounds) *rounds = 0;
    if (count == 0) {
        LSG_CUDA(cudaStreamSynchronize(s));
        return LASAGNA_OK;
    }
    SortCtx c;
    c.status = reinterpret_cast<unsigned long long *>(ws + o_status);
    c.status_bytes = sort_status_bytes(c1, 1);
    c.tile_ctrs = reinterpret_cast<uint32_t *>(ws + o_ctrs);
    c.epoch = 0;
    lasagna_status rc = sort_ctx_reset(c, s);
    if (rc != LASAGNA_OK) return rc;
    unsigned long long *ctr64 = reinterpret_cast<unsigned long long *>(ws + o_ctrs + 4096 * 4);
    LSG_CUDA(cudaMemsetAsync(ctr64, 0, CTR64_N * 8, s));
    uint32_t *claimed = reinterpret_cast<uint32_t *>(ws + o_claimed);
    LSG_CUDA(cudaMemsetAsync(claimed, 0, ceil_div(V, 32) * 4, s));
    // group by length, descending: key (255 - l) << 56 | i, one 8-bit LSD pass
    uint64_t *keys[2] = {reinterpret_cast<uint64_t *>(ws + o_keys),
                         reinterpret_cast<uint64_t *>(ws + o_keys2)};
    if ((rc = launch_lkeys(pl, count, keys[0], s)) != LASAGNA_OK) return rc;
    uint32_t *hist = reinterpret_cast<uint32_t *>(ws + o_hist);
    int which = 0;
    if ((rc = sort_segments(keys, count, 1, 56, 64, hist, false, c, s, &which)) != LASAGNA_OK)
        return rc;
    uint32_t h[256];
    LSG_CUDA(cudaMemcpyAsync(h, hist, sizeof h, cudaMemcpyDeviceToHost, s));
    LSG_CUDA(cudaStreamSynchronize(s));
    GreedyBufs gb;
    gb.pool = reinterpret_cast<unsigned long long *>(ws + o_pool);
    gb.pool2 = reinterpret_cast<unsigned long long *>(ws + o_pool2);
    gb.cnt = ctr64 + CTR_POOL;
    gb.cnt2 = ctr64 + CTR_POOL2;
    gb.cnt3 = ctr64 + CTR_POOL3;
    gb.book = ctr64 + CTR_BOOK;
    gb.work = ctr64 + CTR_WORK;
    gb.best = reinterpret_cast<unsigned long long *>(ws + o_best);
    gb.claimed = claimed;
    gb.cap = c1;
    gb.epoch = 1;
    LSG_CUDA(cudaMemsetAsync(gb.best, 0, V * 8, s));
    const GreedyPeers peers = single_peers(gb, ctr64 + CTR_PEER, succ, olen, V);
    uint64_t pos = 0;
    for (int d = 0; d < 256; ++d) { // digit d = 255 - l: longest lengths first
        const uint64_t m = h[d];
        if (!m) continue;
        const uint8_t l = (uint8_t)(255 - d);
        if ((rc = launch_gather_pairs(keys[which], pos, m, pa, pb, gb.pool, gb.cnt, s)) != LASAGNA_OK)
            return rc;
        if ((rc = old_greedy() ? greedy_length(gb, l, succ, olen, s)
                               : greedy_length_peers(peers, l, s)) != LASAGNA_OK)
            return rc;
        pos += m;
    }
    unsigned long long bk[4];
    LSG_CUDA(cudaMemcpyAsync(bk, old_greedy() ? gb.book : ctr64 + CTR_PEER + PC_BOOK, sizeof bk,
                             cudaMemcpyDeviceToHost, s));
    LSG_CUDA(cudaStreamSynchronize(s));
    if (rounds) *rounds = (uint32_t)bk[3];
    return LASAGNA_OK;
}

// ==================================================================== sharded phases
// Building blocks of the multi-GPU driver (paper_conf_ipps_goswamilsp18_b200/dist.py): the
// same kernels as lasagna_greedy_graph, with global vertex ids and caller-managed buffers.
extern "C" {

uint32_t lasagna_vertex_bits(uint64_t n_total) { return geometry(n_total, 2, 1).vbits; }

uint32_t lasagna_key_sort_bits(uint64_t n_total) { return geometry(n_total, 2, 1).T; }

lasagna_status lasagna_table_keys(const uint64_t *packed, uint64_t n_local, uint64_t read_offset,
                                  uint64_t n_total, uint32_t L, uint32_t l_lo, uint32_t l_hi,
                                  uint64_t *tab, void *stream)
{
    g_err[0] = 0;
    lasagna_status rc = check_shape(n_total, L, l_lo);
    if (rc != LASAGNA_OK) return rc;
    if (l_hi < l_lo || l_hi >= L || l_hi - l_lo + 1 > 64 || read_offset + n_local > n_total) {
        set_error("bad length group [%u, %u] or read range", l_lo, l_hi);
        return LASAGNA_EINVAL;
    }
    if (n_local == 0) return LASAGNA_OK;
    if (!packed || !tab || !aligned(packed, 16) || !aligned(tab, 16)) {
        set_error("NULL or misaligned pointer");
        return LASAGNA_EINVAL;
    }
    Geometry g = geometry(n_total, L, l_lo);
    TableArgs ta;
    ta.packed = packed;
    ta.n = n_local;
    ta.read_offset = read_offset;
    ta.L = L;
    ta.stride = stride_for(L);
    ta.l_lo = l_lo;
    ta.l_hi = l_hi;
    ta.vbits = g.vbits;
    ta.d_shift = 0;
    ta.d_bits = 1;
    ta.tab = tab;
    ta.hist = nullptr;
    return launch_table(ta, (cudaStream_t)stream);
}

lasagna_status lasagna_digit_counts(const uint64_t *keys, uint64_t seg_len, uint32_t n_seg,
                                    uint32_t shift, uint32_t bits, uint32_t *counts, void *stream)
{
    g_err[0] = 0;
    if (bits < 1 || bits > 8 || shift + bits > 64 || !counts || (seg_len && !keys)) {
        set_error("bad digit or NULL pointer");
        return LASAGNA_EINVAL;
    }
    cudaStream_t s = (cudaStream_t)stream;
    LSG_CUDA(cudaMemsetAsync(counts, 0, (size_t)n_seg * 256 * 4, s));
    return launch_hist(keys, seg_len, n_seg, shift, bits, counts, s);
}

lasagna_status lasagna_sort_segments(uint64_t *keys, uint64_t *scratch, uint64_t seg_len,
                                     uint32_t n_seg, uint32_t bit_lo, uint32_t bit_hi,
                                     void *workspace, size_t *workspace_bytes, void *stream)
{
    g_err[0] = 0;
    if (!workspace_bytes || bit_lo >= bit_hi || bit_hi > 64 || n_seg == 0) {
        set_error("bad bit range, segment count or NULL workspace_bytes");
        return LASAGNA_EINVAL;
    }
    const size_t need = align256(sort_status_bytes(seg_len, n_seg)) + align256(CTR_BYTES) +
                        align256((size_t)8 * n_seg * 256 * 4);
    if (!workspace) {
        *workspace_bytes = need;
        return LASAGNA_OK;
    }
    if (*workspace_bytes < need) {
        *workspace_bytes = need;
        set_error("workspace too small");
        return LASAGNA_ENOSPC;
    }
    if (seg_len == 0) return LASAGNA_OK;
    if (!keys || !scratch || !aligned(keys, 8) || !aligned(scratch, 8) || !aligned(workspace, 256)) {
        set_error("NULL or misaligned pointer");
        return LASAGNA_EINVAL;
    }
    if (seg_len > 0xFFFFFFFFull) {
        set_error("segment length must be < 2^32");
        return LASAGNA_ERANGE;
    }
    cudaStream_t s = (cudaStream_t)stream;
    char *ws = (char *)workspace;
    SortCtx c;
    c.status = reinterpret_cast<unsigned long long *>(ws);
    c.status_bytes = sort_status_bytes(seg_len, n_seg);
    c.tile_ctrs = reinterpret_cast<uint32_t *>(ws + align256(c.status_bytes));
    uint32_t *hist = reinterpret_cast<uint32_t *>(ws + align256(c.status_bytes) + align256(CTR_BYTES));
    lasagna_status rc = sort_ctx_reset(c, s);
    if (rc != LASAGNA_OK) return rc;
    uint64_t *bufs[2] = {keys, scratch};
    int which = 0;
    rc = sort_segments(bufs, seg_len, n_seg, bit_lo, bit_hi, hist, false, c, s, &which);
    if (rc != LASAGNA_OK) return rc;
    if (which == 1)
        LSG_CUDA(cudaMemcpyAsync(keys, scratch, seg_len * n_seg * 8, cudaMemcpyDeviceToDevice, s));
    return LASAGNA_OK;
}

lasagna_status lasagna_join(const uint64_t *keys, uint64_t count, const uint64_t *packed_all,
                            uint64_t n_total, uint32_t L, uint32_t l, uint64_t *pairs,
                            uint64_t capacity, uint64_t *counters, void *stream)
{
    g_err[0] = 0;
    lasagna_status rc = check_shape(n_total, L, l);
    if (rc != LASAGNA_OK) return rc;
    if (!counters || (count && (!keys || !packed_all)) || (capacity && !pairs) ||
        !aligned(counters, 8) || (packed_all && !aligned(packed_all, 16))) {
        set_error("NULL or misaligned pointer");
        return LASAGNA_EINVAL;
    }
    if (count == 0) return LASAGNA_OK;
    Geometry g = geometry(n_total, L, l);
    JoinArgs ja;
    ja.packed = packed_all;
    ja.keys = keys;
    ja.N = count;
    ja.V = g.V;
    ja.L = L;
    ja.stride = stride_for(L);
    ja.l = l;
    ja.vbits = g.vbits;
    ja.T = g.T;
    ja.pairs = reinterpret_cast<unsigned long long *>(pairs);
    ja.cap = capacity;
    ja.count = reinterpret_cast<unsigned long long *>(counters);
    ja.false_matches = reinterpret_cast<unsigned long long *>(counters) + 1;
    return launch_join(ja, (cudaStream_t)stream);
}

} // extern "C"

// ==================================================================== sharded fast path
// The multi-GPU driver on the bucketed kernels (P:L204 shuffle re-keyed by
// fingerprint, the paper's future work P:L333).  Rank r holds reads [r n_pad, (r+1) n_pad).
//   lasagna_shard_scatter    a1..a3 + level 1 of its reads, regions in hash-range shard order
//                            (rank o owns level-1 digits [ceil(256 o / g), ceil(256 (o+1) / g)))
//   (caller) all-to-all      equal split sizes: rank o's regions of the G lengths are one
//                            contiguous slice of every sender's buffer
//   lasagna_shard_partition  the remaining levels over the g received slices (multi-source refine)
//   lasagna_shard_join       a5 of one length over this rank's buckets
//   lasagna_greedy_shard_length  a6/a7 over peer memory (greedy_rounds.cu)
namespace lsg {

struct ShardGeom {
    Geometry g; // geometry of the n_total-read set, at least two levels
    uint32_t world, nb_pad;
    uint64_t n_pad, slice, cap1;
};

static ShardGeom shard_geom(uint64_t n_total, uint32_t world, uint32_t L, uint32_t l_min)
{
    ShardGeom s;
    s.g = geometry(n_total, L, l_min);
    if (s.g.P < 2) { // one level would leave nothing to refine after the exchange
        s.g.P = 2;
        s.g.dlast = 8;
        s.g.T = 16;
        s.g.n_buckets = 1ull << 16;
        s.g.half = region_cap((double)s.g.N / (double)(2 * s.g.n_buckets));
    }
    s.world = world;
    s.nb_pad = (256 + world - 1) / world;
    s.n_pad = (ceil_div(n_total, world) + 15) & ~15ull; // a rank's ends: whole bitmap words
    s.slice = 2 * s.n_pad;
    s.cap1 = region_cap(2.0 * (double)s.n_pad / 256.0);
    return s;
}

struct ShardPart {
    size_t out2, fill2, out3, fill3, total;
};

// workspace of lasagna_shard_partition for G lengths: R = G nb_pad level-1 regions
static ShardPart shard_part_layout(const ShardGeom &sg, uint32_t G)
{
    const Geometry &g = sg.g;
    const uint64_t R = (uint64_t)G * sg.nb_pad;
    ShardPart p;
    size_t off = 0;
    auto take = [&](size_t bytes) {
        size_t o = off;
        off += align256(bytes);
        return o;
    };
    if (g.P == 2) {
        p.out2 = take(R * 256 * 2 * g.half * 8);
        p.fill2 = take(R * 512 * 4);
        p.out3 = p.fill3 = 0;
    } else {
        p.out2 = take(R * 256 * g.cap2 * 8);
        p.fill2 = take(R * 256 * 4);
        const uint64_t nb3 = 1ull << g.dlast;
        p.out3 = take(R * 256 * nb3 * 2 * g.half * 8);
        p.fill3 = take(R * 256 * nb3 * 2 * 4);
    }
    p.total = off;
    return p;
}

static lasagna_status shard_check(uint64_t n_total, uint32_t world, uint32_t L, uint32_t l_min,
                                  uint32_t l_lo, uint32_t l_hi)
{
    lasagna_status rc = check_shape(n_total, L, l_min);
    if (rc != LASAGNA_OK) return rc;
    if (world < 1 || world > MAX_PEERS) {
        set_error("world=%u out of range [1, %u]", world, MAX_PEERS);
        return LASAGNA_EINVAL;
    }
    if (l_lo < l_min || l_hi < l_lo || l_hi >= L || l_hi - l_lo + 1 > 64) {
        set_error("bad length group [%u, %u]", l_lo, l_hi);
        return LASAGNA_EINVAL;
    }
    return LASAGNA_OK;
}

} // namespace lsg

extern "C" {

lasagna_status lasagna_shard_geometry(uint64_t n_total, uint32_t world, uint32_t L, uint32_t l_min,
                                      lasagna_shard_geom *out)
{
    g_err[0] = 0;
    lasagna_status rc = shard_check(n_total, world, L, l_min, l_min, l_min);
    if (rc != LASAGNA_OK) return rc;
    if (!out) {
        set_error("NULL output");
        return LASAGNA_EINVAL;
    }
    const ShardGeom sg = shard_geom(n_total, world, L, l_min);
    out->levels = sg.g.P;
    out->last_bits = sg.g.dlast;
    out->nb_pad = sg.nb_pad;
    out->vbits = sg.g.vbits;
    out->n_pad = sg.n_pad;
    out->slice = sg.slice;
    out->cap1 = sg.cap1;
    out->send_entries = (uint64_t)world * sg.nb_pad * sg.cap1;
    out->fill_words = (uint64_t)world * sg.nb_pad;
    out->part_bytes = shard_part_layout(sg, 1).total;
    out->buckets = (uint64_t)sg.nb_pad * 256 * (sg.g.P == 3 ? (1ull << sg.g.dlast) : 1ull);
    return LASAGNA_OK;
}

lasagna_status lasagna_shard_part_bytes(uint64_t n_total, uint32_t world, uint32_t L,
                                        uint32_t l_min, uint32_t lengths, size_t *bytes)
{
    g_err[0] = 0;
    lasagna_status rc = shard_check(n_total, world, L, l_min, l_min, l_min);
    if (rc != LASAGNA_OK) return rc;
    if (!bytes || lengths < 1 || lengths > 64) {
        set_error("NULL output or lengths out of [1, 64]");
        return LASAGNA_EINVAL;
    }
    *bytes = shard_part_layout(shard_geom(n_total, world, L, l_min), lengths).total;
    return LASAGNA_OK;
}

lasagna_status lasagna_shard_scatter(const uint64_t *packed_local, uint64_t n_local,
                                     uint64_t read_offset, uint64_t n_total, uint32_t world,
                                     uint32_t L, uint32_t l_min, uint32_t l_lo, uint32_t l_hi,
                                     const uint32_t *claimed, uint64_t *send, uint32_t *send_fill,
                                     uint64_t *counters, void *stream)
{
    g_err[0] = 0;
    lasagna_status rc = shard_check(n_total, world, L, l_min, l_lo, l_hi);
    if (rc != LASAGNA_OK) return rc;
    const ShardGeom sg = shard_geom(n_total, world, L, l_min);
    if (read_offset % sg.n_pad || n_local > sg.n_pad || read_offset + n_local > n_total) {
        set_error("read range [%llu, +%llu) is not a shard of n_pad=%llu", (unsigned long long)read_offset,
                  (unsigned long long)n_local, (unsigned long long)sg.n_pad);
        return LASAGNA_EINVAL;
    }
    if (!send || !send_fill || !counters || (n_local && !packed_local) || !aligned(send, 16) ||
        !aligned(counters, 8) || (packed_local && !aligned(packed_local, 16))) {
        set_error("NULL or misaligned pointer");
        return LASAGNA_EINVAL;
    }
    cudaStream_t s = (cudaStream_t)stream;
    const uint32_t G = l_hi - l_lo + 1;
    LSG_CUDA(cudaMemsetAsync(send_fill, 0, (size_t)G * world * sg.nb_pad * 4, s));
    if (n_local == 0) return LASAGNA_OK;
    ScatterArgs sa;
    sa.packed = packed_local;
    sa.n = n_local;
    sa.read_offset = read_offset;
    sa.L = L;
    sa.stride = stride_for(L);
    sa.l_lo = l_lo;
    sa.l_hi = l_hi;
    sa.vbits = sg.g.vbits;
    sa.keep = stored_keep(sg.g);
    sa.out = send;
    sa.fill = send_fill;
    sa.split = false;
    sa.cap = sg.cap1;
    sa.overflow = reinterpret_cast<uint32_t *>(counters);
    sa.ascii = nullptr;
    sa.packed_out = nullptr;
    sa.first_bad = nullptr;
    // the caller's bitmap holds this rank's ends [2 read_offset, ...): index it globally
    sa.claimed = claimed ? claimed - (2 * read_offset) / 32 : nullptr;
    sa.pruned = reinterpret_cast<unsigned long long *>(counters) + 1;
    sa.dest_g = world;
    sa.nb_pad = sg.nb_pad;
    return launch_scatter_table(sa, s);
}

lasagna_status lasagna_shard_partition(const uint64_t *recv, const uint32_t *recv_fill,
                                       uint64_t n_total, uint32_t world, uint32_t L,
                                       uint32_t l_min, uint32_t l_lo, uint32_t l_hi, void *part,
                                       uint64_t *counters, void *stream)
{
    g_err[0] = 0;
    lasagna_status rc = shard_check(n_total, world, L, l_min, l_lo, l_hi);
    if (rc != LASAGNA_OK) return rc;
    if (!recv || !recv_fill || !part || !counters || !aligned(part, 256) || !aligned(recv, 16)) {
        set_error("NULL or misaligned pointer");
        return LASAGNA_EINVAL;
    }
    const ShardGeom sg = shard_geom(n_total, world, L, l_min);
    const Geometry &g = sg.g;
    const uint32_t G = l_hi - l_lo + 1;
    const ShardPart pl = shard_part_layout(sg, G);
    char *ws = (char *)part;
    cudaStream_t s = (cudaStream_t)stream;
    const uint64_t R = (uint64_t)G * sg.nb_pad;
    RefineArgs ra;
    ra.in = recv;
    ra.fill_in = recv_fill;
    ra.cap_in = sg.cap1;
    ra.dshift = 56;
    ra.dbits = 8;
    ra.out = reinterpret_cast<uint64_t *>(ws + pl.out2);
    ra.fill_out = reinterpret_cast<uint32_t *>(ws + pl.fill2);
    ra.cap_out = g.P == 2 ? g.half : g.cap2;
    ra.vbits = g.vbits;
    ra.split = g.P == 2;
    ra.overflow = reinterpret_cast<uint32_t *>(counters);
    ra.n_src = world;
    ra.src_stride = R; // sender k's slice for this rank: regions [k R, (k+1) R) of recv
    if ((rc = launch_refine(ra, R, s)) != LASAGNA_OK) return rc;
    if (g.P == 3) {
        ra.in = reinterpret_cast<uint64_t *>(ws + pl.out2);
        ra.fill_in = reinterpret_cast<uint32_t *>(ws + pl.fill2);
        ra.cap_in = g.cap2;
        ra.dshift = 56 - g.dlast;
        ra.dbits = g.dlast;
        ra.out = reinterpret_cast<uint64_t *>(ws + pl.out3);
        ra.fill_out = reinterpret_cast<uint32_t *>(ws + pl.fill3);
        ra.cap_out = g.half;
        ra.split = true;
        ra.n_src = 1;
        ra.src_stride = 0;
        if ((rc = launch_refine(ra, R * 256, s)) != LASAGNA_OK) return rc;
    }
    return LASAGNA_OK;
}

lasagna_status lasagna_shard_join(const void *part, uint64_t n_total, uint32_t world, uint32_t L,
                                  uint32_t l_min, uint32_t l_lo, uint32_t l_hi, uint32_t l,
                                  const uint64_t *packed_all, uint64_t *pool, uint64_t capacity,
                                  uint64_t *pool_count, uint64_t *counters, void *stream)
{
    g_err[0] = 0;
    lasagna_status rc = shard_check(n_total, world, L, l_min, l_lo, l_hi);
    if (rc != LASAGNA_OK) return rc;
    if (l < l_lo || l > l_hi) {
        set_error("length %u outside the group [%u, %u]", l, l_lo, l_hi);
        return LASAGNA_EINVAL;
    }
    if (!part || !packed_all || !pool_count || !counters || (capacity && !pool) ||
        !aligned(part, 256) || !aligned(packed_all, 16)) {
        set_error("NULL or misaligned pointer");
        return LASAGNA_EINVAL;
    }
    const ShardGeom sg = shard_geom(n_total, world, L, l_min);
    const Geometry &g = sg.g;
    const uint32_t G = l_hi - l_lo + 1;
    const ShardPart pl = shard_part_layout(sg, G);
    char *ws = (char *)const_cast<void *>(part);
    cudaStream_t s = (cudaStream_t)stream;
    const uint64_t nbk = (uint64_t)sg.nb_pad * 256 * (g.P == 3 ? (1ull << g.dlast) : 1ull);
    const uint32_t seg = l - l_lo;
    LSG_CUDA(cudaMemsetAsync(pool_count, 0, 8, s));
    BucketJoinArgs bj;
    bj.j.packed = packed_all;
    bj.j.keys = nullptr;
    bj.j.N = 0;
    bj.j.V = g.V;
    bj.j.L = L;
    bj.j.stride = stride_for(L);
    bj.j.l = l;
    bj.j.vbits = g.vbits;
    bj.j.T = g.T;
    bj.j.pairs = reinterpret_cast<unsigned long long *>(pool);
    bj.j.cap = capacity;
    bj.j.count = reinterpret_cast<unsigned long long *>(pool_count);
    bj.j.false_matches = reinterpret_cast<unsigned long long *>(counters) + 3;
    bj.j.claimed = nullptr;
    bj.j.found = nullptr;
    bj.overflow = reinterpret_cast<uint32_t *>(counters);
    const size_t ob = g.P == 2 ? pl.out2 : pl.out3, of = g.P == 2 ? pl.fill2 : pl.fill3;
    bj.buckets = reinterpret_cast<uint64_t *>(ws + ob) + (uint64_t)seg * nbk * 2 * g.half;
    bj.fills = reinterpret_cast<uint32_t *>(ws + of) + (uint64_t)seg * nbk * 2;
    bj.half_cap = g.half;
    bj.n_buckets = nbk;
    if ((rc = launch_bucket_join(bj, s)) != LASAGNA_OK) return rc;
    return LASAGNA_OK;
}

lasagna_status lasagna_greedy_shard_length(const lasagna_greedy_rank *ranks, uint32_t world,
                                           int32_t rank, uint64_t slice, uint64_t capacity,
                                           uint32_t l, void *stream)
{
    g_err[0] = 0;
    if (!ranks || world < 1 || world > MAX_PEERS || rank < -1 || rank >= (int32_t)world ||
        l < 1 || l > 255 || (world > 1 && (slice == 0 || slice % 32 || capacity < GR_TAIL_CAP))) {
        set_error("bad rank layout (world=%u rank=%d slice=%llu) or length %u", world, rank,
                  (unsigned long long)slice, l);
        return LASAGNA_EINVAL;
    }
    GreedyPeers p;
    for (uint32_t q = 0; q < world; ++q) {
        const lasagna_greedy_rank &x = ranks[q];
        p.r[q].pool = reinterpret_cast<unsigned long long *>(x.pool);
        p.r[q].pool2 = reinterpret_cast<unsigned long long *>(x.pool2);
        p.r[q].in_count = reinterpret_cast<unsigned long long *>(x.pool_count);
        p.r[q].ctr = reinterpret_cast<unsigned long long *>(x.ctr);
        p.r[q].best = reinterpret_cast<unsigned long long *>(x.best);
        p.r[q].claimed = x.claimed;
        p.r[q].succ = x.succ;
        p.r[q].olen = x.olen;
        p.r[q].tail = reinterpret_cast<unsigned long long *>(x.tail);
    }
    p.g = world;
    p.slice = world > 1 ? slice : ~0ull >> 1;
    p.cap = capacity;
    p.rank0 = rank < 0 ? 0 : (uint32_t)rank;
    p.nranks_here = rank < 0 ? world : 1;
    return greedy_length_peers(p, (uint8_t)l, (cudaStream_t)stream);
}

lasagna_status lasagna_peer_alloc(size_t bytes, void **dev_ptr, void *handle)
{
    g_err[0] = 0;
    if (!dev_ptr || !handle || bytes == 0) {
        set_error("NULL output or zero size");
        return LASAGNA_EINVAL;
    }
    LSG_CUDA(cudaMalloc(dev_ptr, bytes));
    cudaIpcMemHandle_t h;
    cudaError_t e = cudaIpcGetMemHandle(&h, *dev_ptr);
    if (e != cudaSuccess) {
        cudaFree(*dev_ptr);
        *dev_ptr = nullptr;
        return cuda_status(e, "cudaIpcGetMemHandle");
    }
    memcpy(handle, &h, sizeof h);
    return LASAGNA_OK;
}

lasagna_status lasagna_peer_free(void *dev_ptr)
{
    g_err[0] = 0;
    LSG_CUDA(cudaFree(dev_ptr));
    return LASAGNA_OK;
}

lasagna_status lasagna_peer_open(const void *handle, void **dev_ptr)
{
    g_err[0] = 0;
    if (!handle || !dev_ptr) {
        set_error("NULL handle or output");
        return LASAGNA_EINVAL;
    }
    cudaIpcMemHandle_t h;
    memcpy(&h, handle, sizeof h);
    LSG_CUDA(cudaIpcOpenMemHandle(dev_ptr, h, cudaIpcMemLazyEnablePeerAccess));
    return LASAGNA_OK;
}

lasagna_status lasagna_peer_close(void *dev_ptr)
{
    g_err[0] = 0;
    LSG_CUDA(cudaIpcCloseMemHandle(dev_ptr));
    return LASAGNA_OK;
}

} // extern "C"
