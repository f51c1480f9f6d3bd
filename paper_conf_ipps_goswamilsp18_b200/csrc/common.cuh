// common.cuh — device helpers shared by the sm_100a kernels of liblasagna.so.
// (Nothing here is shared with oracle/: the two sides are independent by construction.)
#pragma once

#include <cuda_runtime.h>
#include <cstdio>
#include <stdint.h>

#include <algorithm>
#include <type_traits>

#include "lasagna.h"

// Device-side bounds checks of the checked build (build.build(checked=True) compiles with
// -DLSG_CHECKS into liblasagna_checked.so; LASAGNA_CHECKED=1 loads it).  compute-sanitizer is
// not available on the GPU pool, so the GPU tests run once against this build: a failed check
// prints its site and traps (the call then returns LASAGNA_ECUDA).  Free in the product build.
#ifdef LSG_CHECKS
#define LSG_DCHECK(cond)                                                                       \
    do {                                                                                       \
        if (!(cond)) {                                                                         \
            printf("LSG_DCHECK failed %s:%d: %s (block %d thread %d)\n", __FILE__, __LINE__,  \
                   #cond, (int)blockIdx.x, (int)threadIdx.x);                                  \
            __trap();                                                                          \
        }                                                                                      \
    } while (0)
#else
#define LSG_DCHECK(cond) do { } while (0)
#endif

namespace lsg {

// ----------------------------------------------------------------- fingerprint arithmetic
// F(s) = sum_k c_k 5^(|s|-1-k) mod q, q = 2^61 - 1 (R2, R4).
constexpr uint64_t Q61 = (1ull << 61) - 1;
constexpr uint32_t NONE = 0xFFFFFFFFu;

// x mod q for any x < 2^64 (Mersenne folding: 2^61 == 1 mod q).
__device__ __forceinline__ uint64_t mod61(uint64_t x)
{
    uint64_t r = (x & Q61) + (x >> 61);
    return r >= Q61 ? r - Q61 : r;
}

// Lazily reduced arithmetic: values are kept in [0, 2^61 + 7) ("folded", congruent mod q);
// fold(x) = (x & q) + (x >> 61) maps any x < 2^64 there with 4 32-bit ops and no compare.
__device__ __forceinline__ uint64_t fold61(uint64_t x) { return (x & Q61) + (x >> 61); }
// exact residue of a folded value
__device__ __forceinline__ uint64_t exact61(uint64_t x) { return x >= Q61 ? x - Q61 : x; }

// Horner step P <- P*5 + c on folded P (5(2^61+7) + 3 < 2^64: no 128-bit product).
__device__ __forceinline__ uint64_t horner5(uint64_t P, uint32_t c)
{
    return fold61((P << 2) + P + c);
}

// Ascending-power step S <- S + c * pw (pw = 5^j mod q, pw2 = 2 pw mod q, c <= 3):
// c*pw = (c&1)pw + (c&2 ? pw2 : 0); folded S + c*pw < 2^61 + 7 + 2^62 < 2^64.
__device__ __forceinline__ uint64_t addpow(uint64_t S, uint32_t c, uint64_t pw, uint64_t pw2)
{
    uint64_t t = S + ((c & 1u) ? pw : 0ull) + ((c & 2u) ? pw2 : 0ull);
    return fold61(t);
}

// Table key mixing: a bijection of the 64-bit word (multiplication by an odd constant mod
// 2^64, Fibonacci hashing), so equal fingerprints <=> equal mixed words, while the TOP bits
// are uniform even for short lengths where F < 5^l < 2^61 has leading zero bits.
constexpr uint64_t MIX = 0x9E3779B97F4A7C15ull;
__device__ __forceinline__ uint64_t mix(uint64_t f) { return f * MIX; }

// ----------------------------------------------------------------- canonical table entries
// ONE table entry per oriented read v and length l.  With
// x = prefix_l(seq(v)), H = F(x) and Hr = F(RC(x)) (= the suffix fingerprint of v^1):
//   key = mix(min(H, Hr)) top (62 - vbits) bits | flag << vbits | v
//   flag = 0 if H < Hr ("build" side), 1 if H > Hr ("probe" side), 2 if H == Hr (both).
// A directed overlap (u, v, l) means suffix_l(seq(u)) == prefix_l(seq(v)), i.e. the prefix
// strings of w = u^1 and v are reverse complements: equal canonical fingerprints and
// opposite flags (or both 2).  So the paper's two lists P_l / S_l collapse
// into one list of V entries whose build side plays P_l and whose probe side plays S_l.
constexpr uint32_t FLAG_BITS = 2;
__device__ __forceinline__ uint64_t key_keep(uint32_t vbits)
{
    return ~((1ull << (vbits + FLAG_BITS)) - 1);
}
// H, Hr folded (congruent mod q); the comparison is on the exact residues
__device__ __forceinline__ uint64_t canon_key(uint64_t H, uint64_t Hr, uint64_t keep,
                                              uint32_t vbits, uint64_t v)
{
    const uint64_t h = exact61(H), hr = exact61(Hr);
    const uint64_t c = h < hr ? h : hr;
    const uint64_t f = h < hr ? 0ull : (h > hr ? 1ull : 2ull);
    return (mix(c) & keep) | (f << vbits) | v;
}
// The bucketed path's form of the same entry (partition_scatter.cu): the top 8 bits of mix(min) pick
// the level-1 region and are implied by the region an entry sits in, so the stored key drops
// them and keeps the next 62 - vbits bits instead — 8 more fingerprint bits in every
// comparison (R12: at vbits = 32, 30 stored + 8 implied = 38 bits instead of 30):
//   key = (mix(min(H, Hr)) << 8) top (62 - vbits) bits | flag << vbits | v,  *d1 = mix >> 56.
// `keep` is key_keep(vbits) in production; a test may clear low fingerprint bits from it.
__device__ __forceinline__ uint64_t canon_key_d1(uint64_t H, uint64_t Hr, uint64_t keep,
                                                 uint32_t vbits, uint64_t v, uint32_t *d1)
{
    const uint64_t h = exact61(H), hr = exact61(Hr);
    const uint64_t c = h < hr ? h : hr;
    const uint64_t f = h < hr ? 0ull : (h > hr ? 1ull : 2ull);
    const uint64_t m = mix(c);
    *d1 = (uint32_t)(m >> 56);
    return ((m << 8) & keep) | (f << vbits) | v;
}
// The same entry from the bucketed path's mod-2^64 key streams (fingerprint.cuh Fp64Streams,
// reading R26): H and Hr are exact residues already.
// fl1 = 1 << vbits, fl2 = 2 << vbits (the flag field); v < 2^vbits <= 2^32.
__device__ __forceinline__ uint64_t canon_key64_d1(uint64_t H, uint64_t Hr, uint64_t keep,
                                                   uint64_t fl1, uint64_t fl2, uint32_t v,
                                                   uint32_t *d1)
{
    const bool lt = H < Hr;
    const uint64_t c = lt ? H : Hr;
    const uint64_t fb = lt ? 0ull : (H == Hr ? fl2 : fl1);
    const uint64_t m = mix(c);
    const uint32_t mlo = (uint32_t)m, mhi = (uint32_t)(m >> 32);
    *d1 = mhi >> 24;
    // (m << 8) & keep | flag | v on 32-bit halves (a funnel shift for the high half: the
    // compiler otherwise folds the shift into a second 64-bit multiply)
    const uint32_t klo = ((mlo << 8) & (uint32_t)keep) | (uint32_t)fb | v;
    const uint32_t khi = (__funnelshift_l(mlo, mhi, 8) & (uint32_t)(keep >> 32)) | (uint32_t)(fb >> 32);
    return ((uint64_t)khi << 32) | klo;
}
__device__ __forceinline__ uint32_t key_flag(uint64_t key, uint32_t vbits)
{
    return (uint32_t)(key >> vbits) & 3u;
}

// ----------------------------------------------------------------- packed reads
// base k of a read at bits [2(k mod 32), +2) of word k/32 (lasagna.h, a1).

// reverse the 32 2-bit groups of a word
__device__ __forceinline__ uint64_t rev2(uint64_t x)
{
    uint64_t y = __brevll(x);
    return ((y >> 1) & 0x5555555555555555ull) | ((y & 0x5555555555555555ull) << 1);
}

// a[] >>= bits (0 <= bits < 64W), zero fill; register-only (no dynamic indexing).
template <int W>
__device__ __forceinline__ void shr_words(uint64_t (&a)[W], uint32_t bits)
{
    uint32_t ws = bits >> 6, bs = bits & 63;
#pragma unroll
    for (int k = 0; k < W - 1; ++k) {
        if ((uint32_t)k < ws) {
#pragma unroll
            for (int j = 0; j < W; ++j) a[j] = (j + 1 < W) ? a[j + 1] : 0ull;
        }
    }
    if (ws >= (uint32_t)W) {
#pragma unroll
        for (int j = 0; j < W; ++j) a[j] = 0;
    }
    if (bs) {
#pragma unroll
        for (int j = 0; j < W; ++j) {
            uint64_t hi = (j + 1 < W) ? a[j + 1] : 0ull;
            a[j] = (a[j] >> bs) | (hi << (64 - bs));
        }
    }
}

// keep the low `bits` bits of the W-word integer a[]
template <int W>
__device__ __forceinline__ void keep_low(uint64_t (&a)[W], uint32_t bits)
{
#pragma unroll
    for (int j = 0; j < W; ++j) {
        uint32_t lo = 64u * j;
        if (bits <= lo) a[j] = 0;
        else if (bits < lo + 64) a[j] &= (1ull << (bits - lo)) - 1;
    }
}

// reverse complement of an L-base packed read (R8: complement = c ^ 2)
template <int W>
__device__ __forceinline__ void rc_words(const uint64_t (&x)[W], uint32_t L, uint64_t (&y)[W])
{
#pragma unroll
    for (int j = 0; j < W; ++j) y[W - 1 - j] = rev2(x[j]);
    shr_words<W>(y, 2u * (32u * W - L));
#pragma unroll
    for (int j = 0; j < W; ++j) y[j] ^= 0xAAAAAAAAAAAAAAAAull;
    keep_low<W>(y, 2u * L);
}

// x[w] for a runtime (block-uniform) w < W without local-memory indexing: a register select
template <int W>
__device__ __forceinline__ uint64_t wsel(const uint64_t (&x)[W], uint32_t w)
{
    uint64_t r = x[0];
#pragma unroll
    for (int j = 1; j < W; ++j)
        if (w == (uint32_t)j) r = x[j];
    return r;
}

template <int W>
__device__ __forceinline__ void load_read(const uint64_t *__restrict__ packed, uint32_t stride,
                                          uint64_t i, uint64_t (&x)[W])
{
    const uint64_t *p = packed + i * stride;
    if constexpr (W == 4) {
        ulonglong4 t = *reinterpret_cast<const ulonglong4 *>(p);
        x[0] = t.x, x[1] = t.y, x[2] = t.z, x[3] = t.w;
    } else if constexpr (W == 2) {
        ulonglong2 t = *reinterpret_cast<const ulonglong2 *>(p);
        x[0] = t.x, x[1] = t.y;
    } else {
#pragma unroll
        for (int j = 0; j < W; ++j) x[j] = p[j];
    }
}

// Exact check of the directed overlap (u, v, l): suffix_l(seq(u)) == prefix_l(seq(v))
// (R12 — every fingerprint hit is verified on the bases).
template <int W>
__device__ __forceinline__ bool verify_overlap(const uint64_t *__restrict__ packed,
                                               uint32_t stride, uint32_t L, uint32_t u,
                                               uint32_t v, uint32_t l)
{
    uint64_t x[W], su[W], y[W], sv[W];
    load_read<W>(packed, stride, u >> 1, x);
    load_read<W>(packed, stride, v >> 1, y);
    if (u & 1) rc_words<W>(x, L, su);
    else {
#pragma unroll
        for (int j = 0; j < W; ++j) su[j] = x[j];
    }
    if (v & 1) rc_words<W>(y, L, sv);
    else {
#pragma unroll
        for (int j = 0; j < W; ++j) sv[j] = y[j];
    }
    shr_words<W>(su, 2u * (L - l));
    keep_low<W>(su, 2u * l);
    keep_low<W>(sv, 2u * l);
    bool eq = true;
#pragma unroll
    for (int j = 0; j < W; ++j) eq &= (su[j] == sv[j]);
    return eq;
}

// ---- approximate mode ("128-bit fingerprints (two 64-bit values
// generated with different radixes and primes)"): a hit is accepted when the fingerprint PAIR
// of the suffix and of the prefix agree — F (radix 5 mod 2^61 - 1) and F2 (radix 7
// mod 2^64 - 59, the largest prime below 2^64; reading R22) — instead of the bases.
constexpr uint64_t Q2_64 = 0xFFFFFFFFFFFFFFC5ull; // 2^64 - 59
// P * 7 + c mod Q2_64 for P < Q2_64: 2^64 == 59 (mod Q2_64)
__device__ __forceinline__ uint64_t horner7_q2(uint64_t P, uint32_t c)
{
    const uint64_t lo = P * 7ull;
    uint64_t hi = __umul64hi(P, 7ull);
    const uint64_t t = lo + c;
    hi += t < lo;
    uint64_t u = t + hi * 59ull;
    if (u < t) u += 59ull; // wrapped past 2^64
    return u >= Q2_64 ? u - Q2_64 : u;
}

template <int W>
__device__ __forceinline__ void fp_pair(const uint64_t (&s)[W], uint32_t l, uint64_t *f1, uint64_t *f2)
{
    uint64_t a = 0, b = 0;
#pragma unroll
    for (int w = 0; w < W; ++w) {
        uint64_t x = s[w];
        const uint32_t kb = 32u * w;
        for (uint32_t j = 0; j < 32u && kb + j < l; ++j) {
            const uint32_t c = (uint32_t)(x & 3u);
            a = horner5(a, c);
            b = horner7_q2(b, c);
            x >>= 2;
        }
    }
    *f1 = exact61(a);
    *f2 = b;
}
// Approximate check of the directed overlap (u, v, l): F and F2 of suffix_l(seq(u)) equal F
// and F2 of prefix_l(seq(v)) (no base comparison).
template <int W>
__device__ __forceinline__ bool verify_fp128(const uint64_t *__restrict__ packed, uint32_t stride,
                                             uint32_t L, uint32_t u, uint32_t v, uint32_t l)
{
    uint64_t x[W], su[W], y[W], sv[W];
    load_read<W>(packed, stride, u >> 1, x);
    load_read<W>(packed, stride, v >> 1, y);
    if (u & 1) rc_words<W>(x, L, su);
    else {
#pragma unroll
        for (int j = 0; j < W; ++j) su[j] = x[j];
    }
    if (v & 1) rc_words<W>(y, L, sv);
    else {
#pragma unroll
        for (int j = 0; j < W; ++j) sv[j] = y[j];
    }
    shr_words<W>(su, 2u * (L - l));
    uint64_t a1, a2, b1, b2;
    fp_pair<W>(su, l, &a1, &a2);
    fp_pair<W>(sv, l, &b1, &b2);
    return a1 == b1 && a2 == b2;
}

__host__ __device__ inline uint32_t words_for(uint32_t L) { return (L + 31) / 32; }

__host__ __device__ inline uint32_t stride_for(uint32_t L)
{
    uint32_t w = words_for(L);
    return w <= 1 ? 1 : w <= 2 ? 2 : w <= 4 ? 4 : 8;
}

// ----------------------------------------------------------------- bulk async copies (TMA engine)
// 1-D cp.async.bulk global -> shared with an mbarrier completing on the transferred bytes
// (SASS UBLKCP): the copy engine moves the next tile while the CTA works on the current one.
__device__ __forceinline__ uint32_t smem_u32(const void *p)
{
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(unsigned long long *bar, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count)
                 : "memory");
}
__device__ __forceinline__ void fence_mbar_init()
{
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async()
{
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
// one elected thread: expect `bytes` on `bar` and start the copy
__device__ __forceinline__ void bulk_load(void *dst, const void *src, uint32_t bytes,
                                          unsigned long long *bar)
{
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
                 "r"(bytes)
                 : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, "
                 "[%3];" ::"r"(smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long *bar, uint32_t phase)
{
    asm volatile("{\n\t.reg .pred p;\n"
                 "WAIT_%=:\n\t"
                 "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
                 "@!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
                 "r"(phase)
                 : "memory");
}

// ----------------------------------------------------------------- host-side error plumbing
void set_error(const char *fmt, ...);
lasagna_status cuda_status(cudaError_t e, const char *what);
void count_launch();
uint64_t launch_count();

// Programmatic dependent launch (PDL) of back-to-back dependent kernels (the greedy's rounds):
// the next grid is scheduled while this one drains and waits in pdl_wait() until this grid's
// memory is visible, hiding the launch gap.  A kernel launched by launch_pdl MUST call
// pdl_wait() before touching anything its predecessor wrote; without PDL both are no-ops.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger()
{
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem,
                              cudaStream_t s, Args... args)
{
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
}

#define LSG_CUDA(call)                                                                         \
    do {                                                                                       \
        cudaError_t e_ = (call);                                                               \
        if (e_ != cudaSuccess) return ::lsg::cuda_status(e_, #call);                           \
    } while (0)

#define LSG_LAUNCHED(what)                                                                     \
    do {                                                                                       \
        ::lsg::count_launch();                                                                 \
        cudaError_t e_ = cudaGetLastError();                                                   \
        if (e_ != cudaSuccess) return ::lsg::cuda_status(e_, what);                            \
    } while (0)

// W dispatch: calls f(std::integral_constant<int, W>{}) for the read's word count.
template <typename F>
lasagna_status dispatch_W(uint32_t L, F &&f)
{
#ifdef LSG_DEV_ONLY_W // SASS inspection builds only: one read width
    if (words_for(L) == LSG_DEV_ONLY_W) return f(std::integral_constant<int, LSG_DEV_ONLY_W>{});
    set_error("L=%u: dev build for W=%d only", L, LSG_DEV_ONLY_W);
    return LASAGNA_EINVAL;
#endif
    switch (words_for(L)) {
    case 1: return f(std::integral_constant<int, 1>{});
    case 2: return f(std::integral_constant<int, 2>{});
    case 3: return f(std::integral_constant<int, 3>{});
    case 4: return f(std::integral_constant<int, 4>{});
    case 5: return f(std::integral_constant<int, 5>{});
    case 6: return f(std::integral_constant<int, 6>{});
    case 7: return f(std::integral_constant<int, 7>{});
    case 8: return f(std::integral_constant<int, 8>{});
    default: set_error("L=%u out of range", L); return LASAGNA_EINVAL;
    }
}

__host__ __device__ __forceinline__ uint64_t min64(uint64_t a, uint64_t b) { return a < b ? a : b; }

__host__ __device__ inline uint64_t ceil_div(uint64_t a, uint64_t b) { return (a + b - 1) / b; }

inline int num_sms()
{
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    return sms;
}

} // namespace lsg
