// fingerprint.cuh — the rolling Rabin-Karp streams of a2 (Fig. 5/6), shared by
// the table kernels (fingerprint.cu, partition_scatter.cu).
#pragma once

#include "kernels.cuh"

namespace lsg {

// Place values M[j] = 5^j mod q and 2 M[j] mod q ("computed once for the entire
// program"), j < 256, built at compile time into constant memory: every lane of a warp reads
// the same j in the same step, so the constant cache broadcasts them.
struct PowTable {
    uint64_t m[256], m2[256];
};
constexpr uint64_t host_fold_exact(uint64_t x)
{
    uint64_t r = (x & Q61) + (x >> 61);
    return r >= Q61 ? r - Q61 : r;
}
constexpr PowTable make_pow_table()
{
    PowTable t{};
    uint64_t p = 1;
    for (int j = 0; j < 256; ++j) {
        t.m[j] = p;
        t.m2[j] = host_fold_exact(p << 1);
        p = host_fold_exact((p << 2) + p);
    }
    return t;
}
static __constant__ PowTable c_pow = make_pow_table(); // one copy per translation unit

struct FpStreams {
    uint64_t P0, P1, S0, S1; // folded (congruent mod q, < 2^61 + 7)
    __device__ __forceinline__ void init() { P0 = P1 = S0 = S1 = 0; }
    // consume base j of r (ca) and of r' (cb)
    __device__ __forceinline__ void step(uint32_t ca, uint32_t cb, uint32_t j)
    {
        const uint64_t pw = c_pow.m[j], pw2 = c_pow.m2[j];
        P0 = horner5(P0, ca);
        P1 = horner5(P1, cb);
        S1 = addpow(S1, ca ^ 2u, pw, pw2);
        S0 = addpow(S0, cb ^ 2u, pw, pw2);
    }
};

// ---- the bucketed path's table keys: the same radix-5 Rabin-Karp polynomial evaluated modulo
// 2^64 (reading R26).  The keys only have to bring equal strings together — every hit is
// verified on the bases (R12) — and modulo 2^64 a step is two multiply-adds on the FMA pipe
// instead of the shifts, folds and exact reductions of mod 2^61 - 1 on the integer ALU pipe,
// which bounds the scatter kernel (ncu: ALU pipe 67 % of peak, FMA 17 %).
struct Pow64Table {
    uint64_t m[256];
};
constexpr Pow64Table make_pow64_table()
{
    Pow64Table t{};
    uint64_t p = 1;
    for (int j = 0; j < 256; ++j) {
        t.m[j] = p;
        p *= 5u;
    }
    return t;
}
static __constant__ Pow64Table c_pow64 = make_pow64_table();

struct Fp64Streams {
    uint64_t P0, P1, S0, S1; // exact values mod 2^64
    __device__ __forceinline__ void step(uint32_t ca, uint32_t cb, uint32_t j)
    {
        const uint64_t pw = c_pow64.m[j];
        P0 = P0 * 5u + ca;
        P1 = P1 * 5u + cb;
        S1 += (uint64_t)(ca ^ 2u) * pw;
        S0 += (uint64_t)(cb ^ 2u) * pw;
    }
};

// ---- absorbing a read's leading bases without per-base modular steps
// Lengths below the first one a kernel emits need no intermediate values, only the stream
// states after them, so whole 16-base half-words are absorbed in 8-base chunks: the chunk's
// Horner value (< 5^8 < 2^19) takes one 32-bit multiply-add per base, and the stream advances
// by one modular multiplication per chunk: P <- P * 5^8 + V (prefix streams, bases in read
// order) and S <- S * 5^8 + V (ascending-power streams, evaluated by Horner from the highest
// base down: sum_{j<m} c_j 5^j = (...(c_{m-1} 5 + c_{m-2}) 5 + ...) 5 + c_0).

// P * m mod q for P < 2^62 and m < 2^32, folded (< 2^61 + 8): P m = hi 2^32 + lo with
// hi 2^32 = (hi >> 29) 2^61 + (hi mod 2^29) 2^32 == (hi >> 29) + (hi mod 2^29) 2^32.
__device__ __forceinline__ uint64_t mulsmall61(uint64_t P, uint32_t m)
{
    const uint64_t lo = (uint64_t)(uint32_t)P * m;
    const uint64_t hi = (uint64_t)(uint32_t)(P >> 32) * m;
    return fold61(fold61(lo) + ((hi & 0x1FFFFFFFull) << 32) + (hi >> 29));
}
constexpr uint32_t POW5_8 = 390625u;
// Horner value of the 8 bases in the low 16 bits of h: base 0 (lowest bits) most significant
__device__ __forceinline__ uint32_t chunk8_fwd(uint32_t h)
{
    uint32_t v = 0;
#pragma unroll
    for (int t = 0; t < 8; ++t) v = v * 5u + ((h >> (2 * t)) & 3u);
    return v;
}
// ... base 7 (highest bits) most significant
__device__ __forceinline__ uint32_t chunk8_bwd(uint32_t h)
{
    uint32_t v = 0;
#pragma unroll
    for (int t = 7; t >= 0; --t) v = v * 5u + ((h >> (2 * t)) & 3u);
    return v;
}

// Stream states after the first 16 * nh bases of r (x) and r' (y), nh <= 2W (block-uniform).
template <int W>
__device__ __forceinline__ void fp_skip(const uint64_t (&x)[W], const uint64_t (&y)[W], uint32_t nh,
                                        FpStreams &st)
{
    uint64_t P0 = 0, P1 = 0, S0 = 0, S1 = 0;
#pragma unroll
    for (int h = 0; h < 2 * W; ++h) {
        if ((uint32_t)h >= nh) break;
        const uint32_t hx = (uint32_t)(x[h >> 1] >> (32 * (h & 1)));
        const uint32_t hy = (uint32_t)(y[h >> 1] >> (32 * (h & 1)));
        P0 = mulsmall61(P0, POW5_8) + chunk8_fwd(hx);
        P0 = mulsmall61(P0, POW5_8) + chunk8_fwd(hx >> 16);
        P1 = mulsmall61(P1, POW5_8) + chunk8_fwd(hy);
        P1 = mulsmall61(P1, POW5_8) + chunk8_fwd(hy >> 16);
    }
#pragma unroll
    for (int h = 2 * W - 1; h >= 0; --h) {
        if ((uint32_t)h >= nh) continue;
        // ascending-power streams consume the complemented bases (c ^ 2)
        const uint32_t hx = (uint32_t)(x[h >> 1] >> (32 * (h & 1))) ^ 0xAAAAAAAAu;
        const uint32_t hy = (uint32_t)(y[h >> 1] >> (32 * (h & 1))) ^ 0xAAAAAAAAu;
        S1 = mulsmall61(S1, POW5_8) + chunk8_bwd(hx >> 16);
        S1 = mulsmall61(S1, POW5_8) + chunk8_bwd(hx);
        S0 = mulsmall61(S0, POW5_8) + chunk8_bwd(hy >> 16);
        S0 = mulsmall61(S0, POW5_8) + chunk8_bwd(hy);
    }
    st.P0 = fold61(P0), st.P1 = fold61(P1), st.S0 = fold61(S0), st.S1 = fold61(S1);
}

// Stream states after exactly the first nb bases of r (x) and r' (y), any nb <= 32 W
// (block-uniform): whole 16-base half-words as in fp_skip, then the remaining nb mod 16 bases
// as one or two chunks of k <= 8 bases.  A forward chunk of k bases is chunk8_fwd of its
// bases moved to the top k positions (P <- P 5^k + value); the ascending-power streams
// evaluate their polynomial from the highest base down, so the partial chunk comes first.
__device__ __forceinline__ uint32_t pow5_small(uint32_t k)
{
    uint32_t p = 1;
    for (uint32_t t = 0; t < k; ++t) p *= 5u;
    return p;
}
template <int W>
__device__ __forceinline__ void fp_absorb(const uint64_t (&x)[W], const uint64_t (&y)[W],
                                          uint32_t nb, FpStreams &st)
{
    const uint32_t nh = nb >> 4, rem = nb & 15u;
    uint64_t P0 = 0, P1 = 0, S0 = 0, S1 = 0;
#pragma unroll
    for (int h = 0; h < 2 * W; ++h) {
        if ((uint32_t)h >= nh) break;
        const uint32_t hx = (uint32_t)(x[h >> 1] >> (32 * (h & 1)));
        const uint32_t hy = (uint32_t)(y[h >> 1] >> (32 * (h & 1)));
        P0 = mulsmall61(P0, POW5_8) + chunk8_fwd(hx);
        P0 = mulsmall61(P0, POW5_8) + chunk8_fwd(hx >> 16);
        P1 = mulsmall61(P1, POW5_8) + chunk8_fwd(hy);
        P1 = mulsmall61(P1, POW5_8) + chunk8_fwd(hy >> 16);
    }
    // the partial half-word nh (bases 16 nh .. 16 nh + rem - 1), rem < 16
    uint32_t px = 0, py = 0;
    if (rem) {
        px = (uint32_t)(wsel<W>(x, nh >> 1) >> (32 * (nh & 1)));
        py = (uint32_t)(wsel<W>(y, nh >> 1) >> (32 * (nh & 1)));
        const uint32_t mask = rem == 16 ? 0xFFFFFFFFu : ((1u << (2 * rem)) - 1u);
        px &= mask;
        py &= mask;
        const uint32_t k1 = min(rem, 8u), k2 = rem - k1; // forward: low chunk first
        const uint32_t m1 = pow5_small(k1);
        P0 = mulsmall61(P0, m1) + chunk8_fwd((px & 0xFFFFu) << (2 * (8 - k1)));
        P1 = mulsmall61(P1, m1) + chunk8_fwd((py & 0xFFFFu) << (2 * (8 - k1)));
        if (k2) {
            const uint32_t m2 = pow5_small(k2);
            P0 = mulsmall61(P0, m2) + chunk8_fwd(((px >> 16) << (2 * (8 - k2))) & 0xFFFFu);
            P1 = mulsmall61(P1, m2) + chunk8_fwd(((py >> 16) << (2 * (8 - k2))) & 0xFFFFu);
        }
        // ascending-power streams: the partial (highest) bases first, high chunk first
        const uint32_t cx = px ^ (0xAAAAAAAAu & mask), cy = py ^ (0xAAAAAAAAu & mask);
        if (k2) {
            S1 = chunk8_bwd(cx >> 16);
            S0 = chunk8_bwd(cy >> 16);
            S1 = mulsmall61(S1, m1) + chunk8_bwd(cx & 0xFFFFu);
            S0 = mulsmall61(S0, m1) + chunk8_bwd(cy & 0xFFFFu);
        } else {
            S1 = chunk8_bwd(cx & 0xFFFFu);
            S0 = chunk8_bwd(cy & 0xFFFFu);
        }
    }
#pragma unroll
    for (int h = 2 * W - 1; h >= 0; --h) {
        if ((uint32_t)h >= nh) continue;
        const uint32_t hx = (uint32_t)(x[h >> 1] >> (32 * (h & 1))) ^ 0xAAAAAAAAu;
        const uint32_t hy = (uint32_t)(y[h >> 1] >> (32 * (h & 1))) ^ 0xAAAAAAAAu;
        S1 = mulsmall61(S1, POW5_8) + chunk8_bwd(hx >> 16);
        S1 = mulsmall61(S1, POW5_8) + chunk8_bwd(hx);
        S0 = mulsmall61(S0, POW5_8) + chunk8_bwd(hy >> 16);
        S0 = mulsmall61(S0, POW5_8) + chunk8_bwd(hy);
    }
    st.P0 = fold61(P0), st.P1 = fold61(P1), st.S0 = fold61(S0), st.S1 = fold61(S1);
}

// Table-driven chunk values: the four 2-bit codes of a byte (code i at bits 2i..2i+1) as a
// base-5 number, code 0 most significant (forward Horner) or least significant (ascending
// powers).  A kernel fills the 256-entry tables into shared memory once (Base5Tabs); an
// 8-base chunk is then two byte extracts, two lookups and one multiply-add instead of eight
// shift/mask/multiply-add steps.
__host__ __device__ constexpr uint32_t base5_fwd(uint32_t b)
{
    return (b & 3u) * 125u + ((b >> 2) & 3u) * 25u + ((b >> 4) & 3u) * 5u + ((b >> 6) & 3u);
}
__host__ __device__ constexpr uint32_t base5_bwd(uint32_t b)
{
    return (b & 3u) + ((b >> 2) & 3u) * 5u + ((b >> 4) & 3u) * 25u + ((b >> 6) & 3u) * 125u;
}
struct Base5Tabs {
    const unsigned short *fwd, *bwd; // shared memory, 256 entries each
};
__device__ __forceinline__ uint32_t byte_k(uint32_t h, uint32_t k) // byte k of h, zero-extended
{
    return __byte_perm(h, 0u, 0x4440u + k);
}
// chunk8_fwd / chunk8_bwd of the 8 bases in bytes k, k+1 of h (k = 0: low half, 2: high half)
__device__ __forceinline__ uint32_t chunk8_fwd_t(const Base5Tabs &t, uint32_t h, uint32_t k)
{
    return (uint32_t)t.fwd[byte_k(h, k)] * 625u + t.fwd[byte_k(h, k + 1u)];
}
__device__ __forceinline__ uint32_t chunk8_bwd_t(const Base5Tabs &t, uint32_t h, uint32_t k)
{
    return (uint32_t)t.bwd[byte_k(h, k + 1u)] * 625u + t.bwd[byte_k(h, k)];
}

// fp_absorb modulo 2^64 (the key streams of the bucketed path, R26)
template <int W>
__device__ __forceinline__ void fp64_absorb(const uint64_t (&x)[W], const uint64_t (&y)[W],
                                          uint32_t nb, Fp64Streams &st, const Base5Tabs &tb)
{
    const uint32_t nh = nb >> 4, rem = nb & 15u;
    uint64_t P0 = 0, P1 = 0, S0 = 0, S1 = 0;
#pragma unroll
    for (int h = 0; h < 2 * W; ++h) {
        if ((uint32_t)h >= nh) break;
        const uint32_t hx = (uint32_t)(x[h >> 1] >> (32 * (h & 1)));
        const uint32_t hy = (uint32_t)(y[h >> 1] >> (32 * (h & 1)));
        P0 = (P0) * (uint64_t)(POW5_8) + chunk8_fwd_t(tb, hx, 0);
        P0 = (P0) * (uint64_t)(POW5_8) + chunk8_fwd_t(tb, hx, 2);
        P1 = (P1) * (uint64_t)(POW5_8) + chunk8_fwd_t(tb, hy, 0);
        P1 = (P1) * (uint64_t)(POW5_8) + chunk8_fwd_t(tb, hy, 2);
    }
    // the partial half-word nh (bases 16 nh .. 16 nh + rem - 1), rem < 16
    uint32_t px = 0, py = 0;
    if (rem) {
        px = (uint32_t)(wsel<W>(x, nh >> 1) >> (32 * (nh & 1)));
        py = (uint32_t)(wsel<W>(y, nh >> 1) >> (32 * (nh & 1)));
        const uint32_t mask = rem == 16 ? 0xFFFFFFFFu : ((1u << (2 * rem)) - 1u);
        px &= mask;
        py &= mask;
        const uint32_t k1 = min(rem, 8u), k2 = rem - k1; // forward: low chunk first
        const uint32_t m1 = pow5_small(k1);
        P0 = (P0) * (uint64_t)(m1) + chunk8_fwd((px & 0xFFFFu) << (2 * (8 - k1)));
        P1 = (P1) * (uint64_t)(m1) + chunk8_fwd((py & 0xFFFFu) << (2 * (8 - k1)));
        if (k2) {
            const uint32_t m2 = pow5_small(k2);
            P0 = (P0) * (uint64_t)(m2) + chunk8_fwd(((px >> 16) << (2 * (8 - k2))) & 0xFFFFu);
            P1 = (P1) * (uint64_t)(m2) + chunk8_fwd(((py >> 16) << (2 * (8 - k2))) & 0xFFFFu);
        }
        // ascending-power streams: the partial (highest) bases first, high chunk first
        const uint32_t cx = px ^ (0xAAAAAAAAu & mask), cy = py ^ (0xAAAAAAAAu & mask);
        if (k2) {
            S1 = chunk8_bwd(cx >> 16);
            S0 = chunk8_bwd(cy >> 16);
            S1 = (S1) * (uint64_t)(m1) + chunk8_bwd(cx & 0xFFFFu);
            S0 = (S0) * (uint64_t)(m1) + chunk8_bwd(cy & 0xFFFFu);
        } else {
            S1 = chunk8_bwd(cx & 0xFFFFu);
            S0 = chunk8_bwd(cy & 0xFFFFu);
        }
    }
#pragma unroll
    for (int h = 2 * W - 1; h >= 0; --h) {
        if ((uint32_t)h >= nh) continue;
        const uint32_t hx = (uint32_t)(x[h >> 1] >> (32 * (h & 1))) ^ 0xAAAAAAAAu;
        const uint32_t hy = (uint32_t)(y[h >> 1] >> (32 * (h & 1))) ^ 0xAAAAAAAAu;
        S1 = (S1) * (uint64_t)(POW5_8) + chunk8_bwd_t(tb, hx, 2);
        S1 = (S1) * (uint64_t)(POW5_8) + chunk8_bwd_t(tb, hx, 0);
        S0 = (S0) * (uint64_t)(POW5_8) + chunk8_bwd_t(tb, hy, 2);
        S0 = (S0) * (uint64_t)(POW5_8) + chunk8_bwd_t(tb, hy, 0);
    }
    st.P0 = P0, st.P1 = P1, st.S0 = S0, st.S1 = S1;
}

// half-words a kernel whose first emitted length is l_first can absorb (bases < l_first - 1)
__host__ __device__ __forceinline__ uint32_t skip_halves(uint32_t l_first)
{
    return l_first > 1 ? (l_first - 1) / 16 : 0;
}

// Visit lengths l = l_first..l_end; call emit(l, st) after base l-1 (values folded: use
// exact61).  The bases before the first 16-base boundary <= l_first - 1 are absorbed by fp_skip.
template <int W, typename Emit>
__device__ __forceinline__ void roll_read(const uint64_t (&x)[W], const uint64_t (&y)[W],
                                          uint32_t l_first, uint32_t l_end, Emit &&emit)
{
    FpStreams st;
    const uint32_t nh = min(skip_halves(l_first), 2u * W);
    fp_skip<W>(x, y, nh, st);
    const uint32_t kskip = 16u * nh;
#pragma unroll
    for (int w = 0; w < W; ++w) {
        const uint32_t k0 = 32u * w;
        if (k0 >= l_end) break;
        if (k0 + 32u <= kskip) continue;
        const uint32_t j0 = kskip > k0 ? kskip - k0 : 0u; // 0 or 16
        uint64_t a = x[w] >> (2 * j0), b = y[w] >> (2 * j0);
        const uint32_t kn = min(32u, l_end - k0);
        for (uint32_t j = j0; j < kn; ++j) {
            st.step((uint32_t)(a & 3u), (uint32_t)(b & 3u), k0 + j);
            a >>= 2;
            b >>= 2;
            if (k0 + j + 1 >= l_first) emit(k0 + j + 1, st);
        }
    }
}

} // namespace lsg
