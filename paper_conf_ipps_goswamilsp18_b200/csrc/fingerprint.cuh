// fingerprint.cuh — the rolling Rabin-Karp streams of a2 (Fig. 5/6), shared by
// the table kernels (fingerprint.cu, partition.cu).
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

// Visit lengths l = 1..l_end; call emit(l, st) after base l-1 (values folded: use exact61).
template <int W, typename Emit>
__device__ __forceinline__ void roll_read(const uint64_t (&x)[W], const uint64_t (&y)[W],
                                          uint32_t l_end, Emit &&emit)
{
    FpStreams st;
    st.init();
#pragma unroll
    for (int w = 0; w < W; ++w) {
        uint64_t a = x[w], b = y[w];
        const uint32_t k0 = 32u * w;
        if (k0 >= l_end) break;
        const uint32_t kn = min(32u, l_end - k0);
        for (uint32_t j = 0; j < kn; ++j) {
            st.step((uint32_t)(a & 3u), (uint32_t)(b & 3u), k0 + j);
            a >>= 2;
            b >>= 2;
            emit(k0 + j + 1, st);
        }
    }
}

} // namespace lsg
