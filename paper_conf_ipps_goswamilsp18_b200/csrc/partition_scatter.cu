// partition_scatter.cu — level 1 fused with a1/a2: scatter_table_kernel (the bucketed fast path; overview in partition.cuh)
#include "partition.cuh"

namespace lsg {

// ------------------------------------------------------------------ level 1: fused with a2
// One thread per read, LPR lengths per partition round: the rolling streams (a2) produce the
// two canonical keys of the read (vertex 2i and 2i+1, common.cuh) for each length; a round
// ranks its 2 * LPR keys per thread by bin in shared memory (atomics: order inside a region is
// irrelevant), reserves space in the regions of its lengths with one global atomic per
// (CTA, bin), stages the keys by bin and writes them out in bin runs.  Bins are
// q * NBL + d1 (split: q * NBL + 2 d1 + flag bit) for the round's q-th length, d1 = the top 8
// bits of the mixed canonical fingerprint, which the stored key no longer carries.
template <int W, bool ASCII, bool SPLIT, int LPR, int NT = SC_THREADS, int MINB = 2>
__global__ void __launch_bounds__(NT, MINB)
scatter_table_kernel(ScatterArgs a)
{
    constexpr int NBL = SPLIT ? 512 : 256; // bins per length
    constexpr int NBIN = LPR * NBL;
    constexpr int BPT = NBIN / NT; // bins per thread in the round's scan
    constexpr int KPT = 2 * LPR;           // keys per thread per round
    static_assert(NBIN % NT == 0 && BPT >= 1 && BPT <= 4, "bins per thread");
    // dynamic: stage[NT * KPT] keys, sbin[NT * KPT] their bins, then (ASCII)
    // the CTA's staged read bytes
    extern __shared__ __align__(16) uint64_t stage[];
    unsigned short *sbin = reinterpret_cast<unsigned short *>(stage + NT * KPT);
    __shared__ uint32_t cnt[NBIN], lstart[NBIN + 1], wsum[16];
    __shared__ uint32_t rbase[SPLIT ? 1 : 256]; // region of (segment 0, digit d); + s * nb_pad
    __shared__ long long gofs[NBIN]; // per bin: element offset of stage slot 0's destination, -1 = overflow

    __shared__ unsigned short s_b5f[256], s_b5b[256]; // base-5 byte tables (fingerprint.cuh)
    for (uint32_t t = threadIdx.x; t < 256; t += NT) {
        s_b5f[t] = (unsigned short)base5_fwd(t);
        s_b5b[t] = (unsigned short)base5_bwd(t);
    }
    // (visible to the prologue: the barriers below precede fp64_absorb)
    const uint64_t i = (uint64_t)blockIdx.x * NT + threadIdx.x;
    const bool valid = i < a.n;
    uint64_t x[W], y[W];
    if constexpr (ASCII) {
        // a1 fused: stage this CTA's ASCII span (zero-copy from host memory over PCIe when
        // the caller passed page-locked host memory), pack, validate, keep the packed rows
        unsigned char *sascii = reinterpret_cast<unsigned char *>(sbin + NT * KPT);
        const uint64_t r0 = (uint64_t)blockIdx.x * NT;
        const uint64_t r1 = min64(a.n, r0 + NT);
        const uint32_t off = stage_ascii(a.ascii, r0 * a.L, r1 * a.L, sascii, NT);
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
    for (uint32_t t = threadIdx.x; t < NBIN; t += NT) cnt[t] = 0;
    if (!SPLIT)
        for (uint32_t d = threadIdx.x; d < 256; d += NT)
            rbase[d] = (uint32_t)(shard_region(0, a.l_hi - a.l_lo + 1u, d, a.dest_g, a.nb_pad) -
                                  (a.keep_owner < 0 ? 0ull
                                                    : (uint64_t)a.keep_owner *
                                                          (a.l_hi - a.l_lo + 1u) * a.nb_pad));
    __syncthreads();
    const uint32_t v0 = (uint32_t)(2 * (a.read_offset + i)); // V < 2^32
    const uint64_t fl1 = 1ull << a.vbits, fl2 = 2ull << a.vbits;
#ifdef LSG_CHECKS
    // regions this call may fill: [G][512] split, else the shard layout (a sub-pass: one range)
    const uint64_t nreg = SPLIT ? (uint64_t)(a.l_hi - a.l_lo + 1u) * 512u
                                : (uint64_t)(a.l_hi - a.l_lo + 1u) * a.nb_pad *
                                      (a.keep_owner >= 0 ? 1u : a.dest_g);
    LSG_DCHECK(v0 / 2u < a.read_offset + a.n || !valid);
#endif
    Fp64Streams st; // key streams modulo 2^64 (R26)
    // the l_lo - 1 bases before the first emitted length, absorbed in 8-base chunks
    fp64_absorb<W>(x, y, a.l_lo - 1u, st, Base5Tabs{s_b5f, s_b5b});
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
                const uint64_t e0 = canon_key64_d1(st.P0, st.S1, a.keep, fl1, fl2, v0, &d0);
                const uint64_t e1 = canon_key64_d1(st.P1, st.S0, a.keep, fl1, fl2, v0 + 1u, &d1);
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
                LSG_DCHECK(!(c[b] && q < kc) || rg[b] < nreg);
                bs[b] = (c[b] && q < kc) ? atomicAdd(&a.fill[rg[b]], c[b]) : 0u;
                sum += c[b];
            }
            uint32_t run = block_scan<NT>(sum, wsum);
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
            if (threadIdx.x == NT - 1) lstart[NBIN] = run;
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
            for (uint32_t u = threadIdx.x; u < total; u += NT) {
                const long long go = gofs[sbin[u]];
                LSG_DCHECK(go < 0 || (uint64_t)(go + u) < nreg * a.cap);
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
        const size_t ascii_row = args.ascii ? (size_t)args.L : 0;
        auto run = [&](auto kern, int lpr, int nt) -> lasagna_status {
            const unsigned blocks = (unsigned)ceil_div(args.n, (uint64_t)nt);
            const size_t smem = (size_t)nt * 2 * lpr * (8 + 2) +
                                (args.ascii ? (size_t)nt * ascii_row + 32 : 0); // + SWAR overread
            LSG_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                          (int)smem));
            kern<<<blocks, nt, smem, s>>>(args);
            LSG_LAUNCHED("scatter_table_kernel");
            return LASAGNA_OK;
        };
        if (args.split)
            return args.ascii ? run(scatter_table_kernel<W, true, true, 1>, 1, SC_THREADS)
                              : run(scatter_table_kernel<W, false, true, 1>, 1, SC_THREADS);
        // CTA geometry: 512 reads x 2 CTAs per SM at the 64-register cap; 256 x 3 (80 registers)
        // and 512 x 1 (128 registers) measured 20-25 % slower (r02e)
        return args.ascii ? run(scatter_table_kernel<W, true, false, 4>, 4, SC_THREADS)
                          : run(scatter_table_kernel<W, false, false, 4>, 4, SC_THREADS);
    });
}

} // namespace lsg
