// partition_refine.cu — level k -> k+1: refine_kernel (the bucketed fast path; overview in partition.cuh)
#include "partition.cuh"

namespace lsg {

// ------------------------------------------------------------------ level k -> k+1
// One CTA owns one region and streams it: the bulk-copy engine prefetches tile t+1 into the
// other half of a double buffer while tile t is ranked (shared atomics: order inside a
// sub-region is irrelevant), staged by digit and written out in digit runs.
template <bool SPLIT, int RF_KPT>
__global__ void __launch_bounds__(RF_THREADS, RF_KPT == 16 ? 1 : 2)
refine_kernel(RefineArgs a)
{
    constexpr int RF_TILE = RF_THREADS * RF_KPT;
    constexpr int NBMAX = 512; // 2^dbits bins (x 2 when split), dbits <= 8
    extern __shared__ __align__(128) uint64_t rsm[];
    uint64_t *inb = rsm;                 // [2][RF_TILE]
    uint64_t *rstage = rsm + 2 * RF_TILE; // [RF_TILE]
    __shared__ __align__(8) unsigned long long mbar[2];
    __shared__ uint32_t cnt[NBMAX], lstart[NBMAX], running[NBMAX], wsum[16];
    __shared__ uint64_t *gdst[NBMAX]; // per bin: a.out + offset - first stage slot; nullptr = overflow
    const uint32_t nb = (1u << a.dbits) << (SPLIT ? 1 : 0);
    const uint32_t dmask = (1u << a.dbits) - 1u;
    auto binof = [&](uint64_t k) -> uint32_t {
        const uint32_t d = (uint32_t)(k >> a.dshift) & dmask;
        if constexpr (SPLIT) return (d << 1) | (uint32_t)((k >> a.vbits) & 1);
        else return d;
    };
    const uint64_t r = blockIdx.x;
    // the region's entries: n_src source segments (multi-GPU: one per sending rank), region
    // k * src_stride + r of `in`, streamed as one sequence of tiles
    __shared__ uint32_t stile[MAX_REFINE_SRC + 1];
    __shared__ uint64_t scount[MAX_REFINE_SRC];
    if (threadIdx.x == 0) {
        uint32_t acc = 0;
        for (uint32_t k = 0; k < a.n_src; ++k) {
            const uint32_t f = a.fill_in[k * a.src_stride + r];
            if (f > a.cap_in) *a.overflow = 1u;
            // an overflowed region dropped whole bin runs (unwritten slots below cap): move
            // nothing from it (the overflow flag makes the caller redo the call)
            scount[k] = f > a.cap_in ? 0u : f;
            stile[k] = acc;
            acc += (uint32_t)ceil_div(scount[k], RF_TILE);
        }
        stile[a.n_src] = acc;
    }
    if (threadIdx.x < NBMAX) cnt[threadIdx.x] = 0, running[threadIdx.x] = 0;
    if (threadIdx.x == 0) {
        mbar_init(&mbar[0], 1);
        mbar_init(&mbar[1], 1);
        fence_mbar_init();
    }
    __syncthreads();
    const uint32_t ntiles = stile[a.n_src];
    // source segment of tile t, and its first entry / length inside that segment
    auto tile_src = [&](uint32_t t, const uint64_t **p, uint32_t *m) {
        uint32_t k = 0;
        while (t >= stile[k + 1]) ++k;
        const uint64_t t0 = (uint64_t)(t - stile[k]) * RF_TILE;
        *p = a.in + ((uint64_t)k * a.src_stride + r) * a.cap_in + t0;
        *m = (uint32_t)min64(RF_TILE, scount[k] - t0);
    };
    // bytes of a tile of m entries (rounded up to 16: the region capacity is even, so the
    // rounding stays inside the region)
    auto tile_bytes = [](uint32_t m) { return (uint32_t)((((uint64_t)m * 8) + 15) & ~15ull); };
    if (threadIdx.x == 0 && ntiles) {
        const uint64_t *p;
        uint32_t m;
        tile_src(0, &p, &m);
        bulk_load(inb, p, tile_bytes(m), &mbar[0]);
    }
    for (uint32_t t = 0; t < ntiles; ++t) {
        const uint32_t bsel = t & 1;
        const uint64_t *pcur;
        uint32_t m;
        tile_src(t, &pcur, &m);
        if (threadIdx.x == 0 && t + 1 < ntiles) {
            const uint64_t *p;
            uint32_t mn;
            tile_src(t + 1, &p, &mn);
            fence_proxy_async();
            bulk_load(inb + (bsel ^ 1) * RF_TILE, p, tile_bytes(mn), &mbar[bsel ^ 1]);
        }
        mbar_wait(&mbar[bsel], (t >> 1) & 1);
        const uint64_t *tin = inb + bsel * RF_TILE;
        uint32_t rk[RF_KPT];
#pragma unroll
        for (int q = 0; q < RF_KPT; ++q) {
            const uint32_t idx = q * RF_THREADS + threadIdx.x;
            if (idx < m) rk[q] = atomicAdd(&cnt[binof(tin[idx])], 1u);
        }
        __syncthreads();
        uint32_t c = 0;
        if (threadIdx.x < nb) {
            c = cnt[threadIdx.x];
            cnt[threadIdx.x] = 0;
        }
        const uint32_t ex = block_scan<RF_THREADS>(c, wsum);
        if (threadIdx.x < nb) {
            lstart[threadIdx.x] = ex;
            const uint32_t run = running[threadIdx.x];
            running[threadIdx.x] = run + c; // this thread's bin only: no barrier needed
            if ((uint64_t)run + c > a.cap_out) {
                gdst[threadIdx.x] = nullptr;
                *a.overflow = 1u;
            } else {
                gdst[threadIdx.x] = a.out + ((r * nb + threadIdx.x) * a.cap_out + run) - ex;
            }
        }
        __syncthreads();
#pragma unroll
        for (int q = 0; q < RF_KPT; ++q) {
            const uint32_t idx = q * RF_THREADS + threadIdx.x;
            if (idx < m) {
                const uint64_t k = tin[idx];
                rstage[lstart[binof(k)] + rk[q]] = k;
            }
        }
        __syncthreads();
#pragma unroll 4
        for (uint32_t u = threadIdx.x; u < m; u += RF_THREADS) {
            const uint64_t k = rstage[u];
            uint64_t *d = gdst[binof(k)];
            LSG_DCHECK(!d || (uint64_t)(d + u - a.out) < (uint64_t)gridDim.x * nb * a.cap_out);
            if (d) __stcg(d + u, k);
        }
        // no barrier here: the next tile's first barrier (after its ranking, which touches only
        // cnt and the other input buffer) orders these reads of rstage/gdst before they are
        // rewritten, and this tile's buffer was last read before the staging barrier above
    }
    if (threadIdx.x < nb) {
        a.fill_out[r * nb + threadIdx.x] = running[threadIdx.x];
        if (running[threadIdx.x] > a.cap_out) *a.overflow = 1u;
    }
}

lasagna_status launch_refine(const RefineArgs &args, uint64_t n_regions, cudaStream_t s)
{
    if (n_regions == 0) return LASAGNA_OK;
    if (args.dbits < 1 || args.dbits > 8) return LASAGNA_EINVAL;
    if (args.n_src < 1 || args.n_src > MAX_REFINE_SRC) return LASAGNA_EINVAL;
    // tile of 16 keys per thread, one 512-thread CTA per SM (8-key tiles at two CTAs per SM
    // measured 15.0 vs 11.0 ms at cfg3: DESIGN.md 6.1, r02g)
    constexpr int kpt = 16;
    const size_t smem = (size_t)3 * RF_THREADS * kpt * 8;
    auto kern = args.split ? refine_kernel<true, kpt> : refine_kernel<false, kpt>;
    LSG_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    kern<<<(unsigned)n_regions, RF_THREADS, smem, s>>>(args);
    LSG_LAUNCHED("refine_kernel");
    return LASAGNA_OK;
}

} // namespace lsg
