// compress.cu — the Compress phase (PAPER §III-D, Fig. 7):
// traverse the greedy string graph into paths and spell one contig per path.
//
// Paper: "Traversal begins with vertices with in-degree 0 and out-degree 1 as seeds ... from
// each seed, we continue to extend the path by appending the read-ID and overhang-length of
// the current vertex ... and stop after we encounter a vertex with no outgoing edge";
// the overhang of a read with an out-edge of length o is L - o, of a read without one L
// (P:L178); contigs are laid out by an exclusive scan of the path sizes and of the overhangs
// (Fig. 7), and each read places its first overhang bases at its offset
// (P:L190).  The paper walks the paths with host threads (the graph lives in host memory);
// here the graph is in HBM and the walk becomes GPU list ranking:
//
//   cp_init     pred(v) = succ[v^1]^1 (the complementary edge of u -> v is v^1 -> u^1, so
//               v's in-edge comes from succ[v^1]^1); ptr = pred (a seed points at itself),
//               val = overhang of pred
//   cp_jump     pointer jumping (Wyllie), double-buffered: val[v] += val[ptr[v]],
//               ptr[v] = ptr[ptr[v]] until every pointer rests on a vertex that points at
//               itself; then val[v] = the offset of v in its contig, ptr[v] = its seed.
//               Vertices on cycles (no seed: in-degree 1 everywhere) never reach a vertex
//               without predecessor; they are in no path (R21) and the round cap stops them.
//   cp_tails    a tail t (no out-edge, an in-edge) closes the path of seed r = ptr[t]:
//               length val[t] + L.  Each path has a complementary path (seed t^1, tail
//               r^1) spelling the reverse complement; the one with the smaller seed is kept
//               (R20).
//   scans       exclusive scans of the kept paths' lengths (contig offsets) and flags
//               (contig index), Fig. 7's two scans
//   cp_place    every vertex on a kept path writes seq(v)[0 .. overhang(v)) at
//               contig offset + val[v]
#include "kernels.cuh"

namespace lsg {

constexpr int CP_THREADS = 256;
constexpr int SC_T = 1024; // scan block
constexpr int SC_IPT = 8;  // items per scan thread
constexpr int SC_TILE = SC_T * SC_IPT;

__device__ __forceinline__ uint32_t cp_pred(const uint32_t *succ, uint32_t v)
{
    const uint32_t s = succ[v ^ 1u];
    return s == NONE ? NONE : s ^ 1u;
}

__global__ void cp_init(const uint32_t *__restrict__ succ, const uint8_t *__restrict__ olen,
                        uint64_t V, uint32_t L, uint32_t *ptr, unsigned long long *val)
{
    for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < V;
         v += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t p = cp_pred(succ, (uint32_t)v);
        ptr[v] = p == NONE ? (uint32_t)v : p;
        val[v] = p == NONE ? 0ull : (unsigned long long)(L - olen[p]);
    }
}

// one synchronous jumping round; *open counts pointers not yet at a self-pointing vertex
__global__ void cp_jump(uint64_t V, const uint32_t *__restrict__ ptr,
                        const unsigned long long *__restrict__ val, uint32_t *__restrict__ nptr,
                        unsigned long long *__restrict__ nval, unsigned long long *open)
{
    uint32_t o = 0;
    for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < V;
         v += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t p = ptr[v];
        const uint32_t pp = ptr[p];
        nptr[v] = pp;
        nval[v] = p == (uint32_t)v ? val[v] : val[v] + val[p];
        o += ptr[pp] != pp;
    }
    for (int k = 16; k; k >>= 1) o += __shfl_xor_sync(0xffffffffu, o, k);
    if ((threadIdx.x & 31) == 0 && o) atomicAdd(open, (unsigned long long)o);
}

// tails close paths: len[r] = contig length of the kept path of seed r, keep[r] = 1
__global__ void cp_tails(const uint32_t *__restrict__ succ, uint64_t V, uint32_t L,
                         const uint32_t *__restrict__ ptr, const unsigned long long *__restrict__ val,
                         unsigned long long *len, uint32_t *keep)
{
    for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < V;
         t += (uint64_t)gridDim.x * blockDim.x) {
        if (succ[t] != NONE || cp_pred(succ, (uint32_t)t) == NONE) continue;
        const uint32_t r = ptr[t];
        if (cp_pred(succ, r) != NONE) continue; // not converged: cannot happen on a path
        if (r < ((uint32_t)t ^ 1u)) {           // R20: keep the path with the smaller seed
            len[r] = val[t] + L;
            keep[r] = 1u;
        }
    }
}

// ---- exclusive scan in place (three phases: tile sums, scan of the sums, tiles)
template <typename T>
__device__ __forceinline__ T block_excl_scan(T x, T *wsum, T *total)
{
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    T y = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const T z = __shfl_up_sync(0xffffffffu, y, o);
        if (lane >= o) y += z;
    }
    if (lane == 31) wsum[warp] = y;
    __syncthreads();
    if (warp == 0) {
        T w = lane < SC_T / 32 ? wsum[lane] : (T)0;
        T s = w;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const T z = __shfl_up_sync(0xffffffffu, s, o);
            if (lane >= o) s += z;
        }
        if (lane < SC_T / 32) wsum[lane] = s - w;
        if (lane == 31) *total = s;
    }
    __syncthreads();
    const T r = wsum[warp] + y - x;
    __syncthreads();
    return r;
}

template <typename T>
__global__ void __launch_bounds__(SC_T) scan_tile_sums(const T *a, uint64_t n, T *sums)
{
    __shared__ T wsum[SC_T / 32];
    __shared__ T tot;
    const uint64_t base = (uint64_t)blockIdx.x * SC_TILE + (uint64_t)threadIdx.x * SC_IPT;
    T s = 0;
#pragma unroll
    for (int k = 0; k < SC_IPT; ++k)
        if (base + k < n) s += a[base + k];
    block_excl_scan<T>(s, wsum, &tot);
    if (threadIdx.x == 0) sums[blockIdx.x] = tot;
}

// one CTA: exclusive scan of the tile sums in place; *grand = their total
template <typename T>
__global__ void __launch_bounds__(SC_T) scan_sums(T *sums, uint64_t m, unsigned long long *grand)
{
    __shared__ T wsum[SC_T / 32];
    __shared__ T tot;
    T carry = 0;
    for (uint64_t b0 = 0; b0 < m; b0 += SC_T) {
        const uint64_t i = b0 + threadIdx.x;
        const T x = i < m ? sums[i] : (T)0;
        const T e = block_excl_scan<T>(x, wsum, &tot);
        if (i < m) sums[i] = carry + e;
        carry += tot;
    }
    if (threadIdx.x == 0) *grand = (unsigned long long)carry;
}

template <typename T>
__global__ void __launch_bounds__(SC_T) scan_tiles(T *a, uint64_t n, const T *sums)
{
    __shared__ T wsum[SC_T / 32];
    __shared__ T tot;
    const uint64_t base = (uint64_t)blockIdx.x * SC_TILE + (uint64_t)threadIdx.x * SC_IPT;
    T x[SC_IPT];
    T s = 0;
#pragma unroll
    for (int k = 0; k < SC_IPT; ++k) {
        x[k] = base + k < n ? a[base + k] : (T)0;
        s += x[k];
    }
    T run = block_excl_scan<T>(s, wsum, &tot) + sums[blockIdx.x];
#pragma unroll
    for (int k = 0; k < SC_IPT; ++k)
        if (base + k < n) {
            a[base + k] = run;
            run += x[k];
        }
}

template <typename T>
static lasagna_status excl_scan(T *a, uint64_t n, T *sums, unsigned long long *grand,
                                cudaStream_t s)
{
    const uint64_t tiles = ceil_div(n, SC_TILE);
    scan_tile_sums<T><<<(unsigned)tiles, SC_T, 0, s>>>(a, n, sums);
    LSG_LAUNCHED("scan_tile_sums");
    scan_sums<T><<<1, SC_T, 0, s>>>(sums, tiles, grand);
    LSG_LAUNCHED("scan_sums");
    scan_tiles<T><<<(unsigned)tiles, SC_T, 0, s>>>(a, n, sums);
    LSG_LAUNCHED("scan_tiles");
    return LASAGNA_OK;
}

__global__ void cp_index(uint64_t V, const uint32_t *__restrict__ keep_scanned,
                         const uint32_t *__restrict__ keep_flag_src,
                         const unsigned long long *__restrict__ off, unsigned long long total,
                         unsigned long long n_contigs, uint64_t *contig_offsets,
                         uint32_t *contig_seed)
{
    (void)keep_flag_src;
    for (uint64_t r = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; r < V;
         r += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t c = keep_scanned[r];
        const uint32_t nx = r + 1 < V ? keep_scanned[r + 1] : (uint32_t)n_contigs;
        if (nx != c) { // r is the c-th kept seed
            contig_offsets[c] = off[r];
            if (contig_seed) contig_seed[c] = (uint32_t)r;
        }
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) contig_offsets[n_contigs] = total;
}

// every vertex of a kept path writes its first overhang bases, as ASCII
template <int W>
__global__ void cp_place(const uint64_t *__restrict__ packed, uint32_t stride, uint32_t L,
                         const uint32_t *__restrict__ succ, const uint8_t *__restrict__ olen,
                         uint64_t V, const uint32_t *__restrict__ ptr,
                         const unsigned long long *__restrict__ val,
                         const uint32_t *__restrict__ keep, const unsigned long long *__restrict__ off,
                         char *__restrict__ contigs)
{
    for (uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; v < V;
         v += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t r = ptr[v];
        if (cp_pred(succ, r) != NONE || !keep[r]) continue; // no kept path (or a cycle)
        if (r == (uint32_t)v && succ[v] == NONE) continue;  // isolated read: no path
        const uint32_t s = succ[v];
        const uint32_t ov = s == NONE ? L : L - olen[v];
        uint64_t x[W], y[W];
        load_read<W>(packed, stride, v >> 1, x);
        if (v & 1) rc_words<W>(x, L, y);
        else {
#pragma unroll
            for (int j = 0; j < W; ++j) y[j] = x[j];
        }
        char *out = contigs + off[r] + val[v];
#pragma unroll
        for (int w = 0; w < W; ++w) {
            uint64_t word = y[w];
            for (uint32_t k = 0; k < 32u; ++k) {
                const uint32_t j = 32u * w + k;
                if (j >= ov) break;
                out[j] = "ACTG"[(uint32_t)(word & 3u)]; // R1: A0 C1 T2 G3
                word >>= 2;
            }
        }
    }
}

lasagna_status compress_impl(const uint64_t *packed, uint64_t n, uint32_t L, const uint32_t *succ,
                             const uint8_t *olen, void *workspace, size_t *workspace_bytes,
                             char *contigs, uint64_t contig_capacity, uint64_t *contig_offsets,
                             uint32_t *contig_seed, uint64_t count_capacity, uint64_t *n_contigs,
                             uint64_t *total_bases, cudaStream_t s)
{
    const uint64_t V = 2 * n;
    auto a256 = [](size_t x) { return (x + 255) & ~(size_t)255; };
    const uint64_t tiles = ceil_div(std::max<uint64_t>(V, 1), SC_TILE);
    // ptrA ptrB | valA valB | keep | sums (u64) | counters
    const size_t o_pa = 0, o_pb = o_pa + a256(V * 4), o_va = o_pb + a256(V * 4),
                 o_vb = o_va + a256(V * 8), o_keep = o_vb + a256(V * 8),
                 o_sums = o_keep + a256(V * 4), o_ctr = o_sums + a256(tiles * 8),
                 total = o_ctr + 256;
    if (!workspace) {
        *workspace_bytes = total;
        return LASAGNA_OK;
    }
    if (*workspace_bytes < total) {
        *workspace_bytes = total;
        set_error("workspace too small");
        return LASAGNA_ENOSPC;
    }
    *n_contigs = 0;
    *total_bases = 0;
    if (V == 0) return LASAGNA_OK;
    char *ws = (char *)workspace;
    uint32_t *ptr[2] = {reinterpret_cast<uint32_t *>(ws + o_pa), reinterpret_cast<uint32_t *>(ws + o_pb)};
    unsigned long long *val[2] = {reinterpret_cast<unsigned long long *>(ws + o_va),
                                  reinterpret_cast<unsigned long long *>(ws + o_vb)};
    uint32_t *keep = reinterpret_cast<uint32_t *>(ws + o_keep);
    unsigned long long *ctr = reinterpret_cast<unsigned long long *>(ws + o_ctr); // [0] open [1] grand
    const unsigned grid = (unsigned)std::max<uint64_t>(
        1, std::min<uint64_t>(ceil_div(V, CP_THREADS), (uint64_t)num_sms() * 16));
    cp_init<<<grid, CP_THREADS, 0, s>>>(succ, olen, V, L, ptr[0], val[0]);
    LSG_LAUNCHED("cp_init");
    // pointer jumping: a path of m vertices converges in ceil(log2 m) rounds; stop when no
    // pointer is open, or after ceil(log2 V) + 1 rounds (only cycle vertices stay open)
    int cur = 0;
    uint32_t cap = 1;
    while ((1ull << cap) < V) ++cap;
    cap += 1;
    for (uint32_t round = 0; round < cap; ++round) {
        LSG_CUDA(cudaMemsetAsync(ctr, 0, 8, s));
        cp_jump<<<grid, CP_THREADS, 0, s>>>(V, ptr[cur], val[cur], ptr[cur ^ 1], val[cur ^ 1], ctr);
        LSG_LAUNCHED("cp_jump");
        cur ^= 1;
        unsigned long long open = 0;
        LSG_CUDA(cudaMemcpyAsync(&open, ctr, 8, cudaMemcpyDeviceToHost, s));
        LSG_CUDA(cudaStreamSynchronize(s));
        if (open == 0) break;
    }
    // tails -> kept seeds and their contig lengths (in the free val buffer)
    unsigned long long *len = val[cur ^ 1];
    LSG_CUDA(cudaMemsetAsync(len, 0, V * 8, s));
    LSG_CUDA(cudaMemsetAsync(keep, 0, V * 4, s));
    cp_tails<<<grid, CP_THREADS, 0, s>>>(succ, V, L, ptr[cur], val[cur], len, keep);
    LSG_LAUNCHED("cp_tails");
    // Fig. 7's scans: contig offsets (over lengths) and contig indices (over kept flags)
    unsigned long long *sums = reinterpret_cast<unsigned long long *>(ws + o_sums);
    lasagna_status rc = excl_scan<unsigned long long>(len, V, sums, ctr + 1, s);
    if (rc != LASAGNA_OK) return rc;
    unsigned long long tot = 0;
    LSG_CUDA(cudaMemcpyAsync(&tot, ctr + 1, 8, cudaMemcpyDeviceToHost, s));
    // keep -> contig index; keep is needed by cp_place too, so scan a copy in ptr[cur ^ 1]
    uint32_t *cidx = ptr[cur ^ 1];
    LSG_CUDA(cudaMemcpyAsync(cidx, keep, V * 4, cudaMemcpyDeviceToDevice, s));
    rc = excl_scan<uint32_t>(cidx, V, reinterpret_cast<uint32_t *>(sums), ctr + 2, s);
    if (rc != LASAGNA_OK) return rc;
    unsigned long long nc = 0;
    LSG_CUDA(cudaMemcpyAsync(&nc, ctr + 2, 8, cudaMemcpyDeviceToHost, s));
    LSG_CUDA(cudaStreamSynchronize(s));
    *n_contigs = nc;
    *total_bases = tot;
    if (tot > contig_capacity || nc + 1 > count_capacity) {
        set_error("contigs need %llu bases and %llu offsets", tot, nc + 1);
        return LASAGNA_ENOSPC;
    }
    if (!contigs || !contig_offsets) {
        set_error("NULL output");
        return LASAGNA_EINVAL;
    }
    cp_index<<<grid, CP_THREADS, 0, s>>>(V, cidx, keep, len, tot, nc, contig_offsets, contig_seed);
    LSG_LAUNCHED("cp_index");
    return dispatch_W(L, [&](auto wc) -> lasagna_status {
        constexpr int Wd = decltype(wc)::value;
        cp_place<Wd><<<grid, CP_THREADS, 0, s>>>(packed, stride_for(L), L, succ, olen, V, ptr[cur],
                                                 val[cur], keep, len, contigs);
        LSG_LAUNCHED("cp_place");
        LSG_CUDA(cudaStreamSynchronize(s));
        return LASAGNA_OK;
    });
}

} // namespace lsg
