/*
 * readgen.c — seeded synthetic read generator shared by the CUDA path's tests/bench
 * and the CPU oracle.  It holds NONE of the method's arithmetic (no fingerprints, no
 * overlaps); it only draws reads.
 *
 * Recipe (reading R18 of PAPER.md §IV-A, where
 * the paper's real Illumina data is replaced by synthetic reads):
 *   genome  g[0..G)      i.i.d. uniform over {A,C,G,T}
 *   read i  start s_i    uniform in [0, G-L]
 *           strand       reverse-complemented with probability 1/2
 *           errors       each base independently substituted with probability p by one of
 *                        the other three bases, uniformly; no indels
 *   order                generation order; read id = index i
 * Every random number is a counter-based splitmix64 draw of (seed, stream, index), so
 * chunked and multi-threaded generation produce identical bytes.
 *
 * Output: n*L ASCII bytes, fixed stride L, no separators, uppercase ACGT.
 */
#include <stdint.h>
#include <stddef.h>

static inline uint64_t splitmix64(uint64_t x)
{
    x += 0x9E3779B97F4A7C15ULL;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ULL;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBULL;
    return x ^ (x >> 31);
}

/* key of a stream: independent of the index; draw(stream, idx) = splitmix64(key + idx) */
static inline uint64_t stream_key(uint64_t seed, uint64_t stream)
{
    return splitmix64(splitmix64(seed) ^ (0xD1B54A32D192ED03ULL * (stream + 1)));
}

enum { S_GENOME = 0, S_START = 1, S_STRAND = 2, S_ERRPOS = 3, S_ERRBASE = 4 };

static const char ACGT[4] = {'A', 'C', 'G', 'T'};

/* genome base g as an index into ACGT (A0 C1 G2 T3 — the generator's own order) */
static inline int genome_base(uint64_t kg, uint64_t g)
{
    return (int)((splitmix64(kg + (g >> 5)) >> ((g & 31) * 2)) & 3);
}

int readgen_version(void) { return 1; }

/* Write G genome bases as ASCII into out[0..G). */
void readgen_genome(uint64_t seed, uint64_t G, char *out)
{
    uint64_t kg = stream_key(seed, S_GENOME);
#pragma omp parallel for schedule(static)
    for (int64_t g = 0; g < (int64_t)G; ++g) out[g] = ACGT[genome_base(kg, (uint64_t)g)];
}

/* Reads [i0, i1) of the set (seed, G, L, p_err) into out (row i at out + (i-i0)*L).
 * Returns 0, or -1 on invalid parameters (L == 0 or L > G). */
int readgen_reads(uint64_t seed, uint64_t G, uint32_t L, double p_err,
                  uint64_t i0, uint64_t i1, char *out, uint64_t *starts, uint8_t *strands)
{
    if (L == 0 || (uint64_t)L > G) return -1;
    const uint64_t kg = stream_key(seed, S_GENOME), ks = stream_key(seed, S_START),
                   kr = stream_key(seed, S_STRAND), ke = stream_key(seed, S_ERRPOS),
                   kb = stream_key(seed, S_ERRBASE);
    const uint64_t span = G - L + 1;
    /* substitution threshold on a 64-bit uniform draw: P(u < thr) = p */
    uint64_t thr;
    if (p_err <= 0.0) thr = 0;
    else if (p_err >= 1.0) thr = UINT64_MAX;
    else thr = (uint64_t)(p_err * 18446744073709551616.0);
#pragma omp parallel for schedule(static)
    for (int64_t ii = (int64_t)i0; ii < (int64_t)i1; ++ii) {
        uint64_t i = (uint64_t)ii;
        uint64_t s = (uint64_t)(((unsigned __int128)splitmix64(ks + i) * span) >> 64);
        int rc = (int)(splitmix64(kr + i) & 1);
        char *row = out + (i - i0) * (uint64_t)L;
        for (uint32_t k = 0; k < L; ++k) {
            int b;
            if (!rc) b = genome_base(kg, s + k);
            else b = 3 - genome_base(kg, s + (L - 1 - k)); /* complement in A0 C1 G2 T3 is 3-b */
            uint64_t e = (uint64_t)i * L + k;
            if (thr && splitmix64(ke + e) < thr) {
                int r = (int)(splitmix64(kb + e) % 3); /* one of the other three, uniformly */
                b = (b + 1 + r) & 3;
            }
            row[k] = ACGT[b];
        }
        if (starts) starts[i - i0] = s;
        if (strands) strands[i - i0] = (uint8_t)rc;
    }
    return 0;
}

/* Start positions only of reads [i0, i1) (the same draws readgen_reads makes; no bases):
 * lets a caller pick the reads of a genome window — a coverage-preserving sample. */
int readgen_starts(uint64_t seed, uint64_t G, uint32_t L, uint64_t i0, uint64_t i1,
                   uint64_t *starts)
{
    if (L == 0 || (uint64_t)L > G) return -1;
    const uint64_t ks = stream_key(seed, S_START);
    const uint64_t span = G - L + 1;
#pragma omp parallel for schedule(static)
    for (int64_t ii = (int64_t)i0; ii < (int64_t)i1; ++ii)
        starts[(uint64_t)ii - i0] =
            (uint64_t)(((unsigned __int128)splitmix64(ks + (uint64_t)ii) * span) >> 64);
    return 0;
}
