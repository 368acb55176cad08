// gsnp_compress.cuh — GPU output compression of gsnp_record tables (§V-B), sm_100a.
// Included once, by gsnp.cu.  Byte format: reading R17 of DESIGN.md (one section per column
// family the paper names; the six quality columns are RLE'd and both the run-value
// and the run-length arrays are DICT-encoded: sorted unique dictionary + parallel binary search +
// least-bit packing of the indices).
//
// Device pipeline, blocks of B records, every block independent:
//   k_cz_columns   records (AoS, 40 B) -> column arrays (SoA), one pass over the input
//   k_cz_sections<false>  grid (section, block): each CTA sizes one section of one block; the
//                  DICT sections build their dictionary with a shared-memory hash set, sort it
//                  (bitonic) and park it in scratch
//   k_cz_scan      exclusive scan of the section sizes -> word offset of every section
//   k_cz_sections<true>   grid (section, block): each CTA writes its section at its offset
//                  (exception lists by CTA scans, RLE runs by run-start compaction with a carry
//                  across chunks, DICT indices by binary search in the sorted dictionary,
//                  bit packing through a shared-memory staging window)
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace gsnp_cz {

constexpr int NT = 512;                    // threads per CTA
#ifndef GSNP_CZ_MINB
#define GSNP_CZ_MINB 4                     // CTAs per SM the section kernels are built for
#endif
#ifndef GSNP_CZ_MINB_W
#define GSNP_CZ_MINB_W 4                   // (the dictionary write pass; 3 measured slower)
#endif
constexpr int NWP = NT / 32;
constexpr int IT = 4;                      // consecutive sites per thread per chunk
constexpr int CH = NT * IT;                // sites per chunk
constexpr uint32_t MAGIC = 0x31435347u;    // "GSC1"
constexpr uint32_t DICT_MAX = 4096;
constexpr uint32_t RAW = 0xFFFFFFFFu;
constexpr uint32_t ONE = 0x3F800000u;      // 1.0f
constexpr uint32_t EMPTY = 0xFFFFFFFFu;
constexpr int HS = 8192;                   // hash slots (> 2 x DICT_MAX: inserts stop past D_MAX)
constexpr int PKW = 800;                   // packer staging words: (CH+1)*12/32 + 2 <= 800
constexpr int NSEC = 16;                   // sections per block, in stream order
constexpr int NDICT = 15;                  // dictionaries per block: S x3, C0..C5 x (values, lengths)
enum : int { SEC_HDR = 0, SEC_P = 1, SEC_N = 2, SEC_G = 5, SEC_K = 6, SEC_R = 7, SEC_Q = 8,
             SEC_S = 9, SEC_C = 10 };

// column ids in record order (gsnp.h): u8 0..7, u16 8..11, u32 12..15
enum : int { C_REF = 0, C_GENO, C_QUAL, C_BASE1, C_BASE2, C_AVGQ1, C_AVGQ2, C_KNOWN,
             C_CU1 = 8, C_CA1, C_CU2, C_CA2, C_DEPTH = 12, C_RANKP, C_COPYN, C_POST1 };

struct Cols {
    uint8_t* u8[8];
    uint16_t* u16[4];
    uint32_t* u32[4];
};

struct CzArgs {
    const gsnp_record* rec;
    uint64_t n;               // records
    uint32_t B;               // records per block
    uint32_t nblk;
    uint32_t DC;              // dictionary capacity per block and dictionary = min(DICT_MAX, B)
    Cols col;
    uint32_t* meta;           // [nblk][NSEC][2]: words, m (or R)
    uint32_t* dD;             // [nblk][NDICT] dictionary sizes (RAW = over DICT_MAX)
    uint32_t* dict;           // [nblk][NDICT][DC] sorted dictionaries
    const uint64_t* off;      // [nblk*NSEC + 1] section word offsets (write pass)
    uint32_t* out;
};

__device__ __forceinline__ uint32_t colv(const Cols& C, int c, uint64_t i) {
    if (c < 8) return C.u8[c][i];
    if (c < 12) return C.u16[c - 8][i];
    return C.u32[c - 12][i];
}

// ------------------------------------------------------------------------ records -> columns
__global__ void __launch_bounds__(256) k_cz_columns(const gsnp_record* rec, uint64_t n, Cols C) {
    for (uint64_t i = blockIdx.x * 256ull + threadIdx.x; i < n; i += (uint64_t)gridDim.x * 256) {
        const uint64_t* r = reinterpret_cast<const uint64_t*>(rec + i);
        const uint64_t b8 = __ldg(r + 1), b16 = __ldg(r + 2), b24 = __ldg(r + 3), b32 = __ldg(r + 4);
#pragma unroll
        for (int k = 0; k < 8; ++k) C.u8[k][i] = (uint8_t)(b8 >> (8 * k));
#pragma unroll
        for (int k = 0; k < 4; ++k) C.u16[k][i] = (uint16_t)(b16 >> (16 * k));
        C.u32[0][i] = (uint32_t)b24;
        C.u32[1][i] = (uint32_t)(b24 >> 32);
        C.u32[2][i] = (uint32_t)b32;
        C.u32[3][i] = (uint32_t)(b32 >> 32);
    }
}

// ------------------------------------------------------------------------ CTA helpers
struct Smem {
    uint32_t ws[NWP + 2];     // scan scratch
    uint32_t bc[8];           // broadcast slots
};

// exclusive scan of one value per thread; *total = CTA sum.  Ends with a barrier.
__device__ __forceinline__ uint32_t cta_scan(uint32_t v, Smem& S, uint32_t* total) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    uint32_t x = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
        if (lane >= d) x += y;
    }
    if (lane == 31) S.ws[w] = x;
    __syncthreads();
    if (w == 0) {
        uint32_t t = lane < NWP ? S.ws[lane] : 0, s = t;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            uint32_t y = __shfl_up_sync(0xFFFFFFFFu, s, d);
            if (lane >= d) s += y;
        }
        if (lane < NWP) S.ws[lane] = s - t;
        if (lane == 31) S.ws[NWP] = s;
    }
    __syncthreads();
    const uint32_t r = S.ws[w] + x - v;
    *total = S.ws[NWP];
    __syncthreads();
    return r;
}

__host__ __device__ __forceinline__ uint32_t bitlen(uint32_t v) {
#ifdef __CUDA_ARCH__
    return v ? 32u - __clz(v) : 0u;
#else
    return v ? 32u - (uint32_t)__builtin_clz(v) : 0u;
#endif
}

__host__ __device__ __forceinline__ uint64_t dict_words(uint64_t m, uint32_t D) {
    if (m == 0) return 0;
    if (D == RAW) return 1 + m;
    const uint32_t b = D <= 1 ? 0 : bitlen(D - 1);
    return 1 + D + (m * b + 31) / 32;
}

// --- set of distinct values (dictionary construction, "sort + unique"): values below
// BMV in a bitmap (sorted by construction), the rest in a hash set sorted at the end
constexpr uint32_t BMV = 65536;            // bitmap range (2048 words)
constexpr uint32_t BMW = BMV / 32;
struct VSet {
    uint32_t* bm;             // BMW words
    uint32_t* slot;           // HS words, EMPTY = free
    uint32_t* cnt;            // [0] distinct hashed values, [1] saw 0xFFFFFFFF
};

__device__ __forceinline__ void vs_clear(VSet h) {
    for (int i = threadIdx.x; i < HS; i += NT) h.slot[i] = EMPTY;
    for (int i = threadIdx.x; i < (int)BMW; i += NT) h.bm[i] = 0;
    if (threadIdx.x == 0) { h.cnt[0] = 0; h.cnt[1] = 0; }
}

__device__ __forceinline__ void vs_insert(VSet h, uint32_t v) {
    if (v < BMV) {
        const uint32_t bit = 1u << (v & 31);
        if (!(h.bm[v >> 5] & bit)) atomicOr(&h.bm[v >> 5], bit);
        return;
    }
    if (v == EMPTY) { h.cnt[1] = 1; return; }
    if (*(volatile uint32_t*)h.cnt > DICT_MAX) return;      // RAW already: stop (bounded fill)
    uint32_t s = (v * 2654435761u) >> 19;                  // 13 bits
    for (;;) {
        uint32_t cur = *(volatile uint32_t*)&h.slot[s];
        if (cur == v) return;
        if (cur == EMPTY) {
            uint32_t old = atomicCAS(&h.slot[s], EMPTY, v);
            if (old == EMPTY) { atomicAdd(h.cnt, 1u); return; }
            if (old == v) return;
        }
        s = (s + 1) & (HS - 1);
    }
}

// Sorted unique list of the set into gdict (capacity >= D); returns D or RAW.  sb: DICT_MAX words
// of sort buffer (may overlap the bitmap: it is read first).
__device__ uint32_t vs_finalize(VSet h, uint32_t* sb, uint32_t* gdict, Smem& S) {
    __syncthreads();
    constexpr int PW = BMW / NT;
    uint32_t w[PW], k = 0;
#pragma unroll
    for (int i = 0; i < PW; ++i) { w[i] = h.bm[threadIdx.x * PW + i]; k += __popc(w[i]); }
    uint32_t nsmall;
    uint32_t at = cta_scan(k, S, &nsmall);               // (ends with a barrier: bm is free)
    const uint32_t c = h.cnt[0], hasmax = h.cnt[1];
    const uint32_t D = nsmall + c + hasmax;
    if (D > DICT_MAX) return RAW;
#pragma unroll
    for (int i = 0; i < PW; ++i)
        while (w[i]) {
            gdict[at++] = (threadIdx.x * PW + i) * 32 + __ffs(w[i]) - 1;
            w[i] &= w[i] - 1;
        }
    if (c) {                                             // hashed values: compact, bitonic sort
        constexpr int PER = HS / NT;
        uint32_t kk = 0;
        for (int i = 0; i < PER; ++i) kk += h.slot[threadIdx.x * PER + i] != EMPTY;
        uint32_t tot;
        uint32_t a2 = cta_scan(kk, S, &tot);
        for (int i = 0; i < PER; ++i) {
            uint32_t v = h.slot[threadIdx.x * PER + i];
            if (v != EMPTY) sb[a2++] = v;
        }
        uint32_t P2 = 1;
        while (P2 < c) P2 <<= 1;
        for (uint32_t i = c + threadIdx.x; i < P2; i += NT) sb[i] = EMPTY;
        __syncthreads();
        for (uint32_t q = 2; q <= P2; q <<= 1)
            for (uint32_t j = q >> 1; j > 0; j >>= 1) {
                for (uint32_t i = threadIdx.x; i < P2; i += NT) {
                    uint32_t ixj = i ^ j;
                    if (ixj > i) {
                        uint32_t x = sb[i], y = sb[ixj];
                        bool up = (i & q) == 0;
                        if ((x > y) == up) { sb[i] = y; sb[ixj] = x; }
                    }
                }
                __syncthreads();
            }
        for (uint32_t i = threadIdx.x; i < c; i += NT) gdict[nsmall + i] = sb[i];
    }
    if (hasmax && threadIdx.x == 0) gdict[nsmall + c] = 0xFFFFFFFFu;
    __syncthreads();
    return D;
}

// --- least-bit packer: element j's b-bit index at bit j*b of the packed area (LSB first)
struct Packer {
    uint32_t* st;             // PKW staging words in shared memory; st[0] is at bit `base`
    uint32_t* g;              // global packed area
    uint64_t base;            // multiple of 32
    uint32_t b;
};

__device__ __forceinline__ void pk_init(Packer& p, uint32_t* st, uint32_t* g, uint32_t b) {
    p.st = st; p.g = g; p.base = 0; p.b = b;
    for (int i = threadIdx.x; i < PKW; i += NT) st[i] = 0;
}

__device__ __forceinline__ void pk_add(const Packer& p, uint64_t j, uint32_t idx) {
    if (p.b == 0) return;
    const uint64_t bit = j * p.b - p.base;
    const uint32_t w = (uint32_t)(bit >> 5), sh = (uint32_t)(bit & 31);
    atomicOr(&p.st[w], idx << sh);
    if (sh + p.b > 32) atomicOr(&p.st[w + 1], idx >> (32 - sh));
}

// all elements < jend added (call after a barrier): store the complete words, keep the partial one
__device__ __forceinline__ void pk_flush(Packer& p, uint64_t jend) {
    if (p.b == 0) return;
    const uint32_t full = (uint32_t)((jend * p.b - p.base) >> 5);
    for (uint32_t w = threadIdx.x; w < full; w += NT) p.g[(p.base >> 5) + w] = p.st[w];
    __syncthreads();
    const uint32_t carry = p.st[full];
    __syncthreads();
    for (uint32_t w = threadIdx.x; w <= full && w < PKW; w += NT) p.st[w] = w == 0 ? carry : 0;
    p.base += (uint64_t)full * 32;
    __syncthreads();
}

__device__ __forceinline__ void pk_final(const Packer& p, uint64_t m) {
    if (p.b && m * p.b > p.base && threadIdx.x == 0) p.g[p.base >> 5] = p.st[0];
}

// --- DICT output of one array: header, dictionary, packed indices (or RAW values).
// The index of a value is found by the paper's binary search in the sorted dictionary
// (P:L779-780); values below LUTN take it from a direct table filled from the same dictionary
// (the same index, one shared-memory load instead of ~12 dependent ones).
constexpr uint32_t LUTN = 4096;
struct DictOut {
    uint32_t D;
    const uint32_t* sd;       // sorted dictionary in shared memory (D words) unless RAW
    const uint16_t* lut;      // lut[v] = index of v, for dictionary values v < LUTN
    uint32_t* g;              // section start in the output
    Packer pk;
};

__device__ __forceinline__ void do_init(DictOut& d, uint32_t D, uint32_t* sd, uint16_t* lut,
                                        const uint32_t* gdict, uint32_t* g, uint32_t* st, uint64_t m) {
    d.D = D; d.sd = sd; d.lut = lut; d.g = g;
    if (m == 0) { d.pk.b = 0; return; }
    if (threadIdx.x == 0) g[0] = D;
    if (D == RAW) { d.pk.b = 0; return; }
    for (uint32_t i = threadIdx.x; i < D; i += NT) {
        uint32_t v = gdict[i];
        sd[i] = v;
        g[1 + i] = v;
        if (v < LUTN) lut[v] = (uint16_t)i;
    }
    pk_init(d.pk, st, g + 1 + D, D <= 1 ? 0 : bitlen(D - 1));
}

__device__ __forceinline__ void do_add(const DictOut& d, uint64_t j, uint32_t v) {
    if (d.D == RAW) { d.g[1 + j] = v; return; }
    uint32_t lo;
    if (v < LUTN) {
        lo = d.lut[v];
    } else {
        uint32_t hi = d.D;                     // parallel binary search
        lo = 0;
        while (lo < hi) {
            uint32_t mid = (lo + hi) >> 1;
            if (d.sd[mid] < v) lo = mid + 1; else hi = mid;
        }
    }
    pk_add(d.pk, j, lo);
}

// ------------------------------------------------------------------------ sections
struct BlockCtx {
    uint64_t g0;              // global index of the block's first record
    uint32_t n;               // records in the block
    uint32_t blk;             // block number
};

// IT (= 4) consecutive elements of a column from element i (n_left of them valid, the rest 0);
// vec: the column and i are aligned for one vector load
static_assert(IT == 4, "vector loads take four elements");
template <typename T>
__device__ __forceinline__ void ld4(const T* col, uint64_t i, bool vec, uint32_t n_left,
                                    uint32_t (&v)[IT]) {
    if (vec && n_left >= 4) {
        if constexpr (sizeof(T) == 1) {
            const uint32_t w = *reinterpret_cast<const uint32_t*>(col + i);
#pragma unroll
            for (int u = 0; u < 4; ++u) v[u] = (w >> (8 * u)) & 255u;
        } else if constexpr (sizeof(T) == 2) {
            const uint2 w = *reinterpret_cast<const uint2*>(col + i);
            v[0] = w.x & 0xFFFFu; v[1] = w.x >> 16; v[2] = w.y & 0xFFFFu; v[3] = w.y >> 16;
        } else {
            const uint4 w = *reinterpret_cast<const uint4*>(col + i);
            v[0] = w.x; v[1] = w.y; v[2] = w.z; v[3] = w.w;
        }
        return;
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) v[u] = (uint32_t)u < n_left ? (uint32_t)col[i + u] : 0u;
}

// exception-list sections N / G / K / R / Q.  The size pass only counts (one
// reduction at the end); the write pass orders the exceptions with a CTA scan per chunk.
template <bool WRITE>
__device__ void sec_exceptions(const CzArgs& A, const BlockCtx& bk, int sec, Smem& S,
                               uint32_t* st) {
    const Cols& C = A.col;
    const uint32_t blk = bk.blk;
    uint32_t* meta = A.meta + ((size_t)blk * NSEC + sec) * 2;
    const uint32_t m = WRITE ? meta[1] : 0;
    uint32_t* o = WRITE ? A.out + A.off[(size_t)blk * NSEC + sec] : nullptr;
    const bool nsec = sec <= SEC_N + 2;
    const uint8_t* ncol = C.u8[sec == SEC_N ? C_REF : sec == SEC_N + 1 ? C_BASE1 : C_BASE2];
    const bool vec = (bk.g0 & 3) == 0;
    Packer pk;
    if (WRITE && (sec == SEC_G || sec == SEC_K)) pk_init(pk, st, o + 1 + m, 8);
    if (WRITE && threadIdx.x == 0) o[0] = m;
    uint32_t run = 0, runE = 0, mine = 0;                    // exceptions (N: run starts, ends)
                                                             // before this chunk
    for (uint32_t c0 = 0; c0 < bk.n; c0 += CH) {
        uint32_t fl[IT], vals[IT], cnt = 0;
        const uint32_t s0 = c0 + threadIdx.x * IT;
        const uint32_t left = s0 < bk.n ? bk.n - s0 : 0;
        const uint64_t gi = bk.g0 + s0;
        if (nsec) {                                          // runs of code 4: start (lo16), end (hi16)
            uint32_t x[IT];
            ld4(ncol, gi, vec, left, x);
            bool pf = s0 > 0 && left && ncol[gi - 1] == 4;
            const bool last_nf = left > 4 && ncol[gi + 4] == 4;
#pragma unroll
            for (int u = 0; u < IT; ++u) {
                const bool f = (uint32_t)u < left && x[u] == 4;
                const bool nf = u + 1 < IT ? ((uint32_t)(u + 1) < left && x[u + 1] == 4) : last_nf;
                fl[u] = (f && !pf ? 1u : 0u) | (f && !nf ? 0x10000u : 0u);
                pf = f;
                vals[u] = 0;
            }
        } else if (sec == SEC_G) {
            uint32_t r[IT];
            ld4(C.u8[C_REF], gi, vec, left, r);
            ld4(C.u8[C_GENO], gi, vec, left, vals);
#pragma unroll
            for (int u = 0; u < IT; ++u) {
                const uint32_t pred = r[u] < 4 ? (0x09070400u >> (8 * r[u])) & 255 : 255;   // HOM[ref]
                fl[u] = (uint32_t)u < left && vals[u] != pred;
            }
        } else if (sec == SEC_K) {
            ld4(C.u8[C_KNOWN], gi, vec, left, vals);
#pragma unroll
            for (int u = 0; u < IT; ++u) fl[u] = vals[u] != 0;
        } else {
            ld4(C.u32[sec == SEC_R ? C_RANKP - 12 : C_POST1 - 12], gi, vec, left, vals);
#pragma unroll
            for (int u = 0; u < IT; ++u) fl[u] = (uint32_t)u < left && vals[u] != ONE;
        }
#pragma unroll
        for (int u = 0; u < IT; ++u) cnt += fl[u];
        if (!WRITE) {
            mine += nsec ? (cnt & 0xFFFF) : cnt;
            continue;
        }
        uint32_t tot;
        uint32_t r = cta_scan(cnt, S, &tot);
        if (nsec) {
            uint32_t rs = run + (r & 0xFFFF), re = runE + (r >> 16);
#pragma unroll
            for (int u = 0; u < IT; ++u) {
                if (fl[u] & 1) o[1 + rs++] = s0 + u;
                if (fl[u] >> 16) o[1 + m + re++] = s0 + u + 1;
            }
        } else {
            uint32_t j = run + r;
#pragma unroll
            for (int u = 0; u < IT; ++u) {
                if (!fl[u]) continue;
                o[1 + j] = s0 + u;
                if (sec == SEC_G || sec == SEC_K) pk_add(pk, j, vals[u]);
                else o[1 + m + j] = vals[u];
                ++j;
            }
        }
        run += nsec ? (tot & 0xFFFF) : tot;
        runE += tot >> 16;
        if (sec == SEC_G || sec == SEC_K) {
            __syncthreads();
            pk_flush(pk, run);
        }
    }
    if (WRITE) {
        if (sec == SEC_G || sec == SEC_K) pk_final(pk, m);
        return;
    }
    cta_scan(mine, S, &run);
    if (threadIdx.x == 0) {
        uint64_t words = nsec || sec == SEC_R || sec == SEC_Q ? 1 + 2ull * run : 1 + run + (run + 3) / 4;
        meta[0] = (uint32_t)words;
        meta[1] = run;
    }
}

// second-allele section S: bitmap of sites with a non-zero second allele, then
// DICT of avgq2, cnt_uni2, cnt_all2 over those sites in order
__device__ __forceinline__ bool s_mask(const Cols& C, uint64_t gi) {
    return (C.u8[C_AVGQ2][gi] | C.u16[C_CU2 - 8][gi] | C.u16[C_CA2 - 8][gi]) != 0;
}

__device__ __forceinline__ int rle_col(int ci) {
    return ci == 0 ? C_QUAL : ci == 1 ? C_AVGQ1 : ci == 2 ? C_CU1 : ci == 3 ? C_CA1
         : ci == 4 ? C_DEPTH : C_COPYN;
}

// One dictionary of one block per CTA (grid nblk x NDICT; dictionary d in dD order): d 0..2 the
// S section's avgq2 / cnt_uni2 / cnt_all2 over the sites with a second allele;
// d = 3 + 2 ci (+1) the run values (lengths) of quality column C<ci>.
// KIND 0: masked values, 1: run values, 2: run lengths.
//   size pass: set of the distinct values -> sorted dictionary in scratch, its size in dD, the
//              element count (S: masked sites, C: runs) in meta[1] (section sizes: k_cz_scan)
//   write pass: the DICT array at its place in the section (S: after the bitmap, written by d = 0
//              and the dictionaries before it; C: R, then the values array, then the lengths)
// shared layout  size:  hash HS + 2 | bitmap BMW | starts CH (bitmap + starts: the sort buffer)
//                write: sd DICT_MAX | lut LUTN/2 | packer PKW | starts CH
constexpr size_t SMEM_DSIZE_WORDS = HS + 2 + BMW + CH;
constexpr size_t SMEM_DWRITE_WORDS = DICT_MAX + LUTN / 2 + PKW + CH;
static_assert(BMW + CH >= DICT_MAX, "sort buffer");
static_assert(BMW % NT == 0, "bitmap words per thread");

template <bool WRITE, int KIND, typename T>
__device__ __forceinline__ void dict_body(const CzArgs& A, const T* col, int d, uint32_t blk,
                                          uint64_t g0, uint32_t n, uint32_t* sm, Smem& S) {
    const Cols& C = A.col;
    const int sec = KIND == 0 ? SEC_S : SEC_C + (d - 3) / 2;
    uint32_t* meta = A.meta + ((size_t)blk * NSEC + sec) * 2;
    const uint32_t* dDb = A.dD + (size_t)blk * NDICT;
    uint32_t* gd = A.dict + ((size_t)blk * NDICT + d) * A.DC;
    VSet h{sm + HS + 2, sm, sm + HS};
    uint32_t* starts = WRITE ? sm + DICT_MAX + LUTN / 2 + PKW : sm + HS + 2 + BMW;
    const bool vec = (g0 & 3) == 0;                      // columns are 16-byte aligned
    DictOut dout;
    if (WRITE) {
        const uint32_t m = meta[1];
        uint32_t* o = A.out + A.off[(size_t)blk * NSEC + sec];
        uint64_t at = 1;
        if (KIND == 0) {
            const uint32_t nbw = (n + 31) / 32;
            at = nbw;
            for (int k = 0; k < d; ++k) at += dict_words(m, dDb[k]);
            if (d == 0)
                for (uint32_t w = threadIdx.x; w < nbw; w += NT) {
                    uint32_t v = 0;
                    if (vec && w * 32 + 32 <= n) {              // eight four-element loads each
#pragma unroll
                        for (int q = 0; q < 8; ++q) {
                            uint32_t a[IT], b[IT], e[IT];
                            const uint64_t i = g0 + w * 32 + 4 * q;
                            ld4(C.u8[C_AVGQ2], i, true, 4, a);
                            ld4(C.u16[C_CU2 - 8], i, true, 4, b);
                            ld4(C.u16[C_CA2 - 8], i, true, 4, e);
#pragma unroll
                            for (int u = 0; u < IT; ++u)
                                v |= (uint32_t)((a[u] | b[u] | e[u]) != 0) << (4 * q + u);
                        }
                    } else {
                        for (uint32_t i = w * 32; i < n && i < w * 32 + 32; ++i)
                            v |= (uint32_t)s_mask(C, g0 + i) << (i % 32);
                    }
                    o[w] = v;
                }
        } else if (KIND == 1) {
            if (threadIdx.x == 0) o[0] = m;
        } else {
            at = 1 + dict_words(m, dDb[d - 1]);
        }
        do_init(dout, dDb[d], sm, reinterpret_cast<uint16_t*>(sm + DICT_MAX), gd, o + at,
                sm + DICT_MAX + LUTN / 2, m);
    } else {
        vs_clear(h);
    }
    __syncthreads();
    uint32_t R0 = 0, pend_s = 0, mine = 0;
    for (uint32_t c0 = 0; c0 < n; c0 += CH) {
        uint32_t fl[IT], v[IT], cnt = 0;
        const uint32_t s0 = c0 + threadIdx.x * IT;
        const uint32_t left = s0 < n ? n - s0 : 0;
        ld4(col, g0 + s0, vec, left, v);
        if (KIND == 0) {
            uint32_t a[IT], b[IT], e[IT];
            ld4(C.u8[C_AVGQ2], g0 + s0, vec, left, a);
            ld4(C.u16[C_CU2 - 8], g0 + s0, vec, left, b);
            ld4(C.u16[C_CA2 - 8], g0 + s0, vec, left, e);
#pragma unroll
            for (int u = 0; u < IT; ++u) {
                fl[u] = (a[u] | b[u] | e[u]) != 0;
                cnt += fl[u];
            }
        } else {
            uint32_t prev = s0 > 0 && s0 < n ? (uint32_t)col[g0 + s0 - 1] : 0;
#pragma unroll
            for (int u = 0; u < IT; ++u) {
                fl[u] = (uint32_t)u < left && (s0 + u == 0 || v[u] != prev);
                prev = v[u];
                cnt += fl[u];
            }
        }
        if (KIND < 2 && !WRITE) {                       // no order needed: insert, count
#pragma unroll
            for (int u = 0; u < IT; ++u)
                if (fl[u]) vs_insert(h, v[u]);
            mine += cnt;
            continue;
        }
        uint32_t k;
        uint32_t r = cta_scan(cnt, S, &k);
        if (KIND < 2) {                                 // write: element R0 + r is this value
#pragma unroll
            for (int u = 0; u < IT; ++u)
                if (fl[u]) do_add(dout, R0 + r++, v[u]);
            R0 += k;
            __syncthreads();
            if (dout.D != RAW) pk_flush(dout.pk, R0);
            continue;
        }
#pragma unroll
        for (int u = 0; u < IT; ++u)                    // lengths: run R0+e-1 ends at starts[e]
            if (fl[u]) starts[r++] = s0 + u;
        __syncthreads();
        for (uint32_t e = threadIdx.x; e < k; e += NT) {
            if (R0 + e == 0) continue;
            const uint32_t len = starts[e] - (e == 0 ? pend_s : starts[e - 1]);
            if (WRITE) do_add(dout, R0 + e - 1, len);
            else vs_insert(h, len);
        }
        __syncthreads();
        if (k) pend_s = starts[k - 1];
        R0 += k;
        if (WRITE && dout.D != RAW) pk_flush(dout.pk, R0 - 1);
        __syncthreads();
    }
    if (KIND == 2 && threadIdx.x == 0) {                // the last run ends at the block end
        if (WRITE) do_add(dout, R0 - 1, n - pend_s);
        else vs_insert(h, n - pend_s);
    }
    __syncthreads();
    if (WRITE) {
        const uint32_t m = meta[1];
        if (dout.D != RAW) { pk_flush(dout.pk, m); pk_final(dout.pk, m); }
        return;
    }
    if (KIND < 2) cta_scan(mine, S, &R0);
    const uint32_t D = vs_finalize(h, sm + HS + 2, gd, S);
    if (threadIdx.x == 0) {
        A.dD[(size_t)blk * NDICT + d] = D;
        if (d == 0 || KIND == 1) meta[1] = R0;
    }
}

template <bool WRITE>
__global__ void __launch_bounds__(NT, WRITE ? GSNP_CZ_MINB_W : GSNP_CZ_MINB) k_cz_dicts(CzArgs A) {
    extern __shared__ __align__(16) uint32_t sm[];
    __shared__ Smem S;
    const int d = (int)(blockIdx.x % NDICT);
    const uint32_t blk = blockIdx.x / NDICT;
    const uint64_t g0 = (uint64_t)blk * A.B;
    const uint32_t n = (uint32_t)(A.n - g0 < A.B ? A.n - g0 : A.B);
    const Cols& C = A.col;
    switch (d) {
    case 0: dict_body<WRITE, 0>(A, C.u8[C_AVGQ2], d, blk, g0, n, sm, S); break;
    case 1: dict_body<WRITE, 0>(A, C.u16[C_CU2 - 8], d, blk, g0, n, sm, S); break;
    case 2: dict_body<WRITE, 0>(A, C.u16[C_CA2 - 8], d, blk, g0, n, sm, S); break;
    default: {
        const int ci = (d - 3) / 2, c = rle_col(ci);
        const bool len = (d - 3) & 1;
        if (c < 8) {
            if (len) dict_body<WRITE, 2>(A, C.u8[c], d, blk, g0, n, sm, S);
            else dict_body<WRITE, 1>(A, C.u8[c], d, blk, g0, n, sm, S);
        } else if (c < 12) {
            if (len) dict_body<WRITE, 2>(A, C.u16[c - 8], d, blk, g0, n, sm, S);
            else dict_body<WRITE, 1>(A, C.u16[c - 8], d, blk, g0, n, sm, S);
        } else {
            if (len) dict_body<WRITE, 2>(A, C.u32[c - 12], d, blk, g0, n, sm, S);
            else dict_body<WRITE, 1>(A, C.u32[c - 12], d, blk, g0, n, sm, S);
        }
    }
    }
}

// grid nblk * nsec: sections [sec0, sec0 + nsec) < SEC_S of every block (header, planes,
// exception lists; the dictionary sections are k_cz_dicts); WRITE = false sizes the sections, true
// writes them
template <bool WRITE>
__global__ void __launch_bounds__(NT, GSNP_CZ_MINB) k_cz_sections(CzArgs A, int sec0, int nsec) {
    extern __shared__ __align__(16) uint32_t sm[];
    __shared__ Smem S;
    const int sec = sec0 + (int)(blockIdx.x % nsec);    // a block's sections are adjacent in
    const uint32_t blk = blockIdx.x / nsec;            // launch order
    BlockCtx bk;
    bk.blk = blk;
    bk.g0 = (uint64_t)blk * A.B;
    bk.n = (uint32_t)(A.n - bk.g0 < A.B ? A.n - bk.g0 : A.B);
    if (sec == SEC_HDR) {
        if (!WRITE) {
            if (threadIdx.x == 0) { A.meta[(size_t)blk * NSEC * 2] = 6; A.meta[(size_t)blk * NSEC * 2 + 1] = 0; }
        } else if (threadIdx.x == 0) {
            uint32_t* o = A.out + A.off[(size_t)blk * NSEC];
            const uint64_t pos0 = A.rec[bk.g0].pos;
            o[0] = MAGIC;
            o[1] = bk.n;
            o[2] = (uint32_t)pos0;
            o[3] = (uint32_t)(pos0 >> 32);
            o[4] = (uint32_t)(A.off[(size_t)(blk + 1) * NSEC] - A.off[(size_t)blk * NSEC]);
            o[5] = A.B;
        }
        return;
    }
    if (sec == SEC_P) {                               // 2-bit planes of ref, base1, base2
        const uint32_t pw = (bk.n + 15) / 16;
        if (!WRITE) {
            if (threadIdx.x == 0) {
                A.meta[((size_t)blk * NSEC + SEC_P) * 2] = 3 * pw;
                A.meta[((size_t)blk * NSEC + SEC_P) * 2 + 1] = 0;
            }
            return;
        }
        uint32_t* o = A.out + A.off[(size_t)blk * NSEC + SEC_P];
        for (uint32_t t = threadIdx.x; t < 3 * pw; t += NT) {
            const int c = t < pw ? C_REF : t < 2 * pw ? C_BASE1 : C_BASE2;
            const uint32_t w = t % pw;
            uint32_t v = 0;
            const uint8_t* col = A.col.u8[c] + bk.g0 + w * 16;
            if ((bk.g0 & 15) == 0 && w * 16 + 16 <= bk.n) {      // one 16-byte load
                const uint4 q = *reinterpret_cast<const uint4*>(col);
                const uint32_t qw[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
                for (int k = 0; k < 4; ++k)
#pragma unroll
                    for (int b = 0; b < 4; ++b) v |= ((qw[k] >> (8 * b)) & 3u) << (2 * (4 * k + b));
            } else {
                for (uint32_t i = w * 16; i < bk.n && i < w * 16 + 16; ++i)
                    v |= (col[i - w * 16] & 3u) << (2 * (i % 16));
            }
            o[t] = v;
        }
        return;
    }
    sec_exceptions<WRITE>(A, bk, sec, S, sm);
}

// words of section sec of block blk: the light sections' size pass stored them in meta[0]; the
// dictionary sections' come from the element counts and dictionary sizes (k_cz_dicts)
__device__ __forceinline__ uint64_t section_words(const CzArgs& A, uint32_t blk, int sec) {
    const uint32_t* meta = A.meta + ((size_t)blk * NSEC + sec) * 2;
    if (sec < SEC_S) return meta[0];
    const uint32_t* dDb = A.dD + (size_t)blk * NDICT;
    const uint32_t m = meta[1];
    if (sec == SEC_S) {
        const uint64_t g0 = (uint64_t)blk * A.B;
        const uint32_t n = (uint32_t)(A.n - g0 < A.B ? A.n - g0 : A.B);
        return (n + 31) / 32 + dict_words(m, dDb[0]) + dict_words(m, dDb[1]) + dict_words(m, dDb[2]);
    }
    const int d = 3 + 2 * (sec - SEC_C);
    return 1 + dict_words(m, dDb[d]) + dict_words(m, dDb[d + 1]);
}

// exclusive scan of the section sizes (block-major, section-minor = stream order)
__global__ void __launch_bounds__(1024) k_cz_scan(const CzArgs A, uint64_t* off) {
    const uint64_t nsec = (uint64_t)A.nblk * NSEC;
    __shared__ uint64_t ws[33];
    uint64_t carry = 0;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (uint64_t c0 = 0; c0 < nsec; c0 += 1024) {
        const uint64_t i = c0 + threadIdx.x;
        const uint64_t v = i < nsec ? section_words(A, (uint32_t)(i / NSEC), (int)(i % NSEC)) : 0;
        uint64_t x = v;
        for (int d = 1; d < 32; d <<= 1) {
            uint64_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
            if (lane >= d) x += y;
        }
        if (lane == 31) ws[w] = x;
        __syncthreads();
        if (w == 0) {
            uint64_t t = ws[lane], s = t;
            for (int d = 1; d < 32; d <<= 1) {
                uint64_t y = __shfl_up_sync(0xFFFFFFFFu, s, d);
                if (lane >= d) s += y;
            }
            ws[lane] = s - t;
            if (lane == 31) ws[32] = s;
        }
        __syncthreads();
        if (i < nsec) off[i] = carry + ws[w] + x - v;
        carry += ws[32];
        __syncthreads();
    }
    if (threadIdx.x == 0) off[nsec] = carry;
}

// dynamic shared memory of k_cz_sections (words): the header, plane and exception sections need
// only the packer's staging window
constexpr size_t SMEM_LIGHT_WORDS = PKW;
static_assert(PKW * 32 >= (CH + 1) * 12 + 64, "packer window");

}  // namespace gsnp_cz
