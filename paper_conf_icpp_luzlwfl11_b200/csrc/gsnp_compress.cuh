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

// --- hash set of distinct values (dictionary construction, "sort + unique")
struct HSet {
    uint32_t* slot;           // HS words, EMPTY = free
    uint32_t* cnt;            // [0] distinct non-EMPTY values, [1] saw 0xFFFFFFFF
};

__device__ __forceinline__ void hs_clear(HSet h) {
    for (int i = threadIdx.x; i < HS; i += NT) h.slot[i] = EMPTY;
    if (threadIdx.x == 0) { h.cnt[0] = 0; h.cnt[1] = 0; }
}

__device__ __forceinline__ void hs_insert(HSet h, uint32_t v) {
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

// Sorted unique list of the set into gdict (capacity >= D); returns D or RAW.  sb: DICT_MAX words.
__device__ uint32_t hs_finalize(HSet h, uint32_t* sb, uint32_t* gdict, Smem& S) {
    __syncthreads();
    const uint32_t c = h.cnt[0], hasmax = h.cnt[1];
    const uint32_t D = c + hasmax;
    __syncthreads();
    if (D > DICT_MAX) return RAW;
    constexpr int PER = HS / NT;
    uint32_t k = 0;
    for (int i = 0; i < PER; ++i) k += h.slot[threadIdx.x * PER + i] != EMPTY;
    uint32_t tot;
    uint32_t at = cta_scan(k, S, &tot);
    for (int i = 0; i < PER; ++i) {
        uint32_t v = h.slot[threadIdx.x * PER + i];
        if (v != EMPTY) sb[at++] = v;
    }
    uint32_t P2 = 1;
    while (P2 < c) P2 <<= 1;
    for (uint32_t i = c + threadIdx.x; i < P2; i += NT) sb[i] = EMPTY;
    __syncthreads();
    for (uint32_t kk = 2; kk <= P2; kk <<= 1)
        for (uint32_t j = kk >> 1; j > 0; j >>= 1) {
            for (uint32_t i = threadIdx.x; i < P2; i += NT) {
                uint32_t ixj = i ^ j;
                if (ixj > i) {
                    uint32_t a = sb[i], b = sb[ixj];
                    bool up = (i & kk) == 0;
                    if ((a > b) == up) { sb[i] = b; sb[ixj] = a; }
                }
            }
            __syncthreads();
        }
    for (uint32_t i = threadIdx.x; i < c; i += NT) gdict[i] = sb[i];
    if (hasmax && threadIdx.x == 0) gdict[c] = 0xFFFFFFFFu;
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

// --- DICT output of one array: header, dictionary, packed indices (or RAW values)
struct DictOut {
    uint32_t D;
    const uint32_t* sd;       // sorted dictionary in shared memory (D words) unless RAW
    uint32_t* g;              // section start in the output
    Packer pk;
};

__device__ __forceinline__ void do_init(DictOut& d, uint32_t D, uint32_t* sd, const uint32_t* gdict,
                                        uint32_t* g, uint32_t* st, uint64_t m) {
    d.D = D; d.sd = sd; d.g = g;
    if (m == 0) { d.pk.b = 0; return; }
    if (threadIdx.x == 0) g[0] = D;
    if (D == RAW) { d.pk.b = 0; return; }
    for (uint32_t i = threadIdx.x; i < D; i += NT) { uint32_t v = gdict[i]; sd[i] = v; g[1 + i] = v; }
    pk_init(d.pk, st, g + 1 + D, D <= 1 ? 0 : bitlen(D - 1));
}

__device__ __forceinline__ void do_add(const DictOut& d, uint64_t j, uint32_t v) {
    if (d.D == RAW) { d.g[1 + j] = v; return; }
    uint32_t lo = 0, hi = d.D;                 // parallel binary search
    while (lo < hi) {
        uint32_t mid = (lo + hi) >> 1;
        if (d.sd[mid] < v) lo = mid + 1; else hi = mid;
    }
    pk_add(d.pk, j, lo);
}

// ------------------------------------------------------------------------ sections
struct BlockCtx {
    uint64_t g0;              // global index of the block's first record
    uint32_t n;               // records in the block
    uint32_t blk;             // block number
};

// exception-list sections N / G / K / R / Q
template <bool WRITE>
__device__ void sec_exceptions(const CzArgs& A, const BlockCtx& bk, int sec, Smem& S,
                               uint32_t* st) {
    const Cols& C = A.col;
    const uint32_t blk = bk.blk;
    uint32_t* meta = A.meta + ((size_t)blk * NSEC + sec) * 2;
    const uint32_t m = WRITE ? meta[1] : 0;
    uint32_t* o = WRITE ? A.out + A.off[(size_t)blk * NSEC + sec] : nullptr;
    const int ncol = sec == SEC_N ? C_REF : sec == SEC_N + 1 ? C_BASE1 : C_BASE2;   // N: base column
    Packer pk;
    if (WRITE && (sec == SEC_G || sec == SEC_K)) pk_init(pk, st, o + 1 + m, 8);
    if (WRITE && threadIdx.x == 0) o[0] = m;
    uint32_t run = 0, runE = 0;                              // exceptions (N: run starts, ends)
                                                             // before this chunk
    for (uint32_t c0 = 0; c0 < bk.n; c0 += CH) {
        uint32_t fl[IT], vals[IT], cnt = 0;
#pragma unroll
        for (int u = 0; u < IT; ++u) {
            const uint32_t s = c0 + threadIdx.x * IT + u;
            fl[u] = 0;
            vals[u] = 0;
            if (s >= bk.n) continue;
            const uint64_t gi = bk.g0 + s;
            if (sec <= SEC_N + 2) {                          // runs of code 4: start (lo16), end (hi16)
                const bool f = C.u8[ncol][gi] == 4;
                const bool pf = s > 0 && C.u8[ncol][gi - 1] == 4;
                const bool nf = s + 1 < bk.n && C.u8[ncol][gi + 1] == 4;
                fl[u] = (f && !pf ? 1u : 0u) | (f && !nf ? 0x10000u : 0u);
            } else if (sec == SEC_G) {
                const uint32_t r = C.u8[C_REF][gi];
                const uint32_t pred = r < 4 ? (0x09070400u >> (8 * r)) & 255 : 255;   // HOM[ref]
                vals[u] = C.u8[C_GENO][gi];
                fl[u] = vals[u] != pred;
            } else if (sec == SEC_K) {
                vals[u] = C.u8[C_KNOWN][gi];
                fl[u] = vals[u] != 0;
            } else {
                vals[u] = C.u32[sec == SEC_R ? C_RANKP - 12 : C_POST1 - 12][gi];
                fl[u] = vals[u] != ONE;
            }
            cnt += fl[u];
        }
        uint32_t tot;
        uint32_t r = cta_scan(cnt, S, &tot);
        if (WRITE) {
            if (sec <= SEC_N + 2) {
                uint32_t rs = run + (r & 0xFFFF), re = runE + (r >> 16);
#pragma unroll
                for (int u = 0; u < IT; ++u) {
                    const uint32_t s = c0 + threadIdx.x * IT + u;
                    if (fl[u] & 1) o[1 + rs++] = s;
                    if (fl[u] >> 16) o[1 + m + re++] = s + 1;
                }
            } else {
                uint32_t j = run + r;
#pragma unroll
                for (int u = 0; u < IT; ++u) {
                    if (!fl[u]) continue;
                    const uint32_t s = c0 + threadIdx.x * IT + u;
                    o[1 + j] = s;
                    if (sec == SEC_G || sec == SEC_K) pk_add(pk, j, vals[u]);
                    else o[1 + m + j] = vals[u];
                    ++j;
                }
            }
        }
        run += sec <= SEC_N + 2 ? (tot & 0xFFFF) : tot;
        runE += tot >> 16;
        if (WRITE && (sec == SEC_G || sec == SEC_K)) {
            __syncthreads();
            pk_flush(pk, run);
        }
    }
    if (WRITE) {
        if (sec == SEC_G || sec == SEC_K) pk_final(pk, m);
    } else if (threadIdx.x == 0) {
        uint64_t words = sec <= SEC_N + 2 || sec == SEC_R || sec == SEC_Q ? 1 + 2ull * run
                                                                           : 1 + run + (run + 3) / 4;
        meta[0] = (uint32_t)words;
        meta[1] = run;
    }
}

// second-allele section S: bitmap of sites with a non-zero second allele, then
// DICT of avgq2, cnt_uni2, cnt_all2 over those sites in order
__device__ __forceinline__ bool s_mask(const Cols& C, uint64_t gi) {
    return (C.u8[C_AVGQ2][gi] | C.u16[C_CU2 - 8][gi] | C.u16[C_CA2 - 8][gi]) != 0;
}

template <bool WRITE>
__device__ void sec_second(const CzArgs& A, const BlockCtx& bk, Smem& S, uint32_t* sm) {
    const Cols& C = A.col;
    const uint32_t blk = bk.blk;
    uint32_t* meta = A.meta + ((size_t)blk * NSEC + SEC_S) * 2;
    uint32_t* dD = A.dD + (size_t)blk * NDICT;
    uint32_t* gd = A.dict + (size_t)blk * NDICT * A.DC;
    const uint32_t nbw = (bk.n + 31) / 32;
    uint32_t* o = WRITE ? A.out + A.off[(size_t)blk * NSEC + SEC_S] : nullptr;
    const uint32_t m = WRITE ? meta[1] : 0;
    if (WRITE)
        for (uint32_t w = threadIdx.x; w < nbw; w += NT) {
            uint32_t v = 0;
            for (uint32_t i = w * 32; i < bk.n && i < w * 32 + 32; ++i)
                v |= (uint32_t)s_mask(C, bk.g0 + i) << (i % 32);
            o[w] = v;
        }
    uint64_t words = nbw, at = nbw;
    uint32_t mm = 0;
    HSet h{sm, sm + HS};
    uint32_t* sb = sm + HS + 2;
    uint32_t* sd = sm;                               // write pass: dictionary
    uint32_t* st = sm + DICT_MAX;                    //             packer staging
    for (int k = 0; k < 3; ++k) {
        const int c = k == 0 ? C_AVGQ2 : k == 1 ? C_CU2 : C_CA2;
        DictOut d;
        if (WRITE) {
            __syncthreads();
            do_init(d, dD[k], sd, gd + (size_t)k * A.DC, o + at, st, m);
            __syncthreads();
        } else {
            hs_clear(h);
            __syncthreads();
        }
        uint32_t run = 0;
        for (uint32_t c0 = 0; c0 < bk.n; c0 += CH) {
            uint32_t fl[IT], cnt = 0;
#pragma unroll
            for (int u = 0; u < IT; ++u) {
                const uint32_t s = c0 + threadIdx.x * IT + u;
                fl[u] = s < bk.n && s_mask(C, bk.g0 + s);
                cnt += fl[u];
                if (!WRITE && fl[u]) hs_insert(h, colv(C, c, bk.g0 + s));
            }
            if (WRITE) {
                uint32_t tot, j;
                j = run + cta_scan(cnt, S, &tot);
#pragma unroll
                for (int u = 0; u < IT; ++u)
                    if (fl[u]) do_add(d, j++, colv(C, c, bk.g0 + c0 + threadIdx.x * IT + u));
                run += tot;
                __syncthreads();
                if (d.D != RAW) pk_flush(d.pk, run);
            } else {
                uint32_t tot;
                cta_scan(cnt, S, &tot);
                run += tot;
            }
        }
        if (WRITE) {
            if (d.D != RAW) pk_final(d.pk, m);
            at += dict_words(m, dD[k]);
        } else {
            mm = run;
            const uint32_t D = hs_finalize(h, sb, gd + (size_t)k * A.DC, S);
            if (threadIdx.x == 0) dD[k] = D;
            words += dict_words(run, D);
        }
    }
    if (!WRITE && threadIdx.x == 0) {
        meta[0] = (uint32_t)words;
        meta[1] = mm;
    }
}

// quality column sections C0..C5: R, DICT(run values), DICT(run lengths)
template <bool WRITE>
__device__ void sec_rle(const CzArgs& A, const BlockCtx& bk, int ci, Smem& S, uint32_t* sm) {
    const Cols& C = A.col;
    const uint32_t blk = bk.blk;
    const int sec = SEC_C + ci;
    const int c = ci == 0 ? C_QUAL : ci == 1 ? C_AVGQ1 : ci == 2 ? C_CU1 : ci == 3 ? C_CA1
                : ci == 4 ? C_DEPTH : C_COPYN;
    uint32_t* meta = A.meta + ((size_t)blk * NSEC + sec) * 2;
    uint32_t* dD = A.dD + (size_t)blk * NDICT + 3 + 2 * ci;
    uint32_t* gd = A.dict + ((size_t)blk * NDICT + 3 + 2 * ci) * A.DC;
    // shared layout: starts[CH], startv[CH], then (size) 2 hash sets + sort buffer
    //                                               (write) 2 dictionaries + 2 packer windows
    uint32_t* starts = sm;
    uint32_t* startv = sm + CH;
    uint32_t* rest = sm + 2 * CH;
    HSet hv{rest, rest + 2 * HS}, hl{rest + HS, rest + 2 * HS + 2};
    uint32_t* sb = rest + 2 * HS + 4;
    DictOut dv, dl;
    const uint32_t R = WRITE ? meta[1] : 0;
    if (WRITE) {
        uint32_t* o = A.out + A.off[(size_t)blk * NSEC + sec];
        if (threadIdx.x == 0) o[0] = R;
        do_init(dv, dD[0], rest, gd, o + 1, rest + 2 * DICT_MAX, R);
        do_init(dl, dD[1], rest + DICT_MAX, gd + A.DC, o + 1 + dict_words(R, dD[0]),
                rest + 2 * DICT_MAX + PKW, R);
    } else {
        hs_clear(hv);
        hs_clear(hl);
    }
    __syncthreads();
    uint32_t R0 = 0, pend_s = 0, pend_v = 0;          // runs started so far; the open run
    for (uint32_t c0 = 0; c0 < bk.n; c0 += CH) {
        uint32_t fl[IT], v[IT], cnt = 0;
        const uint32_t s0 = c0 + threadIdx.x * IT;
        uint32_t prev = s0 > 0 && s0 < bk.n ? colv(C, c, bk.g0 + s0 - 1) : 0;
#pragma unroll
        for (int u = 0; u < IT; ++u) {
            const uint32_t s = s0 + u;
            fl[u] = 0;
            if (s >= bk.n) continue;
            v[u] = colv(C, c, bk.g0 + s);
            fl[u] = s == 0 || v[u] != prev;
            prev = v[u];
            cnt += fl[u];
        }
        uint32_t k;
        uint32_t r = cta_scan(cnt, S, &k);
#pragma unroll
        for (int u = 0; u < IT; ++u)
            if (fl[u]) { starts[r] = s0 + u; startv[r] = v[u]; ++r; }
        __syncthreads();
        // run R0+e-1 ends at starts[e]
        for (uint32_t e = threadIdx.x; e < k; e += NT) {
            if (R0 + e == 0) continue;
            const uint32_t rs = e == 0 ? pend_s : starts[e - 1];
            const uint32_t rv = e == 0 ? pend_v : startv[e - 1];
            const uint32_t len = starts[e] - rs;
            if (WRITE) {
                do_add(dv, R0 + e - 1, rv);
                do_add(dl, R0 + e - 1, len);
            } else {
                hs_insert(hv, rv);
                hs_insert(hl, len);
            }
        }
        __syncthreads();
        if (k) { pend_s = starts[k - 1]; pend_v = startv[k - 1]; }
        R0 += k;
        if (WRITE) {
            if (dv.D != RAW) pk_flush(dv.pk, R0 - 1);
            if (dl.D != RAW) pk_flush(dl.pk, R0 - 1);
        }
        __syncthreads();
    }
    // the last run ends at the block end
    if (threadIdx.x == 0) {
        if (WRITE) {
            do_add(dv, R0 - 1, pend_v);
            do_add(dl, R0 - 1, bk.n - pend_s);
        } else {
            hs_insert(hv, pend_v);
            hs_insert(hl, bk.n - pend_s);
        }
    }
    __syncthreads();
    if (WRITE) {
        if (dv.D != RAW) { pk_flush(dv.pk, R); pk_final(dv.pk, R); }
        if (dl.D != RAW) { pk_flush(dl.pk, R); pk_final(dl.pk, R); }
    } else {
        const uint32_t DV = hs_finalize(hv, sb, gd, S);
        const uint32_t DL = hs_finalize(hl, sb, gd + A.DC, S);
        if (threadIdx.x == 0) {
            dD[0] = DV;
            dD[1] = DL;
            meta[0] = (uint32_t)(1 + dict_words(R0, DV) + dict_words(R0, DL));
            meta[1] = R0;
        }
    }
}

// grid nblk * nsec: sections [sec0, sec0 + nsec) of every block (the exception-list sections and
// the dictionary sections are launched apart, each with the shared memory it needs, so the light
// ones run four CTAs per SM); WRITE = false sizes the sections, true writes them
template <bool WRITE>
__global__ void __launch_bounds__(NT) k_cz_sections(CzArgs A, int sec0, int nsec) {
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
            for (uint32_t i = w * 16; i < bk.n && i < w * 16 + 16; ++i)
                v |= (A.col.u8[c][bk.g0 + i] & 3u) << (2 * (i % 16));
            o[t] = v;
        }
        return;
    }
    if (sec < SEC_S) sec_exceptions<WRITE>(A, bk, sec, S, sm);
    else if (sec == SEC_S) sec_second<WRITE>(A, bk, S, sm);
    else sec_rle<WRITE>(A, bk, sec - SEC_C, S, sm);
}

// exclusive scan of the section sizes (block-major, section-minor = stream order)
__global__ void __launch_bounds__(1024) k_cz_scan(const uint32_t* meta, uint64_t nsec, uint64_t* off) {
    __shared__ uint64_t ws[33];
    uint64_t carry = 0;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (uint64_t c0 = 0; c0 < nsec; c0 += 1024) {
        const uint64_t i = c0 + threadIdx.x;
        const uint64_t v = i < nsec ? meta[i * 2] : 0;
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

// dynamic shared memory of k_cz_sections (words): the RLE section is the largest user; the
// header, plane and exception sections need only the packer's staging window
constexpr size_t SMEM_LIGHT_WORDS = PKW;
constexpr size_t SMEM_SIZE_WORDS = 2 * CH + 2 * HS + 4 + DICT_MAX;
constexpr size_t SMEM_WRITE_WORDS = 2 * CH + 2 * DICT_MAX + 2 * PKW;
static_assert(HS + 2 + DICT_MAX <= SMEM_SIZE_WORDS, "S section (size pass) fits");
static_assert(DICT_MAX + PKW <= SMEM_WRITE_WORDS, "S section (write pass) fits");
static_assert(PKW * 32 >= (CH + 1) * 12 + 64, "packer window");

}  // namespace gsnp_cz
