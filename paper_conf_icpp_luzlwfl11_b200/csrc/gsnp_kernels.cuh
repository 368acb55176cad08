// gsnp_kernels.cuh — device code of libgsnp (sm_100a).  Included once, by gsnp.cu.
//
// Kernels:
//   k_validate_reads  ABI checks on the read arrays (sortedness P:L208-210, ranges)
//   k_calib_count     a1: calibration histogram C[q][cyc][t][o] (cal_p_matrix)
//   k_tile_ranges     a3: per 32-site group, read range [lower_bound(s0-L+1), lower_bound(s1))
//   k_call_tile       a4..a8 fused, one thread per site: counting and
//                     base_word gather walking the sorted reads, likelihood_sort
//                     as an in-register bitonic network bucketed by segment length (multipass,
//                     P:L533-567; deeper sites on the warp / CTA paths), dependency adjust +
//                     likelihood (Alg. 4) from the score table T (Alg. 3,
//                     P:L577-610), posterior, call, rank-sum, record.  Keys never reach HBM.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "gsnp.h"

namespace gsnp_dev {

constexpr int NT = 256;               // threads per CTA
constexpr int NW = NT / 32;           // warps per CTA
constexpr uint32_t FULL = 0xFFFFFFFFu;
constexpr uint32_t KEY_INF = 0xFFFFFFFFu;

enum : int { ERR_RANGE = 1, ERR_UNSORTED = 2, ERR_DEEP = 4, ERR_QUAL = 8 };

struct DevReads {
    const uint64_t* pos;
    const uint16_t* len;
    const uint64_t* off;
    const uint8_t* bases;
    const uint8_t* quals;
    const uint8_t* strand;
    const uint16_t* hits;
    uint64_t n;
    uint64_t off0;                    // bases index of read r, base i = off[r] - off0 + i
};

struct CallArgs {
    DevReads R;
    const uint8_t* ref;               // reference codes, ref[site - origin]
    uint64_t origin, n_sites;
    const uint32_t* known_bits;       // bit (site - origin): site is a known SNP
    const uint64_t* known_pos;        // sorted
    const double* known_lp;           // n_known x 10 log10 priors (host-built)
    uint64_t n_known;
    const double* LP;                 // [5][10] log10 novel priors per reference code (R6)
    const double* T;                  // [64][L][4][10] score table (Alg. 3)
    const uint8_t* adj;               // [64][adjP][adjG] adjust table (R3)
    int adjP, adjG;
    int L, q_max;
    uint32_t flags;
    uint64_t w0, w1;                  // window
    const uint64_t* tile_ra;          // per 32-site group read range [ra, rb)
    const uint64_t* tile_rb;
    gsnp_record* out;                 // out[site - w0]
    int* err;
    // debug (all may be null)
    uint32_t* dbg_nuni;               // count-only pass: unique keys per site
    const uint32_t* dbg_off;          // CSR offsets for the key dumps
    uint32_t* dbg_keys_built;
    uint32_t* dbg_keys_sorted;
    uint32_t* dbg_counters;           // [S][15]
    double* dbg_L10;
    double* dbg_post10;
    int count_only;
};

__device__ __forceinline__ uint32_t lanemask_lt() {
    uint32_t m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// lower_bound over a sorted global array
__device__ __forceinline__ uint64_t lower_bound_u64(const uint64_t* a, uint64_t lo, uint64_t hi,
                                                    uint64_t v) {
    while (lo < hi) {
        uint64_t mid = lo + ((hi - lo) >> 1);
        if (a[mid] < v) lo = mid + 1; else hi = mid;
    }
    return lo;
}

// ------------------------------------------------------------------------------------------
// k_validate_reads: one thread per read.
__global__ void k_validate_reads(DevReads R, uint64_t origin, uint64_t n_sites, int L, int* err) {
    uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (r >= R.n) return;
    uint64_t p = R.pos[r];
    uint32_t l = R.len[r];
    int e = 0;
    if (l == 0 || l > (uint32_t)L) e |= ERR_RANGE;
    if (R.hits[r] == 0 || R.strand[r] > 1) e |= ERR_RANGE;
    if (p < origin || p + l > origin + n_sites) e |= ERR_RANGE;
    if (R.off[r] < R.off0 || R.off[r] + l > R.off[r + 1]) e |= ERR_RANGE;
    if (r > 0 && R.pos[r - 1] > p) e |= ERR_UNSORTED;
    if (e) atomicOr(err, e);
}

// ------------------------------------------------------------------------------------------
// Flattened warp loop over the bases of reads [ra, rb): 32 reads' metadata are staged in a
// per-warp shared slot; lanes then walk the concatenated bases so every lane has work.
struct WarpMeta {
    uint64_t pos[32];
    uint64_t off[32];
    uint32_t pre[33];                 // prefix of lengths
    uint16_t hits[32];
    uint8_t strand[32];
    uint16_t len[32];
};

template <typename F>
__device__ __forceinline__ void for_each_base(const DevReads& R, uint64_t ra, uint64_t rb,
                                              WarpMeta& m, int warp, int nwarps, F&& f) {
    const int lane = threadIdx.x & 31;
    for (uint64_t b0 = ra + (uint64_t)warp * 32; b0 < rb; b0 += (uint64_t)nwarps * 32) {
        uint64_t r = b0 + lane;
        uint32_t l = 0;
        if (r < rb) {
            l = R.len[r];
            m.pos[lane] = R.pos[r];
            m.off[lane] = R.off[r] - R.off0;
            m.hits[lane] = R.hits[r];
            m.strand[lane] = R.strand[r];
            m.len[lane] = (uint16_t)l;
        }
        uint32_t inc = l;                                  // warp inclusive scan of lengths
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            uint32_t y = __shfl_up_sync(FULL, inc, d);
            if (lane >= d) inc += y;
        }
        m.pre[lane + 1] = inc;
        if (lane == 0) m.pre[0] = 0;
        __syncwarp();
        uint32_t total = m.pre[32];
        int k = 0;
        for (uint32_t fi = lane; fi < total; fi += 32) {
            while (m.pre[k + 1] <= fi) ++k;
            f(k, fi - m.pre[k], m);
        }
        __syncwarp();
    }
}

// ------------------------------------------------------------------------------------------
// a1: calibration histogram.  Diagonal cells (t == o, ~98% of bases) go to a shared
// [q][cyc][t] u32 histogram flushed once per CTA; mismatches go straight to global u64 REDs.
struct CalibArgs {
    DevReads R;
    const uint8_t* ref;
    uint64_t origin, n_sites;
    const uint32_t* known_bits;
    int L, q_max;
    unsigned long long* C;            // [64][256][4][4]
    int* err;
    int smem_diag;                    // 1 if the diagonal histogram lives in shared memory
};

__global__ void __launch_bounds__(NT) k_calib_count(CalibArgs A) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ WarpMeta wm[NW];
    uint32_t* diag = reinterpret_cast<uint32_t*>(smem);
    const int nd = (A.q_max + 1) * A.L * 4;
    if (A.smem_diag)
        for (int i = threadIdx.x; i < nd; i += NT) diag[i] = 0;
    __syncthreads();
    const int warp = threadIdx.x >> 5;
    // this CTA's share of the reads
    uint64_t per = (A.R.n + gridDim.x - 1) / gridDim.x;
    uint64_t ra = min(A.R.n, (uint64_t)blockIdx.x * per), rb = min(A.R.n, ra + per);
    for_each_base(A.R, ra, rb, wm[warp], warp, NW, [&](int k, uint32_t i, WarpMeta& m) {
        if (m.hits[k] != 1) return;
        uint64_t site = m.pos[k] + i;
        uint64_t bi = m.off[k] + i;
        uint32_t o = A.R.bases[bi], q = A.R.quals[bi];
        if (o > 4) { atomicOr(A.err, ERR_RANGE); return; }
        if (q > (uint32_t)A.q_max) { atomicOr(A.err, ERR_QUAL); return; }
        if (site < A.origin || site >= A.origin + A.n_sites) return;   // flagged by validate
        uint64_t rs = site - A.origin;
        uint32_t t = A.ref[rs];
        if (t == 4 || o == 4) return;
        if ((A.known_bits[rs >> 5] >> (rs & 31)) & 1u) return;
        uint32_t cyc = m.strand[k] ? m.len[k] - 1 - i : i;
        if (t == o && A.smem_diag) atomicAdd(&diag[(q * A.L + cyc) * 4 + t], 1u);
        else atomicAdd(&A.C[q << 12 | cyc << 4 | t << 2 | o], 1ull);
    });
    __syncthreads();
    if (A.smem_diag)
        for (int i = threadIdx.x; i < nd; i += NT) {
            uint32_t v = diag[i];
            if (v) {
                int t = i & 3, cyc = (i >> 2) % A.L, q = (i >> 2) / A.L;
                atomicAdd(&A.C[q << 12 | cyc << 4 | t << 2 | t], (unsigned long long)v);
            }
        }
}
// ------------------------------------------------------------------------------------------
// a3: read ranges.  For each group of 32 consecutive sites [s0, s0+32) (one warp of
// k_call_tile), the reads that can touch it: pos in [s0 - L + 1, s0 + 32) (input sorted by
// position).
__global__ void k_tile_ranges(const uint64_t* pos, uint64_t n, uint64_t w0, uint64_t w1, int L,
                              uint64_t n_groups, uint64_t* ra, uint64_t* rb) {
    uint64_t g = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (g >= n_groups) return;
    uint64_t s0 = w0 + g * 32, s1 = min(w1, s0 + 32);
    uint64_t lo = s0 >= (uint64_t)(L - 1) ? s0 - (L - 1) : 0;
    ra[g] = lower_bound_u64(pos, 0, n, lo);
    rb[g] = lower_bound_u64(pos, ra[g], n, s1);
}

// ------------------------------------------------------------------------------------------
// k_call_tile: one CTA = TS = 256 consecutive sites, one thread per site (GSNP's baseline
// parallelisation).  Shared-memory layout (host: call_smem_bytes()).
constexpr int TS = NT;
constexpr int COLS = 32;              // key slots per site on the thread-per-site path
constexpr int WBUF = 256;             // per-warp key buffer of the warp path (n <= 256)

struct TileSmem {
    uint32_t* col;       // [COLS][TS] keys in gather order; reused as the CTA deep buffer
    uint32_t* wbuf;      // [NW][WBUF]
    uint8_t* slotcnt;    // [NW][4 * 2L] per-warp (base, strand, coord) counters
    uint32_t* cnt_all;   // [4][TS]
    uint32_t* rep;       // [TS]
    uint32_t* nuni;      // [TS]
    int deep_cap;        // keys the col region holds
};

__host__ __device__ inline size_t align16(size_t x) { return (x + 15) & ~size_t(15); }

__host__ __device__ inline size_t call_smem_bytes(int L, TileSmem* s, unsigned char* base) {
    size_t o = 0;
    auto take = [&](size_t bytes) { size_t r = o; o = align16(o + bytes); return r; };
    size_t o_col = take(4 * (size_t)COLS * TS);
    size_t o_wbuf = take(4 * (size_t)NW * WBUF);
    size_t o_slot = take((size_t)NW * 8 * L);
    size_t o_cnt = take(16 * (size_t)TS);
    size_t o_rep = take(4 * (size_t)TS);
    size_t o_nuni = take(4 * (size_t)TS);
    if (s) {
        s->col = reinterpret_cast<uint32_t*>(base + o_col);
        s->wbuf = reinterpret_cast<uint32_t*>(base + o_wbuf);
        s->slotcnt = base + o_slot;
        s->cnt_all = reinterpret_cast<uint32_t*>(base + o_cnt);
        s->rep = reinterpret_cast<uint32_t*>(base + o_rep);
        s->nuni = reinterpret_cast<uint32_t*>(base + o_nuni);
        s->deep_cap = COLS * TS;
    }
    return o;
}

__device__ __forceinline__ uint32_t key_base(uint32_t k) { return (k >> 15) & 3u; }
__device__ __forceinline__ uint32_t key_q(uint32_t k) { return 63u - ((k >> 9) & 63u); }
__device__ __forceinline__ uint32_t key_cyc(uint32_t k) { return (k >> 1) & 255u; }
__device__ __forceinline__ uint32_t key_slot(uint32_t k) { return k & 511u; }   // cyc<<1|strand
constexpr uint32_t KEY_BSLOT = (3u << 15) | 511u;                               // base + slot

// Score-table row of Alg. 3: 10 consecutive doubles at ((qa*L + coord)*4 + base)*10.
__device__ __forceinline__ void add_row(const double* __restrict__ T, int L, uint32_t qa,
                                        uint32_t cyc, uint32_t b, double* acc) {
    const double2* row =
        reinterpret_cast<const double2*>(T + ((size_t)(qa * (uint32_t)L + cyc) * 4u + b) * 10u);
    double2 v0 = __ldg(row + 0), v1 = __ldg(row + 1), v2 = __ldg(row + 2), v3 = __ldg(row + 3),
            v4 = __ldg(row + 4);
    acc[0] += v0.x; acc[1] += v0.y; acc[2] += v1.x; acc[3] += v1.y; acc[4] += v2.x;
    acc[5] += v2.y; acc[6] += v3.x; acc[7] += v3.y; acc[8] += v4.x; acc[9] += v4.y;
}

// adjust(score, dep_count) through the host-built table (R3): adj[q][min(pcr,P)-1][min(g,G-1)]
__device__ __forceinline__ int adj_lookup(const CallArgs& A, uint32_t q, uint32_t pcr, uint32_t g) {
    uint32_t pi = min(pcr, (uint32_t)A.adjP) - 1u, gi = min(g, (uint32_t)A.adjG - 1u);
    return __ldg(A.adj + ((size_t)q * A.adjP + pi) * A.adjG + gi);
}

// ---- per-site epilogue helpers ---------------------------------------------------------------
__device__ __forceinline__ uint32_t pick4(uint32_t v0, uint32_t v1, uint32_t v2, uint32_t v3, int i) {
    return i == 0 ? v0 : i == 1 ? v1 : i == 2 ? v2 : v3;
}
__device__ __forceinline__ uint32_t f16(uint64_t pack, int b) { return (uint32_t)(pack >> (16 * b)) & 0xFFFFu; }

// Top-2 genotypes over lp (ties -> lowest n, R7).
__device__ __forceinline__ void top2(const double* lp, int& t1, int& t2) {
    t1 = 0;
#pragma unroll
    for (int k = 1; k < 10; ++k) if (lp[k] > lp[t1]) t1 = k;
    t2 = t1 == 0 ? 1 : 0;
#pragma unroll
    for (int k = 0; k < 10; ++k) if (k != t1 && lp[k] > lp[t2]) t2 = k;
}

// genotype n -> alleles, Alg. 4 lines 13-17 order (AA AC AT AG CC CT CG TT TG GG)
__device__ __forceinline__ int geno_a1(int t) { return t < 4 ? 0 : t < 7 ? 1 : t < 9 ? 2 : 3; }
__device__ __forceinline__ int geno_a2(int t) {
    return t < 4 ? t : t < 7 ? t - 3 : t < 9 ? t - 5 : 3;
}

// Known-SNP lookup of a site: the row index into known_lp, or -1 (novel prior, R6).
__device__ __forceinline__ int64_t known_index(const CallArgs& A, uint64_t site) {
    const uint64_t rs = site - A.origin;
    if (!((__ldg(A.known_bits + (rs >> 5)) >> (rs & 31)) & 1u)) return -1;
    return (int64_t)lower_bound_u64(A.known_pos, 0, A.n_known, site);
}

// C8/C9 and the 40-byte record (R8, R9).  Out of line: every path shares one copy.
// cu/qs: unique counts / quality sums per base; ca: all-hits counts; delta = lp[t1] - lp[t2];
// wsum/tie: rank-sum pieces (valid for heterozygous calls with both alleles observed).
__device__ __noinline__ void site_record(const CallArgs& A, uint64_t site, int refb, int known,
                                         int t1, double delta, double post1, uint32_t cu0,
                                         uint32_t cu1, uint32_t cu2, uint32_t cu3, uint32_t qs0,
                                         uint32_t qs1, uint32_t qs2, uint32_t qs3, uint32_t ca0,
                                         uint32_t ca1, uint32_t ca2, uint32_t ca3, uint32_t repeat,
                                         double wsum, double tie) {
    const uint64_t s = site - A.w0;
    const int a1 = geno_a1(t1), a2 = geno_a2(t1);
    const uint32_t dep_uni = cu0 + cu1 + cu2 + cu3;
    const uint32_t depth = ca0 + ca1 + ca2 + ca3;
    // C8 rank-sum (normal approximation with tie correction)
    double rank_p = 1.0;
    if (a1 != a2 && (A.flags & GSNP_RANK_SUM)) {
        const uint32_t n1 = pick4(cu0, cu1, cu2, cu3, a1), n2 = pick4(cu0, cu1, cu2, cu3, a2);
        if (n1 == 0 || n2 == 0) rank_p = 0.0;
        else {
            double n1d = (double)n1, n2d = (double)n2, Nd = (double)(n1 + n2);
            double mu = n1d * (Nd + 1.0) / 2.0;
            double var = n1d * n2d / 12.0 * ((Nd + 1.0) - tie / (Nd * (Nd - 1.0)));
            if (!(var > 0.0)) rank_p = 1.0;
            else {
                double z = (wsum - mu) / sqrt(var);
                rank_p = erfc(fabs(z) / sqrt(2.0));
            }
        }
    }
    // C9 best / second base: rank by q_sum among unique bases (by count_all if none), ties to
    // the lower code.  rank(b) = #{b' present: score(b') > score(b) or (== and b' < b)}.
    const bool uni = dep_uni > 0;
    const uint32_t sc[4] = {uni ? qs0 : ca0, uni ? qs1 : ca1, uni ? qs2 : ca2, uni ? qs3 : ca3};
    const uint32_t pr[4] = {uni ? cu0 : ca0, uni ? cu1 : ca1, uni ? cu2 : ca2, uni ? cu3 : ca3};
    int base1 = -1, base2 = -1, npres = 0;
#pragma unroll
    for (int b = 0; b < 4; ++b) {
        int rk = 0;
#pragma unroll
        for (int c = 0; c < 4; ++c)
            if (c != b && pr[c] > 0 && (sc[c] > sc[b] || (sc[c] == sc[b] && c < b))) ++rk;
        if (pr[b] > 0) {
            ++npres;
            if (rk == 0) base1 = b;
            if (rk == 1) base2 = b;
        }
    }
    if (npres == 0) { base1 = refb; base2 = 4; }
    else if (npres == 1) base2 = base1 != refb ? refb : 4;
    int qsc = rank_p == 0.0 ? 0
              : (int)(10.0 * delta + (rank_p == 1.0 ? 0.0 : 10.0 * log10(rank_p)));
    const uint32_t qb1 = base1 < 4 ? pick4(qs0, qs1, qs2, qs3, base1) : 0u;
    const uint32_t qb2 = base2 < 4 ? pick4(qs0, qs1, qs2, qs3, base2) : 0u;
    if (a1 == a2) {
        if (dep_uni > 0 && base1 != a1) qsc = 0;
        else {
            int c1 = (int)qb1 - (int)qb2;
            if (c1 < qsc) qsc = c1;
        }
    } else {
        if (pick4(ca0, ca1, ca2, ca3, a1) > 0 && pick4(ca0, ca1, ca2, ca3, a2) > 0) {
            uint32_t x = pick4(qs0, qs1, qs2, qs3, a1), y = pick4(qs0, qs1, qs2, qs3, a2);
            int c2 = (int)(x < y ? x : y);
            if (c2 < qsc) qsc = c2;
        } else qsc = 0;
    }
    if (dep_uni == 0) qsc = 0;
    qsc = qsc < 0 ? 0 : qsc > 99 ? 99 : qsc;
    const int geno = (refb == 4 && depth == 0) ? 255 : t1;
    auto sat = [](uint32_t x) -> uint32_t { return x > 65535u ? 65535u : x; };
    const uint32_t u1 = base1 < 4 ? pick4(cu0, cu1, cu2, cu3, base1) : 0u;
    const uint32_t u2 = base2 < 4 ? pick4(cu0, cu1, cu2, cu3, base2) : 0u;
    const uint32_t l1 = base1 < 4 ? pick4(ca0, ca1, ca2, ca3, base1) : 0u;
    const uint32_t l2 = base2 < 4 ? pick4(ca0, ca1, ca2, ca3, base2) : 0u;
    const uint32_t avg1 = u1 ? qb1 / u1 : 0u, avg2 = u2 ? qb2 / u2 : 0u;
    const float copy_num = depth ? (float)((double)repeat / (double)depth) : 0.0f;
    const uint64_t w1 = (uint64_t)refb | (uint64_t)(geno & 255) << 8 |
                        (uint64_t)(geno == 255 ? 0 : qsc) << 16 | (uint64_t)base1 << 24 |
                        (uint64_t)base2 << 32 | (uint64_t)(avg1 & 255) << 40 |
                        (uint64_t)(avg2 & 255) << 48 | (uint64_t)(known ? 1 : 0) << 56;
    const uint64_t w2 = (uint64_t)sat(u1) | (uint64_t)sat(l1) << 16 | (uint64_t)sat(u2) << 32 |
                        (uint64_t)sat(l2) << 48;
    const uint64_t w3 = (uint64_t)depth | (uint64_t)__float_as_uint((float)rank_p) << 32;
    const uint64_t w4 = (uint64_t)__float_as_uint(copy_num) |
                        (uint64_t)__float_as_uint((float)post1) << 32;
    uint64_t* o = reinterpret_cast<uint64_t*>(A.out + s);
    o[0] = site; o[1] = w1; o[2] = w2; o[3] = w3; o[4] = w4;
    if (A.dbg_counters) {
        uint32_t* c = A.dbg_counters + s * 15;
        c[0] = depth; c[1] = dep_uni; c[2] = repeat;
        c[3] = ca0; c[4] = ca1; c[5] = ca2; c[6] = ca3;
        c[7] = cu0; c[8] = cu1; c[9] = cu2; c[10] = cu3;
        c[11] = qs0; c[12] = qs1; c[13] = qs2; c[14] = qs3;
    }
}

// ------------------------------------------------------------------------------------------
// Thread-per-site likelihood for n <= N <= 32 keys (the common case).  Keys come from the
// site's shared-memory column, are sorted by an in-register bitonic network (likelihood_sort),
// then Alg. 4 runs sequentially in canonical order — the same terms in the same order as the
// oracle — followed by C7 and the record.
template <int N>
__device__ __forceinline__ void sort_net(uint32_t (&k)[N]) {
#pragma unroll
    for (int size = 2; size <= N; size <<= 1)
#pragma unroll
        for (int stride = size >> 1; stride > 0; stride >>= 1)
#pragma unroll
            for (int i = 0; i < N; ++i) {
                const int j = i ^ stride;
                if (j > i) {
                    const bool up = (i & size) == 0;
                    const uint32_t a = k[i], b = k[j];
                    k[i] = up ? min(a, b) : max(a, b);
                    k[j] = up ? max(a, b) : min(a, b);
                }
            }
}

template <int N>
__device__ __forceinline__ void thread_site(const CallArgs& A, const TileSmem& sm, uint64_t site,
                                            uint32_t n, bool dup, uint32_t ca0, uint32_t ca1,
                                            uint32_t ca2, uint32_t ca3, uint32_t rep,
                                            const double* sLP) {
    const int tid = threadIdx.x;
    uint32_t k[N];
#pragma unroll
    for (int j = 0; j < N; ++j) k[j] = (j < (int)n) ? sm.col[j * TS + tid] : KEY_INF;
    sort_net<N>(k);
    if (A.dbg_keys_sorted) {
        const uint32_t o = A.dbg_off[site - A.w0];
#pragma unroll
        for (int j = 0; j < N; ++j) if (j < (int)n) A.dbg_keys_sorted[o + j] = k[j];
    }
    // Alg. 4 lines 6-17: dep_count reset per base (l.8-11); pcr = occurrences of this
    // (strand, coord) so far; g = distinct (strand, coord) so far - 1 (R3).  Without duplicate
    // slots (checked during the gather) pcr == 1 and g = position within the base's run.
    double acc[10];
#pragma unroll
    for (int j = 0; j < 10; ++j) acc[j] = 0.0;
    uint64_t cu = 0, qs = 0;
    uint32_t prev_b = 4, distinct = 0;
#pragma unroll
    for (int j = 0; j < N; ++j) {
        if (j < (int)n) {
            const uint32_t kk = k[j], b = key_base(kk), q = key_q(kk);
            uint32_t pcr = 1;
            if (dup) {
#pragma unroll
                for (int i = 0; i < j; ++i) pcr += ((k[i] ^ kk) & KEY_BSLOT) == 0;
            }
            if (b != prev_b) { distinct = 0; prev_b = b; }
            distinct += pcr == 1;
            const int qa = adj_lookup(A, q, pcr, distinct - 1);
            add_row(A.T, A.L, (uint32_t)qa, key_cyc(kk), b, acc);
            cu += 1ull << (16 * b);
            qs += (uint64_t)q << (16 * b);
        }
    }
    // C6/C7: priors, posterior, top-2
    const int refb = A.ref[site - A.origin];
    const int64_t kidx = known_index(A, site);
    const double* prow = kidx >= 0 ? A.known_lp + kidx * 10 : sLP + refb * 10;
    double lp[10], m = -INFINITY;
#pragma unroll
    for (int j = 0; j < 10; ++j) {
        lp[j] = acc[j] + prow[j];
        m = lp[j] > m ? lp[j] : m;
    }
    int t1, t2;
    top2(lp, t1, t2);
    double esum = 0.0;
#pragma unroll
    for (int j = 0; j < 10; ++j) esum += exp10(lp[j] - m);
    // C8 pieces: W = sum of pooled mid-ranks of allele-1 qualities; tie = sum(t^3 - t)
    const int a1 = geno_a1(t1), a2 = geno_a2(t1);
    double wsum = 0.0, tie = 0.0;
    if (a1 != a2 && (A.flags & GSNP_RANK_SUM) && f16(cu, a1) && f16(cu, a2)) {
#pragma unroll 1
        for (int x = 0; x < (int)n; ++x) {
            uint32_t xk = sm.col[x * TS + tid];
            const uint32_t xb = key_base(xk), xq = key_q(xk);
            if (xb != (uint32_t)a1 && xb != (uint32_t)a2) continue;
            uint32_t less = 0, eq = 0;
#pragma unroll 1
            for (int y = 0; y < (int)n; ++y) {
                const uint32_t yk = sm.col[y * TS + tid], yb = key_base(yk), yq = key_q(yk);
                const bool yin = yb == (uint32_t)a1 || yb == (uint32_t)a2;
                less += yin && yq < xq;
                eq += yin && yq == xq;
            }
            if (xb == (uint32_t)a1) wsum += (double)less + ((double)eq + 1.0) / 2.0;
            tie += (double)eq * (double)eq - 1.0;
        }
    }
    if (A.dbg_L10 || A.dbg_post10) {
        const uint64_t s = site - A.w0;
        for (int j = 0; j < 10; ++j) {
            if (A.dbg_L10) A.dbg_L10[s * 10 + j] = acc[j];
            if (A.dbg_post10) A.dbg_post10[s * 10 + j] = exp10(lp[j] - m) / esum;
        }
    }
    site_record(A, site, refb, kidx >= 0, t1, lp[t1] - lp[t2], 1.0 / esum, f16(cu, 0), f16(cu, 1),
                f16(cu, 2), f16(cu, 3), f16(qs, 0), f16(qs, 1), f16(qs, 2), f16(qs, 3), ca0, ca1,
                ca2, ca3, rep, wsum, tie);
}

// ------------------------------------------------------------------------------------------
// Warp path for 32 < n <= 256: the warp gathers the site's keys into its buffer, sorts them
// with a K-per-lane bitonic network, and walks Alg. 4 chunk by chunk (32 keys per chunk) with
// match_any for same-slot peers and per-warp shared counters across chunks.
__device__ __forceinline__ void group_epilogue(const CallArgs& A, uint64_t site, int refb,
                                               int64_t kidx, const double* sLP, const double* L10,
                                               const uint32_t* cu, const uint32_t* qs,
                                               uint32_t ca0, uint32_t ca1, uint32_t ca2,
                                               uint32_t ca3, uint32_t rep, double wsum,
                                               double tie) {
    const int lane = threadIdx.x & 31;
    double lp[10], m = -INFINITY;
    const double* prow = kidx >= 0 ? A.known_lp + kidx * 10 : sLP + refb * 10;
#pragma unroll
    for (int n = 0; n < 10; ++n) {
        lp[n] = L10[n] + prow[n];
        m = lp[n] > m ? lp[n] : m;
    }
    int t1, t2;
    top2(lp, t1, t2);
    double x = -INFINITY;                         // genotype n handled by lane n
#pragma unroll
    for (int n = 0; n < 10; ++n) if (lane == n) x = lp[n] - m;
    const double e = exp10(x);
    double esum = e;
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) esum += __shfl_xor_sync(FULL, esum, d);
    if (A.dbg_post10 && lane < 10) A.dbg_post10[(site - A.w0) * 10 + lane] = e / esum;
    if (lane == 0) {
        if (A.dbg_L10)
            for (int k = 0; k < 10; ++k) A.dbg_L10[(site - A.w0) * 10 + k] = L10[k];
        site_record(A, site, refb, kidx >= 0, t1, lp[t1] - lp[t2], 1.0 / esum, cu[0], cu[1],
                    cu[2], cu[3], qs[0], qs[1], qs[2], qs[3], ca0, ca1, ca2, ca3, rep, wsum, tie);
    }
}

template <int K>
__device__ void warp_site(const CallArgs& A, const uint32_t* buf, uint32_t n, uint64_t site,
                          uint32_t ca0, uint32_t ca1, uint32_t ca2, uint32_t ca3, uint32_t rep,
                          const double* sLP, uint8_t* slotcnt) {
    constexpr int N = 32 * K;
    const int lane = threadIdx.x & 31;
    const int L2 = 2 * A.L;
    const int refb = A.ref[site - A.origin];
    const int64_t kidx = known_index(A, site);
    uint32_t key[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {
        uint32_t e = k * 32 + lane;
        key[k] = (e < n) ? buf[e] : KEY_INF;
    }
    // bitonic network over N = 32*K elements (element e = k*32 + lane)
#pragma unroll
    for (int size = 2; size <= N; size <<= 1) {
#pragma unroll
        for (int stride = size >> 1; stride > 0; stride >>= 1) {
            if (stride >= 32) {
                const int ks = stride / 32;
#pragma unroll
                for (int k = 0; k < K; ++k) {
                    if ((k & ks) == 0) {
                        const uint32_t e = k * 32 + lane;
                        const bool up = (e & size) == 0;
                        uint32_t a = key[k], b = key[k | ks];
                        bool sw = up ? (a > b) : (a < b);
                        key[k] = sw ? b : a;
                        key[k | ks] = sw ? a : b;
                    }
                }
            } else {
#pragma unroll
                for (int k = 0; k < K; ++k) {
                    const uint32_t e = k * 32 + lane;
                    const bool up = (e & size) == 0;
                    const bool lower = (lane & stride) == 0;
                    uint32_t p = __shfl_xor_sync(FULL, key[k], stride);
                    key[k] = (lower == up) ? min(key[k], p) : max(key[k], p);
                }
            }
        }
    }
    if (A.dbg_keys_sorted) {
        const uint32_t o = A.dbg_off[site - A.w0];
#pragma unroll
        for (int k = 0; k < K; ++k) {
            uint32_t e = k * 32 + lane;
            if (e < n) A.dbg_keys_sorted[o + e] = key[k];
        }
    }
    const uint32_t lt = lanemask_lt();
    const uint32_t le = lt | (1u << lane);
    int d0 = 0, d1 = 0, d2 = 0, d3 = 0;          // distinct slots seen per base (chunks < k)
    double acc[10];
#pragma unroll
    for (int j = 0; j < 10; ++j) acc[j] = 0.0;
    uint32_t cu[4] = {0, 0, 0, 0}, qs[4] = {0, 0, 0, 0};
#pragma unroll
    for (int k = 0; k < K; ++k) {
        const uint32_t kk = key[k];
        const bool valid = kk != KEY_INF;
        const uint32_t b = key_base(kk), q = key_q(kk), cyc = key_cyc(kk), slot = key_slot(kk);
        const uint32_t tag = valid ? (b << 9 | slot) : (0x80000000u | lane);
        const uint32_t peers = __match_any_sync(FULL, tag);
        uint32_t pcr = 1u + __popc(peers & lt) + (valid ? slotcnt[b * L2 + slot] : 0u);
        const bool first = valid && pcr == 1u;
        const uint32_t fb = __ballot_sync(FULL, first);
        const uint32_t bmask = __match_any_sync(FULL, valid ? b : (0x80000000u | lane));
        const int db = b == 0 ? d0 : b == 1 ? d1 : b == 2 ? d2 : d3;
        const uint32_t g = (uint32_t)(db + __popc(fb & bmask & le) - 1);
        if (valid && (peers >> lane) == 1u) slotcnt[b * L2 + slot] = (uint8_t)min(pcr, 255u);
        d0 += __popc(fb & __ballot_sync(FULL, valid && b == 0));
        d1 += __popc(fb & __ballot_sync(FULL, valid && b == 1));
        d2 += __popc(fb & __ballot_sync(FULL, valid && b == 2));
        d3 += __popc(fb & __ballot_sync(FULL, valid && b == 3));
        __syncwarp();
        if (valid) {
            const int qa = adj_lookup(A, q, pcr, g);
            add_row(A.T, A.L, (uint32_t)qa, cyc, b, acc);
#pragma unroll
            for (int x = 0; x < 4; ++x) { cu[x] += b == (uint32_t)x; qs[x] += b == (uint32_t)x ? q : 0u; }
        }
    }
#pragma unroll
    for (int k = 0; k < K; ++k)                    // reset this site's slot counters
        if (key[k] != KEY_INF) slotcnt[key_base(key[k]) * L2 + key_slot(key[k])] = 0;
    __syncwarp();
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) {
#pragma unroll
        for (int j = 0; j < 10; ++j) acc[j] += __shfl_xor_sync(FULL, acc[j], d);
#pragma unroll
        for (int x = 0; x < 4; ++x) {
            cu[x] += __shfl_xor_sync(FULL, cu[x], d);
            qs[x] += __shfl_xor_sync(FULL, qs[x], d);
        }
    }
    // rank-sum pieces for a heterozygous call (R8)
    double lp[10];
    const double* prow = kidx >= 0 ? A.known_lp + kidx * 10 : sLP + refb * 10;
#pragma unroll
    for (int j = 0; j < 10; ++j) lp[j] = acc[j] + prow[j];
    int t1, t2;
    top2(lp, t1, t2);
    const int a1 = geno_a1(t1), a2 = geno_a2(t1);
    double wsum = 0.0, tie = 0.0;
    if ((A.flags & GSNP_RANK_SUM) && a1 != a2 && pick4(cu[0], cu[1], cu[2], cu[3], a1) &&
        pick4(cu[0], cu[1], cu[2], cu[3], a2)) {
#pragma unroll 1
        for (int k = 0; k < K; ++k) {
            const uint32_t x = key[k];
            const uint32_t xb = key_base(x), xq = key_q(x);
            const bool xin = x != KEY_INF && (xb == (uint32_t)a1 || xb == (uint32_t)a2);
            uint32_t less = 0, eq = 0;
#pragma unroll 1
            for (uint32_t e = 0; e < n; ++e) {
                const uint32_t y = buf[e], yb = key_base(y), yq = key_q(y);
                const bool yin = yb == (uint32_t)a1 || yb == (uint32_t)a2;
                less += yin && yq < xq;
                eq += yin && yq == xq;
            }
            if (xin) {
                if (xb == (uint32_t)a1) wsum += (double)less + ((double)eq + 1.0) / 2.0;
                tie += (double)eq * (double)eq - 1.0;
            }
        }
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) {
            wsum += __shfl_xor_sync(FULL, wsum, d);
            tie += __shfl_xor_sync(FULL, tie, d);
        }
    }
    group_epilogue(A, site, refb, kidx, sLP, acc, cu, qs, ca0, ca1, ca2, ca3, rep, wsum, tie);
}

// In-place ascending bitonic sort of a[0..n) in shared memory by the whole CTA (n arbitrary:
// the "flip" formulation only ever moves the smaller element to the lower index, so virtual
// +inf padding beyond n never has to move).
__device__ void cta_sort(uint32_t* a, uint32_t n) {
    uint32_t N2 = 1;
    while (N2 < n) N2 <<= 1;
    for (uint32_t size = 2; size <= N2; size <<= 1) {
        const uint32_t half = size >> 1;
        for (uint32_t t = threadIdx.x; t < N2 / 2; t += NT) {
            uint32_t blk = t / half, o = t % half;
            uint32_t i = blk * size + o, j = blk * size + size - 1 - o;
            if (j < n && a[i] > a[j]) { uint32_t x = a[i]; a[i] = a[j]; a[j] = x; }
        }
        __syncthreads();
        for (uint32_t stride = size >> 2; stride > 0; stride >>= 1) {
            for (uint32_t t = threadIdx.x; t < N2 / 2; t += NT) {
                uint32_t i = (t / stride) * 2 * stride + (t % stride), j = i + stride;
                if (j < n && a[i] > a[j]) { uint32_t x = a[i]; a[i] = a[j]; a[j] = x; }
            }
            __syncthreads();
        }
    }
}

// CTA path for 256 < n <= deep_cap: keys gathered into the col region, CTA bitonic sort,
// warp 0 walks the chunks for the dependency counters (q_adj stored in key bits 17..22), all
// warps gather and reduce, warp 0 finishes.
__device__ __noinline__ void cta_site(const CallArgs& A, const TileSmem& sm, uint32_t* a,
                                      uint32_t n, uint64_t site, int site_local,
                                      const double* sLP, double* red) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int L2 = 2 * A.L;
    cta_sort(a, n);
    if (A.dbg_keys_sorted) {
        const uint32_t o = A.dbg_off[site - A.w0];
        for (uint32_t e = threadIdx.x; e < n; e += NT) A.dbg_keys_sorted[o + e] = a[e];
    }
    if (warp == 0) {
        uint8_t* slotcnt = sm.slotcnt;
        int d0 = 0, d1 = 0, d2 = 0, d3 = 0;
        const uint32_t lt = lanemask_lt(), le = lt | (1u << lane);
        for (uint32_t c0 = 0; c0 < n; c0 += 32) {
            const uint32_t e = c0 + lane;
            const bool valid = e < n;
            const uint32_t kk = valid ? a[e] : KEY_INF;
            const uint32_t b = key_base(kk), q = key_q(kk), slot = key_slot(kk);
            const uint32_t peers = __match_any_sync(FULL, valid ? (b << 9 | slot) : (0x80000000u | lane));
            uint32_t pcr = 1u + __popc(peers & lt) + (valid ? slotcnt[b * L2 + slot] : 0u);
            const bool first = valid && pcr == 1u;
            const uint32_t fb = __ballot_sync(FULL, first);
            const uint32_t bmask = __match_any_sync(FULL, valid ? b : (0x80000000u | lane));
            const int db = b == 0 ? d0 : b == 1 ? d1 : b == 2 ? d2 : d3;
            const uint32_t g = (uint32_t)(db + __popc(fb & bmask & le) - 1);
            if (valid && (peers >> lane) == 1u) slotcnt[b * L2 + slot] = (uint8_t)min(pcr, 255u);
            d0 += __popc(fb & __ballot_sync(FULL, valid && b == 0));
            d1 += __popc(fb & __ballot_sync(FULL, valid && b == 1));
            d2 += __popc(fb & __ballot_sync(FULL, valid && b == 2));
            d3 += __popc(fb & __ballot_sync(FULL, valid && b == 3));
            __syncwarp();
            if (valid) a[e] = (kk & 0x1FFFFu) | (uint32_t)adj_lookup(A, q, pcr, g) << 17;
        }
        __syncwarp();
        for (uint32_t e = lane; e < n; e += 32) slotcnt[key_base(a[e]) * L2 + key_slot(a[e])] = 0;
    }
    __syncthreads();
    double acc[10];
#pragma unroll
    for (int j = 0; j < 10; ++j) acc[j] = 0.0;
    uint32_t cu[4] = {0, 0, 0, 0}, qs[4] = {0, 0, 0, 0};
    for (uint32_t e = threadIdx.x; e < n; e += NT) {
        const uint32_t kk = a[e];
        const uint32_t b = key_base(kk);
        add_row(A.T, A.L, kk >> 17, key_cyc(kk), b, acc);
#pragma unroll
        for (int x = 0; x < 4; ++x) { cu[x] += b == (uint32_t)x; qs[x] += b == (uint32_t)x ? key_q(kk) : 0u; }
    }
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) {
#pragma unroll
        for (int j = 0; j < 10; ++j) acc[j] += __shfl_xor_sync(FULL, acc[j], d);
#pragma unroll
        for (int x = 0; x < 4; ++x) {
            cu[x] += __shfl_xor_sync(FULL, cu[x], d);
            qs[x] += __shfl_xor_sync(FULL, qs[x], d);
        }
    }
    if (lane == 0) {
        for (int j = 0; j < 10; ++j) red[warp * 18 + j] = acc[j];
        for (int x = 0; x < 4; ++x) {
            red[warp * 18 + 10 + x] = (double)cu[x];
            red[warp * 18 + 14 + x] = (double)qs[x];
        }
    }
    __syncthreads();
    __shared__ double rk[2];
    const int refb = A.ref[site - A.origin];
    const int64_t kidx = known_index(A, site);
    double L10[10];
    uint32_t cut[4], qst[4];
#pragma unroll
    for (int j = 0; j < 10; ++j) {
        double v = 0.0;
        for (int w = 0; w < NW; ++w) v += red[w * 18 + j];
        L10[j] = v;
    }
#pragma unroll
    for (int x = 0; x < 4; ++x) {
        double c = 0.0, qq = 0.0;
        for (int w = 0; w < NW; ++w) { c += red[w * 18 + 10 + x]; qq += red[w * 18 + 14 + x]; }
        cut[x] = (uint32_t)c;
        qst[x] = (uint32_t)qq;
    }
    if (threadIdx.x == 0) {
        // rank-sum pieces by histogram over the 64 quality values (het calls only)
        double wsum = 0.0, tie = 0.0;
        const double* prow = kidx >= 0 ? A.known_lp + kidx * 10 : sLP + refb * 10;
        double lp[10];
        for (int j = 0; j < 10; ++j) lp[j] = L10[j] + prow[j];
        int t1, t2;
        top2(lp, t1, t2);
        const int a1 = geno_a1(t1), a2 = geno_a2(t1);
        if (a1 != a2 && (A.flags & GSNP_RANK_SUM)) {
            uint32_t hx[64], hy[64];
            for (int v = 0; v < 64; ++v) { hx[v] = 0; hy[v] = 0; }
            for (uint32_t e = 0; e < n; ++e) {
                uint32_t b = key_base(a[e]), q = key_q(a[e]);
                if (b == (uint32_t)a1) hx[q]++;
                else if (b == (uint32_t)a2) hy[q]++;
            }
            double less = 0.0;
            for (int v = 0; v < 64; ++v) {
                double t = (double)hx[v] + (double)hy[v];
                wsum += (double)hx[v] * (less + (t + 1.0) / 2.0);
                tie += t * t * t - t;
                less += t;
            }
        }
        rk[0] = wsum;
        rk[1] = tie;
    }
    __syncthreads();
    if (warp == 0)
        group_epilogue(A, site, refb, kidx, sLP, L10, cut, qst, sm.cnt_all[0 * TS + site_local],
                       sm.cnt_all[1 * TS + site_local], sm.cnt_all[2 * TS + site_local],
                       sm.cnt_all[3 * TS + site_local], sm.rep[site_local], rk[0], rk[1]);
    __syncthreads();
}

// ------------------------------------------------------------------------------------------
// The fused per-tile kernel (a4..a8): counting + base_word gather (site-major, no atomics),
// likelihood_sort + likelihood_comp + posterior + record, per site.
__global__ void __launch_bounds__(NT, 2) k_call_tile(CallArgs A) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ double sLP[50];
    __shared__ double red[NW * 18];
    __shared__ uint64_t wr[NW][2];
    __shared__ uint32_t ovf_n, deep_n;
    __shared__ uint16_t ovf[TS], deep[TS];
    TileSmem sm;
    call_smem_bytes(A.L, &sm, smem);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint64_t t0 = A.w0 + (uint64_t)blockIdx.x * TS;
    const uint64_t site = t0 + tid;
    const bool active = site < A.w1;
    const uint64_t grp = (uint64_t)blockIdx.x * NW + warp;
    const bool wactive = t0 + warp * 32 < A.w1;
    const uint64_t wra = wactive ? A.tile_ra[grp] : 0, wrb = wactive ? A.tile_rb[grp] : 0;
    if (tid < 50) sLP[tid] = A.LP[tid];
    if (tid == 0) { ovf_n = 0; deep_n = 0; }
    if (lane == 0) { wr[warp][0] = wra; wr[warp][1] = wrb; }
    for (int i = tid; i < NW * 2 * A.L; i += NT) reinterpret_cast<uint32_t*>(sm.slotcnt)[i] = 0;

    // ---- counting + base_word gather, one site per lane.  The warp
    // walks the reads covering its 32 sites; metadata for 32 reads is loaded coalesced and
    // broadcast by shuffles; each lane reads the base at its own site (consecutive lanes ->
    // consecutive bytes of the read).
    uint32_t ca0 = 0, ca1 = 0, ca2 = 0, ca3 = 0, rep = 0, n = 0;
    bool dup = false, have_minus = false;
    uint64_t last_plus = ~0ull, last_end = 0;
    int err = 0;
    for (uint64_t r0 = wra; r0 < wrb; r0 += 32) {
        const uint64_t r = r0 + lane;
        uint64_t p = 0, o = 0;
        uint32_t lh = 0;                          // len | hits << 16 ... packed with strand
        uint32_t st = 0;
        if (r < wrb) {
            p = A.R.pos[r];
            o = A.R.off[r] - A.R.off0;
            lh = (uint32_t)A.R.len[r] | (uint32_t)A.R.hits[r] << 16;
            st = A.R.strand[r];
        }
        const int nr = (int)min((uint64_t)32, wrb - r0);
#pragma unroll 4
        for (int k = 0; k < nr; ++k) {
            const uint64_t pk = __shfl_sync(FULL, p, k);
            const uint64_t ok = __shfl_sync(FULL, o, k);
            const uint32_t lhk = __shfl_sync(FULL, lh, k);
            const uint32_t sk = __shfl_sync(FULL, st, k);
            const uint32_t lk = lhk & 0xFFFFu, hk = lhk >> 16;
            const uint64_t i = site - pk;         // wraps (huge) when site < pk
            if (!active || i >= lk) continue;
            const uint32_t b = A.R.bases[ok + i];
            if (b >= 4) { if (b > 4) err |= ERR_RANGE; continue; }
            ca0 += b == 0; ca1 += b == 1; ca2 += b == 2; ca3 += b == 3;
            rep += hk;
            if (hk != 1) continue;
            const uint32_t q = A.R.quals[ok + i];
            if (q > (uint32_t)A.q_max) { err |= ERR_QUAL; continue; }
            const uint32_t cyc = sk ? lk - 1 - (uint32_t)i : (uint32_t)i;
            const uint32_t key = b << 15 | (63u - q) << 9 | cyc << 1 | sk;
            if (n < COLS) sm.col[n * TS + tid] = key;
            if (A.dbg_keys_built) A.dbg_keys_built[A.dbg_off[site - A.w0] + n] = key;
            ++n;
            // same (strand, coord) twice at a site <=> same start on '+', same end on '-'
            if (sk == 0) { dup |= pk == last_plus; last_plus = pk; }
            else { const uint64_t e = pk + lk - 1; dup |= have_minus && e <= last_end; last_end = e; have_minus = true; }
        }
    }
    if (err) atomicOr(A.err, err);
    if (A.count_only) {
        if (active) A.dbg_nuni[site - A.w0] = n;
        return;
    }
    sm.cnt_all[0 * TS + tid] = ca0; sm.cnt_all[1 * TS + tid] = ca1;
    sm.cnt_all[2 * TS + tid] = ca2; sm.cnt_all[3 * TS + tid] = ca3;
    sm.rep[tid] = rep;
    sm.nuni[tid] = n;
    __syncthreads();

    // ---- thread-per-site likelihood for n <= 32 (network size chosen per warp: 8/16/32)
    const bool small = active && n <= COLS;
    if (active && !small) {
        if (n <= WBUF) ovf[atomicAdd(&ovf_n, 1u)] = (uint16_t)tid;
        else deep[atomicAdd(&deep_n, 1u)] = (uint16_t)tid;
    }
    const uint32_t maxn = __reduce_max_sync(FULL, small ? n : 0u);
    if (small) {
        if (maxn <= 8) thread_site<8>(A, sm, site, n, dup, ca0, ca1, ca2, ca3, rep, sLP);
        else if (maxn <= 16) thread_site<16>(A, sm, site, n, dup, ca0, ca1, ca2, ca3, rep, sLP);
        else thread_site<32>(A, sm, site, n, dup, ca0, ca1, ca2, ca3, rep, sLP);
    }
    __syncthreads();

    // ---- warp path: 32 < n <= 256 (keys re-gathered from the owning warp's reads)
    uint32_t* buf = sm.wbuf + warp * WBUF;
    uint8_t* myslot = sm.slotcnt + warp * 8 * A.L;
    for (uint32_t j = warp; j < ovf_n; j += NW) {
        const int sl = ovf[j];
        const uint64_t s = t0 + sl;
        const uint64_t ra = wr[sl >> 5][0], rb = wr[sl >> 5][1];
        uint32_t m = 0;
        for (uint64_t r0 = ra; r0 < rb; r0 += 32) {
            const uint64_t r = r0 + lane;
            uint32_t key = KEY_INF;
            if (r < rb && A.R.hits[r] == 1) {
                const uint64_t i = s - A.R.pos[r];
                const uint32_t l = A.R.len[r];
                if (i < l) {
                    const uint64_t bi = A.R.off[r] - A.R.off0 + i;
                    const uint32_t b = A.R.bases[bi];
                    if (b < 4) {
                        const uint32_t st = A.R.strand[r];
                        const uint32_t cyc = st ? l - 1 - (uint32_t)i : (uint32_t)i;
                        key = b << 15 | (63u - A.R.quals[bi]) << 9 | cyc << 1 | st;
                    }
                }
            }
            const uint32_t v = __ballot_sync(FULL, key != KEY_INF);
            if (key != KEY_INF) buf[m + __popc(v & lanemask_lt())] = key;
            m += __popc(v);
        }
        __syncwarp();
        const uint32_t c0 = sm.cnt_all[sl], c1 = sm.cnt_all[TS + sl], c2 = sm.cnt_all[2 * TS + sl],
                       c3 = sm.cnt_all[3 * TS + sl], rp = sm.rep[sl];
        if (m <= 64) warp_site<2>(A, buf, m, s, c0, c1, c2, c3, rp, sLP, myslot);
        else if (m <= 128) warp_site<4>(A, buf, m, s, c0, c1, c2, c3, rp, sLP, myslot);
        else warp_site<8>(A, buf, m, s, c0, c1, c2, c3, rp, sLP, myslot);
        __syncwarp();
    }
    // ---- CTA path: n > 256, one site at a time in the col region
    for (uint32_t j = 0; j < deep_n; ++j) {
        __syncthreads();
        const int sl = deep[j];
        const uint64_t s = t0 + sl;
        if (sm.nuni[sl] > (uint32_t)sm.deep_cap) {
            if (tid == 0) atomicOr(A.err, ERR_DEEP);
            continue;
        }
        __shared__ uint32_t cnt;
        if (tid == 0) cnt = 0;
        __syncthreads();
        const uint64_t ra = wr[sl >> 5][0], rb = wr[sl >> 5][1];
        for (uint64_t r = ra + tid; r < rb; r += NT) {
            if (A.R.hits[r] != 1) continue;
            const uint64_t i = s - A.R.pos[r];
            const uint32_t l = A.R.len[r];
            if (i >= l) continue;
            const uint64_t bi = A.R.off[r] - A.R.off0 + i;
            const uint32_t b = A.R.bases[bi];
            if (b >= 4) continue;
            const uint32_t st = A.R.strand[r];
            const uint32_t cyc = st ? l - 1 - (uint32_t)i : (uint32_t)i;
            sm.col[atomicAdd(&cnt, 1u)] = b << 15 | (63u - A.R.quals[bi]) << 9 | cyc << 1 | st;
        }
        __syncthreads();
        cta_site(A, sm, sm.col, cnt, s, sl, sLP, red);
    }
}

}  // namespace gsnp_dev
