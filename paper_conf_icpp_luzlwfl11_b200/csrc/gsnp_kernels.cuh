// gsnp_kernels.cuh — device code of libgsnp (sm_100a).  Included once, by gsnp.cu.
//
// Kernels:
//   k_validate_reads  ABI checks on the read arrays (sortedness P:L208-210, ranges)
//   k_calib_count     a1: calibration histogram C[q][cyc][t][o] (cal_p_matrix)
//   k_prep            validation + a3: per 32-site group, read range [lower_bound(s0-L+1),
//                     lower_bound(s1)), and the window's work counters
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

#ifndef GSNP_NT
#define GSNP_NT 256
#endif
constexpr int NT = GSNP_NT;           // threads per CTA
constexpr int NW = NT / 32;           // warps per CTA
constexpr uint32_t FULL = 0xFFFFFFFFu;
constexpr uint32_t KEY_INF = 0xFFFFFFFFu;

enum : int { ERR_RANGE = 1, ERR_UNSORTED = 2, ERR_DEEP = 4, ERR_QUAL = 8, ERR_VALID = 64 };

// k_validate_reads sets ERR_VALID (with the specific bits) when the read arrays break the ABI
// contract (unsorted positions, offsets, lengths or positions out of range).  Every kernel that
// dereferences pos/off/len runs after it on the same stream and returns at once when the flag is
// up, so out-of-contract input yields a status, never an out-of-bounds access.  Only the
// validator writes this bit, so every thread of a launch reads the same value.
__device__ __forceinline__ bool reads_invalid(const int* err) {
    return (*reinterpret_cast<const volatile int*>(err) & ERR_VALID) != 0;
}

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
    const uint8_t* ref;               // ref[site - origin] = code | known << 3 (known SNP)
    uint64_t origin, n_sites;
    const uint64_t* known_pos;        // sorted
    const double* known_lp;           // n_known x 10 log10 priors (host-built)
    uint64_t n_known;
    const double* LP;                 // [5][10] log10 novel priors per reference code (R6)
    const double* T;                  // [64][L][4][TROW] score table (Alg. 3), rows padded
    const double* rank_cdf;           // R20: [(n1*33+n2)*1025 + u] = P(U <= u); null if unused
    const uint8_t* adj;               // [64][adjP][adjG] adjust table (R3)
    int adjP, adjG;
    int L, q_max;
    uint32_t flags;
    uint64_t w0, w1;                  // window
    const uint64_t* tile_ra;          // per 32-site group read range [ra, rb)
    const uint64_t* tile_rb;
    gsnp_record* out;                 // out[site - w0]
    int* err;
    float mid_at, deep_at;            // window depth thresholds of the 64- and 128-slot kernels
    const uint32_t* len_flag;         // == epoch: not every read has the same length (k_prep)
    uint32_t epoch;
    uint32_t list_min;                // listed sites below this count take the warp path
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

// x << s with PTX semantics: shifts of 32 or more give 0
__device__ __forceinline__ uint32_t shl_clamp(uint32_t x, uint32_t s) {
    uint32_t r;
    asm("shl.b32 %0, %1, %2;" : "=r"(r) : "r"(x), "r"(s));
    return r;
}
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
__device__ __forceinline__ void validate_read(const DevReads& R, uint64_t r, uint64_t origin,
                                              uint64_t n_sites, int L, int* err);
__global__ void k_validate_reads(DevReads R, uint64_t origin, uint64_t n_sites, int L, int* err) {
    uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (r < R.n) validate_read(R, r, origin, n_sites, L, err);
}

// ------------------------------------------------------------------------------------------
// k_prep: one launch before a window's calling kernels — blocks [0, nbv) validate the reads (as
// k_validate_reads), the others compute a3's per-32-site-group read ranges,
// and block 0 zeroes the window's three work counters.
__device__ __forceinline__ void validate_read(const DevReads& R, uint64_t r, uint64_t origin,
                                              uint64_t n_sites, int L, int* err) {
    uint64_t p = R.pos[r];
    uint32_t l = R.len[r];
    int e = 0;
    if (l == 0 || l > (uint32_t)L) e |= ERR_RANGE;
    if (R.hits[r] == 0 || R.strand[r] > 1) e |= ERR_RANGE;
    if (p < origin || p + l > origin + n_sites) e |= ERR_RANGE;
    if (R.off[r] < R.off0 || R.off[r] + l > R.off[r + 1]) e |= ERR_RANGE;
    if (r > 0 && R.pos[r - 1] > p) e |= ERR_UNSORTED;
    if (e) atomicOr(err, e | ERR_VALID);
}

// counters[3]: set to `epoch` (this call's number) when some read's length differs from read 0's —
// the calling kernels then check uniformity per group; no reset is needed between calls
__global__ void k_prep(DevReads R, uint64_t origin, uint64_t n_sites, int L, int* err, uint32_t nbv,
                       uint64_t w0, uint64_t w1, uint64_t n_groups, uint64_t* ra, uint64_t* rb,
                       uint32_t* counters, uint32_t epoch) {
    if (blockIdx.x == 0 && (threadIdx.x < 3 || threadIdx.x == 4 || threadIdx.x == 5)) counters[threadIdx.x] = 0;
    if (blockIdx.x < nbv) {
        const uint64_t r = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
        if (r < R.n) {
            validate_read(R, r, origin, n_sites, L, err);
            if (R.len[r] != R.len[0]) counters[3] = epoch;
        }
        return;
    }
    const uint64_t g = (blockIdx.x - nbv) * (uint64_t)blockDim.x + threadIdx.x;
    if (g >= n_groups) return;
    const uint64_t s0 = w0 + g * 32, s1 = min(w1, s0 + 32);
    const uint64_t lo = s0 >= (uint64_t)(L - 1) ? s0 - (L - 1) : 0;
    const uint64_t a = lower_bound_u64(R.pos, 0, R.n, lo);
    ra[g] = a;
    rb[g] = lower_bound_u64(R.pos, a, R.n, s1);
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
// TMA (1-D bulk copy) + mbarrier helpers (sm_90+; SASS UBLKCP / SYNCS).
__host__ __device__ inline size_t align16(size_t x) { return (x + 15) & ~size_t(15); }
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
                 "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n .reg .pred P1;\n"
        "WAIT_%=:\n"
        " mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        " @!P1 bra WAIT_%=;\n}\n" ::"r"(smem_u32(bar)), "r"(parity) : "memory");
}
// global -> shared bulk copy of `bytes` (multiple of 16, both addresses 16-byte aligned)
__device__ __forceinline__ void tma_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
        ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// ------------------------------------------------------------------------------------------
// a1: calibration histogram C[q][cyc][t][o] (cal_p_matrix).
// The CTA streams its share of the reads in batches: the batch's bases and qualities (one
// contiguous byte range) and the reference window under it arrive in shared memory by TMA bulk
// copies, double-buffered and completed on an mbarrier, while the previous batch is counted.
// Warp per read, four consecutive read positions per lane (one 32-bit shared load per array,
// realigned with a funnel shift).  The diagonal cells (t == o, ~98% of bases) go to a shared
// [q][t][cycle] u32 histogram with fire-and-forget shared reductions (lanes of a warp hit
// consecutive cycles: distinct words, distinct banks); mismatches go to global u64 REDs; the
// histogram is added into the global counts once at the end.
struct CalibArgs {
    DevReads R;
    const uint8_t* ref;               // code | known << 3, indexed by site - origin (16 B padded)
    uint64_t origin, n_sites;
    int L, q_max;
    int Lh;                           // cycles [0, Lh) counted in shared memory (Lh <= L)
    int CB;                           // reads per batch
    uint32_t SB;                      // bytes per stage buffer (bases; quals the same)
    uint32_t RB;                      // bytes per reference-window buffer
    unsigned long long* C;            // [64][256][4][4]
    int* err;
    int tma_ok;                       // bases and quals 16-byte aligned (TMA bulk copies allowed)
};

#ifndef GSNP_CAL_NT
#define GSNP_CAL_NT 1024
#endif
constexpr int CAL_NT = GSNP_CAL_NT;
constexpr int CAL_NW = CAL_NT / 32;
constexpr int CAL_MAXB = 512;         // max reads per batch (metadata arrays)

__device__ __forceinline__ void red_shared_add(uint32_t* p, uint32_t v) {
    asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(smem_u32(p)), "r"(v) : "memory");
}
// shared add at a shared-window byte address
__device__ __forceinline__ void red_shared_add_at(uint32_t saddr, uint32_t v) {
    asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(saddr), "r"(v) : "memory");
}
// predicated shared increment (no branch around it)
__device__ __forceinline__ void red_shared_inc_if(uint32_t saddr, uint32_t pred) {
    asm volatile("{\n .reg .pred p;\n setp.ne.u32 p, %1, 0;\n @p red.shared.add.u32 [%0], 1;\n}"
                 ::"r"(saddr), "r"(pred) : "memory");
}

__global__ void __launch_bounds__(CAL_NT, 1) k_calib_count(const __grid_constant__ CalibArgs A) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ uint64_t m_desc[2][CAL_MAXB];          // counted reads: rs | stage offset << 32
    __shared__ uint16_t m_ls[2][CAL_MAXB];            // len | strand << 9
    __shared__ uint32_t m_n[3];                       // counted reads of batch k: m_n[k % 3]
    __shared__ __align__(8) uint64_t bar[2];
    __shared__ uint64_t st_base[2];                   // global byte index of each stage's start
    __shared__ uint32_t st_rs[2];                     // reference index of each ref window's start
    __shared__ int st_direct[2];                      // too wide for the buffers: read global
    // flat mode (every read of the batch has length Lb and the reads' bytes are contiguous):
    // per read of the batch, uncompacted: reference offset in the stage window | minus << 31,
    // or ~0 for a read that is not counted
    __shared__ uint32_t m_flat[2][CAL_MAXB];
    __shared__ uint32_t m_fl[2][5];                   // uniform flag, reads in batch, length Lb,
                                                      // ceil(2^32 / Lb), stage byte offset
    if (reads_invalid(A.err)) return;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int L = A.L, Lh = A.Lh;
    const uint32_t qmax = (uint32_t)A.q_max;
    const int ncell = (A.q_max + 1) * 4 * Lh;
    uint32_t* hist = reinterpret_cast<uint32_t*>(smem);               // [q*4 + t][cycle]
    auto hidx = [&](uint32_t qt, uint32_t cyc) { return qt * (uint32_t)Lh + cyc; };
    unsigned char* stage = smem + align16((size_t)ncell * 4);
    const size_t stage_bytes = 2 * (size_t)A.SB + A.RB;
    for (int i = tid; i < ncell; i += CAL_NT) hist[i] = 0;
    const uint64_t per = (A.R.n + gridDim.x - 1) / gridDim.x;
    const uint64_t ra = min(A.R.n, (uint64_t)blockIdx.x * per), rb = min(A.R.n, ra + per);
    const uint64_t nbatch = (rb - ra + A.CB - 1) / A.CB;
    const int issuer = CAL_NT - 1;
    if (tid == 0) { mbar_init(&bar[0], 1); mbar_init(&bar[1], 1); }
    __syncthreads();
    // thread `issuer`: bulk copies of batch k's bases, quals and reference window into stage k&1
    auto issue = [&](uint64_t k) {
        const uint64_t b0 = ra + k * A.CB, b1 = min(rb, b0 + A.CB);
        const uint64_t o0 = A.R.off[b0] - A.R.off0, o1 = A.R.off[b1] - A.R.off0;
        const uint64_t a0 = o0 & ~15ull, a1 = (o1 + 15) & ~15ull;
        const uint64_t p0 = A.R.pos[b0], p1 = A.R.pos[b1 - 1];
        const int sidx = (int)(k & 1);
        st_base[sidx] = a0;
        const uint64_t r0 = p0 >= A.origin ? ((p0 - A.origin) & ~15ull) : 0;
        const uint64_t r1 = ((p1 + L - A.origin) + 15) & ~15ull;
        st_rs[sidx] = (uint32_t)r0;
        // the rounded-up copy must stay inside the caller's arrays (their last valid byte is
        // off[n] - 1): a batch at the very end whose 16-byte round-up would overrun reads global
        const uint64_t end = A.R.off[A.R.n] - A.R.off0;
        const bool fits = A.tma_ok && a1 <= end && a1 - a0 <= A.SB && p0 >= A.origin &&
                          p1 + L <= A.origin + A.n_sites && r1 - r0 <= A.RB;
        st_direct[sidx] = fits ? 0 : 1;
        if (!fits) return;
        unsigned char* sb = stage + (size_t)sidx * stage_bytes;
        const uint32_t bytes = (uint32_t)(a1 - a0), rbytes = (uint32_t)(r1 - r0);
        fence_proxy_async_smem();
        mbar_arrive_expect_tx(&bar[sidx], 2 * bytes + rbytes);
        tma_g2s(sb, A.R.bases + a0, bytes, &bar[sidx]);
        tma_g2s(sb + A.SB, A.R.quals + a0, bytes, &bar[sidx]);
        tma_g2s(sb + 2 * A.SB, A.ref + r0, rbytes, &bar[sidx]);
    };
    // Descriptor of read b0 + tid of batch k, loaded into registers one batch ahead so its
    // global latency overlaps the count of the batch before.
    struct Meta { uint64_t p, o, base, ob0, p0; uint32_t l, st, hit, l0, nall; bool in; };
    auto meta_load = [&](uint64_t k) {
        Meta m;
        const uint64_t b0 = ra + k * A.CB, b1 = min(rb, b0 + A.CB), r = b0 + tid;
        m.in = tid < A.CB && r < b1;
        m.ob0 = A.R.off[b0];
        m.base = (m.ob0 - A.R.off0) & ~15ull;         // = st_base of batch k (see issue)
        m.p0 = A.R.pos[b0];
        m.l0 = A.R.len[b0];
        m.nall = (uint32_t)(b1 - b0);
        m.p = 0; m.o = 0; m.l = 0; m.st = 0; m.hit = 0;
        if (m.in) {
            m.p = A.R.pos[r]; m.o = A.R.off[r]; m.l = A.R.len[r];
            m.st = A.R.strand[r]; m.hit = A.R.hits[r];
        }
        return m;
    };
    // Compact the counted reads (unique, inside the reference) of a batch into m_desc/m_ls[sidx].
    auto meta_commit = [&](const Meta& m, int sidx, int cidx) {
        const bool keep = m.in && m.hit == 1 && m.p >= A.origin && m.p + m.l <= A.origin + A.n_sites &&
                          m.l >= 1 && m.l <= (uint32_t)L;
        const uint32_t bal = __ballot_sync(FULL, keep);
        uint32_t base = 0;
        if ((tid & 31) == 0 && bal) base = atomicAdd(&m_n[cidx], (uint32_t)__popc(bal));
        base = __shfl_sync(FULL, base, 0);
        if (keep) {
            const uint32_t j = base + __popc(bal & lanemask_lt());
            m_desc[sidx][j] = (uint64_t)(uint32_t)(m.p - A.origin) |
                              (uint64_t)(uint32_t)(m.o - A.R.off0 - m.base) << 32;
            m_ls[sidx][j] = (uint16_t)(m.l | m.st << 9);
        }
        // flat-mode descriptors and the batch's uniformity (all threads take part)
        const uint64_t r0 = m.p0 >= A.origin ? ((m.p0 - A.origin) & ~15ull) : 0;   // = st_rs
        if (m.in)
            m_flat[sidx][tid] = keep ? (uint32_t)(m.p - A.origin - r0) | m.st << 31 : 0xFFFFFFFFu;
        // (flat mode needs Lb >= 2: its read index is a multiply-high by ceil(2^32 / Lb), which
        // wraps to 0 at Lb == 1 — batches of 1-bp reads take the staged path)
#ifdef GSNP_CAL_NOFLAT
        const bool uni = false;
#else
        const bool uni = m.l0 >= 2 && (!m.in || (m.l == m.l0 && m.o - m.ob0 == (uint64_t)tid * m.l0));
#endif
        const int all_uni = __syncthreads_and(uni);
        if (tid == 0) {
            m_fl[sidx][0] = all_uni; m_fl[sidx][1] = m.nall; m_fl[sidx][2] = m.l0;
            m_fl[sidx][3] = m.l0 >= 2 ? (uint32_t)(0xFFFFFFFFull / m.l0 + 1) : 0u;
            m_fl[sidx][4] = (uint32_t)((m.ob0 - A.R.off0) & 15ull);
        }
    };
    // one base: o observed, q quality, rt reference code | known << 3, cycle cyc
    int err = 0;
    auto count1 = [&](uint32_t o, uint32_t q, uint32_t rt, uint32_t cyc) {
        err |= (o > 4 ? ERR_RANGE : 0) | (q > qmax ? ERR_QUAL : 0);
        if (rt >= 4 || o >= 4 || q > qmax) return;                 // N, known SNP, bad
        if (rt == o && cyc < (uint32_t)Lh) red_shared_add(&hist[hidx(q * 4 + rt, cyc)], 1u);
        else atomicAdd(&A.C[q << 12 | cyc << 4 | rt << 2 | o], 1ull);
    };
    if (tid == 0) { m_n[0] = 0; m_n[1] = 0; m_n[2] = 0; }
    __syncthreads();
    if (tid == issuer && nbatch > 0) issue(0);
    Meta nxt{};
    if (nbatch > 0) meta_commit(meta_load(0), 0, 0);
    if (nbatch > 1) nxt = meta_load(1);
    uint32_t phase0 = 0, phase1 = 0;                   // mbarrier parity per stage (TMA'd uses)
    for (uint64_t k = 0; k < nbatch; ++k) {
        const int sidx = (int)(k & 1);
        __syncthreads();                               // metadata of batch k complete
        if (tid == issuer && k + 1 < nbatch) issue(k + 1);
        const uint32_t nr = m_n[k % 3];
        if (tid == 0) m_n[(k + 2) % 3] = 0;           // last read for batch k-1, before the barrier
        const bool direct = st_direct[sidx] != 0;
        const uint64_t* md = m_desc[sidx];
        const uint16_t* ml = m_ls[sidx];
        if (!direct) {
            mbar_wait(&bar[sidx], sidx ? phase1 : phase0);
            if (sidx) phase1 ^= 1u; else phase0 ^= 1u;
        }
        const unsigned char* sb = stage + (size_t)sidx * stage_bytes;
        const unsigned char* rr = sb + 2 * A.SB;
        if (!direct && m_fl[sidx][0]) {
            // flat: thread t takes bytes t, t + 1024, ... of the batch (consecutive threads,
            // consecutive bytes: one read = Lb consecutive bytes; read j = x / Lb exactly by a
            // multiply-high since x < 2^16 and Lb <= 256)
            const uint32_t Lb = m_fl[sidx][2], nb = m_fl[sidx][1] * Lb;
            const uint32_t magic = m_fl[sidx][3], xb = m_fl[sidx][4];
            const unsigned char* fb = sb + xb;
            const uint32_t* mf = m_flat[sidx];
            bool eb = false, eq = false;
            uint32_t ebw = 0, eqw = 0;                                 // error bits (fast path)
            const uint32_t hbase = smem_u32(hist);
            // one byte of the batch (edge words and words that straddle two reads)
            auto one = [&](int64_t x) {
                if (x < 0 || x >= (int64_t)nb) return;
                const uint32_t j = __umulhi((uint32_t)x, magic), i = (uint32_t)x - j * Lb;
                const uint32_t fd = mf[j];
                if (fd == 0xFFFFFFFFu) return;                          // not a counted read
                const uint32_t o = fb[x], q = fb[A.SB + x], rt = rr[(fd & 0xFFFFu) + i];
                const uint32_t cyc = (fd >> 31) ? Lb - 1 - i : i;
                eb |= o > 4;
                eq |= q > qmax;
                if (rt >= 4 || o >= 4 || q > qmax) return;               // N, known SNP, bad
                if (rt == o && cyc < (uint32_t)Lh) red_shared_add(&hist[(q * 4 + rt) * (uint32_t)Lh + cyc], 1u);
                else atomicAdd(&A.C[q << 12 | cyc << 4 | rt << 2 | o], 1ull);
            };
            // thread t: aligned stage words t, t + 1024, ...: four bases, four qualities and the
            // four reference codes under them, checked byte-parallel in 32-bit registers
            const uint32_t* sw = reinterpret_cast<const uint32_t*>(sb);
            const uint32_t w_lo = xb >> 2, w_hi = (xb + nb + 3) >> 2;
            const uint32_t qlim = (qmax + 1) * 0x01010101u;
            const uint32_t L4 = 4u * (uint32_t)Lh, sbw = A.SB >> 2;
            for (uint32_t w = w_lo + tid; w < w_hi; w += CAL_NT) {
                const int64_t x0 = (int64_t)(4 * w) - (int64_t)xb;
                const uint32_t xc = x0 > 0 ? (uint32_t)x0 : 0u;
                const uint32_t j = __umulhi(xc, magic), i0 = xc - j * Lb;
                if (x0 < 0 || x0 + 4 > (int64_t)nb || i0 + 4 > Lb || Lh != L) {   // edge / read boundary
                    for (int u = 0; u < 4; ++u) one(x0 + u);
                    continue;
                }
                const uint32_t fd = mf[j];
                if (fd == 0xFFFFFFFFu) continue;                        // not a counted read
                const uint32_t bw = sw[w], qw = sw[sbw + w];
                const uint32_t ro = (fd & 0xFFFFu) + i0;
                const uint32_t* rw2 = reinterpret_cast<const uint32_t*>(rr + (ro & ~3u));
                const uint32_t rw = __funnelshift_r(rw2[0], rw2[1], (ro & 3u) * 8);
                // per byte, bit 7: b > 4 / q > qmax (errors), byte non-zero tests
                const uint32_t H = 0x80808080u, M = 0x7F7F7F7Fu;
                const uint32_t badb = (((bw | H) - 0x05050505u) | bw) & H;
                const uint32_t badq = (((qw | H) - qlim) | qw) & H;
                ebw |= badb;
                eqw |= badq;
                const uint32_t xd = (rw ^ bw) | (rw & 0xFCFCFCFCu);      // 0 <=> diagonal, t < 4
                const uint32_t xu = (rw | bw) & 0xFCFCFCFCu;             // 0 <=> t < 4 and o < 4
                const uint32_t diag = ~(((xd & M) + M) | xd) & H & ~badq;
                const uint32_t used = ~(((xu & M) + M) | xu) & H & ~badq;
                const uint32_t qt = ((qw & 0x3F3F3F3Fu) << 2) | (rw & 0x03030303u);
                const bool minus = (fd >> 31) != 0;
                const uint32_t c0 = minus ? Lb - 1 - i0 : i0;
                // byte u -> hist[qt_u][c0 +- u]: one unconditional shared add of 0 or 1 per byte
                // (no branch, no warp aggregation)
                const uint32_t a0 = hbase + 4u * c0, st = minus ? 0xFFFFFFFCu : 4u;
                red_shared_add_at(__byte_perm(qt, 0, 0x4440) * L4 + a0, (diag >> 7) & 1u);
                red_shared_add_at(__byte_perm(qt, 0, 0x4441) * L4 + a0 + st, (diag >> 15) & 1u);
                red_shared_add_at(__byte_perm(qt, 0, 0x4442) * L4 + a0 + 2u * st, (diag >> 23) & 1u);
                red_shared_add_at(__byte_perm(qt, 0, 0x4443) * L4 + a0 + 3u * st, diag >> 31);
                uint32_t mis = used & ~diag;                          // ~2% of bases: global
                while (mis) {
                    const int u = (__ffs(mis) - 1) >> 3;
                    mis &= mis - 1;
                    const uint32_t cyc = minus ? c0 - u : c0 + u;
                    atomicAdd(&A.C[((qw >> (8 * u)) & 63u) << 12 | cyc << 4 |
                                   ((rw >> (8 * u)) & 3u) << 2 | ((bw >> (8 * u)) & 3u)], 1ull);
                }
            }
            err |= (eb || ebw ? ERR_RANGE : 0) | (eq || eqw ? ERR_QUAL : 0);
        } else if (!direct) {
            const uint32_t rs = st_rs[sidx];
            // staged: lane covers read positions 4*lane .. 4*lane+3 (+128 per pass)
            for (uint32_t j = warp; j < nr; j += CAL_NW) {
                const uint64_t d = md[j];
                const uint32_t ls = ml[j], l = ls & 511u, minus = ls >> 9;
                const uint32_t bo = (uint32_t)(d >> 32), ro = (uint32_t)d - rs;
                for (uint32_t i0 = 4 * lane; i0 < l; i0 += 128) {
                    const uint32_t ob = bo + i0, orf = ro + i0;
                    const uint32_t* wb = reinterpret_cast<const uint32_t*>(sb + (ob & ~3u));
                    const uint32_t* wq = reinterpret_cast<const uint32_t*>(sb + A.SB + (ob & ~3u));
                    const uint32_t* wr = reinterpret_cast<const uint32_t*>(rr + (orf & ~3u));
                    const uint32_t sh = (ob & 3u) * 8, shr = (orf & 3u) * 8;
                    const uint32_t bw = __funnelshift_r(wb[0], wb[1], sh);
                    const uint32_t qw = __funnelshift_r(wq[0], wq[1], sh);
                    const uint32_t rw = __funnelshift_r(wr[0], wr[1], shr);
                    // byte-parallel (SIMD-in-register) checks of the four bases
                    const uint32_t nv = min(l - i0, 4u);                       // valid bytes
                    const uint32_t vm = nv >= 4 ? 0xFFFFFFFFu : (1u << (8 * nv)) - 1u;
                    const uint32_t badb = __vcmpgtu4(bw, 0x04040404u) & vm;
                    const uint32_t badq = __vcmpgtu4(qw, qmax * 0x01010101u) & vm;
                    err |= (badb ? ERR_RANGE : 0) | (badq ? ERR_QUAL : 0);
                    const uint32_t ok = __vcmpltu4(rw, 0x04040404u) & __vcmpltu4(bw, 0x04040404u) &
                                        ~__vcmpgtu4(qw, qmax * 0x01010101u) & vm;
                    const uint32_t diag = ok & __vcmpeq4(rw, bw);
                    // byte u: (q << 2 | t), the histogram row (q <= 63: no carry between bytes)
                    const uint32_t qt = ((qw & 0x3F3F3F3Fu) << 2) | (rw & 0x03030303u);
                    const int c0 = minus ? (int)(l - 1 - i0) : (int)i0, dir = minus ? -1 : 1;
                    if (Lh == L) {
#pragma unroll
                        for (int u = 0; u < 4; ++u)
                            if (diag & (1u << (8 * u)))
                                red_shared_add(&hist[hidx((qt >> (8 * u)) & 255u, c0 + u * dir)], 1u);
                    } else {
#pragma unroll
                        for (int u = 0; u < 4; ++u)
                            if ((diag & (1u << (8 * u))) && (uint32_t)(c0 + u * dir) < (uint32_t)Lh)
                                red_shared_add(&hist[hidx((qt >> (8 * u)) & 255u, c0 + u * dir)], 1u);
                    }
                    // the rest goes to global REDs: mismatches (~2% of bases) and, when the shared
                    // histogram stops at Lh < L, the diagonal cells of cycles >= Lh
                    uint32_t mis = Lh == L ? ok & ~diag : ok;
                    while (mis) {
                        const int u = (__ffs(mis) - 1) >> 3;
                        mis &= ~(0xFFu << (8 * u));
                        const uint32_t cyc = (uint32_t)(c0 + u * dir);
                        const uint32_t o = (bw >> (8 * u)) & 255u, rt = (rw >> (8 * u)) & 255u;
                        if (rt == o && cyc < (uint32_t)Lh) continue;           // counted in shared
                        count1(o, (qw >> (8 * u)) & 255u, rt, cyc);
                    }
                }
            }
        } else {
            // direct: byte loads from global (batch too wide for the stage buffers)
            const unsigned char* gb = A.R.bases + st_base[sidx];
            const unsigned char* gq = A.R.quals + st_base[sidx];
            for (uint32_t j = warp; j < nr; j += CAL_NW) {
                const uint64_t d = md[j];
                const uint32_t ls = ml[j], l = ls & 511u, minus = ls >> 9;
                const uint32_t bo = (uint32_t)(d >> 32);
                for (uint32_t i = lane; i < l; i += 32)
                    count1(gb[bo + i], gq[bo + i], A.ref[(uint32_t)d + i], minus ? l - 1 - i : i);
            }
        }
        if (k + 1 < nbatch) {
            // batch k+1's buffers were last read by batch k-1 (before this iteration's barrier)
            // and its counter m_n[(k+1)%3] was reset during batch k-1
            const Meta m = nxt;
            if (k + 2 < nbatch) nxt = meta_load(k + 2);
            meta_commit(m, sidx ^ 1, (int)((k + 1) % 3));
        }
    }
    if (err) atomicOr(A.err, err);
    __syncthreads();
    for (int i = tid; i < ncell; i += CAL_NT) {
        const uint32_t v = hist[i];
        if (v) {
            const uint32_t qt = (uint32_t)(i / Lh), c = (uint32_t)(i % Lh), q = qt >> 2, t = qt & 3;
            atomicAdd(&A.C[q << 12 | c << 4 | t << 2 | t], (unsigned long long)v);
        }
    }
}
// ------------------------------------------------------------------------------------------
// k_call_tile: one CTA = TS = 256 consecutive sites, one thread per site (GSNP's baseline
// parallelisation).  Shared-memory layout (host: call_smem_bytes()).
constexpr int TS = NT;
constexpr int COLS = 32;              // key slots per site, shallow kernel (thread path n <= 32)
#ifndef GSNP_CLAIM
#define GSNP_CLAIM 4
#endif
#ifndef GSNP_GB
#define GSNP_GB 2
#endif
constexpr int GB = GSNP_GB;           // reads whose bytes are in flight together in the gather
constexpr int COLS_MID = 64;          // key slots per site, mid-depth kernel (thread path n <= 64)
constexpr int COLS_DEEP = 128;        // key slots per site, deep kernel (thread path n <= 128)

struct TileSmem {
    uint32_t* col;       // [COLS][TS] keys: column of site t at col[j*TS + t]; a warp's 32
                         // columns double as its 1024-key buffer on the warp paths
    uint8_t* slotcnt;    // [NW][4 * 2L] per-warp (base, strand, coord) counters
    uint8_t* adj;        // copy of the adjust table (adj_bytes, 0 = use global)
};

// slot: reserve the per-warp dependency counters of the warp paths (k_warp_sites); k_call_tile
// leaves them out
__host__ __device__ inline size_t call_smem_bytes(int L, size_t adj_bytes, int cols, TileSmem* s,
                                                   unsigned char* base, bool slot = true) {
    size_t o_col = 0;
    size_t o_slot = align16(4 * (size_t)cols * TS);
    size_t o_adj = align16(o_slot + (slot ? (size_t)NW * 8 * L : 0));
    size_t total = align16(o_adj + adj_bytes);
    if (s) {
        s->col = reinterpret_cast<uint32_t*>(base + o_col);
        s->slotcnt = base + o_slot;
        s->adj = base + o_adj;
    }
    return total;
}

__device__ __forceinline__ uint32_t key_base(uint32_t k) { return (k >> 15) & 3u; }
__device__ __forceinline__ uint32_t key_q(uint32_t k) { return 63u - ((k >> 9) & 63u); }
__device__ __forceinline__ uint32_t key_cyc(uint32_t k) { return (k >> 1) & 255u; }
__device__ __forceinline__ uint32_t key_slot(uint32_t k) { return k & 511u; }   // cyc<<1|strand
constexpr uint32_t KEY_BSLOT = (3u << 15) | 511u;                               // base + slot

#ifndef GSNP_T_NOALLOC
#define GSNP_T_NOALLOC 0
#endif
#ifndef GSNP_P2_UNROLL
#define GSNP_P2_UNROLL 1
#endif
constexpr int kP2Unroll = GSNP_P2_UNROLL;      // rows in flight per thread in likelihood pass 2
#ifndef GSNP_FUSED_PASS
#define GSNP_FUSED_PASS 1
#endif
// read-only 16-byte load that does not allocate in L1 (the table has little L1 reuse)
__device__ __forceinline__ double2 ld_na(const double2* p) {
    double2 v;
    asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
    return v;
}
// Score-table row of Alg. 3: the 10 values of (qa, coord, base), stored padded to
// TROW = 12 doubles (96 bytes, 32-byte aligned: exactly three sectors) at
// ((qa*L + coord)*4 + base)*TROW and gathered with three 256-bit loads.
#ifndef GSNP_T256
#define GSNP_T256 1
#endif
constexpr int TROW = GSNP_T256 ? 12 : 10;
#ifndef GSNP_T_HINT
#define GSNP_T_HINT 1
#endif
__device__ __forceinline__ void ld256(const double* p, double& a, double& b, double& c, double& d) {
#if GSNP_T_HINT == 1      // rows do not allocate in L1 (little reuse; keeps the read bytes there)
    asm volatile("ld.global.nc.L1::no_allocate.v4.f64 {%0, %1, %2, %3}, [%4];"
                 : "=d"(a), "=d"(b), "=d"(c), "=d"(d) : "l"(p));
#elif GSNP_T_HINT == 2    // rows marked evict-last in L2 (the table stays resident)
    asm volatile("ld.global.nc.L2::evict_last.v4.f64 {%0, %1, %2, %3}, [%4];"
                 : "=d"(a), "=d"(b), "=d"(c), "=d"(d) : "l"(p));
#else
    asm volatile("ld.global.nc.v4.f64 {%0, %1, %2, %3}, [%4];"
                 : "=d"(a), "=d"(b), "=d"(c), "=d"(d) : "l"(p));
#endif
}
__device__ __forceinline__ void add_row(const double* __restrict__ T, int L, uint32_t qa,
                                        uint32_t cyc, uint32_t b, double* acc) {
    const double* row = T + ((size_t)(qa * (uint32_t)L + cyc) * 4u + b) * TROW;
#if GSNP_T256
    double v0, v1, v2, v3, v4, v5, v6, v7, v8, v9, p0, p1;
    ld256(row, v0, v1, v2, v3);
    ld256(row + 4, v4, v5, v6, v7);
    ld256(row + 8, v8, v9, p0, p1);
    acc[0] += v0; acc[1] += v1; acc[2] += v2; acc[3] += v3; acc[4] += v4;
    acc[5] += v5; acc[6] += v6; acc[7] += v7; acc[8] += v8; acc[9] += v9;
#else
    const double2* r2 = reinterpret_cast<const double2*>(row);
#if GSNP_T_NOALLOC
    double2 v0 = ld_na(r2 + 0), v1 = ld_na(r2 + 1), v2 = ld_na(r2 + 2), v3 = ld_na(r2 + 3),
            v4 = ld_na(r2 + 4);
#else
    double2 v0 = __ldg(r2 + 0), v1 = __ldg(r2 + 1), v2 = __ldg(r2 + 2), v3 = __ldg(r2 + 3),
            v4 = __ldg(r2 + 4);
#endif
    acc[0] += v0.x; acc[1] += v0.y; acc[2] += v1.x; acc[3] += v1.y; acc[4] += v2.x;
    acc[5] += v2.y; acc[6] += v3.x; acc[7] += v3.y; acc[8] += v4.x; acc[9] += v4.y;
#endif
}

// adjust(score, dep_count) through the host-built table (R3): adj[q][min(pcr,P)-1][min(g,G-1)]
__device__ __forceinline__ int adj_lookup(const CallArgs& A, uint32_t q, uint32_t pcr, uint32_t g) {
    uint32_t pi = min(pcr, (uint32_t)A.adjP) - 1u, gi = min(g, (uint32_t)A.adjG - 1u);
    return __ldg(A.adj + ((size_t)q * A.adjP + pi) * A.adjG + gi);
}
// same, from a copy of the table (shared memory in k_call_tile)
__device__ __forceinline__ int adj_lookup_t(const uint8_t* adj, int P, int G, uint32_t q,
                                            uint32_t pcr, uint32_t g) {
    uint32_t pi = min(pcr, (uint32_t)P) - 1u, gi = min(g, (uint32_t)G - 1u);
    return adj[(q * (uint32_t)P + pi) * (uint32_t)G + gi];
}

// ---- per-site epilogue helpers ---------------------------------------------------------------
__device__ __forceinline__ uint32_t pick4(uint32_t v0, uint32_t v1, uint32_t v2, uint32_t v3, int i) {
    return i == 0 ? v0 : i == 1 ? v1 : i == 2 ? v2 : v3;
}
__device__ __forceinline__ uint32_t f16(uint64_t pack, int b) { return (uint32_t)(pack >> (16 * b)) & 0xFFFFu; }

// Top-2 genotypes over lp (ties -> lowest n, R7); returns lp[t1] - lp[t2].  The best values
// are carried in registers (no dynamic index into lp, which would put lp in local memory).
__device__ __forceinline__ double top2(const double* lp, int& t1, int& t2) {
    double v1 = lp[0];
    t1 = 0;
#pragma unroll
    for (int k = 1; k < 10; ++k)
        if (lp[k] > v1) { v1 = lp[k]; t1 = k; }
    double v2 = 0.0;
    t2 = -1;
#pragma unroll
    for (int k = 0; k < 10; ++k)
        if (k != t1 && (t2 < 0 || lp[k] > v2)) { v2 = lp[k]; t2 = k; }
    return v1 - v2;
}

// genotype n -> alleles, Alg. 4 lines 13-17 order (AA AC AT AG CC CT CG TT TG GG)
__device__ __forceinline__ int geno_a1(int t) { return t < 4 ? 0 : t < 7 ? 1 : t < 9 ? 2 : 3; }
__device__ __forceinline__ int geno_a2(int t) {
    return t < 4 ? t : t < 7 ? t - 3 : t < 9 ? t - 5 : 3;
}

// Reference code and known-SNP row of a site (R6: -1 = novel prior).
__device__ __forceinline__ int64_t site_ref(const CallArgs& A, uint64_t site, int& refb) {
    const uint32_t rt = A.ref[site - A.origin];
    refb = (int)(rt & 7u);
    if (!(rt & 8u)) return -1;
    return (int64_t)lower_bound_u64(A.known_pos, 0, A.n_known, site);
}

// C8 p-value from the rank-sum pieces (het calls only: kept out of line, away from the hot path's
// instruction stream).  n1, n2: unique keys of allele 1 / 2; wsum, tie: see thread_finish_tail.
#ifndef GSNP_PIECES_INLINE
#define GSNP_PIECES_INLINE 1   // A/B: inline 10.75 ms vs out of line 11.24 at C2 (layout)
#endif
#ifndef GSNP_COLD_INLINE
__device__ __noinline__
#else
__device__ __forceinline__
#endif
double rank_sum_p(const CallArgs& A, uint32_t n1, uint32_t n2, double wsum, double tie) {
    if (n1 == 0 || n2 == 0) return 0.0;
    double n1d = (double)n1, n2d = (double)n2, Nd = (double)(n1 + n2);
    double mu = n1d * (Nd + 1.0) / 2.0;
    double var = n1d * n2d / 12.0 * ((Nd + 1.0) - tie / (Nd * (Nd - 1.0)));
    if (A.rank_cdf && tie == 0.0 && n1 <= GSNP_RANK_EXACT_MAX && n2 <= GSNP_RANK_EXACT_MAX) {
        // R20 exact: U = W - n1(n1+1)/2 is an integer when nothing ties
        const int u = (int)llrint(wsum - n1d * (n1d + 1.0) / 2.0);
        const double* F = A.rank_cdf + (size_t)(n1 * 33 + n2) * 1025;
        return fmin(1.0, 2.0 * fmin(F[u], F[(int)(n1 * n2) - u]));
    }
    if (!(var > 0.0)) return 1.0;
    double z = (wsum - mu) / sqrt(var);
    return erfc(fabs(z) / sqrt(2.0));
}

// C8/C9 and the 40-byte record (R8, R9).  The 32-slot kernel has one calling path and inlines it
// (measured 0.8% faster at C2); kernels with several paths share one out-of-line copy
// (site_record_ool) — their code must stay within the instruction cache.
// cu/qs: unique counts / quality sums per base; ca: all-hits counts; delta = lp[t1] - lp[t2];
// wsum/tie: rank-sum pieces (valid for heterozygous calls with both alleles observed).
__device__ __forceinline__ void site_record(const CallArgs& A, uint64_t site, int refb, int known,
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
    if (a1 != a2 && (A.flags & GSNP_RANK_SUM))
        rank_p = rank_sum_p(A, pick4(cu0, cu1, cu2, cu3, a1), pick4(cu0, cu1, cu2, cu3, a2), wsum, tie);
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

__device__ __noinline__ void site_record_ool(const CallArgs& A, uint64_t site, int refb, int known,
                                            int t1, double delta, double post1, uint32_t cu0,
                                            uint32_t cu1, uint32_t cu2, uint32_t cu3, uint32_t qs0,
                                            uint32_t qs1, uint32_t qs2, uint32_t qs3, uint32_t ca0,
                                            uint32_t ca1, uint32_t ca2, uint32_t ca3, uint32_t repeat,
                                            double wsum, double tie) {
    site_record(A, site, refb, known, t1, delta, post1, cu0, cu1, cu2, cu3, qs0, qs1, qs2, qs3, ca0,
                ca1, ca2, ca3, repeat, wsum, tie);
}

// ------------------------------------------------------------------------------------------
// Thread-per-site likelihood for n <= N <= 32 keys (the common case).  Each key was stored as
// key << 8 | (pcr - 1) by the gather (pcr = occurrences of its (base, strand, coord) so far in
// canonical order).  An in-register bitonic network sorts them (likelihood_sort; the pcr byte
// only breaks ties between identical keys), then Alg. 4 runs sequentially in canonical order —
// the same terms in the same order as the oracle — followed by C6-C9 and the record.
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

// Sort the first n (<= N) entries of this thread's column in registers and store them back.
template <int N>
__device__ __forceinline__ void sort_column(uint32_t* colp, uint32_t n) {
    uint32_t k[N];
#pragma unroll
    for (int j = 0; j < N; ++j) k[j] = (j < (int)n) ? colp[j * TS] : KEY_INF;
    sort_net<N>(k);
#pragma unroll
    for (int j = 0; j < N; ++j) if (j < (int)n) colp[j * TS] = k[j];
}

// key of a thread-path column entry after the likelihood pass(es)
#if GSNP_FUSED_PASS
#define COLKEY(w) ((w) >> 8)
#else
#define COLKEY(w) ((w) & 0x1FFFFu)
#endif

// C8 pieces of a het call from a column in canonical order (W = sum of pooled mid-ranks of the
// allele-1 qualities, tie = sum(t^3 - t)): each allele's keys are one run with qualities
// descending, so the pooled mid-ranks come from one merge from the low-quality ends.  Het calls
// only, so out of line.
#if !GSNP_PIECES_INLINE
__device__ __noinline__
#else
__device__ __forceinline__
#endif
double2 rank_pieces_sorted(const uint32_t* colp, uint64_t cu, int a1, int a2) {
    double wsum = 0.0, tie = 0.0;
    uint32_t sx = 0, sy = 0;
    for (int b = 0; b < a1; ++b) sx += f16(cu, b);
    for (int b = 0; b < a2; ++b) sy += f16(cu, b);
    uint32_t ix = sx + f16(cu, a1), iy = sy + f16(cu, a2);
    double less = 0.0;
    while (ix > sx || iy > sy) {
        const uint32_t qx = ix > sx ? key_q(COLKEY(colp[(ix - 1) * TS])) : 99u;
        const uint32_t qy = iy > sy ? key_q(COLKEY(colp[(iy - 1) * TS])) : 99u;
        const uint32_t v = min(qx, qy);
        uint32_t cx = 0, cy = 0;
        while (ix > sx && key_q(COLKEY(colp[(ix - 1) * TS])) == v) { ++cx; --ix; }
        while (iy > sy && key_q(COLKEY(colp[(iy - 1) * TS])) == v) { ++cy; --iy; }
        const double t = (double)(cx + cy);
        wsum += (double)cx * (less + (t + 1.0) / 2.0);
        tie += t * t * t - t;
        less += t;
    }
    return make_double2(wsum, tie);
}

// C6-C9 for one site held by one thread: priors, posterior, top-2, rank-sum pieces, record.
// SORTED: the column holds the site's keys in canonical order (rank-sum by one merge).
// HIST (unsorted columns of up to 128 keys): rank-sum pieces from quality histograms instead of
// pairwise counts.
template <bool DBG, bool SORTED, bool INL, bool HIST = false>
// lps: the novel log10 prior rows (R6) staged in shared memory; rt: the site's reference byte
// (code | known << 3), loaded when the site's group was taken.
__device__ __forceinline__ void thread_finish(const CallArgs& A, const double* lps, uint32_t rt,
                                              const uint32_t* colp,
                                              uint64_t site, uint32_t n, const double* acc,
                                              uint64_t cu, uint64_t qs, uint32_t ca0,
                                              uint32_t ca1, uint32_t ca2, uint32_t ca3,
                                              uint32_t rep) {
    // C6/C7: priors, posterior, top-2
    const int refb = (int)(rt & 7u);
    const int64_t kidx = (rt & 8u) ? (int64_t)lower_bound_u64(A.known_pos, 0, A.n_known, site) : -1;
    const double* prow = kidx >= 0 ? A.known_lp + kidx * 10 : lps + refb * 10;
    double lp[10], m = -INFINITY;
#pragma unroll
    for (int j = 0; j < 10; ++j) {
        lp[j] = acc[j] + prow[j];
        m = lp[j] > m ? lp[j] : m;
    }
    int t1, t2;
    const double delta = top2(lp, t1, t2);
    // posterior denominator in genotype order; a term below 1e-18 of the maximum cannot change
    // the double sum (every term is <= 1 and the maximum's term is exactly 1), so it is skipped
    // unless the debug dump wants every posterior
    const bool all_terms = DBG && A.dbg_post10 != nullptr;
    uint32_t need = 0;
#pragma unroll
    for (int j = 0; j < 10; ++j) need |= (all_terms || lp[j] - m > -18.0) ? 1u << j : 0u;
    double esum = 0.0;
    const uint32_t am = __activemask();
    while (__any_sync(am, need != 0)) {                // terms in genotype order, one per pass
        if (need) {
            const int jj = __ffs(need) - 1;
            need &= need - 1;
            double x = lp[0];
#pragma unroll
            for (int j = 1; j < 10; ++j) x = jj == j ? lp[j] : x;
            esum += exp10(x - m);
        }
    }
    // C8 pieces: W = sum of pooled mid-ranks of allele-1 qualities; tie = sum(t^3 - t)
    const int a1 = geno_a1(t1), a2 = geno_a2(t1);
    double wsum = 0.0, tie = 0.0;
    if (SORTED && a1 != a2 && (A.flags & GSNP_RANK_SUM) && f16(cu, a1) && f16(cu, a2)) {
        const double2 wt = rank_pieces_sorted(colp, cu, a1, a2);
        wsum = wt.x;
        tie = wt.y;
    }
    if (!SORTED && a1 != a2 && (A.flags & GSNP_RANK_SUM) && f16(cu, a1) && f16(cu, a2)) {
        if (HIST) {
            // column in chunk order: pooled mid-ranks from the two alleles' quality histograms (6-bit
            // qualities; counts of allele 1 / 2 in the low / high half of one word per quality), walked
            // from the lowest quality as the sorted merge does — every term is an integer or a
            // half-integer, so the sums are exact in either order
            uint32_t hq[64];
#pragma unroll
            for (int q = 0; q < 64; ++q) hq[q] = 0;
            for (uint32_t x = 0; x < n; ++x) {
                const uint32_t xk = colp[x * TS] >> 8;
                const uint32_t xb = key_base(xk), xq = key_q(xk);
                if (xb == (uint32_t)a1) hq[xq] += 1u;
                else if (xb == (uint32_t)a2) hq[xq] += 1u << 16;
            }
            double less = 0.0;
            for (int q = 0; q < 64; ++q) {
                const uint32_t c1 = hq[q] & 0xFFFFu, t = c1 + (hq[q] >> 16);
                if (t) {
                    const double td = (double)t;
                    wsum += (double)c1 * (less + (td + 1.0) / 2.0);
                    tie += td * td * td - td;
                    less += td;
                }
            }
        } else {
            // column in chunk order: pooled mid-ranks by pairwise counts (het calls only)
            for (uint32_t x = 0; x < n; ++x) {
                const uint32_t xk = colp[x * TS] >> 8;
                const uint32_t xb = key_base(xk), xq = key_q(xk);
                if (xb != (uint32_t)a1 && xb != (uint32_t)a2) continue;
                uint32_t less = 0, eq = 0;
                for (uint32_t y = 0; y < n; ++y) {
                    const uint32_t yk = colp[y * TS] >> 8, yb = key_base(yk), yq = key_q(yk);
                    const bool yin = yb == (uint32_t)a1 || yb == (uint32_t)a2;
                    less += yin && yq < xq;
                    eq += yin && yq == xq;
                }
                if (xb == (uint32_t)a1) wsum += (double)less + ((double)eq + 1.0) / 2.0;
                tie += (double)eq * (double)eq - 1.0;
            }
        }
    }
    if (DBG && (A.dbg_L10 || A.dbg_post10)) {
        const uint64_t s = site - A.w0;
        for (int j = 0; j < 10; ++j) {
            if (A.dbg_L10) A.dbg_L10[s * 10 + j] = acc[j];
            if (A.dbg_post10) A.dbg_post10[s * 10 + j] = exp10(lp[j] - m) / esum;
        }
    }
    if (INL)
        site_record(A, site, refb, kidx >= 0, t1, delta, 1.0 / esum, f16(cu, 0), f16(cu, 1),
                    f16(cu, 2), f16(cu, 3), f16(qs, 0), f16(qs, 1), f16(qs, 2), f16(qs, 3), ca0, ca1,
                    ca2, ca3, rep, wsum, tie);
    else
        site_record_ool(A, site, refb, kidx >= 0, t1, delta, 1.0 / esum, f16(cu, 0), f16(cu, 1),
                        f16(cu, 2), f16(cu, 3), f16(qs, 0), f16(qs, 1), f16(qs, 2), f16(qs, 3), ca0,
                        ca1, ca2, ca3, rep, wsum, tie);
}

template <bool DBG, bool INL>
__device__ __forceinline__ void thread_site(const CallArgs& A, const uint8_t* adj, const double* lps,
                                            uint32_t rt, uint32_t* colp,
                                            uint64_t site, uint32_t n, bool slow_pcr, uint32_t ca0,
                                            uint32_t ca1, uint32_t ca2, uint32_t ca3, uint32_t rep) {
    if (DBG && A.dbg_keys_sorted) {
        const uint32_t o = A.dbg_off[site - A.w0];
        for (uint32_t j = 0; j < n; ++j) A.dbg_keys_sorted[o + j] = colp[j * TS] >> 8;
    }
    // Alg. 4 lines 6-17 in canonical order, pass 1 (integers): dep_count reset per base
    // (l.8-11); pcr from the gather, or recounted when '-' strand reads of unequal length can
    // share a coordinate; g = distinct (strand, coord) so far in this base - 1 (R3);
    // q_adj = adjust(q, pcr, g).  Each key becomes key | q_adj << 17.
    uint64_t cu = 0, qs = 0;
    uint32_t prev_b = 4, distinct = 0;
    double acc[10];
#pragma unroll
    for (int j = 0; j < 10; ++j) acc[j] = 0.0;
    const double* __restrict__ T = A.T;
    const uint32_t L = (uint32_t)A.L;
#if GSNP_FUSED_PASS
    // one pass: q_adj and the Alg. 3 row per key (keys keep their key << 8 | pcr-1 form)
#pragma unroll kP2Unroll
    for (uint32_t j = 0; j < n; ++j) {
        const uint32_t kw = colp[j * TS];
        const uint32_t kk = kw >> 8, b = key_base(kk), q = key_q(kk);
        uint32_t pcr = (kw & 255u) + 1u;
        if (slow_pcr) {
            pcr = 1;
            for (uint32_t i = 0; i < j; ++i) pcr += (((colp[i * TS] >> 8) ^ kk) & KEY_BSLOT) == 0;
        }
        if (b != prev_b) { distinct = 0; prev_b = b; }
        distinct += pcr == 1;
        const uint32_t qa = (uint32_t)adj_lookup_t(adj, A.adjP, A.adjG, q, pcr, distinct - 1);
        add_row(T, (int)L, qa, key_cyc(kk), b, acc);
        cu += 1ull << (16 * b);
        qs += (uint64_t)q << (16 * b);
    }
#else
    for (uint32_t j = 0; j < n; ++j) {
        const uint32_t kw = colp[j * TS];
        const uint32_t kk = kw >> 8, b = key_base(kk), q = key_q(kk);
        uint32_t pcr = (kw & 255u) + 1u;
        if (slow_pcr) {
            pcr = 1;
            // entries before j already hold key | q_adj << 17
            for (uint32_t i = 0; i < j; ++i) pcr += ((colp[i * TS] ^ kk) & KEY_BSLOT) == 0;
        }
        if (b != prev_b) { distinct = 0; prev_b = b; }
        distinct += pcr == 1;
        colp[j * TS] = kk | (uint32_t)adj_lookup_t(adj, A.adjP, A.adjG, q, pcr, distinct - 1) << 17;
        cu += 1ull << (16 * b);
        qs += (uint64_t)q << (16 * b);
    }
    // pass 2: type_likely[n] += new_p_matrix[row][n] (Alg. 3) in canonical order; no load
    // depends on another, so several rows are in flight per thread
#pragma unroll kP2Unroll
    for (uint32_t j = 0; j < n; ++j) {
        const uint32_t kk = colp[j * TS];
        add_row(T, (int)L, kk >> 17, key_cyc(kk), key_base(kk), acc);
    }
#endif
    thread_finish<DBG, true, INL>(A, lps, rt, colp, site, n, acc, cu, qs, ca0, ca1, ca2, ca3, rep);
}

#ifndef GSNP_DEEP_U
#define GSNP_DEEP_U 3
#endif
// Deep thread path (32 < n <= 32*NCH, kernels built with 128 slots per site): each 32-key chunk
// of the column is sorted in registers, then an NCH-way streaming merge visits the keys in
// canonical order straight into Alg. 4 (q_adj and the Alg. 3 row per key).
template <bool DBG, int NCH>
__device__ __forceinline__ void thread_site_deep(const CallArgs& A, const uint8_t* adj,
                                                 const double* lps, uint32_t rt,
                                                 uint32_t* colp, uint64_t site, uint32_t n,
                                                 uint32_t ca0, uint32_t ca1, uint32_t ca2,
                                                 uint32_t ca3, uint32_t rep) {
#pragma unroll 1
    for (int c = 0; c < NCH; ++c) {
        const uint32_t cn = n > 32u * c ? min(32u, n - 32u * c) : 0u;
        if (cn) sort_column<32>(colp + (size_t)32 * c * TS, cn);
    }
    // merge heads packed as (column word << 2) | chunk (words are unique and < 2^25), so one
    // minimum gives the next key and its chunk; byte c of cur = position of chunk c's head
    uint32_t hk[NCH], cur = 0;
#pragma unroll
    for (int c = 0; c < NCH; ++c) hk[c] = 32u * c < n ? colp[32u * c * TS] << 2 | (uint32_t)c : KEY_INF;
    uint32_t* dbg = nullptr;
    if (DBG && A.dbg_keys_sorted) dbg = A.dbg_keys_sorted + A.dbg_off[site - A.w0];
    double acc[10];
#pragma unroll
    for (int j = 0; j < 10; ++j) acc[j] = 0.0;
    uint64_t cu = 0, qs = 0;
    uint32_t prev_b = 4, distinct = 0;
    const double* __restrict__ T = A.T;
    const uint32_t L = (uint32_t)A.L;
    // U keys are merged ahead and their rows loaded together (U rows in flight per thread): the
    // 128-slot kernel runs one 384-thread CTA per SM, so it has the registers and needs the
    // memory-level parallelism; the adds stay in canonical order
    constexpr int U = NCH >= 4 ? GSNP_DEEP_U : 1;
    for (uint32_t out0 = 0; out0 < n; out0 += U) {
        uint32_t rowv[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            rowv[u] = 0xFFFFFFFFu;
            if (out0 + u < n) {
                uint32_t best = hk[0];
#pragma unroll
                for (int c = 1; c < NCH; ++c) best = min(best, hk[c]);
                const uint32_t bc = best & 3u;
                const uint32_t ni = ((cur >> (8u * bc)) & 255u) + 1u, gi = 32u * bc + ni;
                cur += 1u << (8u * bc);
                const uint32_t nv = ni < 32u && gi < n ? colp[gi * TS] << 2 | bc : KEY_INF;
#pragma unroll
                for (int c = 0; c < NCH; ++c) hk[c] = (uint32_t)c == bc ? nv : hk[c];
                best >>= 2;                                  // the column word
                const uint32_t kk = best >> 8, b = key_base(kk), q = key_q(kk);
                if (DBG && dbg) dbg[out0 + u] = kk;
                const uint32_t pcr = (best & 255u) + 1u;
                if (b != prev_b) { distinct = 0; prev_b = b; }
                distinct += pcr == 1;
                const uint32_t qa = (uint32_t)adj_lookup_t(adj, A.adjP, A.adjG, q, pcr, distinct - 1);
                rowv[u] = (qa * L + key_cyc(kk)) * 4u + b;
                cu += 1ull << (16 * b);
                qs += (uint64_t)q << (16 * b);
            }
        }
        double v[U][12];
#pragma unroll
        for (int u = 0; u < U; ++u) {
#pragma unroll
            for (int k = 0; k < 12; ++k) v[u][k] = 0.0;
            if (rowv[u] != 0xFFFFFFFFu) {
                const double* row = T + (size_t)rowv[u] * TROW;
                ld256(row, v[u][0], v[u][1], v[u][2], v[u][3]);
                ld256(row + 4, v[u][4], v[u][5], v[u][6], v[u][7]);
                ld256(row + 8, v[u][8], v[u][9], v[u][10], v[u][11]);
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int k = 0; k < 10; ++k) acc[k] += v[u][k];
    }
    thread_finish<DBG, false, false, (NCH >= 4)>(A, lps, rt, colp, site, n, acc, cu, qs, ca0, ca1, ca2,
                                                 ca3, rep);
}

// ------------------------------------------------------------------------------------------
// Warp paths for n > 32.  The warp re-gathers the site's keys (plain 17-bit keys) into its
// slice of the col region: element e lives at col[(e >> 5) * TS + warp * 32 + (e & 31)].
__device__ __forceinline__ uint32_t wslot(int warp, uint32_t e) {
    return (e >> 5) * TS + warp * 32 + (e & 31);
}

__device__ __forceinline__ void group_epilogue(const CallArgs& A, uint64_t site, int refb,
                                               int64_t kidx, const double* L10,
                                               const uint32_t* cu, const uint32_t* qs,
                                               uint32_t ca0, uint32_t ca1, uint32_t ca2,
                                               uint32_t ca3, uint32_t rep, double wsum,
                                               double tie) {
    const int lane = threadIdx.x & 31;
    double lp[10], m = -INFINITY;
    const double* prow = kidx >= 0 ? A.known_lp + kidx * 10 : A.LP + refb * 10;
#pragma unroll
    for (int n = 0; n < 10; ++n) {
        lp[n] = L10[n] + prow[n];
        m = lp[n] > m ? lp[n] : m;
    }
    int t1, t2;
    const double delta = top2(lp, t1, t2);
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
        site_record(A, site, refb, kidx >= 0, t1, delta, 1.0 / esum, cu[0], cu[1],
                    cu[2], cu[3], qs[0], qs[1], qs[2], qs[3], ca0, ca1, ca2, ca3, rep, wsum, tie);
    }
}

// Warp gather of one site's unique non-N keys from the reads [ra, rb) into the warp slice (at
// most cap keys are stored: a deeper site goes to k_big_sites, which gathers again); returns the
// count.
// The same pass counts every read's non-N base at the site (all hits: c[4], their hits in rp,
// this lane's share; the caller reduces across the warp).
__device__ __forceinline__ uint32_t warp_gather(const CallArgs& A, uint32_t* col, int warp,
                                                uint64_t s, uint64_t ra, uint64_t rb, uint32_t cap,
                                                uint32_t (&c)[4], uint32_t& rp) {
    const int lane = threadIdx.x & 31;
    uint32_t m = 0;
    for (uint64_t r0 = ra; r0 < rb; r0 += 32) {
        const uint64_t r = r0 + lane;
        uint32_t key = KEY_INF;
        if (r < rb) {
            const uint64_t i = s - A.R.pos[r];               // huge when the read starts later
            const uint32_t l = A.R.len[r];
            if (i < l) {
                const uint64_t bi = A.R.off[r] - A.R.off0 + i;
                const uint32_t b = A.R.bases[bi];
                if (b < 4) {
                    const uint32_t h = A.R.hits[r];
#pragma unroll
                    for (int x = 0; x < 4; ++x) c[x] += b == (uint32_t)x;
                    rp += h;
                    if (h == 1) {
                        const uint32_t st = A.R.strand[r];
                        const uint32_t cyc = st ? l - 1 - (uint32_t)i : (uint32_t)i;
                        key = b << 15 | (63u - A.R.quals[bi]) << 9 | cyc << 1 | st;
                    }
                }
            }
        }
        const uint32_t v = __ballot_sync(FULL, key != KEY_INF);
        const uint32_t e = m + __popc(v & lanemask_lt());
        if (key != KEY_INF && e < cap) col[wslot(warp, e)] = key;
        m += __popc(v);
    }
    __syncwarp();
    return m;
}

// 32 < n <= 256: K keys per lane in registers, bitonic network over N = 32K, Alg. 4 walked
// chunk by chunk with match_any for same-slot peers and per-warp counters across chunks.
template <int K>
__device__ void warp_site(const CallArgs& A, const uint32_t* col, int warp, uint32_t n,
                          uint64_t site, uint32_t ca0, uint32_t ca1, uint32_t ca2, uint32_t ca3,
                          uint32_t rep, uint8_t* slotcnt) {
    constexpr int N = 32 * K;
    const int lane = threadIdx.x & 31;
    const int L2 = 2 * A.L;
    int refb;
    const int64_t kidx = site_ref(A, site, refb);
    uint32_t key[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {
        uint32_t e = k * 32 + lane;
        key[k] = (e < n) ? col[wslot(warp, e)] : KEY_INF;
    }
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
    const double* prow = kidx >= 0 ? A.known_lp + kidx * 10 : A.LP + refb * 10;
#pragma unroll
    for (int j = 0; j < 10; ++j) lp[j] = acc[j] + prow[j];
    int t1, t2;
    top2(lp, t1, t2);
    const int a1 = geno_a1(t1), a2 = geno_a2(t1);
    double wsum = 0.0, tie = 0.0;
    if ((A.flags & GSNP_RANK_SUM) && a1 != a2 && pick4(cu[0], cu[1], cu[2], cu[3], a1) &&
        pick4(cu[0], cu[1], cu[2], cu[3], a2)) {
#pragma unroll                            // constant indices: key[] stays in registers
        for (int k = 0; k < K; ++k) {
            const uint32_t x = key[k];
            const uint32_t xb = key_base(x), xq = key_q(x);
            const bool xin = x != KEY_INF && (xb == (uint32_t)a1 || xb == (uint32_t)a2);
            uint32_t less = 0, eq = 0;
#pragma unroll 1
            for (uint32_t e = 0; e < n; ++e) {
                const uint32_t y = col[wslot(warp, e)], yb = key_base(y), yq = key_q(y);
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
    group_epilogue(A, site, refb, kidx, acc, cu, qs, ca0, ca1, ca2, ca3, rep, wsum, tie);
}

// Dependency walk over keys already in canonical order, one warp, 32 per chunk: stores q_adj
// into bits 17..22 of each key (shared by the warp-deep and CTA paths).
template <typename Idx>
__device__ __forceinline__ void walk_chunks(const CallArgs& A, uint32_t* a, Idx idx, uint32_t n,
                                            uint8_t* slotcnt) {
    const int lane = threadIdx.x & 31;
    const int L2 = 2 * A.L;
    int d0 = 0, d1 = 0, d2 = 0, d3 = 0;
    const uint32_t lt = lanemask_lt(), le = lt | (1u << lane);
    for (uint32_t c0 = 0; c0 < n; c0 += 32) {
        const uint32_t e = c0 + lane;
        const bool valid = e < n;
        const uint32_t kk = valid ? a[idx(e)] : KEY_INF;
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
        if (valid) a[idx(e)] = (kk & 0x1FFFFu) | (uint32_t)adj_lookup(A, q, pcr, g) << 17;
    }
    __syncwarp();
    for (uint32_t e = lane; e < n; e += 32) slotcnt[key_base(a[idx(e)]) * L2 + key_slot(a[idx(e)])] = 0;
    __syncwarp();
}

// Rank-sum pieces over keys (bits 0..16 valid) by histogram over the 64 quality values.
template <typename Idx>
__device__ void hist_ranks(const uint32_t* a, Idx idx, uint32_t n, int a1, int a2, double& wsum,
                           double& tie) {
    uint32_t hx[64], hy[64];
    for (int v = 0; v < 64; ++v) { hx[v] = 0; hy[v] = 0; }
    for (uint32_t e = 0; e < n; ++e) {
        uint32_t b = key_base(a[idx(e)]), q = key_q(a[idx(e)]);
        if (b == (uint32_t)a1) hx[q]++;
        else if (b == (uint32_t)a2) hy[q]++;
    }
    double less = 0.0;
    wsum = 0.0;
    tie = 0.0;
    for (int v = 0; v < 64; ++v) {
        double t = (double)hx[v] + (double)hy[v];
        wsum += (double)hx[v] * (less + (t + 1.0) / 2.0);
        tie += t * t * t - t;
        less += t;
    }
}

// 256 < n <= 1024: the warp sorts its slice in shared memory (bitonic, arbitrary n), walks the
// chunks, then all lanes gather and reduce.
__device__ __noinline__ void warp_deep_site(const CallArgs& A, uint32_t* col, int warp,
                                            uint32_t n, uint64_t site, uint32_t ca0, uint32_t ca1,
                                            uint32_t ca2, uint32_t ca3, uint32_t rep,
                                            uint8_t* slotcnt) {
    const int lane = threadIdx.x & 31;
    auto idx = [warp](uint32_t e) { return wslot(warp, e); };
    uint32_t N2 = 1;
    while (N2 < n) N2 <<= 1;
    for (uint32_t size = 2; size <= N2; size <<= 1) {
        const uint32_t half = size >> 1;
        for (uint32_t t = lane; t < N2 / 2; t += 32) {
            uint32_t blk = t / half, o = t % half;
            uint32_t i = blk * size + o, j = blk * size + size - 1 - o;
            if (j < n) {
                uint32_t x = col[idx(i)], y = col[idx(j)];
                if (x > y) { col[idx(i)] = y; col[idx(j)] = x; }
            }
        }
        __syncwarp();
        for (uint32_t stride = size >> 2; stride > 0; stride >>= 1) {
            for (uint32_t t = lane; t < N2 / 2; t += 32) {
                uint32_t i = (t / stride) * 2 * stride + (t % stride), j = i + stride;
                if (j < n) {
                    uint32_t x = col[idx(i)], y = col[idx(j)];
                    if (x > y) { col[idx(i)] = y; col[idx(j)] = x; }
                }
            }
            __syncwarp();
        }
    }
    if (A.dbg_keys_sorted) {
        const uint32_t o = A.dbg_off[site - A.w0];
        for (uint32_t e = lane; e < n; e += 32) A.dbg_keys_sorted[o + e] = col[idx(e)];
        __syncwarp();
    }
    walk_chunks(A, col, idx, n, slotcnt);
    double acc[10];
#pragma unroll
    for (int j = 0; j < 10; ++j) acc[j] = 0.0;
    uint32_t cu[4] = {0, 0, 0, 0}, qs[4] = {0, 0, 0, 0};
    for (uint32_t e = lane; e < n; e += 32) {
        const uint32_t kk = col[idx(e)];
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
    int refb;
    const int64_t kidx = site_ref(A, site, refb);
    double wsum = 0.0, tie = 0.0;
    {
        const double* prow = kidx >= 0 ? A.known_lp + kidx * 10 : A.LP + refb * 10;
        double lp[10];
        for (int j = 0; j < 10; ++j) lp[j] = acc[j] + prow[j];
        int t1, t2;
        top2(lp, t1, t2);
        const int a1 = geno_a1(t1), a2 = geno_a2(t1);
        if (a1 != a2 && (A.flags & GSNP_RANK_SUM) && lane == 0) hist_ranks(col, idx, n, a1, a2, wsum, tie);
        wsum = __shfl_sync(FULL, wsum, 0);
        tie = __shfl_sync(FULL, tie, 0);
    }
    group_epilogue(A, site, refb, kidx, acc, cu, qs, ca0, ca1, ca2, ca3, rep, wsum, tie);
    __syncwarp();
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

// CTA path for n > 1024 (k_big_sites): keys in one shared buffer, CTA bitonic sort,
// warp 0 walks the chunks, all warps gather and reduce, warp 0 finishes.
__device__ __noinline__ void cta_site(const CallArgs& A, uint8_t* slotcnt, uint32_t* a,
                                      uint32_t n, uint64_t site, uint32_t ca0, uint32_t ca1,
                                      uint32_t ca2, uint32_t ca3, uint32_t rep, double* red) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    auto flat = [](uint32_t e) { return e; };
    cta_sort(a, n);
    if (A.dbg_keys_sorted) {
        const uint32_t o = A.dbg_off[site - A.w0];
        for (uint32_t e = threadIdx.x; e < n; e += NT) A.dbg_keys_sorted[o + e] = a[e];
    }
    if (warp == 0) walk_chunks(A, a, flat, n, slotcnt);
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
    if (warp == 0) {
        int refb;
        const int64_t kidx = site_ref(A, site, refb);
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
        double wsum = 0.0, tie = 0.0;
        const double* prow = kidx >= 0 ? A.known_lp + kidx * 10 : A.LP + refb * 10;
        double lp[10];
        for (int j = 0; j < 10; ++j) lp[j] = L10[j] + prow[j];
        int t1, t2;
        top2(lp, t1, t2);
        const int a1 = geno_a1(t1), a2 = geno_a2(t1);
        if (a1 != a2 && (A.flags & GSNP_RANK_SUM) && lane == 0) hist_ranks(a, flat, n, a1, a2, wsum, tie);
        wsum = __shfl_sync(FULL, wsum, 0);
        tie = __shfl_sync(FULL, tie, 0);
        group_epilogue(A, site, refb, kidx, L10, cut, qst, ca0, ca1, ca2, ca3, rep, wsum, tie);
    }
    __syncthreads();
}

// ------------------------------------------------------------------------------------------
// Sites with more than 32*CC unique keys are handed to k_big_sites through a global list.
struct BigSite {
    uint64_t site;
    uint32_t n, ca0, ca1, ca2, ca3, rep;
};

// The fused per-tile kernel (a4..a8).  Every warp owns 32 consecutive sites and works
// independently (no CTA barrier): counting + base_word gather (site-major, no atomics), then
// thread-per-site sort + likelihood + posterior + record; its sites with more than 32 keys
// follow on the warp paths; beyond 1024 keys they go to k_big_sites.
#ifndef GSNP_MID_UNIFORM
#define GSNP_MID_UNIFORM 1
#endif
#ifndef GSNP_REC_OOL
#define GSNP_REC_OOL 0
#endif
#ifndef GSNP_CALL_MINB
#define GSNP_CALL_MINB 3
#endif
// Which k_call_tile instantiation calls this window (decided on the device, so gsnp_call needs no
// host round trip): by the window's mean depth = reads overlapping it x L / sites (a3's read
// ranges), the 32-slot kernel below mid_at, the 64-slot kernel below deep_at, the 128-slot kernel
// (gsnp_deep.cu) above.  Every instantiation is launched; all but the chosen one return at once.
// Each sums a site's keys in canonical order while the site fits its thread path; deeper sites go
// to the warp / CTA paths (k_warp_sites, k_big_sites), whose sums may differ from a thread path's
// in the last bits — within the parity rules either way.
__device__ __forceinline__ int pick_variant(const CallArgs& A) {
    const uint64_t ng = (A.w1 - A.w0 + 31) / 32;
    const uint64_t nr = A.tile_rb[ng - 1] - A.tile_ra[0];
    const float depth = (float)((double)nr * A.L / (double)(A.w1 - A.w0));
    return depth >= A.deep_at ? 2 : depth >= A.mid_at ? 1 : 0;
}
template <int CC> __host__ __device__ constexpr int variant_of() { return CC >= 128 ? 2 : CC >= 64 ? 1 : 0; }

template <bool DBG, int CC>
__global__ void __launch_bounds__(NT, GSNP_CALL_MINB)
k_call_tile(const __grid_constant__ CallArgs A, uint32_t* wlist, uint32_t* wlist_n, uint32_t* work, uint32_t adj_smem) {
    if (reads_invalid(A.err) || pick_variant(A) != variant_of<CC>()) return;
    extern __shared__ __align__(16) unsigned char smem[];
    TileSmem sm;
    const size_t adj_bytes = adj_smem ? (size_t)64 * A.adjP * A.adjG : 0;
    call_smem_bytes(A.L, adj_bytes, CC, &sm, smem, false);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    for (size_t i = tid; i < adj_bytes; i += NT) sm.adj[i] = A.adj[i];
    __shared__ double lp_s[50];                             // novel log10 priors [ref][n] (R6)
    for (int i = tid; i < 50; i += NT) lp_s[i] = A.LP[i];
    const uint8_t* adj = adj_smem ? sm.adj : A.adj;
    uint32_t* colp = sm.col + tid;                           // this lane's column
    __syncthreads();
    const uint64_t n_groups = (A.w1 - A.w0 + 31) / 32;
    const bool all_one_len = *A.len_flag != A.epoch;          // every read has read 0's length
    // persistent warps: each takes the next group of 32 consecutive sites from a counter; the
    // next group's index and read range are fetched while the current one is processed
    // groups are claimed GSNP_CLAIM at a time (fewer atomics on the one counter) when every warp
    // gets many claims; a small window (the paper's 256 K sites: ~2 groups per warp) claims one
    // at a time so no warp is left with a tail of several groups
    const uint32_t claim = n_groups >= (uint64_t)8 * GSNP_CLAIM * gridDim.x * (NT / 32) ? GSNP_CLAIM : 1u;
    uint64_t nxt = 0, nra = 0, nrb = 0, claim_end = 0;
    if (lane == 0) nxt = atomicAdd(work, claim);
    nxt = __shfl_sync(FULL, nxt, 0);
    claim_end = nxt + claim;
    if (nxt < n_groups) { nra = A.tile_ra[nxt]; nrb = A.tile_rb[nxt]; }
    for (;;) {
    const uint64_t grp = nxt;
    if (grp >= n_groups) break;
    const uint64_t wra = nra;
    uint64_t wrb = nrb;
    if (grp + 1 < claim_end) {
        nxt = grp + 1;
    } else {
        if (lane == 0) nxt = atomicAdd(work, claim);
        nxt = __shfl_sync(FULL, nxt, 0);
        claim_end = nxt + claim;
    }
    if (nxt < n_groups) { nra = A.tile_ra[nxt]; nrb = A.tile_rb[nxt]; }
    const uint64_t g0 = A.w0 + grp * 32;                     // first site of the group
    const uint64_t site = g0 + lane;
    const bool active = site < A.w1;
    const uint32_t rt = active ? A.ref[site - A.origin] : 4u;   // issued early, used at the end

    // ---- counting + base_word gather, one site per lane.  The warp
    // walks the reads covering its 32 sites: metadata of 32 reads is loaded coalesced and
    // broadcast by shuffles; each lane reads the base and quality at its own site (consecutive
    // lanes -> consecutive bytes of a read).  Loads are issued four reads at a time.
    // Positions are handled relative to the group's first site g0 (32-bit).  If every read in
    // the range has the same length, '-' strand reads share a coordinate only within one start
    // run and the end tracking below is skipped.
    uint32_t one_len = 1;
    if (!all_one_len) {                                       // some read's length differs
        const uint32_t L0 = wra < wrb ? A.R.len[wra] : 0u;
        for (uint64_t r0 = wra; r0 < wrb; r0 += 32) {          // warp-uniform trip count
            const uint64_t r = r0 + lane;
            one_len &= (uint32_t)__all_sync(FULL, r >= wrb || A.R.len[r] == L0);
        }
    }
    uint32_t ca0 = 0, ca1 = 0, ca2 = 0, ca3 = 0, rep = 0, n = 0;
    bool slow_pcr = false, have_minus = false;
    int run_pos = INT32_MIN;
    uint32_t run_start = 0;
    int last_end = 0, last_end_pos = 0;      // read starts relative to g0 fit 32 bits (|pk| < 2^30)
    int err = 0;
    uint32_t bmax = 0, qmx = 0;                              // largest base code / quality seen
    uint32_t* dbg_built = nullptr;
    if (DBG && A.dbg_keys_built) dbg_built = A.dbg_keys_built + (active ? A.dbg_off[site - A.w0] : 0);
    // byte arrays addressed from the warp's first read with 32-bit offsets: the bases of the
    // reads covering 32 consecutive sites must span < 2 GB (else GSNP_E_RANGE)
    const uint64_t ob = wra < wrb ? A.R.off[wra] - A.R.off0 : 0;
    if (wra < wrb && A.R.off[wrb] - A.R.off[wra] >= (1ull << 31)) { err |= ERR_RANGE; wrb = wra; }
    const uint8_t* __restrict__ wbases = A.R.bases + ob;
    const uint8_t* __restrict__ wquals = A.R.quals + ob;
    const int lane_rel = active ? lane : INT32_MIN / 2;     // inactive lanes are never covered
    for (uint64_t r0 = wra; r0 < wrb; r0 += 32) {
        const uint64_t r = r0 + lane;
        int pr = INT32_MAX / 2;                                // read start - g0
        uint32_t o = 0;                                        // bases offset - ob
        uint32_t meta = 0;                                     // len | strand << 9 | hits << 10
        if (r < wrb) {
            pr = (int)((int64_t)A.R.pos[r] - (int64_t)g0);
            o = (uint32_t)(A.R.off[r] - A.R.off0 - ob);
            meta = (uint32_t)A.R.len[r] | (uint32_t)A.R.strand[r] << 9 | (uint32_t)A.R.hits[r] << 10;
        }
        const int nr = (int)min((uint64_t)32, wrb - r0);
        uint32_t cpack = 0;                                    // 4 x 8-bit base counts this batch
        for (int k0 = 0; k0 < nr; k0 += GB) {
            int pk[GB];
            uint32_t ii[GB], mk[GB], bb[GB], qq[GB];
#pragma unroll
            for (int u = 0; u < GB; ++u) {
                const int k = (k0 + u) & 31;
                pk[u] = __shfl_sync(FULL, pr, k);
                const uint32_t ok = __shfl_sync(FULL, o, k);
                mk[u] = __shfl_sync(FULL, meta, k);
                // past the batch: lanes k >= nr hold pr = INT32_MAX / 2 and meta = 0 already; only a
                // GB that does not divide 32 can wrap k past 31 onto lane 0
                if ((32 % GB) != 0 && k0 + u >= nr) pk[u] = INT32_MAX / 2;
                ii[u] = (uint32_t)(lane_rel - pk[u]);           // huge unless 0 <= i < len
                const bool cov = ii[u] < (mk[u] & 511u);
                bb[u] = cov ? wbases[ok + ii[u]] : 4u;
                qq[u] = cov ? wquals[ok + ii[u]] : 0u;
                if (!cov) mk[u] = 0;                           // len 0: not covered below
            }
#pragma unroll
            for (int u = 0; u < GB; ++u) {
                const uint32_t b = bb[u], q = qq[u];
                const uint32_t lk = mk[u] & 511u, sk = (mk[u] >> 9) & 1u, hk = mk[u] >> 10;
                bmax = max(bmax, b);                             // range checks after the group
                qmx = max(qmx, q);                               // (uncovered: b = 4, q = 0)
                const bool nb = b < 4;                           // a non-N aligned base
                cpack += shl_clamp(1u, 8 * b);                   // 0 for N (shift 32)
                rep += nb ? hk : 0u;
                const bool use = nb && hk == 1;                  // uniquely aligned
                const uint32_t i = ii[u];
                const uint32_t cyc = sk ? lk - 1 - i : i;
                // (a quality above 63 is a range error of the call; its bits only reach the masked
                // quality and base fields, never the coordinate)
                const uint32_t key = b << 15 | (63u - q) << 9 | cyc << 1 | sk;
                if (DBG && dbg_built && use) dbg_built[n] = key;
                // pcr: keys sharing (base, strand, coord) come from reads with the same start
                // ('+') or the same end ('-'); with equal starts they are one run of this
                // column.  Canonical order among them is quality descending (R3).
                if (pk[u] != run_pos) { run_pos = pk[u]; run_start = n; }
                uint32_t pcr1 = 0;
                if (use && run_start < n) {
                    const uint32_t jend = min(n, (uint32_t)CC);
                    for (uint32_t j = run_start; j < jend; ++j) {
                        const uint32_t kj = colp[j * TS];
                        if ((((kj >> 8) ^ key) & KEY_BSLOT) == 0) {
                            if (key_q(kj >> 8) >= q) ++pcr1;
                            else if ((kj & 255u) < 255u) colp[j * TS] = kj + 1;
                        }
                    }
                }
                if (!one_len) {       // '-' ends must rise between start runs, else recount pcr
                    const int e = pk[u] + (int)lk - 1;
                    const bool minus = use && sk;
                    slow_pcr |= minus && have_minus &&
                                (e < last_end || (e == last_end && pk[u] != last_end_pos));
                    last_end = minus ? e : last_end;
                    last_end_pos = minus ? pk[u] : last_end_pos;
                    have_minus |= minus;
                }
                if (use && n < CC) colp[n * TS] = key << 8 | min(pcr1, 255u);
                n += use;
            }
        }
        ca0 += cpack & 255u; ca1 += (cpack >> 8) & 255u; ca2 += (cpack >> 16) & 255u; ca3 += cpack >> 24;
    }
    err |= (bmax > 4 || qmx > (uint32_t)A.q_max) ? ERR_RANGE : 0;
    if (err) atomicOr(A.err, err);
    if (DBG && A.count_only) {
        if (active) A.dbg_nuni[site - A.w0] = n;
        continue;
    }

    // ---- thread-per-site sort (in-register 32-key network) + likelihood;
    // the deep kernel also keeps 33..128-key sites on the thread path (chunked sort + merge)
    bool small = active && n <= COLS;
    bool mid = CC > COLS && active && n > COLS && n <= CC && !slow_pcr;
#if GSNP_MID_UNIFORM
    // one path per warp: when any lane needs the chunked path, its small sites take it too (the
    // chunked path visits the keys in the same canonical order, so the sums are the same) instead
    // of the warp running both paths one after the other
    if (CC > COLS && __any_sync(FULL, mid) && small && !slow_pcr) { small = false; mid = true; }
#endif
    if (small) {
        sort_column<32>(colp, n);     // one network for every n <= 32: a second (16-key) network
                                      // measured 1.4% slower at C2 (instruction cache)
        thread_site<DBG, CC == COLS && !GSNP_REC_OOL>(A, adj, lp_s, rt, colp, site, n, slow_pcr, ca0, ca1,
                                                     ca2, ca3, rep);
    } else if (mid) {
        thread_site_deep<DBG, CC / 32>(A, adj, lp_s, rt, colp, site, n, ca0, ca1, ca2, ca3, rep);
    }
    __syncwarp();

    // ---- this warp's deeper sites go to the list that k_warp_sites works through (warp paths,
    // or k_big_sites beyond the warp buffer): their code stays out of this kernel's registers
    const bool deep = active && n > COLS && !mid;
    const uint32_t dv = __ballot_sync(FULL, deep);
    if (dv) {
        uint32_t base = 0;
        if (lane == 0) base = atomicAdd(wlist_n, (uint32_t)__popc(dv));
        base = __shfl_sync(FULL, base, 0);
        if (deep) wlist[base + __popc(dv & lanemask_lt())] = (uint32_t)(site - A.w0);
    }
    }  // persistent loop
}

// Sites listed by the 32-slot k_call_tile (more than 32 unique keys): one thread per listed site,
// 32 listed sites per warp.  Each thread walks its site's group read range (as the gather does,
// reads in position order, so the same pcr runs and '-' end checks apply), gathers the site's keys
// into its own 64-slot column and runs the chunked thread path; sites with more than 64 keys or a
// '-' end recount go on to k_warp_sites through the second list.  (Windows called by the 64- and
// 128-slot kernels return at once: their lists hold only sites beyond those kernels' slots.)
// Below A.list_min listed sites (default 16384; GSNP_LIST_MIN) the warp path takes them all: a
// thread walks its site's ~40 reads one round trip after another (~60 us whatever the count), while
// a warp per site finishes one site in ~14 us with every warp of the GPU in parallel (256 K-site
// windows list ~600 sites).
template <bool DBG>
__global__ void __launch_bounds__(NT, 3) k_list_sites(const __grid_constant__ CallArgs A, const uint32_t* wlist,
                                                      const uint32_t* wlist_n, uint32_t* wlist2,
                                                      uint32_t* wlist2_n, uint32_t* work) {
    if (reads_invalid(A.err) || pick_variant(A) != 0) return;
    const uint32_t count = *wlist_n;
    if (count < A.list_min) return;                     // a short list: the warp path is quicker
    if ((uint64_t)blockIdx.x * NT >= count) return;
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ double lp_s[50];
    const int tid = threadIdx.x, lane = tid & 31;
    for (int i = tid; i < 50; i += NT) lp_s[i] = A.LP[i];
    __syncthreads();
    uint32_t* colp = reinterpret_cast<uint32_t*>(smem) + tid;          // [COLS_MID][TS]
    const bool all_one_len = *A.len_flag != A.epoch;
    for (;;) {
        uint32_t j0 = 0;
        if (lane == 0) j0 = atomicAdd(work, 32u);
        j0 = __shfl_sync(FULL, j0, 0);
        if (j0 >= count) break;
        const uint32_t j = j0 + lane;
        const bool active = j < count;
        const uint64_t site = A.w0 + (active ? wlist[j] : 0u);
        const uint64_t grp = (site - A.w0) / 32;
        const uint64_t ra = A.tile_ra[grp], rb = active ? A.tile_rb[grp] : ra;
        const uint32_t rt = A.ref[site - A.origin];
        uint32_t ca0 = 0, ca1 = 0, ca2 = 0, ca3 = 0, rep = 0, n = 0, run_start = 0;
        uint64_t run_pos = ~0ull, last_end = 0, last_end_pos = 0;
        bool slow_pcr = false, have_minus = false;
        // read r's metadata is loaded one iteration ahead, so each read costs one round trip (its
        // bytes) instead of two
        uint64_t npos = ra < rb ? A.R.pos[ra] : 0, noff = ra < rb ? A.R.off[ra] : 0;
        uint32_t nlen = ra < rb ? A.R.len[ra] : 0u;
        for (uint64_t r = ra; r < rb; ++r) {
            const uint64_t pos = npos, off = noff;
            const uint32_t l = nlen;
            if (r + 1 < rb) { npos = A.R.pos[r + 1]; noff = A.R.off[r + 1]; nlen = A.R.len[r + 1]; }
            if (pos != run_pos) { run_pos = pos; run_start = n; }
            const uint64_t i = site - pos;                    // huge when the read starts later
            if (i >= l) continue;
            const uint64_t bi = off - A.R.off0 + i;
            // the read's bytes and flags in one round
            const uint32_t b = A.R.bases[bi], q = A.R.quals[bi], h = A.R.hits[r], st = A.R.strand[r];
            if (b >= 4) continue;                             // (range errors: the gather checked)
            ca0 += b == 0; ca1 += b == 1; ca2 += b == 2; ca3 += b == 3;
            rep += h;
            if (h != 1) continue;
            const uint32_t cyc = st ? l - 1 - (uint32_t)i : (uint32_t)i;
            const uint32_t key = b << 15 | (63u - q) << 9 | cyc << 1 | st;
            uint32_t pcr1 = 0;                                // pcr - 1 as in the gather (R3)
            const uint32_t jend = min(n, (uint32_t)COLS_MID);
            for (uint32_t k = run_start; k < jend; ++k) {
                const uint32_t kj = colp[k * TS];
                if ((((kj >> 8) ^ key) & KEY_BSLOT) == 0) {
                    if (key_q(kj >> 8) >= q) ++pcr1;
                    else if ((kj & 255u) < 255u) colp[k * TS] = kj + 1;
                }
            }
            if (!all_one_len && st) {                         // '-' ends must rise between runs
                const uint64_t e = pos + l - 1;
                slow_pcr |= have_minus && (e < last_end || (e == last_end && pos != last_end_pos));
                last_end = e;
                last_end_pos = pos;
                have_minus = true;
            }
            if (n < (uint32_t)COLS_MID) colp[n * TS] = key << 8 | min(pcr1, 255u);
            ++n;
        }
        const bool ok = active && n <= (uint32_t)COLS_MID && !slow_pcr;
        if (active && !ok) wlist2[atomicAdd(wlist2_n, 1u)] = wlist[j];
        if (ok) thread_site_deep<DBG, COLS_MID / 32>(A, A.adj, lp_s, rt, colp, site, n, ca0, ca1, ca2, ca3, rep);
        __syncwarp();
    }
}

// Sites listed by k_call_tile (n > COLS keys, or n > CC / '-' ends out of order on the deep
// kernel): one warp per site.  The warp recounts the site's all-hits counters over its group's
// read range, re-gathers the unique keys into its slice of the col region and runs the warp
// paths (n <= 32*CC) or hands the site to k_big_sites.
template <int CC>
__global__ void __launch_bounds__(NT) k_warp_sites(const __grid_constant__ CallArgs A, const uint32_t* wlist,
                                                   const uint32_t* wlist_n, const uint32_t* wlist2,
                                                   const uint32_t* wlist2_n, BigSite* big,
                                                   uint32_t* big_n, uint32_t big_cap) {
    if (reads_invalid(A.err)) return;
    if (pick_variant(A) == 0 && *wlist_n >= A.list_min) { wlist = wlist2; wlist_n = wlist2_n; }   // k_list_sites' leftovers
    const uint32_t count = *wlist_n;
    if ((uint64_t)blockIdx.x * NW >= count) return;     // one warp per listed site
    extern __shared__ __align__(16) unsigned char smem[];
    TileSmem sm;
    call_smem_bytes(A.L, 0, CC, &sm, smem);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    uint8_t* myslot = sm.slotcnt + warp * 8 * A.L;
    for (int i = lane; i < 2 * A.L; i += 32) reinterpret_cast<uint32_t*>(myslot)[i] = 0;
    __syncwarp();
    for (uint32_t j = blockIdx.x * NW + warp; j < count; j += gridDim.x * NW) {
        const uint64_t s = A.w0 + wlist[j];
        const uint64_t grp = (s - A.w0) / 32;
        const uint64_t ra = A.tile_ra[grp], rb = A.tile_rb[grp];
        uint32_t c[4] = {0, 0, 0, 0}, rp = 0;
        const uint32_t m = warp_gather(A, sm.col, warp, s, ra, rb, 32u * CC, c, rp);
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) {
#pragma unroll
            for (int x = 0; x < 4; ++x) c[x] += __shfl_xor_sync(FULL, c[x], d);
            rp += __shfl_xor_sync(FULL, rp, d);
        }
        if (m > 32u * CC) {
            if (lane == 0) {
                const uint32_t k = atomicAdd(big_n, 1u);
                if (k < big_cap) big[k] = BigSite{s, m, c[0], c[1], c[2], c[3], rp};
                else atomicOr(A.err, ERR_DEEP);
            }
            continue;
        }
        if (m <= 64) warp_site<2>(A, sm.col, warp, m, s, c[0], c[1], c[2], c[3], rp, myslot);
        else if (m <= 128) warp_site<4>(A, sm.col, warp, m, s, c[0], c[1], c[2], c[3], rp, myslot);
        else if (m <= 256) warp_site<8>(A, sm.col, warp, m, s, c[0], c[1], c[2], c[3], rp, myslot);
        else warp_deep_site(A, sm.col, warp, m, s, c[0], c[1], c[2], c[3], rp, myslot);
        __syncwarp();
    }
}

// Sites with more than 1024 unique keys: one CTA per site (persistent loop over the list),
// keys gathered into a shared buffer of `cap` keys (GSNP_E_CAPACITY beyond it).
__global__ void __launch_bounds__(NT) k_big_sites(const __grid_constant__ CallArgs A, const BigSite* big,
                                                  const uint32_t* big_n, uint32_t cap) {
    if (reads_invalid(A.err)) return;
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ double red[NW * 18];
    __shared__ uint32_t cnt;
    uint32_t* buf = reinterpret_cast<uint32_t*>(smem);
    uint8_t* slotcnt = smem + 4 * (size_t)cap;
    const int tid = threadIdx.x;
    const uint32_t count = *big_n;
    if (blockIdx.x >= count) return;                    // one CTA per listed site
    for (int i = tid; i < 2 * A.L; i += NT) reinterpret_cast<uint32_t*>(slotcnt)[i] = 0;
    for (uint32_t j = blockIdx.x; j < count; j += gridDim.x) {
        const BigSite bs = big[j];
        if (bs.n > cap) {
            if (tid == 0) atomicOr(A.err, ERR_DEEP);
            continue;
        }
        __syncthreads();
        if (tid == 0) cnt = 0;
        __syncthreads();
        const uint64_t s = bs.site;
        const uint64_t lo = s >= (uint64_t)(A.L - 1) ? s - (A.L - 1) : 0;
        const uint64_t ra = lower_bound_u64(A.R.pos, 0, A.R.n, lo);
        const uint64_t rb = lower_bound_u64(A.R.pos, ra, A.R.n, s + 1);
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
            const uint32_t key = b << 15 | (63u - A.R.quals[bi]) << 9 | cyc << 1 | st;
            const uint32_t slot = atomicAdd(&cnt, 1u);
            buf[slot] = key;
            if (A.dbg_keys_built) A.dbg_keys_built[A.dbg_off[s - A.w0] + slot] = key;
        }
        __syncthreads();
        cta_site(A, slotcnt, buf, cnt, s, bs.ca0, bs.ca1, bs.ca2, bs.ca3, bs.rep, red);
    }
}

}  // namespace gsnp_dev
