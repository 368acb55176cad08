// gsnp_dense.cuh — SURVEY.md §8(f) NEXT #3: the GPU *dense* likelihood ablation (P:L899-917,
// Fig. 5).  SOAPsnp's Alg. 1 on the device, with the paper's dense layout: one
// base_occ[4][64][256][2] array of 1-byte occurrence counts per site (131,072 B, P:L387-394,
// index base<<15 | score<<9 | coord<<1 | strand), filled by `counting`, walked in full
// loop-nest order by `likelihood`, re-zeroed by `recycle`.  The paper
// measured its GPU dense route 14-17x slower than the sparse one; this is the B200
// counterpart of that experiment, built so that it gives the same records as gsnp_call (same
// Alg. 3 terms added in the same canonical order, same posterior/call/record epilogue).
//
//   k_dense_count  one warp per read of the chunk's read range: per-site all-hits counters
//                  (count_all[4], Σhits) by u32 atomics, unique non-N bases into base_occ by
//                  byte-lane u32 atomics (a count reaching 256 would carry into its neighbour:
//                  flagged as ERR_DENSE_SAT -> GSNP_E_CAPACITY, reading R13 / P:L390).
//   k_dense_sites  one warp per site: for base 0..3, score q_max..0 the warp loads the 2L bytes
//                  of coord x strand (one 16-byte vector per lane, four rows in flight), finds the
//                  non-zero counts by ballot, and applies Alg. 1 lines 8-12 to each in order —
//                  dep_count (shared memory, reset per base), the global dependency count, adjust
//                  through the host-built table, and lanes 0..9 add the Alg. 3 row of genotype
//                  n = lane.  C6-C9 and the record follow in lane 0.
//   recycle        cudaMemsetAsync of the chunk's base_occ (the dense route's third cost).
#pragma once

namespace gsnp_dev {

constexpr uint32_t DENSE_SITE_BYTES = 4u * 64u * 256u * 2u;   // 131,072
constexpr int DENSE_NT = 256;                                  // 8 warps = 8 sites per CTA
constexpr int ERR_DENSE_SAT = 16;

struct DenseArgs {
    CallArgs A;                 // reads, tables, window [w0, w1), tile ranges, out, err
    uint64_t c0, c1;            // this chunk's sites
    uint8_t* occ;               // [c1 - c0][131072] base_occ, zero on entry
    uint32_t* cnt;              // [c1 - c0][5] count_all[4], Σhits; zero on entry
};

// counting: every base of every read that can touch [c0, c1)
__global__ void __launch_bounds__(DENSE_NT) k_dense_count(const __grid_constant__ DenseArgs D) {
    const CallArgs& A = D.A;
    if (reads_invalid(A.err)) return;
    const uint64_t ga = (D.c0 - A.w0) / 32, gb = (D.c1 - 1 - A.w0) / 32;
    const uint64_t ra = A.tile_ra[ga], rb = A.tile_rb[gb];
    const int lane = threadIdx.x & 31;
    const uint64_t nwarps = (uint64_t)gridDim.x * (DENSE_NT / 32);
    int err = 0;
    for (uint64_t r = ra + (blockIdx.x * (DENSE_NT / 32) + (threadIdx.x >> 5)); r < rb; r += nwarps) {
        const uint64_t p = A.R.pos[r];
        const uint32_t len = A.R.len[r], sk = A.R.strand[r], hk = A.R.hits[r];
        const uint64_t o = A.R.off[r] - A.R.off0;
        for (uint32_t i = lane; i < len; i += 32) {
            const uint64_t site = p + i;
            if (site < D.c0 || site >= D.c1) continue;
            const uint32_t b = A.R.bases[o + i];
            if (b > 4 || A.R.quals[o + i] > (uint32_t)A.q_max) { err |= ERR_RANGE; continue; }
            if (b == 4) continue;                                   // N: not aligned
            const uint64_t s = site - D.c0;
            atomicAdd(D.cnt + s * 5 + b, 1u);
            atomicAdd(D.cnt + s * 5 + 4, hk);
            if (hk != 1) continue;                                  // uniquely aligned only
            const uint32_t q = A.R.quals[o + i];
            const uint32_t cyc = sk ? len - 1 - i : i;
            const uint32_t idx = b << 15 | q << 9 | cyc << 1 | sk;
            uint8_t* cell = D.occ + s * DENSE_SITE_BYTES + idx;
            uint32_t* word = reinterpret_cast<uint32_t*>(reinterpret_cast<uintptr_t>(cell) & ~(uintptr_t)3);
            const uint32_t sh = 8u * (uint32_t)(reinterpret_cast<uintptr_t>(cell) & 3);
            const uint32_t old = atomicAdd(word, 1u << sh);
            if (((old >> sh) & 255u) == 255u) err |= ERR_DENSE_SAT;
        }
    }
    if (err) atomicOr(A.err, err);
}

// likelihood (Alg. 1) + posterior + record, one warp per site
__global__ void __launch_bounds__(DENSE_NT) k_dense_sites(const __grid_constant__ DenseArgs D) {
    __shared__ uint16_t dep_s[DENSE_NT / 32][512];                 // dep_count[coord<<1|strand]
    __shared__ uint32_t hist_s[DENSE_NT / 32][4][64];              // unique keys per (base, q)
    const CallArgs& A = D.A;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    uint16_t* dep = dep_s[wid];
    uint32_t (*hist)[64] = hist_s[wid];
    const uint32_t L = (uint32_t)A.L;
    const uint32_t nvec = (2 * L + 15) / 16;                       // 16-byte vectors per row
    const uint64_t nsite = D.c1 - D.c0;
    const uint64_t nwarps = (uint64_t)gridDim.x * (DENSE_NT / 32);
    for (uint64_t s = (uint64_t)blockIdx.x * (DENSE_NT / 32) + wid; s < nsite; s += nwarps) {
        const uint8_t* occ = D.occ + s * DENSE_SITE_BYTES;
        for (int j = lane; j < 256; j += 32) (&hist[0][0])[j] = 0;
        double acc = 0.0;                                          // type_likely[n = lane]
        uint32_t cu[4] = {0, 0, 0, 0}, qs[4] = {0, 0, 0, 0};
        for (uint32_t b = 0; b < 4; ++b) {
            for (int j = lane; j < 512; j += 32) dep[j] = 0;       // Alg. 1: dep_count reset per base
            __syncwarp();
            int gdep = -1;                                         // global dependency count
            for (int sc0 = A.q_max; sc0 >= 0; sc0 -= 4) {
                uint4 v[4];
#pragma unroll
                for (int u = 0; u < 4; ++u) {                      // four score rows in flight
                    const int sc = sc0 - u;
                    v[u] = make_uint4(0, 0, 0, 0);
                    if (sc >= 0 && (uint32_t)lane < nvec)
                        v[u] = *reinterpret_cast<const uint4*>(occ + (b << 15 | (uint32_t)sc << 9) + lane * 16);
                }
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const int sc = sc0 - u;
                    if (sc < 0) break;
                    // non-zero bytes of this lane's 16 (coord x strand ascending with the byte)
                    uint32_t nz = 0;
                    const uint32_t w[4] = {v[u].x, v[u].y, v[u].z, v[u].w};
#pragma unroll
                    for (int k = 0; k < 16; ++k) nz |= ((w[k >> 2] >> (8 * (k & 3))) & 255u) ? 1u << k : 0u;
                    uint32_t row_n = 0;
                    for (uint32_t bal = __ballot_sync(FULL, nz != 0); bal; bal = __ballot_sync(FULL, nz != 0)) {
                        const int ld = __ffs(bal) - 1;             // first lane with a count
                        uint32_t e = 0, o = 0;
                        if (lane == ld) {
                            const int k = __ffs(nz) - 1;
                            nz &= nz - 1;
                            e = (uint32_t)lane * 16 + (uint32_t)k;
                            o = (w[k >> 2] >> (8 * (k & 3))) & 255u;
                        }
                        e = __shfl_sync(FULL, e, ld);
                        o = __shfl_sync(FULL, o, ld);
                        const uint32_t c = e >> 1;                 // e = coord << 1 | strand
                        if (c >= L) continue;
                        uint32_t d = dep[e];
                        for (uint32_t k = 0; k < o; ++k) {         // Alg. 1 lines 8-12, occ times
                            if (d == 0) ++gdep;
                            ++d;
                            const uint32_t qa = (uint32_t)adj_lookup(A, (uint32_t)sc, d, (uint32_t)gdep);
                            if (lane < 10)
                                acc += __ldg(A.T + ((size_t)(qa * L + c) * 4u + b) * TROW + lane);
                        }
                        __syncwarp();
                        if (lane == 0) dep[e] = (uint16_t)min(d, 65535u);
                        __syncwarp();
                        row_n += o;
                    }
                    cu[b] += row_n;
                    qs[b] += row_n * (uint32_t)sc;
                    if (lane == 0) hist[b][sc] = row_n;
                }
            }
            __syncwarp();
        }
        // ---- C6/C7 (as thread_finish): lp, top-2, posterior sum in genotype order
        double lp[10];
#pragma unroll
        for (int j = 0; j < 10; ++j) lp[j] = __shfl_sync(FULL, acc, j);
        __syncwarp();
        if (lane == 0) {
            const uint64_t site = D.c0 + s;
            int refb;
            const int64_t kidx = site_ref(A, site, refb);
            const double* prow = kidx >= 0 ? A.known_lp + kidx * 10 : A.LP + refb * 10;
            double m = -INFINITY;
#pragma unroll
            for (int j = 0; j < 10; ++j) {
                lp[j] = lp[j] + __ldg(prow + j);
                m = lp[j] > m ? lp[j] : m;
            }
            int t1, t2;
            const double delta = top2(lp, t1, t2);
            double esum = 0.0;
#pragma unroll
            for (int j = 0; j < 10; ++j)
                if (lp[j] - m > -18.0) esum += exp10(lp[j] - m);
            // C8 pieces from the (base, q) histogram, qualities ascending (= the merge order)
            const int a1 = geno_a1(t1), a2 = geno_a2(t1);
            double wsum = 0.0, tie = 0.0;
            if (a1 != a2 && (A.flags & GSNP_RANK_SUM) && cu[a1] && cu[a2]) {
                double less = 0.0;
                for (int q = 0; q < 64; ++q) {
                    const uint32_t cx = hist[a1][q], cy = hist[a2][q];
                    if (cx + cy == 0) continue;
                    const double t = (double)(cx + cy);
                    wsum += (double)cx * (less + (t + 1.0) / 2.0);
                    tie += t * t * t - t;
                    less += t;
                }
            }
            const uint32_t* cn = D.cnt + s * 5;
            site_record(A, site, refb, kidx >= 0, t1, delta, 1.0 / esum, cu[0], cu[1],
                        cu[2], cu[3], qs[0], qs[1], qs[2], qs[3], cn[0], cn[1], cn[2], cn[3], cn[4],
                        wsum, tie);
        }
        __syncwarp();
    }
}

}  // namespace gsnp_dev
