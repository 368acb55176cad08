// gsnp_parse.cuh — SURVEY.md §8(f) NEXT #2: input packing on the GPU.  The alignment file (input
// file 1; "GSNP uses the same file format as SOAPsnp") arrives as text
// and is turned into the gsnp_reads arrays entirely by kernels (reading R19 of DESIGN.md):
//
//   k_nl_tiles<false>  per 16 KiB tile of text: number of '\n' (16-byte vector loads)
//   k_scan_partials    exclusive scan of the tile counts (one CTA)
//   k_nl_tiles<true>   per tile: block scans give every newline its line number; line_start[]
//   k_parse_meta       one 8-lane group per line (4 lines in flight per warp): the line staged in
//                      shared memory by 16-byte loads, tabs found 32 bytes per lane per step with
//                      a group prefix sum, numeric fields (n_hits, len, location) by a group-
//                      parallel decimal reduction, chromosome compare, validation -> packed
//                      per-line metadata
//   k_sel_tiles / k_scan_partials / k_sel_apply   read index and base offset of every selected
//                      line (exclusive scans of 1 and len over the lines of the wanted chr)
//   k_parse_emit       one 8-lane group per selected line: pos/len/strand/hits, off[], and the
//                      sequence / quality strings staged in shared memory and converted to codes
//                      four characters per 32-bit store
#pragma once

namespace gsnp_dev {

constexpr int PNT = 256;                        // threads per CTA in the parse kernels
constexpr uint32_t PTILE = PNT * 64;            // bytes of text per tile (4 x 16 B per thread)
constexpr uint32_t SEL_TILE = PNT * 16;         // lines per scan tile
constexpr int ERR_PARSE = 32;

// exclusive block scan (PNT threads) of one u64 per thread; *total = block sum
__device__ __forceinline__ uint64_t block_scan_excl(uint64_t v, uint64_t* total, uint64_t* sm) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    uint64_t x = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint64_t y = __shfl_up_sync(FULL, x, d);
        if (lane >= d) x += y;
    }
    if (lane == 31) sm[wid] = x;
    __syncthreads();
    if (wid == 0) {
        uint64_t w = lane < PNT / 32 ? sm[lane] : 0;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint64_t y = __shfl_up_sync(FULL, w, d);
            if (lane >= d) w += y;
        }
        if (lane < PNT / 32) sm[lane] = w;           // inclusive warp totals
    }
    __syncthreads();
    const uint64_t before = wid ? sm[wid - 1] : 0;
    *total = sm[PNT / 32 - 1];
    __syncthreads();
    return before + x - v;
}

__device__ __forceinline__ uint32_t nl_mask16(uint4 v) {     // bit k: byte k == '\n'
    uint32_t m = 0;
    const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int k = 0; k < 16; ++k) m |= (((w[k >> 2] >> (8 * (k & 3))) & 255u) == 10u) ? 1u << k : 0u;
    return m;
}

// WRITE=false: cnt[tile] = newlines in the tile.  WRITE=true: cnt holds the exclusive tile bases;
// line_start[j + 1] = 1 + position of newline j (line_start[0] = 0).
template <bool WRITE>
__global__ void __launch_bounds__(PNT) k_nl_tiles(const uint8_t* text, uint64_t n, uint64_t* cnt,
                                                  uint64_t* line_start) {
    __shared__ uint64_t sm[PNT / 32];
    const uint64_t t0 = (uint64_t)blockIdx.x * PTILE;
    uint64_t base = WRITE ? cnt[blockIdx.x] : 0, mine = 0;
    if (WRITE && blockIdx.x == 0 && threadIdx.x == 0) line_start[0] = 0;
#pragma unroll 1
    for (int k = 0; k < 4; ++k) {
        const uint64_t p = t0 + ((uint64_t)k * PNT + threadIdx.x) * 16;
        uint32_t m = 0;
        if (p + 16 <= n) m = nl_mask16(*reinterpret_cast<const uint4*>(text + p));
        else
            for (uint64_t i = p; i < n; ++i) m |= text[i] == '\n' ? 1u << (i - p) : 0u;
        if (!WRITE) { mine += __popc(m); continue; }
        uint64_t tot;
        uint64_t ex = block_scan_excl((uint64_t)__popc(m), &tot, sm);
        for (; m; m &= m - 1) line_start[base + ex++ + 1] = p + (uint64_t)(__ffs(m) - 1) + 1;
        base += tot;
    }
    if (!WRITE) {
        uint64_t tot;
        block_scan_excl(mine, &tot, sm);
        if (threadIdx.x == 0) cnt[blockIdx.x] = tot;
    }
}

// in-place exclusive scan of a[0..n) by one CTA; a[n] = total
__global__ void __launch_bounds__(PNT) k_scan_partials(uint64_t* a, uint64_t n) {
    __shared__ uint64_t sm[PNT / 32];
    uint64_t carry = 0;
    for (uint64_t i0 = 0; i0 < n; i0 += PNT) {
        const uint64_t i = i0 + threadIdx.x;
        const uint64_t v = i < n ? a[i] : 0;
        uint64_t tot;
        const uint64_t ex = block_scan_excl(v, &tot, sm);
        if (i < n) a[i] = carry + ex;
        carry += tot;
    }
    if (threadIdx.x == 0) a[n] = carry;
}

// per-line metadata: len | strand << 9 | sel << 10 | hits << 11 (16 bits) | seq offset in the
// line << 32.  sel = the line is a well-formed alignment on the wanted chromosome.
struct ParseArgs {
    const uint8_t* text;
    uint64_t n_bytes, n_lines;
    const uint64_t* ls;           // [n_lines + 1] line starts (ls[n_lines] = end of the last line + 1)
    const uint8_t* chr;           // wanted chromosome name (device), chr_len 0 = any
    uint32_t chr_len, q_offset;
    uint64_t loc_base;            // pos = location - 1 + loc_base
    uint64_t* meta;
    uint64_t* pos;
    uint64_t* ridx;               // exclusive scan of sel
    uint64_t* boff;               // exclusive scan of sel * len
    int* err;
    unsigned long long* bad_line; // first malformed line (atomicMin)
    // outputs (gsnp_reads arrays, device)
    uint64_t* o_pos; uint16_t* o_len; uint64_t* o_off; uint8_t* o_bases; uint8_t* o_quals;
    uint8_t* o_strand; uint16_t* o_hits;
};

__device__ __constant__ uint64_t kPow10[20] = {
    1ull, 10ull, 100ull, 1000ull, 10000ull, 100000ull, 1000000ull, 10000000ull, 100000000ull,
    1000000000ull, 10000000000ull, 100000000000ull, 1000000000000ull, 10000000000000ull,
    100000000000000ull, 1000000000000000ull, 10000000000000000ull, 100000000000000000ull,
    1000000000000000000ull, 10000000000000000000ull};

// Lines are handled by groups of PG = 8 lanes (four lines in flight per warp).  A group stages
// its line's bytes in shared memory with 16-byte loads (lines up to PSTAGE - 15 bytes; longer
// lines are read from global memory byte by byte — same code, slower source).
constexpr int PG = 8;
constexpr int PSTAGE = 640;                     // staging bytes per group
constexpr int PGROUPS = PNT / PG;               // groups per CTA

__device__ __forceinline__ uint32_t group_mask(int lane) { return 0xFFu << (lane & ~(PG - 1)); }

// group sum (lanes of one 8-lane group)
__device__ __forceinline__ uint64_t group_sum(uint64_t v) {
#pragma unroll
    for (int d = PG / 2; d; d >>= 1) v += __shfl_xor_sync(FULL, v, d);
    return v;
}

__global__ void __launch_bounds__(PNT) k_parse_meta(ParseArgs P) {
    __shared__ __align__(16) uint8_t stage_s[PGROUPS][PSTAGE + 32];    // + the scan's overhang
    __shared__ uint64_t tab_s[PGROUPS][9];
    const int lane = threadIdx.x & 31, sub = lane & (PG - 1), g = threadIdx.x / PG;
    const int gbase = lane & ~(PG - 1);                       // first lane of this group
    uint8_t* buf = stage_s[g];
    uint64_t* tabs = tab_s[g];
    const uint64_t ngroups = (uint64_t)gridDim.x * PGROUPS;
    // warp-uniform rounds; in each, group g takes line l0 + g
    for (uint64_t l0 = (uint64_t)blockIdx.x * PGROUPS + (threadIdx.x / 32) * (32 / PG);
         __any_sync(FULL, l0 + (lane / PG) < P.n_lines); l0 += ngroups) {
        const uint64_t l = l0 + (lane / PG);
        const bool act = l < P.n_lines;
        uint64_t a = 0, b = 0;
        if (act) {
            a = P.ls[l];
            b = P.ls[l + 1] - 1;                                 // the '\n' (or n_bytes)
            if (b > P.n_bytes) b = P.n_bytes;
            if (b < a) b = a;
        }
        const uint64_t A0 = a & ~15ull;
        const uint32_t nchunk = (uint32_t)((b - A0 + 15) / 16);
        const bool fast = nchunk * 16 <= PSTAGE;
        // stage the line: chunk c = sub + 8k, five 16-byte loads per lane at most
        uint4 v[PSTAGE / 16 / PG];
#pragma unroll
        for (int k = 0; k < PSTAGE / 16 / PG; ++k) {
            const uint32_t c = sub + PG * k;
            v[k] = make_uint4(0, 0, 0, 0);
            if (act && fast && c < nchunk) {
                const uint64_t q = A0 + 16 * (uint64_t)c;
                if (q + 16 <= P.n_bytes) v[k] = *reinterpret_cast<const uint4*>(P.text + q);
                else {                                         // the text's last, partial chunk
                    uint32_t w[4] = {0, 0, 0, 0};
                    for (uint64_t i = q; i < P.n_bytes; ++i) w[(i - q) >> 2] |= (uint32_t)P.text[i] << (8 * ((i - q) & 3));
                    v[k] = make_uint4(w[0], w[1], w[2], w[3]);
                }
            }
        }
#pragma unroll
        for (int k = 0; k < PSTAGE / 16 / PG; ++k) {
            const uint32_t c = sub + PG * k;
            if (act && fast && c < nchunk) *reinterpret_cast<uint4*>(buf + 16 * c) = v[k];
        }
        __syncwarp();
        auto at = [&](uint64_t p) -> uint32_t { return fast ? buf[p - A0] : P.text[p]; };
        // tabs in order: each lane scans 32 bytes per step; group prefix of the counts
        uint32_t ntab = 0;
        for (uint64_t p0 = A0; __any_sync(FULL, act && p0 < b && ntab < 9); p0 += 32 * PG) {
            const uint64_t q0 = p0 + 32 * (uint64_t)sub;
            uint32_t m = 0;
            if (act && p0 < b && ntab < 9) {
                if (fast && q0 < b) {
                    const uint4 x = *reinterpret_cast<const uint4*>(buf + (q0 - A0));
                    const uint4 y = *reinterpret_cast<const uint4*>(buf + (q0 - A0) + 16);
                    const uint32_t w[8] = {x.x, x.y, x.z, x.w, y.x, y.y, y.z, y.w};
#pragma unroll
                    for (int j = 0; j < 8; ++j) {          // byte == '\t' -> bit, 4 per word
                        const uint32_t e = __vcmpeq4(w[j], 0x09090909u) & 0x01010101u;
                        m |= ((e * 0x00204081u) >> 21 & 15u) << (4 * j);
                    }
                } else if (!fast) {
                    for (int k = 0; k < 32; ++k)
                        if (q0 + k < b && P.text[q0 + k] == '\t') m |= 1u << k;
                }
                // keep bytes inside [a, b)
                const uint64_t lo = q0 < a ? a - q0 : 0, hi = b > q0 ? b - q0 : 0;
                const uint32_t keep_hi = hi >= 32 ? ~0u : (1u << hi) - 1u;
                const uint32_t keep_lo = lo >= 32 ? 0u : ~((1u << lo) - 1u);
                m &= keep_hi & keep_lo;
            }
            uint32_t cnt = __popc(m), inc = cnt;
#pragma unroll
            for (int d = 1; d < PG; d <<= 1) {
                const uint32_t y = __shfl_up_sync(FULL, inc, d);
                if (sub >= d) inc += y;
            }
            uint32_t idx = ntab + inc - cnt;
            for (; m && idx < 9; m &= m - 1, ++idx) tabs[idx] = q0 + (uint64_t)(__ffs(m) - 1);
            ntab += __shfl_sync(FULL, inc, gbase + PG - 1);
        }
        __syncwarp();
        uint64_t tab[9];
#pragma unroll
        for (int k = 0; k < 9; ++k) tab[k] = (uint32_t)k < ntab ? tabs[k] : b;
        bool ok = ntab >= 8;                                     // 9 fields: id .. location
        bool want = act && b > a && ok;
        // chromosome (field 8: tab[6]+1 .. tab[7])
        bool eq = true;
        if (want && P.chr_len) {
            const uint64_t ca = tab[6] + 1;
            eq = tab[7] - ca == P.chr_len;
            if (eq)
                for (uint32_t i = sub; i < P.chr_len; i += PG) eq &= at(ca + i) == P.chr[i];
        }
        const uint32_t neq = __ballot_sync(FULL, !eq);          // every lane votes (no short circuit)
        want = want && (neq & group_mask(lane)) == 0;
        // numeric fields n_hits (3), len (5), location (8): digits spread over the group
        uint64_t fa[3] = {tab[2] + 1, tab[4] + 1, tab[7] + 1};
        uint64_t fb[3] = {tab[3], tab[5], ntab >= 9 ? tab[8] : b};
        uint64_t val[3];
        bool dig_ok = true;
#pragma unroll
        for (int f = 0; f < 3; ++f) {
            const uint64_t nd = want ? fb[f] - fa[f] : 0;
            uint64_t v = 0;
            if (want && (nd < 1 || nd > 19)) dig_ok = false;
            if (want && nd >= 1 && nd <= 19)
                for (uint32_t i = sub; i < nd; i += PG) {
                    const uint32_t c = at(fa[f] + i);
                    dig_ok &= c >= '0' && c <= '9';
                    v += (uint64_t)(c - '0') * kPow10[nd - 1 - i];
                }
            val[f] = group_sum(v);
        }
        const bool digits = (__ballot_sync(FULL, !dig_ok) & group_mask(lane)) == 0;
        uint64_t meta = 0, pos = 0;
        bool bad = act && b > a && !ok;
        if (want) {
            const uint64_t hits = val[0], len = val[1], loc = val[2];
            const uint64_t seq_a = tab[0] + 1, seq_len = tab[1] - seq_a;
            const uint64_t qual_len = tab[2] - (tab[1] + 1);
            const uint32_t sc = tab[6] - tab[5] == 2 ? at(tab[5] + 1) : 0u;
            const bool good = digits && hits >= 1 && len >= 1 && len <= 256 && seq_len == len &&
                              qual_len == len && loc >= 1 && (sc == '+' || sc == '-') &&
                              seq_a - a < (1ull << 32);
            if (good) {
                const uint64_t h = hits > 65535 ? 65535 : hits;
                meta = len | (uint64_t)(sc == '-') << 9 | 1ull << 10 | h << 11 | (seq_a - a) << 32;
                pos = loc - 1 + P.loc_base;
            } else {
                bad = true;
            }
        }
        if (act && sub == 0) {
            P.meta[l] = meta;
            P.pos[l] = pos;
            if (bad) {
                atomicOr(P.err, ERR_PARSE);
                atomicMin(P.bad_line, (unsigned long long)l);
            }
        }
        __syncwarp();
    }
}

__device__ __forceinline__ uint64_t sel_of(uint64_t m) { return (m >> 10) & 1u; }
__device__ __forceinline__ uint64_t len_of(uint64_t m) { return m & 511u; }

// per scan tile of SEL_TILE lines: number of selected lines and their bases -> part[2*tile]
__global__ void __launch_bounds__(PNT) k_sel_tiles(const uint64_t* meta, uint64_t n, uint64_t* part_n,
                                                   uint64_t* part_b) {
    __shared__ uint64_t sm[PNT / 32];
    const uint64_t i0 = (uint64_t)blockIdx.x * SEL_TILE;
    uint64_t cn = 0, cb = 0;
    for (uint32_t k = threadIdx.x; k < SEL_TILE; k += PNT) {
        const uint64_t i = i0 + k;
        if (i < n) {
            const uint64_t m = meta[i];
            cn += sel_of(m);
            cb += sel_of(m) * len_of(m);
        }
    }
    uint64_t tn, tb;
    block_scan_excl(cn, &tn, sm);
    block_scan_excl(cb, &tb, sm);
    if (threadIdx.x == 0) { part_n[blockIdx.x] = tn; part_b[blockIdx.x] = tb; }
}

// ridx / boff of every line (exclusive, in line order) from the scanned tile bases
__global__ void __launch_bounds__(PNT) k_sel_apply(ParseArgs P, const uint64_t* part_n,
                                                   const uint64_t* part_b) {
    __shared__ uint64_t sm[PNT / 32];
    const uint64_t i0 = (uint64_t)blockIdx.x * SEL_TILE;
    uint64_t bn = part_n[blockIdx.x], bb = part_b[blockIdx.x];
    for (uint32_t k0 = 0; k0 < SEL_TILE; k0 += PNT) {
        const uint64_t i = i0 + k0 + threadIdx.x;
        const uint64_t m = i < P.n_lines ? P.meta[i] : 0;
        uint64_t tn, tb;
        const uint64_t en = block_scan_excl(sel_of(m), &tn, sm);
        const uint64_t eb = block_scan_excl(sel_of(m) * len_of(m), &tb, sm);
        if (i < P.n_lines) { P.ridx[i] = bn + en; P.boff[i] = bb + eb; }
        bn += tn;
        bb += tb;
    }
}

// one 8-lane group per selected line (four lines in flight per warp): the gsnp_reads arrays.
// The line's sequence and quality strings are staged in shared memory with 16-byte loads; each
// lane then converts four characters at a time and writes them as one 32-bit store (the unaligned
// head and tail bytes of each output run are stored singly).
__device__ __forceinline__ uint32_t base_code(uint32_t c) {
    c &= 0xDFu;                                                // upper case
    return c == 'A' ? 0u : c == 'C' ? 1u : c == 'T' ? 2u : c == 'G' ? 3u : c == 'N' ? 4u : 255u;
}

__global__ void __launch_bounds__(PNT) k_parse_emit(ParseArgs P, uint64_t n_sel, uint64_t n_bases) {
    __shared__ __align__(16) uint8_t stage_s[PGROUPS][2 * 256 + 48];
    const int lane = threadIdx.x & 31, sub = lane & (PG - 1), g = threadIdx.x / PG;
    uint8_t* buf = stage_s[g];
    const uint64_t ngroups = (uint64_t)gridDim.x * PGROUPS;
    bool good = true;
    unsigned long long bad = ~0ull;
    for (uint64_t l0 = (uint64_t)blockIdx.x * PGROUPS + (threadIdx.x / 32) * (32 / PG);
         __any_sync(FULL, l0 + (lane / PG) < P.n_lines); l0 += ngroups) {
        const uint64_t l = l0 + (lane / PG);
        uint64_t m = 0, r = 0, o = 0, sp = 0;
        if (l < P.n_lines) {
            m = P.meta[l];
            if (sel_of(m)) { r = P.ridx[l]; o = P.boff[l]; sp = P.ls[l] + (m >> 32); }
        }
        const bool act = sel_of(m) != 0;
        const uint32_t len = (uint32_t)len_of(m);
        // stage seq '\t' qual: bytes [S0, sp + 2 len + 1) with S0 = sp rounded down to 16
        const uint64_t S0 = sp & ~15ull, S1 = sp + 2 * (uint64_t)len + 1;
        const uint32_t nchunk = act ? (uint32_t)((S1 - S0 + 15) / 16) : 0u;   // <= 33
#pragma unroll
        for (int k = 0; k < 5; ++k) {
            const uint32_t c = sub + PG * k;
            if (c < nchunk) {
                const uint64_t q = S0 + 16 * (uint64_t)c;
                uint4 v;
                if (q + 16 <= P.n_bytes) v = *reinterpret_cast<const uint4*>(P.text + q);
                else {
                    uint32_t w[4] = {0, 0, 0, 0};
                    for (uint64_t i = q; i < P.n_bytes; ++i) w[(i - q) >> 2] |= (uint32_t)P.text[i] << (8 * ((i - q) & 3));
                    v = make_uint4(w[0], w[1], w[2], w[3]);
                }
                *reinterpret_cast<uint4*>(buf + 16 * c) = v;
            }
        }
        __syncwarp();
        if (act) {
            if (sub == 0) {
                P.o_pos[r] = P.pos[l];
                P.o_len[r] = (uint16_t)len;
                P.o_off[r] = o;
                P.o_strand[r] = (uint8_t)((m >> 9) & 1u);
                P.o_hits[r] = (uint16_t)((m >> 11) & 0xFFFFu);
                if (r + 1 == n_sel) P.o_off[n_sel] = n_bases;
            }
            const uint32_t sb = (uint32_t)(sp - S0), qb = sb + len + 1;
            // word stores need bases and quals equally aligned (else every byte singly)
            const uintptr_t ab = reinterpret_cast<uintptr_t>(P.o_bases + o);
            const bool words = ((ab ^ reinterpret_cast<uintptr_t>(P.o_quals + o)) & 3) == 0;
            const uint32_t head = words ? min(len, (uint32_t)((4u - (uint32_t)(ab & 3)) & 3u)) : len;
            const uint32_t nw = (len - head) / 4, tail0 = head + 4 * nw;
            const uint32_t qo = P.q_offset;
            // single bytes: head [0, head) and tail [tail0, len): at most 6, one per lane
            for (uint32_t t = sub; t < head + (len - tail0); t += PG) {     // <= 6, or all if !words
                const uint32_t i = t < head ? t : tail0 + (t - head);
                const uint32_t bc = base_code(buf[sb + i]), qc = buf[qb + i];
                good &= bc != 255u && qc >= qo && qc - qo <= 63u;
                P.o_bases[o + i] = (uint8_t)bc;
                P.o_quals[o + i] = (uint8_t)(qc - qo);
            }
            for (uint32_t wi = sub; wi < nw; wi += PG) {
                const uint32_t i = head + 4 * wi;
                uint32_t wb = 0, wq = 0;
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const uint32_t bc = base_code(buf[sb + i + k]), qc = buf[qb + i + k];
                    good &= bc != 255u && qc >= qo && qc - qo <= 63u;
                    wb |= (bc & 255u) << (8 * k);
                    wq |= ((qc - qo) & 255u) << (8 * k);
                }
                *reinterpret_cast<uint32_t*>(P.o_bases + o + i) = wb;
                *reinterpret_cast<uint32_t*>(P.o_quals + o + i) = wq;
            }
            if (!good) bad = min(bad, (unsigned long long)l);
        }
        __syncwarp();
    }
    if (!good) {
        atomicOr(P.err, ERR_PARSE);
        atomicMin(P.bad_line, bad);
    }
}

}  // namespace gsnp_dev
