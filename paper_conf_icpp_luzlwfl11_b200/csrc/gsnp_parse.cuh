// gsnp_parse.cuh — SURVEY.md §8(f) NEXT #2: input packing on the GPU.  The alignment file (input
// file 1; "GSNP uses the same file format as SOAPsnp") arrives as text
// and is turned into the gsnp_reads arrays entirely by kernels (reading R19 of DESIGN.md):
//
//   k_nl_tiles<false>  per 16 KiB tile of text: number of '\n' (16-byte vector loads)
//   k_scan_partials    exclusive scan of the tile counts (one CTA)
//   k_nl_tiles<true>   per tile: block scans give every newline its line number; line_start[]
//   k_parse_meta       one warp per line: tab positions by ballot over 32-byte steps, the numeric
//                      fields (n_hits, len, location) by a warp-parallel decimal reduction, the
//                      chromosome compare, field validation -> packed per-line metadata
//   k_sel_tiles / k_scan_partials / k_sel_apply   read index and base offset of every selected
//                      line (exclusive scans of 1 and len over the lines of the wanted chr)
//   k_parse_emit       one warp per selected line: pos/len/strand/hits, off[], and the sequence /
//                      quality characters converted to codes (coalesced byte lanes)
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

// decimal field text[a, b) -> value (warp-parallel; b - a <= 19 digits); ok = all digits
__device__ __forceinline__ uint64_t warp_decimal(const uint8_t* text, uint64_t a, uint64_t b,
                                                 int lane, bool& ok) {
    const uint32_t nd = (uint32_t)(b - a);
    ok = nd >= 1 && nd <= 19;
    if (!ok) return 0;
    uint64_t v = 0;
    bool good = true;
    if ((uint32_t)lane < nd) {
        const uint32_t c = text[a + lane];
        good = c >= '0' && c <= '9';
        v = (uint64_t)(c - '0') * kPow10[nd - 1 - lane];
    }
    ok = __all_sync(FULL, good);
#pragma unroll
    for (int d = 16; d; d >>= 1) v += __shfl_xor_sync(FULL, v, d);
    return v;
}

__global__ void __launch_bounds__(PNT) k_parse_meta(ParseArgs P) {
    const int lane = threadIdx.x & 31;
    const uint64_t nw = (uint64_t)gridDim.x * (PNT / 32);
    for (uint64_t l = (uint64_t)blockIdx.x * (PNT / 32) + (threadIdx.x >> 5); l < P.n_lines; l += nw) {
        const uint64_t a = P.ls[l];
        uint64_t b = P.ls[l + 1] - 1;                    // the '\n' (or n_bytes for the last line)
        if (b > P.n_bytes) b = P.n_bytes;
        uint64_t meta = 0, pos = 0;
        if (b > a) {                                     // empty lines are skipped
            // tab positions t[0..8] (fields 1..9 start after them)
            uint64_t tab[9];
#pragma unroll
            for (int k = 0; k < 9; ++k) tab[k] = b;
            uint32_t ntab = 0;
            for (uint64_t p0 = a; p0 < b && ntab < 9; p0 += 32) {
                const uint64_t p = p0 + lane;
                const bool is_tab = p < b && P.text[p] == '\t';
                uint32_t m = __ballot_sync(FULL, is_tab);
                while (m && ntab < 9) {
                    const uint64_t tp = p0 + (uint64_t)(__ffs(m) - 1);
#pragma unroll
                    for (int k = 0; k < 9; ++k) tab[k] = (k == (int)ntab) ? tp : tab[k];
                    ++ntab;
                    m &= m - 1;
                }
            }
            bool ok = ntab >= 8;                          // 9 fields: id .. location
            const uint64_t f9_end = ntab >= 9 ? tab[8] : b;
            // chromosome (field 8: tab[6]+1 .. tab[7])
            bool want = ok;
            if (ok && P.chr_len) {
                const uint64_t ca = tab[6] + 1, cl = tab[7] - ca;
                bool eq = cl == P.chr_len;
                if (eq)
                    for (uint32_t i = lane; i < P.chr_len; i += 32) eq &= P.text[ca + i] == P.chr[i];
                want = __all_sync(FULL, eq);
            }
            if (want) {
                bool o1, o2, o3;
                const uint64_t hits = warp_decimal(P.text, tab[2] + 1, tab[3], lane, o1);
                const uint64_t len = warp_decimal(P.text, tab[4] + 1, tab[5], lane, o2);
                const uint64_t loc = warp_decimal(P.text, tab[7] + 1, f9_end, lane, o3);
                const uint64_t seq_a = tab[0] + 1, seq_len = tab[1] - seq_a;
                const uint64_t qual_len = tab[2] - (tab[1] + 1);
                const uint32_t sc = tab[6] - tab[5] == 2 ? P.text[tab[5] + 1] : 0u;
                ok = o1 && o2 && o3 && hits >= 1 && len >= 1 && len <= 256 && seq_len == len &&
                     qual_len == len && loc >= 1 && (sc == '+' || sc == '-') && seq_a - a < (1ull << 32);
                if (ok) {
                    const uint64_t h = hits > 65535 ? 65535 : hits;
                    meta = len | (uint64_t)(sc == '-') << 9 | 1ull << 10 | h << 11 |
                           (seq_a - a) << 32;
                    pos = loc - 1 + P.loc_base;
                }
            }
            if (!ok && lane == 0) {
                atomicOr(P.err, ERR_PARSE);
                atomicMin(P.bad_line, (unsigned long long)l);
            }
        }
        if (lane == 0) {
            P.meta[l] = meta;
            P.pos[l] = pos;
        }
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

// one warp per selected line: the gsnp_reads arrays
__global__ void __launch_bounds__(PNT) k_parse_emit(ParseArgs P, uint64_t n_sel, uint64_t n_bases) {
    const int lane = threadIdx.x & 31;
    const uint64_t nw = (uint64_t)gridDim.x * (PNT / 32);
    int err = 0;
    unsigned long long bad = ~0ull;
    for (uint64_t l = (uint64_t)blockIdx.x * (PNT / 32) + (threadIdx.x >> 5); l < P.n_lines; l += nw) {
        const uint64_t m = P.meta[l];
        if (!sel_of(m)) continue;
        const uint64_t r = P.ridx[l], o = P.boff[l];
        const uint32_t len = (uint32_t)len_of(m);
        const uint8_t* seq = P.text + P.ls[l] + (m >> 32);
        const uint8_t* qual = seq + len + 1;
        if (lane == 0) {
            P.o_pos[r] = P.pos[l];
            P.o_len[r] = (uint16_t)len;
            P.o_off[r] = o;
            P.o_strand[r] = (uint8_t)((m >> 9) & 1u);
            P.o_hits[r] = (uint16_t)((m >> 11) & 0xFFFFu);
            if (r + 1 == n_sel) P.o_off[n_sel] = n_bases;
        }
        bool good = true;
        for (uint32_t i = lane; i < len; i += 32) {
            const uint32_t c = seq[i] & 0xDFu;            // upper case
            const uint32_t code = c == 'A' ? 0u : c == 'C' ? 1u : c == 'T' ? 2u : c == 'G' ? 3u
                                : c == 'N' ? 4u : 255u;
            const uint32_t qc = qual[i];
            good &= code != 255u && qc >= P.q_offset && qc - P.q_offset <= 63u;
            P.o_bases[o + i] = (uint8_t)code;
            P.o_quals[o + i] = (uint8_t)(qc - P.q_offset);
        }
        if (!__all_sync(FULL, good)) { err = ERR_PARSE; bad = min(bad, (unsigned long long)l); }
    }
    if (err && lane == 0) {
        atomicOr(P.err, err);
        atomicMin(P.bad_line, bad);
    }
}

}  // namespace gsnp_dev
