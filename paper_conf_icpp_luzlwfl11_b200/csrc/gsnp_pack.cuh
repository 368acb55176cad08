// gsnp_pack.cuh — packed read format R21 (second half: GSNP's first pass
// writes a compressed copy of the input, about a third of its size, for the second pass to read,
// PAPER.md P:L708-727 §V-A, Fig. 10b).  On B200 the reads cross PCIe packed — 2-bit
// bases with an N exception list, qualities as runs of equal value, 6 bytes of
// metadata per read — and are unpacked in HBM by k_unpack.  Byte layout: DESIGN.md §3 R21 and
// oracle/pack.py (the test oracle, which shares no code with this file).
//
// Host side: pack_reads() (multi-threaded over blocks of reads), the header parser.
// Device side: k_unpack, one CTA per block of reads.
#pragma once
#include <cstdint>
#include <cstring>
#include <cuda_runtime.h>

namespace gsnp_pk {

constexpr uint32_t MAGIC = 0x31525347u;       // "GSR1" little-endian
constexpr uint32_t HDR = 128;
constexpr uint32_t MAX_BLOCK = 4096;          // reads per block (decoder's shared arrays)
constexpr int UNT = 256;                      // k_unpack threads per CTA

__host__ __device__ inline uint64_t a16(uint64_t x) { return (x + 15) & ~uint64_t(15); }

struct Header {                               // the 128-byte header, parsed
    uint32_t version;                         // 1: 2-bit bases; 2: reference-relative bases
    uint64_t n_reads, n_bases, n_runs, n_nexc, n_hexc;
    uint32_t n_blocks, block_reads;
    uint64_t sec[6];                          // blocks, meta, bases, runs, nexc, hexc
    // meta sub-arrays (each 16-byte aligned inside the meta section)
    uint64_t m_pos, m_len, m_sh, m_nrun;
};

inline void meta_offsets(Header& h) {
    h.m_pos = h.sec[1];
    h.m_len = a16(h.m_pos + 4 * h.n_reads);
    h.m_sh = a16(h.m_len + h.n_reads);
    h.m_nrun = a16(h.m_sh + h.n_reads);
}

// Parse and sanity-check a header (host memory); false if the bytes are not a GSR1 stream that
// fits in n_bytes.
inline bool parse_header(const uint8_t* p, uint64_t n_bytes, Header& h) {
    if (n_bytes < HDR) return false;
    uint32_t magic, ver;
    memcpy(&magic, p, 4);
    memcpy(&ver, p + 4, 4);
    if (magic != MAGIC || (ver != 1 && ver != 2)) return false;
    h.version = ver;
    memcpy(&h.n_reads, p + 8, 8);
    memcpy(&h.n_bases, p + 16, 8);
    memcpy(&h.n_runs, p + 24, 8);
    memcpy(&h.n_nexc, p + 32, 8);
    memcpy(&h.n_hexc, p + 40, 8);
    memcpy(&h.n_blocks, p + 48, 4);
    memcpy(&h.block_reads, p + 52, 4);
    memcpy(h.sec, p + 56, 48);
    if (h.block_reads == 0 || h.block_reads > MAX_BLOCK) return false;
    if ((uint64_t)h.n_blocks != (h.n_reads + h.block_reads - 1) / h.block_reads) return false;
    meta_offsets(h);
    const uint64_t end[6] = {h.sec[0] + 40ull * h.n_blocks, a16(h.m_nrun + h.n_reads),
                             h.sec[2] + (h.version == 1 ? (h.n_bases + 3) / 4 : 0), h.sec[3] + 2 * h.n_runs,
                             h.sec[4] + 4 * h.n_nexc, h.sec[5] + 8 * h.n_hexc};
    for (int k = 0; k < 6; ++k)
        if (h.sec[k] < HDR || end[k] > n_bytes || end[k] < h.sec[k]) return false;
    return true;
}

// ------------------------------------------------------------------------------------------
// Device: k_unpack.  CTA per block of reads: block-wide scans of the read lengths and run counts
// give every read's base and run offsets; warps then expand one read at a time (lanes take four
// consecutive positions: 2-bit codes from the base plane, the quality from a binary search of the
// read's run starts staged in shared memory); finally the block's N and hits exceptions are
// patched in.  Outputs are the gsnp_reads arrays, off[] rebuilt contiguous from 0.
struct UnpackArgs {
    const uint8_t* buf;                       // device copy of the stream (same byte offsets)
    Header h;
    const uint8_t* ref;                       // version 2: the context's reference codes
    uint64_t origin, n_sites;                 //            (code | known << 3) and its span
    uint32_t blk0;                            // first block of this launch
    uint64_t* pos;
    uint16_t* len;
    uint64_t* off;
    uint8_t* bases;
    uint8_t* quals;
    uint8_t* strand;
    uint16_t* hits;
};

__global__ void __launch_bounds__(UNT) k_unpack(const __grid_constant__ UnpackArgs U) {
    __shared__ uint32_t s_boff[MAX_BLOCK];    // base offset of each read inside the block
    __shared__ uint32_t s_roff[MAX_BLOCK];    // run offset of each read inside the block
    __shared__ uint32_t s_part[2][UNT / 32];
    __shared__ uint16_t s_rst[UNT / 32][257]; // per warp: run start positions of one read (+ end)
    __shared__ uint8_t s_rq[UNT / 32][256];   // per warp: run qualities
    const Header& h = U.h;
    const uint32_t b = U.blk0 + blockIdx.x;
    if (b >= h.n_blocks) return;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint64_t* bt = reinterpret_cast<const uint64_t*>(U.buf + h.sec[0]) + 5ull * b;
    const uint64_t pos0 = bt[0], base0 = bt[1], run0 = bt[2], ne0 = bt[3], he0 = bt[4];
    const uint64_t ne1 = b + 1 < h.n_blocks ? bt[8] : h.n_nexc;
    const uint64_t he1 = b + 1 < h.n_blocks ? bt[9] : h.n_hexc;
    const uint64_t r0 = (uint64_t)b * h.block_reads;
    const uint32_t nr = (uint32_t)min((uint64_t)h.block_reads, h.n_reads - r0);
    const uint32_t* m_pos = reinterpret_cast<const uint32_t*>(U.buf + h.m_pos) + r0;
    const uint8_t* m_len = U.buf + h.m_len + r0;
    const uint8_t* m_sh = U.buf + h.m_sh + r0;
    const uint8_t* m_nrun = U.buf + h.m_nrun + r0;
    // ---- block scans: thread t owns reads [t*per, (t+1)*per)
    const uint32_t per = (nr + UNT - 1) / UNT;
    const uint32_t i0 = min(nr, tid * per), i1 = min(nr, i0 + per);
    uint32_t sb = 0, sr = 0;
    for (uint32_t i = i0; i < i1; ++i) { sb += m_len[i] + 1u; sr += m_nrun[i] + 1u; }
    uint32_t xb = sb, xr = sr;                               // warp inclusive scans
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t yb = __shfl_up_sync(0xFFFFFFFFu, xb, d), yr = __shfl_up_sync(0xFFFFFFFFu, xr, d);
        if (lane >= d) { xb += yb; xr += yr; }
    }
    if (lane == 31) { s_part[0][warp] = xb; s_part[1][warp] = xr; }
    __syncthreads();
    uint32_t wb = 0, wr = 0;
    for (int k = 0; k < warp; ++k) { wb += s_part[0][k]; wr += s_part[1][k]; }
    uint32_t eb = wb + xb - sb, er = wr + xr - sr;           // exclusive prefix of thread's reads
    for (uint32_t i = i0; i < i1; ++i) {
        const uint32_t L = m_len[i] + 1u, sh = m_sh[i];
        s_boff[i] = eb;
        s_roff[i] = er;
        const uint64_t r = r0 + i;
        U.pos[r] = pos0 + m_pos[i];
        U.len[r] = (uint16_t)L;
        U.off[r] = base0 + eb;
        U.strand[r] = (uint8_t)(sh >> 7);
        U.hits[r] = (uint16_t)((sh & 127u) + 1u);
        eb += L;
        er += m_nrun[i] + 1u;
    }
    if (r0 + nr == h.n_reads && tid == UNT - 1) U.off[h.n_reads] = base0 + eb;   // last block
    __syncthreads();
    // ---- expand: warp per read
    const uint8_t* plane = U.buf + h.sec[2];
    const uint16_t* runs = reinterpret_cast<const uint16_t*>(U.buf + h.sec[3]);
    for (uint32_t i = warp; i < nr; i += UNT / 32) {
        const uint32_t L = m_len[i] + 1u, nrun = m_nrun[i] + 1u;
        const uint64_t kb = base0 + s_boff[i];               // first base (global index)
        const uint16_t* rr = runs + run0 + s_roff[i];
        uint32_t carry = 0;
        for (uint32_t j0 = 0; j0 < nrun; j0 += 32) {          // run starts by a warp scan
            const uint32_t j = j0 + lane;
            const uint32_t v = j < nrun ? rr[j] : 0u;
            const uint32_t rl = j < nrun ? (v & 255u) + 1u : 0u;
            uint32_t x = rl;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
                if (lane >= d) x += y;
            }
            if (j < nrun) { s_rst[warp][j] = (uint16_t)(carry + x - rl); s_rq[warp][j] = (uint8_t)(v >> 8); }
            carry += __shfl_sync(0xFFFFFFFFu, x, 31);
        }
        __syncwarp();
        // version 2: the predicted base is the reference code at the site (N where it is N)
        const uint64_t rs = h.version == 2 ? pos0 + m_pos[i] - U.origin : 0;
        for (uint32_t p0 = 4 * lane; p0 < L; p0 += 128) {
#pragma unroll
            for (uint32_t u = 0; u < 4; ++u) {
                const uint32_t p = p0 + u;
                if (p >= L) break;
                const uint64_t k = kb + p;
                uint32_t code;
                if (h.version == 1) code = (plane[k >> 2] >> (2 * (uint32_t)(k & 3))) & 3u;
                else {
                    const uint32_t rc = rs + p < U.n_sites ? U.ref[rs + p] & 7u : 4u;
                    code = rc < 4 ? rc : 4u;
                }
                uint32_t lo = 0, hi = nrun;                   // last run with start <= p
                while (hi - lo > 1) {
                    const uint32_t mid = (lo + hi) >> 1;
                    if (s_rst[warp][mid] <= p) lo = mid; else hi = mid;
                }
                U.bases[k] = (uint8_t)code;
                U.quals[k] = s_rq[warp][lo];
            }
        }
        __syncwarp();
    }
    __syncthreads();
    // ---- exceptions of this block
    const uint32_t* nexc = reinterpret_cast<const uint32_t*>(U.buf + h.sec[4]);
    if (h.version == 1)
        for (uint64_t e = ne0 + tid; e < ne1; e += UNT) U.bases[base0 + nexc[e]] = 4;
    else                                      // (block-relative base << 3 | code) of mismatches
        for (uint64_t e = ne0 + tid; e < ne1; e += UNT) U.bases[base0 + (nexc[e] >> 3)] = (uint8_t)(nexc[e] & 7u);
    const uint32_t* hexc = reinterpret_cast<const uint32_t*>(U.buf + h.sec[5]);
    for (uint64_t e = he0 + tid; e < he1; e += UNT) U.hits[r0 + hexc[2 * e]] = (uint16_t)hexc[2 * e + 1];
}

}  // namespace gsnp_pk

// ------------------------------------------------------------------------------------------
// Host encoder (the library's; the oracle's is oracle/pack.py).  Reads r0..n of host arrays in
// blocks of block_reads, spread over nt threads: pass 1 sizes every block (and validates), the
// block table and section offsets follow from prefix sums, pass 2 writes every block at its
// offsets.  The 2-bit plane is shared between neighbouring blocks only at their edge bytes, which
// are combined with atomic ORs.  Returns 0, or -1 (value out of range) / -2 (capacity).
namespace gsnp_pk {

struct HostReads {
    const uint8_t* ref;               // version 2: reference codes (NULL: version 1)
    uint64_t origin, n_sites;
    uint64_t n;
    const uint64_t* pos;
    const uint16_t* len;
    const uint64_t* off;
    const uint8_t* bases;
    const uint8_t* quals;
    const uint8_t* strand;
    const uint16_t* hits;
};

struct BlockSize { uint64_t bases, runs, nexc, hexc; int bad; };

inline BlockSize size_block(const HostReads& R, uint64_t r0, uint64_t r1) {
    BlockSize s{0, 0, 0, 0, 0};
    const uint64_t p0 = R.pos[r0];
    for (uint64_t r = r0; r < r1; ++r) {
        const uint32_t L = R.len[r];
        if (L < 1 || L > 256 || R.strand[r] > 1 || R.hits[r] < 1 || R.pos[r] < p0 ||
            R.pos[r] - p0 >= (1ull << 32)) { s.bad = 1; return s; }
        const uint8_t* b = R.bases + R.off[r];
        const uint8_t* q = R.quals + R.off[r];
        const uint8_t* rf = nullptr;
        if (R.ref) {
            if (R.pos[r] < R.origin || R.pos[r] - R.origin + L > R.n_sites) { s.bad = 1; return s; }
            rf = R.ref + (R.pos[r] - R.origin);
        }
        for (uint32_t i = 0; i < L; ++i) {
            if (b[i] > 4 || q[i] > 63) { s.bad = 1; return s; }
            if (rf) {
                const uint32_t rc = rf[i] & 7u;
                s.nexc += b[i] != (rc < 4 ? rc : 4u);
            } else {
                s.nexc += b[i] == 4;
            }
            s.runs += (i == 0 || q[i] != q[i - 1]);
        }
        s.bases += L;
        s.hexc += R.hits[r] >= 128;
    }
    return s;
}

inline void write_block(const HostReads& R, uint64_t r0, uint64_t r1, const Header& h,
                        const uint64_t* brow, uint8_t* out) {
    const uint64_t p0 = R.pos[r0];
    uint32_t* m_pos = reinterpret_cast<uint32_t*>(out + h.m_pos);
    uint8_t* m_len = out + h.m_len;
    uint8_t* m_sh = out + h.m_sh;
    uint8_t* m_nrun = out + h.m_nrun;
    uint8_t* plane = out + h.sec[2];
    uint16_t* runs = reinterpret_cast<uint16_t*>(out + h.sec[3]) + brow[2];
    uint32_t* nexc = reinterpret_cast<uint32_t*>(out + h.sec[4]) + brow[3];
    uint32_t* hexc = reinterpret_cast<uint32_t*>(out + h.sec[5]) + 2 * brow[4];
    const uint64_t kb0 = brow[1];
    uint64_t k = kb0;                                  // global base index
    const uint64_t kend = kb0 + [&] { uint64_t t = 0; for (uint64_t r = r0; r < r1; ++r) t += R.len[r]; return t; }();
    uint32_t acc = 0;                                  // the byte being assembled
    auto put_byte = [&](uint64_t byte, uint8_t v) {
        const bool edge = byte == (kb0 >> 2) || byte == ((kend - 1) >> 2);
        if (edge) __atomic_fetch_or(plane + byte, v, __ATOMIC_RELAXED);
        else plane[byte] = v;
    };
    for (uint64_t r = r0; r < r1; ++r) {
        const uint32_t L = R.len[r], hm = R.hits[r] - 1u;
        m_pos[r] = (uint32_t)(R.pos[r] - p0);
        m_len[r] = (uint8_t)(L - 1);
        m_sh[r] = (uint8_t)(R.strand[r] << 7 | (hm < 127 ? hm : 127u));
        if (hm >= 127) { *hexc++ = (uint32_t)(r - r0); *hexc++ = R.hits[r]; }
        const uint8_t* b = R.bases + R.off[r];
        const uint8_t* q = R.quals + R.off[r];
        const uint8_t* rf = R.ref ? R.ref + (R.pos[r] - R.origin) : nullptr;
        uint32_t nrun = 0;
        for (uint32_t i = 0; i < L; ++i, ++k) {
            uint32_t c = b[i];
            if (rf) {                                  // version 2: mismatches vs the reference
                const uint32_t rc = rf[i] & 7u;
                if (c != (rc < 4 ? rc : 4u)) *nexc++ = (uint32_t)(k - kb0) << 3 | c;
            } else {
                if (c == 4) { *nexc++ = (uint32_t)(k - kb0); c = 0; }
                acc |= c << (2 * (k & 3));
                if ((k & 3) == 3) { put_byte(k >> 2, (uint8_t)acc); acc = 0; }
            }
            if (i == 0 || q[i] != q[i - 1]) {
                uint32_t e = i + 1;
                while (e < L && q[e] == q[i]) ++e;
                *runs++ = (uint16_t)(q[i] << 8 | (e - i - 1));
                ++nrun;
            }
        }
        m_nrun[r] = (uint8_t)(nrun - 1);
    }
    if (!R.ref && (k & 3)) put_byte(k >> 2, (uint8_t)acc);
}

}  // namespace gsnp_pk
