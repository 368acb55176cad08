/*
 * compress.c — CPU ORACLE for GSNP's output compression (§V-B).
 * TEST INFRASTRUCTURE ONLY (same rules as oracle.c: tests/, smoke() and bench.py only; shares
 * no code with libgsnp).
 *
 * The paper describes the scheme in prose; the byte format below is the reading R17 of
 * DESIGN.md, one section per column family the paper names:
 *   - "sequence name and the number of sites"    -> block header (pos0, n)
 *   - "three columns containing four base types, two bits"     -> planes P (+ N runs)
 *
 *   - "columns related to SNPs ... only store differences"    -> exception lists G K R Q
 *
 *   - "columns related to the second allele are sparse ...    -> bitmap + present values S
 *     only store non-zero elements"
 *   - six quality columns: RLE then DICT of both the run value -> sections C0..C5
 *     and run length arrays; DICT = sorted
 *     unique dictionary + index in least bits
 *
 * Stream = blocks of B consecutive records (the paper compresses per window).
 * All fields are little-endian uint32 words.  Block layout:
 *   w0 magic 0x31435347 ("GSC1"); w1 n (sites in the block); w2,w3 pos0 lo/hi; w4 total words
 *   of the block incl. header; w5 B.
 *   P  for ref, base1, base2: ceil(n/16) words; site i -> bits 2(i%16) of word i/16 = code & 3
 *   N  for ref, base1, base2: m; m run starts; m run ends (exclusive) — maximal runs of code 4
 *   G  genotype != (ref < 4 ? HOM[ref] : 255): m; m site indices; ceil(m/4) words of bytes
 *   K  known != 0: same layout
 *   R  rank_p bits != 0x3F800000 (1.0f): m; m indices; m value words
 *   Q  post1 bits != 0x3F800000: same layout
 *   S  ceil(n/32) bitmap words, bit i%32 of word i/32 = (avgq2|cnt_uni2|cnt_all2) != 0; then
 *      DICT(avgq2), DICT(cnt_uni2), DICT(cnt_all2) over the set sites in order
 *   C0..C5 for quality, avgq1, cnt_uni1, cnt_all1, depth, copy_num (float bits): R (number of
 *      maximal runs of equal values); DICT(run values); DICT(run lengths)
 * DICT(x[0..m)), nothing when m = 0; else D = number of distinct values; if D > 4096 the word
 *   0xFFFFFFFF then m raw words; else D, the D distinct values ascending, then the index of each
 *   x[j] in that list in b = (D == 1 ? 0 : bit length of D-1) bits, element j at bit j*b of the
 *   packed area (LSB first, spilling into the next word), ceil(m*b/32) words.
 * Byte bytes are packed 4 per word, byte j at bits 8(j%4) of word j/4.
 *
 * Parity pins (tests/test_oracle_pins.py): decode(encode(x)) == x on adversarial records; a
 * hand-derived golden block (tests/golden/compress_tiny.txt); size identities.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {             /* identical layout to or_record in oracle.c (40 bytes) */
    uint64_t pos;
    uint8_t ref, genotype, quality, base1, base2, avgq1, avgq2, known;
    uint16_t cnt_uni1, cnt_all1, cnt_uni2, cnt_all2;
    uint32_t depth;
    float rank_p, copy_num, post1;
} oc_record;

#define OC_MAGIC 0x31435347u
#define OC_DICT_MAX 4096u
#define OC_RAW 0xFFFFFFFFu
#define OC_ONE 0x3F800000u

/* homozygous genotype of each base code, genotype order of Alg. 4: AA CC TT GG */
static const uint8_t HOM[4] = {0, 4, 7, 9};

typedef struct { uint32_t* w; uint64_t n, cap; int overflow; } obuf;

static void put(obuf* o, uint32_t v) {
    if (o->n < o->cap) o->w[o->n] = v; else o->overflow = 1;
    o->n++;
}

static uint32_t f2u(float f) { uint32_t u; memcpy(&u, &f, 4); return u; }
static float u2f(uint32_t u) { float f; memcpy(&f, &u, 4); return f; }

static int cmp_u32(const void* a, const void* b) {
    uint32_t x = *(const uint32_t*)a, y = *(const uint32_t*)b;
    return (x > y) - (x < y);
}

static uint32_t bitlen(uint32_t v) { uint32_t b = 0; while (v) { b++; v >>= 1; } return b; }

/* DICT encode: sort + unique, index of each element by binary search, least bits */
static void dict_put(obuf* o, const uint32_t* x, uint64_t m) {
    if (m == 0) return;
    uint32_t* s = malloc(m * sizeof(uint32_t));
    memcpy(s, x, m * sizeof(uint32_t));
    qsort(s, m, sizeof(uint32_t), cmp_u32);
    uint64_t D = 0;
    for (uint64_t j = 0; j < m; ++j)
        if (j == 0 || s[j] != s[j - 1]) s[D++] = s[j];
    if (D > OC_DICT_MAX) {
        put(o, OC_RAW);
        for (uint64_t j = 0; j < m; ++j) put(o, x[j]);
        free(s);
        return;
    }
    put(o, (uint32_t)D);
    for (uint64_t j = 0; j < D; ++j) put(o, s[j]);
    const uint32_t b = D == 1 ? 0 : bitlen((uint32_t)(D - 1));
    const uint64_t words = (m * b + 31) / 32;
    uint32_t* pk = calloc(words + 1, sizeof(uint32_t));
    for (uint64_t j = 0; j < m; ++j) {
        const uint32_t* f = bsearch(&x[j], s, D, sizeof(uint32_t), cmp_u32);
        const uint64_t idx = (uint64_t)(f - s), bit = j * b;
        pk[bit / 32] |= (uint32_t)(idx << (bit % 32));
        if (bit % 32 + b > 32) pk[bit / 32 + 1] |= (uint32_t)(idx >> (32 - bit % 32));
    }
    for (uint64_t j = 0; j < words; ++j) put(o, pk[j]);
    free(pk);
    free(s);
}

static void bytes_put(obuf* o, const uint8_t* v, uint64_t m) {
    for (uint64_t j = 0; j < m; j += 4) {
        uint32_t w = 0;
        for (uint64_t k = 0; k < 4 && j + k < m; ++k) w |= (uint32_t)v[j + k] << (8 * k);
        put(o, w);
    }
}

static uint32_t col6(const oc_record* r, int c) {
    switch (c) {
    case 0: return r->quality;
    case 1: return r->avgq1;
    case 2: return r->cnt_uni1;
    case 3: return r->cnt_all1;
    case 4: return r->depth;
    default: return f2u(r->copy_num);
    }
}

static uint8_t base_col(const oc_record* r, int c) { return c == 0 ? r->ref : c == 1 ? r->base1 : r->base2; }

static void encode_block(obuf* o, const oc_record* rec, uint64_t n, uint32_t B) {
    const uint64_t start = o->n;
    put(o, OC_MAGIC);
    put(o, (uint32_t)n);
    put(o, (uint32_t)rec[0].pos);
    put(o, (uint32_t)(rec[0].pos >> 32));
    put(o, 0);                                         /* total words, patched below */
    put(o, B);
    /* P: 2-bit planes */
    for (int c = 0; c < 3; ++c)
        for (uint64_t w = 0; w < (n + 15) / 16; ++w) {
            uint32_t v = 0;
            for (uint64_t i = w * 16; i < n && i < w * 16 + 16; ++i)
                v |= (uint32_t)(base_col(&rec[i], c) & 3) << (2 * (i % 16));
            put(o, v);
        }
    /* N: runs of code 4 */
    uint32_t* a = malloc((n + 1) * sizeof(uint32_t));
    uint32_t* b = malloc((n + 1) * sizeof(uint32_t));
    for (int c = 0; c < 3; ++c) {
        uint64_t m = 0;
        for (uint64_t i = 0; i < n; ++i) {
            const int f = base_col(&rec[i], c) == 4, pf = i > 0 && base_col(&rec[i - 1], c) == 4;
            if (f && !pf) a[m] = (uint32_t)i;
            if (!f && pf) b[m++] = (uint32_t)i;
        }
        if (n > 0 && base_col(&rec[n - 1], c) == 4) b[m++] = (uint32_t)n;
        put(o, (uint32_t)m);
        for (uint64_t j = 0; j < m; ++j) put(o, a[j]);
        for (uint64_t j = 0; j < m; ++j) put(o, b[j]);
    }
    /* G, K: byte exceptions */
    uint8_t* v8 = malloc(n + 1);
    for (int c = 0; c < 2; ++c) {
        uint64_t m = 0;
        for (uint64_t i = 0; i < n; ++i) {
            const uint8_t val = c == 0 ? rec[i].genotype : rec[i].known;
            const uint8_t pred = c == 0 ? (rec[i].ref < 4 ? HOM[rec[i].ref] : 255) : 0;
            if (val != pred) { a[m] = (uint32_t)i; v8[m++] = val; }
        }
        put(o, (uint32_t)m);
        for (uint64_t j = 0; j < m; ++j) put(o, a[j]);
        bytes_put(o, v8, m);
    }
    /* R, Q: float exceptions vs 1.0f */
    for (int c = 0; c < 2; ++c) {
        uint64_t m = 0;
        for (uint64_t i = 0; i < n; ++i) {
            const uint32_t u = f2u(c == 0 ? rec[i].rank_p : rec[i].post1);
            if (u != OC_ONE) { a[m] = (uint32_t)i; b[m++] = u; }
        }
        put(o, (uint32_t)m);
        for (uint64_t j = 0; j < m; ++j) put(o, a[j]);
        for (uint64_t j = 0; j < m; ++j) put(o, b[j]);
    }
    /* S: second allele, non-zero sites only */
    uint64_t m = 0;
    for (uint64_t w = 0; w < (n + 31) / 32; ++w) {
        uint32_t v = 0;
        for (uint64_t i = w * 32; i < n && i < w * 32 + 32; ++i)
            if (rec[i].avgq2 | rec[i].cnt_uni2 | rec[i].cnt_all2) v |= 1u << (i % 32);
        put(o, v);
    }
    for (uint64_t i = 0; i < n; ++i)
        if (rec[i].avgq2 | rec[i].cnt_uni2 | rec[i].cnt_all2) a[m++] = (uint32_t)i;
    for (int c = 0; c < 3; ++c) {
        for (uint64_t j = 0; j < m; ++j) {
            const oc_record* r = &rec[a[j]];
            b[j] = c == 0 ? r->avgq2 : c == 1 ? r->cnt_uni2 : r->cnt_all2;
        }
        dict_put(o, b, m);
    }
    /* C0..C5: RLE then DICT of values and of lengths */
    for (int c = 0; c < 6; ++c) {
        uint64_t R = 0;
        for (uint64_t i = 0; i < n; ++i) {
            if (i == 0 || col6(&rec[i], c) != col6(&rec[i - 1], c)) { a[R] = col6(&rec[i], c); b[R++] = 1; }
            else b[R - 1]++;
        }
        put(o, (uint32_t)R);
        dict_put(o, a, R);
        dict_put(o, b, R);
    }
    free(v8);
    free(a);
    free(b);
    if (start + 4 < o->cap) o->w[start + 4] = (uint32_t)(o->n - start);
}

/* Compress records [0, n) in blocks of B.  Returns the number of words written (or needed, if
 * larger than cap; nothing past cap is written). */
uint64_t oc_compress(const oc_record* rec, uint64_t n, uint32_t B, uint32_t* out, uint64_t cap) {
    obuf o = {out, 0, cap, 0};
    for (uint64_t s = 0; s < n; s += B) encode_block(&o, rec + s, n - s < B ? n - s : B, B);
    return o.n;
}

/* ------------------------------------------------------------------------------------------ */
typedef struct { const uint32_t* w; uint64_t n, i; int bad; } ibuf;

static uint32_t get(ibuf* in) {
    if (in->i >= in->n) { in->bad = 1; return 0; }
    return in->w[in->i++];
}

static int dict_get(ibuf* in, uint32_t* x, uint64_t m) {
    if (m == 0) return 0;
    const uint32_t D = get(in);
    if (D == OC_RAW) {
        for (uint64_t j = 0; j < m; ++j) x[j] = get(in);
        return in->bad;
    }
    if (D == 0 || D > OC_DICT_MAX) return 1;
    uint32_t* s = malloc(D * sizeof(uint32_t));
    for (uint32_t j = 0; j < D; ++j) s[j] = get(in);
    const uint32_t b = D == 1 ? 0 : bitlen(D - 1);
    const uint64_t words = (m * b + 31) / 32, base = in->i;
    if (base + words > in->n) { free(s); return 1; }
    for (uint64_t j = 0; j < m; ++j) {
        const uint64_t bit = j * b;
        uint64_t v = in->w[base + bit / 32] >> (bit % 32);
        if (bit % 32 + b > 32) v |= (uint64_t)in->w[base + bit / 32 + 1] << (32 - bit % 32);
        const uint32_t idx = b == 0 ? 0 : (uint32_t)(v & ((1ull << b) - 1));
        if (idx >= D) { free(s); return 1; }
        x[j] = s[idx];
    }
    in->i = base + words;
    free(s);
    return 0;
}

/* Decompress a stream of `words` words into rec (capacity cap).  Returns the number of records,
 * or -1 on a malformed stream. */
int64_t oc_decompress(const uint32_t* w, uint64_t words, oc_record* rec, uint64_t cap) {
    ibuf in = {w, words, 0, 0};
    uint64_t total = 0;
    while (in.i < words) {
        const uint64_t start = in.i;
        if (get(&in) != OC_MAGIC) return -1;
        const uint64_t n = get(&in);
        uint64_t pos0 = get(&in);
        pos0 |= (uint64_t)get(&in) << 32;
        const uint64_t W = get(&in);
        get(&in);                                      /* B */
        if (in.bad || n == 0 || total + n > cap || start + W > words) return -1;
        oc_record* r = rec + total;
        memset(r, 0, n * sizeof(oc_record));
        for (uint64_t i = 0; i < n; ++i) r[i].pos = pos0 + i;
        for (int c = 0; c < 3; ++c)
            for (uint64_t wd = 0; wd < (n + 15) / 16; ++wd) {
                const uint32_t v = get(&in);
                for (uint64_t i = wd * 16; i < n && i < wd * 16 + 16; ++i) {
                    const uint8_t code = (v >> (2 * (i % 16))) & 3;
                    if (c == 0) r[i].ref = code; else if (c == 1) r[i].base1 = code; else r[i].base2 = code;
                }
            }
        for (int c = 0; c < 3; ++c) {
            const uint64_t m = get(&in);
            if (in.bad || in.i + 2 * m > words) return -1;
            const uint32_t* st = w + in.i;
            const uint32_t* en = w + in.i + m;
            for (uint64_t j = 0; j < m; ++j) {
                if (st[j] >= en[j] || en[j] > n) return -1;
                for (uint64_t i = st[j]; i < en[j]; ++i) {
                    if (c == 0) r[i].ref = 4; else if (c == 1) r[i].base1 = 4; else r[i].base2 = 4;
                }
            }
            in.i += 2 * m;
        }
        for (uint64_t i = 0; i < n; ++i) r[i].genotype = r[i].ref < 4 ? HOM[r[i].ref] : 255;
        for (int c = 0; c < 2; ++c) {
            const uint64_t m = get(&in);
            if (in.bad || in.i + m + (m + 3) / 4 > words) return -1;
            for (uint64_t j = 0; j < m; ++j) {
                const uint32_t i = w[in.i + j];
                if (i >= n) return -1;
                const uint8_t val = (w[in.i + m + j / 4] >> (8 * (j % 4))) & 255;
                if (c == 0) r[i].genotype = val; else r[i].known = val;
            }
            in.i += m + (m + 3) / 4;
        }
        for (uint64_t i = 0; i < n; ++i) { r[i].rank_p = 1.0f; r[i].post1 = 1.0f; }
        for (int c = 0; c < 2; ++c) {
            const uint64_t m = get(&in);
            if (in.bad || in.i + 2 * m > words) return -1;
            for (uint64_t j = 0; j < m; ++j) {
                const uint32_t i = w[in.i + j];
                if (i >= n) return -1;
                if (c == 0) r[i].rank_p = u2f(w[in.i + m + j]); else r[i].post1 = u2f(w[in.i + m + j]);
            }
            in.i += 2 * m;
        }
        uint32_t* idx = malloc((n + 1) * sizeof(uint32_t));
        uint32_t* val = malloc((n + 1) * sizeof(uint32_t));
        uint32_t* len = malloc((n + 1) * sizeof(uint32_t));
        uint64_t m = 0;
        for (uint64_t wd = 0; wd < (n + 31) / 32; ++wd) {
            const uint32_t v = get(&in);
            for (uint64_t i = wd * 32; i < n && i < wd * 32 + 32; ++i)
                if (v >> (i % 32) & 1) idx[m++] = (uint32_t)i;
        }
        int bad = in.bad;
        for (int c = 0; c < 3 && !bad; ++c) {
            bad |= dict_get(&in, val, m);
            for (uint64_t j = 0; j < m && !bad; ++j) {
                if (c == 0) r[idx[j]].avgq2 = (uint8_t)val[j];
                else if (c == 1) r[idx[j]].cnt_uni2 = (uint16_t)val[j];
                else r[idx[j]].cnt_all2 = (uint16_t)val[j];
            }
        }
        for (int c = 0; c < 6 && !bad; ++c) {
            const uint64_t R = get(&in);
            if (in.bad || R > n) { bad = 1; break; }
            bad |= dict_get(&in, val, R) | dict_get(&in, len, R);
            uint64_t i = 0;
            for (uint64_t j = 0; j < R && !bad; ++j) {
                if (len[j] == 0 || i + len[j] > n) { bad = 1; break; }
                for (uint64_t k = 0; k < len[j]; ++k, ++i) {
                    const uint32_t v = val[j];
                    switch (c) {
                    case 0: r[i].quality = (uint8_t)v; break;
                    case 1: r[i].avgq1 = (uint8_t)v; break;
                    case 2: r[i].cnt_uni1 = (uint16_t)v; break;
                    case 3: r[i].cnt_all1 = (uint16_t)v; break;
                    case 4: r[i].depth = v; break;
                    default: r[i].copy_num = u2f(v);
                    }
                }
            }
            if (!bad && i != n) bad = 1;
        }
        free(idx);
        free(val);
        free(len);
        if (bad || in.bad || in.i != start + W) return -1;
        total += n;
    }
    return (int64_t)total;
}
