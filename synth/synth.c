/*
 * synth.c — seeded synthetic workload generator (reference, diploid sample, aligned reads).
 *
 * This module is shared INPUT infrastructure: the CUDA path (via bench.py / tests) and the CPU
 * oracle both consume what it produces.  It holds none of the GSNP method's arithmetic (no keys,
 * no calibration, no likelihoods); it only draws a reference, plants SNPs and samples reads with
 * sequencing errors, following the workload recipe in DESIGN.md §"Input recipe"
 * (the paper's data: 100 bp reads, ~2% error).
 *
 * Randomness is counter based: every draw is hash(seed, tag, a, b), so the output depends only on
 * the config, never on the thread count.
 */
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
    uint64_t seed;
    uint64_t n_sites;       /* reference length */
    uint64_t origin;        /* global coordinate of ref[0] */
    double depth;           /* mean depth over read-eligible sites */
    uint32_t read_len;      /* all generated reads have this length (<= 256) */
    uint32_t q_hi;          /* highest generated quality (<= 63) */
    double n_frac;          /* total fraction of N sites (leading block + interior blocks) */
    double n_lead_frac;     /* fraction of n_sites in the leading N block */
    uint32_t n_blocks;      /* number of interior N blocks */
    double het_rate;        /* planted heterozygous SNPs per non-N site */
    double hom_rate;        /* planted homozygous-alt SNPs per non-N site */
    double multi_hit_rate;  /* fraction of reads with hits in [2,5] */
    double dup_rate;        /* fraction of fragments sequenced twice (PCR duplicate) */
    double base_n_rate;     /* fraction of read bases called N (quality 2) */
    double known_frac;      /* fraction of planted SNPs put in the known-SNP list (+ as many decoys) */
    uint32_t n_threads;
    uint32_t _pad;
    uint64_t region_lo, region_hi; /* generate only genome sites [lo, hi) + read halo (0,0 = all) */
} syn_config;

/* ---- counter-based hashing ---------------------------------------------------------------- */
static inline uint64_t sm64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}
static inline uint64_t h4(uint64_t seed, uint64_t tag, uint64_t a, uint64_t b) {
    return sm64(sm64(sm64(seed ^ (tag * 0xD1B54A32D192ED03ull)) ^ a) ^ b);
}
static inline double u01(uint64_t h) { return (double)(h >> 11) * (1.0 / 9007199254740992.0); }

enum { T_REF = 1, T_SNP, T_SNPALT, T_SNPHAP, T_NBLK, T_FRAG, T_READ, T_QRUN, T_QVAL, T_ERR,
       T_ERRB, T_NB, T_KNOWN, T_DECOY, T_DECOYALT };

/* ---- reference + planted SNPs ---------------------------------------------------------------
 * ref: 0=A 1=C 2=T 3=G 4=N with human-like composition A/T 29.5%, C/G 20.5%.
 * snp: 0 none, 1 het (alt on hap 0), 2 het (alt on hap 1), 3 hom-alt.  alt: the alt base.
 * Transition:transversion 2:1.  Transition partner of b is 3-b (A<->G, C<->T). */
static void make_reference(const syn_config* c, uint64_t g0, uint64_t g1, uint8_t* ref,
                           uint8_t* snp, uint8_t* alt) {
    uint64_t n = c->n_sites;
    for (uint64_t s = g0; s < g1; ++s) {
        double u = u01(h4(c->seed, T_REF, s, 0));
        ref[s - g0] = u < 0.295 ? 0 : u < 0.5 ? 1 : u < 0.795 ? 2 : 3;
    }
    /* N blocks (placed by global coordinates) */
    uint64_t lead = (uint64_t)(c->n_lead_frac * (double)n);
    for (uint64_t s = g0; s < lead && s < g1; ++s) ref[s - g0] = 4;
    double rest = c->n_frac - c->n_lead_frac;
    if (rest > 0 && c->n_blocks > 0 && n > lead) {
        uint64_t blk = (uint64_t)(rest * (double)n / c->n_blocks);
        uint64_t span = (n - lead) / c->n_blocks;
        for (uint32_t j = 0; j < c->n_blocks; ++j) {
            uint64_t jit = span > blk ? h4(c->seed, T_NBLK, j, 0) % (span - blk) : 0;
            uint64_t st = lead + (uint64_t)j * span + jit;
            uint64_t a = st > g0 ? st : g0, b = st + blk < g1 ? st + blk : g1;
            for (uint64_t s = a; s < b && s < n; ++s) ref[s - g0] = 4;
        }
    }
    for (uint64_t s = g0; s < g1; ++s) {
        uint64_t k = s - g0;
        snp[k] = 0;
        alt[k] = 4;
        if (ref[k] == 4) continue;
        double u = u01(h4(c->seed, T_SNP, s, 0));
        if (u >= c->het_rate + c->hom_rate) continue;
        int b = ref[k];
        double v = u01(h4(c->seed, T_SNPALT, s, 0));
        int a;
        if (v < 2.0 / 3.0) a = 3 - b;                  /* transition */
        else {                                         /* one of the two transversions */
            int tv[2], m = 0;
            for (int x = 0; x < 4; ++x) if (x != b && x != 3 - b) tv[m++] = x;
            a = tv[v < 5.0 / 6.0 ? 0 : 1];
        }
        alt[k] = (uint8_t)a;
        if (u < c->het_rate) snp[k] = (h4(c->seed, T_SNPHAP, s, 0) & 1) ? 2 : 1;
        else snp[k] = 3;
    }
}

/* ---- read placement -------------------------------------------------------------------------
 * A site is read-eligible when [s, s+L) holds no N.  Fragment starts per eligible site are
 * Poisson(depth / (L (1+dup))); each fragment is sequenced twice with probability dup_rate.
 * Everything is keyed by the global site s, so any region of the genome can be generated on its
 * own and agrees with the whole-genome generation (multi-GPU shards).  Arrays cover the window
 * [g0, g1) of the genome: ref/snp/alt/elig[s - g0]. */
typedef struct {
    const syn_config* c;
    const uint8_t* ref;
    const uint8_t* snp;
    const uint8_t* alt;
    const uint8_t* elig;
    uint64_t g0;             /* window origin (genome index of array element 0) */
    double lam_frag;
    uint64_t s0, s1;         /* read starts handled by this job (genome indices) */
    uint64_t n_reads;        /* count pass result */
    uint64_t r0;             /* fill pass: first read index */
    uint64_t* pos; uint16_t* len; uint64_t* off; uint8_t* bases; uint8_t* quals;
    uint8_t* strand; uint16_t* hits;
} job_t;

static inline uint32_t poisson(double lam, double u) {
    double p = exp(-lam), F = p;
    uint32_t k = 0;
    while (u > F && k < 1000) { ++k; p *= lam / k; F += p; }
    return k;
}

static inline uint32_t site_frags(const job_t* j, uint64_t s) {
    if (!j->elig[s - j->g0]) return 0;
    return poisson(j->lam_frag, u01(h4(j->c->seed, T_FRAG, s, 0)));
}
static inline uint32_t frag_copies(const job_t* j, uint64_t s, uint32_t f) {
    return 1u + (u01(h4(j->c->seed, T_FRAG, s, 1 + f)) < j->c->dup_rate ? 1u : 0u);
}

static void* count_job(void* arg) {
    job_t* j = (job_t*)arg;
    uint64_t n = 0;
    for (uint64_t s = j->s0; s < j->s1; ++s) {
        uint32_t nf = site_frags(j, s);
        for (uint32_t f = 0; f < nf; ++f) n += frag_copies(j, s, f);
    }
    j->n_reads = n;
    return NULL;
}

/* quality mixture: 80% U[30,40], 12% U[15,29], 8% U[2,14] (clipped to q_hi) */
static inline uint8_t draw_q(const syn_config* c, uint64_t h) {
    double u = u01(h);
    uint64_t h2 = sm64(h);
    int q;
    if (u < 0.80) q = 30 + (int)(h2 % 11);
    else if (u < 0.92) q = 15 + (int)(h2 % 15);
    else q = 2 + (int)(h2 % 13);
    if (q > (int)c->q_hi) q = (int)c->q_hi;
    return (uint8_t)q;
}

static void* fill_job(void* arg) {
    job_t* j = (job_t*)arg;
    const syn_config* c = j->c;
    const uint32_t L = c->read_len;
    uint64_t r = j->r0;
    uint8_t qcyc[256];
    for (uint64_t s = j->s0; s < j->s1; ++s) {
        uint32_t nf = site_frags(j, s);
        for (uint32_t f = 0; f < nf; ++f) {
            uint32_t nc = frag_copies(j, s, f);
            uint64_t fh = h4(c->seed, T_READ, s, f);
            uint8_t st = (uint8_t)(fh & 1);
            int hap = (int)((fh >> 1) & 1);
            for (uint32_t k = 0; k < nc; ++k, ++r) {
                uint64_t rid = ((uint64_t)f << 8) | k;
                uint64_t rh = h4(c->seed, T_READ, s, 0x100000000ull | rid);
                j->pos[r] = c->origin + s;
                j->len[r] = (uint16_t)L;
                j->off[r] = r * (uint64_t)L;
                j->strand[r] = st;
                j->hits[r] = (uint16_t)(u01(rh) < c->multi_hit_rate ? 2 + (int)(sm64(rh) % 4) : 1);
                /* quality string in sequencing-cycle order, in runs */
                uint32_t cyc = 0, run = 0;
                while (cyc < L) {
                    uint64_t qh = h4(c->seed, T_QRUN, s, (rid << 16) | cyc);
                    uint32_t rl = 1 + (uint32_t)(-log(1.0 - u01(qh)) * 14.0);
                    uint8_t q = draw_q(c, h4(c->seed, T_QVAL, s, (rid << 16) | run));
                    for (uint32_t t = 0; t < rl && cyc < L; ++t) qcyc[cyc++] = q;
                    ++run;
                }
                uint8_t* bb = j->bases + r * (uint64_t)L;
                uint8_t* qq = j->quals + r * (uint64_t)L;
                for (uint32_t i = 0; i < L; ++i) {
                    uint64_t site = s + i - j->g0;
                    uint32_t cy = st ? L - 1 - i : i;
                    uint8_t q = qcyc[cy];
                    int tb = j->ref[site];
                    int sk = j->snp[site];
                    if (sk == 3 || (sk == 1 && hap == 0) || (sk == 2 && hap == 1)) tb = j->alt[site];
                    uint64_t eh = h4(c->seed, T_ERR, s, (rid << 16) | i);
                    if (u01(h4(c->seed, T_NB, s, (rid << 16) | i)) < c->base_n_rate) {
                        bb[i] = 4;
                        qq[i] = 2;
                        continue;
                    }
                    double perr = pow(10.0, -(double)q / 10.0);
                    if (u01(eh) < perr) tb = (tb + 1 + (int)(sm64(eh) % 3)) & 3;
                    bb[i] = (uint8_t)tb;
                    qq[i] = q;
                }
            }
        }
    }
    return NULL;
}

/* ---- public API -------------------------------------------------------------------------- */
/* The generated window: reads starting in [start_lo, start_hi) (all reads that can touch the
 * region [lo, hi)) and the reference [g0, g1) under them. */
typedef struct { uint64_t lo, hi, start_lo, start_hi, g0, g1; } syn_win;

static syn_win window(const syn_config* c) {
    syn_win w;
    uint64_t n = c->n_sites, L = c->read_len;
    w.lo = c->region_hi > c->region_lo ? c->region_lo : 0;
    w.hi = c->region_hi > c->region_lo ? (c->region_hi < n ? c->region_hi : n) : n;
    w.start_lo = w.lo + 1 >= L ? w.lo + 1 - L : 0;
    w.start_hi = w.hi;
    w.g0 = w.start_lo;
    w.g1 = w.hi + L - 1 < n ? w.hi + L - 1 : n;
    if (w.g1 < w.hi) w.g1 = w.hi;
    return w;
}

/* Window bounds: out[0] = g0, out[1] = g1 (reference array length g1 - g0). */
void syn_window(const syn_config* c, uint64_t* out) {
    syn_win w = window(c);
    out[0] = w.g0;
    out[1] = w.g1;
}

static uint64_t run_jobs(const syn_config* c, const uint8_t* ref, const uint8_t* snp,
                         const uint8_t* alt, const uint8_t* elig, int fill, uint64_t* pos,
                         uint16_t* len, uint64_t* off, uint8_t* bases, uint8_t* quals,
                         uint8_t* strand, uint16_t* hits) {
    syn_win w = window(c);
    uint32_t nt = c->n_threads ? c->n_threads : 1;
    if (nt > 256) nt = 256;
    uint64_t n = w.start_hi - w.start_lo;
    uint64_t chunk = (n + nt - 1) / nt;
    job_t jobs[256];
    pthread_t th[256];
    for (uint32_t t = 0; t < nt; ++t) {
        job_t* j = &jobs[t];
        memset(j, 0, sizeof *j);
        j->c = c; j->ref = ref; j->snp = snp; j->alt = alt; j->elig = elig; j->g0 = w.g0;
        j->lam_frag = c->depth / ((double)c->read_len * (1.0 + c->dup_rate));
        j->s0 = w.start_lo + (t * chunk < n ? t * chunk : n);
        j->s1 = w.start_lo + ((t + 1) * chunk < n ? (t + 1) * chunk : n);
    }
    for (uint32_t t = 0; t < nt; ++t) pthread_create(&th[t], NULL, count_job, &jobs[t]);
    for (uint32_t t = 0; t < nt; ++t) pthread_join(th[t], NULL);
    uint64_t total = 0;
    for (uint32_t t = 0; t < nt; ++t) { jobs[t].r0 = total; total += jobs[t].n_reads; }
    if (!fill) return total;
    for (uint32_t t = 0; t < nt; ++t) {
        job_t* j = &jobs[t];
        j->pos = pos; j->len = len; j->off = off; j->bases = bases; j->quals = quals;
        j->strand = strand; j->hits = hits;
    }
    for (uint32_t t = 0; t < nt; ++t) pthread_create(&th[t], NULL, fill_job, &jobs[t]);
    for (uint32_t t = 0; t < nt; ++t) pthread_join(th[t], NULL);
    off[total] = total * (uint64_t)c->read_len;
    return total;
}

/* The N blocks of the whole genome as [begin, end) genome indices (the leading block first, then
 * the interior blocks in order; empty blocks omitted), the same placement make_reference uses.
 * out holds 2 * (n_blocks + 1) entries (NULL: count only); returns the number of intervals.
 * Lets a multi-GPU run plan shards by expected aligned bases without generating the genome. */
uint64_t syn_n_intervals(const syn_config* c, uint64_t* out) {
    uint64_t n = c->n_sites, k = 0;
    uint64_t lead = (uint64_t)(c->n_lead_frac * (double)n);
    if (lead > n) lead = n;
    if (lead) { if (out) { out[0] = 0; out[1] = lead; } ++k; }
    double rest = c->n_frac - c->n_lead_frac;
    if (rest > 0 && c->n_blocks > 0 && n > lead) {
        uint64_t blk = (uint64_t)(rest * (double)n / c->n_blocks);
        uint64_t span = (n - lead) / c->n_blocks;
        for (uint32_t j = 0; j < c->n_blocks; ++j) {
            uint64_t jit = span > blk ? h4(c->seed, T_NBLK, j, 0) % (span - blk) : 0;
            uint64_t st = lead + (uint64_t)j * span + jit, en = st + blk < n ? st + blk : n;
            if (en > st) { if (out) { out[2 * k] = st; out[2 * k + 1] = en; } ++k; }
        }
    }
    return k;
}

/* Phase 1: reference window, SNPs, eligibility (arrays of g1 - g0); returns the read count. */
uint64_t syn_plan(const syn_config* c, uint8_t* ref, uint8_t* snp, uint8_t* alt, uint8_t* elig) {
    if (c->read_len == 0 || c->read_len > 256 || c->n_sites == 0) return (uint64_t)-1;
    syn_win w = window(c);
    make_reference(c, w.g0, w.g1, ref, snp, alt);
    uint64_t L = c->read_len, run = 0, m = w.g1 - w.g0;
    /* elig[s] = 1 iff ref[s..s+L) has no N (and lies in the genome): right-to-left non-N run */
    for (uint64_t k = m; k-- > 0;) {
        run = ref[k] == 4 ? 0 : run + 1;
        elig[k] = run >= L;
    }
    return run_jobs(c, ref, snp, alt, elig, 0, 0, 0, 0, 0, 0, 0, 0);
}

/* Phase 2: fill reads (arrays sized by syn_plan's count; off has n_reads+1 entries). */
uint64_t syn_fill(const syn_config* c, uint8_t* ref, uint8_t* snp, uint8_t* alt, uint8_t* elig,
                  uint64_t* pos, uint16_t* len, uint64_t* off, uint8_t* bases, uint8_t* quals,
                  uint8_t* strand, uint16_t* hits) {
    return run_jobs(c, ref, snp, alt, elig, 1, pos, len, off, bases, quals, strand, hits);
}

/* Known-SNP list over the reference window: known_frac of the planted SNPs plus decoys at the
 * same rate over non-SNP non-N sites.  Priors (linear, > 0) per genotype n (order AA AC AT AG
 * CC CT CG TT TG GG): ref-hom 0.85, ref/alt het 0.1, alt-hom 0.05, any other genotype 1e-4.
 * Pass known_pos == NULL to count. */
uint64_t syn_known(const syn_config* c, const uint8_t* ref, const uint8_t* snp, const uint8_t* alt,
                   uint64_t* known_pos, double* prior10) {
    static const int A1[10] = {0, 0, 0, 0, 1, 1, 1, 2, 2, 3};
    static const int A2[10] = {0, 1, 2, 3, 1, 2, 3, 2, 3, 3};
    syn_win w = window(c);
    double decoy_rate = c->known_frac * (c->het_rate + c->hom_rate);
    uint64_t k = 0;
    for (uint64_t s = w.g0; s < w.g1; ++s) {
        uint64_t i = s - w.g0;
        if (ref[i] == 4) continue;
        int a = -1;
        if (snp[i]) {
            if (u01(h4(c->seed, T_KNOWN, s, 0)) < c->known_frac) a = alt[i];
        } else if (u01(h4(c->seed, T_DECOY, s, 0)) < decoy_rate) {
            a = (ref[i] + 1 + (int)(h4(c->seed, T_DECOYALT, s, 0) % 3)) & 3;
        }
        if (a < 0) continue;
        if (known_pos) {
            int r = ref[i];
            known_pos[k] = c->origin + s;
            for (int n = 0; n < 10; ++n) {
                int x = A1[n], y = A2[n];
                double pr = 1e-4;
                if (x == r && y == r) pr = 0.85;
                else if ((x == r && y == a) || (x == a && y == r)) pr = 0.1;
                else if (x == a && y == a) pr = 0.05;
                prior10[k * 10 + n] = pr;
            }
        }
        ++k;
    }
    return k;
}

/* ------------------------------------------------------------------------------------------
 * SOAP alignment text (input file 1 of P:L206-212 in SOAPsnp's format; reading R19 of
 * DESIGN.md): one line per read, tab-separated
 *   id  seq  qual  n_hits  a  len  strand  chr  location(1-based)  n_mismatch
 * seq in reference-forward orientation (ACGTN), qual = chr(q + q_offset).  Writes the lines of
 * reads [0, n) to out (NULL: size query); returns the number of bytes.
 */
static uint32_t put_u64(char* o, uint64_t v) {
    char t[24];
    uint32_t k = 0;
    do { t[k++] = (char)('0' + v % 10); v /= 10; } while (v);
    for (uint32_t i = 0; i < k; ++i) o[i] = t[k - 1 - i];
    return k;
}

uint64_t syn_soap_text(uint64_t n, const uint64_t* pos, const uint16_t* len, const uint64_t* off,
                       const uint8_t* bases, const uint8_t* quals, const uint8_t* strand,
                       const uint16_t* hits, const char* chr, uint32_t q_offset,
                       uint64_t loc_base, char* out) {
    static const char B[5] = {'A', 'C', 'T', 'G', 'N'};
    char buf[1024];
    uint64_t tot = 0;
    size_t cl = strlen(chr);
    for (uint64_t r = 0; r < n; ++r) {
        char* o = buf;
        *o++ = 'r';
        o += put_u64(o, r);
        *o++ = '\t';
        for (uint32_t i = 0; i < len[r]; ++i) *o++ = B[bases[off[r] + i] > 4 ? 4 : bases[off[r] + i]];
        *o++ = '\t';
        for (uint32_t i = 0; i < len[r]; ++i) *o++ = (char)(quals[off[r] + i] + q_offset);
        *o++ = '\t';
        o += put_u64(o, hits[r]);
        *o++ = '\t'; *o++ = (r & 1) ? 'b' : 'a'; *o++ = '\t';
        o += put_u64(o, len[r]);
        *o++ = '\t'; *o++ = strand[r] ? '-' : '+'; *o++ = '\t';
        memcpy(o, chr, cl); o += cl;
        *o++ = '\t';
        o += put_u64(o, pos[r] - loc_base + 1);
        *o++ = '\t'; *o++ = '0'; *o++ = '\n';
        uint64_t k = (uint64_t)(o - buf);
        if (out) memcpy(out + tot, buf, k);
        tot += k;
    }
    return tot;
}
