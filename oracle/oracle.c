/*
 * oracle.c — CPU ORACLE for the GSNP hot path.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline / --impl reference) may load
 * this file's library.  The product path (libgsnp, paper_conf_icpp_luzlwfl11_b200) never does.
 * It shares no code, header, table or constant generator with the CUDA library.
 *
 * Plain, slow, single-threaded C.  fp64 throughout, glibc log10/pow/erfc, built with
 * -O2 -ffp-contract=off.  Each function cites the passage of PAPER.md ("P:L<n>") it follows,
 * or the DESIGN.md reading (R<n>) where the paper is silent.
 *
 * Pins (tests/test_oracle_pins.py): Fig. 3 keys; dense Alg. 1 == sparse Alg. 4; brute-force
 * products vs log-sums; closed forms; scipy's Mann-Whitney asymptotic and exact p (R20);
 * calibration invariants.
 * Functions without an external pin say "parity unpinned" in their comment.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
    uint32_t max_read_len;   /* L: reads are 1..L long; coord field 8 bits */
    uint32_t q_max;          /* qualities 0..q_max <= 63 (P:L389, 6-bit score) */
    double het_novel;        /* R6 prior of a novel ref/alt heterozygote */
    double althom_novel;     /* R6 prior of a novel alt homozygote */
    double global_dep;       /* R3 global dependency coefficient (linear) */
    double pcr_dep;          /* R3 PCR dependency coefficient (linear) */
    uint32_t calib_min_count;/* R1 tau */
    uint32_t rank_sum;       /* R8: 1 = apply the rank-sum test to het calls; 2 = R20 exact */
    uint32_t prior_mode;     /* R18: bit 0 monoploid, bit 1 ti/tv 2:1 */
} or_params;

typedef struct {
    uint64_t n_reads;
    const uint64_t* pos;     /* leftmost reference coordinate, non-decreasing */
    const uint16_t* len;
    const uint64_t* off;     /* n_reads+1 offsets into bases/quals */
    const uint8_t* bases;    /* 0=A 1=C 2=T 3=G 4=N, reference-forward orientation (R11) */
    const uint8_t* quals;
    const uint8_t* strand;   /* 0 '+', 1 '-' */
    const uint16_t* hits;    /* 1 = uniquely aligned */
} or_reads;

typedef struct {             /* one output row: the record of DESIGN.md */
    uint64_t pos;
    uint8_t ref, genotype, quality, base1, base2, avgq1, avgq2, known;
    uint16_t cnt_uni1, cnt_all1, cnt_uni2, cnt_all2;
    uint32_t depth;
    float rank_p, copy_num, post1;
} or_record;

/* genotype n -> (allele1, allele2), Alg. 4 lines 13-17 order */
static const int GA1[10] = {0, 0, 0, 0, 1, 1, 1, 2, 2, 3};
static const int GA2[10] = {0, 1, 2, 3, 1, 2, 3, 2, 3, 3};

int or_sizeof_record(void) { return (int)sizeof(or_record); }

/* ------------------------------------------------------------------------------------------
 * C2 — base_word key (Fig. 3) with the score field inverted (reading R2/G1)
 * so that an ascending sort visits base 0..3, score high..low, coord 0..L, strand 0..1 — the
 * loop nest of Alg. 1 lines 2-6.
 */
uint32_t or_key(int base, int q, int coord, int strand) {
    return (uint32_t)base << 15 | (uint32_t)(63 - q) << 9 | (uint32_t)coord << 1 | (uint32_t)strand;
}
/* The paper's own (uninverted) layout, used only by the Fig. 3 pin: base<<15|score<<9|coord<<1|strand */
uint32_t or_key_paper(int base, int score, int coord, int strand) {
    return (uint32_t)base << 15 | (uint32_t)score << 9 | (uint32_t)coord << 1 | (uint32_t)strand;
}

/* ------------------------------------------------------------------------------------------
 * C3 — adjust(score, dep_count) (Alg. 1 l.10 P:L365, Alg. 4 l.12 P:L650; body PAPER SILENT,
 * reading R3):  q_adj = max(1, (int)(10^(log10 q + (pcr-1)*log10(pcr_dep) + g*log10(global_dep)) + 0.5))
 */
int or_adjust(const or_params* P, int q, int pcr, int g) {
    double lq = log10((double)q);
    double e = lq + (double)(pcr - 1) * log10(P->pcr_dep) + (double)g * log10(P->global_dep);
    int qa = (int)(pow(10.0, e) + 0.5);
    return qa < 1 ? 1 : qa;
}

/* ------------------------------------------------------------------------------------------
 * C1 — calibration counts (cal_p_matrix; which bases count: reading R1):
 * C[q][cyc][t][o] += 1 for every non-N base of a uniquely aligned read at a reference site that
 * is neither N nor a known SNP.  t = reference base, o = observed base, cyc = sequencing cycle.
 * C is uint64[64][256][4][4], index q<<12 | cyc<<4 | t<<2 | o.
 */
static int is_known(uint64_t n_known, const uint64_t* known_pos, uint64_t site, uint64_t* idx) {
    uint64_t lo = 0, hi = n_known;
    while (lo < hi) {
        uint64_t mid = lo + (hi - lo) / 2;
        if (known_pos[mid] < site) lo = mid + 1; else hi = mid;
    }
    if (lo < n_known && known_pos[lo] == site) { if (idx) *idx = lo; return 1; }
    return 0;
}

int or_calib_counts(const or_params* P, const uint8_t* ref, uint64_t n_sites, uint64_t origin,
                    uint64_t n_known, const uint64_t* known_pos, const or_reads* R, uint64_t* C) {
    memset(C, 0, sizeof(uint64_t) * 64 * 256 * 16);
    for (uint64_t r = 0; r < R->n_reads; ++r) {
        if (R->hits[r] != 1) continue;
        int L = R->len[r];
        for (int i = 0; i < L; ++i) {
            uint64_t site = R->pos[r] + (uint64_t)i;
            if (site < origin || site >= origin + n_sites) return -2;
            int t = ref[site - origin];
            int o = R->bases[R->off[r] + i];
            int q = R->quals[R->off[r] + i];
            if (t == 4 || o == 4) continue;
            if (is_known(n_known, known_pos, site, 0)) continue;
            int cyc = R->strand[r] ? L - 1 - i : i;
            C[(uint64_t)q << 12 | (uint64_t)cyc << 4 | (uint64_t)t << 2 | (uint64_t)o] += 1;
        }
    }
    (void)P;
    return 0;
}

/* ------------------------------------------------------------------------------------------
 * C1 — p_matrix estimate (PAPER SILENT on the estimator, reading R1).  p is double
 * [64][256][4][4], index q<<12 | coord<<4 | allele<<2 | base (Alg. 2), meaning
 * P(observed base | true allele, quality, coord).  For each cell the first rule that applies:
 *   1. n      > tau : p = n / N_ct                  (this cycle's row)
 *   2. n_pool > tau : p = n_pool / N_pool           (pooled over cycles)
 *   3. 0 < mm < tot : p = o==t ? (tot-mm)/tot : mm/(3 tot)   (quality-wide mismatch rate)
 *   4. otherwise     : e = min(0.75, 10^(-q/10)), p = o==t ? 1-e : e/3   (theoretical)
 */
int or_p_matrix(const or_params* P, const uint64_t* C, double* p) {
    int L = (int)P->max_read_len;
    double tau = (double)P->calib_min_count;
    for (int i = 0; i < 64 * 256 * 16; ++i) p[i] = 0.0;
    for (int q = 0; q < 64; ++q) {
        double tot = 0, mm = 0;
        for (int c = 0; c < L; ++c)
            for (int t = 0; t < 4; ++t)
                for (int o = 0; o < 4; ++o) {
                    double v = (double)C[q << 12 | c << 4 | t << 2 | o];
                    tot += v;
                    if (t != o) mm += v;
                }
        for (int t = 0; t < 4; ++t) {
            double n_pool[4] = {0, 0, 0, 0}, N_pool = 0;
            for (int c = 0; c < L; ++c)
                for (int o = 0; o < 4; ++o) {
                    double v = (double)C[q << 12 | c << 4 | t << 2 | o];
                    n_pool[o] += v;
                    N_pool += v;
                }
            for (int c = 0; c < L; ++c) {
                double N_ct = 0;
                for (int o = 0; o < 4; ++o) N_ct += (double)C[q << 12 | c << 4 | t << 2 | o];
                for (int o = 0; o < 4; ++o) {
                    double n = (double)C[q << 12 | c << 4 | t << 2 | o];
                    double v;
                    if (n > tau) v = n / N_ct;
                    else if (n_pool[o] > tau) v = n_pool[o] / N_pool;
                    else if (mm > 0 && mm < tot) v = (o == t) ? (tot - mm) / tot : mm / (3.0 * tot);
                    else {
                        double e = pow(10.0, -(double)q / 10.0);
                        if (e > 0.75) e = 0.75;
                        v = (o == t) ? 1.0 - e : e / 3.0;
                    }
                    p[q << 12 | c << 4 | t << 2 | o] = v;
                }
            }
        }
    }
    return 0;
}

/* ------------------------------------------------------------------------------------------
 * Alg. 2 likely_update: log10(0.5 p_matrix[p1] + 0.5 p_matrix[p2]),
 * p1 = q<<12 | coord<<4 | allele1<<2 | base, p2 = ... allele2 ...
 */
static double likely_update(const double* p, int q_adj, int coord, int base, int a1, int a2) {
    int p1 = q_adj << 12 | coord << 4 | a1 << 2 | base;
    int p2 = q_adj << 12 | coord << 4 | a2 << 2 | base;
    return log10(0.5 * p[p1] + 0.5 * p[p2]);
}

/* ------------------------------------------------------------------------------------------
 * C2+C3+C4 — sparse likelihood of one site, Alg. 4 over keys already sorted
 * ascending (likelihood_sort, Alg. 4 l.1).  dep_count[strand*L + coord] reset when the base
 * changes (l.8-11); pcr = dep_count after the increment; g = (#non-zero dep_count entries) - 1
 * (reading R3, SOAPsnp's global dependency count).  type_likely[10] in Alg. 4 n order.
 */
static int cmp_u32(const void* a, const void* b) {
    uint32_t x = *(const uint32_t*)a, y = *(const uint32_t*)b;
    return x < y ? -1 : x > y;
}

static void likelihood_comp(const or_params* P, const double* p, const uint32_t* keys, uint64_t n,
                            double* L10) {
    int L = (int)P->max_read_len;
    int dep_count[512];
    int distinct = 0;
    memset(dep_count, 0, sizeof dep_count);
    for (int k = 0; k < 10; ++k) L10[k] = 0.0;
    int last_base = 0;
    for (uint64_t i = 0; i < n; ++i) {
        int base = (int)(keys[i] >> 15 & 3);
        int score = 63 - (int)(keys[i] >> 9 & 63);
        int coord = (int)(keys[i] >> 1 & 255);
        int strand = (int)(keys[i] & 1);
        if (base > last_base) {
            memset(dep_count, 0, sizeof dep_count);
            distinct = 0;
            last_base = base;
        }
        if (dep_count[strand * L + coord] == 0) distinct += 1;
        dep_count[strand * L + coord] += 1;
        int q_adj = or_adjust(P, score, dep_count[strand * L + coord], distinct - 1);
        int n = 0;
        for (int a1 = 0; a1 <= 3; ++a1)
            for (int a2 = a1; a2 <= 3; ++a2) {
                L10[n] += likely_update(p, q_adj, coord, base, a1, a2);
                n += 1;
            }
    }
}

/* Sparse route for a list of aligned bases in input order: build keys (C2), sort (Alg. 4 l.1),
 * likelihood_comp (Alg. 4 l.2).  Used by the pins and by or_call_window. */
int or_sparse_likelihood(const or_params* P, const double* p, uint64_t n, const uint8_t* base,
                         const uint8_t* q, const uint8_t* coord, const uint8_t* strand,
                         double* L10, uint32_t* keys_sorted) {
    uint32_t* keys = (uint32_t*)malloc(sizeof(uint32_t) * (n ? n : 1));
    for (uint64_t i = 0; i < n; ++i) keys[i] = or_key(base[i], q[i], coord[i], strand[i]);
    qsort(keys, n, sizeof(uint32_t), cmp_u32);
    likelihood_comp(P, p, keys, n, L10);
    if (keys_sorted) memcpy(keys_sorted, keys, sizeof(uint32_t) * n);
    free(keys);
    return 0;
}

/* C5 — dense route, Alg. 1 literally: materialise base_occ[4][64][256][2]
 * (occurrence counts, here 16-bit so that no count saturates, reading G13) and walk
 * base 0..3, score q_max..0 (q_min = 0), coord 0..L-1, strand 0..1. */
int or_dense_likelihood(const or_params* P, const double* p, uint64_t n, const uint8_t* base,
                        const uint8_t* q, const uint8_t* coord, const uint8_t* strand, double* L10) {
    int L = (int)P->max_read_len;
    uint16_t* base_occ = (uint16_t*)calloc(4 * 64 * 256 * 2, sizeof(uint16_t));
    for (uint64_t i = 0; i < n; ++i)
        base_occ[base[i] << 15 | q[i] << 9 | coord[i] << 1 | strand[i]] += 1;
    double type_likely[16];                       /* index allele1<<2 | allele2 (Alg. 1 l.13) */
    for (int k = 0; k < 16; ++k) type_likely[k] = 0.0;
    int dep_count[512];
    for (int b = 0; b <= 3; ++b) {
        memset(dep_count, 0, sizeof dep_count);
        int global_dep_count = -1;
        for (int score = (int)P->q_max; score >= 0; --score)
            for (int c = 0; c < L; ++c)
                for (int s = 0; s <= 1; ++s) {
                    int occ = base_occ[b << 15 | score << 9 | c << 1 | s];
                    for (int k = 0; k < occ; ++k) {
                        if (dep_count[s * L + c] == 0) global_dep_count += 1;
                        dep_count[s * L + c] += 1;
                        int q_adj = or_adjust(P, score, dep_count[s * L + c], global_dep_count);
                        for (int a1 = 0; a1 <= 3; ++a1)
                            for (int a2 = a1; a2 <= 3; ++a2)
                                type_likely[a1 << 2 | a2] += likely_update(p, q_adj, c, b, a1, a2);
                    }
                }
    }
    for (int k = 0; k < 10; ++k) L10[k] = type_likely[GA1[k] << 2 | GA2[k]];
    free(base_occ);
    return 0;
}

/* ------------------------------------------------------------------------------------------
 * C6 — priors ("prior probability for known SNPs"; the novel prior is PAPER SILENT,
 * reading R6).  Returns log10 prior of genotype n at a site with reference base ref.
 */
/* R18 prior variants (P:L216 names only "prior probability for known
 * SNPs", so every variant is a reading):
 *  - ti/tv (prior_mode bit 1): the transition:transversion ratio of novel alleles is 2:1.  Of the
 *    three alternative alleles of ref, one is the transition (A<->G, C<->T: code XOR 3) and two are
 *    transversions; per-allele weights with mean 1 and ratio 2:1 overall are w_ti = 2,
 *    w_tv = 1/2.  ref/x het: het_novel w(x); x/x: althom_novel w(x); x/y: het_novel althom_novel
 *    w(x) w(y).  No effect at ref N.
 *  - monoploid (bit 0): heterozygous genotypes have prior 0 (log10 = -inf) at every site,
 *    known SNP rows included. */
static double titv_w(const or_params* P, int ref, int x) {
    if (!(P->prior_mode & 2u)) return 1.0;
    return (ref ^ x) == 3 ? 2.0 : 0.5;
}

static double log10_prior(const or_params* P, int ref, int n, const double* known_row) {
    int a1 = GA1[n], a2 = GA2[n];
    if ((P->prior_mode & 1u) && a1 != a2) return log10(0.0);   /* -inf */
    if (known_row) return log10(known_row[n]);
    if (ref == 4) return 0.0;
    double pr;
    if (a1 == ref && a2 == ref) pr = 1.0;
    else if (a1 == ref) pr = P->het_novel * titv_w(P, ref, a2);
    else if (a2 == ref) pr = P->het_novel * titv_w(P, ref, a1);
    else if (a1 == a2) pr = P->althom_novel * titv_w(P, ref, a1);
    else pr = P->het_novel * P->althom_novel * titv_w(P, ref, a1) * titv_w(P, ref, a2);
    return log10(pr);
}

/* R18 known-SNP priors from allele frequencies (the known-SNP file of P:L216 as SOAPsnp's:
 * per-site frequencies of A, C, T, G): Hardy-Weinberg genotype frequencies, f_a^2 for a/a and
 * 2 f_a f_b for a/b (frequencies normalised to sum 1), each floored at floor_prior > 0 so every
 * prior stays positive.  freq: n x 4; prior10: n x 10.  Returns -1 if a row sums to <= 0. */
int or_priors_from_freq(const double* freq, uint64_t n, double floor_prior, double* prior10) {
    for (uint64_t i = 0; i < n; ++i) {
        const double* f = freq + 4 * i;
        double tot = f[0] + f[1] + f[2] + f[3];
        if (!(tot > 0) || f[0] < 0 || f[1] < 0 || f[2] < 0 || f[3] < 0) return -1;
        for (int k = 0; k < 10; ++k) {
            double fa = f[GA1[k]] / tot, fb = f[GA2[k]] / tot;
            double v = GA1[k] == GA2[k] ? fa * fa : 2.0 * fa * fb;
            prior10[10 * i + k] = v > floor_prior ? v : floor_prior;
        }
    }
    return 0;
}

/* C8 — Wilcoxon rank-sum, normal approximation with tie correction (PAPER SILENT, reading R8).
 * X, Y = raw qualities; returns the two-sided p-value erfc(|z|/sqrt(2)). */
double or_rank_sum(uint64_t n1, const uint8_t* X, uint64_t n2, const uint8_t* Y) {
    if (n1 == 0 || n2 == 0) return 0.0;
    uint64_t N = n1 + n2;
    double W = 0.0, tie = 0.0;
    /* pooled mid-ranks: rank(v) = #{pooled < v} + (#{pooled == v} + 1) / 2 */
    for (uint64_t i = 0; i < n1; ++i) {
        uint64_t less = 0, eq = 0;
        for (uint64_t j = 0; j < n1; ++j) { less += X[j] < X[i]; eq += X[j] == X[i]; }
        for (uint64_t j = 0; j < n2; ++j) { less += Y[j] < X[i]; eq += Y[j] == X[i]; }
        W += (double)less + ((double)eq + 1.0) / 2.0;
    }
    /* tie groups: sum over distinct values of t^3 - t */
    for (int v = 0; v < 256; ++v) {
        double t = 0;
        for (uint64_t j = 0; j < n1; ++j) t += X[j] == v;
        for (uint64_t j = 0; j < n2; ++j) t += Y[j] == v;
        tie += t * t * t - t;
    }
    double n1d = (double)n1, n2d = (double)n2, Nd = (double)N;
    double mu = n1d * (Nd + 1.0) / 2.0;
    double var = n1d * n2d / 12.0 * ((Nd + 1.0) - tie / (Nd * (Nd - 1.0)));
    if (!(var > 0.0)) return 1.0;
    double z = (W - mu) / sqrt(var);
    return erfc(fabs(z) / sqrt(2.0));
}

/* C8 exact variant (PAPER SILENT, reading R20; SURVEY §8(f) NEXT #4 "exact small-N rank-sum").
 * When n1, n2 <= 32 and no two pooled qualities tie, W = sum of the integer ranks of X and the
 * p-value is the definition of the exact two-sided test: under H0 every n1-subset of the ranks
 * {1..N} is equally likely, so P(W <= w) = #{subsets with rank sum <= w} / C(N, n1).  The subset
 * counts come from the plain 0/1-knapsack over ranks 1..N (cnt[k][s]: k ranks summing to s).
 * p = min(1, 2 min(P(W <= w), P(W >= w))).  Otherwise the normal approximation (or_rank_sum). */
double or_rank_sum_exact(uint64_t n1, const uint8_t* X, uint64_t n2, const uint8_t* Y) {
    if (n1 == 0 || n2 == 0) return 0.0;
    if (n1 > 32 || n2 > 32) return or_rank_sum(n1, X, n2, Y);
    uint64_t N = n1 + n2;
    for (uint64_t i = 0; i < N; ++i)
        for (uint64_t j = i + 1; j < N; ++j) {
            uint8_t a = i < n1 ? X[i] : Y[i - n1], b = j < n1 ? X[j] : Y[j - n1];
            if (a == b) return or_rank_sum(n1, X, n2, Y);
        }
    uint64_t W = 0;
    for (uint64_t i = 0; i < n1; ++i) {
        uint64_t less = 0;
        for (uint64_t j = 0; j < n1; ++j) less += X[j] < X[i];
        for (uint64_t j = 0; j < n2; ++j) less += Y[j] < X[i];
        W += less + 1;
    }
    uint64_t smax = N * (N + 1) / 2;
    double* cnt = (double*)calloc((n1 + 1) * (smax + 1), sizeof(double));
    cnt[0] = 1.0;
    for (uint64_t r = 1; r <= N; ++r)                   /* add rank r to every subset */
        for (uint64_t k = (r < n1 ? r : n1); k >= 1; --k)
            for (uint64_t s = smax; s >= r; --s)
                cnt[k * (smax + 1) + s] += cnt[(k - 1) * (smax + 1) + s - r];
    double tot = 0.0, le = 0.0, ge = 0.0;
    for (uint64_t s = 0; s <= smax; ++s) {
        double c = cnt[n1 * (smax + 1) + s];
        tot += c;
        if (s <= W) le += c;
        if (s >= W) ge += c;
    }
    free(cnt);
    double p = 2.0 * (le < ge ? le : ge) / tot;
    return p < 1.0 ? p : 1.0;
}

/* ------------------------------------------------------------------------------------------
 * One window [w0, w1): C0 gathering, then per site C2..C9.  Optional debug outputs (may be NULL):
 *   off[S+1] (u32 CSR offsets of keys), keys_sorted, counters[S][15] =
 *   {depth, dep_uni, repeat, count_all[4], count_uni[4], q_sum[4]}, L10[S][10], post10[S][10].
 * Returns 0, or -2 if a read leaves the reference.
 */
typedef struct { uint8_t b, q, cyc, strand; } tuple_t;

int or_call_window(const or_params* P, const uint8_t* ref, uint64_t n_sites, uint64_t origin,
                   uint64_t n_known, const uint64_t* known_pos, const double* known_prior10,
                   const double* p, const or_reads* R, uint64_t w0, uint64_t w1, or_record* rec,
                   uint32_t* off_out, uint32_t* keys_out, uint32_t* counters, double* L10_out,
                   double* post10_out) {
    if (w1 < w0 || w0 < origin || w1 > origin + n_sites) return -2;
    uint64_t S = w1 - w0;
    uint32_t* depth = (uint32_t*)calloc(S + 1, 4);
    uint32_t* repeat = (uint32_t*)calloc(S + 1, 4);
    uint32_t* count_all = (uint32_t*)calloc(4 * (S + 1), 4);
    uint64_t* n_uni = (uint64_t*)calloc(S + 1, 8);
    /* C0 pass 1: per-site counts (reading R10) */
    for (uint64_t r = 0; r < R->n_reads; ++r) {
        for (int i = 0; i < R->len[r]; ++i) {
            uint64_t site = R->pos[r] + (uint64_t)i;
            if (site < w0 || site >= w1) continue;
            int b = R->bases[R->off[r] + i];
            if (b == 4) continue;
            uint64_t s = site - w0;
            depth[s] += 1;
            count_all[s * 4 + b] += 1;
            repeat[s] += R->hits[r];
            if (R->hits[r] == 1) n_uni[s] += 1;
        }
    }
    uint64_t* start = (uint64_t*)calloc(S + 1, 8);
    for (uint64_t s = 0; s < S; ++s) start[s + 1] = start[s] + n_uni[s];
    tuple_t* tup = (tuple_t*)malloc(sizeof(tuple_t) * (start[S] ? start[S] : 1));
    uint64_t* fill = (uint64_t*)calloc(S + 1, 8);
    /* C0 pass 2: the (b, q, cyc, strand) tuple of every uniquely aligned non-N base */
    for (uint64_t r = 0; r < R->n_reads; ++r) {
        if (R->hits[r] != 1) continue;
        for (int i = 0; i < R->len[r]; ++i) {
            uint64_t site = R->pos[r] + (uint64_t)i;
            if (site < w0 || site >= w1) continue;
            int b = R->bases[R->off[r] + i];
            if (b == 4) continue;
            uint64_t s = site - w0;
            tuple_t t;
            t.b = (uint8_t)b;
            t.q = R->quals[R->off[r] + i];
            t.cyc = (uint8_t)(R->strand[r] ? R->len[r] - 1 - i : i);
            t.strand = R->strand[r];
            tup[start[s] + fill[s]++] = t;
        }
    }
    uint8_t* bb = (uint8_t*)malloc(4096), *qq = NULL, *cc = NULL, *ss = NULL;
    uint64_t cap = 0;
    uint32_t* keys = NULL;
    for (uint64_t s = 0; s < S; ++s) {
        uint64_t site = w0 + s, n = n_uni[s];
        int refb = ref[site - origin];
        if (n > cap) {
            cap = n * 2;
            free(bb); free(qq); free(cc); free(ss); free(keys);
            bb = (uint8_t*)malloc(cap); qq = (uint8_t*)malloc(cap); cc = (uint8_t*)malloc(cap);
            ss = (uint8_t*)malloc(cap); keys = (uint32_t*)malloc(cap * 4);
        }
        uint32_t count_uni[4] = {0, 0, 0, 0}, q_sum[4] = {0, 0, 0, 0};
        for (uint64_t k = 0; k < n; ++k) {
            tuple_t t = tup[start[s] + k];
            bb[k] = t.b; qq[k] = t.q; cc[k] = t.cyc; ss[k] = t.strand;
            count_uni[t.b] += 1;
            q_sum[t.b] += t.q;
        }
        /* C2-C4 */
        double L10[10];
        or_sparse_likelihood(P, p, n, bb, qq, cc, ss, L10, keys);
        /* C6-C7 */
        uint64_t kidx = 0;
        int known = is_known(n_known, known_pos, site, &kidx);
        const double* krow = known ? known_prior10 + kidx * 10 : NULL;
        double lp[10], m = -INFINITY;
        for (int k = 0; k < 10; ++k) {
            lp[k] = L10[k] + log10_prior(P, refb, k, krow);
            if (lp[k] > m) m = lp[k];
        }
        double post[10], sum = 0.0;
        for (int k = 0; k < 10; ++k) { post[k] = pow(10.0, lp[k] - m); sum += post[k]; }
        for (int k = 0; k < 10; ++k) post[k] = post[k] / sum;
        int t1 = 0;
        for (int k = 1; k < 10; ++k) if (lp[k] > lp[t1]) t1 = k;
        int t2 = t1 == 0 ? 1 : 0;
        for (int k = 0; k < 10; ++k) if (k != t1 && lp[k] > lp[t2]) t2 = k;
        int a1 = GA1[t1], a2 = GA2[t1];
        uint32_t dep_uni = (uint32_t)n;
        /* C8 */
        double rank_p = 1.0;
        if (a1 != a2 && P->rank_sum) {
            uint8_t* X = (uint8_t*)malloc(n + 1);
            uint8_t* Y = (uint8_t*)malloc(n + 1);
            uint64_t nx = 0, ny = 0;
            for (uint64_t k = 0; k < n; ++k) {
                if (bb[k] == a1) X[nx++] = qq[k];
                else if (bb[k] == a2) Y[ny++] = qq[k];
            }
            rank_p = P->rank_sum == 2 ? or_rank_sum_exact(nx, X, ny, Y)
                                      : or_rank_sum(nx, X, ny, Y);
            free(X); free(Y);
        }
        /* C9 — best and second base: rank by q_sum (unique bases) or, with no unique base, by
         * count_all; descending, ties to the lower code. */
        const uint32_t* score = dep_uni > 0 ? q_sum : count_all + s * 4;
        const uint32_t* present = dep_uni > 0 ? count_uni : count_all + s * 4;
        int order[4], no = 0;
        for (int b = 0; b < 4; ++b) if (present[b] > 0) order[no++] = b;
        for (int i = 1; i < no; ++i)          /* insertion sort, stable: ties keep lower code */
            for (int j = i; j > 0 && score[order[j]] > score[order[j - 1]]; --j) {
                int tmp = order[j]; order[j] = order[j - 1]; order[j - 1] = tmp;
            }
        int base1, base2;
        if (no == 0) { base1 = refb; base2 = 4; }
        else {
            base1 = order[0];
            base2 = no >= 2 ? order[1] : (order[0] != refb ? refb : 4);
        }
        /* C9 — consensus quality */
        int qs = rank_p == 0.0 ? 0 : (int)(10.0 * (lp[t1] - lp[t2]) + 10.0 * log10(rank_p));
        if (a1 == a2) {
            if (dep_uni > 0 && base1 != a1) qs = 0;
            else {
                int cap1 = (base1 < 4 ? (int)q_sum[base1] : 0) - (base2 < 4 ? (int)q_sum[base2] : 0);
                if (cap1 < qs) qs = cap1;
            }
        } else {
            if (count_all[s * 4 + a1] > 0 && count_all[s * 4 + a2] > 0) {
                int cap2 = (int)(q_sum[a1] < q_sum[a2] ? q_sum[a1] : q_sum[a2]);
                if (cap2 < qs) qs = cap2;
            } else qs = 0;
        }
        if (dep_uni == 0) qs = 0;
        if (qs < 0) qs = 0;
        if (qs > 99) qs = 99;
        or_record* o = &rec[s];
        memset(o, 0, sizeof *o);
        o->pos = site;
        o->ref = (uint8_t)refb;
        o->genotype = (refb == 4 && depth[s] == 0) ? 255 : (uint8_t)t1;
        o->quality = o->genotype == 255 ? 0 : (uint8_t)qs;
        o->base1 = (uint8_t)base1;
        o->base2 = (uint8_t)base2;
        o->avgq1 = (uint8_t)(base1 < 4 && count_uni[base1] ? q_sum[base1] / count_uni[base1] : 0);
        o->avgq2 = (uint8_t)(base2 < 4 && count_uni[base2] ? q_sum[base2] / count_uni[base2] : 0);
        o->known = (uint8_t)known;
#define SAT16(x) ((uint16_t)((x) > 65535u ? 65535u : (x)))
        o->cnt_uni1 = base1 < 4 ? SAT16(count_uni[base1]) : 0;
        o->cnt_all1 = base1 < 4 ? SAT16(count_all[s * 4 + base1]) : 0;
        o->cnt_uni2 = base2 < 4 ? SAT16(count_uni[base2]) : 0;
        o->cnt_all2 = base2 < 4 ? SAT16(count_all[s * 4 + base2]) : 0;
        o->depth = depth[s];
        o->rank_p = (float)rank_p;
        o->copy_num = depth[s] ? (float)((double)repeat[s] / (double)depth[s]) : 0.0f;
        o->post1 = (float)post[t1];
        if (off_out) off_out[s] = (uint32_t)start[s];
        if (keys_out) memcpy(keys_out + start[s], keys, sizeof(uint32_t) * n);
        if (counters) {
            uint32_t* c = counters + s * 15;
            c[0] = depth[s]; c[1] = dep_uni; c[2] = repeat[s];
            for (int b = 0; b < 4; ++b) {
                c[3 + b] = count_all[s * 4 + b];
                c[7 + b] = count_uni[b];
                c[11 + b] = q_sum[b];
            }
        }
        if (L10_out) memcpy(L10_out + s * 10, L10, sizeof L10);
        if (post10_out) memcpy(post10_out + s * 10, post, sizeof post);
    }
    if (off_out) off_out[S] = (uint32_t)start[S];
    free(bb); free(qq); free(cc); free(ss); free(keys);
    free(tup); free(fill); free(start); free(depth); free(repeat); free(count_all); free(n_uni);
    return 0;
}
