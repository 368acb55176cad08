/*
 * gsnp.h — C ABI of libgsnp, the B200 (sm_100a) GSNP hot path.
 *
 * GSNP (Lu et al., ICPP 2011; /root/reference/PAPER.md, cited "P:L<line>") detects SNPs with the
 * SOAPsnp Bayesian model: a calibration pass over all aligned reads (cal_p_matrix, P:L193-196,
 * P:L714-727), then per window of sites (read_site): counting (§IV-B),
 * likelihood = sort + comp (Alg. 4), posterior and output.  This
 * library computes that path on one GPU; every step runs in its CUDA kernels.  Readings of what
 * the paper leaves silent (R1..R15) are listed in DESIGN.md §3.
 *
 * Conventions for every call:
 *  - Status: 0 = GSNP_OK, negative = error (below); never exit()/abort().  After an error the
 *    context stays usable; gsnp_last_error() holds a one-line description.
 *  - Ownership: every input pointer is borrowed for the duration of the call only.  The context
 *    copies what it keeps (reference codes, known-SNP list, tables).  Outputs go to caller-owned
 *    buffers, which may be host memory or device memory (detected per pointer).
 *  - Concurrency: one context per device per process; a context is not thread-safe.  Work is
 *    enqueued on params.stream (NULL = the legacy default stream); calls that return results to
 *    the host synchronise that stream before returning.
 *  - Base codes 0=A 1=C 2=T 3=G 4=N; genotype n = 0..9 is AA AC AT AG CC CT CG TT TG GG
 *    (Alg. 4 lines 13-17).
 */
#ifndef GSNP_H
#define GSNP_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GSNP_ABI_VERSION 1u

typedef int32_t gsnp_status;
#define GSNP_OK 0
#define GSNP_E_INVAL (-1)     /* NULL/invalid argument or parameter */
#define GSNP_E_RANGE (-2)     /* value out of range: len > max_read_len, qual > q_max, base > 4,
                                 strand > 1, hits == 0, read/window outside the reference */
#define GSNP_E_UNSORTED (-3)  /* read positions decrease (input must be sorted) */
#define GSNP_E_STATE (-4)     /* call order violated (gsnp_call before calibration) */
#define GSNP_E_NOMEM (-5)     /* host or device allocation failed */
#define GSNP_E_CUDA (-6)      /* CUDA runtime error (message in gsnp_last_error) */
#define GSNP_E_CAPACITY (-7)  /* output buffer too small; *n_out holds the required count */

#define GSNP_RANK_SUM 0x1u    /* apply the rank-sum test to heterozygous calls (reading R8) */
#define GSNP_TIMING 0x2u      /* record per-stage device times with CUDA events (see below) */
/* Prior variants (reading R18; P:L216 names only known-SNP priors): */
#define GSNP_MONOPLOID 0x4u   /* heterozygous genotypes get prior 0 at every site (known rows too) */
#define GSNP_TITV 0x8u        /* novel priors weighted for transition:transversion 2:1: the
                                 transition allele of ref (A<->G, C<->T) x2, transversions x1/2 */
/* Exact small-sample rank-sum (reading R20, SURVEY §8(f) NEXT #4 "exact small-N rank-sum table";
 * the paper never names the test).  With GSNP_RANK_SUM also set: when both
 * allele groups hold <= GSNP_RANK_EXACT_MAX unique reads and the pooled qualities have no ties,
 * rank_p is the exact two-sided p-value min(1, 2 min(P(U <= u), P(U >= u))) of the Mann-Whitney
 * U = W - n1(n1+1)/2 under H0 (all C(n1+n2, n1) rank sets equally likely), read from a table the
 * library builds at gsnp_create; otherwise the normal approximation of R8 stays. */
#define GSNP_RANK_EXACT 0x10u
#define GSNP_RANK_EXACT_MAX 32

/* stages reported by gsnp_stage_times */
#define GSNP_STAGE_VALIDATE 0     /* k_validate_reads (calibration) */
#define GSNP_STAGE_CALIB 1        /* k_calib_count (a1) */
#define GSNP_STAGE_RANGES 2       /* k_prep: read validation + per-group read ranges (a3) */
#define GSNP_STAGE_CALL 3         /* k_call_tile (a4..a8): the three instantiations of one call */
#define GSNP_STAGE_FINALIZE 4     /* host tables + upload (a2), wall time on the host */
#define GSNP_STAGE_BIG 5          /* k_big_sites (sites with > 1024 unique keys) */
#define GSNP_STAGE_COMPRESS 6     /* k_cz_* (output compression, §V-B) */
#define GSNP_STAGE_WARP 7         /* k_warp_sites (sites with more keys than the thread path) */
#define GSNP_STAGE_DENSE_COUNT 8    /* k_dense_count (dense ablation, gsnp_call_dense) */
#define GSNP_STAGE_DENSE_LIK 9      /* k_dense_sites (dense Alg. 1 + posterior + record) */
#define GSNP_STAGE_DENSE_RECYCLE 10 /* re-zeroing base_occ after each chunk (memset) */
#define GSNP_STAGE_PARSE 11         /* k_nl_tiles, k_parse_meta, k_sel_*, k_parse_emit (gsnp_parse_soap) */
#define GSNP_STAGE_UNPACK 12        /* k_unpack (gsnp_unpack_reads, packed reads R21) */
#define GSNP_N_STAGES 13

typedef struct gsnp_ctx gsnp_ctx;  /* opaque; owned by the library until gsnp_destroy */

typedef struct {
    uint32_t abi_version;     /* must be GSNP_ABI_VERSION */
    uint32_t max_read_len;    /* L, 1..256 (8-bit coord field); default 100 */
    uint32_t q_max;           /* highest quality, <= 63 (6-bit score field); default 40 */
    uint32_t calib_min_count; /* tau of the calibration estimator (R1); default 10 */
    double het_novel;         /* novel heterozygote prior (R6); default 1e-3 */
    double althom_novel;      /* novel alt-homozygote prior (R6); default 5e-4 */
    double global_dep;        /* global dependency coefficient in (0,1] (R3); default 0.9 */
    double pcr_dep;           /* PCR dependency coefficient in (0,1] (R3); default 0.5 */
    uint32_t flags;           /* GSNP_RANK_SUM (default set) */
    int32_t device;           /* CUDA device ordinal; default 0 */
    void* stream;             /* cudaStream_t to enqueue on, or NULL; e.g. a torch stream */
} gsnp_params;

typedef struct {              /* the reference sequence (input file 2) */
    const uint8_t* code;      /* n_sites codes 0..4, host memory */
    uint64_t n_sites;
    uint64_t origin;          /* global coordinate of code[0] (a shard's offset) */
} gsnp_reference;

typedef struct {              /* known SNPs with priors (input file 3) */
    uint64_t n;
    const uint64_t* pos;      /* strictly increasing global coordinates, host memory */
    const double* prior10;    /* n x 10 linear priors (> 0), genotype order n = 0..9 */
} gsnp_priors;

typedef struct {              /* aligned reads sorted by position (input file 1) */
    uint64_t n_reads;
    const uint64_t* pos;      /* leftmost global coordinate, non-decreasing */
    const uint16_t* len;      /* 1..max_read_len */
    const uint64_t* off;      /* n_reads+1 offsets into bases/quals (base i of read r at off[r]+i);
                                 off[0] need not be 0 */
    const uint8_t* bases;     /* 0..4, reference-forward orientation (R11) */
    const uint8_t* quals;     /* 0..q_max */
    const uint8_t* strand;    /* 0 '+', 1 '-' */
    const uint16_t* hits;     /* >= 1; 1 = uniquely aligned */
    int32_t on_device;        /* 0: host arrays (copied by the library); 1: device arrays on the
                                 context's device (e.g. torch CUDA tensors), used in place */
} gsnp_reads;

typedef struct {              /* 40 bytes: one output row (fields R9) */
    uint64_t pos;             /* global coordinate */
    uint8_t ref;              /* reference code */
    uint8_t genotype;         /* 0..9, 255 = no call (ref N and depth 0) */
    uint8_t quality;          /* consensus quality 0..99 (R9) */
    uint8_t base1, base2;     /* best / second base, 4 = none (R9) */
    uint8_t avgq1, avgq2;     /* mean quality of the unique base1/base2 observations */
    uint8_t known;            /* 1 if the site is in the known-SNP list */
    uint16_t cnt_uni1, cnt_all1, cnt_uni2, cnt_all2;  /* unique / all counts (saturating) */
    uint32_t depth;           /* non-N aligned bases (all hits) */
    float rank_p;             /* rank-sum p-value of het calls, else 1 (R8) */
    float copy_num;           /* sum(hits) / depth (R9) */
    float post1;              /* posterior probability of the called genotype (R7) */
} gsnp_record;

/* Fill *out with the defaults listed above. */
gsnp_status gsnp_params_default(gsnp_params* out);

/* Known-SNP priors from allele frequencies (reading R18; the known-SNP file of P:L216 as
 * SOAPsnp's per-site A/C/T/G frequencies): Hardy-Weinberg genotype frequencies f_a^2 (a/a) and
 * 2 f_a f_b (a/b) of the row-normalised frequencies, each floored at floor_prior (> 0) so every
 * prior is positive, as gsnp_priors requires.  freq: n x 4 (A, C, T, G; >= 0, row sum > 0), host;
 * prior10: n x 10 out, host, genotype order n = 0..9.  A bad row -> GSNP_E_RANGE (rows before it
 * are written).  Host arithmetic only; no context needed. */
gsnp_status gsnp_priors_from_freq(const double* freq, uint64_t n, double floor_prior,
                                  double* prior10);

/* Create a context on params->device: copies the reference and known-SNP list to the device and
 * builds the adjust table (R3) on the host.  priors may be NULL (no known SNPs). */
gsnp_status gsnp_create(const gsnp_reference* ref, const gsnp_priors* priors,
                        const gsnp_params* params, gsnp_ctx** out);

/* Calibration = count (GPU histogram, a1) + finalize (host tables, a2).  Needs all reads before
 * any window is called.  Reads must lie inside the reference. */
gsnp_status gsnp_calibrate(gsnp_ctx* ctx, const gsnp_reads* reads);

/* Multi-process split of gsnp_calibrate.  _count writes this shard's counts
 * C[q][cyc][t][o] (uint64[64][256][4][4], index q<<12|cyc<<4|t<<2|o; host or device buffer).
 * Count each read on exactly one rank.  The caller sums the buffers across ranks (e.g.
 * torch.distributed.all_reduce) and passes the sum to _finalize, which builds the p matrix, the
 * score table T (Alg. 3) and the priors on the host and uploads them. */
gsnp_status gsnp_calibrate_count(gsnp_ctx* ctx, const gsnp_reads* reads, uint64_t* counts);
gsnp_status gsnp_calibrate_finalize(gsnp_ctx* ctx, const uint64_t* counts);

/* input packing on the GPU: SOAP alignment text (input file 1,
 * P:L206-212, in SOAPsnp's format; reading R19) -> the gsnp_reads arrays.  One
 * alignment per '\n'-terminated line (the last line may be unterminated; empty lines are
 * skipped), tab-separated fields
 *   id  seq  qual  n_hits  a/b  len  strand(+/-)  chr  location(1-based)  [further fields ignored]
 * seq in reference-forward orientation, ACGTN (either case) -> 0 1 2 3 4; qual characters minus
 * q_offset (33 or 64), each 0..63; n_hits >= 1 (saturates at 65535); len == |seq| == |qual|,
 * 1..256.  Lines whose chr differs from chr_name (NULL or "" = any) are skipped; the others, in
 * input order, become reads with pos = location - 1 + loc_base.
 *   text: n_bytes bytes, host or device (device text is used in place when 16-byte aligned).
 *   outputs: reads_cap entries of pos/len/strand/hits, reads_cap+1 of off (off[0] = 0),
 *   bases_cap of bases/quals; all host or all device (judged by pos).
 *   *n_reads / *n_bases: the selected reads and their bases — also set on GSNP_E_CAPACITY (caps
 *   too small; nothing written), so a call with caps 0 and NULL outputs is a size query.
 * A malformed selected line (missing fields, bad number, |seq| != len, strand not +/-, a base
 * or quality character out of range) -> GSNP_E_RANGE naming the first bad line.  Sortedness
 * and the reference range are checked later, by gsnp_calibrate / gsnp_call. */
gsnp_status gsnp_parse_soap(gsnp_ctx* ctx, const char* text, uint64_t n_bytes, const char* chr_name,
                            uint32_t q_offset, uint64_t loc_base, uint64_t* pos, uint16_t* len,
                            uint64_t* off, uint8_t* bases, uint8_t* quals, uint8_t* strand,
                            uint16_t* hits, uint64_t reads_cap, uint64_t bases_cap,
                            uint64_t* n_reads, uint64_t* n_bases);

/* SURVEY.md §8(f) NEXT #2, second half — the compressed copy of the input (PAPER.md P:L708-727,
 * §V-A: GSNP's first pass writes it, about a third of the input's size, for the second pass).  Here
 * it is what crosses PCIe: reading R21 of DESIGN.md (oracle/pack.py), a stream of 2-bit bases
 * with an N exception list, qualities as maximal runs of equal value inside each read
 * (P:L761-764), and 6 bytes of metadata per read (position relative to its block of block_reads
 * reads, length, strand | hits, run count; hits >= 128 as exceptions) — ~47 bytes per 100-bp read
 * against 221 unpacked.
 *
 * gsnp_pack_reads: encode host reads (on_device 0; bases contiguous per read at off[r]) on the
 *   host's cores.  ref NULL: version 1 (2-bit bases); ref given (host codes, the reference the
 *   reads are aligned to): version 2 — a base is predicted as the reference code at its site and
 *   only the bases that differ are stored (u32 block-relative index << 3 | code), ~0.3 B/base
 *   instead of ~0.5; such a stream must be unpacked by a context created on the same reference.
 *   block_reads 1..4096.  out: host buffer of cap bytes; *n_bytes receives the
 *   stream size (also on GSNP_E_CAPACITY, when out is NULL or cap too small — a size query).
 *   A length outside 1..256, base > 4, quality > 63, strand > 1, hits 0, a position before its
 *   block's first read or >= 2^32 past it, or (version 2) a read outside ref -> GSNP_E_RANGE.
 *   No context needed.
 * gsnp_packed_sizes: n_reads / n_bases of a stream (host memory; the header is checked).
 * gsnp_unpack_reads: decode a stream (host — copied H2D in chunks on the library's copy stream,
 *   overlapped with the decode — or device memory) into DEVICE arrays sized by gsnp_packed_sizes
 *   (off: n_reads + 1 entries, rebuilt contiguous from 0).  Work is stream-ordered on
 *   params.stream; the call returns once a host stream has been copied (it may be reused).  The
 *   decoded reads are then passed to gsnp_calibrate / gsnp_call like any device reads (they are
 *   validated there).  A bad header -> GSNP_E_INVAL. */
gsnp_status gsnp_pack_reads(const gsnp_reads* reads, const gsnp_reference* ref, uint32_t block_reads,
                            void* out, uint64_t cap, uint64_t* n_bytes);
gsnp_status gsnp_packed_sizes(const void* packed, uint64_t n_bytes, uint64_t* n_reads,
                              uint64_t* n_bases);
gsnp_status gsnp_unpack_reads(gsnp_ctx* ctx, const void* packed, uint64_t n_bytes, uint64_t* pos,
                              uint16_t* len, uint64_t* off, uint8_t* bases, uint8_t* quals,
                              uint8_t* strand, uint16_t* hits);

/* Call sites [w0, w1) (global coordinates inside the reference): one gsnp_record per site,
 * written to out[0 .. w1-w0).  reads must include every read overlapping the window (the
 * read-length halo: pos in [w0-L+1, w1)); bases outside [w0, w1) are ignored.  out may be host or
 * device memory.  out_cap < w1-w0 -> GSNP_E_CAPACITY with *n_out = w1-w0. */
gsnp_status gsnp_call(gsnp_ctx* ctx, const gsnp_reads* reads, uint64_t w0, uint64_t w1,
                      gsnp_record* out, uint64_t out_cap, uint64_t* n_out);

/* Windowed calling without host round trips (the paper calls windows of >= 256 K sites,
 * P:L835-840): gsnp_call_async enqueues the same work as gsnp_call on params.stream and returns at
 * once — reads must be device arrays and out device memory.  Nothing is read back: out-of-range
 * input and capacity conditions found on the device are recorded in the context's error flag,
 * later windows skip their work once an input is invalid, and gsnp_wait synchronises the stream
 * and returns the first such status (then clears it).  Argument errors found on the host are
 * returned directly.  gsnp_call (synchronous) clears the flag when it starts. */
gsnp_status gsnp_call_async(gsnp_ctx* ctx, const gsnp_reads* reads, uint64_t w0, uint64_t w1,
                            gsnp_record* out, uint64_t out_cap);
gsnp_status gsnp_wait(gsnp_ctx* ctx);

/* the dense ablation (Fig. 5): the same records as
 * gsnp_call, computed the way SOAPsnp's Alg. 1 does on the GPU: per site a dense
 * base_occ[4][64][256][2] of 1-byte occurrence counts (131,072 B, index base<<15 | score<<9 |
 * coord<<1 | strand) is filled (`counting`), walked in full loop-nest order
 * (`likelihood`: base 0..3, score q_max..0, coord 0..L-1, strand 0..1) and re-zeroed
 * (`recycle`), chunk_sites sites at a time (the paper's window of sites).  Arguments
 * as gsnp_call; chunk_sites: a multiple of 32 in [32, 2^20] (device memory chunk_sites x 128 KiB,
 * owned by the context).  A cell reaching 256 occurrences (more than 255 identical unique bases
 * at one site: the paper's 1-byte cell) -> GSNP_E_CAPACITY. */
gsnp_status gsnp_call_dense(gsnp_ctx* ctx, const gsnp_reads* reads, uint64_t w0, uint64_t w1,
                            uint32_t chunk_sites, gsnp_record* out, uint64_t out_cap,
                            uint64_t* n_out);

/* Debug dump of the same pipeline for [w0, w1) into HOST buffers (any may be NULL):
 *   off[S+1]        u32 CSR offsets of each site's unique keys (S = w1-w0)
 *   keys_built      u32 keys as the builder scattered them (per-site order unspecified)
 *   keys_sorted     u32 keys after the sort (ascending)  — both sized off[S]
 *   site_counters   u32[S][15] = depth, dep_uni, repeat, count_all[4], count_uni[4], q_sum[4]
 *   L10, post10     f64[S][10] log10 likelihoods and posteriors
 *   records         gsnp_record[S]
 * Buffers for keys must hold at least the number of bases in reads. */
gsnp_status gsnp_debug_window(gsnp_ctx* ctx, const gsnp_reads* reads, uint64_t w0, uint64_t w1,
                              uint32_t* off, uint32_t* keys_built, uint32_t* keys_sorted,
                              uint32_t* site_counters, double* L10, double* post10,
                              gsnp_record* records);

/* Copy the context's tables to host buffers (any may be NULL):
 *   counts u64[64*256*16]; p_matrix f64[64*256*16] (index q<<12|coord<<4|allele<<2|base);
 *   T f64[64*L*4*10] (index ((q*L+coord)*4+base)*10+n, Alg. 3; rows q = 1..q_max are built —
 *   adjust() never leaves that range — the others are zero); adj u8[64*adj_pcr*adj_g].
 * dims (may be NULL) receives {L, adj_pcr, adj_g}. */
gsnp_status gsnp_get_tables(gsnp_ctx* ctx, uint64_t* counts, double* p_matrix, double* T,
                            uint8_t* adj, uint32_t* dims);

/* Output compression (§V-B): compress records rec[0 .. n) into a stream of uint32
 * words, in blocks of block_sites consecutive records (1 .. 2^24; the paper compresses per window,
 * P:L749).  The byte format is reading R17 of DESIGN.md: per block a header (magic "GSC1", n,
 * pos of the first record, block words, block_sites), 2-bit planes of ref/base1/base2 + runs of
 * N, exception lists for genotype/known/rank_p/post1, the sparse
 * second-allele columns, and the six quality columns quality, avgq1, cnt_uni1,
 * cnt_all1, depth, copy_num as RLE with both run arrays DICT-encoded.  Records are
 * expected in ascending pos order with pos[i+1] = pos[i] + 1 inside a block (what gsnp_call
 * writes); pos is not stored beyond the block's first record.
 *   rec: host or device memory (device: used in place).  out: host or device memory.
 *   out_cap: capacity in words.  *n_words: words of the stream (also on GSNP_E_CAPACITY, when
 *   out_cap is too small; nothing is written then).  out may be NULL with out_cap 0 to query.
 * Every step runs in the library's kernels (k_cz_*); the host only reads the total size.
 * Device output is written stream-ordered on params.stream (the call returns once the size is
 * known; synchronise that stream, or order work after it, before reading the words); host
 * output has landed when the call returns. */
gsnp_status gsnp_compress(gsnp_ctx* ctx, const gsnp_record* rec, uint64_t n, uint32_t block_sites,
                          uint32_t* out, uint64_t out_cap, uint64_t* n_words);

/* gsnp_call followed by gsnp_compress of the window's records without the records leaving the
 * device (a8 -> §V-B fused at the library level): the result is the compressed stream only. */
gsnp_status gsnp_call_compressed(gsnp_ctx* ctx, const gsnp_reads* reads, uint64_t w0, uint64_t w1,
                                 uint32_t block_sites, uint32_t* out, uint64_t out_cap,
                                 uint64_t* n_words);

/* Number of kernel launches this context has issued so far (for bench accounting). */
uint64_t gsnp_launch_count(const gsnp_ctx* ctx);

/* With GSNP_TIMING set in params.flags: accumulated milliseconds and launch counts per stage
 * (GSNP_STAGE_*), measured with CUDA events recorded on params.stream around each launch
 * (finalize: host wall time).  ms/launches may be NULL; n_stages <= GSNP_N_STAGES entries are
 * written; reset != 0 clears the accumulators after reading. */
gsnp_status gsnp_stage_times(gsnp_ctx* ctx, double* ms, uint64_t* launches, int n_stages,
                             int reset);

const char* gsnp_strerror(gsnp_status s);
const char* gsnp_last_error(const gsnp_ctx* ctx);
void gsnp_destroy(gsnp_ctx* ctx);

#ifdef __cplusplus
}
#endif
#endif /* GSNP_H */
