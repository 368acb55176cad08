// gsnp.cu — libgsnp: the C ABI of include/gsnp.h (host orchestration + table builders) and the
// sm_100a kernels of gsnp_kernels.cuh.  See DESIGN.md for the path, readings and roofline.
//
// Host arithmetic that feeds integer decisions (the adjust table, R3) or the score table T
// (Alg. 3; built on the CPU for CPU/GPU consistency, §IV-G) is compiled
// with -ffp-contract=off and uses glibc log10/pow.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <condition_variable>
#include <functional>
#include <mutex>
#include <cmath>
#include <cstdarg>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <map>
#include <string>
#include <thread>
#include <vector>

#include "gsnp.h"
#include "gsnp_kernels.cuh"
#include "gsnp_compress.cuh"
#include "gsnp_dense.cuh"
#include "gsnp_parse.cuh"
#include "gsnp_pack.cuh"

using namespace gsnp_dev;

namespace gsnp_deep {   // gsnp_deep.cu: the deep-window k_call_tile with 384-thread CTAs
const void* call_tile_kernel(bool dbg);
int call_tile_nt();
size_t call_tile_smem(int L, size_t adj_bytes, uint32_t* adj_smem);
}

namespace {

template <typename T>
struct DevBuf {  // grow-only device buffer
    T* p = nullptr;
    size_t n = 0;
    cudaError_t ensure(size_t want) {
        if (want <= n && p) return cudaSuccess;
        if (p) cudaFree(p);
        p = nullptr;
        n = 0;
        cudaError_t e = cudaMalloc(&p, std::max<size_t>(want, 1) * sizeof(T));
        if (e == cudaSuccess) n = std::max<size_t>(want, 1);
        return e;
    }
    void release() {
        if (p) cudaFree(p);
        p = nullptr;
        n = 0;
    }
};

const double kLog10Zero = 0.0;
constexpr size_t REF_PAD = 64;      // N bytes before and after the device reference

}  // namespace

namespace {
// Persistent host worker threads of a context (the table build of every calibration runs on
// them; creating threads per call would cost more than the work).  run(f) executes f on every
// worker and on the caller, and returns when all are done.
struct HostPool {
    std::vector<std::thread> th;
    std::mutex m;
    std::condition_variable cv, done_cv;
    std::function<void()> job;
    uint64_t gen = 0;
    int busy = 0;
    bool stop = false;
    void start(int n) {
        for (int i = 0; i < n; ++i)
            th.emplace_back([this] {
                uint64_t seen = 0;
                for (;;) {
                    std::function<void()> j;
                    {
                        std::unique_lock<std::mutex> l(m);
                        cv.wait(l, [&] { return stop || gen != seen; });
                        if (stop) return;
                        seen = gen;
                        j = job;
                    }
                    j();
                    std::lock_guard<std::mutex> l(m);
                    if (--busy == 0) done_cv.notify_all();
                }
            });
    }
    void run(const std::function<void()>& f) {
        {
            std::lock_guard<std::mutex> l(m);
            job = f;
            busy = (int)th.size();
            ++gen;
        }
        cv.notify_all();
        f();
        std::unique_lock<std::mutex> l(m);
        done_cv.wait(l, [&] { return busy == 0; });
    }
    ~HostPool() {
        {
            std::lock_guard<std::mutex> l(m);
            stop = true;
        }
        cv.notify_all();
        for (auto& t : th) t.join();
    }
};
}  // namespace

struct gsnp_ctx {
    HostPool pool;                 // started at gsnp_create
    gsnp_params prm{};
    cudaStream_t stream = nullptr;
    std::string err;
    // reference + known SNPs
    uint64_t n_sites = 0, origin = 0;
    DevBuf<uint8_t> ref;           // code | known << 3, with REF_PAD bytes of N on both sides
    const uint8_t* ref_code = nullptr;   // = ref.p + REF_PAD: code of site origin
    DevBuf<uint64_t> known_pos;
    DevBuf<double> known_lp;
    uint64_t n_known = 0;
    std::vector<uint64_t> h_known_pos;
    // tables
    std::vector<uint8_t> h_adj;
    int adjP = 1, adjG = 1;
    DevBuf<uint8_t> adj;
    DevBuf<double> LP;
    DevBuf<double> rank_cdf;       // R20 exact rank-sum table (GSNP_RANK_EXACT only)
    std::vector<uint64_t> h_counts;
    std::vector<double> h_p;   // [64][256][4][4]
    double* h_T = nullptr;     // [64][L][4][10], pinned host copy of the score table
    size_t h_T_n = 0;
    uint64_t* h_cnt_pinned = nullptr;   // staging for device-resident counts
    DevBuf<double> T;
    bool T_zeroed = false;
    bool calibrated = false;
    // scratch
    DevBuf<int> d_err;
    DevBuf<unsigned long long> d_counts;
    DevBuf<uint64_t> tile_ra, tile_rb;
    DevBuf<gsnp_record> rec;
    DevBuf<BigSite> big;
    DevBuf<uint32_t> big_n;
    DevBuf<uint32_t> wlist;
    DevBuf<uint32_t> wlist2;       // k_list_sites' leftovers for k_warp_sites
    // dense ablation (§8(f) NEXT #3): base_occ of one chunk of sites + per-site all-hits counters
    DevBuf<uint8_t> dense_occ;
    DevBuf<uint32_t> dense_cnt;
    // SOAP text parsing (§8(f) NEXT #2)
    DevBuf<uint8_t> p_text, p_chr;
    DevBuf<uint64_t> p_cnt, p_ls, p_meta, p_pos, p_ridx, p_boff, p_part, p_scal;
    // staged host reads
    DevBuf<uint64_t> r_pos, r_off;
    DevBuf<uint16_t> r_len, r_hits;
    DevBuf<uint8_t> r_bases, r_quals, r_strand;
    // debug
    DevBuf<uint32_t> dbg_u32a, dbg_u32b, dbg_u32c, dbg_u32d, dbg_u32e;
    DevBuf<double> dbg_f64a, dbg_f64b;
    // output compression scratch (§V-B)
    DevBuf<uint8_t> cz_cols;
    DevBuf<uint32_t> cz_meta, cz_dD, cz_dict, cz_out;
    DevBuf<uint64_t> cz_off;
    DevBuf<gsnp_record> cz_rec;
    uint64_t* h_cz_total = nullptr;     // pinned
    // mapped pinned mailbox for the few scalars the host reads on the call path (status flag,
    // window read range, compressed size): written by k_peek over PCIe with SM stores, so a
    // caller's large device->host copy in flight on another stream (same DMA engine) cannot
    // delay the read
    uint64_t* mbox = nullptr;
    uint64_t launches = 0;
    // packed reads (R21): device copy of a host stream, the copy stream and its chunk events
    DevBuf<uint8_t> pk_buf;
    cudaStream_t copy_stream = nullptr;
    std::vector<cudaEvent_t> pk_ev;
    // per-device facts, read at gsnp_create on prm.device (a process may hold contexts on
    // several devices)
    int num_sms = 148;
    // (kernel, dynamic smem) -> resident CTAs per SM, with the smem attribute set: host API calls
    // made once, not on every window of a windowed run
    std::map<std::pair<const void*, size_t>, int> occ;
    int occupancy(const void* kern, int nt, size_t smem) {
        auto key = std::make_pair(kern, smem);
        auto it = occ.find(key);
        if (it != occ.end()) return it->second;
        int per = 0;
        static const int carve = [] { const char* e = getenv("GSNP_CARVEOUT"); return e ? atoi(e) : -1; }();
        if (carve >= 0) cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, carve);
        if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess ||
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, kern, nt, smem) != cudaSuccess) {
            cudaGetLastError();
            return -1;
        }
        occ[key] = per;
        return per;
    }
    // window depth thresholds of the 64- / 128-slot k_call_tile instantiations (pick_variant)
    // window mean depth (reads x L / sites) at which the 64- / 128-slot kernels take over; the 32-slot
    // kernel + k_list_sites wins below ~29.5 (tools/thr_probe.sh: 10.7 vs 11.4 ms at 27.6, 14.8 vs
    // 12.4 at 31.3 per 24 M sites)
    float mid_at = 29.5f, deep_at = 48.0f;
    uint32_t epoch = 0;               // calls so far (k_prep's read-length flag)
    uint32_t list_min = 16384;        // k_list_sites below this many listed sites: warp path instead
    bool mid_adj_smem = false;        // the 64-slot kernel reads adj from L1/L2: 3 CTAs per SM
    size_t cal_budget = 0;            // k_calib_count shared-memory budget (0 = not yet sized)
    // per-stage timing (GSNP_TIMING)
    struct Pending { int stage; cudaEvent_t a, b; };
    std::vector<cudaEvent_t> ev_pool;
    std::vector<Pending> pending;
    double stage_ms[GSNP_N_STAGES] = {};
    uint64_t stage_n[GSNP_N_STAGES] = {};
    bool timing() const { return (prm.flags & GSNP_TIMING) != 0; }
    cudaEvent_t ev() {
        if (ev_pool.empty()) {
            cudaEvent_t e;
            cudaEventCreate(&e);
            return e;
        }
        cudaEvent_t e = ev_pool.back();
        ev_pool.pop_back();
        return e;
    }
    // bracket one launch of a stage: call begin() before and end() after the launch
    cudaEvent_t cur_a = nullptr;
    void begin() {
        if (!timing()) return;
        cur_a = ev();
        cudaEventRecord(cur_a, stream);
    }
    void end(int stage) {
        if (!timing()) return;
        cudaEvent_t b = ev();
        cudaEventRecord(b, stream);
        pending.push_back({stage, cur_a, b});
        cur_a = nullptr;
    }
    // after a stream sync: fold completed pairs into the accumulators
    void flush() {
        for (auto& p : pending) {
            float ms = 0;
            if (cudaEventElapsedTime(&ms, p.a, p.b) == cudaSuccess) {
                stage_ms[p.stage] += ms;
                stage_n[p.stage] += 1;
            } else {
                cudaGetLastError();
            }
            ev_pool.push_back(p.a);
            ev_pool.push_back(p.b);
        }
        pending.clear();
    }
};

namespace {

gsnp_status fail(gsnp_ctx* c, gsnp_status s, const char* fmt, ...) {
    if (c) {
        char buf[512];
        va_list ap;
        va_start(ap, fmt);
        vsnprintf(buf, sizeof buf, fmt, ap);
        va_end(ap);
        c->err = buf;
    }
    return s;
}

#define CK(call)                                                                              \
    do {                                                                                      \
        cudaError_t e_ = (call);                                                              \
        if (e_ != cudaSuccess)                                                                \
            return fail(ctx, e_ == cudaErrorMemoryAllocation ? GSNP_E_NOMEM : GSNP_E_CUDA,    \
                        "%s: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, __LINE__); \
    } while (0)

bool is_device_ptr(const void* p) {
    if (!p) return false;
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// R3: q_adj = max(1, (int)(10^(log10 q + (pcr-1) log10 pcr_dep + g log10 global_dep) + 0.5))
int adjust_expr(double lpd, double lgd, int q, int pcr, int g) {
    double lq = log10((double)q);
    double e = lq + (double)(pcr - 1) * lpd + (double)g * lgd;
    int qa = (int)(pow(10.0, e) + 0.5);
    return qa < 1 ? 1 : qa;
}

// R20 table F[(m*33+n)*1025 + u] = P(U <= u) of the Mann-Whitney U for sample sizes m, n <= 32
// under H0.  Frequencies by the recursion on the largest pooled observation:
// c(m,n,u) = c(m-1,n,u-n) + c(m,n-1,u), c(0,n,u) = c(m,0,u) = [u == 0]; doubles are exact up to
// 2^53 and relative 1e-16 beyond (C(64,32) ~ 1.8e18).
void build_rank_cdf(std::vector<double>& F) {
    const int M = GSNP_RANK_EXACT_MAX, S = (M + 1) * (M + 1) * 1025;
    std::vector<double> c(S, 0.0);
    auto at = [&](int m, int n) { return c.data() + (size_t)(m * 33 + n) * 1025; };
    for (int m = 0; m <= M; ++m)
        for (int n = 0; n <= M; ++n) {
            double* cm = at(m, n);
            if (m == 0 || n == 0) { cm[0] = 1.0; continue; }
            const double *a = at(m - 1, n), *b = at(m, n - 1);
            for (int u = 0; u <= m * n; ++u) cm[u] = (u >= n ? a[u - n] : 0.0) + b[u];
        }
    F.assign(S, 1.0);
    for (int m = 0; m <= M; ++m)
        for (int n = 0; n <= M; ++n) {
            const double* cm = at(m, n);
            double tot = 0.0, run = 0.0;
            for (int u = 0; u <= m * n; ++u) tot += cm[u];
            double* f = F.data() + (size_t)(m * 33 + n) * 1025;
            for (int u = 0; u <= m * n; ++u) { run += cm[u]; f[u] = run / tot; }
        }
}

// Build adj[64][P][G].  The expression is non-increasing in pcr and g (coefficients <= 1), so
// P = first pcr with adjust(63, P, 0) == 1 and G = first g with adjust(63, 1, G) == 1 bound
// where it saturates at 1; beyond them every cell is 1 and indices clamp.
gsnp_status build_adj(gsnp_ctx* ctx) {
    const double lpd = log10(ctx->prm.pcr_dep), lgd = log10(ctx->prm.global_dep);
    int P = 1, G = 1;
    if (ctx->prm.pcr_dep < 1.0) {
        while (adjust_expr(lpd, lgd, 63, P, 0) > 1) {
            if (++P > 255) return fail(ctx, GSNP_E_INVAL, "pcr_dep too close to 1 (table > 255)");
        }
    }
    if (ctx->prm.global_dep < 1.0) {
        while (adjust_expr(lpd, lgd, 63, 1, G - 1) > 1) {
            if (++G > 4096) return fail(ctx, GSNP_E_INVAL, "global_dep too close to 1");
        }
    } else {
        G = 1;
    }
    // with global_dep == 1, g has no effect (G = 1); with pcr_dep == 1, P = 1.
    ctx->adjP = P;
    ctx->adjG = G;
    ctx->h_adj.assign((size_t)64 * P * G, 1);
    for (int q = 0; q < 64; ++q)
        for (int p = 1; p <= P; ++p)
            for (int g = 0; g < G; ++g)
                ctx->h_adj[((size_t)q * P + (p - 1)) * G + g] = (uint8_t)adjust_expr(lpd, lgd, q, p, g);
    return GSNP_OK;
}

// R1 estimator (host) for one quality q: p[q][c][t][o], index q<<12 | c<<4 | t<<2 | o.
void estimate_p_q(const gsnp_params& prm, const uint64_t* C, double* p, int q) {
    const int L = (int)prm.max_read_len;
    const double tau = (double)prm.calib_min_count;
    double tot = 0, mm = 0;
    for (int c = 0; c < L; ++c)
        for (int t = 0; t < 4; ++t)
            for (int o = 0; o < 4; ++o) {
                double v = (double)C[q << 12 | c << 4 | t << 2 | o];
                tot += v;
                if (t != o) mm += v;
            }
    for (int t = 0; t < 4; ++t) {
        double npool[4] = {0, 0, 0, 0}, Npool = 0;
        for (int c = 0; c < L; ++c)
            for (int o = 0; o < 4; ++o) {
                double v = (double)C[q << 12 | c << 4 | t << 2 | o];
                npool[o] += v;
                Npool += v;
            }
        for (int c = 0; c < L; ++c) {
            double Nct = 0;
            for (int o = 0; o < 4; ++o) Nct += (double)C[q << 12 | c << 4 | t << 2 | o];
            for (int o = 0; o < 4; ++o) {
                double n = (double)C[q << 12 | c << 4 | t << 2 | o], v;
                if (n > tau) v = n / Nct;
                else if (npool[o] > tau) v = npool[o] / Npool;
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

// Alg. 3 score-table rows of quality qa: T[qa][c][b][n] = log10(0.5 p[qa][c][a1][b] +
// 0.5 p[qa][c][a2][b]), the value Alg. 2 returns, built on the CPU (§IV-G).
// Rows are stored with TROW (>= 10) doubles each; the padding stays zero.
void build_T_q(int L, const double* p, double* T, int qa, int c_lo, int c_hi) {
    static const int A1[10] = {0, 0, 0, 0, 1, 1, 1, 2, 2, 3};
    static const int A2[10] = {0, 1, 2, 3, 1, 2, 3, 2, 3, 3};
    for (int c = c_lo; c < c_hi; ++c)
        for (int b = 0; b < 4; ++b)
            for (int n = 0; n < 10; ++n) {
                int p1 = qa << 12 | c << 4 | A1[n] << 2 | b;
                int p2 = qa << 12 | c << 4 | A2[n] << 2 | b;
                T[(((size_t)qa * L + c) * 4 + b) * TROW + n] = log10(0.5 * p[p1] + 0.5 * p[p2]);
            }
}

gsnp_status check_params(gsnp_ctx* ctx, const gsnp_params* p) {
    if (!p || p->abi_version != GSNP_ABI_VERSION) return fail(ctx, GSNP_E_INVAL, "bad params/abi");
    if (p->max_read_len < 1 || p->max_read_len > 256) return fail(ctx, GSNP_E_INVAL, "max_read_len");
    if (p->q_max > 63) return fail(ctx, GSNP_E_INVAL, "q_max > 63");
    if (!(p->global_dep > 0 && p->global_dep <= 1) || !(p->pcr_dep > 0 && p->pcr_dep <= 1))
        return fail(ctx, GSNP_E_INVAL, "dependency coefficients must be in (0,1]");
    if (!(p->het_novel > 0) || !(p->althom_novel > 0)) return fail(ctx, GSNP_E_INVAL, "priors");
    return GSNP_OK;
}

// Stage reads on the device (host arrays are copied; device arrays used in place).
gsnp_status stage_reads(gsnp_ctx* ctx, const gsnp_reads* r, DevReads& d) {
    if (!r) return fail(ctx, GSNP_E_INVAL, "reads == NULL");
    d.n = r->n_reads;
    if (r->n_reads == 0) {
        d.pos = nullptr; d.len = nullptr; d.off = nullptr; d.bases = nullptr; d.quals = nullptr;
        d.strand = nullptr; d.hits = nullptr; d.off0 = 0;
        return GSNP_OK;
    }
    if (!r->pos || !r->len || !r->off || !r->bases || !r->quals || !r->strand || !r->hits)
        return fail(ctx, GSNP_E_INVAL, "NULL read array");
    if (r->on_device) {
        d.pos = r->pos; d.len = r->len; d.off = r->off; d.bases = r->bases; d.quals = r->quals;
        d.strand = r->strand; d.hits = r->hits; d.off0 = 0;
        return GSNP_OK;
    }
    const uint64_t n = r->n_reads;
    const uint64_t o0 = r->off[0], o1 = r->off[n];
    if (o1 < o0) return fail(ctx, GSNP_E_RANGE, "off[n] < off[0]");
    const uint64_t nb = o1 - o0;
    cudaStream_t s = ctx->stream;
    CK(ctx->r_pos.ensure(n));
    CK(ctx->r_off.ensure(n + 1));
    CK(ctx->r_len.ensure(n));
    CK(ctx->r_hits.ensure(n));
    CK(ctx->r_strand.ensure(n));
    CK(ctx->r_bases.ensure(nb));
    CK(ctx->r_quals.ensure(nb));
    CK(cudaMemcpyAsync(ctx->r_pos.p, r->pos, n * 8, cudaMemcpyHostToDevice, s));
    CK(cudaMemcpyAsync(ctx->r_off.p, r->off, (n + 1) * 8, cudaMemcpyHostToDevice, s));
    CK(cudaMemcpyAsync(ctx->r_len.p, r->len, n * 2, cudaMemcpyHostToDevice, s));
    CK(cudaMemcpyAsync(ctx->r_hits.p, r->hits, n * 2, cudaMemcpyHostToDevice, s));
    CK(cudaMemcpyAsync(ctx->r_strand.p, r->strand, n, cudaMemcpyHostToDevice, s));
    CK(cudaMemcpyAsync(ctx->r_bases.p, r->bases + o0, nb, cudaMemcpyHostToDevice, s));
    CK(cudaMemcpyAsync(ctx->r_quals.p, r->quals + o0, nb, cudaMemcpyHostToDevice, s));
    d.pos = ctx->r_pos.p; d.len = ctx->r_len.p; d.off = ctx->r_off.p; d.bases = ctx->r_bases.p;
    d.quals = ctx->r_quals.p; d.strand = ctx->r_strand.p; d.hits = ctx->r_hits.p; d.off0 = o0;
    return GSNP_OK;
}

gsnp_status map_err(gsnp_ctx* ctx, int e) {
    if (!e) return GSNP_OK;
    if (e & ERR_UNSORTED) return fail(ctx, GSNP_E_UNSORTED, "read positions decrease");
    if (e & (ERR_RANGE | ERR_QUAL))
        return fail(ctx, GSNP_E_RANGE, "read value out of range (len/base/qual/strand/hits/pos)");
    if (e & ERR_DENSE_SAT)
        return fail(ctx, GSNP_E_CAPACITY, "a dense base_occ count exceeds 255 (1-byte cells, P:L390)");
    if (e & ERR_DEEP)
        return fail(ctx, GSNP_E_CAPACITY, "a site's unique depth exceeds the shared-memory key buffer");
    return fail(ctx, GSNP_E_CUDA, "device error flag %d", e);
}

__global__ void k_peek(uint8_t* dst, const uint8_t* src, uint32_t n) {
    for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) dst[i] = src[i];
}

// copy n (<= 8) bytes at device address src into mailbox slot `slot` (read after a sync)
gsnp_status peek(gsnp_ctx* ctx, int slot, const void* src, uint32_t n) {
    if (!ctx->mbox) {
        CK(cudaHostAlloc(&ctx->mbox, 16 * sizeof(uint64_t), cudaHostAllocMapped));
        memset(ctx->mbox, 0, 16 * sizeof(uint64_t));
    }
    ctx->mbox[slot] = 0;
    k_peek<<<1, 32, 0, ctx->stream>>>(reinterpret_cast<uint8_t*>(ctx->mbox + slot),
                                      reinterpret_cast<const uint8_t*>(src), n);
    ctx->launches++;
    CK(cudaGetLastError());
    return GSNP_OK;
}

gsnp_status launch_validate(gsnp_ctx* ctx, const DevReads& d) {
    if (d.n == 0) return GSNP_OK;
    unsigned blocks = (unsigned)((d.n + 255) / 256);
    ctx->begin();
    k_validate_reads<<<blocks, 256, 0, ctx->stream>>>(d, ctx->origin, ctx->n_sites,
                                                      (int)ctx->prm.max_read_len, ctx->d_err.p);
    ctx->end(GSNP_STAGE_VALIDATE);
    ctx->launches++;
    CK(cudaGetLastError());
    return GSNP_OK;
}

// a3: per-32-site-group read ranges of [w0, w1) (k_prep, with read validation) and the kernels' arguments
gsnp_status prep_window(gsnp_ctx* ctx, const DevReads& d, uint64_t w0, uint64_t w1,
                        gsnp_record* d_out, CallArgs& A) {
    cudaStream_t s = ctx->stream;
    const uint64_t n_groups = (w1 - w0 + 31) / 32;
    CK(ctx->tile_ra.ensure(n_groups));
    CK(ctx->tile_rb.ensure(n_groups));
    CK(ctx->big_n.ensure(6));
    const uint32_t epoch = ++ctx->epoch;               // k_prep's read-length flag (no reset)
    // one launch: validate the reads (ABI contract; the calling kernels return at once on a
    // violation), the per-group read ranges, and zero the window's work counters
    const uint32_t nbv = (uint32_t)((d.n + 255) / 256);
    ctx->begin();
    k_prep<<<(unsigned)(nbv + (n_groups + 255) / 256), 256, 0, s>>>(
        d, ctx->origin, ctx->n_sites, (int)ctx->prm.max_read_len, ctx->d_err.p, nbv, w0, w1, n_groups,
        ctx->tile_ra.p, ctx->tile_rb.p, ctx->big_n.p, epoch);
    ctx->end(GSNP_STAGE_RANGES);
    ctx->launches++;
    CK(cudaGetLastError());
    A.R = d;
    A.len_flag = ctx->big_n.p + 3;
    A.epoch = epoch;
    A.list_min = ctx->list_min;
    A.ref = ctx->ref_code;
    A.origin = ctx->origin;
    A.n_sites = ctx->n_sites;
    A.known_pos = ctx->known_pos.p;
    A.known_lp = ctx->known_lp.p;
    A.n_known = ctx->n_known;
    A.LP = ctx->LP.p;
    A.T = ctx->T.p;
    A.rank_cdf = (ctx->prm.flags & GSNP_RANK_EXACT) ? ctx->rank_cdf.p : nullptr;
    A.adj = ctx->adj.p;
    A.adjP = ctx->adjP;
    A.adjG = ctx->adjG;
    A.L = (int)ctx->prm.max_read_len;
    A.q_max = (int)ctx->prm.q_max;
    A.flags = ctx->prm.flags;
    A.w0 = w0;
    A.w1 = w1;
    A.tile_ra = ctx->tile_ra.p;
    A.tile_rb = ctx->tile_rb.p;
    A.out = d_out;
    A.err = ctx->d_err.p;
    return GSNP_OK;
}

gsnp_status run_window(gsnp_ctx* ctx, const DevReads& d, uint64_t w0, uint64_t w1,
                       gsnp_record* d_out, CallArgs& A) {
    cudaStream_t s = ctx->stream;
    const uint64_t n_tiles = (w1 - w0 + TS - 1) / TS;
    if (n_tiles == 0) return GSNP_OK;
    gsnp_status st = prep_window(ctx, d, w0, w1, d_out, A);
    if (st) return st;
    const uint64_t n_groups = (w1 - w0 + 31) / 32;
    // persistent CTAs; warps pull 32-site groups from a counter.  The adjust table rides in
    // shared memory when small (it is 64 x 7 x 37 bytes at the default coefficients).
    const size_t adj_bytes = (size_t)64 * A.adjP * A.adjG;
#ifndef GSNP_ADJ_SMEM_MAX
#define GSNP_ADJ_SMEM_MAX (48 * 1024)
#endif
    const uint32_t adj_smem = adj_bytes <= GSNP_ADJ_SMEM_MAX ? 1u : 0u;
    // the three k_call_tile instantiations (32 / 64 / 128 key slots per thread) are all launched;
    // each reads the window's depth from the read ranges on the device and only the one that fits
    // the window does the work (pick_variant) — no host round trip
    A.mid_at = ctx->mid_at;
    A.deep_at = ctx->deep_at;
    const uint32_t big_cap = (uint32_t)std::min<uint64_t>(w1 - w0, 1u << 22);
    CK(ctx->big.ensure(big_cap));
    CK(ctx->wlist.ensure(w1 - w0));                 // sites for k_warp_sites (at most all)
    const bool dbg = A.count_only || A.dbg_off || A.dbg_counters || A.dbg_L10 || A.dbg_post10;
    auto launch_tile = [&](auto kern, int cols, uint32_t adj_on) -> gsnp_status {
        const size_t smem = call_smem_bytes(A.L, adj_on ? adj_bytes : 0, cols, nullptr, nullptr, false);
        const int per_sm = ctx->occupancy(reinterpret_cast<const void*>(kern), NT, smem);
        if (per_sm < 0) return fail(ctx, GSNP_E_CUDA, "k_call_tile: shared memory %zu B", smem);
        const uint64_t want = (uint64_t)ctx->num_sms * std::max(per_sm, 1);
        const unsigned grid = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(want, n_tiles));
        ctx->begin();
        kern<<<grid, NT, smem, s>>>(A, ctx->wlist.p, ctx->big_n.p + 2, ctx->big_n.p + 1, adj_on);
        ctx->end(GSNP_STAGE_CALL);
        ctx->launches++;
        CK(cudaGetLastError());
        return GSNP_OK;
    };
    gsnp_status lst;
    if ((lst = launch_tile(dbg ? k_call_tile<true, COLS> : k_call_tile<false, COLS>, COLS, adj_smem))) return lst;
    if ((lst = launch_tile(dbg ? k_call_tile<true, COLS_MID> : k_call_tile<false, COLS_MID>, COLS_MID,
                           adj_smem && ctx->mid_adj_smem))) return lst;
    {                                                // the 128-slot kernel (gsnp_deep.cu)
        uint32_t adj_on = adj_smem;
        const size_t smem = gsnp_deep::call_tile_smem(A.L, adj_bytes, &adj_on);
        const void* kern = gsnp_deep::call_tile_kernel(dbg);
        const int nt = gsnp_deep::call_tile_nt();
        const int per_sm = ctx->occupancy(kern, nt, smem);
        if (per_sm < 0) return fail(ctx, GSNP_E_CUDA, "deep k_call_tile: shared memory %zu B", smem);
        const uint64_t tiles = (w1 - w0 + nt - 1) / nt;
        const unsigned grid = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(
            (uint64_t)ctx->num_sms * std::max(per_sm, 1), tiles));
        uint32_t* wl = ctx->wlist.p;
        uint32_t* wln = ctx->big_n.p + 2;
        uint32_t* work = ctx->big_n.p + 1;
        void* kargs[] = {&A, &wl, &wln, &work, &adj_on};
        ctx->begin();
        CK(cudaLaunchKernel(kern, dim3(grid), dim3(nt), kargs, smem, s));
        ctx->end(GSNP_STAGE_CALL);
        ctx->launches++;
    }
    if (!A.count_only) {
        // sites the 32-slot kernel listed (33..64 keys): thread per listed site, chunked thread path
        CK(ctx->wlist2.ensure(w1 - w0));
        auto lk = dbg ? k_list_sites<true> : k_list_sites<false>;
        const size_t lsm = (size_t)4 * COLS_MID * TS;
        const int lper = ctx->occupancy(reinterpret_cast<const void*>(lk), NT, lsm);
        if (lper < 0) return fail(ctx, GSNP_E_CUDA, "k_list_sites: shared memory %zu B", lsm);
        ctx->begin();
        lk<<<(unsigned)(ctx->num_sms * std::max(lper, 1)), NT, lsm, s>>>(A, ctx->wlist.p, ctx->big_n.p + 2,
                                                                       ctx->wlist2.p, ctx->big_n.p + 4,
                                                                       ctx->big_n.p + 5);
        ctx->end(GSNP_STAGE_WARP);
        ctx->launches++;
        CK(cudaGetLastError());
        // what is left (n > 64 keys, '-' end recounts, or beyond the deep kernels' thread paths):
        // warp per site
        auto wk = k_warp_sites<COLS>;
        const size_t wsm = call_smem_bytes(A.L, 0, COLS, nullptr, nullptr);
        const int wper = ctx->occupancy(reinterpret_cast<const void*>(wk), NT, wsm);
        if (wper < 0) return fail(ctx, GSNP_E_CUDA, "k_warp_sites: shared memory %zu B", wsm);
        ctx->begin();
        wk<<<(unsigned)(ctx->num_sms * std::max(wper, 1)), NT, wsm, s>>>(A, ctx->wlist.p, ctx->big_n.p + 2,
                                                                       ctx->wlist2.p, ctx->big_n.p + 4,
                                                                       ctx->big.p, ctx->big_n.p, big_cap);
        ctx->end(GSNP_STAGE_WARP);
        ctx->launches++;
        CK(cudaGetLastError());
        // sites beyond 1024 unique keys: one CTA each, shared buffer of up to ~200 KB
        const uint32_t cap = (uint32_t)((200 * 1024 - (size_t)8 * A.L) / 4);
        const size_t bsm = 4 * (size_t)cap + (size_t)8 * A.L;
        if (ctx->occupancy(reinterpret_cast<const void*>(k_big_sites), NT, bsm) < 0)
            return fail(ctx, GSNP_E_CUDA, "k_big_sites: shared memory %zu B", bsm);
        ctx->begin();
        k_big_sites<<<(unsigned)ctx->num_sms, NT, bsm, s>>>(A, ctx->big.p, ctx->big_n.p, cap);
        ctx->end(GSNP_STAGE_BIG);
        ctx->launches++;
        CK(cudaGetLastError());
    }
    return GSNP_OK;
}

// synchronise the stream, read and clear the device error flag (a clean flag for what follows,
// e.g. a run of gsnp_call_async windows)
gsnp_status read_err(gsnp_ctx* ctx) {
    int h = 0;
    gsnp_status pst = peek(ctx, 2, ctx->d_err.p, sizeof(int));
    if (pst) return pst;
    CK(cudaStreamSynchronize(ctx->stream));
    memcpy(&h, ctx->mbox + 2, sizeof(int));
    if (h) CK(cudaMemsetAsync(ctx->d_err.p, 0, sizeof(int), ctx->stream));
    ctx->flush();
    return map_err(ctx, h);
}

gsnp_status count_impl(gsnp_ctx* ctx, const gsnp_reads* reads) {
    DevReads d;
    gsnp_status st = stage_reads(ctx, reads, d);
    if (st) return st;
    cudaStream_t s = ctx->stream;
    CK(ctx->d_counts.ensure(64 * 256 * 16));
    CK(cudaMemsetAsync(ctx->d_counts.p, 0, 64 * 256 * 16 * 8, s));
    CK(cudaMemsetAsync(ctx->d_err.p, 0, sizeof(int), s));
    if ((st = launch_validate(ctx, d))) return st;
    if (d.n) {
        CalibArgs A;
        A.R = d;
        A.ref = ctx->ref_code;
        A.origin = ctx->origin;
        A.n_sites = ctx->n_sites;
        A.L = (int)ctx->prm.max_read_len;
        A.q_max = (int)ctx->prm.q_max;
        A.C = ctx->d_counts.p;
        A.err = ctx->d_err.p;
        A.tma_ok = ((reinterpret_cast<uintptr_t>(d.bases) | reinterpret_cast<uintptr_t>(d.quals)) & 15) == 0;
        // shared memory: u32 diagonal histogram [q][t][cycle] + two stages of (bases, quals,
        // reference window).  Cycles beyond Lh (only for long reads at high q_max) use global REDs.
        // budget: the opt-in maximum per CTA less the kernel's static shared memory (larger
        // batches amortise the per-batch barriers and metadata over more words per thread)
        size_t& budget = ctx->cal_budget;
        if (!budget) {
            int optin = 0;
            cudaFuncAttributes fa{};
            cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, ctx->prm.device);
            CK(cudaFuncGetAttributes(&fa, k_calib_count));
            budget = optin > (int)fa.sharedSizeBytes + 64 * 1024 ? (size_t)optin - fa.sharedSizeBytes - 256
                                                                 : 200 * 1024;
            if (const char* e = getenv("GSNP_CAL_BUDGET_KB")) budget = (size_t)atoi(e) * 1024;
        }
        A.RB = 8 * 1024;                               // reference window per stage
        A.SB = 32 * 1024;                              // bases (and quals) per stage
        const size_t per_cyc = (size_t)(A.q_max + 1) * 4 * 4;
        A.Lh = std::min<int>(A.L, (int)((budget - 2 * (2 * 4096 + A.RB) - 16) / per_cyc) & ~3);
        const size_t hist = align16(per_cyc * ((A.Lh + 3) / 4 * 4));
        while (A.SB > 4096 && hist + 2 * (2 * (size_t)A.SB + A.RB) + 16 > budget) A.SB -= 4096;
        A.CB = std::max(1, std::min<int>(std::min(CAL_MAXB, CAL_NT), (int)(A.SB - 32) / A.L));
        const size_t smem = hist + 2 * (2 * (size_t)A.SB + A.RB) + 16;
        unsigned grid = (unsigned)std::min<uint64_t>((uint64_t)ctx->num_sms, (d.n + A.CB - 1) / A.CB);
        grid = std::max(grid, 1u);
        CK(cudaFuncSetAttribute(k_calib_count, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        ctx->begin();
        k_calib_count<<<grid, CAL_NT, smem, s>>>(A);
        ctx->end(GSNP_STAGE_CALIB);
        ctx->launches++;
        CK(cudaGetLastError());
    }
    return GSNP_OK;
}

gsnp_status finalize_impl(gsnp_ctx* ctx, const uint64_t* counts_host) {
    auto t0 = std::chrono::steady_clock::now();
    const int L = (int)ctx->prm.max_read_len;
    const int qmax = (int)ctx->prm.q_max;
    if (ctx->h_counts.size() != (size_t)64 * 256 * 16) ctx->h_counts.assign((size_t)64 * 256 * 16, 0);
    if (ctx->h_p.size() != (size_t)64 * 256 * 16) ctx->h_p.assign((size_t)64 * 256 * 16, 0.0);
    const size_t tn = (size_t)64 * L * 4 * TROW;
    if (!ctx->h_T || ctx->h_T_n != tn) {
        if (ctx->h_T) cudaFreeHost(ctx->h_T);
        ctx->h_T = nullptr;
        CK(cudaMallocHost(&ctx->h_T, tn * sizeof(double)));
        ctx->h_T_n = tn;
        memset(ctx->h_T, 0, tn * sizeof(double));     // rows 0 and > q_max are never indexed
    }
    // p for every quality; T rows only for q_adj in [1, q_max] (adjust never leaves that range)
    const uint64_t* C = ctx->h_counts.data();
    double* p = ctx->h_p.data();
    double* T = ctx->h_T;
    const gsnp_params prm = ctx->prm;
    // two phases over all host threads: p rows per quality, then T rows per (quality, cycle
    // chunk) — the log10 calls of Alg. 2 dominate (built once on the CPU)
    const int CCH = 10;                                  // cycles per T work item
    const int nch = (L + CCH - 1) / CCH;
    const int nT = qmax * nch;
    std::atomic<int> next_p{0}, done_p{0}, next_t{0};
    auto work = [&]() {
        for (int q; (q = next_p.fetch_add(1)) < 64;) {
            // this quality's counts into the context's copy (rows copied in parallel)
            memcpy(ctx->h_counts.data() + ((size_t)q << 12), counts_host + ((size_t)q << 12), 4096 * 8);
            estimate_p_q(prm, C, p, q);
            done_p.fetch_add(1);
        }
        while (done_p.load() < 64) std::this_thread::yield();
        for (int it; (it = next_t.fetch_add(1)) < nT;) {
            const int q = 1 + it / nch, c0 = (it % nch) * CCH;
            build_T_q(L, p, T, q, c0, std::min(L, c0 + CCH));
        }
    };
    static const int nt_env = [] { const char* e = getenv("GSNP_HOST_THREADS"); return e ? atoi(e) : 0; }();
    const int nt = nt_env > 0 ? nt_env
                              : (int)std::max(1u, std::min(32u, std::thread::hardware_concurrency()));
    if (ctx->pool.th.empty() && nt > 1) ctx->pool.start(nt - 1);
    ctx->pool.run(work);
    CK(ctx->T.ensure(tn));
    if (!ctx->T_zeroed) {                                  // rows of q > q_max stay zero
        CK(cudaMemsetAsync(ctx->T.p, 0, tn * 8, ctx->stream));
        ctx->T_zeroed = true;
    }
    const size_t tq = (size_t)(qmax + 1) * L * 4 * TROW;  // rows q = 0..q_max (the built ones)
    // no host wait: the calls that read T are queued behind the copy on the same stream, and h_T is
    // rewritten only by the next finalize, after the next count's synchronising read-back
    CK(cudaMemcpyAsync(ctx->T.p, ctx->h_T, tq * 8, cudaMemcpyHostToDevice, ctx->stream));
    ctx->calibrated = true;
    if (ctx->timing()) {
        ctx->stage_ms[GSNP_STAGE_FINALIZE] +=
            std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
        ctx->stage_n[GSNP_STAGE_FINALIZE] += 1;
    }
    return GSNP_OK;
}

// §V-B output compression of device records d_rec[0, n) (format R17, kernels k_cz_*)
gsnp_status compress_impl(gsnp_ctx* ctx, const gsnp_record* d_rec, uint64_t n, uint32_t B,
                          uint32_t* out, uint64_t out_cap, uint64_t* n_words) {
    using namespace gsnp_cz;
    cudaStream_t s = ctx->stream;
    const uint64_t nblk = (n + B - 1) / B;
    if (nblk * NSEC > 0x7FFFFFFFull) return fail(ctx, GSNP_E_RANGE, "too many compression blocks");
    const uint32_t DC = std::min<uint32_t>(DICT_MAX, B);
    const uint64_t npad = (n + 15) & ~15ull;         // every column 16-byte aligned (vector loads)
    CK(ctx->cz_cols.ensure(32 * npad));
    CK(ctx->cz_meta.ensure(nblk * NSEC * 2));
    CK(ctx->cz_dD.ensure(nblk * NDICT));
    CK(ctx->cz_dict.ensure(nblk * NDICT * DC));
    CK(ctx->cz_off.ensure(nblk * NSEC + 1));
    if (!ctx->h_cz_total) CK(cudaMallocHost(&ctx->h_cz_total, 8));
    CzArgs A;
    memset(&A, 0, sizeof A);
    A.rec = d_rec;
    A.n = n;
    A.B = B;
    A.nblk = (uint32_t)nblk;
    A.DC = DC;
    uint8_t* base = ctx->cz_cols.p;                  // u32 columns, then u16, then u8
    for (int k = 0; k < 4; ++k) A.col.u32[k] = reinterpret_cast<uint32_t*>(base + (size_t)4 * npad * k);
    for (int k = 0; k < 4; ++k) A.col.u16[k] = reinterpret_cast<uint16_t*>(base + 16 * npad + (size_t)2 * npad * k);
    for (int k = 0; k < 8; ++k) A.col.u8[k] = base + 24 * npad + (size_t)npad * k;
    A.meta = ctx->cz_meta.p;
    A.dD = ctx->cz_dD.p;
    A.dict = ctx->cz_dict.p;
    A.off = ctx->cz_off.p;
    const size_t sm_size = SMEM_DSIZE_WORDS * 4, sm_write = SMEM_DWRITE_WORDS * 4;
    const size_t sm_light = SMEM_LIGHT_WORDS * 4;
    CK(cudaFuncSetAttribute(k_cz_dicts<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm_size));
    CK(cudaFuncSetAttribute(k_cz_dicts<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm_write));
    // sections [0, SEC_S): header, planes, exception lists (k_cz_sections, one CTA per block and
    // section); [SEC_S, NSEC): dictionary sections (k_cz_dicts, one CTA per block and dictionary)
    const int nlight = SEC_S;
    ctx->begin();
    const unsigned g0 = (unsigned)std::min<uint64_t>((n + 255) / 256, (uint64_t)ctx->num_sms * 8);
    k_cz_columns<<<g0, 256, 0, s>>>(d_rec, n, A.col);
    k_cz_sections<false><<<(unsigned)(nblk * nlight), gsnp_cz::NT, sm_light, s>>>(A, 0, nlight);
    k_cz_dicts<false><<<(unsigned)(nblk * NDICT), gsnp_cz::NT, sm_size, s>>>(A);
    k_cz_scan<<<1, 1024, 0, s>>>(A, ctx->cz_off.p);
    ctx->launches += 4;
    CK(cudaGetLastError());
    gsnp_status pst = peek(ctx, 3, ctx->cz_off.p + nblk * NSEC, 8);
    if (pst) return pst;
    CK(cudaStreamSynchronize(s));
    const uint64_t total = ctx->mbox[3];
    if (n_words) *n_words = total;
    if (total > out_cap) {
        ctx->end(GSNP_STAGE_COMPRESS);
        return fail(ctx, GSNP_E_CAPACITY, "compressed stream needs %llu words, out_cap %llu",
                    (unsigned long long)total, (unsigned long long)out_cap);
    }
    const bool dev_out = is_device_ptr(out);
    if (dev_out) {
        A.out = out;
    } else {
        CK(ctx->cz_out.ensure(total));
        A.out = ctx->cz_out.p;
    }
    k_cz_sections<true><<<(unsigned)(nblk * nlight), gsnp_cz::NT, sm_light, s>>>(A, 0, nlight);
    k_cz_dicts<true><<<(unsigned)(nblk * NDICT), gsnp_cz::NT, sm_write, s>>>(A);
    ctx->launches += 2;
    ctx->end(GSNP_STAGE_COMPRESS);
    CK(cudaGetLastError());
    if (!dev_out) {              // host output: the words must have landed when we return
        CK(cudaMemcpyAsync(out, A.out, total * 4, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        ctx->flush();
    }                            // device output: ordered on the caller's stream, no host wait
    return GSNP_OK;
}

}  // namespace

// ============================================================================ public ABI
extern "C" {

gsnp_status gsnp_params_default(gsnp_params* out) {
    if (!out) return GSNP_E_INVAL;
    memset(out, 0, sizeof *out);
    out->abi_version = GSNP_ABI_VERSION;
    out->max_read_len = 100;
    out->q_max = 40;
    out->calib_min_count = 10;
    out->het_novel = 1e-3;
    out->althom_novel = 5e-4;
    out->global_dep = 0.9;
    out->pcr_dep = 0.5;
    out->flags = GSNP_RANK_SUM;
    out->device = 0;
    out->stream = nullptr;
    return GSNP_OK;
}

gsnp_status gsnp_priors_from_freq(const double* freq, uint64_t n, double floor_prior,
                                  double* prior10) {
    static const int A1[10] = {0, 0, 0, 0, 1, 1, 1, 2, 2, 3};
    static const int A2[10] = {0, 1, 2, 3, 1, 2, 3, 2, 3, 3};
    if (n && (!freq || !prior10)) return GSNP_E_INVAL;
    if (!(floor_prior > 0)) return GSNP_E_INVAL;
    for (uint64_t i = 0; i < n; ++i) {
        const double* f = freq + 4 * i;
        const double tot = f[0] + f[1] + f[2] + f[3];
        if (!(tot > 0) || !(f[0] >= 0) || !(f[1] >= 0) || !(f[2] >= 0) || !(f[3] >= 0))
            return GSNP_E_RANGE;
        for (int k = 0; k < 10; ++k) {
            const double fa = f[A1[k]] / tot, fb = f[A2[k]] / tot;
            const double v = A1[k] == A2[k] ? fa * fa : 2.0 * fa * fb;
            prior10[10 * i + k] = v > floor_prior ? v : floor_prior;
        }
    }
    return GSNP_OK;
}

gsnp_status gsnp_create(const gsnp_reference* ref, const gsnp_priors* priors,
                        const gsnp_params* params, gsnp_ctx** out) {
    if (!out) return GSNP_E_INVAL;
    *out = nullptr;
    if (!ref || !ref->code || ref->n_sites == 0) return GSNP_E_INVAL;
    if (ref->n_sites >= (1ull << 32)) return GSNP_E_RANGE;   // per-context shard < 4 Gb
    gsnp_ctx* ctx = new (std::nothrow) gsnp_ctx();
    if (!ctx) return GSNP_E_NOMEM;
    gsnp_status st = check_params(ctx, params);
    if (st) { delete ctx; return st; }
    ctx->prm = *params;
    ctx->stream = (cudaStream_t)params->stream;
    auto bail = [&](gsnp_status s) { gsnp_destroy(ctx); return s; };
    if (cudaSetDevice(params->device) != cudaSuccess) { cudaGetLastError(); return bail(GSNP_E_CUDA); }
    {
        int sms = 0;
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, params->device);
        ctx->num_sms = sms > 0 ? sms : 148;
        if (const char* e = getenv("GSNP_MID_AT")) ctx->mid_at = (float)atof(e);
        if (const char* e = getenv("GSNP_LIST_MIN")) ctx->list_min = (uint32_t)strtoul(e, nullptr, 10);
        if (const char* e = getenv("GSNP_DEEP_AT")) ctx->deep_at = (float)atof(e);
        if (const char* e = getenv("GSNP_MID_ADJ_SMEM")) ctx->mid_adj_smem = atoi(e) != 0;
    }
    ctx->n_sites = ref->n_sites;
    ctx->origin = ref->origin;
    for (uint64_t i = 0; i < ref->n_sites; ++i)
        if (ref->code[i] > 4) return bail(GSNP_E_RANGE);
    // known SNPs: sorted positions, log10 prior rows (C6), site bitmap
    uint64_t nk = priors ? priors->n : 0;
    std::vector<double> lp(std::max<uint64_t>(nk, 1) * 10);
    std::vector<uint8_t> code(ref->code, ref->code + ref->n_sites);
    ctx->h_known_pos.assign(nk, 0);
    for (uint64_t k = 0; k < nk; ++k) {
        uint64_t p = priors->pos[k];
        if (k && p <= priors->pos[k - 1]) return bail(GSNP_E_UNSORTED);
        if (p < ref->origin || p >= ref->origin + ref->n_sites) return bail(GSNP_E_RANGE);
        for (int n = 0; n < 10; ++n) {
            double v = priors->prior10[k * 10 + n];
            if (!(v > 0)) return bail(GSNP_E_RANGE);
            lp[k * 10 + n] = log10(v);
        }
        code[p - ref->origin] |= 8u;                     // known-SNP flag rides on the code
        ctx->h_known_pos[k] = p;
    }
    ctx->n_known = nk;
    // novel log10 priors per reference code (R6); ref N: flat
    double LP[50];
    static const int A1[10] = {0, 0, 0, 0, 1, 1, 1, 2, 2, 3};
    static const int A2[10] = {0, 1, 2, 3, 1, 2, 3, 2, 3, 3};
    // R18 variants: ti/tv 2:1 weights of the alternative alleles; monoploid zeroes het priors
    const bool mono = (params->flags & GSNP_MONOPLOID) != 0, titv = (params->flags & GSNP_TITV) != 0;
    auto wt = [&](int r, int x) { return !titv ? 1.0 : (r ^ x) == 3 ? 2.0 : 0.5; };
    for (int r = 0; r < 5; ++r)
        for (int n = 0; n < 10; ++n) {
            double v;
            if (mono && A1[n] != A2[n]) { LP[r * 10 + n] = log10(0.0); continue; }
            if (r == 4) { LP[r * 10 + n] = kLog10Zero; continue; }
            if (A1[n] == r && A2[n] == r) v = 1.0;
            else if (A1[n] == r) v = params->het_novel * wt(r, A2[n]);
            else if (A2[n] == r) v = params->het_novel * wt(r, A1[n]);
            else if (A1[n] == A2[n]) v = params->althom_novel * wt(r, A1[n]);
            else v = params->het_novel * params->althom_novel * wt(r, A1[n]) * wt(r, A2[n]);
            LP[r * 10 + n] = log10(v);
        }
    if (mono)
        for (uint64_t k = 0; k < nk; ++k)
            for (int n = 0; n < 10; ++n)
                if (A1[n] != A2[n]) lp[k * 10 + n] = log10(0.0);
    if ((st = build_adj(ctx))) return bail(st);
    gsnp_ctx* c = ctx;
#define CKC(x) do { if ((x) != cudaSuccess) { cudaGetLastError(); return bail(fail(c, GSNP_E_CUDA, "%s", #x)); } } while (0)
    // padded with N on both sides: 16-byte TMA reference windows may reach past either end
    CKC(ctx->ref.ensure(ref->n_sites + 2 * REF_PAD));
    CKC(cudaMemset(ctx->ref.p, 4, ref->n_sites + 2 * REF_PAD));
    CKC(cudaMemcpy(ctx->ref.p + REF_PAD, code.data(), ref->n_sites, cudaMemcpyHostToDevice));
    ctx->ref_code = ctx->ref.p + REF_PAD;
    CKC(ctx->known_pos.ensure(std::max<uint64_t>(nk, 1)));
    if (nk) CKC(cudaMemcpy(ctx->known_pos.p, ctx->h_known_pos.data(), nk * 8, cudaMemcpyHostToDevice));
    CKC(ctx->known_lp.ensure(lp.size()));
    CKC(cudaMemcpy(ctx->known_lp.p, lp.data(), lp.size() * 8, cudaMemcpyHostToDevice));
    CKC(ctx->LP.ensure(50));
    CKC(cudaMemcpy(ctx->LP.p, LP, sizeof LP, cudaMemcpyHostToDevice));
    CKC(ctx->adj.ensure(ctx->h_adj.size()));
    CKC(cudaMemcpy(ctx->adj.p, ctx->h_adj.data(), ctx->h_adj.size(), cudaMemcpyHostToDevice));
    if (params->flags & GSNP_RANK_EXACT) {
        std::vector<double> F;
        build_rank_cdf(F);
        CKC(ctx->rank_cdf.ensure(F.size()));
        CKC(cudaMemcpy(ctx->rank_cdf.p, F.data(), F.size() * 8, cudaMemcpyHostToDevice));
    }
    CKC(ctx->d_err.ensure(1));
#undef CKC
    *out = ctx;
    return GSNP_OK;
}

gsnp_status gsnp_calibrate_count(gsnp_ctx* ctx, const gsnp_reads* reads, uint64_t* counts) {
    if (!ctx || !counts) return GSNP_E_INVAL;
    if (cudaSetDevice(ctx->prm.device) != cudaSuccess) return fail(ctx, GSNP_E_CUDA, "set device");
    gsnp_status st = count_impl(ctx, reads);
    if (st) return st;
    if ((st = read_err(ctx))) return st;
    cudaMemcpyKind kind = is_device_ptr(counts) ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost;
    CK(cudaMemcpyAsync(counts, ctx->d_counts.p, 64 * 256 * 16 * 8, kind, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    return GSNP_OK;
}

gsnp_status gsnp_calibrate_finalize(gsnp_ctx* ctx, const uint64_t* counts) {
    if (!ctx || !counts) return GSNP_E_INVAL;
    if (cudaSetDevice(ctx->prm.device) != cudaSuccess) return fail(ctx, GSNP_E_CUDA, "set device");
    if (is_device_ptr(counts)) {
        if (!ctx->h_cnt_pinned) {
            CK(cudaMallocHost(&ctx->h_cnt_pinned, 64 * 256 * 16 * 8));
            memset(ctx->h_cnt_pinned, 0, 64 * 256 * 16 * 8);
        }
        // only the cells a count can reach (q <= q_max, cycle < max_read_len): k_calib_count rejects
        // the other qualities and never forms a later cycle, so the rest stays zero
        CK(cudaMemcpy2DAsync(ctx->h_cnt_pinned, 4096 * 8, counts, 4096 * 8,
                             (size_t)ctx->prm.max_read_len * 16 * 8, (size_t)ctx->prm.q_max + 1,
                             cudaMemcpyDeviceToHost, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        return finalize_impl(ctx, ctx->h_cnt_pinned);
    }
    return finalize_impl(ctx, counts);
}

gsnp_status gsnp_calibrate(gsnp_ctx* ctx, const gsnp_reads* reads) {
    if (!ctx) return GSNP_E_INVAL;
    if (cudaSetDevice(ctx->prm.device) != cudaSuccess) return fail(ctx, GSNP_E_CUDA, "set device");
    gsnp_status st = count_impl(ctx, reads);
    if (st) return st;
    if ((st = read_err(ctx))) return st;
    std::vector<uint64_t> h(64 * 256 * 16);
    CK(cudaMemcpyAsync(h.data(), ctx->d_counts.p, h.size() * 8, cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    return finalize_impl(ctx, h.data());
}

static gsnp_status check_window(gsnp_ctx* ctx, const gsnp_reads* reads, uint64_t w0, uint64_t w1) {
    if (!ctx->calibrated) return fail(ctx, GSNP_E_STATE, "gsnp_call before calibration");
    if (!reads) return fail(ctx, GSNP_E_INVAL, "reads == NULL");
    if (w1 < w0 || w0 < ctx->origin || w1 > ctx->origin + ctx->n_sites)
        return fail(ctx, GSNP_E_RANGE, "window outside the reference");
    return GSNP_OK;
}

gsnp_status gsnp_call(gsnp_ctx* ctx, const gsnp_reads* reads, uint64_t w0, uint64_t w1,
                      gsnp_record* out, uint64_t out_cap, uint64_t* n_out) {
    if (!ctx) return GSNP_E_INVAL;
    if (cudaSetDevice(ctx->prm.device) != cudaSuccess) return fail(ctx, GSNP_E_CUDA, "set device");
    gsnp_status st = check_window(ctx, reads, w0, w1);
    if (st) return st;
    const uint64_t S = w1 - w0;
    if (n_out) *n_out = S;
    if (out_cap < S) return fail(ctx, GSNP_E_CAPACITY, "out_cap %llu < %llu", (unsigned long long)out_cap,
                                 (unsigned long long)S);
    if (S && !out) return fail(ctx, GSNP_E_INVAL, "out == NULL");
    if (S == 0) return GSNP_OK;
    DevReads d;
    if ((st = stage_reads(ctx, reads, d))) return st;
    CK(cudaMemsetAsync(ctx->d_err.p, 0, sizeof(int), ctx->stream));
    const bool dev_out = is_device_ptr(out);
    gsnp_record* d_out = out;
    if (!dev_out) {
        CK(ctx->rec.ensure(S));
        d_out = ctx->rec.p;
    }
    CallArgs A;
    memset(&A, 0, sizeof A);
    if ((st = run_window(ctx, d, w0, w1, d_out, A))) return st;
    if ((st = read_err(ctx))) return st;           // on an error the records were not written
    if (!dev_out) {
        CK(cudaMemcpyAsync(out, d_out, S * sizeof(gsnp_record), cudaMemcpyDeviceToHost, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
    }
    return GSNP_OK;
}

gsnp_status gsnp_call_async(gsnp_ctx* ctx, const gsnp_reads* reads, uint64_t w0, uint64_t w1,
                            gsnp_record* out, uint64_t out_cap) {
    if (!ctx) return GSNP_E_INVAL;
    if (cudaSetDevice(ctx->prm.device) != cudaSuccess) return fail(ctx, GSNP_E_CUDA, "set device");
    gsnp_status st = check_window(ctx, reads, w0, w1);
    if (st) return st;
    const uint64_t S = w1 - w0;
    if (out_cap < S) return fail(ctx, GSNP_E_CAPACITY, "out_cap %llu < %llu", (unsigned long long)out_cap,
                                 (unsigned long long)S);
    if (S == 0) return GSNP_OK;
    if (!out || !is_device_ptr(out)) return fail(ctx, GSNP_E_INVAL, "gsnp_call_async: out must be device memory");
    if (reads->n_reads && !reads->on_device)
        return fail(ctx, GSNP_E_INVAL, "gsnp_call_async: reads must be device arrays");
    DevReads d;
    if ((st = stage_reads(ctx, reads, d))) return st;
    CallArgs A;
    memset(&A, 0, sizeof A);
    return run_window(ctx, d, w0, w1, out, A);
}

gsnp_status gsnp_wait(gsnp_ctx* ctx) {
    if (!ctx) return GSNP_E_INVAL;
    if (cudaSetDevice(ctx->prm.device) != cudaSuccess) return fail(ctx, GSNP_E_CUDA, "set device");
    return read_err(ctx);
}

gsnp_status gsnp_call_dense(gsnp_ctx* ctx, const gsnp_reads* reads, uint64_t w0, uint64_t w1,
                            uint32_t chunk_sites, gsnp_record* out, uint64_t out_cap,
                            uint64_t* n_out) {
    if (!ctx) return GSNP_E_INVAL;
    if (cudaSetDevice(ctx->prm.device) != cudaSuccess) return fail(ctx, GSNP_E_CUDA, "set device");
    gsnp_status st = check_window(ctx, reads, w0, w1);
    if (st) return st;
    if (chunk_sites < 32 || chunk_sites % 32 || chunk_sites > (1u << 20))
        return fail(ctx, GSNP_E_INVAL, "chunk_sites must be a multiple of 32 in [32, 2^20]");
    const uint64_t S = w1 - w0;
    if (n_out) *n_out = S;
    if (out_cap < S) return fail(ctx, GSNP_E_CAPACITY, "out_cap %llu < %llu", (unsigned long long)out_cap,
                                 (unsigned long long)S);
    if (S && !out) return fail(ctx, GSNP_E_INVAL, "out == NULL");
    if (S == 0) return GSNP_OK;
    cudaStream_t s = ctx->stream;
    DevReads d;
    if ((st = stage_reads(ctx, reads, d))) return st;
    CK(cudaMemsetAsync(ctx->d_err.p, 0, sizeof(int), s));
    const bool dev_out = is_device_ptr(out);
    gsnp_record* d_out = out;
    if (!dev_out) {
        CK(ctx->rec.ensure(S));
        d_out = ctx->rec.p;
    }
    DenseArgs D;
    memset(&D, 0, sizeof D);
    if ((st = prep_window(ctx, d, w0, w1, d_out, D.A))) return st;
    const uint64_t chunk = std::min<uint64_t>(chunk_sites, S);
    const bool fresh = ctx->dense_occ.n < chunk * DENSE_SITE_BYTES;
    CK(ctx->dense_occ.ensure(chunk * DENSE_SITE_BYTES));
    CK(ctx->dense_cnt.ensure(chunk * 5));
    if (fresh) CK(cudaMemsetAsync(ctx->dense_occ.p, 0, chunk * DENSE_SITE_BYTES, s));
    D.occ = ctx->dense_occ.p;
    D.cnt = ctx->dense_cnt.p;
    for (uint64_t c0 = w0; c0 < w1; c0 += chunk) {
        D.c0 = c0;
        D.c1 = std::min(w1, c0 + chunk);
        const uint64_t n = D.c1 - D.c0;
        CK(cudaMemsetAsync(D.cnt, 0, n * 5 * 4, s));
        if (d.n) {
            ctx->begin();
            k_dense_count<<<(unsigned)(ctx->num_sms * 8), DENSE_NT, 0, s>>>(D);
            ctx->end(GSNP_STAGE_DENSE_COUNT);
            ctx->launches++;
            CK(cudaGetLastError());
        }
        ctx->begin();
        k_dense_sites<<<(unsigned)std::min<uint64_t>((n + 7) / 8, (uint64_t)ctx->num_sms * 8), DENSE_NT, 0, s>>>(D);
        ctx->end(GSNP_STAGE_DENSE_LIK);
        ctx->launches++;
        CK(cudaGetLastError());
        ctx->begin();                       // recycle: re-zero the whole dense array
        CK(cudaMemsetAsync(D.occ, 0, n * DENSE_SITE_BYTES, s));
        ctx->end(GSNP_STAGE_DENSE_RECYCLE);
    }
    st = read_err(ctx);
    if (st == GSNP_E_CAPACITY)              // a saturated cell leaves residue behind: start clean
        cudaMemsetAsync(ctx->dense_occ.p, 0, ctx->dense_occ.n, s);
    if (st) return st;                      // on an error the records were not all written
    if (!dev_out) {
        CK(cudaMemcpyAsync(out, d_out, S * sizeof(gsnp_record), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
    }
    return GSNP_OK;
}

gsnp_status gsnp_parse_soap(gsnp_ctx* ctx, const char* text, uint64_t n_bytes, const char* chr_name,
                            uint32_t q_offset, uint64_t loc_base, uint64_t* pos, uint16_t* len,
                            uint64_t* off, uint8_t* bases, uint8_t* quals, uint8_t* strand,
                            uint16_t* hits, uint64_t reads_cap, uint64_t bases_cap,
                            uint64_t* n_reads, uint64_t* n_bases) {
    if (!ctx) return GSNP_E_INVAL;
    if (n_reads) *n_reads = 0;
    if (n_bases) *n_bases = 0;
    if (cudaSetDevice(ctx->prm.device) != cudaSuccess) return fail(ctx, GSNP_E_CUDA, "set device");
    if (n_bytes && !text) return fail(ctx, GSNP_E_INVAL, "text == NULL");
    if (q_offset > 255) return fail(ctx, GSNP_E_INVAL, "q_offset > 255");
    const size_t chr_len = chr_name ? strlen(chr_name) : 0;
    if (chr_len > 4096) return fail(ctx, GSNP_E_INVAL, "chr_name longer than 4096");
    cudaStream_t s = ctx->stream;
    // the text on the device, 16-byte aligned (host text or an unaligned device pointer: copied)
    const uint8_t* t = reinterpret_cast<const uint8_t*>(text);
    const bool dev_text = is_device_ptr(text);
    if (!dev_text || (reinterpret_cast<uintptr_t>(text) & 15)) {
        CK(ctx->p_text.ensure(n_bytes + 16));
        CK(cudaMemcpyAsync(ctx->p_text.p, text, n_bytes, dev_text ? cudaMemcpyDeviceToDevice
                                                                    : cudaMemcpyHostToDevice, s));
        t = ctx->p_text.p;
    }
    uint8_t last = '\n';
    if (n_bytes) {
        if (dev_text) CK(cudaMemcpyAsync(&last, t + n_bytes - 1, 1, cudaMemcpyDeviceToHost, s));
        else last = (uint8_t)text[n_bytes - 1];
    }
    CK(ctx->p_chr.ensure(chr_len + 1));
    if (chr_len) CK(cudaMemcpyAsync(ctx->p_chr.p, chr_name, chr_len, cudaMemcpyHostToDevice, s));
    CK(ctx->p_scal.ensure(8));
    CK(cudaMemsetAsync(ctx->d_err.p, 0, sizeof(int), s));
    CK(cudaMemsetAsync(ctx->p_scal.p, 0xFF, 8, s));                 // bad_line = max
    // newlines: per-tile counts -> scan -> line starts
    const uint64_t n_tiles = (n_bytes + PTILE - 1) / PTILE;
    CK(ctx->p_cnt.ensure(n_tiles + 1));
    uint64_t n_nl = 0;
    if (n_tiles) {
        ctx->begin();
        k_nl_tiles<false><<<(unsigned)n_tiles, PNT, 0, s>>>(t, n_bytes, ctx->p_cnt.p, nullptr);
        k_scan_partials<<<1, PNT, 0, s>>>(ctx->p_cnt.p, n_tiles);
        ctx->end(GSNP_STAGE_PARSE);
        ctx->launches += 2;
        CK(cudaGetLastError());
        CK(cudaMemcpyAsync(&n_nl, ctx->p_cnt.p + n_tiles, 8, cudaMemcpyDeviceToHost, s));
    }
    CK(cudaStreamSynchronize(s));
    const uint64_t n_lines = n_nl + ((n_bytes && last != '\n') ? 1 : 0);
    CK(ctx->p_ls.ensure(n_nl + 2));
    uint64_t ls_end = n_bytes + 1;                                    // end of an unterminated line
    if (n_tiles) {
        ctx->begin();
        k_nl_tiles<true><<<(unsigned)n_tiles, PNT, 0, s>>>(t, n_bytes, ctx->p_cnt.p, ctx->p_ls.p);
        ctx->end(GSNP_STAGE_PARSE);
        ctx->launches++;
        CK(cudaGetLastError());
    }
    if (n_lines > n_nl) CK(cudaMemcpyAsync(ctx->p_ls.p + n_lines, &ls_end, 8, cudaMemcpyHostToDevice, s));
    uint64_t tot[2] = {0, 0};
    ParseArgs P;
    memset(&P, 0, sizeof P);
    P.text = t; P.n_bytes = n_bytes; P.n_lines = n_lines; P.ls = ctx->p_ls.p;
    P.chr = ctx->p_chr.p; P.chr_len = (uint32_t)chr_len; P.q_offset = q_offset; P.loc_base = loc_base;
    P.err = ctx->d_err.p; P.bad_line = reinterpret_cast<unsigned long long*>(ctx->p_scal.p);
    const uint64_t n_sel_tiles = (n_lines + SEL_TILE - 1) / SEL_TILE;
    if (n_lines) {
        CK(ctx->p_meta.ensure(n_lines));
        CK(ctx->p_pos.ensure(n_lines));
        CK(ctx->p_ridx.ensure(n_lines));
        CK(ctx->p_boff.ensure(n_lines));
        CK(ctx->p_part.ensure(2 * (n_sel_tiles + 1)));
        P.meta = ctx->p_meta.p; P.pos = ctx->p_pos.p; P.ridx = ctx->p_ridx.p; P.boff = ctx->p_boff.p;
        const unsigned wgrid = (unsigned)std::min<uint64_t>((n_lines + PGROUPS - 1) / PGROUPS,
                                                            (uint64_t)ctx->num_sms * 8);
        uint64_t* part_n = ctx->p_part.p;
        uint64_t* part_b = ctx->p_part.p + n_sel_tiles + 1;
        ctx->begin();
        k_parse_meta<<<wgrid, PNT, 0, s>>>(P);
        k_sel_tiles<<<(unsigned)n_sel_tiles, PNT, 0, s>>>(P.meta, n_lines, part_n, part_b);
        k_scan_partials<<<1, PNT, 0, s>>>(part_n, n_sel_tiles);
        k_scan_partials<<<1, PNT, 0, s>>>(part_b, n_sel_tiles);
        ctx->end(GSNP_STAGE_PARSE);
        ctx->launches += 4;
        CK(cudaGetLastError());
        CK(cudaMemcpyAsync(&tot[0], part_n + n_sel_tiles, 8, cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(&tot[1], part_b + n_sel_tiles, 8, cudaMemcpyDeviceToHost, s));
    }
    int herr = 0;
    unsigned long long bad = 0;
    CK(cudaMemcpyAsync(&herr, ctx->d_err.p, sizeof(int), cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(&bad, ctx->p_scal.p, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    ctx->flush();
    if (herr) return fail(ctx, GSNP_E_RANGE, "malformed SOAP alignment line %llu (0-based)", bad);
    if (n_reads) *n_reads = tot[0];
    if (n_bases) *n_bases = tot[1];
    if (reads_cap < tot[0] || bases_cap < tot[1])
        return fail(ctx, GSNP_E_CAPACITY, "need %llu reads / %llu bases", (unsigned long long)tot[0],
                    (unsigned long long)tot[1]);
    if (!pos && !len && !off && !bases && !quals && !strand && !hits && tot[0] == 0)
        return GSNP_OK;                                               // size query of an empty parse
    if (!pos || !len || !off || !bases || !quals || !strand || !hits)
        return fail(ctx, GSNP_E_INVAL, "NULL output array");
    // outputs: device arrays written in place, host arrays through the staging buffers
    const bool dev_out = is_device_ptr(pos);
    P.o_pos = pos; P.o_len = len; P.o_off = off; P.o_bases = bases; P.o_quals = quals;
    P.o_strand = strand; P.o_hits = hits;
    if (!dev_out) {
        CK(ctx->r_pos.ensure(tot[0] + 1)); CK(ctx->r_off.ensure(tot[0] + 1));
        CK(ctx->r_len.ensure(tot[0] + 1)); CK(ctx->r_hits.ensure(tot[0] + 1));
        CK(ctx->r_strand.ensure(tot[0] + 1));
        CK(ctx->r_bases.ensure(tot[1] + 1)); CK(ctx->r_quals.ensure(tot[1] + 1));
        P.o_pos = ctx->r_pos.p; P.o_len = ctx->r_len.p; P.o_off = ctx->r_off.p;
        P.o_bases = ctx->r_bases.p; P.o_quals = ctx->r_quals.p; P.o_strand = ctx->r_strand.p;
        P.o_hits = ctx->r_hits.p;
    }
    if (tot[0] == 0) {
        const uint64_t z = 0;
        CK(cudaMemcpyAsync(P.o_off, &z, 8, cudaMemcpyHostToDevice, s));
        CK(cudaStreamSynchronize(s));
    } else {
        const uint64_t* part_n = ctx->p_part.p;
        const uint64_t* part_b = ctx->p_part.p + n_sel_tiles + 1;
        ctx->begin();
        k_sel_apply<<<(unsigned)n_sel_tiles, PNT, 0, s>>>(P, part_n, part_b);
        k_parse_emit<<<(unsigned)std::min<uint64_t>((n_lines + PGROUPS - 1) / PGROUPS, (uint64_t)ctx->num_sms * 8), PNT, 0, s>>>(
            P, tot[0], tot[1]);
        ctx->end(GSNP_STAGE_PARSE);
        ctx->launches += 2;
        CK(cudaGetLastError());
        CK(cudaMemcpyAsync(&herr, ctx->d_err.p, sizeof(int), cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(&bad, ctx->p_scal.p, 8, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        ctx->flush();
        if (herr) return fail(ctx, GSNP_E_RANGE, "bad base or quality character on line %llu", bad);
    }
    if (!dev_out) {
        const uint64_t nr = tot[0], nb = tot[1];
        CK(cudaMemcpyAsync(pos, P.o_pos, nr * 8, cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(len, P.o_len, nr * 2, cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(off, P.o_off, (nr + 1) * 8, cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(strand, P.o_strand, nr, cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(hits, P.o_hits, nr * 2, cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(bases, P.o_bases, nb, cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(quals, P.o_quals, nb, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
    }
    return GSNP_OK;
}

gsnp_status gsnp_pack_reads(const gsnp_reads* reads, const gsnp_reference* ref, uint32_t block_reads,
                            void* out, uint64_t cap, uint64_t* n_bytes) {
    using namespace gsnp_pk;
    if (n_bytes) *n_bytes = 0;
    if (!reads || reads->on_device) return GSNP_E_INVAL;
    if (block_reads < 1 || block_reads > MAX_BLOCK) return GSNP_E_INVAL;
    const uint64_t n = reads->n_reads;
    if (n && (!reads->pos || !reads->len || !reads->off || !reads->bases || !reads->quals ||
              !reads->strand || !reads->hits)) return GSNP_E_INVAL;
    if (ref && (!ref->code || ref->n_sites == 0)) return GSNP_E_INVAL;
    HostReads R{ref ? ref->code : nullptr, ref ? ref->origin : 0, ref ? ref->n_sites : 0,
                n, reads->pos, reads->len, reads->off, reads->bases, reads->quals, reads->strand,
                reads->hits};
    const uint32_t version = ref ? 2u : 1u;
    const uint64_t nblk = (n + block_reads - 1) / block_reads;
    std::vector<BlockSize> bs(nblk);
    const int nt = (int)std::max(1u, std::min(32u, std::thread::hardware_concurrency()));
    auto par = [&](auto&& fn) {                  // fn(block) over all blocks on nt threads
        std::atomic<uint64_t> next{0};
        auto work = [&] { for (uint64_t b; (b = next.fetch_add(1)) < nblk;) fn(b); };
        std::vector<std::thread> th;
        for (int i = 1; i < nt && (uint64_t)i < nblk; ++i) th.emplace_back(work);
        work();
        for (auto& t : th) t.join();
    };
    par([&](uint64_t b) {
        bs[b] = size_block(R, b * block_reads, std::min(n, (b + 1) * block_reads));
    });
    std::vector<uint64_t> table(5 * nblk);
    Header h{};
    for (uint64_t b = 0; b < nblk; ++b) {
        if (bs[b].bad) return GSNP_E_RANGE;
        uint64_t* t = table.data() + 5 * b;
        t[0] = R.pos[b * block_reads];
        t[1] = h.n_bases; t[2] = h.n_runs; t[3] = h.n_nexc; t[4] = h.n_hexc;
        h.n_bases += bs[b].bases; h.n_runs += bs[b].runs; h.n_nexc += bs[b].nexc; h.n_hexc += bs[b].hexc;
    }
    h.n_reads = n;
    h.n_blocks = (uint32_t)nblk;
    h.block_reads = block_reads;
    h.sec[0] = HDR;
    h.sec[1] = a16(h.sec[0] + 40 * nblk);
    meta_offsets(h);
    h.sec[2] = a16(h.m_nrun + n);
    h.version = version;
    h.sec[3] = a16(h.sec[2] + (version == 1 ? (h.n_bases + 3) / 4 : 0));
    h.sec[4] = a16(h.sec[3] + 2 * h.n_runs);
    h.sec[5] = a16(h.sec[4] + 4 * h.n_nexc);
    const uint64_t total = a16(h.sec[5] + 8 * h.n_hexc);
    if (n_bytes) *n_bytes = total;
    if (!out || cap < total) return GSNP_E_CAPACITY;
    uint8_t* o = static_cast<uint8_t*>(out);
    memset(o, 0, HDR);
    const uint32_t magic = MAGIC, ver = version;
    memcpy(o, &magic, 4); memcpy(o + 4, &ver, 4);
    memcpy(o + 8, &h.n_reads, 8); memcpy(o + 16, &h.n_bases, 8); memcpy(o + 24, &h.n_runs, 8);
    memcpy(o + 32, &h.n_nexc, 8); memcpy(o + 40, &h.n_hexc, 8); memcpy(o + 48, &h.n_blocks, 4);
    memcpy(o + 52, &h.block_reads, 4); memcpy(o + 56, h.sec, 48);
    // zero every padding gap and the 2-bit plane (edge bytes are OR-ed by neighbouring blocks)
    auto zero = [&](uint64_t a, uint64_t b) { if (b > a) memset(o + a, 0, b - a); };
    zero(h.sec[0] + 40 * nblk, h.sec[1]);
    zero(h.m_pos + 4 * n, h.m_len); zero(h.m_len + n, h.m_sh); zero(h.m_sh + n, h.m_nrun);
    zero(h.m_nrun + n, h.sec[2]);
    zero(h.sec[2], h.sec[3]);
    zero(h.sec[3] + 2 * h.n_runs, h.sec[4]); zero(h.sec[4] + 4 * h.n_nexc, h.sec[5]);
    zero(h.sec[5] + 8 * h.n_hexc, total);
    if (nblk) memcpy(o + h.sec[0], table.data(), 40 * nblk);
    par([&](uint64_t b) {
        write_block(R, b * block_reads, std::min(n, (b + 1) * block_reads), h, table.data() + 5 * b, o);
    });
    return GSNP_OK;
}

gsnp_status gsnp_packed_sizes(const void* packed, uint64_t n_bytes, uint64_t* n_reads,
                              uint64_t* n_bases) {
    gsnp_pk::Header h;
    if (!packed || !gsnp_pk::parse_header(static_cast<const uint8_t*>(packed), n_bytes, h))
        return GSNP_E_INVAL;
    if (n_reads) *n_reads = h.n_reads;
    if (n_bases) *n_bases = h.n_bases;
    return GSNP_OK;
}

gsnp_status gsnp_unpack_reads(gsnp_ctx* ctx, const void* packed, uint64_t n_bytes, uint64_t* pos,
                              uint16_t* len, uint64_t* off, uint8_t* bases, uint8_t* quals,
                              uint8_t* strand, uint16_t* hits) {
    using namespace gsnp_pk;
    if (!ctx) return GSNP_E_INVAL;
    if (cudaSetDevice(ctx->prm.device) != cudaSuccess) return fail(ctx, GSNP_E_CUDA, "set device");
    if (!packed) return fail(ctx, GSNP_E_INVAL, "packed == NULL");
    cudaStream_t s = ctx->stream;
    const uint8_t* pk = static_cast<const uint8_t*>(packed);
    const bool dev_in = is_device_ptr(packed);
    Header h;
    uint8_t hb[HDR];
    if (n_bytes < HDR) return fail(ctx, GSNP_E_INVAL, "packed stream shorter than its header");
    if (dev_in) {
        CK(cudaMemcpyAsync(hb, pk, HDR, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
    } else {
        memcpy(hb, pk, HDR);
    }
    if (!parse_header(hb, n_bytes, h)) return fail(ctx, GSNP_E_INVAL, "not a GSR1 packed-read stream");
    if (!off || (h.n_reads && (!pos || !len || !strand || !hits)) || (h.n_bases && (!bases || !quals)))
        return fail(ctx, GSNP_E_INVAL, "NULL output array");
    if (!is_device_ptr(off) || (h.n_reads && !is_device_ptr(pos)) || (h.n_bases && !is_device_ptr(bases)))
        return fail(ctx, GSNP_E_INVAL, "outputs must be device arrays");
    UnpackArgs U;
    memset(&U, 0, sizeof U);
    U.h = h;
    U.ref = ctx->ref_code;
    U.origin = ctx->origin;
    U.n_sites = ctx->n_sites;
    U.pos = pos; U.len = len; U.off = off; U.bases = bases; U.quals = quals; U.strand = strand;
    U.hits = hits;
    if (h.n_reads == 0) {
        CK(cudaMemsetAsync(off, 0, 8, s));
        CK(cudaStreamSynchronize(s));
        return GSNP_OK;
    }
    if (dev_in && (reinterpret_cast<uintptr_t>(pk) & 15) == 0) {
        U.buf = pk;                                  // in place: one launch over every block
        ctx->begin();
        k_unpack<<<h.n_blocks, UNT, 0, s>>>(U);
        ctx->end(GSNP_STAGE_UNPACK);
        ctx->launches++;
        CK(cudaGetLastError());
        return GSNP_OK;
    }
    CK(ctx->pk_buf.ensure(n_bytes));
    U.buf = ctx->pk_buf.p;
    if (dev_in) {                                    // unaligned device stream: one D2D copy
        CK(cudaMemcpyAsync(ctx->pk_buf.p, pk, n_bytes, cudaMemcpyDeviceToDevice, s));
        ctx->begin();
        k_unpack<<<h.n_blocks, UNT, 0, s>>>(U);
        ctx->end(GSNP_STAGE_UNPACK);
        ctx->launches++;
        CK(cudaGetLastError());
        return GSNP_OK;
    }
    // host stream: the header and block table first, then chunks of blocks — each chunk's slices
    // of every section on the copy stream, its decode on the library stream once they landed
    if (!ctx->copy_stream) CK(cudaStreamCreateWithFlags(&ctx->copy_stream, cudaStreamNonBlocking));
    cudaStream_t cs = ctx->copy_stream;
    const uint64_t* bt = reinterpret_cast<const uint64_t*>(pk + h.sec[0]);
    const uint32_t K = (uint32_t)std::min<uint64_t>(h.n_blocks, 8);
    while (ctx->pk_ev.size() < K + 1) {
        cudaEvent_t e;
        CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        ctx->pk_ev.push_back(e);
    }
    CK(cudaEventRecord(ctx->pk_ev[K], s));           // the buffer is free once earlier work is done
    CK(cudaStreamWaitEvent(cs, ctx->pk_ev[K], 0));
    CK(cudaMemcpyAsync(ctx->pk_buf.p, pk, h.sec[1], cudaMemcpyHostToDevice, cs));
    auto cp = [&](uint64_t a, uint64_t b) -> cudaError_t {
        return b > a ? cudaMemcpyAsync(ctx->pk_buf.p + a, pk + a, b - a, cudaMemcpyHostToDevice, cs)
                     : cudaSuccess;
    };
    auto brow = [&](uint32_t b, int f) -> uint64_t {  // block b's counter f (b == n_blocks: totals)
        if (b < h.n_blocks) return bt[5ull * b + f];
        const uint64_t tot[5] = {0, h.n_bases, h.n_runs, h.n_nexc, h.n_hexc};
        return tot[f];
    };
    for (uint32_t k = 0; k < K; ++k) {
        const uint32_t b0 = (uint32_t)((uint64_t)h.n_blocks * k / K);
        const uint32_t b1 = (uint32_t)((uint64_t)h.n_blocks * (k + 1) / K);
        const uint64_t r0 = (uint64_t)b0 * h.block_reads, r1 = std::min(h.n_reads, (uint64_t)b1 * h.block_reads);
        CK(cp(h.m_pos + 4 * r0, h.m_pos + 4 * r1));
        CK(cp(h.m_len + r0, h.m_len + r1));
        CK(cp(h.m_sh + r0, h.m_sh + r1));
        CK(cp(h.m_nrun + r0, h.m_nrun + r1));
        if (h.version == 1) CK(cp(h.sec[2] + brow(b0, 1) / 4, h.sec[2] + (brow(b1, 1) + 3) / 4));
        CK(cp(h.sec[3] + 2 * brow(b0, 2), h.sec[3] + 2 * brow(b1, 2)));
        CK(cp(h.sec[4] + 4 * brow(b0, 3), h.sec[4] + 4 * brow(b1, 3)));
        CK(cp(h.sec[5] + 8 * brow(b0, 4), h.sec[5] + 8 * brow(b1, 4)));
        CK(cudaEventRecord(ctx->pk_ev[k], cs));
        CK(cudaStreamWaitEvent(s, ctx->pk_ev[k], 0));
        U.blk0 = b0;
        ctx->begin();
        k_unpack<<<b1 - b0, UNT, 0, s>>>(U);
        ctx->end(GSNP_STAGE_UNPACK);
        ctx->launches++;
        CK(cudaGetLastError());
    }
    CK(cudaStreamSynchronize(cs));                   // the host stream may be reused on return
    return GSNP_OK;
}

gsnp_status gsnp_compress(gsnp_ctx* ctx, const gsnp_record* rec, uint64_t n, uint32_t block_sites,
                          uint32_t* out, uint64_t out_cap, uint64_t* n_words) {
    if (!ctx) return GSNP_E_INVAL;
    if (n_words) *n_words = 0;
    if (cudaSetDevice(ctx->prm.device) != cudaSuccess) return fail(ctx, GSNP_E_CUDA, "set device");
    if (block_sites < 1 || block_sites > (1u << 24)) return fail(ctx, GSNP_E_INVAL, "block_sites");
    if (n == 0) return GSNP_OK;
    if (!rec) return fail(ctx, GSNP_E_INVAL, "rec == NULL");
    if (out_cap && !out) return fail(ctx, GSNP_E_INVAL, "out == NULL");
    const gsnp_record* d_rec = rec;
    if (!is_device_ptr(rec)) {
        CK(ctx->cz_rec.ensure(n));
        CK(cudaMemcpyAsync(ctx->cz_rec.p, rec, n * sizeof(gsnp_record), cudaMemcpyHostToDevice,
                           ctx->stream));
        d_rec = ctx->cz_rec.p;
    }
    return compress_impl(ctx, d_rec, n, block_sites, out, out_cap, n_words);
}

gsnp_status gsnp_call_compressed(gsnp_ctx* ctx, const gsnp_reads* reads, uint64_t w0, uint64_t w1,
                                 uint32_t block_sites, uint32_t* out, uint64_t out_cap,
                                 uint64_t* n_words) {
    if (!ctx) return GSNP_E_INVAL;
    if (n_words) *n_words = 0;
    if (cudaSetDevice(ctx->prm.device) != cudaSuccess) return fail(ctx, GSNP_E_CUDA, "set device");
    if (block_sites < 1 || block_sites > (1u << 24)) return fail(ctx, GSNP_E_INVAL, "block_sites");
    if (out_cap && !out) return fail(ctx, GSNP_E_INVAL, "out == NULL");
    if (w1 < w0) return fail(ctx, GSNP_E_RANGE, "window outside the reference");
    const uint64_t S = w1 - w0;
    if (S == 0) return check_window(ctx, reads, w0, w1);
    CK(ctx->rec.ensure(S));
    uint64_t nrec = 0;
    gsnp_status st = gsnp_call(ctx, reads, w0, w1, ctx->rec.p, S, &nrec);
    if (st) return st;
    return compress_impl(ctx, ctx->rec.p, S, block_sites, out, out_cap, n_words);
}

gsnp_status gsnp_debug_window(gsnp_ctx* ctx, const gsnp_reads* reads, uint64_t w0, uint64_t w1,
                              uint32_t* off, uint32_t* keys_built, uint32_t* keys_sorted,
                              uint32_t* site_counters, double* L10, double* post10,
                              gsnp_record* records) {
    if (!ctx) return GSNP_E_INVAL;
    if (cudaSetDevice(ctx->prm.device) != cudaSuccess) return fail(ctx, GSNP_E_CUDA, "set device");
    gsnp_status st = check_window(ctx, reads, w0, w1);
    if (st) return st;
    const uint64_t S = w1 - w0;
    if (S == 0) return GSNP_OK;
    cudaStream_t s = ctx->stream;
    DevReads d;
    if ((st = stage_reads(ctx, reads, d))) return st;
    CK(cudaMemsetAsync(ctx->d_err.p, 0, sizeof(int), s));
    // pass 1: unique keys per site -> CSR offsets (host scan)
    CK(ctx->dbg_u32a.ensure(S));
    CK(ctx->rec.ensure(S));
    CallArgs A;
    memset(&A, 0, sizeof A);
    A.count_only = 1;
    A.dbg_nuni = ctx->dbg_u32a.p;
    if ((st = run_window(ctx, d, w0, w1, ctx->rec.p, A))) return st;
    std::vector<uint32_t> nuni(S), hoff(S + 1);
    CK(cudaMemcpyAsync(nuni.data(), ctx->dbg_u32a.p, S * 4, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if ((st = read_err(ctx))) return st;
    hoff[0] = 0;
    for (uint64_t i = 0; i < S; ++i) hoff[i + 1] = hoff[i] + nuni[i];
    const uint64_t K = hoff[S];
    CK(ctx->dbg_u32b.ensure(S + 1));
    CK(ctx->dbg_u32c.ensure(std::max<uint64_t>(K, 1)));
    CK(ctx->dbg_u32d.ensure(std::max<uint64_t>(K, 1)));
    CK(ctx->dbg_u32e.ensure(S * 15));
    CK(ctx->dbg_f64a.ensure(S * 10));
    CK(ctx->dbg_f64b.ensure(S * 10));
    CK(cudaMemcpyAsync(ctx->dbg_u32b.p, hoff.data(), (S + 1) * 4, cudaMemcpyHostToDevice, s));
    memset(&A, 0, sizeof A);
    A.dbg_off = ctx->dbg_u32b.p;
    A.dbg_keys_built = ctx->dbg_u32c.p;
    A.dbg_keys_sorted = ctx->dbg_u32d.p;
    A.dbg_counters = ctx->dbg_u32e.p;
    A.dbg_L10 = ctx->dbg_f64a.p;
    A.dbg_post10 = ctx->dbg_f64b.p;
    if ((st = run_window(ctx, d, w0, w1, ctx->rec.p, A))) return st;
    if ((st = read_err(ctx))) return st;
    if (off) memcpy(off, hoff.data(), (S + 1) * 4);
    if (keys_built && K) CK(cudaMemcpyAsync(keys_built, ctx->dbg_u32c.p, K * 4, cudaMemcpyDeviceToHost, s));
    if (keys_sorted && K) CK(cudaMemcpyAsync(keys_sorted, ctx->dbg_u32d.p, K * 4, cudaMemcpyDeviceToHost, s));
    if (site_counters) CK(cudaMemcpyAsync(site_counters, ctx->dbg_u32e.p, S * 60, cudaMemcpyDeviceToHost, s));
    if (L10) CK(cudaMemcpyAsync(L10, ctx->dbg_f64a.p, S * 80, cudaMemcpyDeviceToHost, s));
    if (post10) CK(cudaMemcpyAsync(post10, ctx->dbg_f64b.p, S * 80, cudaMemcpyDeviceToHost, s));
    if (records) CK(cudaMemcpyAsync(records, ctx->rec.p, S * sizeof(gsnp_record), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    return GSNP_OK;
}

gsnp_status gsnp_get_tables(gsnp_ctx* ctx, uint64_t* counts, double* p_matrix, double* T,
                            uint8_t* adj, uint32_t* dims) {
    if (!ctx) return GSNP_E_INVAL;
    if (dims) {
        dims[0] = ctx->prm.max_read_len;
        dims[1] = (uint32_t)ctx->adjP;
        dims[2] = (uint32_t)ctx->adjG;
    }
    if (adj) memcpy(adj, ctx->h_adj.data(), ctx->h_adj.size());
    if ((counts || p_matrix || T) && !ctx->calibrated) return fail(ctx, GSNP_E_STATE, "not calibrated");
    if (counts) memcpy(counts, ctx->h_counts.data(), ctx->h_counts.size() * 8);
    if (p_matrix) memcpy(p_matrix, ctx->h_p.data(), ctx->h_p.size() * 8);
    if (T) {                                        // unpadded [64][L][4][10] view
        const size_t rows = ctx->h_T_n / TROW;
        for (size_t r = 0; r < rows; ++r) memcpy(T + r * 10, ctx->h_T + r * TROW, 10 * 8);
    }
    return GSNP_OK;
}

uint64_t gsnp_launch_count(const gsnp_ctx* ctx) { return ctx ? ctx->launches : 0; }

gsnp_status gsnp_stage_times(gsnp_ctx* ctx, double* ms, uint64_t* launches, int n_stages,
                             int reset) {
    if (!ctx || n_stages < 0) return GSNP_E_INVAL;
    ctx->flush();
    for (int i = 0; i < n_stages && i < GSNP_N_STAGES; ++i) {
        if (ms) ms[i] = ctx->stage_ms[i];
        if (launches) launches[i] = ctx->stage_n[i];
    }
    if (reset)
        for (int i = 0; i < GSNP_N_STAGES; ++i) { ctx->stage_ms[i] = 0; ctx->stage_n[i] = 0; }
    return GSNP_OK;
}

const char* gsnp_strerror(gsnp_status s) {
    switch (s) {
        case GSNP_OK: return "ok";
        case GSNP_E_INVAL: return "invalid argument";
        case GSNP_E_RANGE: return "value out of range";
        case GSNP_E_UNSORTED: return "reads not sorted by position";
        case GSNP_E_STATE: return "call order violated";
        case GSNP_E_NOMEM: return "out of memory";
        case GSNP_E_CUDA: return "CUDA error";
        case GSNP_E_CAPACITY: return "capacity exceeded";
        default: return "unknown status";
    }
}

const char* gsnp_last_error(const gsnp_ctx* ctx) { return ctx ? ctx->err.c_str() : ""; }

void gsnp_destroy(gsnp_ctx* ctx) {
    if (!ctx) return;
    cudaSetDevice(ctx->prm.device);
    ctx->ref.release(); ctx->known_pos.release(); ctx->known_lp.release();
    ctx->adj.release(); ctx->LP.release(); ctx->rank_cdf.release(); ctx->T.release(); ctx->d_err.release();
    ctx->d_counts.release(); ctx->tile_ra.release(); ctx->tile_rb.release(); ctx->rec.release();
    ctx->big.release(); ctx->big_n.release(); ctx->wlist.release(); ctx->wlist2.release();
    ctx->dense_occ.release(); ctx->dense_cnt.release();
    ctx->p_text.release(); ctx->p_chr.release(); ctx->p_cnt.release(); ctx->p_ls.release();
    ctx->p_meta.release(); ctx->p_pos.release(); ctx->p_ridx.release(); ctx->p_boff.release();
    ctx->p_part.release(); ctx->p_scal.release();
    ctx->r_pos.release(); ctx->r_off.release(); ctx->r_len.release(); ctx->r_hits.release();
    ctx->r_bases.release(); ctx->r_quals.release(); ctx->r_strand.release();
    ctx->dbg_u32a.release(); ctx->dbg_u32b.release(); ctx->dbg_u32c.release();
    ctx->dbg_u32d.release(); ctx->dbg_u32e.release(); ctx->dbg_f64a.release(); ctx->dbg_f64b.release();
    ctx->cz_cols.release(); ctx->cz_meta.release(); ctx->cz_dD.release(); ctx->cz_dict.release();
    ctx->cz_out.release(); ctx->cz_off.release(); ctx->cz_rec.release();
    if (ctx->h_cz_total) cudaFreeHost(ctx->h_cz_total);
    if (ctx->mbox) cudaFreeHost(ctx->mbox);
    if (ctx->h_T) cudaFreeHost(ctx->h_T);
    if (ctx->h_cnt_pinned) cudaFreeHost(ctx->h_cnt_pinned);
    ctx->pk_buf.release();
    for (auto e : ctx->pk_ev) cudaEventDestroy(e);
    if (ctx->copy_stream) cudaStreamDestroy(ctx->copy_stream);
    for (auto& p : ctx->pending) { cudaEventDestroy(p.a); cudaEventDestroy(p.b); }
    for (auto e : ctx->ev_pool) cudaEventDestroy(e);
    delete ctx;
}

}  // extern "C"
