// gsnp_deep.cu — the deep-window instantiation of k_call_tile (COLS_DEEP = 128 key slots per
// thread, chosen for windows with >= 48 reads per site, e.g. C5's 100X exome-like target) built
// with 384-thread CTAs.  Its key columns take COLS_DEEP x NT x 4 bytes of shared memory, so only
// one CTA fits per SM either way: 12 warps at NT = 384 instead of 8 at 256 — the row gathers of
// deep sites are latency-bound and the extra warps hide more of it (C5: 46.7 -> 33.2 ms per three
// calls, tools/nt_ab.sh).  Same device source as gsnp_kernels.cuh, compiled in its own namespace;
// the shallow kernel keeps 256-thread CTAs (three per SM).
#include <cstring>

#ifndef GSNP_DEEP_NT
#define GSNP_DEEP_NT 384
#endif
#define GSNP_NT GSNP_DEEP_NT
#define GSNP_CALL_MINB 1
#define gsnp_dev gsnp_dev384
#include "gsnp_kernels.cuh"
#undef gsnp_dev

namespace gsnp_deep {

// Launch k_call_tile<DBG, COLS_DEEP> with NT = 384 on stream s.  args: the caller's CallArgs
// (identical layout in both namespaces: same header); returns the CUDA status of the launch.
cudaError_t launch_call_tile_deep(const void* args, size_t args_size, bool dbg, int num_sms,
                                  size_t adj_bytes, uint32_t adj_smem, uint32_t* wlist,
                                  uint32_t* wlist_n, uint32_t* work, cudaStream_t s) {
    using namespace gsnp_dev384;
    static_assert(sizeof(CallArgs) > 0, "");
    if (args_size != sizeof(CallArgs)) return cudaErrorInvalidValue;
    CallArgs A;
    memcpy(&A, args, sizeof A);
    size_t smem = call_smem_bytes(A.L, adj_smem ? adj_bytes : 0, COLS_DEEP, nullptr, nullptr, false);
    if (adj_smem && smem > 227 * 1024) {     // no room for the adjust table: read it from global
        adj_smem = 0;
        smem = call_smem_bytes(A.L, 0, COLS_DEEP, nullptr, nullptr, false);
    }
    auto kern = dbg ? k_call_tile<true, COLS_DEEP> : k_call_tile<false, COLS_DEEP>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    int per_sm = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, NT, smem);
    if (e != cudaSuccess) return e;
    const uint64_t n_tiles = (A.w1 - A.w0 + TS - 1) / TS;
    const uint64_t want = (uint64_t)num_sms * (per_sm > 0 ? per_sm : 1);
    const unsigned grid = (unsigned)(want < n_tiles ? want : (n_tiles ? n_tiles : 1));
    kern<<<grid, NT, smem, s>>>(A, wlist, wlist_n, work, adj_smem);
    return cudaGetLastError();
}

}  // namespace gsnp_deep
