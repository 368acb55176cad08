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
// reads whose bytes the gather keeps in flight: a deep window has ~L reads per 32-site group
// start, and this kernel has the registers (one CTA per SM) to hide more of their latency
#ifndef GSNP_DEEP_GB
#define GSNP_DEEP_GB 4
#endif
#define GSNP_GB GSNP_DEEP_GB
#define GSNP_CALL_MINB 1
#define gsnp_dev gsnp_dev384
#include "gsnp_kernels.cuh"
#undef gsnp_dev

namespace gsnp_deep {

// The k_call_tile<DBG, COLS_DEEP> instantiation with NT = 384, for the caller to launch through
// cudaLaunchKernel (CallArgs has the same layout in both namespaces: same header).
const void* call_tile_kernel(bool dbg) {
    using namespace gsnp_dev384;
    return dbg ? reinterpret_cast<const void*>(k_call_tile<true, COLS_DEEP>)
               : reinterpret_cast<const void*>(k_call_tile<false, COLS_DEEP>);
}
int call_tile_nt() { return gsnp_dev384::NT; }
// dynamic shared memory of the deep kernel; clears *adj_smem when the adjust table does not fit
size_t call_tile_smem(int L, size_t adj_bytes, uint32_t* adj_smem) {
    using namespace gsnp_dev384;
    size_t smem = call_smem_bytes(L, *adj_smem ? adj_bytes : 0, COLS_DEEP, nullptr, nullptr, false);
    if (*adj_smem && smem > 227 * 1024) {    // no room for the adjust table: read it from global
        *adj_smem = 0;
        smem = call_smem_bytes(L, 0, COLS_DEEP, nullptr, nullptr, false);
    }
    return smem;
}

}  // namespace gsnp_deep
