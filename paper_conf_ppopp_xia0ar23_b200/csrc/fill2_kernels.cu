// Host-side dispatch of the fill2 traversal kernels over the CTA size (per-NT translation units
// fill2_nt*.cu instantiate the kernels of fill2_impl.cuh).
#include "internal.h"

#include <cstdlib>
#include <map>
#include <mutex>
#include <tuple>

namespace lusym {

// header | visited words held in shared memory (smem_words, whole swizzle groups) | level-1
// summary (one bit per visited word, all n) | two frontier queues of q entries
size_t fill2_smem_bytes(int n, int smem_words, int q)
{
    const size_t words = (size_t)((n + 31) / 32);
    size_t b = kHdrBytes + 2 * (size_t)q * sizeof(int32_t);
    b += (words + 31) / 32 * sizeof(uint32_t);
    b += (size_t)smem_words * sizeof(uint32_t);
    return (b + 15) & ~(size_t)15;
}

namespace {
__global__ void k_smem_base(unsigned *out)
{
    extern __shared__ __align__(16) unsigned char smem[];
    if (threadIdx.x == 0) *out = (unsigned)__cvta_generic_to_shared(smem);
}
}  // namespace

// The shared-memory fill2 variants address their visited words at the constant offset
// 0x400 + kHdrBytes (fill2_impl.cuh kDynSmemBase): probe where a kernel's dynamic shared
// memory actually starts on this device (once per device); false sends the planner to the
// kVisGlobal variants, which take every shared address from the runtime window.
bool fill2_smem_base_ok(int dev)
{
    static int cached[64];
    static bool init[64];
    if (dev < 0 || dev >= 64) return false;
    if (getenv("LUSYM_ASSUME_SMEM_BASE_MISMATCH")) return false;  // test knob
    if (init[dev]) return cached[dev] != 0;
    unsigned *d = nullptr, h = 0;
    bool ok = false;
    if (cudaMalloc(&d, sizeof(unsigned)) == cudaSuccess) {
        k_smem_base<<<1, 32, 16384>>>(d);
        if (cudaMemcpy(&h, d, sizeof(unsigned), cudaMemcpyDeviceToHost) == cudaSuccess)
            ok = h == 0x400u;
        cudaFree(d);
    }
    cudaGetLastError();
    cached[dev] = ok;
    init[dev] = true;
    return ok;
}

#define LUSYM_NT_SWITCH(FN, ...)                                                             \
    switch (nt) {                                                                            \
    case 64: return FN<64>(__VA_ARGS__);                                                     \
    case 128: return FN<128>(__VA_ARGS__);                                                   \
    case 256: return FN<256>(__VA_ARGS__);                                                   \
    case 512: return FN<512>(__VA_ARGS__);                                                   \
    case 1024: return FN<1024>(__VA_ARGS__);                                                 \
    case 1025: return FN<1025>(__VA_ARGS__);                                                 \
    default: return cudaErrorInvalidValue;                                                   \
    }

namespace {
cudaError_t configure_impl(int nt, int w, int vis, size_t smem)
{
    LUSYM_NT_SWITCH(fill2_configure_nt, w, vis, smem)
}
cudaError_t occupancy_impl(int nt, int w, int vis, size_t smem, int *occ)
{
    LUSYM_NT_SWITCH(fill2_occupancy_nt, w, vis, smem, occ)
}
// the planner queries many (CTA size, W, visited mode, shared bytes) combinations per handle:
// set each kernel's attribute and compute each occupancy once per device and process
std::mutex g_mu;
std::map<std::tuple<int, int, int, int, size_t>, int> g_occ;
std::map<std::tuple<int, int, int, int>, size_t> g_conf;
int cur_dev()
{
    int d = 0;
    cudaGetDevice(&d);
    return d;
}
}  // namespace

cudaError_t fill2_configure(int nt, int w, int vis, size_t smem)
{
    const auto key = std::make_tuple(cur_dev(), nt, w, vis);
    std::lock_guard<std::mutex> lock(g_mu);
    auto it = g_conf.find(key);
    if (it != g_conf.end() && it->second >= smem) return cudaSuccess;
    cudaError_t e = configure_impl(nt, w, vis, smem);
    if (e == cudaSuccess) g_conf[key] = smem;
    return e;
}

cudaError_t fill2_occupancy(int nt, int w, int vis, size_t smem, int *occ)
{
    const auto key = std::make_tuple(cur_dev(), nt, w, vis, smem);
    std::lock_guard<std::mutex> lock(g_mu);
    auto it = g_occ.find(key);
    if (it != g_occ.end()) {
        *occ = it->second;
        return cudaSuccess;
    }
    cudaError_t e = occupancy_impl(nt, w, vis, smem, occ);
    if (e == cudaSuccess) g_occ[key] = *occ;
    return e;
}

cudaError_t fill2_launch(const Fill2Params &p, int nt, int w, int mode, int vis, int grid,
                         size_t smem, cudaStream_t s)
{
    LUSYM_NT_SWITCH(fill2_launch_nt, p, w, mode, vis, grid, smem, s)
}

}  // namespace lusym
