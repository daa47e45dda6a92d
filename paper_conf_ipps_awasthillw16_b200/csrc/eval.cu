// eval.cu -- batched sequence evaluation (cdd_eval_batch / ucddcp_eval_batch).
//
// The paper's fitness kernel runs the sequential O(n) walk in one thread per sequence with alpha,
// beta staged in shared memory.  Here a group of G lanes evaluates one sequence:
// the instance's packed records are staged in shared memory once per CTA, each lane loads a
// contiguous chunk of E job ids with vector loads, gathers the records, and the group runs the
// scan/ballot evaluator of device_common.cuh.  Persistent grid: #SM x resident CTAs.
#include <cuda_runtime.h>

#include "device_common.cuh"
#include "internal.h"

namespace cdd {
namespace {

constexpr int kEvalThreads = 256;

template <int E, bool VEC>
__device__ __forceinline__ void load_ids(const int16_t* __restrict__ row, int l, int n,
                                         int16_t (&ids)[E]) {
    const int k0 = l * E;
    if constexpr (VEC && E >= 8) {
#pragma unroll
        for (int v = 0; v < E / 8; ++v) {
            int4 x = make_int4(0, 0, 0, 0);
            if (k0 + 8 * v < n) x = __ldg(reinterpret_cast<const int4*>(row + k0 + 8 * v));
            const int16_t* h = reinterpret_cast<const int16_t*>(&x);
#pragma unroll
            for (int j = 0; j < 8; ++j) ids[8 * v + j] = h[j];
        }
    } else if constexpr (VEC && E == 4) {
        int2 x = make_int2(0, 0);
        if (k0 < n) x = __ldg(reinterpret_cast<const int2*>(row + k0));
        const int16_t* h = reinterpret_cast<const int16_t*>(&x);
#pragma unroll
        for (int j = 0; j < 4; ++j) ids[j] = h[j];
    } else {
#pragma unroll
        for (int j = 0; j < E; ++j) ids[j] = (k0 + j < n) ? __ldg(row + k0 + j) : (int16_t)0;
    }
}

template <int G, int E, bool UCD, bool VEC>
__global__ void __launch_bounds__(kEvalThreads) eval_batch_kernel(
    const uint32_t* __restrict__ table, int n, int32_t d, RecLayout L,
    const int16_t* __restrict__ perms, int64_t ld, int64_t batch, int64_t* __restrict__ out,
    int* __restrict__ err) {
    extern __shared__ uint32_t s_tab[];
    for (int i = threadIdx.x; i < n; i += blockDim.x) s_tab[i] = table[i];
    __syncthreads();

    const int lane = threadIdx.x & 31;
    const int l = lane % G;
    const int gbase = lane - l;
    constexpr int kGroupsPerWarp = 32 / G;
    const int warp = threadIdx.x >> 5;
    const int64_t warps_total = (int64_t)gridDim.x * (kEvalThreads / 32);
    const int64_t stride = warps_total * kGroupsPerWarp;

    for (int64_t row0 = ((int64_t)blockIdx.x * (kEvalThreads / 32) + warp) * kGroupsPerWarp;
         row0 < batch; row0 += stride) {  // warp-uniform trip count
        const int64_t row = row0 + lane / G;
        const bool rv = row < batch;
        const int16_t* rp = perms + (rv ? row : 0) * ld;
        int16_t ids[E];
        load_ids<E, VEC>(rp, rv ? l : 31, rv ? n : 0, ids);
        uint32_t rec[E];
        bool bad = false;
#pragma unroll
        for (int i = 0; i < E; ++i) {
            const int k = l * E + i;
            const uint32_t id = (uint32_t)(uint16_t)ids[i];
            const bool in = rv && k < n;
            bad |= in && id >= (uint32_t)n;
            rec[i] = (in && id < (uint32_t)n) ? s_tab[id] : 0u;
        }
        if (bad) atomicOr(err, 1);
        auto elem = [&](int k) -> uint32_t {
            const uint32_t id = (uint32_t)(uint16_t)__ldg(rp + k);
            return (rv && id < (uint32_t)n) ? s_tab[id] : 0u;
        };
        int32_t Z;
        if constexpr (UCD)
            Z = eval_ucddcp<G, E>(rec, l, gbase, n, L, elem);
        else
            Z = eval_cdd<G, E>(rec, l, gbase, n, d, L, elem);
        if (rv && l == 0) out[row] = (int64_t)Z;
    }
}

template <int G, int E, bool UCD>
cudaError_t launch_ge(const Instance& I, const int16_t* perms, int64_t ld, int64_t batch,
                      int64_t* out, cudaStream_t s) {
    const bool vec = (ld % 8 == 0) && ((reinterpret_cast<uintptr_t>(perms) & 15) == 0);
    const size_t smem = sizeof(uint32_t) * (size_t)I.n;
    const uint32_t* tab = UCD ? I.rec_ucd : I.rec_cdd;
    const RecLayout& L = UCD ? I.lay_ucd : I.lay_cdd;
    int dev_sms = 0, occ = 0;
    cudaError_t e = cudaDeviceGetAttribute(&dev_sms, cudaDevAttrMultiProcessorCount, I.device);
    if (e != cudaSuccess) return e;
    auto kern = vec ? eval_batch_kernel<G, E, UCD, true> : eval_batch_kernel<G, E, UCD, false>;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kEvalThreads, smem);
    if (e != cudaSuccess) return e;
    const int64_t rows_per_block = (kEvalThreads / 32) * (32 / G);
    int64_t blocks = (batch + rows_per_block - 1) / rows_per_block;
    const int64_t cap = (int64_t)dev_sms * (occ > 0 ? occ : 1);
    if (blocks > cap) blocks = cap;
    if (blocks < 1) blocks = 1;
    kern<<<(unsigned)blocks, kEvalThreads, smem, s>>>(tab, I.n, I.d_eff, L, perms, ld, batch, out,
                                                      I.err);
    return cudaGetLastError();
}

template <bool UCD>
cudaError_t dispatch(const Instance& I, const int16_t* perms, int64_t ld, int64_t batch,
                     int64_t* out, cudaStream_t s) {
    const int n = I.n;
    if (n <= 16) return launch_ge<4, 4, UCD>(I, perms, ld, batch, out, s);
    if (n <= 32) return launch_ge<8, 4, UCD>(I, perms, ld, batch, out, s);
    if (n <= 64) return launch_ge<8, 8, UCD>(I, perms, ld, batch, out, s);
    if (n <= 128) return launch_ge<16, 8, UCD>(I, perms, ld, batch, out, s);
    if (n <= 256) return launch_ge<32, 8, UCD>(I, perms, ld, batch, out, s);
    if (n <= 512) return launch_ge<32, 16, UCD>(I, perms, ld, batch, out, s);
    return launch_ge<32, 32, UCD>(I, perms, ld, batch, out, s);
}

}  // namespace

cudaError_t launch_eval_batch(const Instance& I, bool ucd, const int16_t* perms, int64_t ld,
                              int64_t batch, int64_t* out, cudaStream_t s) {
    if (batch <= 0) return cudaSuccess;
    return ucd ? dispatch<true>(I, perms, ld, batch, out, s)
               : dispatch<false>(I, perms, ld, batch, out, s);
}

}  // namespace cdd
