// eval.cu -- batched sequence evaluation (cdd_eval_batch / ucddcp_eval_batch).
//
// The paper's fitness kernel runs the sequential O(n) walk in one thread per sequence with alpha,
// beta staged in shared memory.  Here a group of G lanes evaluates one sequence:
// the instance's packed records are staged in shared memory once per CTA (a power-of-two table,
// zero records past n, aligned so that a gather address is one OR), each lane loads a contiguous
// chunk of E job ids with 16-byte loads (the next row's ids are prefetched while the current row
// is evaluated), gathers the records with masked indices (no bounds branches; ids >= n are
// detected with a 16x2 SIMD max and raise the data-error flag), and the group runs the
// scan/ballot evaluator of device_common.cuh.  Persistent grid: #SM x resident CTAs.
#include <cuda_runtime.h>

#include "device_common.cuh"
#include "internal.h"

namespace cdd {
namespace {

constexpr int kEvalThreads = 256;
constexpr int kGatherCopies = 8;  // bank-partitioned table copies (see eval_batch_kernel)

__device__ __forceinline__ uint32_t lds32(uint32_t addr) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr));
    return v;
}

// The lane's E ids as E/2 packed words (two int16 per word).  Vectors starting at or past n (and
// rows past the batch, signalled by n = 0) are not read and hold `s2` (two sentinel ids that index
// zero records).  vmax accumulates the ids of fully valid vectors; a vector straddling n (only
// when n % 8 != 0) is checked and patched element by element.
template <int E, bool VEC>
__device__ __forceinline__ void load_words(const int16_t* __restrict__ row, int k0, int n,
                                           uint32_t s2, uint32_t (&w)[E / 2], uint32_t& vmax,
                                           bool& bad) {
    if constexpr (VEC && E >= 8) {
#pragma unroll
        for (int v = 0; v < E / 8; ++v) {
            const int p0 = k0 + 8 * v;
            uint4 x = make_uint4(s2, s2, s2, s2);
            if (p0 < n) {
                x = __ldg(reinterpret_cast<const uint4*>(row + p0));
                if (p0 + 8 > n) {
                    uint32_t xs[4] = {x.x, x.y, x.z, x.w};
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        uint32_t lo = xs[j] & 0xffffu, hi = xs[j] >> 16;
                        if (p0 + 2 * j < n) bad |= lo >= (uint32_t)n; else lo = s2 & 0xffffu;
                        if (p0 + 2 * j + 1 < n) bad |= hi >= (uint32_t)n; else hi = s2 & 0xffffu;
                        xs[j] = lo | (hi << 16);
                    }
                    x = make_uint4(xs[0], xs[1], xs[2], xs[3]);
                }
            }
            w[4 * v] = x.x; w[4 * v + 1] = x.y; w[4 * v + 2] = x.z; w[4 * v + 3] = x.w;
        }
    } else {
#pragma unroll
        for (int j = 0; j < E / 2; ++j) {
            uint32_t lo = s2 & 0xffffu, hi = s2 & 0xffffu;
            if (k0 + 2 * j < n) {
                lo = (uint32_t)(uint16_t)__ldg(row + k0 + 2 * j);
                bad |= lo >= (uint32_t)n;
            }
            if (k0 + 2 * j + 1 < n) {
                hi = (uint32_t)(uint16_t)__ldg(row + k0 + 2 * j + 1);
                bad |= hi >= (uint32_t)n;
            }
            w[j] = lo | (hi << 16);
        }
    }
}

#ifndef CDD_EVAL_MIN_BLOCKS
#define CDD_EVAL_MIN_BLOCKS 2
#endif
template <int G, int E, bool UCD, bool VEC>
__global__ void __launch_bounds__(kEvalThreads, CDD_EVAL_MIN_BLOCKS) eval_batch_kernel(
    const uint32_t* __restrict__ table, int n, int npow2, int32_t d, RecLayout L,
    const int16_t* __restrict__ perms, int64_t ld, int64_t batch, int64_t* __restrict__ out,
    int* __restrict__ err) {
    extern __shared__ __align__(16) uint32_t s_raw[];
    // KC bank-partitioned copies of the table: record id, copy c at word id*KC + c, so lane L
    // (copy L % KC) only ever touches banks == L (mod KC) and competes with 32/KC lanes instead
    // of 32 for the random gather.  The table is aligned to its size, so an address is
    // ((id << log2(4*KC)) & mask) | (base | 4c).
    constexpr int KC = kGatherCopies;
    const uint32_t raw = (uint32_t)__cvta_generic_to_shared(s_raw);
    const uint32_t tbytes = (uint32_t)npow2 * 4u * KC;
    const uint32_t tab = (raw + tbytes - 1u) & ~(tbytes - 1u);
    uint32_t* s_tab = s_raw + (tab - raw) / 4u;
    for (int i = threadIdx.x; i < npow2 * KC; i += blockDim.x) {
        const int id = i / KC;
        s_tab[i] = id < n ? table[id] : 0u;
    }
    __syncthreads();
    const uint32_t amask = tbytes - 4u * KC;
    const uint32_t s2 = (uint32_t)n * 0x10001u;  // table[n] is a zero record (npow2 > n)

    const int lane = threadIdx.x & 31;
    const uint32_t tabc = tab | (uint32_t)((lane % KC) * 4);
    constexpr int SH = KC == 16 ? 6 : (KC == 8 ? 5 : 2);  // log2(4*KC)
    const int l = lane % G;
    const int gbase = lane - l;
    constexpr int kGroupsPerWarp = 32 / G;
    constexpr int NW = E / 2;
    const int warp = threadIdx.x >> 5;
    const int64_t warps_total = (int64_t)gridDim.x * (kEvalThreads / 32);
    const int64_t stride = warps_total * kGroupsPerWarp;
    const int k0 = l * E;
    uint32_t vmax = 0;
    bool bad = false;

    int64_t row0 = ((int64_t)blockIdx.x * (kEvalThreads / 32) + warp) * kGroupsPerWarp;
    uint32_t wn[NW];
    {
        const int64_t row = row0 + lane / G;
        const bool rv = row < batch;
        load_words<E, VEC>(perms + (rv ? row : 0) * ld, k0, rv ? n : 0, s2, wn, vmax, bad);
    }
    for (; row0 < batch; row0 += stride) {  // warp-uniform trip count
        const int64_t row = row0 + lane / G;
        const bool rv = row < batch;
        const int16_t* rp = perms + (rv ? row : 0) * ld;
        uint32_t w[NW];
#pragma unroll
        for (int j = 0; j < NW; ++j) w[j] = wn[j];
        {  // prefetch the next row of this group
            const int64_t nrow = row + stride;
            const bool nv = nrow < batch;
            load_words<E, VEC>(perms + (nv ? nrow : 0) * ld, k0, nv ? n : 0, s2, wn, vmax, bad);
        }
        if constexpr (VEC && E >= 8) {  // ids of fully valid vectors (checked at use, not at load)
#pragma unroll
            for (int v = 0; v < E / 8; ++v)
                if (rv && k0 + 8 * v + 8 <= n)
                    vmax = __vmaxu2(__vmaxu2(vmax, w[4 * v]), __vmaxu2(w[4 * v + 1], __vmaxu2(w[4 * v + 2], w[4 * v + 3])));
        }
        uint32_t rec[E];
#pragma unroll
        for (int j = 0; j < NW; ++j) {
            rec[2 * j] = lds32(((w[j] << SH) & amask) | tabc);
            rec[2 * j + 1] = lds32(((w[j] >> (16 - SH)) & amask) | tabc);
        }
        auto elem = [&](int k) -> uint32_t {
            const uint32_t id = rv ? (uint32_t)(uint16_t)__ldg(rp + k) : (uint32_t)n;
            return lds32(((id << SH) & amask) | tabc);
        };
        int32_t Z;
        if constexpr (UCD)
            Z = eval_ucddcp<G, E>(rec, l, gbase, n, L, elem);
        else
            Z = eval_cdd<G, E>(rec, l, gbase, n, d, L, elem);
        if (rv && l == 0) out[row] = (int64_t)Z;
    }
    if (bad || (vmax & 0xffffu) >= (uint32_t)n || (vmax >> 16) >= (uint32_t)n) atomicOr(err, 1);
}

template <int G, int E, bool UCD>
cudaError_t launch_ge(const Instance& I, const int16_t* perms, int64_t ld, int64_t batch,
                      int64_t* out, cudaStream_t s) {
    const bool vec = (ld % 8 == 0) && ((reinterpret_cast<uintptr_t>(perms) & 15) == 0);
    int npow2 = 1;
    while (npow2 <= I.n) npow2 <<= 1;  // strictly greater than n: table[n] is the zero sentinel
    // room to align the table (KC copies) to its own size
    const size_t smem = 2 * sizeof(uint32_t) * (size_t)npow2 * kGatherCopies;
    if (smem > 48 * 1024) {
        auto k1 = eval_batch_kernel<G, E, UCD, true>;
        auto k2 = eval_batch_kernel<G, E, UCD, false>;
        cudaFuncSetAttribute(k1, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        cudaFuncSetAttribute(k2, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    }
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
    kern<<<(unsigned)blocks, kEvalThreads, smem, s>>>(tab, I.n, npow2, I.d_eff, L, perms, ld, batch,
                                                      out, I.err);
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
