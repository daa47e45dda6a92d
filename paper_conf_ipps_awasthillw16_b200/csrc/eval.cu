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

// ------------------------------------------------------------------------------------------
// CDD with 512 < n <= 1024: 64 units of 16 positions, lane L owns units L and 32+L.  The ids of
// unit u are bytes [32u, 32u+32) of the row, so a warp's 256-bit loads of one chunk are fully
// coalesced (1 KB contiguous) -- with lane-contiguous 64-position chunks they would touch 16
// lines per instruction.  The evaluator is eval_cdd's, over units instead of lanes.
// ------------------------------------------------------------------------------------------
template <class Elem>
__device__ __forceinline__ int32_t eval_cdd_u16(const uint32_t (&r0)[16], const uint32_t (&r1)[16],
                                                int lane, int n, int32_t d, const RecLayout& L,
                                                Elem&& elem) {
    const uint32_t t0 = lane_total<16>(r0), t1 = lane_total<16>(r1);
    const uint32_t P0 = t0 & L.pmask, P1 = t1 & L.pmask;
    const uint32_t AB0 = ((t0 >> L.sa) & L.amask) | ((t0 >> L.sb) << 16);
    const uint32_t AB1 = ((t1 >> L.sa) & L.amask) | ((t1 >> L.sb) << 16);
    const uint32_t iP0 = group_incl_scan<32>(P0, lane), iP1 = group_incl_scan<32>(P1, lane);
    const uint32_t iAB0 = group_incl_scan<32>(AB0, lane), iAB1 = group_incl_scan<32>(AB1, lane);
    const uint32_t totP0 = __shfl_sync(kFull, iP0, 31);
    const uint32_t totAB0 = __shfl_sync(kFull, iAB0, 31), totAB1 = __shfl_sync(kFull, iAB1, 31);
    const int32_t Pb0 = (int32_t)(iP0 - P0), Pb1 = (int32_t)(totP0 + iP1 - P1);
    const uint32_t ABb0 = iAB0 - AB0, ABb1 = totAB0 + iAB1 - AB1;
    const int32_t Btot = (int32_t)((totAB0 + totAB1) >> 16);
    const int32_t Ab0 = (int32_t)(ABb0 & 0xffffu), Bb0 = (int32_t)(ABb0 >> 16);
    const int32_t Ab1 = (int32_t)(ABb1 & 0xffffu), Bb1 = (int32_t)(ABb1 >> 16);
    const bool v0 = 16 * lane < n, v1 = 512 + 16 * lane < n;
    const uint32_t k0b = __ballot_sync(kFull, v0 && Ab0 + Bb0 <= Btot);
    const uint32_t k1b = __ballot_sync(kFull, v1 && Ab1 + Bb1 <= Btot);
    const uint32_t t0b = __ballot_sync(kFull, v0 && Pb0 <= d);
    const uint32_t t1b = __ballot_sync(kFull, v1 && Pb1 <= d);
    const int Lk = k1b ? 32 + hibit(k1b) : hibit(k0b);
    const int Lt = t1b ? 32 + hibit(t1b) : hibit(t0b);
    const int Ls = min(Lk, Lt);
    const bool s_hi = Ls >= 32;
    const int32_t PbS = __shfl_sync(kFull, s_hi ? Pb1 : Pb0, Ls & 31);
    const uint32_t ABbS = __shfl_sync(kFull, s_hi ? ABb1 : ABb0, Ls & 31);
    // boundary unit, one element per lane (lanes 0..15)
    const int kb = 16 * Ls + lane;
    const bool ev = lane < 16 && kb < n;
    const uint32_t r = ev ? elem(kb) : 0u;
    const uint32_t ex = group_incl_scan<32, 16>(r, lane) - r;
    const int32_t pj = (int32_t)(r & L.pmask);
    const int32_t Cex = PbS + (int32_t)(ex & L.pmask);
    const int32_t Sex = (int32_t)(ABbS & 0xffffu) + (int32_t)((ex >> L.sa) & L.amask) +
                        (int32_t)(ABbS >> 16) + (int32_t)(ex >> L.sb);
    const uint32_t bke = __ballot_sync(kFull, ev && (Sex <= Btot));
    const int32_t Ck0 = __shfl_sync(kFull, Cex + pj, hibit(bke | 1u));
    const int32_t D = (Ls == Lk) ? min(Ck0, d) : d;
    const int32_t corr = ev ? (Sex - Btot) * min(pj, max(0, D - Cex)) : 0;
    // F(C_{m'}) per unit: early weights left of unit Ls, tardy weights from it on
    int32_t contrib = corr;
    {
        const bool am = lane < Ls;
        const int sh = am ? L.sa : L.sb;
        const uint32_t mk = am ? L.amask : kFull;
        uint32_t s = 0, acc = 0;
#pragma unroll
        for (int i = 0; i < 16; ++i) {
            acc += (r0[i] & L.pmask) * ((s >> sh) & mk);
            s += r0[i];
        }
        contrib += (am ? Ab0 : (Btot - Bb0)) * (int32_t)P0 + (am ? (int32_t)acc : -(int32_t)acc);
    }
    {
        const bool am = 32 + lane < Ls;
        const int sh = am ? L.sa : L.sb;
        const uint32_t mk = am ? L.amask : kFull;
        uint32_t s = 0, acc = 0;
#pragma unroll
        for (int i = 0; i < 16; ++i) {
            acc += (r1[i] & L.pmask) * ((s >> sh) & mk);
            s += r1[i];
        }
        contrib += (am ? Ab1 : (Btot - Bb1)) * (int32_t)P1 + (am ? (int32_t)acc : -(int32_t)acc);
    }
    return (int32_t)__reduce_add_sync(kFull, (uint32_t)contrib);
}

__device__ __forceinline__ void ld256(const int16_t* p, uint32_t* w) {
    // volatile: keeps the prefetch where it is written (a pure asm gets sunk to its first use)
    asm volatile("ld.global.nc.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]),
                   "=r"(w[6]), "=r"(w[7])
                 : "l"(p));
}

// ids of units `lane` and `32+lane` (8 words each); positions >= n -> sentinel
template <bool W32>
__device__ __forceinline__ void load_u16(const int16_t* __restrict__ row, int lane, int n,
                                         uint32_t s2, uint32_t (&w)[16], bool& bad) {
#pragma unroll
    for (int c = 0; c < 2; ++c) {
        const int p0 = 512 * c + 16 * lane;
        uint32_t* x = w + 8 * c;
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j] = s2;
        if (W32 && p0 + 16 <= n) {
            ld256(row + p0, x);
        } else {
#pragma unroll
            for (int h = 0; h < 2; ++h)
                if (p0 + 8 * h < n) {
                    const uint4 v = __ldg(reinterpret_cast<const uint4*>(row + p0 + 8 * h));
                    x[4 * h] = v.x; x[4 * h + 1] = v.y; x[4 * h + 2] = v.z; x[4 * h + 3] = v.w;
                }
            if (p0 < n && p0 + 16 > n && (n & 7)) {  // a straddling 8-vector (n % 8 != 0)
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                    uint32_t lo = x[j] & 0xffffu, hi = x[j] >> 16;
                    if (p0 + 2 * j < n) bad |= lo >= (uint32_t)n; else lo = s2 & 0xffffu;
                    if (p0 + 2 * j + 1 < n) bad |= hi >= (uint32_t)n; else hi = s2 & 0xffffu;
                    x[j] = lo | (hi << 16);
                }
            }
        }
    }
}

template <bool W32>
__global__ void __launch_bounds__(kEvalThreads, CDD_EVAL_MIN_BLOCKS) eval_cdd_u16_kernel(
    const uint32_t* __restrict__ table, int n, int npow2, int32_t d, RecLayout L,
    const int16_t* __restrict__ perms, int64_t ld, int64_t batch, int64_t* __restrict__ out,
    int* __restrict__ err) {
    extern __shared__ __align__(16) uint32_t s_raw[];
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
    const uint32_t s2 = (uint32_t)n * 0x10001u;
    const int lane = threadIdx.x & 31;
    const uint32_t tabc = tab | (uint32_t)((lane % KC) * 4);
    constexpr int SH = KC == 16 ? 6 : (KC == 8 ? 5 : 2);
    const int64_t warps_total = (int64_t)gridDim.x * (kEvalThreads / 32);
    uint32_t vmax = 0;
    bool bad = false;
    int64_t row = (int64_t)blockIdx.x * (kEvalThreads / 32) + (threadIdx.x >> 5);
    // evaluate the row whose ids are in w; once its records are gathered, w is refilled with the
    // ids of the row two steps ahead (prefetch distance ~2 rows without extra registers)
    auto process = [&](int64_t r, uint32_t (&w)[16]) {
        const int16_t* rp = perms + r * ld;
#pragma unroll
        for (int c = 0; c < 2; ++c)
#pragma unroll
            for (int h = 0; h < 2; ++h)
                if (512 * c + 16 * lane + 8 * h + 8 <= n)
                    vmax = __vmaxu2(__vmaxu2(vmax, w[8 * c + 4 * h]),
                                    __vmaxu2(w[8 * c + 4 * h + 1], __vmaxu2(w[8 * c + 4 * h + 2], w[8 * c + 4 * h + 3])));
        uint32_t r0[16], r1[16];
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            r0[2 * j] = lds32(((w[j] << SH) & amask) | tabc);
            r0[2 * j + 1] = lds32(((w[j] >> (16 - SH)) & amask) | tabc);
            r1[2 * j] = lds32(((w[8 + j] << SH) & amask) | tabc);
            r1[2 * j + 1] = lds32(((w[8 + j] >> (16 - SH)) & amask) | tabc);
        }
        {
            const int64_t nrow = r + 2 * warps_total;
            const bool nv = nrow < batch;
            load_u16<W32>(perms + (nv ? nrow : 0) * ld, lane, nv ? n : 0, s2, w, bad);
        }
        auto elem = [&](int k) -> uint32_t {
            const uint32_t id = (uint32_t)(uint16_t)__ldg(rp + k);
            return lds32(((id << SH) & amask) | tabc);
        };
        const int32_t Z = eval_cdd_u16(r0, r1, lane, n, d, L, elem);
        if (lane == 0) out[r] = (int64_t)Z;
    };
    uint32_t wa[16], wb[16];
    {
        const bool v0 = row < batch, v1 = row + warps_total < batch;
        load_u16<W32>(perms + (v0 ? row : 0) * ld, lane, v0 ? n : 0, s2, wa, bad);
        load_u16<W32>(perms + (v1 ? row + warps_total : 0) * ld, lane, v1 ? n : 0, s2, wb, bad);
    }
    for (; row < batch; row += 2 * warps_total) {  // one row per warp, warp-uniform; ping-pong
        process(row, wa);
        if (row + warps_total < batch) process(row + warps_total, wb);
    }
    if (bad || (vmax & 0xffffu) >= (uint32_t)n || (vmax >> 16) >= (uint32_t)n) atomicOr(err, 1);
}

cudaError_t launch_u16(const Instance& I, const int16_t* perms, int64_t ld, int64_t batch,
                       int64_t* out, cudaStream_t s) {
    const bool w32 = (ld % 16 == 0) && ((reinterpret_cast<uintptr_t>(perms) & 31) == 0);
    int npow2 = 1;
    while (npow2 <= I.n) npow2 <<= 1;
    const size_t smem = 2 * sizeof(uint32_t) * (size_t)npow2 * kGatherCopies;
    auto kern = w32 ? eval_cdd_u16_kernel<true> : eval_cdd_u16_kernel<false>;
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int dev_sms = 0, occ = 0;
    cudaError_t e = cudaDeviceGetAttribute(&dev_sms, cudaDevAttrMultiProcessorCount, I.device);
    if (e != cudaSuccess) return e;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kEvalThreads, smem);
    if (e != cudaSuccess) return e;
    int64_t blocks = (batch + (kEvalThreads / 32) - 1) / (kEvalThreads / 32);
    const int64_t cap = (int64_t)dev_sms * (occ > 0 ? occ : 1);
    if (blocks > cap) blocks = cap;
    if (blocks < 1) blocks = 1;
    kern<<<(unsigned)blocks, kEvalThreads, smem, s>>>(I.rec_cdd, I.n, npow2, I.d_eff, I.lay_cdd, perms,
                                                      ld, batch, out, I.err);
    return cudaGetLastError();
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
    const bool vec = (ld % 8 == 0) && ((reinterpret_cast<uintptr_t>(perms) & 15) == 0);
    if (!UCD && vec) return launch_u16(I, perms, ld, batch, out, s);
    return launch_ge<32, 32, UCD>(I, perms, ld, batch, out, s);
}

}  // namespace

cudaError_t launch_eval_batch(const Instance& I, bool ucd, const int16_t* perms, int64_t ld,
                              int64_t batch, int64_t* out, cudaStream_t s) {
    if (batch <= 0) return cudaSuccess;
#ifndef CDD_EVAL_V1
    {
        const cudaError_t e = ucd ? launch_eval2_ucddcp(I, perms, ld, batch, out, s)
                                  : launch_eval2_cdd(I, perms, ld, batch, out, s);
        if (e != cudaErrorNotSupported) return e;
    }
#endif
    return ucd ? dispatch<true>(I, perms, ld, batch, out, s)
               : dispatch<false>(I, perms, ld, batch, out, s);
}

}  // namespace cdd
