// sa_group.cuh -- the CDD SA kernel: G lanes per chain, 32/G chains per warp.
//
// Differences from the warp-per-chain kernel (sa.cu, used for UCDDCP):
//  * every warp instruction of the fixed per-step work (move decode, scans, ballots, Metropolis,
//    bookkeeping) serves 32/G chains at once;
//  * the per-lane totals of the packed records are kept in shared memory and updated by the
//    movers with shared atomics (delta of the <= 4 moved positions), so no full pass is needed to
//    form them; the records are streamed from shared memory once per step (pass 2);
//  * the job ids of the current sequence live in a per-chain global slot (L2-resident), written
//    only when a move is accepted.
// The arithmetic is the evaluator of device_common.cuh / chain.cuh.
#pragma once
#include <cuda_runtime.h>

#include <climits>

#include "device_common.cuh"
#include "internal.h"

namespace cdd {

// One chain of G lanes x E positions.  CDD: ab = alpha|beta<<16 (u32), pb = P (u8).  UCDDCP also:
// pb = M (u8), xb = X = P - M (u8), gh = gamma (u16).  Rows are padded so that lane-contiguous
// vector reads are bank-conflict free.
template <int G, int E, bool UCD = false>
struct GChain {
    static constexpr int NP = G * E;
    static constexpr int ABS = E >= 8 ? E + 4 : E;                         // words per lane row
    static constexpr int PS = E == 64 ? 80 : (E == 32 ? 48 : E);            // bytes per lane row
    static constexpr int GS = E >= 16 ? 2 * E + 16 : 2 * E;                // bytes per lane row (gamma)
    static constexpr int SPR = E >= G ? E / G : 1;                         // boundary elements per lane
    static constexpr int AB_BYTES = G * ABS * 4;
    static constexpr int P_BYTES = (G * PS + 15) / 16 * 16;
    static constexpr int X_BYTES = UCD ? P_BYTES : 0;
    static constexpr int G_BYTES = UCD ? (G * GS + 15) / 16 * 16 : 0;
    static constexpr int TOT_BYTES = G * 8;
    static constexpr int OFF_P = AB_BYTES, OFF_X = OFF_P + P_BYTES, OFF_G = OFF_X + X_BYTES,
                         OFF_T = OFF_G + G_BYTES;
    static constexpr int BYTES = (OFF_T + TOT_BYTES + 15) / 16 * 16;
    uint8_t* base;
    __device__ __forceinline__ uint32_t* ab() const { return reinterpret_cast<uint32_t*>(base); }
    __device__ __forceinline__ uint8_t* pb() const { return base + OFF_P; }
    __device__ __forceinline__ uint8_t* xb() const { return base + OFF_X; }
    __device__ __forceinline__ uint16_t* gh() const { return reinterpret_cast<uint16_t*>(base + OFF_G); }
    __device__ __forceinline__ uint2* tot() const { return reinterpret_cast<uint2*>(base + OFF_T); }
    static __device__ __forceinline__ int ab_w(int k) { return (k / E) * ABS + (k % E); }
    static __device__ __forceinline__ int pb_b(int k) { return (k / E) * PS + (k % E); }
    static __device__ __forceinline__ int gh_h(int k) { return (k / E) * (GS / 2) + (k % E); }
};

// Inclusive scan over G-lane segments (predicated shuffle, see device_common.cuh).
template <int G>
__device__ __forceinline__ uint32_t gscan(uint32_t v) {
    return group_incl_scan<G>(v, 0);
}

template <int G>
__device__ __forceinline__ uint32_t gsum(uint32_t v) {
    if constexpr (G == 32) {
        return __reduce_add_sync(kFull, v);
    } else {
#pragma unroll
        for (int off = G / 2; off > 0; off >>= 1) v += __shfl_xor_sync(kFull, v, off, G);
        return v;
    }
}

// CDD penalty of the group's chain.  tAB / tP: this lane's totals (maintained incrementally).
template <int G, int E>
__device__ __forceinline__ int32_t gchain_eval_cdd(const GChain<G, E>& ch, int l, int gbase, int n,
                                                   int32_t d, uint32_t tAB, uint32_t tP) {
    using C = GChain<G, E>;
    constexpr int SPR = C::SPR;
    // pass-2 operands are loaded first so their latency hides behind the scans and the spread
    const uint32_t* abr = ch.ab() + l * C::ABS;
    const uint8_t* pbr = ch.pb() + l * C::PS;
    uint32_t rr[E];
    uint32_t pw[E / 4];
#pragma unroll
    for (int v = 0; v < E / 4; ++v) {
        const uint4 x = *reinterpret_cast<const uint4*>(abr + 4 * v);
        rr[4 * v] = x.x; rr[4 * v + 1] = x.y; rr[4 * v + 2] = x.z; rr[4 * v + 3] = x.w;
    }
    if constexpr (E >= 16) {
#pragma unroll
        for (int q = 0; q < E / 16; ++q) {
            const uint4 x = *reinterpret_cast<const uint4*>(pbr + 16 * q);
            pw[4 * q] = x.x; pw[4 * q + 1] = x.y; pw[4 * q + 2] = x.z; pw[4 * q + 3] = x.w;
        }
    } else if constexpr (E == 8) {
        const uint2 x = *reinterpret_cast<const uint2*>(pbr);
        pw[0] = x.x; pw[1] = x.y;
    } else {
        pw[0] = *reinterpret_cast<const uint32_t*>(pbr);
    }
    const uint32_t iP = gscan<G>(tP);
    const uint32_t iAB = gscan<G>(tAB);
    const int32_t Pb = (int32_t)(iP - tP);
    const uint32_t ABb = iAB - tAB;
    const int32_t Ab = (int32_t)(ABb & 0xffffu), Bb = (int32_t)(ABb >> 16);
    const int32_t Btot = (int32_t)(__shfl_sync(kFull, iAB, G - 1, G) >> 16);
    const bool lane_valid = l * E < n;
    const int Lk = hibit(group_ballot<G>(lane_valid && (Ab + Bb <= Btot), gbase));
    const int Lt = hibit(group_ballot<G>(lane_valid && (Pb <= d), gbase));
    const int Ls = min(Lk, Lt);

    // ---- boundary lane Ls: SPR consecutive elements per lane
    const int32_t PbS = __shfl_sync(kFull, Pb, Ls, G);
    const uint32_t ABbS = __shfl_sync(kFull, ABb, Ls, G);
    const int32_t SbS = (int32_t)(ABbS & 0xffffu) + (int32_t)(ABbS >> 16);
    const int e0 = l * SPR;  // first element (within the row) of this lane
    const bool lane_in = e0 < E;
    uint32_t rv[SPR];
    uint32_t pv = 0;
    if constexpr (SPR == 4) {
        const uint4 x = *reinterpret_cast<const uint4*>(ch.ab() + Ls * C::ABS + e0);
        rv[0] = x.x; rv[1] = x.y; rv[2] = x.z; rv[3] = x.w;
        pv = *reinterpret_cast<const uint32_t*>(ch.pb() + Ls * C::PS + e0);
    } else if constexpr (SPR == 2) {
        const uint2 x = *reinterpret_cast<const uint2*>(ch.ab() + Ls * C::ABS + e0);
        rv[0] = x.x; rv[1] = x.y;
        pv = *reinterpret_cast<const uint16_t*>(ch.pb() + Ls * C::PS + e0);
    } else {
        rv[0] = lane_in ? ch.ab()[Ls * C::ABS + e0] : 0u;
        pv = lane_in ? ch.pb()[Ls * C::PS + e0] : 0u;
    }
    uint32_t v[SPR];
    uint32_t lsum = 0;
#pragma unroll
    for (int i = 0; i < SPR; ++i) {
        const uint32_t pi = (pv >> (8 * i)) & 0xffu;
        v[i] = pi | (((rv[i] & 0xffffu) + (rv[i] >> 16)) << 16);
        lsum += v[i];
    }
    uint32_t ex = gscan<G>(lsum) - lsum;
    int32_t Cex[SPR], Sex[SPR], pe[SPR];
    uint32_t cnt = 0;
    const int kbase = Ls * E + e0;
#pragma unroll
    for (int i = 0; i < SPR; ++i) {
        Cex[i] = PbS + (int32_t)(ex & 0xffffu);
        Sex[i] = SbS + (int32_t)(ex >> 16);
        pe[i] = (int32_t)(v[i] & 0xffffu);
        const bool ok = lane_in && (kbase + i < n) && (Sex[i] <= Btot);
        cnt += ok ? 1u : 0u;
        ex += v[i];
    }
    const int ik = (int)gsum<G>(cnt) - 1;  // k0 - Ls*E when Ls == Lk
    const int own = ik < 0 ? 0 : ik / SPR, ei = ik < 0 ? 0 : ik % SPR;
    int32_t csel = Cex[0] + pe[0];
#pragma unroll
    for (int i = 1; i < SPR; ++i) csel = (ei == i) ? Cex[i] + pe[i] : csel;
    const int32_t Ck0 = __shfl_sync(kFull, csel, own, G);
    const int32_t D = (Ls == Lk) ? min(Ck0, d) : d;
    int32_t corr = 0;
#pragma unroll
    for (int i = 0; i < SPR; ++i) {
        const bool vi = lane_in && (kbase + i < n);
        corr += vi ? (Sex[i] - Btot) * min(pe[i], max(0, D - Cex[i])) : 0;
    }

    // ---- F(C_{m'}): two positions per PRMT (16-bit prefix halves) + IDP.2A (x 8-bit p)
    const bool amode = l < Ls;
    const uint32_t sel = amode ? 0x5410u : 0x7632u;
    uint32_t s = 0, acc = 0;
#pragma unroll
    for (int j = 0; j < E; j += 2) {
        const uint32_t t = s + rr[j];
        acc = (j & 2) ? __dp2a_hi(__byte_perm(s, t, sel), pw[j >> 2], acc)
                      : __dp2a_lo(__byte_perm(s, t, sel), pw[j >> 2], acc);
        s = t + rr[j + 1];
    }
    const int32_t base = amode ? Ab : (Btot - Bb);
    const int32_t contrib = base * (int32_t)tP + (amode ? (int32_t)acc : -(int32_t)acc) + corr;
    return (int32_t)gsum<G>((uint32_t)contrib);
}

// UCDDCP penalty of the group's chain (same quantities as chain_eval_ucddcp in chain.cuh):
// due-date position C_{k0} (d >= sum P), Z = sum_j M_j w_j + X_j min(w_j, gamma_j).
template <int G, int E>
__device__ __forceinline__ int32_t gchain_eval_ucddcp(const GChain<G, E, true>& ch, int l, int gbase,
                                                      int n, uint32_t tAB) {
    using C = GChain<G, E, true>;
    constexpr int SPR = C::SPR;
    const uint32_t* abr = ch.ab() + l * C::ABS;
    uint32_t rr[E];
#pragma unroll
    for (int v = 0; v < E / 4; ++v) {
        const uint4 x = *reinterpret_cast<const uint4*>(abr + 4 * v);
        rr[4 * v] = x.x; rr[4 * v + 1] = x.y; rr[4 * v + 2] = x.z; rr[4 * v + 3] = x.w;
    }
    uint32_t mw[E / 4], xw[E / 4], gw[E / 2];
    {
        const uint8_t* mp = ch.pb() + l * C::PS;
        const uint8_t* xp = ch.xb() + l * C::PS;
        const uint8_t* gp = reinterpret_cast<const uint8_t*>(ch.gh()) + l * C::GS;
        if constexpr (E >= 16) {
#pragma unroll
            for (int q = 0; q < E / 16; ++q) {
                const uint4 a = *reinterpret_cast<const uint4*>(mp + 16 * q);
                const uint4 b = *reinterpret_cast<const uint4*>(xp + 16 * q);
                mw[4 * q] = a.x; mw[4 * q + 1] = a.y; mw[4 * q + 2] = a.z; mw[4 * q + 3] = a.w;
                xw[4 * q] = b.x; xw[4 * q + 1] = b.y; xw[4 * q + 2] = b.z; xw[4 * q + 3] = b.w;
            }
        } else if constexpr (E == 8) {
            const uint2 a = *reinterpret_cast<const uint2*>(mp);
            const uint2 b = *reinterpret_cast<const uint2*>(xp);
            mw[0] = a.x; mw[1] = a.y; xw[0] = b.x; xw[1] = b.y;
        } else {
            mw[0] = *reinterpret_cast<const uint32_t*>(mp);
            xw[0] = *reinterpret_cast<const uint32_t*>(xp);
        }
        if constexpr (E >= 8) {
#pragma unroll
            for (int q = 0; q < E / 8; ++q) {
                const uint4 a = *reinterpret_cast<const uint4*>(gp + 16 * q);
                gw[4 * q] = a.x; gw[4 * q + 1] = a.y; gw[4 * q + 2] = a.z; gw[4 * q + 3] = a.w;
            }
        } else {
            const uint2 a = *reinterpret_cast<const uint2*>(gp);
            gw[0] = a.x; gw[1] = a.y;
        }
    }
    const uint32_t iAB = gscan<G>(tAB);
    const uint32_t ABb = iAB - tAB;
    const int32_t Ab = (int32_t)(ABb & 0xffffu), Bb = (int32_t)(ABb >> 16);
    const int32_t Btot = (int32_t)(__shfl_sync(kFull, iAB, G - 1, G) >> 16);
    const bool lane_valid = l * E < n;
    const int Lk = hibit(group_ballot<G>(lane_valid && (Ab + Bb <= Btot), gbase));

    // boundary lane Lk: SPR consecutive elements per lane
    const uint32_t ABbS = __shfl_sync(kFull, ABb, Lk, G);
    const int e0 = l * SPR;
    const bool lane_in = e0 < E;
    uint32_t rv[SPR], mv[SPR], xv[SPR], gv[SPR];
#pragma unroll
    for (int i = 0; i < SPR; ++i) {
        const bool ok = lane_in;
        const int k = Lk * E + e0 + i;
        rv[i] = ok ? ch.ab()[C::ab_w(k)] : 0u;
        mv[i] = ok ? ch.pb()[C::pb_b(k)] : 0u;
        xv[i] = ok ? ch.xb()[C::pb_b(k)] : 0u;
        gv[i] = ok ? ch.gh()[C::gh_h(k)] : 0u;
    }
    uint32_t lsum = 0;
#pragma unroll
    for (int i = 0; i < SPR; ++i) lsum += rv[i];
    uint32_t ex = gscan<G>(lsum) - lsum;
    int32_t wA[SPR], wB[SPR];
    uint32_t cnt = 0;
    const int kbase = Lk * E + e0;
#pragma unroll
    for (int i = 0; i < SPR; ++i) {
        const int32_t Aex = (int32_t)(ABbS & 0xffffu) + (int32_t)(ex & 0xffffu);
        const int32_t Bex = (int32_t)(ABbS >> 16) + (int32_t)(ex >> 16);
        wA[i] = Aex;
        wB[i] = Btot - Bex;
        cnt += (lane_in && kbase + i < n && Aex + Bex <= Btot) ? 1u : 0u;
        ex += rv[i];
    }
    const int ik = (int)gsum<G>(cnt) - 1;  // k0 - Lk*E
    int32_t corr = 0;
#pragma unroll
    for (int i = 0; i < SPR; ++i) {
        const int32_t g = (int32_t)gv[i];
        if (lane_in && e0 + i <= ik)
            corr += (int32_t)mv[i] * (wA[i] - wB[i]) + (int32_t)xv[i] * (min(wA[i], g) - min(wB[i], g));
    }

    // pass 2: pairs of weights as 16-bit halves
    const bool amode = l < Lk;
    const uint32_t base = (uint32_t)(amode ? Ab : (Btot - Bb));
    const uint32_t base2 = base | (base << 16);
    const uint32_t sgn = amode ? 1u : 0xffffffffu;
    const uint32_t sel = amode ? 0x5410u : 0x7632u;
    uint32_t s = 0, acc = 0;
#pragma unroll
    for (int j = 0; j < E; j += 2) {
        const uint32_t t = s + rr[j];
        const uint32_t w2 = __byte_perm(s, t, sel) * sgn + base2;
        const uint32_t mn2 = __vminu2(w2, gw[j >> 1]);
        if (j & 2) {
            acc = __dp2a_hi(w2, mw[j >> 2], acc);
            acc = __dp2a_hi(mn2, xw[j >> 2], acc);
        } else {
            acc = __dp2a_lo(w2, mw[j >> 2], acc);
            acc = __dp2a_lo(mn2, xw[j >> 2], acc);
        }
        s = t + rr[j + 1];
    }
    return (int32_t)gsum<G>(acc + (uint32_t)corr);
}

}  // namespace cdd
