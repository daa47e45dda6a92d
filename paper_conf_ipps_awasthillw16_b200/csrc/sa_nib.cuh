// sa_nib.cuh -- the CDD chain layout of the headline SA configuration for instances with small
// weights: 4-bit alpha and beta packed in one byte per position, P in a byte row, and a cached
// summary per sub-block (16 positions at E = 128, 8 at E = 64) of every lane row.
//
// Why: at n = 1000 (G = 8 lanes x E = 128 positions) the group kernel's per-step pass streams the
// whole chain (5 instructions per 4 positions, a third of the step), and the boundary row's level
// 1 streams one more row.  A move of <= 4 positions changes <= 4 sub-blocks, and the quantities
// the evaluator needs from a lane row are sums over its sub-blocks:
//     acc_row = sum_k p_k * X_k            (X_k: exclusive prefix of x within the row)
//             = sum_b ( acc_b + Xbefore_b * P_b ),
// with acc_b = sum_{k in b} p_k * (prefix of x within b), X_b = sum_{k in b} x_k, P_b = sum p_k.
// So each sub-block keeps {acc_b for x = alpha and for x = beta, A_b, B_b, P_b}; the movers
// recompute the <= 4 sub-blocks they touched (restored on rejection), and the evaluation
// aggregates 8 summaries per lane instead of streaming 128 positions.  The boundary row's level 1
// (sa_group.cuh, boundary_two_level) reads lane l's sub-block summary directly: the dot of p with
// the alpha+beta prefix is acc_A + acc_B.
//
// Applies when alpha, beta <= 15 and pmax * max(alpha, beta) * 120 < 2^16 (acc_b fits 16 bits;
// 120 = sum of the in-block prefix counts 0..15), at G = 8 lanes per chain with E = 128 (n in
// (512, 1024], 16-position sub-blocks) or E = 64 (n in (256, 512], 8-position sub-blocks; one
// sub-block per lane of the boundary's level 1 either way): the OR-library ranges (p <= 20,
// alpha <= 10, beta <= 15), e.g. BASELINE config 5.  The records take 2 bytes per position
// instead of 3 and no padding, so at n = 1000 5 CTAs (20 warps) fit an SM instead of 4.
// The arithmetic is exactly the evaluator of sa_group.cuh: same penalties, same trajectories.
#pragma once
#include <cuda_runtime.h>

#include "device_common.cuh"
#include "sa_group.cuh"

namespace cdd {

template <int G, int E>
struct GChainNib {
    // (layout checks in nib_summary: overload resolution of the chain functions completes this
    // type for every (G, E) of the byte-row layout too)
    static constexpr int NP = G * E;
    static constexpr int SPR = E / G;          // boundary elements per lane (= sub-block length)
    static constexpr int SB = E / G;           // positions per sub-block (16 at E = 128, 8 at E = 64)
    static constexpr int NSB = E / SB;         // sub-blocks per lane row (= G)
    static constexpr int OFF_P = NP, OFF_S = 2 * NP, OFF_T = 2 * NP + 8 * G * NSB;
    // chains are BYTES apart: BYTES % 128 == 64 puts the summaries of a warp's even and odd chains
    // in opposite bank halves (the aggregation's LDS.64 then takes the minimum two wavefronts)
    static constexpr int RAW = OFF_T + 8 * G;
    static constexpr int BYTES = ((RAW + 63) / 64 * 64) % 128 == 64 ? (RAW + 63) / 64 * 64
                                                                        : (RAW + 63) / 64 * 64 + 64;
    uint8_t* base;
    __device__ __forceinline__ uint8_t* ab() const { return base; }         // alpha | beta << 4
    __device__ __forceinline__ uint8_t* pb() const { return base + OFF_P; }
    // summary of sub-block b of lane row r at sum()[b * G + r]:
    //   .x = acc_A | acc_B << 16,  .y = A_b | B_b << 8 | P_b << 16
    __device__ __forceinline__ uint2* sum() const { return reinterpret_cast<uint2*>(base + OFF_S); }
    __device__ __forceinline__ uint2* tot() const { return reinterpret_cast<uint2*>(base + OFF_T); }
    static __device__ __forceinline__ int sidx(int k) { return ((k % E) / SB) * G + k / E; }
};

// u0 = alpha | beta << 8 | P << 16 (the shuffle / lane-total format of pos_read)
template <int G, int E>
__device__ __forceinline__ uint32_t nib_read(const GChainNib<G, E>& ch, int k) {
    const uint32_t w = ch.ab()[k];
    return (w & 15u) | ((w >> 4) << 8) | ((uint32_t)ch.pb()[k] << 16);
}
template <int G, int E>
__device__ __forceinline__ void nib_write(const GChainNib<G, E>& ch, int k, uint32_t v) {
    ch.ab()[k] = (uint8_t)((v & 15u) | ((v >> 4) & 0xf0u));
    ch.pb()[k] = (uint8_t)(v >> 16);
}

// Summary of the Q quads of positions [k0, k0 + 4Q) (k0 a multiple of 4Q): the quad form of the SA
// pass on x = alpha and x = beta (byte-wise prefixes of three 4-bit weights fit a byte).
template <int Q>
__device__ __forceinline__ uint2 nib_quads(const uint8_t* ab, const uint8_t* pb) {
    uint32_t w[Q], q[Q];
    if constexpr (Q == 4) {
        const uint4 w4 = *reinterpret_cast<const uint4*>(ab), q4 = *reinterpret_cast<const uint4*>(pb);
        w[0] = w4.x; w[1] = w4.y; w[2] = w4.z; w[3] = w4.w;
        q[0] = q4.x; q[1] = q4.y; q[2] = q4.z; q[3] = q4.w;
    } else if constexpr (Q == 2) {
        const uint2 w2 = *reinterpret_cast<const uint2*>(ab), q2 = *reinterpret_cast<const uint2*>(pb);
        w[0] = w2.x; w[1] = w2.y;
        q[0] = q2.x; q[1] = q2.y;
    } else {
        w[0] = *reinterpret_cast<const uint32_t*>(ab);
        q[0] = *reinterpret_cast<const uint32_t*>(pb);
    }
    uint32_t accA = 0, accB = 0, sA = 0, sB = 0, P = 0;
#pragma unroll
    for (int j = 0; j < Q; ++j) {
        const uint32_t a = w[j] & 0x0f0f0f0fu, b = (w[j] >> 4) & 0x0f0f0f0fu;
        const uint32_t pq = __dp4a(q[j], 0x01010101u, 0u);
        accA = __dp4a(a * 0x01010100u, q[j], accA) + sA * pq;
        accB = __dp4a(b * 0x01010100u, q[j], accB) + sB * pq;
        sA = __dp4a(a, 0x01010101u, sA);
        sB = __dp4a(b, 0x01010101u, sB);
        P += pq;
    }
    return make_uint2(accA | (accB << 16), sA | (sB << 8) | (P << 16));
}

// Summary of sub-block [k0, k0 + SB) (k0 a multiple of SB).
template <int G, int E>
__device__ __forceinline__ uint2 nib_summary(const GChainNib<G, E>& ch, int k0) {
    using C = GChainNib<G, E>;
    static_assert(C::SB == 16 || C::SB == 8, "16- or 8-position sub-blocks, one per lane of the boundary's level 1");
    static_assert(2 * C::NP + 16 * G <= C::BYTES, "FY staging (ids + Philox words) must fit");
    return nib_quads<C::SB / 4>(ch.ab() + k0, ch.pb() + k0);
}

// Half of a sub-block's summary, positions [k0, k0 + SB/2) (k0 a multiple of SB/2), in the same
// packed format; the summary of the sub-block is nib_join(half at k0, half at k0 + SB/2).  The
// kernel splits a mover's recomputation between the mover (lanes 0-3) and lane l ^ 4 of its group.
template <int G, int E>
__device__ __forceinline__ uint2 nib_half(const GChainNib<G, E>& ch, int k0) {
    static_assert(G == 8, "mover lanes 0-3 pair with lanes 4-7 of their group");
    return nib_quads<GChainNib<G, E>::SB / 8>(ch.ab() + k0, ch.pb() + k0);
}
// lo then hi: acc = acc_lo + acc_hi + X_lo * P_hi for both weights (no carry between the 16-bit
// halves: the joined forms fit 16 bits), the byte sums and P add field-wise
__device__ __forceinline__ uint2 nib_join(uint2 lo, uint2 hi) {
    const uint32_t ph = hi.y >> 16;
    const uint32_t cross = (lo.y & 0xffu) * ph + (((lo.y >> 8) & 0xffu) * ph << 16);
    return make_uint2(lo.x + hi.x + cross, lo.y + hi.y);
}

// ---- hooks of boundary_two_level (sa_group.cuh) for this layout
// level 1: sub-block l of row Ls from its summary
template <int G, int E>
__device__ __forceinline__ void bt_level1(const GChainNib<G, E>& ch, int Ls, int l, int /*quad*/, uint32_t& Pb1,
                                          uint32_t& Sb1, uint32_t& dot) {
    const uint2 s = ch.sum()[l * G + Ls];
    Pb1 = s.y >> 16;
    Sb1 = __dp4a(s.y, 0x0101u, 0u);       // A_b + B_b
    dot = __dp2a_lo(s.x, 0x0101u, 0u);    // acc_A + acc_B
}
// level 2: L2 <= 4 consecutive positions from e (row-relative) of row Ls as alpha|beta<<8 pair
// words and a P word
template <int L2, int G, int E>
__device__ __forceinline__ void bt_spread_load(const GChainNib<G, E>& ch, int Ls, int e,
                                               uint32_t (&a2)[(L2 + 1) / 2], uint32_t& pp) {
    const int k = Ls * E + e;
    if constexpr (L2 == 2) {
        const uint32_t w = *reinterpret_cast<const uint16_t*>(ch.ab() + k);
        a2[0] = __byte_perm(w & 0x0f0fu, (w >> 4) & 0x0f0fu, 0x5140u);
        pp = *reinterpret_cast<const uint16_t*>(ch.pb() + k);
    } else if constexpr (L2 == 4) {
        const uint32_t w = *reinterpret_cast<const uint32_t*>(ch.ab() + k);
        const uint32_t lo = w & 0x0f0f0f0fu, hi = (w >> 4) & 0x0f0f0f0fu;
        a2[0] = __byte_perm(lo, hi, 0x5140u);
        a2[1] = __byte_perm(lo, hi, 0x7362u);
        pp = *reinterpret_cast<const uint32_t*>(ch.pb() + k);
    } else {
        const uint32_t w = ch.ab()[k];
        a2[0] = (w & 15u) | ((w >> 4) << 8);
        pp = ch.pb()[k];
    }
}

// CDD penalty of the group's chain: scans and boundary as gchain_eval_cdd, the row forms from the
// sub-block summaries.
template <int G, int E>
__device__ __forceinline__ int32_t gchain_eval_nib(const GChainNib<G, E>& ch, int l, int gbase, int n,
                                                   int32_t d, uint32_t tAB, uint32_t tP, int quad) {
    using C = GChainNib<G, E>;
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
    const int32_t PbS = __shfl_sync(kFull, Pb, Ls, G);
    const uint32_t ABbS = __shfl_sync(kFull, ABb, Ls, G);
    const int32_t SbS = (int32_t)(ABbS & 0xffffu) + (int32_t)(ABbS >> 16);
    const int32_t thr = Btot - SbS;
    const uint32_t key = ((uint32_t)min(thr, 0xffff) << 16) | 0xffffu;
    const int32_t corr = boundary_two_level<G, E>(ch, l, gbase, Ls, Lk, d, PbS, thr, key, quad);
    // F(C_{m'}): the row form of x = alpha (lanes left of Ls) or beta from the 8 summaries
    // per sub-block: IDP.2A picks and adds acc_A or acc_B (16-bit halves x (1, 0) / (0, 1)),
    // IDP.4A picks and adds A_b or B_b, one IMAD for Xbefore * P_b
    const bool amode = l < Ls;
    const uint32_t asel = amode ? 0x0001u : 0x0100u, xsel = amode ? 0x0001u : 0x0100u;
    const uint2* srow = ch.sum() + l;
    uint32_t acc = 0, xb = 0;
#pragma unroll
    for (int b = 0; b < C::NSB; ++b) {
        const uint2 s = srow[b * G];
        acc = __dp2a_lo(s.x, asel, acc) + xb * (s.y >> 16);
        xb = __dp4a(s.y, xsel, xb);
    }
    const int32_t base = amode ? Ab : (Btot - Bb);
    const int32_t contrib = base * (int32_t)tP + (amode ? (int32_t)acc : -(int32_t)acc) + corr;
    return (int32_t)gsum<G>((uint32_t)contrib);
}

}  // namespace cdd
