// sa_group.cuh -- the SA chain layout and evaluators of the group kernel: G lanes per chain,
// 32/G chains per warp (sa.cu: sa_group_kernel).
//
// Differences from the warp-per-chain kernel (sa.cu: sa_kernel, used for n <= 64):
//  * every warp instruction of the fixed per-step work (move decode, scans, ballots, Metropolis,
//    bookkeeping) serves 32/G chains at once;
//  * the per-lane totals of the records are kept in shared memory and updated by the movers with
//    shared atomics (delta of the <= 4 moved positions), so no pass is needed to form them;
//  * records are 16 bits (alpha | beta << 8) -- half the shared-memory traffic and registers of
//    32-bit records -- and the per-position pass works on them directly: for a pair of positions
//    (2j, 2j+1) packed in one word w, the pair of 16-bit exclusive prefixes is
//    f2 = s * 0x10001 + (x_{2j} << 16) (one PRMT, one IMAD), it is dotted with the pair of
//    processing times by IDP.2A, and the running prefix advances by IDP.4A(w, weights);
//  * the job ids of the current sequence live in a per-chain global slot (L2-resident), written
//    only when a move is accepted.
// The arithmetic is the evaluator of device_common.cuh / chain.cuh.
#pragma once
#include <cuda_runtime.h>

#include <climits>

#include "device_common.cuh"
#include "internal.h"

// 1: the CDD pass-2 records are loaded into registers before the scans (latency hidden by ILP);
// 0: streamed in chunks of 16 positions (fewer registers, more resident warps)
#ifndef CDD_SAG_PREFETCH
#define CDD_SAG_PREFETCH 0
#endif
// timing experiment only (wrong results): the CDD quad pass streams 1/CDD_SAG_PASSDIV of each row
#ifndef CDD_SAG_PASSDIV
#define CDD_SAG_PASSDIV 1
#endif
// 1: the CDD pass runs the two halves of a lane row as independent dependency chains (experiment)
#ifndef CDD_SAG_SPLITPASS
#define CDD_SAG_SPLITPASS 0
#endif

namespace cdd {

// One chain of G lanes x E positions.  ab = alpha | beta << 8 (u16), pb = P (CDD) or M (UCDDCP)
// (u8), UCDDCP also xb = X = P - M (u8), gh = gamma (u16).  Rows are padded so that
// lane-contiguous vector reads are bank-conflict free.
template <int G, int E, bool UCD = false>
struct GChain {
    static constexpr int NP = G * E;
    static constexpr int AS = E >= 16 ? 2 * E + 16 : 2 * E;               // bytes per lane row (ab)
    static constexpr int PS = E >= 32 ? E + 16 : E;                        // bytes per lane row (p)
    static constexpr int GS = E >= 16 ? 2 * E + 16 : 2 * E;                // bytes per lane row (gamma)
    static constexpr int SPR = E >= G ? E / G : 1;                         // boundary elements per lane
    static constexpr int AB_BYTES = (G * AS + 15) / 16 * 16;
    static constexpr int P_BYTES = (G * PS + 15) / 16 * 16;
    static constexpr int X_BYTES = UCD ? P_BYTES : 0;
    static constexpr int G_BYTES = UCD ? (G * GS + 15) / 16 * 16 : 0;
    static constexpr int TOT_BYTES = G * 8;
    static constexpr int OFF_P = AB_BYTES, OFF_X = OFF_P + P_BYTES, OFF_G = OFF_X + X_BYTES,
                         OFF_T = OFF_G + G_BYTES;
    static constexpr int BYTES = (OFF_T + TOT_BYTES + 15) / 16 * 16;
    static_assert(2 * NP + 16 * G <= BYTES, "FY staging (ids + Philox words) must fit");
    uint8_t* base;
    __device__ __forceinline__ uint16_t* ab() const { return reinterpret_cast<uint16_t*>(base); }
    __device__ __forceinline__ uint8_t* pb() const { return base + OFF_P; }
    __device__ __forceinline__ uint8_t* xb() const { return base + OFF_X; }
    __device__ __forceinline__ uint16_t* gh() const { return reinterpret_cast<uint16_t*>(base + OFF_G); }
    __device__ __forceinline__ uint2* tot() const { return reinterpret_cast<uint2*>(base + OFF_T); }
    static __device__ __forceinline__ int ab_h(int k) { return (k / E) * (AS / 2) + (k % E); }
    static __device__ __forceinline__ int pb_b(int k) { return (k / E) * PS + (k % E); }
    static __device__ __forceinline__ int gh_h(int k) { return (k / E) * (GS / 2) + (k % E); }
};

// CDD chain: three byte rows per lane -- alpha, beta, P -- so that four consecutive positions of
// one field are one 32-bit word.  With max(alpha, beta) <= 85 the pass then handles a quad of
// positions in five instructions (byte-wise prefixes by one IMAD, IDP.4A against the P quad);
// larger weights use 16-bit prefix pairs as the UCDDCP layout does.  Lane rows are padded by 16
// bytes (E >= 32) so the lane-contiguous LDS.128 of a group is bank-conflict free.
template <int G, int E>
struct GChain<G, E, false> {
    static constexpr int NP = G * E;
    static constexpr int RS = E >= 32 ? E + 16 : E;  // bytes per lane row (each field)
    static constexpr int PS = RS;
    static constexpr int SPR = E >= G ? E / G : 1;   // boundary elements per lane
    static constexpr int ROW_BYTES = (G * RS + 15) / 16 * 16;
    static constexpr int OFF_B = ROW_BYTES, OFF_P = 2 * ROW_BYTES, OFF_T = 3 * ROW_BYTES;
    static constexpr int BYTES = (OFF_T + G * 8 + 15) / 16 * 16;
    static_assert(2 * NP + 16 * G <= BYTES, "FY staging (ids + Philox words) must fit");
    uint8_t* base;
    __device__ __forceinline__ uint8_t* a8() const { return base; }
    __device__ __forceinline__ uint8_t* b8() const { return base + OFF_B; }
    __device__ __forceinline__ uint8_t* pb() const { return base + OFF_P; }
    __device__ __forceinline__ uint2* tot() const { return reinterpret_cast<uint2*>(base + OFF_T); }
    static __device__ __forceinline__ int rb(int k) { return (k / E) * RS + (k % E); }
    static __device__ __forceinline__ int pb_b(int k) { return rb(k); }
};

// N alpha bytes and N beta bytes (N >= 2, a multiple of 2) as N/2 words alpha|beta<<8 per
// position, two positions per word (the 16-bit record pairs of the UCDDCP layout)
template <int N>
__device__ __forceinline__ void ab_pairs(const uint8_t* ar, const uint8_t* br, uint32_t (&w)[N / 2]) {
    if constexpr (N >= 4) {
        uint32_t a[N / 4], b[N / 4];
        if constexpr (N >= 16) {
#pragma unroll
            for (int q = 0; q < N / 16; ++q) {
                const uint4 x = *reinterpret_cast<const uint4*>(ar + 16 * q);
                const uint4 y = *reinterpret_cast<const uint4*>(br + 16 * q);
                a[4 * q] = x.x; a[4 * q + 1] = x.y; a[4 * q + 2] = x.z; a[4 * q + 3] = x.w;
                b[4 * q] = y.x; b[4 * q + 1] = y.y; b[4 * q + 2] = y.z; b[4 * q + 3] = y.w;
            }
        } else if constexpr (N == 8) {
            const uint2 x = *reinterpret_cast<const uint2*>(ar);
            const uint2 y = *reinterpret_cast<const uint2*>(br);
            a[0] = x.x; a[1] = x.y; b[0] = y.x; b[1] = y.y;
        } else {
            a[0] = *reinterpret_cast<const uint32_t*>(ar);
            b[0] = *reinterpret_cast<const uint32_t*>(br);
        }
#pragma unroll
        for (int q = 0; q < N / 4; ++q) {
            w[2 * q] = __byte_perm(a[q], b[q], 0x5140u);
            w[2 * q + 1] = __byte_perm(a[q], b[q], 0x7362u);
        }
    } else {
        const uint32_t a = *reinterpret_cast<const uint16_t*>(ar), b = *reinterpret_cast<const uint16_t*>(br);
        w[0] = __byte_perm(a, b, 0x5140u);
    }
}

// alpha | beta << 8 (u16) -> alpha | beta << 16
__device__ __forceinline__ uint32_t ab_wide(uint32_t r16) { return __byte_perm(r16, 0u, 0x4140u); }

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

// E/2 words of the lane's 16-bit records (two positions per word)
template <int E>
__device__ __forceinline__ void load_ab16(const uint8_t* row, uint32_t (&rr)[E / 2]) {
    if constexpr (E >= 8) {
#pragma unroll
        for (int v = 0; v < E / 8; ++v) {
            const uint4 x = *reinterpret_cast<const uint4*>(row + 16 * v);
            rr[4 * v] = x.x; rr[4 * v + 1] = x.y; rr[4 * v + 2] = x.z; rr[4 * v + 3] = x.w;
        }
    } else {
        const uint2 x = *reinterpret_cast<const uint2*>(row);
        rr[0] = x.x; rr[1] = x.y;
    }
}

// E bytes of the lane as E/4 words
template <int E>
__device__ __forceinline__ void load_b8(const uint8_t* row, uint32_t (&w)[E / 4]) {
    if constexpr (E >= 16) {
#pragma unroll
        for (int q = 0; q < E / 16; ++q) {
            const uint4 x = *reinterpret_cast<const uint4*>(row + 16 * q);
            w[4 * q] = x.x; w[4 * q + 1] = x.y; w[4 * q + 2] = x.z; w[4 * q + 3] = x.w;
        }
    } else if constexpr (E == 8) {
        const uint2 x = *reinterpret_cast<const uint2*>(row);
        w[0] = x.x; w[1] = x.y;
    } else {
        w[0] = *reinterpret_cast<const uint32_t*>(row);
    }
}

// SPR consecutive records of unit (lane row) `ls` starting at element e0, widened to alpha | beta << 16
// (CDD byte rows)
template <int SPR, int G, int E>
__device__ __forceinline__ void load_spread(const GChain<G, E, false>& ch, int ls, int e0, bool in,
                                            uint32_t (&rv)[SPR]) {
    using C = GChain<G, E, false>;
    const int o = ls * C::RS + e0;
    if constexpr (SPR >= 2) {
        uint32_t w[SPR / 2];
        ab_pairs<SPR>(ch.a8() + o, ch.b8() + o, w);
#pragma unroll
        for (int i = 0; i < SPR / 2; ++i) {
            rv[2 * i] = ab_wide(w[i] & 0xffffu);
            rv[2 * i + 1] = ab_wide(w[i] >> 16);
        }
    } else {
        rv[0] = in ? ((uint32_t)ch.a8()[o] | ((uint32_t)ch.b8()[o] << 16)) : 0u;
    }
}

template <int SPR, class C>
__device__ __forceinline__ void load_spread(const C& ch, int ls, int e0, bool in, uint32_t (&rv)[SPR]) {
    const uint16_t* src = ch.ab() + ls * (C::AS / 2) + e0;
    if constexpr (SPR >= 8) {
#pragma unroll
        for (int v = 0; v < SPR / 8; ++v) {
            const uint4 x = reinterpret_cast<const uint4*>(src)[v];
            const uint32_t w[4] = {x.x, x.y, x.z, x.w};
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                rv[8 * v + 2 * i] = ab_wide(w[i] & 0xffffu);
                rv[8 * v + 2 * i + 1] = ab_wide(w[i] >> 16);
            }
        }
    } else if constexpr (SPR == 4) {
        const uint2 x = *reinterpret_cast<const uint2*>(src);
        rv[0] = ab_wide(x.x & 0xffffu); rv[1] = ab_wide(x.x >> 16);
        rv[2] = ab_wide(x.y & 0xffffu); rv[3] = ab_wide(x.y >> 16);
    } else if constexpr (SPR == 2) {
        const uint32_t x = *reinterpret_cast<const uint32_t*>(src);
        rv[0] = ab_wide(x & 0xffffu); rv[1] = ab_wide(x >> 16);
    } else {
        rv[0] = in ? ab_wide(src[0]) : 0u;
    }
}

// Boundary row Ls for rows of E >= G^2 positions, in two levels, returning this lane's share of
// corr = sum_k (S_k - Btot) * clamp(D - C_{k-1}, 0, p_k) over the row (row-relative: c_k, s_k
// exclusive prefixes of p and alpha + beta, thr = Btot - S at the row start).
//  level 1: lane l takes sub-block l (SB = E/G consecutive positions): its sums of p and
//           alpha + beta (IDP.4A), its local dot  sum_k p_k * s^loc_k  (f2 pairs + IDP.2A), and a
//           G-lane scan of the packed sums gives every sub-block's start.  Sub-blocks wholly left
//           of D contribute  dot + (s_b - thr) * P_b  each.
//  level 2: the sub-block holding k0 (last start with S <= Btot) is spread over the G lanes
//           (SB/G positions each) to find C_{k0}, hence D; then the sub-block holding D (last start
//           with c < D) is spread the same way for its partial term.
// Level 1 of the byte-row layout: sub-block l of row Ls streamed (the nibble layout of sa_nib.cuh
// reads a cached summary instead).
template <int G, int E>
__device__ __forceinline__ void bt_level1(const GChain<G, E>& ch, int Ls, int l, int quad, uint32_t& Pb1,
                                          uint32_t& Sb1, uint32_t& dot) {
    using C = GChain<G, E>;
    constexpr int SB = E / G;
    const uint8_t* arow = ch.a8() + Ls * C::RS;
    const uint8_t* brow = ch.b8() + Ls * C::RS;
    const uint8_t* prow = ch.pb() + Ls * C::RS;
    uint32_t q[SB / 4];
    load_b8<SB>(prow + SB * l, q);
    Pb1 = 0, Sb1 = 0, dot = 0;
    if (quad == 2) {
        // max(alpha + beta) <= 85: the alpha and beta words add bytewise without carries, and the
        // byte-wise exclusive prefixes of a quad (<= 3 * 85) fit a byte -- the main pass's quad
        // form on x = alpha + beta (one IMAD + IDP.4A per quad, the cross term s * P_quad)
        uint32_t a[SB / 4], b[SB / 4];
        load_b8<SB>(arow + SB * l, a);
        load_b8<SB>(brow + SB * l, b);
#pragma unroll
        for (int j = 0; j < SB / 4; ++j) {
            const uint32_t x = a[j] + b[j];
            const uint32_t pq = __dp4a(q[j], 0x01010101u, 0u);
            dot = __dp4a(x * 0x01010100u, q[j], dot);
            dot += Sb1 * pq;
            Sb1 = __dp4a(x, 0x01010101u, Sb1);
            Pb1 += pq;
        }
    } else {
        uint32_t w[SB / 2];
        ab_pairs<SB>(arow + SB * l, brow + SB * l, w);
        uint32_t sig2 = 0;
#pragma unroll
        for (int j = 0; j < SB / 4; ++j) Pb1 = __dp4a(q[j], 0x01010101u, Pb1);
#pragma unroll
        for (int j = 0; j < SB / 2; ++j) {
            // positions 2j, 2j+1: f2 = (s, s + s_{2j}) in 16-bit halves, dotted with (p_{2j}, p_{2j+1})
            const uint32_t f2 = __dp4a(w[j], 0x00000101u, 0u) * 0x10000u + sig2;
            dot = (j & 1) ? __dp2a_hi(f2, q[j >> 1], dot) : __dp2a_lo(f2, q[j >> 1], dot);
            const uint32_t pair = __dp4a(w[j], 0x01010101u, 0u);
            sig2 += pair * 0x10001u;
            Sb1 += pair;
        }
    }
}

// Level 2 of the byte-row layout: L2 consecutive positions from e (row-relative) of row Ls as
// alpha|beta<<8 pair words and a P word.
template <int L2, int G, int E>
__device__ __forceinline__ void bt_spread_load(const GChain<G, E>& ch, int Ls, int e, uint32_t (&a2)[(L2 + 1) / 2],
                                               uint32_t& pp) {
    using C = GChain<G, E>;
    const uint8_t* arow = ch.a8() + Ls * C::RS;
    const uint8_t* brow = ch.b8() + Ls * C::RS;
    const uint8_t* prow = ch.pb() + Ls * C::RS;
    if constexpr (L2 >= 2) {
        ab_pairs<L2>(arow + e, brow + e, a2);
        pp = L2 == 4 ? *reinterpret_cast<const uint32_t*>(prow + e) : (uint32_t)*reinterpret_cast<const uint16_t*>(prow + e);
    } else {
        a2[0] = (uint32_t)arow[e] | ((uint32_t)brow[e] << 8);
        pp = prow[e];
    }
}

// Boundary row Ls for rows of E >= G^2 positions, in two levels, returning this lane's share of
// corr = sum_k (S_k - Btot) * clamp(D - C_{k-1}, 0, p_k) over the row (row-relative: c_k, s_k
// exclusive prefixes of p and alpha + beta, thr = Btot - S at the row start).
//  level 1: lane l takes sub-block l (SB = E/G consecutive positions): its sums of p and
//           alpha + beta (IDP.4A), its local dot  sum_k p_k * s^loc_k  (f2 pairs + IDP.2A), and a
//           G-lane scan of the packed sums gives every sub-block's start.  Sub-blocks wholly left
//           of D contribute  dot + (s_b - thr) * P_b  each.
//  level 2: the sub-block holding k0 (last start with S <= Btot) is spread over the G lanes
//           (SB/G positions each) to find C_{k0}, hence D; then the sub-block holding D (last start
//           with c < D) is spread the same way for its partial term.
// The layout's loads are the bt_level1 / bt_spread_load overloads (GChain here, GChainNib in
// sa_nib.cuh).
template <int G, int E, class C>
__device__ __forceinline__ int32_t boundary_two_level(const C& ch, int l, int gbase,
                                                      int Ls, int Lk, int32_t d, int32_t PbS,
                                                      int32_t thr, uint32_t key, int quad) {
    constexpr int SB = E / G;   // positions per sub-block (16 for E = 128, G = 8)
    constexpr int L2 = SB / G;  // positions per lane in level 2
    static_assert(SB % 8 == 0 && L2 >= 1 && L2 <= 4, "two-level boundary layout");
    // ---- level 1
    uint32_t Pb1, Sb1, dot;
    bt_level1(ch, Ls, l, quad, Pb1, Sb1, dot);
    const uint32_t lsum = Pb1 | (Sb1 << 16);
    const uint32_t ex = gscan<G>(lsum) - lsum;  // c_b | s_b << 16 at the sub-block start
    const int32_t cb = (int32_t)(ex & 0xffffu), sb = (int32_t)(ex >> 16);
    const int32_t full = (int32_t)dot + (sb - thr) * (int32_t)Pb1;
    const int own = max(0, hibit(group_ballot<G>(ex <= key, gbase)));  // lane 0 always qualifies

    // ---- level 2a: k0 inside sub-block `own`, C_{k0} (inclusive) -> D
    auto spread = [&](int blk, uint32_t (&v)[L2]) -> uint32_t {
        const int e = SB * blk + L2 * l;
        uint32_t a2[(L2 + 1) / 2], pp;
        bt_spread_load<L2>(ch, Ls, e, a2, pp);
        uint32_t tot = 0;
#pragma unroll
        for (int i = 0; i < L2; ++i) {
            const uint32_t si = __dp4a(a2[i >> 1], (i & 1) ? 0x01010000u : 0x00000101u, 0u);
            v[i] = __byte_perm(pp, 0u, 0x4440u + i) + (si << 16);
            tot += v[i];
        }
        return gscan<G>(tot) - tot + __shfl_sync(kFull, ex, blk, G);  // row-relative start
    };
    uint32_t v[L2];
    uint32_t run, run0 = 0;
    // D - C at the row start.  C_{k0} matters only when the boundary row is k0's (Ls == Lk); when
    // d's row comes first (Lt < Lk), C_{k0} > d and D = d -- the usual case for restrictive due
    // dates -- so a warp whose chains all have Ls < Lk skips the search for C_{k0}
    int32_t Dr = d - PbS;
    const bool s2a = __any_sync(kFull, Ls == Lk);
    if (s2a) {
        run = spread(own, v);
        run0 = run;
        uint32_t cinc = 0;
        const bool first_sat = run <= key;
#pragma unroll
        for (int i = 0; i < L2; ++i) {
            const bool sat = run <= key;
            run += v[i];
            cinc = sat ? run : cinc;
        }
        const int own2 = max(0, hibit(group_ballot<G>(first_sat, gbase)));
        const int32_t Ck0 = PbS + (int32_t)(__shfl_sync(kFull, cinc, own2, G) & 0xffffu);
        if (Ls == Lk) Dr = min(Ck0, d) - PbS;
    }

    // ---- level 2b: sub-blocks left of the one holding D count in full; that one in part
    const int ownD = hibit(group_ballot<G>(cb < Dr, gbase));  // -1 iff Dr <= 0 (then corr = 0)
    // D = C_{k0} (the unrestrictive case) lies in k0's sub-block: level 2a's spread is re-used
    if (!s2a || !__all_sync(kFull, max(ownD, 0) == own)) run = spread(max(ownD, 0), v);
    else run = run0;
    int32_t corr = (l < ownD) ? full : 0;
#pragma unroll
    for (int i = 0; i < L2; ++i) {
        const int32_t ci = (int32_t)(run & 0xffffu), si = (int32_t)(run >> 16);
        const int32_t pi = (int32_t)(v[i] & 0xffu);
        corr += (si - thr) * min(pi, max(0, Dr - ci));
        run += v[i];
    }
    return corr;
}

// CDD penalty of the group's chain.  tAB / tP: this lane's totals (maintained incrementally).
// quad: max(alpha, beta) <= 85 (the byte-wise prefix of three weights never carries).
template <int G, int E>
__device__ __forceinline__ int32_t gchain_eval_cdd(const GChain<G, E>& ch, int l, int gbase, int n,
                                                   int32_t d, uint32_t tAB, uint32_t tP, int quad) {
    using C = GChain<G, E>;
    constexpr int SPR = C::SPR;
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
    // Everything below is relative to the start of the row: C - PbS and S - SbS, both < 2^16 per
    // row (E * 255, E * 510 for E <= 128), so they travel packed as c | s << 16.  thr = Btot - SbS >= 0 since
    // Ls <= Lk.  Padded positions (k >= n) hold zero records: they add nothing to c or s, and where
    // they pass the S <= Btot test (only if every alpha is 0) they repeat C_n, so no index test.
    const int32_t thr = Btot - SbS;
    // (s >> 16) <= thr  <=>  s <= key  for a packed c | s << 16 (s <= E * 510 < 2^16, so
    // thr >= 0xffff admits every element)
    const uint32_t key = ((uint32_t)min(thr, 0xffff) << 16) | 0xffffu;
    int32_t corr = 0;
    if constexpr (E < G * G || E / G < 8) {  // one level: SPR = E/G positions per lane
        const int e0 = l * SPR;
        const bool lane_in = e0 < E;
        uint32_t rv[SPR];
        load_spread<SPR>(ch, Ls, e0, lane_in, rv);
        constexpr int PW = SPR >= 4 ? SPR / 4 : 1;
        uint32_t pv[PW];
        const uint8_t* psrc = ch.pb() + Ls * C::RS + e0;
        if constexpr (SPR >= 16) {
#pragma unroll
            for (int q = 0; q < SPR / 16; ++q) {
                const uint4 x = reinterpret_cast<const uint4*>(psrc)[q];
                pv[4 * q] = x.x; pv[4 * q + 1] = x.y; pv[4 * q + 2] = x.z; pv[4 * q + 3] = x.w;
            }
        } else if constexpr (SPR == 8) {
            const uint2 x = *reinterpret_cast<const uint2*>(psrc);
            pv[0] = x.x; pv[1] = x.y;
        } else if constexpr (SPR == 4) pv[0] = *reinterpret_cast<const uint32_t*>(psrc);
        else if constexpr (SPR == 2) pv[0] = *reinterpret_cast<const uint16_t*>(psrc);
        else pv[0] = lane_in ? psrc[0] : 0u;
        uint32_t v[SPR];
        uint32_t lsum = 0;
#pragma unroll
        for (int i = 0; i < SPR; ++i) {
            // p | (alpha + beta) << 16 from the widened record alpha | beta << 16
            v[i] = __byte_perm(pv[i / 4], 0u, 0x4440u + (i & 3)) + (rv[i] << 16) + (rv[i] & 0xffff0000u);
            lsum += v[i];
        }
        const uint32_t ex = gscan<G>(lsum) - lsum;
        // k0: the last element of the row with S_excl <= Btot (a prefix of the row); its inclusive C
        // (needed only when the boundary row is k0's, see boundary_two_level)
        int32_t Dr = d - PbS;  // D - C at the row start
        if (__any_sync(kFull, Ls == Lk)) {
            uint32_t run = ex, cinc = 0;
            const bool sat0 = lane_in && ex <= key;
#pragma unroll
            for (int i = 0; i < SPR; ++i) {
                const bool sat = run <= key;
                run += v[i];
                cinc = sat ? run : cinc;
            }
            const int own = hibit(group_ballot<G>(sat0, gbase));  // >= 0: element 0 of the row has S = SbS
            const int32_t Ck0 = PbS + (int32_t)(__shfl_sync(kFull, cinc, own < 0 ? 0 : own, G) & 0xffffu);
            if (Ls == Lk) Dr = min(Ck0, d) - PbS;
        }
        uint32_t run = ex;
#pragma unroll
        for (int i = 0; i < SPR; ++i) {
            const int32_t ci = (int32_t)(run & 0xffffu), si = (int32_t)(run >> 16);
            const int32_t pi = (int32_t)(v[i] & 0xffu);
            corr += (si - thr) * min(pi, max(0, Dr - ci));
            run += v[i];
        }
    } else {
        corr = boundary_two_level<G, E>(ch, l, gbase, Ls, Lk, d, PbS, thr, key, quad);
    }

    // ---- F(C_{m'}) = sum_j p_j * (exclusive prefix of x within the lane row), x = alpha in early
    // lanes, beta in tardy lanes
    const bool amode = l < Ls;
    const uint8_t* xrow = (amode ? ch.a8() : ch.b8()) + l * C::RS;
    const uint8_t* prow = ch.pb() + l * C::RS;
    constexpr int CH = E >= 16 ? 16 : E;  // positions per chunk (32 measured: same speed)
    uint32_t s = 0, acc = 0;
    if (quad) {
        // per quad: byte-wise exclusive prefixes [0, x0, x0+x1, x0+x1+x2] by one IMAD, their dot
        // with the P quad by IDP.4A, plus s * (sum of the P quad)
#pragma unroll
        for (int c0 = 0; c0 < E / CDD_SAG_PASSDIV; c0 += CH) {
            uint32_t x[CH / 4], q[CH / 4];
            load_b8<CH>(xrow + c0, x);
            load_b8<CH>(prow + c0, q);
#pragma unroll
            for (int j = 0; j < CH / 4; ++j) {
                acc = __dp4a(x[j] * 0x01010100u, q[j], acc);
                acc += s * __dp4a(q[j], 0x01010101u, 0u);
                s = __dp4a(x[j], 0x01010101u, s);
            }
        }
    } else {
        // pairs: f2 = (s, s + x_{2j}) in 16-bit halves, IDP.2A with the pair of p bytes
#pragma unroll
        for (int c0 = 0; c0 < E; c0 += CH) {
            uint32_t x[CH / 4], q[CH / 4];
            load_b8<CH>(xrow + c0, x);
            load_b8<CH>(prow + c0, q);
#pragma unroll
            for (int j = 0; j < CH / 4; ++j) {
                const uint32_t f0 = s * 0x10001u + __byte_perm(x[j], 0u, 0x4044u);
                acc = __dp2a_lo(f0, q[j], acc);
                s = __dp4a(x[j], 0x00000101u, s);
                const uint32_t f1 = s * 0x10001u + __byte_perm(x[j], 0u, 0x4244u);
                acc = __dp2a_hi(f1, q[j], acc);
                s = __dp4a(x[j], 0x01010000u, s);
            }
        }
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
#if CDD_SAG_PREFETCH
    uint32_t rr[E / 2], mw[E / 4], xw[E / 4], gw[E / 2];
    load_ab16<E>(reinterpret_cast<const uint8_t*>(ch.ab()) + l * C::AS, rr);
    load_b8<E>(ch.pb() + l * C::PS, mw);
    load_b8<E>(ch.xb() + l * C::PS, xw);
    load_ab16<E>(reinterpret_cast<const uint8_t*>(ch.gh()) + l * C::GS, gw);
#endif
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
    load_spread<SPR>(ch, Lk, e0, lane_in, rv);
#pragma unroll
    for (int i = 0; i < SPR; ++i) {
        const int k = Lk * E + e0 + i;
        mv[i] = lane_in ? ch.pb()[C::pb_b(k)] : 0u;
        xv[i] = lane_in ? ch.xb()[C::pb_b(k)] : 0u;
        gv[i] = lane_in ? ch.gh()[C::gh_h(k)] : 0u;
    }
    uint32_t lsum = 0;
#pragma unroll
    for (int i = 0; i < SPR; ++i) lsum += rv[i];
    uint32_t ex = gscan<G>(lsum) - lsum;
    // The elements at or before k0 are those with A_excl + B_excl <= Btot (a prefix of the row);
    // each of them switches from the tardy weight wB to the early weight wA.  Padded positions
    // have M = X = 0 and add nothing, so no index test.
    int32_t corr = 0;
#pragma unroll
    for (int i = 0; i < SPR; ++i) {
        const int32_t wA = (int32_t)(ABbS & 0xffffu) + (int32_t)(ex & 0xffffu);
        const int32_t Bex = (int32_t)(ABbS >> 16) + (int32_t)(ex >> 16);
        const int32_t wB = Btot - Bex;
        const int32_t g = (int32_t)gv[i];
        const int32_t c = (int32_t)mv[i] * (wA - wB) + (int32_t)xv[i] * (min(wA, g) - min(wB, g));
        corr += (wA + Bex <= Btot) ? c : 0;
        ex += rv[i];
    }

    // pass 2: pairs of weights as 16-bit halves, w2 = base2 +- f2
    const bool amode = l < Lk;
    const uint32_t base = (uint32_t)(amode ? Ab : (Btot - Bb));
    const uint32_t base2 = base | (base << 16);
    const uint32_t sgn = amode ? 1u : 0xffffffffu;
    const uint32_t psel = amode ? 0x4044u : 0x4144u;
    const uint32_t wsum = amode ? 0x00010001u : 0x01000100u;
    uint32_t s = 0, acc = 0;
#if CDD_SAG_PREFETCH
#pragma unroll
    for (int j = 0; j < E / 2; ++j) {
        const uint32_t f2 = s * 0x10001u + __byte_perm(rr[j], 0u, psel);
        const uint32_t w2 = f2 * sgn + base2;
        const uint32_t mn2 = __vminu2(w2, gw[j]);
        if (j & 1) {
            acc = __dp2a_hi(w2, mw[j >> 1], acc);
            acc = __dp2a_hi(mn2, xw[j >> 1], acc);
        } else {
            acc = __dp2a_lo(w2, mw[j >> 1], acc);
            acc = __dp2a_lo(mn2, xw[j >> 1], acc);
        }
        s = __dp4a(rr[j], wsum, s);
    }
#else
    const uint8_t* arow = reinterpret_cast<const uint8_t*>(ch.ab()) + l * C::AS;
    const uint8_t* grow = reinterpret_cast<const uint8_t*>(ch.gh()) + l * C::GS;
    const uint8_t* mrow = ch.pb() + l * C::PS;
    const uint8_t* xrow = ch.xb() + l * C::PS;
    constexpr int CH = E >= 16 ? 16 : E;  // positions per chunk
#pragma unroll
    for (int c0 = 0; c0 < E; c0 += CH) {
        uint32_t r[CH / 2], g2[CH / 2], mq[CH / 4], xq[CH / 4];
        load_ab16<CH>(arow + 2 * c0, r);
        load_ab16<CH>(grow + 2 * c0, g2);
        load_b8<CH>(mrow + c0, mq);
        load_b8<CH>(xrow + c0, xq);
#pragma unroll
        for (int j = 0; j < CH / 2; ++j) {
            const uint32_t f2 = s * 0x10001u + __byte_perm(r[j], 0u, psel);
            const uint32_t w2 = f2 * sgn + base2;
            const uint32_t mn2 = __vminu2(w2, g2[j]);
            if (j & 1) {
                acc = __dp2a_hi(w2, mq[j >> 1], acc);
                acc = __dp2a_hi(mn2, xq[j >> 1], acc);
            } else {
                acc = __dp2a_lo(w2, mq[j >> 1], acc);
                acc = __dp2a_lo(mn2, xq[j >> 1], acc);
            }
            s = __dp4a(r[j], wsum, s);
        }
    }
#endif
    return (int32_t)gsum<G>(acc + (uint32_t)corr);
}

}  // namespace cdd
