// device_common.cuh -- device-side building blocks of the sm_100a hot path.
//
//  * Philox4x32-10 counter-based RNG (replaces the paper's cuRand calls) with the
//    counter layout of DESIGN.md so every random draw is replayable;
//  * det_exp: the deterministic exp of the Metropolis test (Alg. 1 line 7), explicit
//    round-to-nearest double operations only (no FMA contraction);
//  * packed 32-bit job records and the group-parallel O(n) evaluators for CDD and
//    UCDDCP -- see DESIGN.md "Evaluator" for the derivation.
#pragma once
#include <cstdint>

#include "internal.h"

namespace cdd {

constexpr uint32_t kFull = 0xffffffffu;

// ------------------------------------------------------------------------------ Philox4x32-10
__device__ __forceinline__ uint4 philox4x32_10(uint4 c, uint32_t k0, uint32_t k1) {
#pragma unroll
    for (int r = 0; r < 10; ++r) {
        if (r) {
            k0 += 0x9E3779B9u;
            k1 += 0xBB67AE85u;
        }
        const uint32_t lo0 = 0xD2511F53u * c.x, hi0 = __umulhi(0xD2511F53u, c.x);
        const uint32_t lo1 = 0xCD9E8D57u * c.z, hi1 = __umulhi(0xCD9E8D57u, c.z);
        c = make_uint4(hi1 ^ c.y ^ k0, lo1, hi0 ^ c.w ^ k1, lo0);
    }
    return c;
}

// counter = (x0, id_lo, id_hi, tag << 16 | sub), key = (seed_lo, seed_hi)
__device__ __forceinline__ uint4 rng_block(uint64_t seed, uint32_t x0, uint64_t id, uint32_t tag,
                                           uint32_t sub) {
    return philox4x32_10(make_uint4(x0, (uint32_t)id, (uint32_t)(id >> 32), (tag << 16) | sub),
                         (uint32_t)seed, (uint32_t)(seed >> 32));
}

__device__ __forceinline__ uint32_t bnd(uint32_t w, uint32_t m) { return __umulhi(w, m); }

__device__ __forceinline__ uint32_t word_of(const uint4& v, int i) {
    return i == 0 ? v.x : (i == 1 ? v.y : (i == 2 ? v.z : v.w));
}

// ------------------------------------------------------------------------------ det_exp
// k = rint(x/ln2); r = (x - k ln2_hi) - k ln2_lo; Horner Taylor degree 12; times 2^k.
__device__ __forceinline__ double det_exp(double x) {
    const double inv_ln2 = 1.4426950408889634074;
    const double ln2_hi = 6.93147180369123816490e-01;
    const double ln2_lo = 1.90821492927058770002e-10;
    if (!(x >= -700.0)) return 0.0;
    const double kd = rint(__dmul_rn(x, inv_ln2));
    const double r = __dsub_rn(__dsub_rn(x, __dmul_rn(kd, ln2_hi)), __dmul_rn(kd, ln2_lo));
    const double c[13] = {1.0,           1.0,            1.0 / 2.0,        1.0 / 6.0,
                          1.0 / 24.0,    1.0 / 120.0,    1.0 / 720.0,      1.0 / 5040.0,
                          1.0 / 40320.0, 1.0 / 362880.0, 1.0 / 3628800.0,  1.0 / 39916800.0,
                          1.0 / 479001600.0};
    double p = c[12];
#pragma unroll
    for (int j = 11; j >= 0; --j) p = __dadd_rn(__dmul_rn(p, r), c[j]);
    const long long k = (long long)kd;
    return __dmul_rn(p, __longlong_as_double((k + 1023) << 52));
}

// Metropolis test of Alg. 1 line 7 for delta = E - E_new < 0 (delta >= 0 always accepts).
__device__ __forceinline__ bool metropolis_accept(int64_t delta, double T, uint32_t uw) {
    const double dd = (double)delta;
    if (!(dd >= __dmul_rn(-24.0, T))) return false;  // then delta/T < -23: rejected below anyway
    const double x = __ddiv_rn(dd, T);
    if (!(x >= -23.0)) return false;
    const double u = __dmul_rn(__dadd_rn((double)uw, 0.5), 2.3283064365386962890625e-10);
    return det_exp(x) >= u;
}

// ------------------------------------------------------------------------------ group helpers
template <int G>
__device__ __forceinline__ uint32_t gmask() {
    return G == 32 ? kFull : ((1u << G) - 1u);
}

template <int G>
__device__ __forceinline__ uint32_t group_ballot(bool pred, int gbase) {
    return (__ballot_sync(kFull, pred) >> gbase) & gmask<G>();
}

// Inclusive scan over the first LIMIT lanes of each G-lane segment.  One predicated SHFL.UP + add
// per step: the shuffle's in-range predicate replaces the lane-index compare/select.
template <int G, int LIMIT = G>
__device__ __forceinline__ uint32_t group_incl_scan(uint32_t v, int /*l*/) {
    constexpr uint32_t c = (uint32_t)(32 - G) << 8;
#pragma unroll
    for (int off = 1; off < LIMIT; off <<= 1) {
        asm volatile(
            "{\n\t.reg .pred p;\n\t.reg .b32 t;\n\t"
            "shfl.sync.up.b32 t|p, %0, %1, %2, 0xffffffff;\n\t"
            "@p add.u32 %0, %0, t;\n\t}"
            : "+r"(v)
            : "r"(off), "r"(c));
    }
    return v;
}

template <int G>
__device__ __forceinline__ int32_t group_sum(int32_t v) {
    if constexpr (G == 32) {
        return (int32_t)__reduce_add_sync(kFull, (uint32_t)v);
    } else {
#pragma unroll
        for (int off = G / 2; off > 0; off >>= 1) v += __shfl_xor_sync(kFull, v, off, G);
        return v;
    }
}

// Sum of a lane's E packed records with two independent 3-input add chains.
template <int E>
__device__ __forceinline__ uint32_t lane_total(const uint32_t (&r)[E]) {
    if constexpr (E == 1) {
        return r[0];
    } else {
        uint32_t a0 = 0, a1 = 0;
#pragma unroll
        for (int i = 0; i + 1 < E; i += 2) {
            if ((i >> 1) & 1)
                a1 += r[i] + r[i + 1];
            else
                a0 += r[i] + r[i + 1];
        }
        return a0 + a1;
    }
}

// highest set bit index (x != 0)
__device__ __forceinline__ int hibit(uint32_t x) { return 31 - __clz(x); }

// ------------------------------------------------------------------------------ evaluators
// Positions k = l*E + i of the group's sequence live in lane l's registers rec[i] (packed job
// records, 0 for k >= n).  `elem(k)` re-reads the record at position k (used for the one lane
// that holds the due-date boundary).  All G lanes of the group must call with the same n/d.
//
// CDD.  With S_k = sum_{j<k}(a_j+b_j) and Btot = sum b, the breakpoint index
// k0 = max{k : S_k <= Btot} is where Theorem 1's sign change happens; the optimal
// due-date position is D = min(C_{k0}, d) (start at t=0 when C_{k0} > d) and the penalty is
// F(D) = sum_k max(a_k (D - C_k), b_k (C_k - D)).  F is evaluated as F(C_{m'}) (m' = last position
// before the boundary lane: early weights A_{j-1} left of it, tardy weights B_j right of it) plus
// the integral of F' over the boundary lane, computed one element per lane.
template <int G, int E, class Elem>
__device__ __forceinline__ int32_t eval_cdd(const uint32_t (&rec)[E], int l, int gbase, int n,
                                            int32_t d, const RecLayout& L, Elem&& elem) {
    const uint32_t tot = lane_total<E>(rec);
    const uint32_t tP = tot & L.pmask;
    const uint32_t tAB = ((tot >> L.sa) & L.amask) | ((tot >> L.sb) << 16);
    const uint32_t iP = group_incl_scan<G>(tP, l);
    const uint32_t iAB = group_incl_scan<G>(tAB, l);
    const int32_t Pb = (int32_t)(iP - tP);
    const uint32_t ABb = iAB - tAB;
    const int32_t Ab = (int32_t)(ABb & 0xffffu), Bb = (int32_t)(ABb >> 16);
    const int32_t Btot = (int32_t)(__shfl_sync(kFull, iAB, G - 1, G) >> 16);
    const bool lane_valid = l * E < n;
    const int Lk = hibit(group_ballot<G>(lane_valid && (Ab + Bb <= Btot), gbase));
    const int Lt = hibit(group_ballot<G>(lane_valid && (Pb <= d), gbase));
    const int Ls = min(Lk, Lt);

    // boundary lane Ls, one element per lane
    const int kb = Ls * E + l;
    const bool ev = (l < E) && (kb < n);
    const uint32_t r = ev ? elem(kb) : 0u;
    const uint32_t ex = group_incl_scan<G, E>(r, l) - r;
    const int32_t PbS = __shfl_sync(kFull, Pb, Ls, G);
    const uint32_t ABbS = __shfl_sync(kFull, ABb, Ls, G);
    const int32_t pj = (int32_t)(r & L.pmask);
    const int32_t Cex = PbS + (int32_t)(ex & L.pmask);
    const int32_t Sex = (int32_t)(ABbS & 0xffffu) + (int32_t)((ex >> L.sa) & L.amask) +
                        (int32_t)(ABbS >> 16) + (int32_t)(ex >> L.sb);
    const uint32_t bke = group_ballot<G>(ev && (Sex <= Btot), gbase);
    const int32_t Ck0 = __shfl_sync(kFull, Cex + pj, hibit(bke | 1u), G);
    const int32_t D = (Ls == Lk) ? min(Ck0, d) : d;
    const int32_t corr = ev ? (Sex - Btot) * min(pj, max(0, D - Cex)) : 0;

    // F(C_{m'}) = sum_j p_j * (j in early lanes ? A_{j-1} : B_j)
    const bool amode = l < Ls;
    const int sh = amode ? L.sa : L.sb;
    const uint32_t mk = amode ? L.amask : kFull;
    uint32_t s = 0, acc = 0;
#pragma unroll
    for (int i = 0; i < E; ++i) {
        acc += (rec[i] & L.pmask) * ((s >> sh) & mk);
        s += rec[i];
    }
    const int32_t base = amode ? Ab : (Btot - Bb);
    const int32_t contrib = base * (int32_t)tP + (amode ? (int32_t)acc : -(int32_t)acc) + corr;
    return group_sum<G>(contrib);
}

// UCDDCP, d >= sum p so the due-date position is C_{k0} (Property 1).  Each job pays
// its weight w_j (A_{j-1} early/on-time, B_j tardy) per unit of its minimum time M_j and
// min(w_j, gamma_j) per unit of its compressible part X_j = P_j - M_j (Property 2).
template <int G, int E, class Elem>
__device__ __forceinline__ int32_t eval_ucddcp(const uint32_t (&rec)[E], int l, int gbase, int n,
                                               const RecLayout& L, Elem&& elem) {
    const uint32_t tot = lane_total<E>(rec);
    const uint32_t tAB = (tot & L.amask) | (((tot >> L.sb) & L.bmask) << 16);
    const uint32_t iAB = group_incl_scan<G>(tAB, l);
    const uint32_t ABb = iAB - tAB;
    const int32_t Ab = (int32_t)(ABb & 0xffffu), Bb = (int32_t)(ABb >> 16);
    const int32_t Btot = (int32_t)(__shfl_sync(kFull, iAB, G - 1, G) >> 16);
    const bool lane_valid = l * E < n;
    const int Lk = hibit(group_ballot<G>(lane_valid && (Ab + Bb <= Btot), gbase));

    const int kb = Lk * E + l;
    const bool ev = (l < E) && (kb < n);
    const uint32_t r = ev ? elem(kb) : 0u;
    const uint32_t ex = group_incl_scan<G, E>(r, l) - r;
    const uint32_t ABbS = __shfl_sync(kFull, ABb, Lk, G);
    const int32_t Aex = (int32_t)(ABbS & 0xffffu) + (int32_t)(ex & L.amask);
    const int32_t Bex = (int32_t)(ABbS >> 16) + (int32_t)((ex >> L.sb) & L.bmask);
    const int ik = hibit(group_ballot<G>(ev && (Aex + Bex <= Btot), gbase) | 1u);
    int32_t corr = 0;
    {
        const int32_t m = (int32_t)((r >> L.sm) & L.mmask), x = (int32_t)((r >> L.sx) & L.xmask);
        const int32_t g = (int32_t)(r >> L.sg);
        const int32_t wA = Aex, wB = Btot - Bex;
        if (ev && l <= ik) corr = m * (wA - wB) + x * (min(wA, g) - min(wB, g));
    }
    const bool amode = l < Lk;
    const int sh = amode ? 0 : L.sb;
    const uint32_t mk = amode ? L.amask : L.bmask;
    const int32_t base = amode ? Ab : (Btot - Bb);
    const int32_t sgn = amode ? 1 : -1;
    uint32_t s = 0;
    int32_t acc = 0;
#pragma unroll
    for (int i = 0; i < E; ++i) {
        const uint32_t v = rec[i];
        const int32_t w = base + sgn * (int32_t)((s >> sh) & mk);
        const int32_t m = (int32_t)((v >> L.sm) & L.mmask), x = (int32_t)((v >> L.sx) & L.xmask);
        const int32_t g = (int32_t)(v >> L.sg);
        acc += m * w + x * min(w, g);
        s += v;
    }
    return group_sum<G>(acc + corr);
}

// ------------------------------------------------------------------------------ smem layout
// Per-chain record array: position k at word swz(k).  Rows of 32 words; the 16-byte chunk index
// within a row is XORed with the row index, so the lane-contiguous LDS.128 reads of the
// evaluator (lane l reads chunk v of positions [l*E, l*E+E)) are bank-conflict free.
__device__ __forceinline__ int swz(int k) {
    return (k & ~31) | ((((k >> 2) ^ (k >> 5)) & 7) << 2) | (k & 3);
}

template <int E>
__device__ __forceinline__ void load_records(const uint32_t* rec, int lane, uint32_t (&r)[E]) {
    if constexpr (E >= 4) {
#pragma unroll
        for (int v = 0; v < E / 4; ++v) {
            const uint4 x = *reinterpret_cast<const uint4*>(rec + swz(lane * E + 4 * v));
            r[4 * v + 0] = x.x;
            r[4 * v + 1] = x.y;
            r[4 * v + 2] = x.z;
            r[4 * v + 3] = x.w;
        }
    } else if constexpr (E == 2) {
        const uint2 x = *reinterpret_cast<const uint2*>(rec + swz(lane * 2));
        r[0] = x.x;
        r[1] = x.y;
    } else {
        r[0] = rec[swz(lane)];
    }
}

}  // namespace cdd
