// sa_impl.cuh -- the SA kernels shared by the translation units of libcdd's SA (sa.cu: warp per
// chain and the host dispatch; sag_*.cu: the group kernel per problem / trace / move variant, so
// that nvcc compiles the many (G, E) instantiations in parallel).  Everything here is in an
// anonymous namespace: each translation unit owns the copies it instantiates.
#pragma once
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>
#include <cstdlib>

#include "chain.cuh"
#include "device_common.cuh"
#include "internal.h"
#include "peer.cuh"
#include "sa_group.cuh"
#include "sa_nib.cuh"

namespace cdd {
namespace {

constexpr int kSaWarps = 8;  // warps per CTA of the warp-per-chain kernel (sa.cu)
constexpr int kSaThreads = kSaWarps * 32;

// Moves of steps k0 .. k0+15: even lane 2s holds the sorted positions of step k0+s (Floyd sample of
// P distinct positions, packed 16 bits each), odd lane 2s+1 the slot permutation (2 bits per
// slot) and the uniform word of the Metropolis test.
__device__ __forceinline__ void precompute_moves(uint64_t seed, uint64_t g, uint32_t k0, int lane,
                                                 int n, int P, int move, uint32_t& R0,
                                                 uint32_t& R1) {
    const uint32_t sub = (uint32_t)(lane & 1);
    const uint4 w = rng_block(seed, k0 + (uint32_t)(lane >> 1), g, kTagSa, sub);
    if (sub == 0) {
        if (move == 2) {
            // insertion (R11b): (from, to) uniform over ordered pairs of distinct positions;
            // n < 2: no move (from = to = 0)
            const int from = n >= 2 ? (int)bnd(w.x, (uint32_t)n) : 0;
            int to = n >= 2 ? (int)bnd(w.y, (uint32_t)(n - 1)) : 0;
            to += (n >= 2 && to >= from) ? 1 : 0;
            R0 = (uint32_t)from | ((uint32_t)to << 16);
            R1 = 0x7fff7fffu;
            return;
        }
        int c[4] = {0, 0, 0, 0};
        if (move == 3) {
            // contiguous window of P positions (R11c): already ascending
            const int st = (int)bnd(w.x, (uint32_t)(n - P + 1));
#pragma unroll
            for (int t = 0; t < 4; ++t) c[t] = t < P ? st + t : 0x7fff;
        } else {
#pragma unroll
            for (int t = 0; t < 4; ++t) {
                if (t < P) {
                    const int j = n - P + t;
                    int r = (int)bnd(word_of(w, t), (uint32_t)j + 1u);
#pragma unroll
                    for (int e = 0; e < t; ++e) r = (c[e] == r) ? j : r;
                    c[t] = r;
                }
            }
#pragma unroll
            for (int t = 0; t < 4; ++t)
                if (t >= P) c[t] = 0x7fff;
#pragma unroll
            for (int a = 0; a < 3; ++a)
#pragma unroll
                for (int b = 0; b < 3 - a; ++b)
                    if (c[b] > c[b + 1]) {
                        const int t = c[b];
                        c[b] = c[b + 1];
                        c[b + 1] = t;
                    }
        }
        R0 = (uint32_t)(c[0] & 0xffff) | ((uint32_t)(c[1] & 0xffff) << 16);
        R1 = (uint32_t)(c[2] & 0xffff) | ((uint32_t)(c[3] & 0xffff) << 16);
    } else {
        int s[4] = {0, 1, 2, 3};
        if (move == 1) {
            if (P == 2) {
                s[0] = 1;
                s[1] = 0;
            }
        } else if (move != 2) {  // Pert-FY and window: Fisher-Yates over the P slots
#pragma unroll
            for (int i = 3; i >= 1; --i) {
                if (i <= P - 1) {
                    const int j = (int)bnd(word_of(w, P - 1 - i), (uint32_t)i + 1u);
                    int si = s[0], sj = s[0];
#pragma unroll
                    for (int e = 0; e < 4; ++e) {
                        if (e == i) si = s[e];
                        if (e == j) sj = s[e];
                    }
#pragma unroll
                    for (int e = 0; e < 4; ++e) {
                        if (e == i) s[e] = sj;
                        else if (e == j) s[e] = si;
                    }
                }
            }
        }
        R0 = (uint32_t)s[0] | ((uint32_t)s[1] << 2) | ((uint32_t)s[2] << 4) | ((uint32_t)s[3] << 6);
        R1 = w.w;
    }
}

// Copies the winning chain slot's best sequence to the instance's best buffer.  Chain c ran in
// slot c % slots_total; a slot's best sequence is at slots + slot*stride + best_off.
__global__ void sa_finalize(const unsigned long long* key, const int16_t* slots, int64_t stride,
                            int64_t best_off, int n, uint64_t chain_offset, int64_t slots_total,
                            int16_t* best_perm, int64_t share = 0, int64_t steps = 0, int cpw = 1) {
    const unsigned long long k = *key;
    if (k == ULLONG_MAX) return;
    const uint64_t c = (uint64_t)(uint32_t)(k & 0xffffffffu) - chain_offset;
    // the group that finished chain c: c % slots (round robin), or under the balanced schedule
    // the warp whose share holds the last step of c's quad
    const int64_t sl = share ? (((int64_t)(c / cpw) + 1) * steps - 1) / share * cpw + (int64_t)(c % cpw)
                             : (int64_t)(c % (uint64_t)slots_total);
    const int16_t* src = slots + (size_t)sl * stride + best_off;
    for (int i = threadIdx.x; i < n; i += blockDim.x) best_perm[i] = src[i];
}

// T0 = population std: exact 128-bit moments, N^2 var = N S2 - S1^2, one conversion, one sqrt.
__global__ void t0_reduce_kernel(const int64_t* __restrict__ Z, int64_t N, double* T0) {
    // per thread, then per warp (64-bit shuffles, carry into the high word), then thread 0
    __shared__ unsigned long long s1s[32], s2lo[32], s2hi[32];
    unsigned long long s1 = 0, lo = 0, hi = 0;
    for (int64_t i = threadIdx.x; i < N; i += blockDim.x) {
        const unsigned long long z = (unsigned long long)Z[i];
        s1 += z;
        const unsigned __int128 q = (unsigned __int128)z * z;
        const unsigned long long qlo = (unsigned long long)q, nlo = lo + qlo;
        hi += (unsigned long long)(q >> 64) + (nlo < lo ? 1ull : 0ull);
        lo = nlo;
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
        s1 += __shfl_down_sync(kFull, s1, off);
        const unsigned long long olo = __shfl_down_sync(kFull, lo, off), ohi = __shfl_down_sync(kFull, hi, off);
        const unsigned long long nlo = lo + olo;
        hi += ohi + (nlo < lo ? 1ull : 0ull);
        lo = nlo;
    }
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    if (lane == 0) {
        s1s[wid] = s1;
        s2lo[wid] = lo;
        s2hi[wid] = hi;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned __int128 S1 = 0, S2 = 0;
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) {
            S1 += s1s[w];
            S2 += ((unsigned __int128)s2hi[w] << 64) | s2lo[w];
        }
        const unsigned __int128 num = (unsigned __int128)(unsigned long long)N * S2 - S1 * S1;
        const double h = (double)(unsigned long long)(num >> 64);
        const double l = (double)(unsigned long long)num;
        const double x = __dadd_rn(__dmul_rn(h, 18446744073709551616.0), l);
        *T0 = __ddiv_rn(__dsqrt_rn(x), (double)N);
    }
}

// ------------------------------------------------------------------ CDD: G lanes per chain
#ifndef CDD_SAG_MIN_BLOCKS
#define CDD_SAG_MIN_BLOCKS 6  // 6 CTAs x 4 warps per SM -> <= 80 registers
#endif
// resident CTAs the register budget is sized for: as many as shared memory admits, at most
// CDD_SAG_MIN_BLOCKS (UCDDCP at E = 64 holds 58 KB of chains per CTA -> 3)
// the chain layout of a group-kernel variant: MV = 2 is the nibble layout with sub-block
// summaries (sa_nib.cuh; CDD, moves of <= 4 positions, G = 8, E = 128 or 64)
template <int G, int E, bool UCD, int MV>
struct SagChainT {
    using type = GChain<G, E, UCD>;
};
template <int G, int E>
struct SagChainT<G, E, false, 2> {
    using type = GChainNib<G, E>;
};
template <int G, int E, bool UCD, int MV>
using SagChain = typename SagChainT<G, E, UCD, MV>::type;

template <int G, int E, bool UCD, int MV = 0>
constexpr int sag_min_blocks() {
    constexpr int per_cta = 4 * (32 / G) * SagChain<G, E, UCD, MV>::BYTES + 2048;
    constexpr int fit = (228 * 1024) / per_cta;
    return fit < 1 ? 1 : (fit < CDD_SAG_MIN_BLOCKS ? fit : CDD_SAG_MIN_BLOCKS);
}
constexpr int kGWarps = 4;
constexpr int kGThreads = kGWarps * 32;

struct SaGArgs {
    ChainTables T;
    int n;
    int32_t d;
    int64_t chains;
    uint32_t steps;
    double mu;
    double T0;
    const double* T0_ptr;
    double* T0_out;
    int pert, move;
    uint64_t seed, chain_offset;
    int16_t* slots;  // [groups][3 or 4][NP]: current ids, scratch best, group best (, group final)
    unsigned long long* best_key;
    int64_t *trace, *chain_best, *chain_final;
    // synchronous SA (sa_sync_*): every chain starts from init_perm (NULL: its own random state),
    // move counters start at step0, and the minimum (final penalty << 32 | id) goes to final_key
    // with the final state in the group's 4th slot
    const int16_t* init_perm;
    uint32_t step0;
    unsigned long long* final_key;
    // asynchronous SA with the caller's initial sequences (row c at c * init_ld; NULL: random)
    const int16_t* init_user;
    int64_t init_ld;
    int* err;
    // synchronous SA, levels j >= 1: the shared-memory image of a chain holding s^min_{j-1}
    // (records, padding, lane totals; GChain::BYTES) and its ids (NP, zero-padded), built once per
    // level by sync_level_prepare; every chain copies them instead of re-gathering the records
    const uint8_t* init_image;
    const int16_t* init_ids;
    // balanced schedule (share > 0): warp w runs (quad, step) work [w*share, (w+1)*share) of the
    // quad-major space; chains split between two warps hand their state over through `hand`
    int64_t share;
    uint8_t* hand;
    // CDD: the evaluator's quad level (Instance::quad_level, sa_group.cuh)
    int quad;
};

// State of one chain handed from the warp that ran its first steps to the warp finishing it.
struct SaHand {
    int32_t Ecur, Ebest, cur_is_best, pad;
    double T;
};
// per warp: a 16-byte ready flag, CPW records, then per chain the current and best ids (2 NP)
__host__ __device__ constexpr size_t hand_warp_bytes(int np, int cpw) {
    return (16 + (size_t)cpw * sizeof(SaHand) + (size_t)cpw * 2 * np * sizeof(int16_t) + 255) / 256 * 256;
}

// Alg. 1 line 1 for the group's chain: Fisher-Yates of the identity (ids staged in the AB area,
// Philox words in batches of 4G behind them, swaps on the group's lane 0), ids to the global
// current slot, then the records and the per-lane totals.
// This lane's totals of its row: alpha | beta << 16 and P (UCDDCP: M).
template <int G, int E, bool UCD>
__device__ __forceinline__ uint2 gchain_lane_totals(const GChain<G, E, UCD>& ch, int l) {
    using C = GChain<G, E, UCD>;
    uint32_t tAB = 0, tP = 0;
    if constexpr (UCD) {
        for (int i = 0; i < E; ++i) {
            tAB += ab_wide(ch.ab()[l * (C::AS / 2) + i]);
            tP += ch.pb()[l * C::PS + i];
        }
    } else {
        const uint8_t* ar = ch.a8() + l * C::RS;
        const uint8_t* br = ch.b8() + l * C::RS;
        const uint8_t* pr = ch.pb() + l * C::RS;
        uint32_t ta = 0, tb = 0;
        for (int i = 0; i < E; i += 4) {
            ta = __dp4a(*reinterpret_cast<const uint32_t*>(ar + i), 0x01010101u, ta);
            tb = __dp4a(*reinterpret_cast<const uint32_t*>(br + i), 0x01010101u, tb);
            tP = __dp4a(*reinterpret_cast<const uint32_t*>(pr + i), 0x01010101u, tP);
        }
        tAB = ta | (tb << 16);
    }
    return make_uint2(tAB, tP);
}

// Alg. 1 line 1, the sequence: Fisher-Yates of the identity (or the caller's sequence) staged in
// the chain's shared memory at base (NP ids then 4G Philox words), copied to the global slot cur.
template <int G, int NP>
__device__ void gchain_ids(uint8_t* base, int16_t* cur, int n, uint64_t seed, uint64_t g, int l,
                           const int16_t* init, int* err, uint32_t tag) {
    uint16_t* ids = reinterpret_cast<uint16_t*>(base);
    uint32_t* words = reinterpret_cast<uint32_t*>(ids + NP);
    if (init)
        for (int k = l; k < NP; k += G) {
            uint32_t v = k < n ? (uint16_t)init[k] : 0u;
            if (v >= (uint32_t)n) {  // only a caller's sequence can hold one
                if (err) atomicOr(err, 1);
                v = 0;
            }
            ids[k] = (uint16_t)v;
        }
    else
        for (int k = l; k < NP; k += G) ids[k] = (uint16_t)(k < n ? k : 0);
    const int nw = init ? 0 : n - 1;
    for (int r0 = 0; r0 < nw; r0 += 4 * G) {
        __syncwarp();
        const int b = r0 / 4 + l;
        if (4 * b < nw) reinterpret_cast<uint4*>(words)[l] = rng_block(seed, (uint32_t)b, g, tag, 0);
        __syncwarp();
        if (l == 0) {
            // the swaps are serial through ids[]; their words are loaded 4 at a time up front so
            // that only the ids[j] load -> stores chain stays on the critical path
            const int r1 = min(nw, r0 + 4 * G);
            int q = r0;
            for (; q + 4 <= r1; q += 4) {
                const uint4 w4 = *reinterpret_cast<const uint4*>(words + (q - r0));
                const uint32_t wv[4] = {w4.x, w4.y, w4.z, w4.w};
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const int i = n - 1 - (q + u);
                    const uint32_t j = bnd(wv[u], (uint32_t)i + 1u);
                    const uint16_t t = ids[i];
                    ids[i] = ids[j];
                    ids[j] = t;
                }
            }
            for (; q < r1; ++q) {
                const int i = n - 1 - q;
                const uint32_t j = bnd(words[q - r0], (uint32_t)i + 1u);
                const uint16_t t = ids[i];
                ids[i] = ids[j];
                ids[j] = t;
            }
        }
    }
    __syncwarp();
    for (int k = l; k < NP; k += G) cur[k] = (int16_t)ids[k];
    __syncwarp();
}

template <int G, int E, bool UCD>
__device__ void gchain_init(const GChain<G, E, UCD>& ch, int16_t* cur, int n, uint64_t seed,
                            uint64_t g, int l, const ChainTables& T, const int16_t* init, int* err,
                            uint32_t tag = kTagSaInit) {
    using C = GChain<G, E, UCD>;
    constexpr int NP = C::NP;
    // staging: NP ids then 4G Philox words, 2 NP + 16 G bytes <= C::BYTES (static_assert there)
    gchain_ids<G, NP>(ch.base, cur, n, seed, g, l, init, err, tag);
    // records in batches of 8 positions per lane: 8 independent id loads, then 8 independent
    // table loads (E is a multiple of 8, so NP is a multiple of 8 G)
    for (int k0 = l; k0 < NP; k0 += 8 * G) {
        int jj[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) jj[u] = k0 + u * G < n ? cur[k0 + u * G] : 0;
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const int k = k0 + u * G;
            const bool v = k < n;
            const uint32_t ab = v ? __ldg(T.ab16 + jj[u]) : 0u;
            ch.pb()[C::pb_b(k)] = v ? __ldg(T.p + jj[u]) : (uint8_t)0;
            if constexpr (UCD) {
                ch.ab()[C::ab_h(k)] = (uint16_t)ab;
                ch.xb()[C::pb_b(k)] = v ? __ldg(T.x + jj[u]) : (uint8_t)0;
                ch.gh()[C::gh_h(k)] = v ? __ldg(T.g + jj[u]) : (uint16_t)0;
            } else {
                ch.a8()[C::rb(k)] = (uint8_t)ab;
                ch.b8()[C::rb(k)] = (uint8_t)(ab >> 8);
            }
        }
    }
    __syncwarp();
    ch.tot()[l] = gchain_lane_totals(ch, l);
    __syncwarp();
}

// The nibble layout (sa_nib.cuh): records alpha | beta << 4 and P, lane totals, and the summaries
// of the lane's 8 sub-blocks.
template <int G, int E, bool UCD>
__device__ void gchain_init(const GChainNib<G, E>& ch, int16_t* cur, int n, uint64_t seed,
                            uint64_t g, int l, const ChainTables& T, const int16_t* init, int* err,
                            uint32_t tag = kTagSaInit) {
    using C = GChainNib<G, E>;
    constexpr int NP = C::NP;
    gchain_ids<G, NP>(ch.base, cur, n, seed, g, l, init, err, tag);
    for (int k0 = l; k0 < NP; k0 += 8 * G) {
        int jj[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) jj[u] = k0 + u * G < n ? cur[k0 + u * G] : 0;
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const int k = k0 + u * G;
            const bool v = k < n;
            const uint32_t ab = v ? __ldg(T.ab16 + jj[u]) : 0u;
            ch.ab()[k] = (uint8_t)((ab & 15u) | ((ab >> 4) & 0xf0u));
            ch.pb()[k] = v ? __ldg(T.p + jj[u]) : (uint8_t)0;
        }
    }
    __syncwarp();
    uint32_t tA = 0, tB = 0, tP = 0;
#pragma unroll
    for (int b = 0; b < C::NSB; ++b) {
        const uint2 sm = nib_summary(ch, l * E + C::SB * b);
        ch.sum()[b * G + l] = sm;
        tA += sm.y & 0xffu;
        tB += (sm.y >> 8) & 0xffu;
        tP += sm.y >> 16;
    }
    ch.tot()[l] = make_uint2(tA | (tB << 16), tP);
    __syncwarp();
}

template <int G, int E, bool UCD>
__device__ __forceinline__ int32_t gchain_eval(const GChainNib<G, E>& ch, int l, int gbase, int n,
                                               int32_t d, uint2 t, int quad) {
    return gchain_eval_nib<G, E>(ch, l, gbase, n, d, t.x, t.y, quad);
}

template <int G, int E, bool UCD>
__device__ __forceinline__ uint2 pos_read(const GChainNib<G, E>& ch, int k) {
    return make_uint2(nib_read(ch, k), 0u);
}

template <int G, int E, bool UCD>
__device__ __forceinline__ void pos_write(const GChainNib<G, E>& ch, int k, uint2 v) {
    nib_write(ch, k, v.x);
}

template <int G, int E, bool UCD>
__device__ __forceinline__ int32_t gchain_eval(const GChain<G, E, UCD>& ch, int l, int gbase, int n,
                                               int32_t d, uint2 t, int quad) {
    if constexpr (UCD)
        return gchain_eval_ucddcp<G, E>(ch, l, gbase, n, t.x);
    else
        return gchain_eval_cdd<G, E>(ch, l, gbase, n, d, t.x, t.y, quad);
}

// The data of one position, packed for shuffles: u0 = alpha|beta<<8 | P << 16 (CDD) or
// alpha|beta<<8 | gamma << 16 (UCDDCP); u1 = M | X << 8 (UCDDCP only).
template <int G, int E, bool UCD>
__device__ __forceinline__ uint2 pos_read(const GChain<G, E, UCD>& ch, int k) {
    using C = GChain<G, E, UCD>;
    uint2 v;
    if constexpr (UCD) {
        v.x = (uint32_t)ch.ab()[C::ab_h(k)] | ((uint32_t)ch.gh()[C::gh_h(k)] << 16);
        v.y = (uint32_t)ch.pb()[C::pb_b(k)] | ((uint32_t)ch.xb()[C::pb_b(k)] << 8);
    } else {
        const int i = C::rb(k);
        v.x = (uint32_t)ch.a8()[i] | ((uint32_t)ch.b8()[i] << 8) | ((uint32_t)ch.pb()[i] << 16);
        v.y = 0;
    }
    return v;
}

template <int G, int E, bool UCD>
__device__ __forceinline__ void pos_write(const GChain<G, E, UCD>& ch, int k, uint2 v) {
    using C = GChain<G, E, UCD>;
    if constexpr (UCD) {
        ch.ab()[C::ab_h(k)] = (uint16_t)v.x;
        ch.gh()[C::gh_h(k)] = (uint16_t)(v.x >> 16);
        ch.pb()[C::pb_b(k)] = (uint8_t)v.y;
        ch.xb()[C::pb_b(k)] = (uint8_t)(v.y >> 8);
    } else {
        const int i = C::rb(k);
        ch.a8()[i] = (uint8_t)v.x;
        ch.b8()[i] = (uint8_t)(v.x >> 8);
        ch.pb()[i] = (uint8_t)(v.x >> 16);
    }
}

// ---- insertion move (R11b) on the group layout: rotation by one position of [lo, hi] --
// left: new[k] = old[k+1] (lo <= k < hi), new[hi] = old[lo]; right: new[k] = old[k-1]
// (lo < k <= hi), new[lo] = old[hi].  Chunks of 8 positions (16 B of a 16-bit array, 8 B of a byte
// array; E is a multiple of 8, so a chunk never straddles a lane row): the lane of the group that
// owns a chunk loads it and the one neighbouring element, shifts it with funnel shifts and keeps
// the positions outside the rotated range by a mask.  Chunks advance in the rotation's direction,
// G per round, every load of a round before its stores.

// bits e of the chunk at c whose position is rotated: [lo, hi) (left) or (lo, hi] (right)
__device__ __forceinline__ uint32_t rot_mask8(int c, int lo, int hi, bool left) {
    const int a = max((left ? lo : lo + 1) - c, 0), b = min((left ? hi : hi + 1) - c, 8);
    return a < b ? ((1u << b) - 1u) & ~((1u << a) - 1u) : 0u;
}
// 16-bit lane masks of a word from 2 mask bits, byte masks from 4 mask bits
__device__ __forceinline__ uint32_t half_mask(uint32_t v2) { return ((v2 * 0x8001u) & 0x10001u) * 0xffffu; }
__device__ __forceinline__ uint32_t byte_mask(uint32_t v4) { return ((v4 * 0x00204081u) & 0x01010101u) * 0xffu; }

// chunk of 8 16-bit elements; nb = the element after (left) / before (right) the chunk
__device__ __forceinline__ uint4 rot16(uint4 A, uint32_t nb, bool left, uint32_t m8) {
    uint4 S;
    if (left) {
        S.x = __funnelshift_r(A.x, A.y, 16);
        S.y = __funnelshift_r(A.y, A.z, 16);
        S.z = __funnelshift_r(A.z, A.w, 16);
        S.w = __funnelshift_r(A.w, nb, 16);
    } else {
        S.x = __funnelshift_l(nb << 16, A.x, 16);
        S.y = __funnelshift_l(A.x, A.y, 16);
        S.z = __funnelshift_l(A.y, A.z, 16);
        S.w = __funnelshift_l(A.z, A.w, 16);
    }
    uint4 R;
    R.x = (S.x & half_mask(m8 & 3u)) | (A.x & ~half_mask(m8 & 3u));
    R.y = (S.y & half_mask((m8 >> 2) & 3u)) | (A.y & ~half_mask((m8 >> 2) & 3u));
    R.z = (S.z & half_mask((m8 >> 4) & 3u)) | (A.z & ~half_mask((m8 >> 4) & 3u));
    R.w = (S.w & half_mask(m8 >> 6)) | (A.w & ~half_mask(m8 >> 6));
    return R;
}
// chunk of 8 byte elements
__device__ __forceinline__ uint2 rot8(uint2 A, uint32_t nb, bool left, uint32_t m8) {
    uint2 S;
    if (left) {
        S.x = __funnelshift_r(A.x, A.y, 8);
        S.y = __funnelshift_r(A.y, nb, 8);
    } else {
        S.x = __funnelshift_l(nb << 24, A.x, 8);
        S.y = __funnelshift_l(A.x, A.y, 8);
    }
    uint2 R;
    R.x = (S.x & byte_mask(m8 & 15u)) | (A.x & ~byte_mask(m8 & 15u));
    R.y = (S.y & byte_mask(m8 >> 4)) | (A.y & ~byte_mask(m8 >> 4));
    return R;
}

// CDD byte rows in chunks of 16 positions (one 16-byte word per row; E a multiple of 16): half
// the rounds of the 8-position chunks, and chunks wholly inside the range skip the masks.
__device__ __forceinline__ uint32_t rot_mask16(int c, int lo, int hi, bool left) {
    const int a = max((left ? lo : lo + 1) - c, 0), b = min((left ? hi : hi + 1) - c, 16);
    return a < b ? ((b >= 32 ? 0xffffffffu : (1u << b) - 1u) & ~((1u << a) - 1u)) : 0u;
}
__device__ __forceinline__ uint4 rot_b16(uint4 A, uint32_t nb, bool left, uint32_t m16) {
    uint4 S;
    if (left) {
        S.x = __funnelshift_r(A.x, A.y, 8);
        S.y = __funnelshift_r(A.y, A.z, 8);
        S.z = __funnelshift_r(A.z, A.w, 8);
        S.w = __funnelshift_r(A.w, nb, 8);
    } else {
        S.x = __funnelshift_l(nb << 24, A.x, 8);
        S.y = __funnelshift_l(A.x, A.y, 8);
        S.z = __funnelshift_l(A.y, A.z, 8);
        S.w = __funnelshift_l(A.z, A.w, 8);
    }
    if (m16 == 0xffffu) return S;
    const uint32_t b0 = byte_mask(m16 & 15u), b1 = byte_mask((m16 >> 4) & 15u), b2 = byte_mask((m16 >> 8) & 15u),
                   b3 = byte_mask(m16 >> 12);
    return make_uint4((S.x & b0) | (A.x & ~b0), (S.y & b1) | (A.y & ~b1), (S.z & b2) | (A.z & ~b2),
                      (S.w & b3) | (A.w & ~b3));
}
template <int G, int E>
__device__ __forceinline__ void group_rotate_rows16(const GChain<G, E, false>& ch, int lo, int hi, bool left,
                                                    bool act, int l) {
    using C = GChain<G, E, false>;
    static_assert(E % 16 == 0, "16-position chunks stay inside a lane row");
    const int c0 = lo & ~15, c1 = hi & ~15;
    const int nch = act && hi > lo ? (c1 - c0) / 16 + 1 : 0;
    const int rounds = (int)__reduce_max_sync(kFull, (uint32_t)((nch + G - 1) / G));
    const int wsrc = left ? lo : hi;
    uint2 wv = make_uint2(0u, 0u);
    if (l == 0 && nch) wv = pos_read<G, E, false>(ch, wsrc);
    for (int r = 0; r < rounds; ++r) {
        const int j = r * G + l;
        const bool v = j < nch;
        const int c = left ? c0 + 16 * j : c1 - 16 * j;
        const uint32_t m16 = v ? rot_mask16(c, lo, hi, left) : 0u;
        const bool nbv = left ? ((m16 >> 15) & 1u) : (m16 & 1u);
        const int kn = left ? c + 16 : c - 1;
        uint4 Ra = make_uint4(0, 0, 0, 0), Rb = Ra, Rp = Ra;
        if (v) {
            const int i = C::rb(c), in = C::rb(kn);
            Ra = *reinterpret_cast<const uint4*>(ch.a8() + i);
            Rb = *reinterpret_cast<const uint4*>(ch.b8() + i);
            Rp = *reinterpret_cast<const uint4*>(ch.pb() + i);
            uint32_t na = 0u, nb = 0u, np = 0u;
            if (nbv) {
                na = ch.a8()[in];
                nb = ch.b8()[in];
                np = ch.pb()[in];
            }
            Ra = rot_b16(Ra, na, left, m16);
            Rb = rot_b16(Rb, nb, left, m16);
            Rp = rot_b16(Rp, np, left, m16);
        }
        __syncwarp();
        if (v && m16) {
            const int i = C::rb(c);
            *reinterpret_cast<uint4*>(ch.a8() + i) = Ra;
            *reinterpret_cast<uint4*>(ch.b8() + i) = Rb;
            *reinterpret_cast<uint4*>(ch.pb() + i) = Rp;
        }
        __syncwarp();
    }
    if (l == 0 && nch) pos_write<G, E, false>(ch, left ? hi : lo, wv);
    __syncwarp();
}

// Rotates the records (IDS = false: ab, p / M, X, gamma in shared memory) or the job ids of the
// group's current slot (IDS = true, global) over [lo, hi].  act: this group has a move (the other
// groups of the warp run the same number of rounds with nothing to do).
template <int G, int E, bool UCD, bool IDS>
__device__ __forceinline__ void group_rotate(const GChain<G, E, UCD>& ch, int16_t* ids, int lo, int hi,
                                             bool left, bool act, int l) {
    using C = GChain<G, E, UCD>;
    if constexpr (!IDS && !UCD && E % 16 == 0) {
        group_rotate_rows16<G, E>(ch, lo, hi, left, act, l);
        return;
    }
    const int c0 = lo & ~7, c1 = hi & ~7;
    const int nch = act && hi > lo ? (c1 - c0) / 8 + 1 : 0;
    const int rounds = (int)__reduce_max_sync(kFull, (uint32_t)((nch + G - 1) / G));
    // the wrapped element, read before any store (group lane 0 stores it after the rounds)
    const int wsrc = left ? lo : hi;
    uint2 wv = make_uint2(0u, 0u);
    int16_t wid = 0;
    if (l == 0 && nch) {
        if constexpr (IDS) wid = ids[wsrc];
        else wv = pos_read<G, E, UCD>(ch, wsrc);
    }
    for (int r = 0; r < rounds; ++r) {
        const int j = r * G + l;
        const bool v = j < nch;
        const int c = left ? c0 + 8 * j : c1 - 8 * j;
        const uint32_t m8 = v ? rot_mask8(c, lo, hi, left) : 0u;
        // the neighbour is needed iff the chunk's edge position is rotated
        const bool nbv = left ? ((m8 >> 7) & 1u) : (m8 & 1u);
        const int kn = left ? c + 8 : c - 1;
        uint4 A16 = make_uint4(0, 0, 0, 0), G16 = make_uint4(0, 0, 0, 0);
        uint2 P8 = make_uint2(0, 0), X8 = make_uint2(0, 0);
        if (v) {
            if constexpr (IDS) {
                A16 = *reinterpret_cast<const uint4*>(ids + c);
                const uint32_t nb = nbv ? (uint32_t)(uint16_t)ids[kn] : 0u;
                A16 = rot16(A16, nb, left, m8);
            } else if constexpr (UCD) {
                uint8_t* abb = reinterpret_cast<uint8_t*>(ch.ab());
                uint8_t* ghb = reinterpret_cast<uint8_t*>(ch.gh());
                A16 = *reinterpret_cast<const uint4*>(abb + 2 * C::ab_h(c));
                P8 = *reinterpret_cast<const uint2*>(ch.pb() + C::pb_b(c));
                const uint32_t nab = nbv ? (uint32_t)ch.ab()[C::ab_h(kn)] : 0u;
                const uint32_t np8 = nbv ? (uint32_t)ch.pb()[C::pb_b(kn)] : 0u;
                A16 = rot16(A16, nab, left, m8);
                P8 = rot8(P8, np8, left, m8);
                G16 = *reinterpret_cast<const uint4*>(ghb + 2 * C::gh_h(c));
                X8 = *reinterpret_cast<const uint2*>(ch.xb() + C::pb_b(c));
                const uint32_t ng = nbv ? (uint32_t)ch.gh()[C::gh_h(kn)] : 0u;
                const uint32_t nx = nbv ? (uint32_t)ch.xb()[C::pb_b(kn)] : 0u;
                G16 = rot16(G16, ng, left, m8);
                X8 = rot8(X8, nx, left, m8);
            } else {
                // CDD: the alpha, beta and P byte rows (A16.x/.y carry alpha, .z/.w beta)
                const int i = C::rb(c), in = C::rb(kn);
                const uint2 a8 = *reinterpret_cast<const uint2*>(ch.a8() + i);
                const uint2 b8 = *reinterpret_cast<const uint2*>(ch.b8() + i);
                P8 = *reinterpret_cast<const uint2*>(ch.pb() + i);
                const uint2 ra = rot8(a8, nbv ? (uint32_t)ch.a8()[in] : 0u, left, m8);
                const uint2 rbt = rot8(b8, nbv ? (uint32_t)ch.b8()[in] : 0u, left, m8);
                A16 = make_uint4(ra.x, ra.y, rbt.x, rbt.y);
                P8 = rot8(P8, nbv ? (uint32_t)ch.pb()[in] : 0u, left, m8);
            }
        }
        __syncwarp();
        if (v && m8) {
            if constexpr (IDS) {
                *reinterpret_cast<uint4*>(ids + c) = A16;
            } else if constexpr (UCD) {
                *reinterpret_cast<uint4*>(reinterpret_cast<uint8_t*>(ch.ab()) + 2 * C::ab_h(c)) = A16;
                *reinterpret_cast<uint2*>(ch.pb() + C::pb_b(c)) = P8;
                *reinterpret_cast<uint4*>(reinterpret_cast<uint8_t*>(ch.gh()) + 2 * C::gh_h(c)) = G16;
                *reinterpret_cast<uint2*>(ch.xb() + C::pb_b(c)) = X8;
            } else {
                const int i = C::rb(c);
                *reinterpret_cast<uint2*>(ch.a8() + i) = make_uint2(A16.x, A16.y);
                *reinterpret_cast<uint2*>(ch.b8() + i) = make_uint2(A16.z, A16.w);
                *reinterpret_cast<uint2*>(ch.pb() + i) = P8;
            }
        }
        __syncwarp();
    }
    if (l == 0 && nch) {
        const int wdst = left ? hi : lo;
        if constexpr (IDS) ids[wdst] = wid;
        else pos_write<G, E, UCD>(ch, wdst, wv);
    }
    __syncwarp();
}

// Change of lane row l's totals (alpha|beta<<16 wide, P or M) under the rotation of [lo, hi]: the
// row loses the element leaving it and gains the one entering it.  Read before the rotation.
template <int G, int E, bool UCD>
__device__ __forceinline__ uint2 rot_tot_delta(const GChain<G, E, UCD>& ch, int lo, int hi, bool left,
                                               bool act, int l) {
    const int a0 = max(lo, l * E), b0 = min(hi, l * E + E - 1);
    if (!act || a0 > b0 || hi <= lo) return make_uint2(0u, 0u);
    const int ko = left ? a0 : b0;
    const int ki = left ? (b0 < hi ? b0 + 1 : lo) : (a0 > lo ? a0 - 1 : hi);
    const uint2 o = pos_read<G, E, UCD>(ch, ko), i = pos_read<G, E, UCD>(ch, ki);
    const uint32_t po = UCD ? (o.y & 0xffu) : (o.x >> 16), pi = UCD ? (i.y & 0xffu) : (i.x >> 16);
    return make_uint2(ab_wide(i.x & 0xffffu) - ab_wide(o.x & 0xffffu), pi - po);
}

// MV: 0 = moves of <= 4 positions (Pert-FY, swap, window), 1 = insertion (a segment rotation),
// 2 = moves of <= 4 positions on the nibble layout with sub-block summaries (sa_nib.cuh)
template <int G, int E, bool UCD, bool TRACE, int MV>
__global__ void __launch_bounds__(kGThreads, sag_min_blocks<G, E, UCD, MV>()) sa_group_kernel(SaGArgs a) {
    using C = SagChain<G, E, UCD, MV>;
    constexpr int NP = C::NP;
    constexpr int CPW = 32 / G;   // chains per warp
    constexpr int SPG = G / 2;    // steps of moves per precompute
    extern __shared__ __align__(16) uint8_t smem[];
    __shared__ unsigned long long s_key[kGWarps * CPW], s_fkey[kGWarps * CPW];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int grp = lane / G, l = lane % G, gbase = grp * G;
    const C ch{smem + (size_t)(wib * CPW + grp) * C::BYTES};
    const int64_t groups = (int64_t)gridDim.x * kGWarps * CPW;
    const int64_t wglob = (int64_t)blockIdx.x * kGWarps + wib;
    const int64_t wfirst = wglob * CPW;
    const int64_t gg = wfirst + grp;
    int16_t* cur = a.slots + (size_t)gg * (a.final_key ? 4 : 3) * NP;
    int16_t* scratch = cur + NP;
    int16_t* gbest = cur + 2 * NP;
    int16_t* gfinal = cur + 3 * NP;  // synchronous SA only
    unsigned long long gfkey = ULLONG_MAX;
    const int n = a.n;
    const int P = a.move == 1 ? min(2, n) : min(min(a.pert, 4), n);
    const double T0 = a.T0_ptr ? *a.T0_ptr : a.T0;
    if (a.T0_out && gg == 0 && l == 0) *a.T0_out = T0;
    unsigned long long gkey = ULLONG_MAX;

    // One piece of work for the warp's CPW chains c0 .. c0+CPW-1: steps [k0, k1), started fresh
    // (k0 = 0) or resumed from a handoff, finished (k1 = steps) or handed off to warp wglob + 1.
    auto run_piece = [&](int64_t c0, uint32_t k0, uint32_t k1, bool restore, bool hout) {
        const int64_t c = c0 + grp;
        const bool active = c < a.chains;
        const uint64_t g = a.chain_offset + (uint64_t)c;
        const int16_t* s0 = a.init_perm;
        if (!s0 && a.init_user) s0 = a.init_user + (active ? c : a.chains - 1) * a.init_ld;
        // a resumed piece starts from the state its first part handed over (balanced schedule)
        SaHand* hand_rec = nullptr;
        const int16_t* hand_best = nullptr;
        if (restore || hout) {
            uint8_t* hw = a.hand + (size_t)(restore ? wglob : wglob + 1) * hand_warp_bytes(NP, CPW);
            hand_rec = reinterpret_cast<SaHand*>(hw + 16);
            int16_t* hids = reinterpret_cast<int16_t*>(hw + 16 + CPW * sizeof(SaHand)) + (size_t)grp * 2 * NP;
            if (restore) {
                if (lane == 0) {
                    unsigned int v;
                    do {
                        asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(hw) : "memory");
                    } while (v == 0u);
                }
                __syncwarp();
                s0 = hids;
                hand_best = hids + NP;
            }
        }
        if (a.init_image && !restore) {
            // every lane issues its independent 16-byte loads back to back
#pragma unroll 4
            for (int o = l * 16; o < C::BYTES; o += 16 * G)
                *reinterpret_cast<int4*>(ch.base + o) = __ldg(reinterpret_cast<const int4*>(a.init_image + o));
#pragma unroll 4
            for (int o = l * 8; o < NP; o += 8 * G)
                *reinterpret_cast<int4*>(cur + o) = __ldg(reinterpret_cast<const int4*>(a.init_ids + o));
            __syncwarp();
        } else {
            gchain_init<G, E, UCD>(ch, cur, n, a.seed, g, l, a.T, s0, a.err);
        }
        uint2 tt;
        int32_t Ecur, Ebest;
        bool cur_is_best;
        double T;
        if (!restore) {
            tt = ch.tot()[l];
            Ecur = gchain_eval<G, E, UCD>(ch, l, gbase, n, a.d, tt, a.quad);
            Ebest = Ecur;
            cur_is_best = true;
            T = T0;
        } else {
            tt = ch.tot()[l];
            const SaHand h = hand_rec[grp];
            Ecur = h.Ecur;
            Ebest = h.Ebest;
            cur_is_best = h.cur_is_best != 0;
            T = h.T;
            if (!cur_is_best)
                for (int o = l * 8; o < NP; o += 8 * G)
                    *reinterpret_cast<int4*>(scratch + o) = *reinterpret_cast<const int4*>(hand_best + o);
            __syncwarp();
        }
        uint32_t R0 = 0, R1 = 0;
        if (k0 % SPG) precompute_moves(a.seed, g, a.step0 + k0 - k0 % SPG, l, n, P, a.move, R0, R1);
        for (uint32_t k = k0; k < k1; ++k) {
            const int sk = (int)(k % SPG);
            if (sk == 0) precompute_moves(a.seed, g, a.step0 + k, l, n, P, a.move, R0, R1);
            const uint32_t q01 = __shfl_sync(kFull, R0, 2 * sk, G);
            const uint32_t q23 = __shfl_sync(kFull, R1, 2 * sk, G);
            const uint32_t sig = __shfl_sync(kFull, R0, 2 * sk + 1, G);
            const uint32_t uw = __shfl_sync(kFull, R1, 2 * sk + 1, G);
            if constexpr (MV == 1) {
                // Alg. 1 line 5, insertion (R11b): the job at `from` moves to `to`
                const int from = (int)(q01 & 0xffffu), to = (int)(q01 >> 16);
                const int lo = min(from, to), hi = max(from, to);
                const bool left = from < to;
                const uint2 dt = rot_tot_delta<G, E, UCD>(ch, lo, hi, left, true, l);
                group_rotate<G, E, UCD, false>(ch, cur, lo, hi, left, true, l);
                const uint2 tn = make_uint2(tt.x + dt.x, tt.y + dt.y);
                ch.tot()[l] = tn;
                __syncwarp();
                const int32_t En = gchain_eval<G, E, UCD>(ch, l, gbase, n, a.d, tn, a.quad);
                const int32_t delta = Ecur - En;
                const bool acc = delta >= 0 || metropolis_accept(delta, T, uw);
                if (TRACE && active && l == 0)
                    a.trace[c * (int64_t)a.steps + (int64_t)k] =
                        (int64_t)(((uint64_t)(uint32_t)En) << 1) | (acc ? 1 : 0);
                // leaving the best state: the current slot still holds the pre-move sequence
                const bool mat = acc && En > Ebest && cur_is_best;
                if (__any_sync(kFull, mat)) {
                    if (mat)
                        for (int o = l * 8; o < NP; o += 8 * G)
                            *reinterpret_cast<int4*>(scratch + o) = *reinterpret_cast<const int4*>(cur + o);
                    __syncwarp();
                }
                // accepted: the ids follow; rejected: the records rotate back
                group_rotate<G, E, UCD, true>(ch, cur, lo, hi, left, acc, l);
                group_rotate<G, E, UCD, false>(ch, cur, lo, hi, !left, !acc, l);
                if (acc) {
                    tt = tn;
                    if (En <= Ebest) {
                        Ebest = En;
                        cur_is_best = true;
                    } else if (mat) {
                        cur_is_best = false;
                    }
                    Ecur = En;
                } else {
                    ch.tot()[l] = tt;
                }
                __syncwarp();
                T = __dmul_rn(T, a.mu);  // line 10
                continue;
            }
            // Alg. 1 line 5: position q_i receives the job of position q_sigma(i)
            const bool mover = l < P;
            const int myq = mover ? (int)(((l < 2 ? q01 : q23) >> (16 * (l & 1))) & 0xffffu) : 0;
            const uint2 old_v = pos_read<G, E, UCD>(ch, myq);
            // nibble layout: the summary of the mover's sub-block (every mover reads before any
            // writes).  Movers sharing a sub-block store the same value with the same warp
            // instruction (the join below, the restore on rejection), where CUDA keeps exactly one
            // of the lanes' writes -- so the result is that value.  (Electing one writer per
            // sub-block was measured 2.5 % slower.)
            uint2 old_s = make_uint2(0u, 0u);
            int sidx = 0;
            if constexpr (MV == 2) {
                sidx = C::sidx(myq);
                old_s = ch.sum()[sidx];
            }
            // unconditional (myq = 0 for non-movers): consumed only after the evaluation
            const int16_t old_id = cur[myq];
            const int src = (int)((sig >> (2 * (l & 3))) & 3u);
            uint2 new_v;
            new_v.x = __shfl_sync(kFull, old_v.x, src, G);
            new_v.y = UCD ? __shfl_sync(kFull, old_v.y, src, G) : 0u;
            __syncwarp();
            if (mover) {
                pos_write<G, E, UCD>(ch, myq, new_v);
                uint32_t* t2 = reinterpret_cast<uint32_t*>(ch.tot() + myq / E);
                atomicAdd(t2, ab_wide(new_v.x & 0xffffu) - ab_wide(old_v.x & 0xffffu));
                if constexpr (!UCD) atomicAdd(t2 + 1, (new_v.x >> 16) - (old_v.x >> 16));
            }
            __syncwarp();
            if constexpr (MV == 2) {
                // the moved sub-blocks' summaries: mover h (lane h < P) joins its half [k0, k0+8)
                // with lane h + 4's [k0+8, k0+16) (movers sharing a sub-block write equal values)
                const int h = l & 3;
                const int hq = h < P ? (int)(((h < 2 ? q01 : q23) >> (16 * (h & 1))) & 0xffffu) : 0;
                const uint2 part = nib_half(ch, (hq & ~(C::SB - 1)) | (l & 4 ? C::SB / 2 : 0));
                const uint2 other = make_uint2(__shfl_xor_sync(kFull, part.x, 4, G), __shfl_xor_sync(kFull, part.y, 4, G));
                if (mover) ch.sum()[sidx] = nib_join(part, other);
                __syncwarp();
            }
            const uint2 tn = ch.tot()[l];
            // line 6
            const int32_t En = gchain_eval<G, E, UCD>(ch, l, gbase, n, a.d, tn, a.quad);
            // line 7
            const int32_t delta = Ecur - En;
            const bool acc = delta >= 0 || metropolis_accept(delta, T, uw);
            if (TRACE && active && l == 0)
                a.trace[c * (int64_t)a.steps + (int64_t)k] =
                    (int64_t)(((uint64_t)(uint32_t)En) << 1) | (acc ? 1 : 0);
            // leaving the best state: the current slot still holds the pre-move sequence
            const bool mat = acc && En > Ebest && cur_is_best;
            if (__any_sync(kFull, mat)) {
                if (mat)
                    for (int o = l * 8; o < NP; o += 8 * G)
                        *reinterpret_cast<int4*>(scratch + o) = *reinterpret_cast<const int4*>(cur + o);
                __syncwarp();
            }
            const int16_t new_id = (int16_t)__shfl_sync(kFull, (uint32_t)(uint16_t)old_id, src, G);
            __syncwarp();
            if (acc) {
                if (mover) cur[myq] = new_id;
                tt = tn;
                if (En <= Ebest) {
                    Ebest = En;
                    cur_is_best = true;
                } else if (mat) {
                    cur_is_best = false;
                }
                Ecur = En;
            } else {
                if (mover) {
                    pos_write<G, E, UCD>(ch, myq, old_v);
                    if constexpr (MV == 2) ch.sum()[sidx] = old_s;
                }
                ch.tot()[l] = tt;
            }
            __syncwarp();
            T = __dmul_rn(T, a.mu);  // line 10
        }
        if (hout) {  // first part of a split chain: hand the state to the warp finishing it
            int16_t* hids = reinterpret_cast<int16_t*>(reinterpret_cast<uint8_t*>(hand_rec) + CPW * sizeof(SaHand)) +
                            (size_t)grp * 2 * NP;
            for (int o = l * 8; o < NP; o += 8 * G) {
                *reinterpret_cast<int4*>(hids + o) = *reinterpret_cast<const int4*>(cur + o);
                if (!cur_is_best)
                    *reinterpret_cast<int4*>(hids + NP + o) = *reinterpret_cast<const int4*>(scratch + o);
            }
            if (l == 0) hand_rec[grp] = SaHand{Ecur, Ebest, cur_is_best ? 1 : 0, 0, T};
            __threadfence();
            __syncwarp();
            if (lane == 0)
                asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(reinterpret_cast<uint8_t*>(hand_rec) - 16),
                             "r"(1u) : "memory");
            __syncwarp();
            return;
        }
        if (active && l == 0) {
            if (a.chain_best) a.chain_best[c] = Ebest;
            if (a.chain_final) a.chain_final[c] = Ecur;
        }
        const unsigned long long key = ((unsigned long long)(uint32_t)Ebest << 32) | (uint32_t)g;
        const bool better = active && key < gkey;
        if (better) gkey = key;
        __syncwarp();
        if (better) {
            const int16_t* src = cur_is_best ? cur : scratch;
            for (int o = l * 8; o < NP; o += 8 * G)
                *reinterpret_cast<int4*>(gbest + o) = *reinterpret_cast<const int4*>(src + o);
        }
        if (a.final_key) {  // synchronous SA: the minimum final state
            const unsigned long long fkey = ((unsigned long long)(uint32_t)Ecur << 32) | (uint32_t)g;
            const bool fbetter = active && fkey < gfkey;
            if (fbetter) {
                gfkey = fkey;
                for (int o = l * 8; o < NP; o += 8 * G)
                    *reinterpret_cast<int4*>(gfinal + o) = *reinterpret_cast<const int4*>(cur + o);
            }
        }
        __syncwarp();
    };
    if (a.share == 0) {
        for (int64_t c0 = wfirst; c0 < a.chains; c0 += groups)  // warp-uniform trip count
            run_piece(c0, 0, a.steps, false, false);
    } else {
        // balanced schedule: the (quad of chains, step) space in quad-major order, a contiguous
        // share per warp; a warp runs the head of its last quad first (and hands it over), then
        // its whole quads, and the tail of its first quad last (after the previous warp's
        // handover, which that warp produced first) -- every warp does the same number of steps
        const int64_t S = a.steps, W = ((a.chains + CPW - 1) / CPW) * S;
        const int64_t b = wglob * a.share, e = min(W, b + a.share);
        if (b < e) {
            const int64_t qa = b / S, qb = (e - 1) / S;
            const uint32_t ka = (uint32_t)(b - qa * S), kbe = (uint32_t)(e - qb * S);
            if (kbe < (uint32_t)S) run_piece(qb * CPW, 0, kbe, false, true);
            const int64_t f0 = ka ? qa + 1 : qa, f1 = kbe < (uint32_t)S ? qb - 1 : qb;
            for (int64_t q = f0; q <= f1; ++q) run_piece(q * CPW, 0, a.steps, false, false);
            if (ka) run_piece(qa * CPW, ka, a.steps, true, false);
        }
    }
    if (l == 0) {
        s_key[wib * CPW + grp] = gkey;
        s_fkey[wib * CPW + grp] = gfkey;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long m = s_key[0], f = s_fkey[0];
        for (int i = 1; i < kGWarps * CPW; ++i) {
            m = s_key[i] < m ? s_key[i] : m;
            f = s_fkey[i] < f ? s_fkey[i] : f;
        }
        if (m != ULLONG_MAX) atomicMin(a.best_key, m);
        if (a.final_key && f != ULLONG_MAX) atomicMin(a.final_key, f);
    }
}

// T0 rule on the group layout: G lanes per sample, so 32/G of the serial Fisher-Yates
// shuffles (R10, the bulk of a sample's work) run side by side in a warp and far more samples are
// resident at once than with a warp per sample.  Same words (tag T0, id = sample) and the same
// evaluator as the SA chains, so Z is bit-identical to t0_sample_kernel's.
template <int G, int E, bool UCD>
__global__ void __launch_bounds__(kGThreads) t0_group_kernel(ChainTables T, int n, int32_t d, int quad, uint64_t seed,
                                                            int64_t samples, int16_t* scratch, int64_t* Z) {
    using C = GChain<G, E, UCD>;
    constexpr int CPW = 32 / G;
    extern __shared__ __align__(16) uint8_t smem[];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int grp = lane / G, l = lane % G, gbase = grp * G;
    const C ch{smem + (size_t)(wib * CPW + grp) * C::BYTES};
    const int64_t groups = (int64_t)gridDim.x * kGWarps * CPW;
    for (int64_t s0 = ((int64_t)blockIdx.x * kGWarps + wib) * CPW; s0 < samples; s0 += groups) {
        const int64_t sm = s0 + grp;
        const bool active = sm < samples;
        // (groups past the last sample shuffle sample 0 into a spare slot and write nothing)
        int16_t* cur = scratch + (size_t)(active ? sm : samples + grp) * C::NP;
        gchain_init<G, E, UCD>(ch, cur, n, seed, (uint64_t)(active ? sm : 0), l, T, nullptr, nullptr, kTagT0);
        const int32_t z = gchain_eval<G, E, UCD>(ch, l, gbase, n, d, ch.tot()[l], quad);
        if (active && l == 0) Z[sm] = z;
        __syncwarp();
    }
}

// ------------------------------------------------------------------------------- host side
struct Grid {
    int blocks;
    size_t smem;
};

ChainTables tables(const Instance& I, bool ucd) {
    return ucd ? ChainTables{I.tab_ab, I.tab_m, I.tab_x, I.tab_g, I.tab_ab16}
               : ChainTables{I.tab_ab, I.tab_p, nullptr, nullptr, I.tab_ab16};
}

constexpr size_t kAlign = 256;
inline size_t align_up(size_t x) { return (x + kAlign - 1) / kAlign * kAlign; }

struct WsLayout {
    size_t t0_off, z_off, t0s_off, slots_off, total;
};

int t0_pow2_at_least(int c) {
    int e = 1;
    while (e < c) e <<= 1;
    return e;
}

// Layout of the group T0 kernel (0: warp-per-sample kernel): the SA base layouts by n, unwidened.
struct T0Cfg {
    int G, E;
};
T0Cfg t0_cfg(const Instance& I, bool ucd) {
    if (!I.ab16_ok) return {0, 0};
    const int G = !ucd ? (I.n <= 256 ? 4 : 8) : (I.n <= 64 ? 4 : (I.n <= 512 ? 8 : 16));
    const int E = std::max(8, t0_pow2_at_least((I.n + G - 1) / G));
    if (E > (G == 8 ? 128 : 64)) return {0, 0};
    return {G, E};
}
// per-sample id slots of the group T0 kernel (+32 spares for the groups past the last sample)
size_t t0_scratch_bytes(const Instance& I, bool ucd, int64_t samples) {
    const T0Cfg c = t0_cfg(I, ucd);
    return c.G && samples > 0 ? (size_t)(samples + 32) * (size_t)(c.G * c.E) * sizeof(int16_t) : 0;
}

WsLayout ws_layout(int np, int64_t samples, int blocks, size_t t0s) {
    WsLayout w{};
    w.t0_off = 0;
    w.z_off = align_up(sizeof(double));
    w.t0s_off = align_up(w.z_off + sizeof(int64_t) * (size_t)(samples > 0 ? samples : 0));
    w.slots_off = align_up(w.t0s_off + t0s);
    w.total = align_up(w.slots_off + (size_t)blocks * kSaWarps * 2 * (size_t)np * sizeof(int16_t));
    return w;
}

template <int G, int E, bool UCD>
cudaError_t t0_group_impl(const Instance& I, uint64_t seed, int64_t samples, double* T0_dev, void* ws,
                          cudaStream_t s) {
    using C = GChain<G, E, UCD>;
    constexpr int CPB = kGWarps * (32 / G);
    const size_t smem = (size_t)CPB * C::BYTES;
    int sms = 148, occ = 1;
    resident_ctas(reinterpret_cast<const void*>(t0_group_kernel<G, E, UCD>), I.device, kGThreads, smem, &sms, &occ);
    int64_t blocks = (samples + CPB - 1) / CPB;
    if (blocks > (int64_t)sms * occ) blocks = (int64_t)sms * occ;
    if (blocks < 1) blocks = 1;
    const WsLayout w = ws_layout(0, samples, 0, 0);
    uint8_t* base = static_cast<uint8_t*>(ws);
    int64_t* Z = reinterpret_cast<int64_t*>(base + w.z_off);
    int16_t* scratch = reinterpret_cast<int16_t*>(base + w.t0s_off);
    t0_group_kernel<G, E, UCD><<<(unsigned)blocks, kGThreads, smem, s>>>(tables(I, UCD), I.n, I.d_eff, I.quad_level(), seed,
                                                                       samples, scratch, Z);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    t0_reduce_kernel<<<1, 1024, 0, s>>>(Z, samples, T0_dev);
    return cudaGetLastError();
}

// ---- group kernel (16 lanes per chain)
template <int G, int E, bool UCD, bool TRACE, int MV>
Grid sag_grid(const Instance& I, int64_t chains) {
    constexpr int CPB = kGWarps * (32 / G);  // chains per CTA
    Grid gr{1, (size_t)CPB * SagChain<G, E, UCD, MV>::BYTES};
    int sms = 148, occ = 1;
    resident_ctas(reinterpret_cast<const void*>(sa_group_kernel<G, E, UCD, TRACE, MV>), I.device, kGThreads, gr.smem,
                  &sms, &occ);
    // CDD_SA_OCC=k: at most k CTAs per SM (occupancy experiments)
    if (const char* v = getenv("CDD_SA_OCC")) occ = std::max(1, std::min(occ, atoi(v)));
    const int64_t need = (chains + CPB - 1) / CPB;
    const int64_t cap = (int64_t)sms * occ;
    gr.blocks = (int)(need < cap ? (need < 1 ? 1 : need) : cap);
    return gr;
}

// Balanced schedule for runs whose chains fill the resident slots for more than one round but
// leave the last one mostly empty (e.g. 16384 UCDDCP chains at n=200 over 14208 slots: two rounds
// for 1.15 rounds of work): 0 = round robin (also when the last round is > 75 % full -- config 5:
// 6.92 rounds -- or with traces).  CDD_SA_BALANCE=0 disables it.
template <int G>
int64_t sag_share(const SaLaunch& p, const Grid& gr) {
    if (p.trace || p.steps < 1) return 0;
    const char* v = getenv("CDD_SA_BALANCE");  // "0": never, "2": whenever the last round is partial
    if (v && v[0] == '0') return 0;
    constexpr int CPW = 32 / G;
    const int64_t Rw = (int64_t)gr.blocks * kGWarps;
    const int64_t Q = (p.chains + CPW - 1) / CPW;
    if (Q <= Rw) return 0;
    const int64_t full = Q / Rw, rem = Q % Rw;
    if (rem == 0 || (4 * rem > 3 * Rw && !(v && v[0] == '2'))) return 0;
    (void)full;
    const int64_t W = Q * p.steps;
    return (W + Rw - 1) / Rw;  // >= steps since Q > Rw
}

template <int G, int E, bool UCD, bool TRACE, int MV>
size_t sag_ws(const Instance& I, const SaLaunch& p) {
    const Grid gr = sag_grid<G, E, UCD, TRACE, MV>(I, p.chains);
    const int64_t groups = (int64_t)gr.blocks * kGWarps * (32 / G);
    // slots: 3 * NP ids per group (current, scratch best, group best)
    WsLayout w = ws_layout(G * E, p.t0_samples, 0, t0_scratch_bytes(I, p.ucd, p.t0_samples));
    w.total = align_up(w.slots_off + (size_t)groups * 3 * G * E * sizeof(int16_t));
    if (sag_share<G>(p, gr))  // handover area of the balanced schedule
        w.total += (size_t)gr.blocks * kGWarps * hand_warp_bytes(G * E, 32 / G);
    return w.total;
}

template <int G, int E, bool UCD, bool TRACE, int MV>
cudaError_t sag_impl(Instance& I, const SaLaunch& p, void* ws, cudaStream_t s) {
    constexpr int NP = G * E;
    const Grid gr = sag_grid<G, E, UCD, TRACE, MV>(I, p.chains);
    const int64_t groups = (int64_t)gr.blocks * kGWarps * (32 / G);
    const WsLayout w = ws_layout(NP, p.t0_samples, 0, t0_scratch_bytes(I, UCD, p.t0_samples));
    uint8_t* base = static_cast<uint8_t*>(ws);
    const double* T0_dev = p.T0_in;
    if (!T0_dev && !(p.T0 > 0)) {
        double* t0w = reinterpret_cast<double*>(base + w.t0_off);
        cudaError_t e = launch_t0(I, UCD, p.seed, p.t0_samples, t0w, ws, s);
        if (e != cudaSuccess) return e;
        T0_dev = t0w;
    }
    cudaError_t e = cudaMemsetAsync(I.best_key, 0xff, sizeof(unsigned long long), s);
    if (e != cudaSuccess) return e;
    SaGArgs a{};
    a.quad = I.quad_level();
    a.T = tables(I, UCD);
    a.n = I.n;
    a.d = I.d_eff;
    a.chains = p.chains;
    a.steps = (uint32_t)p.steps;
    a.mu = p.mu;
    a.T0 = p.T0;
    a.T0_ptr = T0_dev;
    a.T0_out = p.T0_out;
    a.pert = p.pert;
    a.move = p.move;
    a.seed = p.seed;
    a.chain_offset = p.chain_offset;
    a.slots = reinterpret_cast<int16_t*>(base + w.slots_off);
    a.best_key = I.best_key;
    a.trace = p.trace;
    a.chain_best = p.chain_best;
    a.chain_final = p.chain_final;
    a.init_user = p.init;
    a.init_ld = p.init_ld;
    a.err = I.err;
    a.share = sag_share<G>(p, gr);
    if (a.share) {
        // handover area after the slots; ready flags cleared; all warps co-resident (a warp may
        // wait for the previous one's handover), hence a cooperative launch
        const size_t hb = hand_warp_bytes(NP, 32 / G);
        a.hand = base + align_up(w.slots_off + (size_t)groups * 3 * NP * sizeof(int16_t));
        e = cudaMemset2DAsync(a.hand, hb, 0, 16, (size_t)gr.blocks * kGWarps, s);
        if (e != cudaSuccess) return e;
        void* args[] = {&a};
        e = cudaLaunchCooperativeKernel(reinterpret_cast<const void*>(sa_group_kernel<G, E, UCD, TRACE, MV>),
                                        dim3(gr.blocks), dim3(kGThreads), args, gr.smem, s);
        if (e == cudaErrorCooperativeLaunchTooLarge || e == cudaErrorNotSupported) {
            (void)cudaGetLastError();  // co-residency not available here: round robin
            a.share = 0;
            sa_group_kernel<G, E, UCD, TRACE, MV><<<gr.blocks, kGThreads, gr.smem, s>>>(a);
        } else if (e != cudaSuccess) {
            return e;
        }
    } else {
        sa_group_kernel<G, E, UCD, TRACE, MV><<<gr.blocks, kGThreads, gr.smem, s>>>(a);
    }
    e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    sa_finalize<<<1, 256, 0, s>>>(I.best_key, a.slots, 3 * NP, 2 * NP, I.n, p.chain_offset, groups,
                                  I.best_perm, a.share, p.steps, 32 / G);
    return cudaGetLastError();
}

// ---- synchronous SA (Fig. 8): one launch of the group kernel per temperature level
__global__ void sync_scale_T(double* T, double mu, const double* T0_in, double T0_value, int mode) {
    // mode 0: T = T0_value, 1: T = *T0_in, 2: T = T * mu (next temperature level)
    if (mode == 0) *T = T0_value;
    else if (mode == 1) *T = *T0_in;
    else *T = __dmul_rn(*T, mu);
}

// Peer exchange of s^min across ranks inside the finalisation (sa_sync_run_peer): regions, world,
// rank, chains per rank, region sequence stride.
struct SyncPeer {
    uint8_t* const* regions;
    int world, rank;
    int64_t per_rank;
    int np;
    int* err;
};

__global__ void sync_level_finalize(unsigned long long* keys, const int16_t* slots, int64_t stride,
                                    int np, int n, uint64_t chain_offset, int64_t groups, int16_t* smin,
                                    unsigned long long* best_key, int16_t* best_perm,
                                    int64_t* level_min, int64_t j, SyncPeer px) {
    const unsigned long long b = keys[0];
    unsigned long long f = keys[1];
    const unsigned long long cur = *best_key;
    __syncthreads();  // every thread has read the old best before thread 0 may replace it
    if (f != ULLONG_MAX) {  // s^min_j: the final state of minimal cost (lowest id on ties)
        const uint64_t c = (uint64_t)(uint32_t)(f & 0xffffffffu) - chain_offset;
        const int16_t* src = slots + (size_t)(c % (uint64_t)groups) * stride + 3 * np;
        for (int i = threadIdx.x; i < n; i += blockDim.x) smin[i] = src[i];
    }
    if (px.world > 1) {  // s^min over the chains of all ranks, fused (peer.cuh)
        __syncthreads();
        f = peer_exchange_block(px.regions, px.world, px.rank, px.per_rank, px.np, (uint32_t)j,
                                (int)(j & 1), f, smin, n, px.err);
        if (threadIdx.x == 0) keys[1] = f;
    }
    // best-ever (R18): the minimum of (penalty, chain id) over all levels -- the packed key's order,
    // so the per-rank results reduce across GPUs with one MIN; an exact tie keeps the earlier level
    if (b != ULLONG_MAX && b < cur) {
        const uint64_t c = (uint64_t)(uint32_t)(b & 0xffffffffu) - chain_offset;
        const int16_t* src = slots + (size_t)(c % (uint64_t)groups) * stride + 2 * np;
        for (int i = threadIdx.x; i < n; i += blockDim.x) best_perm[i] = src[i];
        if (threadIdx.x == 0) *best_key = b;
    }
    if (level_min && threadIdx.x == 0) level_min[j] = (int64_t)(f >> 32);
}

// Start of level j >= 1: T_j = T_{j-1} * mu, level keys reset, and the shared-memory image of a
// chain holding s^min_{j-1} (exactly what gchain_init writes for it, zero padding elsewhere).
// After the cross-GPU exchange smin holds the global s^min, so the image is built here, not in
// sync_level_finalize.
template <int G, int E, bool UCD, int MV>
__global__ void sync_level_prepare(double* T, double mu, unsigned long long* keys, const int16_t* smin,
                                   int n, ChainTables tb, uint8_t* image, int16_t* ids, int* err) {
    using C = SagChain<G, E, UCD, MV>;
    constexpr int NP = C::NP;
    if (threadIdx.x == 0) {
        *T = __dmul_rn(*T, mu);
        keys[0] = ULLONG_MAX;
        keys[1] = ULLONG_MAX;
    }
    // built in shared memory (the lane totals re-read it), then copied out
    __shared__ __align__(16) uint8_t buf[C::BYTES];
    for (int i = threadIdx.x; i < C::BYTES / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(buf)[i] = 0u;
    __syncthreads();
    const C ch{buf};
    for (int k = threadIdx.x; k < NP; k += blockDim.x) {
        uint32_t j = k < n ? (uint16_t)smin[k] : 0u;
        if (j >= (uint32_t)n) {  // never from this library's kernels
            atomicOr(err, 1);
            j = 0;
        }
        ids[k] = (int16_t)j;
        const bool v = k < n;
        const uint32_t ab = v ? tb.ab16[j] : 0u;
        if constexpr (MV == 2) {  // nibble layout (sa_nib.cuh)
            ch.ab()[k] = (uint8_t)((ab & 15u) | ((ab >> 4) & 0xf0u));
            ch.pb()[k] = v ? tb.p[j] : (uint8_t)0;
        } else if constexpr (UCD) {
            ch.pb()[C::pb_b(k)] = v ? tb.p[j] : (uint8_t)0;
            ch.ab()[C::ab_h(k)] = (uint16_t)ab;
            ch.xb()[C::pb_b(k)] = v ? tb.x[j] : (uint8_t)0;
            ch.gh()[C::gh_h(k)] = v ? tb.g[j] : (uint16_t)0;
        } else {
            ch.pb()[C::pb_b(k)] = v ? tb.p[j] : (uint8_t)0;
            ch.a8()[C::rb(k)] = (uint8_t)ab;
            ch.b8()[C::rb(k)] = (uint8_t)(ab >> 8);
        }
    }
    __syncthreads();
    if constexpr (MV == 2) {
        if (threadIdx.x < G) {  // the lane row's sub-block summaries and totals, as gchain_init
            const int l = (int)threadIdx.x;
            uint32_t tA = 0, tB = 0, tP = 0;
            for (int b = 0; b < C::NSB; ++b) {
                const uint2 sm = nib_summary(ch, l * E + C::SB * b);
                ch.sum()[b * G + l] = sm;
                tA += sm.y & 0xffu;
                tB += (sm.y >> 8) & 0xffu;
                tP += sm.y >> 16;
            }
            ch.tot()[l] = make_uint2(tA | (tB << 16), tP);
        }
    } else {
        if (threadIdx.x < G) ch.tot()[threadIdx.x] = gchain_lane_totals(ch, (int)threadIdx.x);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < C::BYTES / 16; i += blockDim.x)
        reinterpret_cast<int4*>(image)[i] = reinterpret_cast<const int4*>(buf)[i];
}

struct SyncWs {
    size_t slots_off, T_off, keys_off, smin_off, image_off, ids_off, total;
    int64_t groups;
};

template <int G, int E, bool UCD, int MV>
SyncWs sync_layout(const Instance& I, const SaLaunch& p) {
    constexpr int NP = G * E;
    const Grid gr = sag_grid<G, E, UCD, false, MV>(I, p.chains);
    SyncWs w{};
    w.groups = (int64_t)gr.blocks * kGWarps * (32 / G);
    const WsLayout b = ws_layout(NP, p.t0_samples, 0, t0_scratch_bytes(I, UCD, p.t0_samples));
    w.slots_off = b.slots_off;
    w.T_off = align_up(w.slots_off + (size_t)w.groups * 4 * NP * sizeof(int16_t));
    w.keys_off = align_up(w.T_off + sizeof(double));
    w.smin_off = align_up(w.keys_off + 2 * sizeof(unsigned long long));
    w.image_off = align_up(w.smin_off + (size_t)NP * sizeof(int16_t));
    w.ids_off = align_up(w.image_off + (size_t)SagChain<G, E, UCD, MV>::BYTES);
    w.total = align_up(w.ids_off + (size_t)NP * sizeof(int16_t));
    return w;
}

template <int G, int E, bool UCD, int MV>
cudaError_t sag_sync_level(Instance& I, const SaLaunch& p, int64_t j, int64_t* level_min, void* ws,
                           cudaStream_t s) {
    constexpr int NP = G * E;
    const Grid gr = sag_grid<G, E, UCD, false, MV>(I, p.chains);
    const SyncWs w = sync_layout<G, E, UCD, MV>(I, p);
    uint8_t* base = static_cast<uint8_t*>(ws);
    double* T = reinterpret_cast<double*>(base + w.T_off);
    auto* keys = reinterpret_cast<unsigned long long*>(base + w.keys_off);
    int16_t* smin = reinterpret_cast<int16_t*>(base + w.smin_off);
    int16_t* slots = reinterpret_cast<int16_t*>(base + w.slots_off);
    cudaError_t e = cudaSuccess;
    if (j == 0) {
        if (p.T0_in) {
            sync_scale_T<<<1, 1, 0, s>>>(T, 1.0, p.T0_in, 0.0, 1);
        } else if (p.T0 > 0) {
            sync_scale_T<<<1, 1, 0, s>>>(T, 1.0, nullptr, p.T0, 0);
        } else {
            e = launch_t0(I, UCD, p.seed, p.t0_samples, T, ws, s);
            if (e != cudaSuccess) return e;
        }
        if (p.T0_out) {
            e = cudaMemcpyAsync(p.T0_out, T, sizeof(double), cudaMemcpyDeviceToDevice, s);
            if (e != cudaSuccess) return e;
        }
        e = cudaMemsetAsync(I.best_key, 0xff, sizeof(unsigned long long), s);
        if (e != cudaSuccess) return e;
        e = cudaMemsetAsync(keys, 0xff, 2 * sizeof(unsigned long long), s);
        if (e != cudaSuccess) return e;
    } else {
        sync_level_prepare<G, E, UCD, MV><<<1, 256, 0, s>>>(T, p.mu, keys, smin, I.n, tables(I, UCD),
                                                        base + w.image_off,
                                                        reinterpret_cast<int16_t*>(base + w.ids_off), I.err);
        e = cudaGetLastError();
        if (e != cudaSuccess) return e;
    }
    SaGArgs a{};
    a.quad = I.quad_level();
    a.T = tables(I, UCD);
    a.n = I.n;
    a.d = I.d_eff;
    a.chains = p.chains;
    a.steps = (uint32_t)p.steps;  // M
    a.mu = 1.0;                   // constant temperature within a level
    a.T0 = 0.0;
    a.T0_ptr = T;
    a.pert = p.pert;
    a.move = p.move;
    a.seed = p.seed;
    a.chain_offset = p.chain_offset;
    a.slots = slots;
    a.best_key = keys;
    a.init_perm = nullptr;  // level 0: each chain's own random state
    a.init_image = j == 0 ? nullptr : base + w.image_off;
    a.init_ids = j == 0 ? nullptr : reinterpret_cast<const int16_t*>(base + w.ids_off);
    a.step0 = (uint32_t)((uint64_t)j * (uint64_t)p.steps);
    a.final_key = keys + 1;
    sa_group_kernel<G, E, UCD, false, MV><<<gr.blocks, kGThreads, gr.smem, s>>>(a);
    e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    SyncPeer px{nullptr, 0, 0, 1, 0, I.err};
    if (p.peer && I.peer && I.peer->open)
        px = SyncPeer{I.peer->d_regions, I.peer->world, I.peer->rank, p.chains, I.peer->np, I.err};
    sync_level_finalize<<<1, 256, 0, s>>>(keys, slots, 4 * NP, NP, I.n, p.chain_offset, w.groups, smin,
                                          I.best_key, I.best_perm, level_min, j, px);
    return cudaGetLastError();
}

int pow2_at_least(int c) {
    int e = 1;
    while (e < c) e <<= 1;
    return e;
}

#define CDD_SAG_DISPATCH(CFG, CALL)                                                             \
    switch ((CFG).G * 1000 + (CFG).E) {                                                         \
        case 16008: CALL(16, 8)                                                                 \
        case 16016: CALL(16, 16)                                                                \
        case 16032: CALL(16, 32)                                                                \
        case 16064: CALL(16, 64)                                                                \
        case 4008: CALL(4, 8)                                                                   \
        case 4016: CALL(4, 16)                                                                  \
        case 4032: CALL(4, 32)                                                                  \
        case 4064: CALL(4, 64)                                                                  \
        case 8008: CALL(8, 8)                                                                   \
        case 8016: CALL(8, 16)                                                                  \
        case 8032: CALL(8, 32)                                                                  \
        case 8064: CALL(8, 64)                                                                  \
        case 8128: CALL(8, 128)                                                                 \
        default: break;                                                                         \
    }

}  // namespace

// The functions one variant translation unit (sag_*.cu) exports: NAME_ws / NAME_run for the async
// kernel of (UCD, TRACE, MV); with SYNC also the synchronous-SA levels and the group T0 kernel.
#define CDD_SAG_CASES(X, UCD, TR, MV)                                                             \
    X(16, 8, UCD, TR, MV) X(16, 16, UCD, TR, MV) X(16, 32, UCD, TR, MV) X(16, 64, UCD, TR, MV)   \
    X(4, 8, UCD, TR, MV) X(4, 16, UCD, TR, MV) X(4, 32, UCD, TR, MV) X(4, 64, UCD, TR, MV)       \
    X(8, 8, UCD, TR, MV) X(8, 16, UCD, TR, MV) X(8, 32, UCD, TR, MV) X(8, 64, UCD, TR, MV)       \
    X(8, 128, UCD, TR, MV)
#define CDD_SAG_C_WS(GG, EE, UCD, TR, MV) case GG * 1000 + EE: return sag_ws<GG, EE, UCD, TR, MV>(I, p);
#define CDD_SAG_C_RUN(GG, EE, UCD, TR, MV) case GG * 1000 + EE: return sag_impl<GG, EE, UCD, TR, MV>(I, p, ws, s);
#define CDD_SAG_C_SW(GG, EE, UCD, TR, MV) case GG * 1000 + EE: return sync_layout<GG, EE, UCD, MV>(I, p).total;
#define CDD_SAG_C_SL(GG, EE, UCD, TR, MV) \
    case GG * 1000 + EE: return sag_sync_level<GG, EE, UCD, MV>(I, p, j, level_min, ws, s);
#define CDD_SAG_C_SP(GG, EE, UCD, TR, MV) case GG * 1000 + EE: w = sync_layout<GG, EE, UCD, MV>(I, p); break;
#define CDD_SAG_C_T0(GG, EE, UCD, TR, MV) \
    case GG * 1000 + EE: return t0_group_impl<GG, EE, UCD>(I, seed, samples, T0_dev, ws, s);
#define CDD_SAG_SWITCH(cfg, X, UCD, TR, MV) \
    switch ((cfg).G * 1000 + (cfg).E) { CDD_SAG_CASES(X, UCD, TR, MV) default: break; }

#define CDD_SAG_VARIANT(NAME, UCD, TR, MV)                                                        \
    size_t NAME##_ws(const Instance& I, const SaLaunch& p, GroupCfg cfg) {                       \
        CDD_SAG_SWITCH(cfg, CDD_SAG_C_WS, UCD, TR, MV)                                           \
        return 0;                                                                                \
    }                                                                                            \
    cudaError_t NAME##_run(Instance& I, const SaLaunch& p, GroupCfg cfg, void* ws, cudaStream_t s) { \
        CDD_SAG_SWITCH(cfg, CDD_SAG_C_RUN, UCD, TR, MV)                                          \
        return cudaErrorInvalidValue;                                                            \
    }

#define CDD_SAG_SYNC_VARIANT(NAME, UCD, MV)                                                       \
    size_t NAME##_sync_ws(const Instance& I, const SaLaunch& p, GroupCfg cfg) {                  \
        CDD_SAG_SWITCH(cfg, CDD_SAG_C_SW, UCD, false, MV)                                        \
        return 0;                                                                                \
    }                                                                                            \
    cudaError_t NAME##_sync_level(Instance& I, const SaLaunch& p, GroupCfg cfg, int64_t j,       \
                                  int64_t* level_min, void* ws, cudaStream_t s) {                \
        CDD_SAG_SWITCH(cfg, CDD_SAG_C_SL, UCD, false, MV)                                        \
        return cudaErrorInvalidValue;                                                            \
    }                                                                                            \
    void NAME##_sync_ptrs(const Instance& I, const SaLaunch& p, GroupCfg cfg, void* ws,          \
                          unsigned long long** key, int16_t** perm) {                            \
        SyncWs w{};                                                                              \
        CDD_SAG_SWITCH(cfg, CDD_SAG_C_SP, UCD, false, MV)                                        \
        uint8_t* base = static_cast<uint8_t*>(ws);                                               \
        *key = reinterpret_cast<unsigned long long*>(base + w.keys_off) + 1;                     \
        *perm = reinterpret_cast<int16_t*>(base + w.smin_off);                                   \
    }

// The nibble-layout variant (MV = 2, sa_nib.cuh): CDD, G = 8, E = 128 only.
#define CDD_SAG_NIB_VARIANT(NAME, TR)                                                             \
    size_t NAME##_ws(const Instance& I, const SaLaunch& p, GroupCfg cfg) {                       \
        if (cfg.G == 8 && cfg.E == 128) return sag_ws<8, 128, false, TR, 2>(I, p);               \
        if (cfg.G == 8 && cfg.E == 64) return sag_ws<8, 64, false, TR, 2>(I, p);                 \
        return 0;                                                                                \
    }                                                                                            \
    cudaError_t NAME##_run(Instance& I, const SaLaunch& p, GroupCfg cfg, void* ws, cudaStream_t s) { \
        if (cfg.G == 8 && cfg.E == 128) return sag_impl<8, 128, false, TR, 2>(I, p, ws, s);      \
        if (cfg.G == 8 && cfg.E == 64) return sag_impl<8, 64, false, TR, 2>(I, p, ws, s);        \
        return cudaErrorInvalidValue;                                                            \
    }
// ... and its synchronous-SA levels
#define CDD_SAG_NIB_SYNC_VARIANT(NAME)                                                            \
    size_t NAME##_sync_ws(const Instance& I, const SaLaunch& p, GroupCfg cfg) {                  \
        if (cfg.G == 8 && cfg.E == 128) return sync_layout<8, 128, false, 2>(I, p).total;        \
        if (cfg.G == 8 && cfg.E == 64) return sync_layout<8, 64, false, 2>(I, p).total;          \
        return 0;                                                                                \
    }                                                                                            \
    cudaError_t NAME##_sync_level(Instance& I, const SaLaunch& p, GroupCfg cfg, int64_t j,       \
                                  int64_t* level_min, void* ws, cudaStream_t s) {                \
        if (cfg.G == 8 && cfg.E == 128) return sag_sync_level<8, 128, false, 2>(I, p, j, level_min, ws, s); \
        if (cfg.G == 8 && cfg.E == 64) return sag_sync_level<8, 64, false, 2>(I, p, j, level_min, ws, s); \
        return cudaErrorInvalidValue;                                                            \
    }                                                                                            \
    void NAME##_sync_ptrs(const Instance& I, const SaLaunch& p, GroupCfg cfg, void* ws,          \
                          unsigned long long** key, int16_t** perm) {                            \
        const SyncWs w = cfg.E == 128 ? sync_layout<8, 128, false, 2>(I, p) : sync_layout<8, 64, false, 2>(I, p); \
        uint8_t* base = static_cast<uint8_t*>(ws);                                               \
        *key = reinterpret_cast<unsigned long long*>(base + w.keys_off) + 1;                     \
        *perm = reinterpret_cast<int16_t*>(base + w.smin_off);                                   \
    }

#define CDD_SAG_T0_VARIANT(NAME, UCD)                                                             \
    cudaError_t NAME##_t0(const Instance& I, GroupCfg cfg, uint64_t seed, int64_t samples,       \
                          double* T0_dev, void* ws, cudaStream_t s) {                            \
        CDD_SAG_SWITCH(cfg, CDD_SAG_C_T0, UCD, false, 0)                                         \
        return cudaErrorInvalidValue;                                                            \
    }

}  // namespace cdd
