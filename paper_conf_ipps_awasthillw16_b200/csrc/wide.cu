// wide.cu -- the generic ("wide") path of libcdd: instances outside the packed 8/16-bit record
// ranges of the fast kernels (n up to 32767, any non-negative int32 P, alpha, beta, M, gamma, int64
// d; include/cdd.h "Fast and generic paths").
//
// Same method, same closed form as the fast kernels: with S_k = sum_{j<k}(a_j + b_j)
// and Btot = sum b, the due-date position is k0 = max{k : S_k <= Btot} (Theorem 1), the
// CDD due date in unshifted coordinates is D = min(C_{k0}, d), and the UCDDCP weight of
// position k is A_{k-1} (k <= k0) or B_k (k > k0) with compression iff the weight exceeds gamma
// (P:137-166).  Everything is int64 and the records are plain int32 fields gathered by job id
// (int4 {P, alpha, beta, gamma}, int2 {M, X = P - M}) -- no packing, so no value-range limit
// beyond int64 penalties.
//
// A group of TH threads (one warp, or one CTA for long sequences) evaluates one sequence: thread t
// owns the contiguous positions [t*S, t*S+S), S = ceil(n/TH).  Pass 1: per-thread sums of P,
// alpha, beta and a group exclusive scan; the thread whose first position still has S <= Btot
// walks its segment for k0 and C_{k0}.  Pass 2: the objective itself, eq. (1) at D (CDD) or the
// weights of eq. (2) (UCDDCP), summed over the group.
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>

#include "device_common.cuh"
#include "internal.h"
#include "sa_impl.cuh"

namespace cdd {
namespace {

constexpr int kWideWarpThreads = 256;   // warp-per-sequence kernels: 8 sequences per CTA
constexpr int kWideBlockThreads = 256;  // block-per-sequence kernels (n > kWideWarpMaxN)
constexpr int kWideWarpMaxN = 2048;

// ---------------------------------------------------------------------------- group primitives
// Group = one warp (TH = 32) or the whole CTA (TH = blockDim.x).  `sm` is TH/32 + 1 int64 of
// shared memory per group (CTA groups only).
template <int TH>
__device__ __forceinline__ long long wgroup_excl_scan(long long v, long long& total, long long* sm) {
    const int lane = threadIdx.x & 31;
    long long x = v;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const long long y = __shfl_up_sync(kFull, x, off);
        if (lane >= off) x += y;
    }
    if constexpr (TH == 32) {
        total = __shfl_sync(kFull, x, 31);
        return x - v;
    } else {
        const int w = threadIdx.x >> 5;
        __syncthreads();
        if (lane == 31) sm[w] = x;
        __syncthreads();
        long long off = 0, tot = 0;
#pragma unroll 1
        for (int i = 0; i < TH / 32; ++i) {
            const long long t = sm[i];
            off += i < w ? t : 0;
            tot += t;
        }
        total = tot;
        return x - v + off;
    }
}

template <int TH>
__device__ __forceinline__ long long wgroup_sum(long long v, long long* sm) {
    long long tot;
    (void)wgroup_excl_scan<TH>(v, tot, sm);
    return tot;
}

template <int TH>
__device__ __forceinline__ int wgroup_max(int v, long long* sm) {
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) v = max(v, __shfl_xor_sync(kFull, v, off));
    if constexpr (TH == 32) {
        return v;
    } else {
        __syncthreads();
        if ((threadIdx.x & 31) == 0) sm[threadIdx.x >> 5] = v;
        __syncthreads();
        int m = INT_MIN;
#pragma unroll 1
        for (int i = 0; i < TH / 32; ++i) m = max(m, (int)sm[i]);
        return m;
    }
}

// value of thread `src` of the group (CTA groups: through sm[TH/32])
template <int TH>
__device__ __forceinline__ long long wgroup_bcast(long long v, int src, long long* sm) {
    if constexpr (TH == 32) {
        return __shfl_sync(kFull, v, src);
    } else {
        __syncthreads();
        if ((int)threadIdx.x == src) sm[TH / 32] = v;
        __syncthreads();
        return sm[TH / 32];
    }
}

struct WideTab {
    const int4* w0;  // {P, alpha, beta, gamma} by job id
    const int2* w1;  // {M, X = P - M} by job id (UCDDCP)
};

// The due-date position of the group's sequence: k0 = max{k : S_k <= Btot} and the inclusive
// completion time C_{k0} (start at 0), plus this thread's exclusive prefixes.
struct WideSplit {
    int k0;
    long long Ck0, Pex, Aex, Bex, Btot;
};

template <int TH, class IdAt>
__device__ __forceinline__ WideSplit wide_split(const WideTab& T, int n, int t, IdAt&& id_at, long long* sm) {
    const int S = (n + TH - 1) / TH;
    const int ka = min(n, t * S), kb = min(n, ka + S);
    long long Pt = 0, At = 0, Bt = 0;
    for (int k = ka; k < kb; ++k) {
        const int4 r = __ldg(T.w0 + id_at(k));
        Pt += r.x;
        At += r.y;
        Bt += r.z;
    }
    WideSplit w;
    long long Ptot, Atot;
    w.Pex = wgroup_excl_scan<TH>(Pt, Ptot, sm);
    w.Aex = wgroup_excl_scan<TH>(At, Atot, sm);
    w.Bex = wgroup_excl_scan<TH>(Bt, w.Btot, sm);
    // S is non-decreasing, so {k : S_k <= Btot} is a prefix; its last element lies in the segment
    // of the last thread whose first position passes (thread 0 always does: S_0 = 0)
    const int own = wgroup_max<TH>((ka < kb && w.Aex + w.Bex <= w.Btot) ? t : 0, sm);
    long long kc = 0, cc = 0;
    if (t == own) {
        long long s = w.Aex + w.Bex, c = w.Pex;
        for (int k = ka; k < kb; ++k) {
            const int4 r = __ldg(T.w0 + id_at(k));
            c += r.x;
            if (s <= w.Btot) {
                kc = k;
                cc = c;
            }
            s += (long long)r.y + r.z;
        }
    }
    w.k0 = (int)wgroup_bcast<TH>(kc, own, sm);
    w.Ck0 = wgroup_bcast<TH>(cc, own, sm);
    return w;
}

// Optimal penalty of the group's sequence: eq. (1) at D = min(C_{k0}, d) (CDD) or eq. (2) with the
// Property 1/2 weights (UCDDCP, d >= sum P).  Every thread of the group returns it.
// CDD in one gather pass: besides the sums, each thread keeps DA = sum alpha_k c_k and
// DB = sum beta_k c_k over its segment (c_k = completion time from the segment start), so a segment
// wholly before the due date D contributes A (D - C_start) - DA, one wholly after it
// B (C_start - D) + DB; only the thread whose segment holds D walks it again (and the owner of
// k0, for C_{k0}) -- the split F(C) = F(C_m') + integral of the fast kernels.
// Warp inclusive scan of int64 values (one warp group, TH = 32).
__device__ __forceinline__ long long warp_incl_scan64(long long x, int lane) {
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const long long y = __shfl_up_sync(kFull, x, off);
        if (lane >= off) x += y;
    }
    return x;
}

// One warp per sequence: the two segment walks of wide_eval_cdd (C_{k0} in the owner's segment,
// the objective over the segment holding D) spread over the 32 lanes, 32 positions per round, with
// warp scans of P and alpha + beta instead of one thread walking S positions.
template <class IdAt>
__device__ __forceinline__ long long wide_walk_k0_warp(const WideTab& T, int ka, int kb, long long s0, long long c0,
                                                       long long Btot, int lane, IdAt&& id_at) {
    long long cc = 0;
    for (int k1 = ka; k1 < kb; k1 += 32) {  // warp-uniform
        const int k = k1 + lane;
        long long p = 0, w = 0;
        if (k < kb) {
            const int4 r = __ldg(T.w0 + id_at(k));
            p = r.x;
            w = (long long)r.y + r.z;
        }
        const long long ip = warp_incl_scan64(p, lane), iw = warp_incl_scan64(w, lane);
        // S_k (exclusive) <= Btot: a prefix of the positions; the last one's inclusive C
        const unsigned m = __ballot_sync(kFull, k < kb && s0 + iw - w <= Btot);
        if (m) cc = __shfl_sync(kFull, c0 + ip, 31 - __clz(m));
        if (!(m >> 31)) break;  // the prefix ended inside this round (or the segment did)
        s0 += __shfl_sync(kFull, iw, 31);
        c0 += __shfl_sync(kFull, ip, 31);
    }
    return cc;
}

template <class IdAt>
__device__ __forceinline__ long long wide_walk_D_warp(const WideTab& T, int ka, int kb, long long c0, long long D,
                                                      int lane, IdAt&& id_at) {
    long long z = 0;
    for (int k1 = ka; k1 < kb; k1 += 32) {
        const int k = k1 + lane;
        long long p = 0, a = 0, b = 0;
        if (k < kb) {
            const int4 r = __ldg(T.w0 + id_at(k));
            p = r.x;
            a = r.y;
            b = r.z;
        }
        const long long ip = warp_incl_scan64(p, lane);
        const long long c = c0 + ip;
        if (k < kb) z += D > c ? a * (D - c) : b * (c - D);
        c0 += __shfl_sync(kFull, ip, 31);
    }
    return z;  // this lane's share
}

template <int TH, class IdAt>
__device__ __forceinline__ long long wide_eval_cdd(const WideTab& T, int n, long long d, int t, IdAt&& id_at,
                                                   long long* sm) {
    const int S = (n + TH - 1) / TH;
    const int ka = min(n, t * S), kb = min(n, ka + S);
    long long Pt = 0, At = 0, Bt = 0, DA = 0, DB = 0;
    for (int k = ka; k < kb; ++k) {
        const int4 r = __ldg(T.w0 + id_at(k));
        Pt += r.x;
        At += r.y;
        Bt += r.z;
        DA += (long long)r.y * Pt;
        DB += (long long)r.z * Pt;
    }
    long long Ptot, Atot, Btot;
    const long long Pex = wgroup_excl_scan<TH>(Pt, Ptot, sm);
    const long long Aex = wgroup_excl_scan<TH>(At, Atot, sm);
    const long long Bex = wgroup_excl_scan<TH>(Bt, Btot, sm);
    // k0 = max{k : S_k <= Btot} (a prefix): the owner's segment is walked for C_{k0}
    const int own = wgroup_max<TH>((ka < kb && Aex + Bex <= Btot) ? t : 0, sm);
    long long cc = 0;
    if constexpr (TH == 32) {
        const int oka = min(n, own * S), okb = min(n, oka + S);
        cc = wide_walk_k0_warp(T, oka, okb, __shfl_sync(kFull, Aex + Bex, own), __shfl_sync(kFull, Pex, own),
                               Btot, t, id_at);
    } else if (t == own) {
        long long s = Aex + Bex, c = Pex;
        for (int k = ka; k < kb; ++k) {
            const int4 r = __ldg(T.w0 + id_at(k));
            c += r.x;
            if (s <= Btot) cc = c;
            s += (long long)r.y + r.z;
        }
    }
    const long long D = TH == 32 ? min(cc, d) : min(wgroup_bcast<TH>(cc, own, sm), d);
    long long z = 0;
    const bool holds = ka < kb && Pex < D && Pex + Pt > D;  // the segment that holds D (at most one)
    if (ka < kb && !holds) z = Pex + Pt <= D ? At * (D - Pex) - DA : Bt * (Pex - D) + DB;
    if constexpr (TH == 32) {
        const unsigned hm = __ballot_sync(kFull, holds);
        if (hm) {
            const int th = __ffs(hm) - 1;
            const int hka = min(n, th * S), hkb = min(n, hka + S);
            z += wide_walk_D_warp(T, hka, hkb, __shfl_sync(kFull, Pex, th), D, t, id_at);
        }
    } else if (holds) {
        long long c = Pex;
        for (int k = ka; k < kb; ++k) {
            const int4 r = __ldg(T.w0 + id_at(k));
            c += r.x;
            z += D > c ? (long long)r.y * (D - c) : (long long)r.z * (c - D);
        }
    }
    return wgroup_sum<TH>(z, sm);
}

template <int TH, bool UCD, class IdAt>
__device__ __forceinline__ long long wide_eval(const WideTab& T, int n, long long d, int t, IdAt&& id_at,
                                               long long* sm) {
    if constexpr (!UCD) return wide_eval_cdd<TH>(T, n, d, t, id_at, sm);
    const WideSplit w = wide_split<TH>(T, n, t, id_at, sm);
    const int S = (n + TH - 1) / TH;
    const int ka = min(n, t * S), kb = min(n, ka + S);
    long long z = 0;
    {
        long long a = w.Aex, b = w.Btot - w.Bex;
        for (int k = ka; k < kb; ++k) {
            const int j = id_at(k);
            const int4 r = __ldg(T.w0 + j);
            const int2 q = __ldg(T.w1 + j);
            const long long wt = k <= w.k0 ? a : b;
            z += (long long)q.x * wt + (long long)q.y * min(wt, (long long)r.w);
            a += r.y;
            b -= r.z;
        }
    }
    return wgroup_sum<TH>(z, sm);
}

WideTab wide_tab(const Instance& I) { return WideTab{I.tab_w0, I.tab_w1}; }

// ------------------------------------------------------------------------- batched evaluation
// ids outside [0, n) raise the data-error flag and are read as job 0 (no out-of-bounds access)
struct RowIds {
    const int16_t* row;
    int n;
    int* err;
    __device__ __forceinline__ int operator()(int k) const {
        const int j = row[k];
        if ((unsigned)j >= (unsigned)n) {
            atomicOr(err, 1);
            return 0;
        }
        return j;
    }
};

template <bool UCD>
__global__ void __launch_bounds__(kWideWarpThreads) wide_eval_warp_kernel(WideTab T, int n, long long d,
                                                                          const int16_t* perms, int64_t ld,
                                                                          int64_t batch, int64_t* out, int* err) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = (int64_t)gridDim.x * (kWideWarpThreads / 32);
    for (int64_t b = (int64_t)blockIdx.x * (kWideWarpThreads / 32) + (threadIdx.x >> 5); b < batch; b += warps) {
        const long long z = wide_eval<32, UCD>(T, n, d, lane, RowIds{perms + b * ld, n, err}, nullptr);
        if (lane == 0) out[b] = z;
    }
}

template <bool UCD>
__global__ void __launch_bounds__(kWideBlockThreads) wide_eval_block_kernel(WideTab T, int n, long long d,
                                                                            const int16_t* perms, int64_t ld,
                                                                            int64_t batch, int64_t* out, int* err) {
    __shared__ long long sm[kWideBlockThreads / 32 + 1];
    for (int64_t b = blockIdx.x; b < batch; b += gridDim.x) {
        const long long z = wide_eval<kWideBlockThreads, UCD>(T, n, d, threadIdx.x, RowIds{perms + b * ld, n, err}, sm);
        if (threadIdx.x == 0) out[b] = z;
    }
}

// ------------------------------------------------------------------------------- schedules (F1)
// Completion times of the optimal schedule: CDD -- start s = d - D, C_k + s; UCDDCP -- X_k = P_k - M_k
// iff the weight exceeds gamma_k (R4), job k0 completes at d, C'_k = d + Q_k - Q_{k0} with Q the
// inclusive prefix of P - X.  penalty = eq. (1) / (2) of exactly these times.
template <bool UCD>
__global__ void __launch_bounds__(kWideBlockThreads) wide_schedule_kernel(WideTab T, int n, long long d,
                                                                          const int16_t* perms, int64_t ld,
                                                                          int64_t batch, int64_t* C, int32_t* X,
                                                                          int64_t* start, int64_t* pen, int* err) {
    constexpr int TH = kWideBlockThreads;
    __shared__ long long sm[TH / 32 + 1];
    const int t = threadIdx.x;
    const int S = (n + TH - 1) / TH;
    const int ka = min(n, t * S), kb = min(n, ka + S);
    for (int64_t b = blockIdx.x; b < batch; b += gridDim.x) {
        const RowIds ids{perms + b * ld, n, err};
        const WideSplit w = wide_split<TH>(T, n, t, ids, sm);
        int64_t* Cr = C + b * (int64_t)n;
        long long z = 0;
        if constexpr (!UCD) {
            const long long D = min(w.Ck0, d), s = d - D;
            long long c = w.Pex;
            for (int k = ka; k < kb; ++k) {
                const int4 r = __ldg(T.w0 + ids(k));
                c += r.x;
                const long long ck = c + s;
                Cr[k] = ck;
                z += ck < d ? (long long)r.y * (d - ck) : (long long)r.z * (ck - d);
            }
            z = wgroup_sum<TH>(z, sm);
            if (t == 0) {
                start[b] = s;
                pen[b] = z;
            }
        } else {
            int32_t* Xr = X + b * (int64_t)n;
            long long a = w.Aex, bb = w.Btot - w.Bex, q = 0;
            for (int k = ka; k < kb; ++k) {  // compressions, then the thread's sum of P - X
                const int j = ids(k);
                const int4 r = __ldg(T.w0 + j);
                const int2 m = __ldg(T.w1 + j);
                const long long wt = k <= w.k0 ? a : bb;
                const int x = wt > (long long)r.w ? m.y : 0;
                Xr[k] = x;
                q += (long long)r.x - x;
                a += r.y;
                bb -= r.z;
            }
            long long Qtot;
            const long long Qex = wgroup_excl_scan<TH>(q, Qtot, sm);
            // Q_{k0} (inclusive): the owner of position k0 sums its segment up to k0
            const int own = w.k0 / S;
            long long qk = 0;
            if (t == own) {
                qk = Qex;
                for (int k = ka; k <= w.k0; ++k) qk += (long long)__ldg(T.w0 + ids(k)).x - Xr[k];
            }
            const long long Qk0 = wgroup_bcast<TH>(qk, own, sm);
            long long Q = Qex;
            for (int k = ka; k < kb; ++k) {
                const int j = ids(k);
                const int4 r = __ldg(T.w0 + j);
                const int x = Xr[k];
                Q += (long long)r.x - x;
                const long long ck = d + Q - Qk0;
                Cr[k] = ck;
                z += (ck < d ? (long long)r.y * (d - ck) : (long long)r.z * (ck - d)) + (long long)r.w * x;
            }
            z = wgroup_sum<TH>(z, sm);
            if (t == 0) {
                start[b] = d - Qk0;
                pen[b] = z;
            }
        }
        __syncthreads();
    }
}

// ------------------------------------------------------------------------------------- SA (Alg. 1)
constexpr int kWSaWarps = 8;

struct WideSaArgs {
    WideTab T;
    int n;
    long long d;
    int64_t chains;
    uint32_t steps;
    double mu, T0;
    const double* T0_ptr;
    double* T0_out;
    int pert, move;
    uint64_t seed, chain_offset;
    int16_t* slots;  // per warp [3][NP]: current ids, scratch best, warp best
    int np;
    long long* cta_best;  // per CTA {E, g, warp slot}
    int64_t *trace, *chain_best, *chain_final;
    const int16_t* init;
    int64_t init_ld;
    int* err;
};

struct GIds {
    const int16_t* ids;
    __device__ __forceinline__ int operator()(int k) const { return ids[k]; }
};

// Alg. 1 line 1: s0 = Fisher-Yates of the identity (R10, the Philox words of (tag, id)) on lane 0,
// or the caller's row (ids outside [0, n) flag the instance and become 0)
__device__ void wide_init_ids(int16_t* cur, int n, uint64_t seed, uint32_t tag, uint64_t id, const int16_t* init,
                              int* err, int lane) {
    if (init) {
        for (int k = lane; k < n; k += 32) {
            int v = init[k];
            if ((unsigned)v >= (unsigned)n) {
                atomicOr(err, 1);
                v = 0;
            }
            cur[k] = (int16_t)v;
        }
        __syncwarp();
        return;
    }
    for (int k = lane; k < n; k += 32) cur[k] = (int16_t)k;
    __syncwarp();
    if (lane == 0) {
        uint4 w = make_uint4(0, 0, 0, 0);
        for (int q = 0; q < n - 1; ++q) {
            if ((q & 3) == 0) w = rng_block(seed, (uint32_t)(q >> 2), id, tag, 0);
            const int i = n - 1 - q;
            const int j = (int)bnd(word_of(w, q & 3), (uint32_t)i + 1u);
            const int16_t t = cur[i];
            cur[i] = cur[j];
            cur[j] = t;
        }
    }
    __syncwarp();
}

// insertion (R11b) on global ids: rotation by one of [lo, hi], 32 destinations per round
__device__ void wide_rotate(int16_t* ids, int lo, int hi, bool left, int lane) {
    const int16_t x = ids[left ? lo : hi];
    const int L = hi - lo;
    for (int i0 = 0; i0 < L; i0 += 32) {
        const int t = i0 + lane;
        const int k = left ? lo + t : hi - t;
        int16_t v = 0;
        if (t < L) v = ids[left ? k + 1 : k - 1];
        __syncwarp();
        if (t < L) ids[k] = v;
        __syncwarp();
    }
    if (lane == 0 && L > 0) ids[left ? hi : lo] = x;
    __syncwarp();
}

template <bool UCD>
__global__ void __launch_bounds__(kWSaWarps * 32) wide_sa_kernel(WideSaArgs a) {
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    __shared__ long long s_E[kWSaWarps];
    __shared__ long long s_g[kWSaWarps];
    const int64_t total_warps = (int64_t)gridDim.x * kWSaWarps;
    const int64_t gw = (int64_t)blockIdx.x * kWSaWarps + wib;
    int16_t* cur = a.slots + (size_t)gw * 3 * a.np;
    int16_t* scratch = cur + a.np;
    int16_t* wbest = cur + 2 * a.np;
    const int n = a.n;
    const int P = a.move == 1 ? min(2, n) : (a.move == 2 ? 0 : min(min(a.pert, 4), n));
    const double T0 = a.T0_ptr ? *a.T0_ptr : a.T0;
    if (a.T0_out && gw == 0 && lane == 0) *a.T0_out = T0;
    long long wE = LLONG_MAX, wg = -1;
    for (int64_t c = gw; c < a.chains; c += total_warps) {
        const uint64_t g = a.chain_offset + (uint64_t)c;
        wide_init_ids(cur, n, a.seed, kTagSaInit, g, a.init ? a.init + c * a.init_ld : nullptr, a.err, lane);
        long long Ecur = wide_eval<32, UCD>(a.T, n, a.d, lane, GIds{cur}, nullptr);
        long long Ebest = Ecur;
        bool cur_is_best = true;
        double T = T0;
        uint32_t R0 = 0, R1 = 0;
        for (uint32_t k = 0; k < a.steps; ++k) {
            const int s16 = (int)(k & 15);
            if (s16 == 0) precompute_moves(a.seed, g, k, lane, n, P, a.move, R0, R1);
            const uint32_t q01 = __shfl_sync(kFull, R0, 2 * s16);
            const uint32_t q23 = __shfl_sync(kFull, R1, 2 * s16);
            const uint32_t sig = __shfl_sync(kFull, R0, 2 * s16 + 1);
            const uint32_t uw = __shfl_sync(kFull, R1, 2 * s16 + 1);
            // line 5: the move on the ids (slot moves: position q_i receives the job of q_sigma(i))
            const bool ins = a.move == 2;
            const int from = (int)(q01 & 0xffffu), to = (int)(q01 >> 16);
            const int lo = min(from, to), hi = max(from, to);
            const bool mover = !ins && lane < P;
            const int myq = mover ? (int)(((lane < 2 ? q01 : q23) >> (16 * (lane & 1))) & 0xffffu) : 0;
            const int src = (int)((sig >> (2 * (lane & 3))) & 3u);
            const int16_t old_id = mover ? cur[myq] : (int16_t)0;
            const int16_t new_id = (int16_t)__shfl_sync(kFull, (uint32_t)(uint16_t)old_id, src);
            __syncwarp();
            if (ins) wide_rotate(cur, lo, hi, from < to, lane);
            else if (mover) cur[myq] = new_id;
            __syncwarp();
            const long long En = wide_eval<32, UCD>(a.T, n, a.d, lane, GIds{cur}, nullptr);  // line 6
            const long long delta = Ecur - En;                                                 // line 7
            const bool acc = delta >= 0 || metropolis_accept(delta, T, uw);
            if (a.trace && lane == 0)
                a.trace[c * (int64_t)a.steps + (int64_t)k] = (int64_t)(((uint64_t)En) << 1) | (acc ? 1 : 0);
            if (!acc) {  // revert
                if (ins) wide_rotate(cur, lo, hi, !(from < to), lane);
                else if (mover) cur[myq] = old_id;
                __syncwarp();
            } else {
                if (En <= Ebest) {
                    Ebest = En;
                    cur_is_best = true;
                } else if (cur_is_best) {
                    // leaving the best state: copy the pre-move sequence (move undone, copied, redone)
                    if (ins) wide_rotate(cur, lo, hi, !(from < to), lane);
                    else if (mover) cur[myq] = old_id;
                    __syncwarp();
                    for (int i = lane; i < n; i += 32) scratch[i] = cur[i];
                    __syncwarp();
                    if (ins) wide_rotate(cur, lo, hi, from < to, lane);
                    else if (mover) cur[myq] = new_id;
                    __syncwarp();
                    cur_is_best = false;
                }
                Ecur = En;
            }
            T = __dmul_rn(T, a.mu);  // line 10
        }
        if (lane == 0) {
            if (a.chain_best) a.chain_best[c] = Ebest;
            if (a.chain_final) a.chain_final[c] = Ecur;
        }
        // warp best: min (E_best, g) over this warp's chains (lowest id on ties: ids increase)
        if (Ebest < wE) {
            wE = Ebest;
            wg = (long long)g;
            const int16_t* s = cur_is_best ? cur : scratch;
            for (int i = lane; i < n; i += 32) wbest[i] = s[i];
        }
        __syncwarp();
    }
    if (lane == 0) {
        s_E[wib] = wE;
        s_g[wib] = wg;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        int bi = 0;
        for (int i = 1; i < kWSaWarps; ++i)
            if (s_E[i] < s_E[bi] || (s_E[i] == s_E[bi] && (unsigned long long)s_g[i] < (unsigned long long)s_g[bi])) bi = i;
        long long* o = a.cta_best + 3 * blockIdx.x;
        o[0] = s_E[bi];
        o[1] = s_g[bi];
        o[2] = (long long)blockIdx.x * kWSaWarps + bi;
    }
}

// min over the CTAs' (E, g); the winner's sequence and (penalty, id) into the instance's best
__global__ void wide_sa_finalize(const long long* cta_best, int ctas, const int16_t* slots, int np, int n,
                                 long long* best_wide, unsigned long long* best_key, int16_t* best_perm) {
    __shared__ int s_bi;
    if (threadIdx.x == 0) {
        int bi = 0;
        for (int i = 1; i < ctas; ++i) {
            const long long E = cta_best[3 * i], g = cta_best[3 * i + 1];
            const long long Eb = cta_best[3 * bi], gb = cta_best[3 * bi + 1];
            if (E < Eb || (E == Eb && (unsigned long long)g < (unsigned long long)gb)) bi = i;
        }
        s_bi = bi;
        const long long E = cta_best[3 * bi], g = cta_best[3 * bi + 1];
        best_wide[0] = E;
        best_wide[1] = g;
        *best_key = (E >= 0 && E < 0xffffffffll) ? (((unsigned long long)E << 32) | (unsigned long long)(uint32_t)g)
                                                  : ULLONG_MAX;
    }
    __syncthreads();
    const int16_t* src = slots + (size_t)cta_best[3 * s_bi + 2] * 3 * np + 2 * np;
    for (int i = threadIdx.x; i < n; i += blockDim.x) best_perm[i] = src[i];
}

// ------------------------------------------------------------------------------------------ T0
__global__ void __launch_bounds__(kWSaWarps * 32) wide_t0_kernel(WideTab T, int n, long long d, bool ucd,
                                                                 uint64_t seed, int64_t samples, int16_t* scratch,
                                                                 int np, int64_t* Z) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = (int64_t)gridDim.x * kWSaWarps;
    const int64_t gw = (int64_t)blockIdx.x * kWSaWarps + (threadIdx.x >> 5);
    int16_t* ids = scratch + (size_t)gw * np;
    for (int64_t s = gw; s < samples; s += warps) {
        wide_init_ids(ids, n, seed, kTagT0, (uint64_t)s, nullptr, nullptr, lane);
        const long long z = ucd ? wide_eval<32, true>(T, n, d, lane, GIds{ids}, nullptr)
                                : wide_eval<32, false>(T, n, d, lane, GIds{ids}, nullptr);
        if (lane == 0) Z[s] = z;
        __syncwarp();
    }
}

// ------------------------------------------------------------------------------------ host side
int wide_blocks(const void* kern, const Instance& I, int threads, int64_t want) {
    int sms = 148, occ = 1;
    resident_ctas(kern, I.device, threads, 0, &sms, &occ);
    const int64_t cap = (int64_t)sms * occ;
    return (int)std::max<int64_t>(1, std::min<int64_t>(want, cap));
}

struct WideWs {
    size_t t0_off, z_off, t0s_off, slots_off, cta_off, total;
    int blocks, t0_blocks;
};

WideWs wide_ws(const Instance& I, const SaLaunch& p) {
    WideWs w{};
    const int np = (I.n + 7) / 8 * 8;
    w.blocks = wide_blocks(reinterpret_cast<const void*>(p.ucd ? wide_sa_kernel<true> : wide_sa_kernel<false>), I,
                           kWSaWarps * 32, (p.chains + kWSaWarps - 1) / kWSaWarps);
    w.t0_blocks = p.t0_samples > 0 ? wide_blocks(reinterpret_cast<const void*>(wide_t0_kernel), I, kWSaWarps * 32,
                                                 (p.t0_samples + kWSaWarps - 1) / kWSaWarps)
                                   : 0;
    w.t0_off = 0;
    w.z_off = align_up(sizeof(double));
    w.t0s_off = align_up(w.z_off + sizeof(int64_t) * (size_t)std::max<int64_t>(p.t0_samples, 0));
    w.slots_off = align_up(w.t0s_off + (size_t)w.t0_blocks * kWSaWarps * np * sizeof(int16_t));
    w.cta_off = align_up(w.slots_off + (size_t)w.blocks * kWSaWarps * 3 * np * sizeof(int16_t));
    w.total = align_up(w.cta_off + (size_t)w.blocks * 3 * sizeof(long long));
    return w;
}

}  // namespace

cudaError_t launch_wide_eval(const Instance& I, bool ucd, const int16_t* perms, int64_t ld, int64_t batch,
                             int64_t* out, cudaStream_t s) {
    if (batch <= 0) return cudaSuccess;
    const WideTab T = wide_tab(I);
    if (I.n <= kWideWarpMaxN) {
        const void* k = ucd ? reinterpret_cast<const void*>(wide_eval_warp_kernel<true>)
                            : reinterpret_cast<const void*>(wide_eval_warp_kernel<false>);
        const int blocks = wide_blocks(k, I, kWideWarpThreads, (batch + kWideWarpThreads / 32 - 1) / (kWideWarpThreads / 32));
        if (ucd) wide_eval_warp_kernel<true><<<blocks, kWideWarpThreads, 0, s>>>(T, I.n, I.d, perms, ld, batch, out, I.err);
        else wide_eval_warp_kernel<false><<<blocks, kWideWarpThreads, 0, s>>>(T, I.n, I.d, perms, ld, batch, out, I.err);
    } else {
        const void* k = ucd ? reinterpret_cast<const void*>(wide_eval_block_kernel<true>)
                            : reinterpret_cast<const void*>(wide_eval_block_kernel<false>);
        const int blocks = wide_blocks(k, I, kWideBlockThreads, batch);
        if (ucd) wide_eval_block_kernel<true><<<blocks, kWideBlockThreads, 0, s>>>(T, I.n, I.d, perms, ld, batch, out, I.err);
        else wide_eval_block_kernel<false><<<blocks, kWideBlockThreads, 0, s>>>(T, I.n, I.d, perms, ld, batch, out, I.err);
    }
    return cudaGetLastError();
}

cudaError_t launch_wide_schedule(const Instance& I, bool ucd, const int16_t* perms, int64_t ld, int64_t batch,
                                 int64_t* C, int32_t* X, int64_t* start, int64_t* pen, cudaStream_t s) {
    if (batch <= 0) return cudaSuccess;
    const WideTab T = wide_tab(I);
    const void* k = ucd ? reinterpret_cast<const void*>(wide_schedule_kernel<true>)
                        : reinterpret_cast<const void*>(wide_schedule_kernel<false>);
    const int blocks = wide_blocks(k, I, kWideBlockThreads, batch);
    if (ucd) wide_schedule_kernel<true><<<blocks, kWideBlockThreads, 0, s>>>(T, I.n, I.d, perms, ld, batch, C, X, start, pen, I.err);
    else wide_schedule_kernel<false><<<blocks, kWideBlockThreads, 0, s>>>(T, I.n, I.d, perms, ld, batch, C, X, start, pen, I.err);
    return cudaGetLastError();
}

size_t wide_sa_workspace_bytes(const Instance& I, const SaLaunch& p) { return wide_ws(I, p).total; }

cudaError_t launch_wide_t0(const Instance& I, bool ucd, uint64_t seed, int64_t samples, double* T0_dev, void* ws,
                           cudaStream_t s) {
    SaLaunch p{};
    p.ucd = ucd;
    p.chains = 1;
    p.t0_samples = samples;
    const WideWs w = wide_ws(I, p);
    uint8_t* base = static_cast<uint8_t*>(ws);
    int64_t* Z = reinterpret_cast<int64_t*>(base + w.z_off);
    const int np = (I.n + 7) / 8 * 8;
    wide_t0_kernel<<<w.t0_blocks, kWSaWarps * 32, 0, s>>>(wide_tab(I), I.n, I.d, ucd, seed, samples,
                                                          reinterpret_cast<int16_t*>(base + w.t0s_off), np, Z);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    t0_reduce_kernel<<<1, 1024, 0, s>>>(Z, samples, T0_dev);
    return cudaGetLastError();
}

cudaError_t launch_wide_sa(Instance& I, const SaLaunch& p, void* ws, cudaStream_t s) {
    const WideWs w = wide_ws(I, p);
    uint8_t* base = static_cast<uint8_t*>(ws);
    const double* T0_dev = p.T0_in;
    if (!T0_dev && !(p.T0 > 0)) {
        double* t0w = reinterpret_cast<double*>(base + w.t0_off);
        const cudaError_t e = launch_wide_t0(I, p.ucd, p.seed, p.t0_samples, t0w, ws, s);
        if (e != cudaSuccess) return e;
        T0_dev = t0w;
    }
    WideSaArgs a{};
    a.T = wide_tab(I);
    a.n = I.n;
    a.d = I.d;
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
    a.np = (I.n + 7) / 8 * 8;
    a.cta_best = reinterpret_cast<long long*>(base + w.cta_off);
    a.trace = p.trace;
    a.chain_best = p.chain_best;
    a.chain_final = p.chain_final;
    a.init = p.init;
    a.init_ld = p.init_ld;
    a.err = I.err;
    if (p.ucd) wide_sa_kernel<true><<<w.blocks, kWSaWarps * 32, 0, s>>>(a);
    else wide_sa_kernel<false><<<w.blocks, kWSaWarps * 32, 0, s>>>(a);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    wide_sa_finalize<<<1, 256, 0, s>>>(a.cta_best, w.blocks, a.slots, a.np, I.n, I.best_wide, I.best_key,
                                       I.best_perm);
    return cudaGetLastError();
}

}  // namespace cdd
