// dpso_group.cu -- discrete PSO (Alg. 2; update eq. (3)) on the group layout:
// G = 8 lanes per particle, 4 particles per warp, the particle's sequence (ids) and the position of
// every job (inv) in shared memory, and the SA group evaluator (sa_group.cuh) for line 7.
//
// Against the warp-per-particle kernel of dpso.cu (kept for instances whose alpha or beta exceed 8
// bits), per particle and iteration:
//  * inv is persistent (global, next to the position): the crossovers keep it up to date as they
//    place jobs, so it is loaded with 16-byte loads instead of being rebuilt by n scattered stores;
//  * the Philox words of eq. (3)'s decisions cost one block per lane for four particles;
//  * the swarm best of iteration t (Alg. 2 line 5) is needed only by F3 (line 6's third term): every
//    warp loads its particle, applies F1 and F2 and only then waits for the release of the swarm
//    best -- the grid-wide barrier of lines 4-5 is split into an arrival (the publish at the end of
//    iteration t-1) and a wait that overlaps the first part of iteration t;
//  * every particle of the swarm is resident at once when the grid allows (8192 particles at
//    n = 500: 2048 warps), so an iteration has no partial last round.
// Bit-identical to the oracle (same Philox words, same operators R15, same ties R16).
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>
#include <cstdlib>

#include "device_common.cuh"
#include "internal.h"
#include "peer.cuh"
#include "sa_group.cuh"

namespace cdd {
namespace {

constexpr int kDgSmemBudget = 224 * 1024;  // per CTA: one big CTA per SM -> few publish atomics

struct DgArgs {
    int n;
    int32_t d;
    int64_t particles;
    uint64_t offset;
    double w, c1, c2;
    uint64_t seed;
    int16_t* pos;               // [N][np]
    int16_t* inv;               // [N][np]: position of each job in pos
    int16_t* pb;                // [N][np]
    int32_t* zb;                // [N]
    unsigned long long* gkey;   // [2]
    int16_t* gperm;             // [2][np]
    int pw, pr;                 // fused cross-GPU exchange: world, rank (pw > 1)
    int64_t pper;
    uint8_t* const* pregions;
    int* err;
    unsigned int* counter;      // [0] CTA arrivals, [3] iterations whose swarm best is released;
                                // [1], [2]: arrivals per parity, [4..7]: running keys per parity
                                // (single-GPU publish)
    int16_t* slots;             // [2][gridDim][np]: each CTA's best personal-best row per parity
    unsigned long long* fkey;   // [2] = counter + 4: the single-GPU publish's running minima
    int64_t* trace;
    int np;
    int quad;  // CDD: the evaluator's quad level (Instance::quad_level)
    // tables by job id (global; staged in shared memory per CTA): CDD alpha|beta<<8 | p<<16;
    // UCDDCP alpha|beta<<8 | gamma<<16 and M | X<<8
    const uint16_t* ab16;
    const uint8_t* p;
    const uint8_t* m;
    const uint8_t* x;
    const uint16_t* g;
};

// Shared memory of a CTA: the instance tables, the swarm best of the current iteration (staged once
// per CTA), then per particle its chain records (inv aliases them) and its ids.  W warps per CTA:
// as many as the budget holds (<= 16), so a swarm needs few CTAs (one publish atomic each).
template <int DG, int E, bool UCD>
struct DgSmem {
    using C = GChain<DG, E, UCD>;
    static constexpr int NP = C::NP;
    static constexpr int GROUP = (C::BYTES + 4 * NP + 15) / 16 * 16;  // chain records, ids, inv
    static constexpr int IDS = C::BYTES, INV = C::BYTES + 2 * NP;
    static constexpr int TAB = UCD ? NP * 6 : NP * 4;
    static constexpr int TAB_AL = (TAB + 15) / 16 * 16;
    static constexpr int G_OFF = TAB_AL;                  // swarm best ids [NP]
    static constexpr int P_OFF = G_OFF + 2 * NP;
    static constexpr int PPW = 32 / DG;                   // particles per warp
    static constexpr int FIT = (kDgSmemBudget - P_OFF) / (PPW * GROUP);
    static constexpr int W = FIT >= 16 ? 16 : (FIT >= 1 ? FIT : 1);
    static constexpr int THREADS = 32 * W;
    static constexpr int PER_CTA = W * PPW;
    static constexpr int CTA = P_OFF + PER_CTA * GROUP;
};

__device__ __forceinline__ uint32_t half16(const uint4& v, int j) {
    const uint32_t w = j < 4 ? (j < 2 ? v.x : v.y) : (j < 6 ? v.z : v.w);
    return (j & 1) ? (w >> 16) : (w & 0xffffu);
}

// minimum of a u64 over the 32 lanes
__device__ __forceinline__ unsigned long long warp_min64(unsigned long long v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const unsigned long long u = __shfl_xor_sync(kFull, v, o);
        v = u < v ? u : v;
    }
    return v;
}

// Alg. 2 line 5 for the swarm after iteration `done` (0: after line 2): CTA min of the particles'
// keys, one atomicMin per CTA on gkey[nxt] (no round trip: a reduction in L2), the arrival, and the
// last CTA to arrive copies the winner's personal best to gperm[nxt] (exchanging it across GPUs
// first when pw > 1), re-arms gkey[cur] and releases counter[3] = done.  The swarm best of Alg. 2 is
// the minimum over the personal bests, which never increase, so an unchanged key means an unchanged
// row: then the copy is skipped (every CTA still holds that row in shared memory), except on the
// last publish of a launch (`final`), whose row the next launch and the end kernel read.
template <int W>
__device__ void dg_publish(const DgArgs& a, unsigned long long wkey, int nxt, int cur, bool rearm, uint32_t done,
                           bool trace, bool final) {
    __shared__ unsigned long long s_key[2];
    __shared__ unsigned long long s_wkey[W];
    __shared__ bool s_last;
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int nw = (int)(blockDim.x >> 5);
    wkey = warp_min64(wkey);
    if (lane == 0) s_wkey[wib] = wkey;
    __syncthreads();  // the CTA's personal-best writes happen before thread 0's (cumulative) fence
    if (threadIdx.x == 0) {
        unsigned long long mk = s_wkey[0];
        for (int i = 1; i < nw; ++i) mk = s_wkey[i] < mk ? s_wkey[i] : mk;
        if (mk != ULLONG_MAX) atomicMin(a.gkey + nxt, mk);
        __threadfence();
        const unsigned int prev = atomicAdd(a.counter, 1u);
        s_last = prev == gridDim.x - 1;
        if (s_last) {
            __threadfence();  // every other CTA's writes (fenced before its arrival) visible
            s_key[0] = __ldcg(a.gkey + nxt);
            s_key[1] = rearm ? __ldcg(a.gkey + cur) : ULLONG_MAX;  // the previous release's key
        }
    }
    __syncthreads();
    if (s_last) {
        const unsigned long long k = s_key[0];
        const bool copy = final || a.pw > 1 || k != s_key[1];
        const int64_t li = (int64_t)((k & 0xffffffffull) - a.offset);
        const int16_t* src = a.pb + (size_t)li * a.np;
        int16_t* dst = a.gperm + (size_t)nxt * a.np;
        if (copy)
            for (int i = threadIdx.x; i < a.np; i += blockDim.x) dst[i] = __ldcg(src + i);
        unsigned long long gk = k;
        if (a.pw > 1) {
            __syncthreads();
            gk = peer_exchange_block(a.pregions, a.pw, a.pr, a.pper, a.np, done, nxt, k, dst, a.np, a.err);
            if (threadIdx.x == 0) a.gkey[nxt] = gk;
            __threadfence();
            __syncthreads();
        }
        if (threadIdx.x == 0) {
            if (trace && a.trace) a.trace[done] = (int64_t)(gk >> 32);  // line 5 of iteration `done`
            a.gkey[nxt] = gk;
            if (rearm) a.gkey[cur] = ULLONG_MAX;
            *a.counter = 0u;
            __threadfence();
            asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(a.counter + 3), "r"(done) : "memory");
        }
    }
}

// The split barrier of Alg. 2 lines 4-5: every warp of the CTA finishes the part of iteration t
// that does not need the swarm best (F1, F2), then one CTA barrier; warp 0 waits for the release
// of iteration t's swarm best (acquire on L2) and copies it into shared memory; a second barrier
// and the CTA goes on with F3.  Waiting warps sit at the barrier (no spinning), and the swarm
// best crosses L2 once per CTA.
__device__ __forceinline__ uint32_t dg_acquire(const unsigned int* p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

template <int NP>
__device__ __forceinline__ void dg_cta_stage(const DgArgs& a, uint16_t* g_sm, uint32_t t, unsigned long long* s_gk) {
    __syncthreads();
    if (threadIdx.x < 32) {
        unsigned long long k = 0;
        if (threadIdx.x == 0) {
            while ((int32_t)(dg_acquire(a.counter + 3) - t) < 0) {
            }
            k = __ldcg(a.gkey + (t & 1));
        }
        k = __shfl_sync(kFull, k, 0);
        // the swarm best row changes only with its key (the copy of an unchanged row is skipped)
        if (k != *s_gk) {
            const int16_t* src = a.gperm + (size_t)(t & 1) * a.np;
            for (int o = 8 * (int)threadIdx.x; o < NP; o += 256)
                *reinterpret_cast<uint4*>(g_sm + o) = __ldcg(reinterpret_cast<const uint4*>(src + o));
            __syncwarp();
            if (threadIdx.x == 0) *s_gk = k;
        }
    }
    __syncthreads();
}

// Single-GPU publish (no last-CTA step on the critical path).  Every CTA keeps the row of its own
// best key in slots[parity][cta] (rewritten only when that key changes, before the arrival), adds
// the key to gkey[nxt] by atomicMin and arrives on the parity's counter; the waiting CTAs see the
// count, read the swarm key and copy the row from the winner's slot.  Slot rows of a parity are
// rewritten two publishes later, after every CTA has passed the publish in between, i.e. after
// every CTA has read them.  The keys go to fkey[parity], which is never re-armed inside a launch:
// the minimum over the personal bests never increases, so the running minimum of a parity is the
// swarm best of its latest publish (fkey only ever holds keys of this launch's particles; gkey,
// which a host-side exchange may overwrite between launches, is read at the launch's first stage
// only).  The last publish of a launch (`final`) writes gkey[nxt] and gperm[nxt], releases
// counter[3] (the end kernel, the next launch and the multi-GPU protocol read those) and re-arms
// the parity counters and fkey for the next launch.
__device__ __forceinline__ unsigned int dg_target(int64_t done, int64_t t0) {
    return (unsigned int)((((done - (t0 + 1)) >> 1) + 1) * (int64_t)gridDim.x);
}
__device__ __forceinline__ int dg_cta_of(const DgArgs& a, unsigned long long k, int per_cta) {
    const int64_t li = (int64_t)((k & 0xffffffffull) - a.offset);
    return (int)((li / per_cta) % (int64_t)gridDim.x);
}

template <int W>
__device__ void dg_publish_fast(const DgArgs& a, unsigned long long wkey, int nxt, int64_t done, int64_t t0,
                                bool final, unsigned long long* s_slot, int per_cta) {
    __shared__ unsigned long long s_wk[W];
    __shared__ unsigned long long s_mk;
    __shared__ bool s_last;
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int nw = (int)(blockDim.x >> 5);
    wkey = warp_min64(wkey);
    if (lane == 0) s_wk[wib] = wkey;
    __syncthreads();  // also: the CTA's personal-best rows are written
    if (threadIdx.x == 0) {
        unsigned long long mk = s_wk[0];
        for (int i = 1; i < nw; ++i) mk = s_wk[i] < mk ? s_wk[i] : mk;
        s_mk = mk;
    }
    __syncthreads();
    const unsigned long long mk = s_mk;
    int16_t* slot = a.slots + ((size_t)nxt * gridDim.x + blockIdx.x) * a.np;
    if (mk != ULLONG_MAX && mk != s_slot[nxt]) {  // CTA-uniform
        const int64_t li = (int64_t)((mk & 0xffffffffull) - a.offset);
        const uint4* src = reinterpret_cast<const uint4*>(a.pb + (size_t)li * a.np);
        for (int o = threadIdx.x; o < a.np / 8; o += blockDim.x) reinterpret_cast<uint4*>(slot)[o] = __ldcg(src + o);
        __syncthreads();
        if (threadIdx.x == 0) s_slot[nxt] = mk;
    }
    if (threadIdx.x == 0) {
        if (mk != ULLONG_MAX) atomicMin(a.fkey + nxt, mk);
        __threadfence();
        if (!final) {
            atomicAdd(a.counter + 1 + nxt, 1u);
        } else {
            const unsigned int prev = atomicAdd(a.counter + 1 + nxt, 1u);
            s_last = prev + 1u == dg_target(done, t0);
        }
    }
    if (!final) return;
    __syncthreads();
    if (!s_last) return;
    __shared__ unsigned long long s_k;
    if (threadIdx.x == 0) {
        __threadfence();
        s_k = __ldcg(a.fkey + nxt);
    }
    __syncthreads();
    const unsigned long long k = s_k;
    const uint4* src = reinterpret_cast<const uint4*>(a.slots + ((size_t)nxt * gridDim.x + dg_cta_of(a, k, per_cta)) * a.np);
    for (int o = threadIdx.x; o < a.np / 8; o += blockDim.x)
        reinterpret_cast<uint4*>(a.gperm + (size_t)nxt * a.np)[o] = __ldcg(src + o);
    __syncthreads();
    if (threadIdx.x == 0) {
        a.gkey[nxt] = k;
        a.counter[1] = 0u;
        a.counter[2] = 0u;
        a.fkey[0] = a.fkey[1] = ULLONG_MAX;
        __threadfence();
        asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(a.counter + 3), "r"((uint32_t)done) : "memory");
    }
}

template <int NP>
__device__ __forceinline__ void dg_stage_fast(const DgArgs& a, uint16_t* g_sm, int64_t t, int64_t t0,
                                              unsigned long long* s_gk, int per_cta) {
    __syncthreads();
    if (threadIdx.x < 32) {
        unsigned long long k = 0;
        if (threadIdx.x == 0) {
            if (t > t0) {
                const unsigned int target = dg_target(t, t0);
                while (dg_acquire(a.counter + 1 + (int)(t & 1)) < target) {
                }
            }
            k = __ldcg((t > t0 ? a.fkey : a.gkey) + (t & 1));
            if (t > t0 && blockIdx.x == 0 && a.trace) a.trace[t] = (int64_t)(k >> 32);  // line 5 of iteration t
        }
        k = __shfl_sync(kFull, k, 0);
        if (k != *s_gk) {  // the swarm best row changes only with its key
            const int16_t* src = t > t0 ? a.slots + ((size_t)(t & 1) * gridDim.x + dg_cta_of(a, k, per_cta)) * a.np
                                        : a.gperm + (size_t)(t & 1) * a.np;
            for (int o = 8 * (int)threadIdx.x; o < NP; o += 256)
                *reinterpret_cast<uint4*>(g_sm + o) = __ldcg(reinterpret_cast<const uint4*>(src + o));
            __syncwarp();
            if (threadIdx.x == 0) *s_gk = k;
        }
    }
    __syncthreads();
}

template <int DG, int E, bool UCD>
__device__ __forceinline__ void dg_stage_tables(uint8_t* t, const DgArgs& a) {
    constexpr int NP = DgSmem<DG, E, UCD>::NP;
    uint32_t* t32 = reinterpret_cast<uint32_t*>(t);
    for (int j = threadIdx.x; j < NP; j += blockDim.x) {
        const bool v = j < a.n;
        if constexpr (UCD) {
            t32[j] = v ? (uint32_t)__ldg(a.ab16 + j) | ((uint32_t)__ldg(a.g + j) << 16) : 0u;
            reinterpret_cast<uint16_t*>(t + 4 * NP)[j] =
                v ? (uint16_t)((uint32_t)__ldg(a.m + j) | ((uint32_t)__ldg(a.x + j) << 8)) : (uint16_t)0;
        } else {
            t32[j] = v ? (uint32_t)__ldg(a.ab16 + j) | ((uint32_t)__ldg(a.p + j) << 16) : 0u;
        }
    }
}

// Crossover fill on the group: the jobs of the donor row (global) for which keep(inv[job]) holds
// are written, in donor order, to positions dst(0), dst(1), ... of ids, and inv follows them.
// Lane l filters donor positions [l*E, l*E+E) (16-byte chunks), a group scan of the counts gives
// each lane's first rank, and a second pass over the (L1-resident) chunks places the kept jobs.
// Every lane of the warp must call (act = false: this group has nothing to do).
// CG: the donor is the swarm best, written by another SM during this launch -- read from L2
template <int DG, int E, bool CG, class Keep, class Dst>
__device__ __forceinline__ void dg_fill(uint16_t* ids, uint16_t* inv, const int16_t* donor, int n, int l,
                                        bool act, Keep&& keep, Dst&& dst) {
    auto ld = [&](int k) -> uint4 {
        const uint4* p = reinterpret_cast<const uint4*>(donor + k);
        return CG ? __ldcg(p) : *p;
    };
    constexpr int NCH = E / 8;
    uint32_t bits[(NCH + 3) / 4];
#pragma unroll
    for (int i = 0; i < (NCH + 3) / 4; ++i) bits[i] = 0u;
    int cnt = 0;
    if (act) {
#pragma unroll
        for (int ch = 0; ch < NCH; ++ch) {
            const int k0 = l * E + 8 * ch;
            if (k0 < n) {
                const uint4 v = ld(k0);
                uint32_t m = 0;
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                    const uint32_t job = half16(v, j);
                    if (k0 + j < n && keep((int)inv[job])) m |= 1u << j;
                }
                bits[ch >> 2] |= m << (8 * (ch & 3));
                cnt += __popc(m);
            }
        }
    }
    const int base = (int)(gscan<DG>((uint32_t)cnt) - (uint32_t)cnt);
    if (act && cnt) {
        int idx = base;
#pragma unroll
        for (int ch = 0; ch < NCH; ++ch) {
            const uint32_t m = (bits[ch >> 2] >> (8 * (ch & 3))) & 0xffu;
            if (m) {
                const uint4 v = ld(l * E + 8 * ch);
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                    if ((m >> j) & 1u) {
                        const uint32_t job = half16(v, j);
                        const int pos = dst(idx++);
                        ids[pos] = (uint16_t)job;
                        inv[job] = (uint16_t)pos;
                    }
                }
            }
        }
    }
    __syncwarp();
}

// Records of the group's sequence (ids) into the chain rows, and this lane's totals.
template <int DG, int E, bool UCD>
__device__ __forceinline__ uint2 dg_build(const GChain<DG, E, UCD>& ch, const uint16_t* ids, const uint8_t* tab,
                                          int n, int l) {
    using C = GChain<DG, E, UCD>;
    constexpr int NP = C::NP;
    const uint32_t* t32 = reinterpret_cast<const uint32_t*>(tab);
    const uint16_t* t16 = reinterpret_cast<const uint16_t*>(tab + 4 * NP);
    uint8_t* pr = ch.pb() + l * C::PS;
    uint32_t tAB = 0, tP = 0;
#pragma unroll 2
    for (int c = 0; c < E; c += 8) {
        const int k0 = l * E + c;
        const uint4 q = *reinterpret_cast<const uint4*>(ids + k0);
        uint32_t r[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) r[j] = t32[half16(q, j)];  // pads hold ids >= n: zero records
        if constexpr (UCD) {
            uint8_t* abr = reinterpret_cast<uint8_t*>(ch.ab()) + l * C::AS;
            uint32_t w[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                w[j] = __byte_perm(r[2 * j], r[2 * j + 1], 0x5410u);  // alpha|beta of two positions
                tAB = __dp4a(w[j], 0x00010001u, tAB);
                tAB += __dp4a(w[j], 0x01000100u, 0u) << 16;
            }
            *reinterpret_cast<uint4*>(abr + 2 * c) = make_uint4(w[0], w[1], w[2], w[3]);
            uint32_t g2[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) g2[j] = __byte_perm(r[2 * j], r[2 * j + 1], 0x7632u);  // gamma pairs
            *reinterpret_cast<uint4*>(reinterpret_cast<uint8_t*>(ch.gh()) + l * C::GS + 2 * c) =
                make_uint4(g2[0], g2[1], g2[2], g2[3]);
            uint32_t mx[8];
#pragma unroll
            for (int j = 0; j < 8; ++j) mx[j] = (uint32_t)t16[half16(q, j)];
            // M bytes and X bytes of the 8 positions
            const uint32_t m0 = __byte_perm(__byte_perm(mx[0], mx[1], 0x0040u), __byte_perm(mx[2], mx[3], 0x0040u), 0x5410u);
            const uint32_t m1 = __byte_perm(__byte_perm(mx[4], mx[5], 0x0040u), __byte_perm(mx[6], mx[7], 0x0040u), 0x5410u);
            const uint32_t x0 = __byte_perm(__byte_perm(mx[0], mx[1], 0x0051u), __byte_perm(mx[2], mx[3], 0x0051u), 0x5410u);
            const uint32_t x1 = __byte_perm(__byte_perm(mx[4], mx[5], 0x0051u), __byte_perm(mx[6], mx[7], 0x0051u), 0x5410u);
            *reinterpret_cast<uint2*>(pr + c) = make_uint2(m0, m1);
            *reinterpret_cast<uint2*>(ch.xb() + l * C::PS + c) = make_uint2(x0, x1);
            tP = __dp4a(m0, 0x01010101u, __dp4a(m1, 0x01010101u, tP));
        } else {
            // CDD byte rows: alpha (byte 0 of a record), beta (byte 1), P (byte 2)
            auto quad = [&](int b, uint32_t sel) {
                return __byte_perm(__byte_perm(r[b], r[b + 1], sel), __byte_perm(r[b + 2], r[b + 3], sel), 0x5410u);
            };
            const uint32_t a0 = quad(0, 0x0040u), a1 = quad(4, 0x0040u);
            const uint32_t b0 = quad(0, 0x0051u), b1 = quad(4, 0x0051u);
            const uint32_t p0 = quad(0, 0x0062u), p1 = quad(4, 0x0062u);
            const int o = l * C::RS + c;
            *reinterpret_cast<uint2*>(ch.a8() + o) = make_uint2(a0, a1);
            *reinterpret_cast<uint2*>(ch.b8() + o) = make_uint2(b0, b1);
            *reinterpret_cast<uint2*>(pr + c) = make_uint2(p0, p1);
            tAB += __dp4a(a0, 0x01010101u, __dp4a(a1, 0x01010101u, 0u)) |
                   (__dp4a(b0, 0x01010101u, __dp4a(b1, 0x01010101u, 0u)) << 16);
            tP = __dp4a(p0, 0x01010101u, __dp4a(p1, 0x01010101u, tP));
        }
    }
    __syncwarp();
    return make_uint2(tAB, tP);
}

template <int DG, int E, bool UCD>
__device__ __forceinline__ int32_t dg_eval(const GChain<DG, E, UCD>& ch, int l, int gbase, int n, int32_t d, uint2 t,
                                          int quad) {
    if constexpr (UCD)
        return gchain_eval_ucddcp<DG, E>(ch, l, gbase, n, t.x);
    else
        return gchain_eval_cdd<DG, E>(ch, l, gbase, n, d, t.x, t.y, quad);
}

// row copies between global memory and the group's shared-memory arrays (16 bytes per lane-step)
template <int DG, int NP>
__device__ __forceinline__ void dg_load_row(uint16_t* dst, const int16_t* src, int l) {
#pragma unroll 4
    for (int o = 8 * l; o < NP; o += 8 * DG)
        *reinterpret_cast<uint4*>(dst + o) = *reinterpret_cast<const uint4*>(src + o);
}
template <int DG, int NP>
__device__ __forceinline__ void dg_store_row(int16_t* dst, const uint16_t* src, int l) {
#pragma unroll 4
    for (int o = 8 * l; o < NP; o += 8 * DG)
        *reinterpret_cast<uint4*>(dst + o) = *reinterpret_cast<const uint4*>(src + o);
}

// Alg. 2 lines 1-2 and lines 4-5 of iteration 0.
template <int DG, int E, bool UCD>
__global__ void __launch_bounds__(DgSmem<DG, E, UCD>::THREADS) dpsog_init_kernel(DgArgs a) {
    using S = DgSmem<DG, E, UCD>;
    using C = GChain<DG, E, UCD>;
    constexpr int NP = S::NP;
    extern __shared__ __align__(16) uint8_t smem[];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int grp = lane / DG, l = lane % DG, gbase = grp * DG;
    dg_stage_tables<DG, E, UCD>(smem, a);
    __syncthreads();
    uint8_t* gb = smem + S::P_OFF + (size_t)(wib * (32 / DG) + grp) * S::GROUP;
    const C ch{gb};
    uint16_t* ids = reinterpret_cast<uint16_t*>(gb + C::BYTES);
    uint16_t* inv = reinterpret_cast<uint16_t*>(gb + S::INV);
    uint32_t* words = reinterpret_cast<uint32_t*>(ch.pb());  // Philox staging (P rows are free here)
    const int n = a.n;
    const int per_cta = (int)(blockDim.x >> 5) * (32 / DG);
    const int64_t groups = (int64_t)gridDim.x * per_cta;
    unsigned long long wkey = ULLONG_MAX;
    for (int64_t i0 = (int64_t)blockIdx.x * per_cta + wib * (32 / DG); i0 < a.particles; i0 += groups) {
        const int64_t i = i0 + grp;
        const bool active = i < a.particles;
        const uint64_t gid = a.offset + (uint64_t)(active ? i : 0);
        // R10: Fisher-Yates of the identity with the words of (TAG_DPSO_INIT, gid), on group lane 0
        // position k >= n holds the sentinel id k (>= n: a zero record in the tables; distinct, so
        // the crossovers' inv lookups of the pads stay in bounds and never collide)
        for (int k = l; k < NP; k += DG) ids[k] = (uint16_t)k;
        const int nw = n - 1;
        for (int r0 = 0; r0 < nw; r0 += 4 * DG) {
            __syncwarp();
            const int b = r0 / 4 + l;
            if (4 * b < nw) reinterpret_cast<uint4*>(words)[l] = rng_block(a.seed, (uint32_t)b, gid, kTagDpsoInit, 0);
            __syncwarp();
            if (l == 0) {
                const int r1 = min(nw, r0 + 4 * DG);
                for (int q = r0; q < r1; ++q) {
                    const int ii = n - 1 - q;
                    const uint32_t j = bnd(words[q - r0], (uint32_t)ii + 1u);
                    const uint16_t t = ids[ii];
                    ids[ii] = ids[j];
                    ids[j] = t;
                }
            }
        }
        __syncwarp();
        for (int k = l; k < NP; k += DG) inv[ids[k]] = (uint16_t)k;
        __syncwarp();
        if (active) {
            dg_store_row<DG, NP>(a.pos + (size_t)i * a.np, ids, l);
            dg_store_row<DG, NP>(a.pb + (size_t)i * a.np, ids, l);
            dg_store_row<DG, NP>(a.inv + (size_t)i * a.np, inv, l);
        }
        __syncwarp();
        const uint2 t = dg_build<DG, E, UCD>(ch, ids, smem, n, l);
        const int32_t z = dg_eval<DG, E, UCD>(ch, l, gbase, n, a.d, t, a.quad);
        if (active && l == 0) a.zb[i] = z;
        const unsigned long long key = active ? ((unsigned long long)(uint32_t)z << 32) | (uint32_t)gid : ULLONG_MAX;
        wkey = key < wkey ? key : wkey;
        __syncwarp();
    }
    dg_publish<S::W>(a, wkey, 0, 1, false, 0u, false, true);
}

// ---- warp-wide crossovers (one particle at a time, all 32 lanes): a crossover is applied with
// probability c1 / c2 per particle, so a warp only pays for the particles that apply it (with the
// four particles of a warp in lockstep it would pay whenever any of them does).

template <int NP>
__device__ __forceinline__ void dw_load_row(uint16_t* dst, const int16_t* src, int lane) {
#pragma unroll
    for (int o = 8 * lane; o < NP; o += 256)
        *reinterpret_cast<uint4*>(dst + o) = *reinterpret_cast<const uint4*>(src + o);
}
template <int NP>
__device__ __forceinline__ void dw_store_row(int16_t* dst, const uint16_t* src, int lane) {
#pragma unroll
    for (int o = 8 * lane; o < NP; o += 256)
        *reinterpret_cast<uint4*>(dst + o) = *reinterpret_cast<const uint4*>(src + o);
}

// The donor row's jobs for which keep(inv[job]) holds, in donor order, to positions dst(0),
// dst(1), ... of ids (inv follows).  Lane L holds donor positions [L*K, L*K+K) in registers
// (K = NP/32, pairs of 16-bit ids), filters them with one shared-memory lookup each, and a warp
// scan of the counts gives its first rank.
template <int NP, class Keep, class Dst>
__device__ __forceinline__ void dw_fill(uint16_t* ids, uint16_t* inv, const int16_t* donor, int n, int lane,
                                        Keep&& keep, Dst&& dst) {
    constexpr int K = NP / 32;
    static_assert(K >= 2 && K <= 32, "2..32 positions per lane");
    uint32_t w[K / 2];
    const int16_t* src = donor + lane * K;
    if constexpr (K >= 8) {
#pragma unroll
        for (int v = 0; v < K / 8; ++v) {
            const uint4 q = *reinterpret_cast<const uint4*>(src + 8 * v);
            w[4 * v] = q.x; w[4 * v + 1] = q.y; w[4 * v + 2] = q.z; w[4 * v + 3] = q.w;
        }
    } else if constexpr (K == 4) {
        const uint2 q = *reinterpret_cast<const uint2*>(src);
        w[0] = q.x; w[1] = q.y;
    } else {
        w[0] = *reinterpret_cast<const uint32_t*>(src);
    }
    uint32_t m = 0;
#pragma unroll
    for (int j = 0; j < K; ++j) {
        const uint32_t job = (j & 1) ? (w[j >> 1] >> 16) : (w[j >> 1] & 0xffffu);
        m |= (keep((int)inv[job]) ? 1u : 0u) << j;
    }
    const int lim = n - lane * K;  // positions past n (padding) never count
    if (lim < K) m &= lim <= 0 ? 0u : ((1u << lim) - 1u);
    const uint32_t cnt = (uint32_t)__popc(m);
    uint32_t x = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(kFull, x, o);
        if (lane >= o) x += y;
    }
    int idx = (int)(x - cnt);
    if (m) {
#pragma unroll
        for (int j = 0; j < K; ++j) {
            if ((m >> j) & 1u) {
                const uint32_t job = (j & 1) ? (w[j >> 1] >> 16) : (w[j >> 1] & 0xffffu);
                const int pos = dst(idx++);
                ids[pos] = (uint16_t)job;
                inv[job] = (uint16_t)pos;
            }
        }
    }
    __syncwarp();
}

// Iterations t0..t1-1: lines 6-7 of iteration t, then lines 4-5 of iteration t+1.
template <int DG, int E, bool UCD>
__global__ void __launch_bounds__(DgSmem<DG, E, UCD>::THREADS, 1) dpsog_iter_kernel(DgArgs a, int64_t t0, int64_t t1) {
    using S = DgSmem<DG, E, UCD>;
    using C = GChain<DG, E, UCD>;
    constexpr int NP = S::NP;
    extern __shared__ __align__(16) uint8_t smem[];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int grp = lane / DG, l = lane % DG, gbase = grp * DG;
    dg_stage_tables<DG, E, UCD>(smem, a);
    __syncthreads();
    constexpr int PPW = 32 / DG;
    uint8_t* wb = smem + S::P_OFF + (size_t)(wib * PPW) * S::GROUP;  // this warp's particles
    auto ids_of = [&](int p) { return reinterpret_cast<uint16_t*>(wb + (size_t)p * S::GROUP + S::IDS); };
    auto inv_of = [&](int p) { return reinterpret_cast<uint16_t*>(wb + (size_t)p * S::GROUP + S::INV); };
    const C ch{wb + (size_t)grp * S::GROUP};
    uint16_t* ids = ids_of(grp);
    const int n = a.n;
    const int per_cta = (int)(blockDim.x >> 5) * PPW;  // the launch may use fewer than S::W warps
    const int64_t groups = (int64_t)gridDim.x * per_cta;
    // resident: every particle has its own slot, so its position and inv stay in shared memory
    // from the first iteration of the launch to the last (loaded / stored once per launch)
    const bool resident = groups >= a.particles;
    const int64_t i0r = (int64_t)blockIdx.x * per_cta + wib * PPW;
    // every slot starts from the identity (valid ids < NP): the slots past the swarm are evaluated
    // too (their results are discarded) and must not gather outside the tables
    for (int p = 0; p < PPW; ++p)
        for (int k = lane; k < NP; k += 32) {
            ids_of(p)[k] = (uint16_t)k;
            inv_of(p)[k] = (uint16_t)k;
        }
    __syncwarp();
    if (resident)
        for (int p = 0; p < PPW; ++p)
            if (i0r + p < a.particles) {
                dw_load_row<NP>(ids_of(p), a.pos + (size_t)(i0r + p) * a.np, lane);
                dw_load_row<NP>(inv_of(p), a.inv + (size_t)(i0r + p) * a.np, lane);
            }
    const double u2 = 2.3283064365386962890625e-10;
    uint16_t* g_sm = reinterpret_cast<uint16_t*>(smem + S::G_OFF);
    __shared__ unsigned long long s_gk;  // key of the swarm best row held in g_sm
    __shared__ unsigned long long s_slot[2];  // keys of this CTA's slot rows (single-GPU publish)
    if (threadIdx.x == 0) s_gk = s_slot[0] = s_slot[1] = ULLONG_MAX;
    const bool fast = a.pw <= 1;
    auto stage = [&](int64_t t) {
        if (fast)
            dg_stage_fast<NP>(a, g_sm, t, t0, &s_gk, per_cta);
        else
            dg_cta_stage<NP>(a, g_sm, (uint32_t)t, &s_gk);
    };
    // swarm best at line 5 of iteration t0 (after a host-side exchange when stepping across GPUs)
    if (a.trace && blockIdx.x == 0 && threadIdx.x == 0) a.trace[t0] = (int64_t)(a.gkey[t0 & 1] >> 32);
    for (int64_t t = t0; t < t1; ++t) {
        const int cur = (int)(t & 1), nxt = cur ^ 1;
        bool have_g = false;
        unsigned long long wkey = ULLONG_MAX;
        // CTA-uniform trip count (the split barrier is a CTA barrier); warps past the swarm idle
        for (int64_t ib = (int64_t)blockIdx.x * per_cta; ib < a.particles; ib += groups) {
            const int64_t i0 = ib + wib * PPW;
            const int64_t i = i0 + grp;
            const bool active = i < a.particles;
            const uint64_t gid = a.offset + (uint64_t)(active ? i : 0);
            // the warp's particles, one at a time: position and inv rows
#pragma unroll
            for (int p = 0; p < PPW; ++p)
                if (!resident && i0 + p < a.particles) {
                    dw_load_row<NP>(ids_of(p), a.pos + (size_t)(i0 + p) * a.np, lane);
                    dw_load_row<NP>(inv_of(p), a.inv + (size_t)(i0 + p) * a.np, lane);
                }
            const int32_t zb = active ? a.zb[i] : 0;
            // eq. (3)'s words of particle p: block 0 on lane 2p, block 1 on lane 2p+1 (R15, D4)
            const int pp = (lane >> 1) & (PPW - 1);
            const uint4 wv = rng_block(a.seed, (uint32_t)t, a.offset + (uint64_t)(i0 + pp), kTagDpso, (uint32_t)(lane & 1));
            __syncwarp();
#pragma unroll
            for (int p = 0; p < PPW; ++p) {
                if (i0 + p >= a.particles) break;
                const uint32_t a0 = __shfl_sync(kFull, wv.x, 2 * p), a1 = __shfl_sync(kFull, wv.y, 2 * p);
                const uint32_t a2 = __shfl_sync(kFull, wv.z, 2 * p), a3 = __shfl_sync(kFull, wv.w, 2 * p);
                const uint32_t b0 = __shfl_sync(kFull, wv.x, 2 * p + 1);
                uint16_t* id = ids_of(p);
                uint16_t* iv = inv_of(p);
                // lambda = w (+) F1(p): swap of two distinct positions (Floyd)
                if (lane == 0 && __dmul_rn(__dadd_rn((double)a0, 0.5), u2) < a.w) {
                    const int pa = (int)bnd(a1, (uint32_t)n - 1u);
                    int qb = (int)bnd(a2, (uint32_t)n);
                    if (qb == pa) qb = n - 1;
                    const uint16_t x = id[pa], y = id[qb];
                    id[pa] = y;
                    id[qb] = x;
                    iv[y] = (uint16_t)pa;
                    iv[x] = (uint16_t)qb;
                }
                __syncwarp();
                // delta = c1 (+) F2(lambda, p^b): lambda's first c jobs stay, the others follow in
                // personal-best order
                if (__dmul_rn(__dadd_rn((double)a3, 0.5), u2) < a.c1) {
                    const int c = 1 + (int)bnd(b0, (uint32_t)n - 1u);
                    dw_fill<NP>(id, iv, a.pb + (size_t)(i0 + p) * a.np, n, lane, [c](int at) { return at >= c; },
                                [c](int idx) { return c + idx; });
                }
            }
            // everything below needs the swarm best of iteration t (F3) or writes the personal
            // best the last CTA of the previous publish may still be copying
            if (!have_g) {
                stage(t);
                have_g = true;
            }
#pragma unroll
            for (int p = 0; p < PPW; ++p) {
                if (i0 + p >= a.particles) break;
                const uint32_t b1 = __shfl_sync(kFull, wv.y, 2 * p + 1), b2 = __shfl_sync(kFull, wv.z, 2 * p + 1);
                const uint32_t b3 = __shfl_sync(kFull, wv.w, 2 * p + 1);
                // p(t+1) = c2 (+) F3(delta, g): delta[q0..q1] stays, the other positions take the
                // remaining jobs in swarm-best order
                if (__dmul_rn(__dadd_rn((double)b1, 0.5), u2) < a.c2) {
                    int q0 = (int)bnd(b2, (uint32_t)n - 1u);
                    int q1 = (int)bnd(b3, (uint32_t)n);
                    if (q1 == q0) q1 = n - 1;
                    if (q0 > q1) {
                        const int x = q0;
                        q0 = q1;
                        q1 = x;
                    }
                    const int span = q1 - q0 + 1;
                    const uint32_t ext = (uint32_t)(q1 - q0);
                    dw_fill<NP>(ids_of(p), inv_of(p), reinterpret_cast<const int16_t*>(g_sm), n, lane,
                                [q0, ext](int at) { return (uint32_t)(at - q0) > ext; },
                                [q0, span](int idx) { return idx < q0 ? idx : idx + span; });
                }
                if (!resident || t + 1 == t1) {
                    dw_store_row<NP>(a.pos + (size_t)(i0 + p) * a.np, ids_of(p), lane);
                    dw_store_row<NP>(a.inv + (size_t)(i0 + p) * a.np, inv_of(p), lane);
                }
            }
            __syncwarp();
            // line 7: evaluate
            const uint2 tt = dg_build<DG, E, UCD>(ch, ids, smem, n, l);
            const int32_t z = dg_eval<DG, E, UCD>(ch, l, gbase, n, a.d, tt, a.quad);
            // line 4 (iteration t+1): personal best
            int32_t best = zb;
            if (active && z < zb) {
                best = z;
                dg_store_row<DG, NP>(a.pb + (size_t)i * a.np, ids, l);
                if (l == 0) a.zb[i] = z;
            }
            const unsigned long long key =
                active ? ((unsigned long long)(uint32_t)best << 32) | (uint32_t)gid : ULLONG_MAX;
            wkey = key < wkey ? key : wkey;
            __syncwarp();
        }
        // a warp without particles never waited: the previous publish must be complete before
        // this one re-uses its key slot and counter
        if (!have_g) stage(t);
        // line 5 (iteration t+1): swarm best (traced here when iteration t+1 runs in this launch)
        if (fast)
            dg_publish_fast<S::W>(a, wkey, nxt, t + 1, t0, t + 1 == t1, s_slot, per_cta);
        else
            dg_publish<S::W>(a, wkey, nxt, cur, true, (uint32_t)(t + 1), t + 1 < t1, t + 1 == t1);
    }
}

__global__ void dpsog_end_kernel(const unsigned long long* gkey, const int16_t* gperm, int n,
                                 unsigned long long* best_key, int16_t* best_perm) {
    if (threadIdx.x == 0) *best_key = *gkey;
    for (int i = threadIdx.x; i < n; i += blockDim.x) best_perm[i] = gperm[i];
}

int dg_pow2(int c) {
    int e = 1;
    while (e < c) e <<= 1;
    return e;
}

// Launch shape: as few warps per CTA as spread the swarm over every SM (one CTA per SM, all
// particles resident when they fit), else the widest CTA and as many rounds as needed.
struct DgShape {
    int blocks, warps;
    size_t smem;
};
template <int DG, int E, bool UCD, class K>
DgShape dg_shape(const Instance& I, K kern, int64_t particles) {
    using S = DgSmem<DG, E, UCD>;
    int sms = 148, occ = 1;
    resident_ctas(reinterpret_cast<const void*>(kern), I.device, S::THREADS, S::CTA, &sms, &occ);
    int warps = (int)std::min<int64_t>(S::W, std::max<int64_t>(1, (particles + (int64_t)sms * S::PPW - 1) /
                                                                        ((int64_t)sms * S::PPW)));
    DgShape sh{0, warps, (size_t)S::P_OFF + (size_t)warps * S::PPW * S::GROUP};
    int occ2 = 1;
    resident_ctas(reinterpret_cast<const void*>(kern), I.device, warps * 32, sh.smem, &sms, &occ2);
    const int64_t per = (int64_t)warps * S::PPW;
    const int64_t need = (particles + per - 1) / per;
    sh.blocks = (int)std::max<int64_t>(1, std::min<int64_t>(std::min<int64_t>(need, (int64_t)sms * occ2), kDpsoMaxCtas));
    return sh;
}

template <int DG, int E, bool UCD>
cudaError_t dg_begin(const Instance& I, const DgArgs& a, int64_t particles, cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(a.gkey, 0xff, 2 * sizeof(unsigned long long), s);
    if (e == cudaSuccess) e = cudaMemsetAsync(a.counter, 0, 4 * sizeof(unsigned int), s);
    if (e == cudaSuccess) e = cudaMemsetAsync(a.fkey, 0xff, 2 * sizeof(unsigned long long), s);
    if (e != cudaSuccess) return e;
    const DgShape sh = dg_shape<DG, E, UCD>(I, dpsog_init_kernel<DG, E, UCD>, particles);
    dpsog_init_kernel<DG, E, UCD><<<sh.blocks, sh.warps * 32, sh.smem, s>>>(a);
    return cudaGetLastError();
}

template <int DG, int E, bool UCD>
cudaError_t dg_iter(const Instance& I, const DgArgs& a, int64_t particles, int64_t t0, int64_t t1, cudaStream_t s) {
    if (t1 <= t0) return cudaSuccess;
    auto kern = dpsog_iter_kernel<DG, E, UCD>;
    const DgShape sh = dg_shape<DG, E, UCD>(I, kern, particles);
    // persistent launch for t0..t1-1: the CTAs wait for each other's publish between iterations, so
    // they must be co-resident -- a cooperative launch guarantees it
    void* args[] = {const_cast<DgArgs*>(&a), &t0, &t1};
    cudaError_t e = cudaLaunchCooperativeKernel(reinterpret_cast<const void*>(kern), dim3(sh.blocks),
                                                dim3(sh.warps * 32), args, sh.smem, s);
    if (e == cudaErrorCooperativeLaunchTooLarge || e == cudaErrorNotSupported) {
        (void)cudaGetLastError();  // no co-residency: one launch per iteration
        for (int64_t t = t0; t < t1; ++t) {
            kern<<<sh.blocks, sh.warps * 32, sh.smem, s>>>(a, t, t + 1);
            const cudaError_t le = cudaGetLastError();
            if (le != cudaSuccess) return le;
        }
        return cudaSuccess;
    }
    return e;
}

}  // namespace

// lanes per particle (CDD_DPSO_G=8 / 16 overrides; measured in DESIGN.md §8) and positions per lane
int dpsog_lanes() {
    static const int g = [] {
        const char* v = getenv("CDD_DPSO_G");
        const int x = v ? atoi(v) : 8;
        return x == 16 ? 16 : 8;
    }();
    return g;
}
int dpsog_e(int G, int n) { return std::max(8, dg_pow2((n + G - 1) / G)); }

// the workspace rows of the DPSO kernels (every layout uses the same stride)
int dpso_np(int n) { return std::max(32 * sa_e_for_n(n), std::max(8 * dpsog_e(8, n), 16 * dpsog_e(16, n))); }

// the group layout for n <= 512 (all particles resident in shared memory at config 4's 8192 x n=500);
// longer rows need two rounds of 7.4 KB particles and the warp-per-particle kernel is faster there
// (n = 1000: 2.6e8 vs 2.2e8 particle-evaluations/s); CDD_DPSO=group / warp forces one
bool dpsog_usable(const Instance& I) {
    if (!I.ab16_ok || I.wide) return false;
    const char* v = getenv("CDD_DPSO");
    if (v && v[0] == 'w') return false;
    if (v && v[0] == 'g') return I.n <= 1024;
    return I.n <= 512;
}

#define CDD_DG_SWITCH(G_, E_, CALL)                           \
    switch ((G_) * 1000 + (E_)) {                             \
        case 8008: CALL(8, 8)                                 \
        case 8016: CALL(8, 16)                                \
        case 8032: CALL(8, 32)                                \
        case 8064: CALL(8, 64)                                \
        case 8128: CALL(8, 128)                               \
        case 16008: CALL(16, 8)                               \
        case 16016: CALL(16, 16)                              \
        case 16032: CALL(16, 32)                              \
        default: CALL(16, 64)                                 \
    }

static DgArgs dg_args(const Instance& I, const DpsoLaunch& p, const DpsoWsPtrs& w) {
    DgArgs a{};
    a.n = I.n;
    a.d = I.d_eff;
    a.particles = p.particles;
    a.offset = p.particle_offset;
    a.w = p.w;
    a.c1 = p.c1;
    a.c2 = p.c2;
    a.seed = p.seed;
    a.pos = w.pos;
    a.inv = w.inv;
    a.pb = w.pb;
    a.zb = w.zb;
    a.gkey = w.gkey;
    a.gperm = w.gperm;
    a.counter = w.counter;
    a.slots = w.slots;
    a.fkey = reinterpret_cast<unsigned long long*>(w.counter + 4);
    a.err = I.err;
    if (p.peer && I.peer && I.peer->open) {
        a.pw = I.peer->world;
        a.pr = I.peer->rank;
        a.pper = p.particles;
        a.pregions = I.peer->d_regions;
    }
    a.trace = p.gbest_trace;
    a.np = w.np;
    a.quad = I.quad_level();
    a.ab16 = I.tab_ab16;
    a.p = I.tab_p;
    a.m = I.tab_m;
    a.x = I.tab_x;
    a.g = I.tab_g;
    return a;
}

cudaError_t dpsog_begin(Instance& I, const DpsoLaunch& p, const DpsoWsPtrs& w, cudaStream_t s) {
    const DgArgs a = dg_args(I, p, w);
    const int G = dpsog_lanes();
#define CDD_DG_BEGIN(GG, EE) \
    return p.ucd ? dg_begin<GG, EE, true>(I, a, p.particles, s) : dg_begin<GG, EE, false>(I, a, p.particles, s);
    CDD_DG_SWITCH(G, dpsog_e(G, I.n), CDD_DG_BEGIN)
#undef CDD_DG_BEGIN
}

cudaError_t dpsog_iterate(Instance& I, const DpsoLaunch& p, const DpsoWsPtrs& w, int64_t t0, int64_t t1,
                          cudaStream_t s) {
    const DgArgs a = dg_args(I, p, w);
    const int G = dpsog_lanes();
#define CDD_DG_ITER(GG, EE)                                                                   \
    return p.ucd ? dg_iter<GG, EE, true>(I, a, p.particles, t0, t1, s)                        \
                 : dg_iter<GG, EE, false>(I, a, p.particles, t0, t1, s);
    CDD_DG_SWITCH(G, dpsog_e(G, I.n), CDD_DG_ITER)
#undef CDD_DG_ITER
}

}  // namespace cdd
