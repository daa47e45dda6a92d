// dpso.cu -- discrete PSO (Alg. 2) with the position update of eq. (3).
//
// One warp per particle; the particle's sequence is rebuilt in the warp's shared-memory chain
// (chain.cuh) every iteration.  Per iteration ONE kernel does lines 6-7 of iteration t (eq. (3)
// then the O(n) evaluation) and lines 4-5 of iteration t+1 (personal best, then the swarm best by a
// CTA argmin + one atomicMin per CTA on the packed (value << 32 | particle id); the last CTA to
// finish copies the winner's personal best into the double-buffered swarm-best sequence).  The
// kernel boundary is the swarm-wide barrier Alg. 2 needs between lines 5 and 6.
//
// The crossovers keep the position of every job (inv) next to the sequence: a donor job is missing
// from the kept part iff its position lies outside it, so the donor row (read from global memory
// with 16-byte loads issued up front) is filtered with one shared-memory lookup per job, and the
// kept jobs are ranked by a warp scan of per-lane counts.  The instance tables are staged in
// shared memory once per CTA.
#include <cuda_runtime.h>

#include <climits>
#include <cstdlib>

#include "chain.cuh"
#include "device_common.cuh"
#include "internal.h"
#include "peer.cuh"

namespace cdd {
namespace {

constexpr int kDpWarps = 8;
constexpr int kDpThreads = kDpWarps * 32;
// resident CTAs per SM the iteration kernel is compiled for (registers: 3 -> 80, 4 -> 64, 5 -> 48)
#ifndef CDD_DP_MINB
#define CDD_DP_MINB 3
#endif

struct DpArgs {
    ChainTables T;
    int n;
    int32_t d;
    int64_t particles;
    uint64_t offset;
    double w, c1, c2;
    uint64_t seed;
    int16_t* pos;                  // [N][NP]
    int16_t* pb;                   // [N][NP]
    int32_t* zb;                   // [N]
    unsigned long long* gkey;      // [2]
    int16_t* gperm;                // [2][NP]
    // fused cross-GPU exchange (dpso_run_peer): world, rank, particles per rank, regions [world]
    int pw, pr;
    int64_t pper;
    uint8_t* const* pregions;
    int* err;  // instance error flag (bit 2: a peer never arrived)
    unsigned int* counter;         // [4]: CTA arrivals, the work counters of even / odd iterations,
                                   // the number of completed iterations (persistent kernel)
    int64_t* trace;
    int np;
};

template <int E, bool UCD>
struct DpSmem {
    static constexpr int NP = Chain<E, UCD>::NP;
    // per warp: the chain only (in the iteration kernel the position-of-job array lives in the
    // record area, which is rebuilt after the crossovers) ...
    static constexpr int BYTES = Chain<E, UCD>::BYTES;
    static constexpr int WARP = BYTES;
    // ... and, per CTA, the instance tables by job id: ab u32, p (or M) u8 [, X u8, gamma u16]
    static constexpr int TAB = NP * (UCD ? 8 : 5);
};

template <int E, bool UCD>
__device__ __forceinline__ void copy_out(int16_t* dst, const uint16_t* ids, int lane) {
    constexpr int NP = Chain<E, UCD>::NP;
    for (int o = lane * 8; o < NP; o += 256)
        *reinterpret_cast<int4*>(dst + o) = *reinterpret_cast<const int4*>(ids + o);
}

// CTA min of the warps' keys, one atomicMin per CTA, and the last CTA to finish copies the
// winning personal best into gperm[nxt] (and re-arms gkey[cur] for iteration t+2).
template <int E, bool UCD>
__device__ __forceinline__ void publish(const DpArgs& a, unsigned long long wkey, int nxt, int cur,
                                       bool rearm, uint32_t done = 0) {
    __shared__ unsigned long long s_key[kDpWarps];
    __shared__ bool s_last;
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    __threadfence();  // this CTA's personal-best writes before the arrival counter
    if (lane == 0) s_key[wib] = wkey;
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long m = s_key[0];
        for (int i = 1; i < kDpWarps; ++i) m = s_key[i] < m ? s_key[i] : m;
        if (m != ULLONG_MAX) atomicMin(&a.gkey[nxt], m);
        __threadfence();
        const unsigned int prev = atomicAdd(a.counter, 1u);
        s_last = prev == gridDim.x - 1;
    }
    __syncthreads();
    if (s_last) {
        __threadfence();
        const unsigned long long k = *(volatile unsigned long long*)&a.gkey[nxt];
        const int64_t li = (int64_t)((k & 0xffffffffull) - a.offset);
        const int16_t* src = a.pb + (size_t)li * a.np;
        for (int i = threadIdx.x; i < a.np; i += blockDim.x) a.gperm[(size_t)nxt * a.np + i] = src[i];
        if (a.pw > 1) {  // Alg. 2 line 5 over the global swarm (peer.cuh)
            __syncthreads();
            const unsigned long long local = *(volatile unsigned long long*)&a.gkey[nxt];
            const unsigned long long gk = peer_exchange_block(a.pregions, a.pw, a.pr, a.pper, a.np, done, nxt,
                                                              local, a.gperm + (size_t)nxt * a.np, a.np, a.err);
            if (threadIdx.x == 0) a.gkey[nxt] = gk;
            __threadfence();
            __syncthreads();
        }
        if (threadIdx.x == 0) {
            if (rearm) {
                a.gkey[cur] = ULLONG_MAX;
                a.counter[1 + cur] = 0u;  // every CTA has left its particle loop
            }
            *a.counter = 0u;
            if (done) {  // iteration done-1 complete: release the CTAs waiting for it
                __threadfence();
                asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(a.counter + 3), "r"(done) : "memory");
            }
        }
    }
}

// Alg. 2 lines 1-2 (random initial positions, evaluation) and lines 4-5 of iteration 0.
template <int E, bool UCD>
__global__ void __launch_bounds__(kDpThreads) dpso_init_kernel(DpArgs a) {
    using C = Chain<E, UCD>;
    extern __shared__ __align__(16) uint8_t smem[];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const C ch{smem + (size_t)wib * DpSmem<E, UCD>::BYTES};
    const int64_t total = (int64_t)gridDim.x * kDpWarps;
    unsigned long long wkey = ULLONG_MAX;
    for (int64_t i = (int64_t)blockIdx.x * kDpWarps + wib; i < a.particles; i += total) {
        const uint64_t gid = a.offset + (uint64_t)i;
        chain_fy_init<E, UCD>(ch, a.n, a.seed, kTagDpsoInit, gid, lane);
        // position k >= n carries the sentinel id k (>= n: a zero record in the iteration kernel's
        // table; distinct, so the position-of-job writes of the pads never collide); the
        // crossovers never move them
        for (int k = a.n + lane; k < C::NP; k += 32) ch.id()[k] = (uint16_t)k;
        __syncwarp();
        chain_build<E, UCD>(ch, a.T, a.n, lane);
        const int32_t z = chain_eval<E, UCD>(ch, lane, a.n, a.d);
        copy_out<E, UCD>(a.pos + (size_t)i * a.np, ch.id(), lane);
        copy_out<E, UCD>(a.pb + (size_t)i * a.np, ch.id(), lane);
        if (lane == 0) a.zb[i] = z;
        const unsigned long long key = ((unsigned long long)(uint32_t)z << 32) | (uint32_t)gid;
        wkey = key < wkey ? key : wkey;
        __syncwarp();
    }
    publish<E, UCD>(a, wkey, 0, 1, false);
}

// Instance tables by job id, staged in shared memory once per CTA at `t`: ab u32 [NP], p (or M)
// u8 [NP], UCDDCP: X u8 [NP], gamma u16 [NP].
template <int E, bool UCD>
struct DpTab {
    static constexpr int NP = Chain<E, UCD>::NP;
    const uint8_t* t;
    __device__ __forceinline__ uint32_t ab(int j) const { return reinterpret_cast<const uint32_t*>(t)[j]; }
    __device__ __forceinline__ uint8_t p(int j) const { return t[4 * NP + j]; }
    __device__ __forceinline__ uint8_t x(int j) const { return t[5 * NP + j]; }
    __device__ __forceinline__ uint16_t g(int j) const { return reinterpret_cast<const uint16_t*>(t + 6 * NP)[j]; }
};

template <int E, bool UCD>
__device__ __forceinline__ void stage_tables(uint8_t* t, const ChainTables& T, int n, bool fast) {
    constexpr int NP = Chain<E, UCD>::NP;
    if (fast) {  // CDD with 8-bit alpha, beta: one record alpha | beta << 8 | p << 16, zero past n
        for (int j = threadIdx.x; j < NP; j += blockDim.x)
            reinterpret_cast<uint32_t*>(t)[j] =
                j < n ? (uint32_t)__ldg(T.ab16 + j) | ((uint32_t)__ldg(T.p + j) << 16) : 0u;
        return;
    }
    for (int j = threadIdx.x; j < n; j += blockDim.x) {
        reinterpret_cast<uint32_t*>(t)[j] = __ldg(T.ab + j);
        t[4 * NP + j] = __ldg(T.p + j);
        if constexpr (UCD) {
            t[5 * NP + j] = __ldg(T.x + j);
            reinterpret_cast<uint16_t*>(t + 6 * NP)[j] = __ldg(T.g + j);
        }
    }
}

// Records of the sequence in id[] from the shared-memory tables (positions >= n: zero records).
template <int E, bool UCD>
__device__ __forceinline__ void chain_build_s(const Chain<E, UCD>& ch, const DpTab<E, UCD>& S, int n,
                                              int lane) {
    using C = Chain<E, UCD>;
    const uint16_t* ids = ch.id();
#pragma unroll 4
    for (int k = lane; k < C::NP; k += 32) {
        const bool v = k < n;
        const int j = v ? ids[k] : 0;
        ch.ab()[C::ab_w(k)] = v ? S.ab(j) : 0u;
        ch.pb()[C::pb_b(k)] = v ? S.p(j) : (uint8_t)0;
        if constexpr (UCD) {
            ch.xb()[C::pb_b(k)] = v ? S.x(j) : (uint8_t)0;
            ch.gh()[C::gh_h(k)] = v ? S.g(j) : (uint16_t)0;
        }
    }
    __syncwarp();
}

// The same records from the packed table (CDD, E >= 8): lane l builds its own segment
// [l*E, l*E+E) -- ids by 16-byte loads, one table load per position, the alpha|beta words and p
// bytes assembled by PRMT and written with 16-byte stores.  Positions past n hold the sentinel id,
// whose record is zero.
template <int E>
__device__ __forceinline__ void chain_build_fast(const Chain<E, false>& ch, const uint32_t* rtab, int lane) {
    using C = Chain<E, false>;
    static_assert(E >= 8, "16-byte segments");
    const uint16_t* ids = ch.id() + lane * E;
    uint32_t* abw = ch.ab() + lane * C::AB_STRIDE;
    uint8_t* pb = ch.pb() + lane * C::PB_STRIDE;
#pragma unroll
    for (int v = 0; v < E / 8; ++v) {
        const uint4 q = *reinterpret_cast<const uint4*>(ids + 8 * v);
        const uint32_t w[4] = {q.x, q.y, q.z, q.w};
        uint32_t r[8];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            r[2 * j] = rtab[w[j] & 0xffffu];
            r[2 * j + 1] = rtab[w[j] >> 16];
        }
        uint32_t a[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) a[j] = __byte_perm(r[j], 0u, 0x4140u);  // alpha | beta << 16
        *reinterpret_cast<uint4*>(abw + 8 * v) = make_uint4(a[0], a[1], a[2], a[3]);
        *reinterpret_cast<uint4*>(abw + 8 * v + 4) = make_uint4(a[4], a[5], a[6], a[7]);
        const uint32_t p0 = __byte_perm(__byte_perm(r[0], r[1], 0x0062u), __byte_perm(r[2], r[3], 0x0062u), 0x5410u);
        const uint32_t p1 = __byte_perm(__byte_perm(r[4], r[5], 0x0062u), __byte_perm(r[6], r[7], 0x0062u), 0x5410u);
        *reinterpret_cast<uint2*>(pb + 8 * v) = make_uint2(p0, p1);
    }
    __syncwarp();
}

__device__ __forceinline__ uint32_t warp_excl_scan(uint32_t v, int lane, uint32_t* total) {
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(kFull, x, o);
        if (lane >= o) x += y;
    }
    *total = __shfl_sync(kFull, x, 31);
    return x - v;
}

// Crossover fill: the jobs of `donor` (global row, n entries) for which keep(inv[job]) holds are
// written, in donor order, to positions dst(0), dst(1), ... of ids[], and inv[] follows them.
// The donor row is read with 16-byte loads issued up front (lane L holds donor positions
// [8L + 256 r, 8L + 256 r + 8)); the rank of a kept job is a warp scan of per-lane counts.
template <int E>
constexpr int kDonorRounds = (32 * E + 255) / 256;  // 16-byte rounds per lane

template <int E>
__device__ __forceinline__ void load_donor(const int16_t* __restrict__ donor, int lane,
                                           uint4 (&q)[kDonorRounds<E>]) {
#pragma unroll
    for (int r = 0; r < kDonorRounds<E>; ++r) {
        const int o = 8 * lane + 256 * r;
        q[r] = o < 32 * E ? __ldg(reinterpret_cast<const uint4*>(donor + o)) : make_uint4(0, 0, 0, 0);
    }
}

// (the donor row already in registers, loaded by load_donor)
template <int E, class Keep, class Dst>
__device__ __forceinline__ void fill_from(uint16_t* ids, uint16_t* inv, const uint4 (&q)[kDonorRounds<E>],
                                          int n, int lane, Keep&& keep, Dst&& dst) {
    constexpr int R = kDonorRounds<E>;
    uint32_t km[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const uint32_t w[4] = {q[r].x, q[r].y, q[r].z, q[r].w};
        uint32_t m = 0;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const int k = 8 * lane + 256 * r + j;
            const uint32_t job = (j & 1) ? (w[j >> 1] >> 16) : (w[j >> 1] & 0xffffu);
            if (k < n && keep((int)inv[job])) m |= 1u << j;
        }
        km[r] = m;
    }
    __syncwarp();
    int out = 0;
#pragma unroll
    for (int r = 0; r < R; ++r) {
        uint32_t tot;
        int idx = out + (int)warp_excl_scan((uint32_t)__popc(km[r]), lane, &tot);
        out += (int)tot;
        const uint32_t w[4] = {q[r].x, q[r].y, q[r].z, q[r].w};
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            if ((km[r] >> j) & 1u) {
                const uint32_t job = (j & 1) ? (w[j >> 1] >> 16) : (w[j >> 1] & 0xffffu);
                const int pos = dst(idx++);
                ids[pos] = (uint16_t)job;
                inv[job] = (uint16_t)pos;
            }
        }
    }
    __syncwarp();
}

// Lines 6-7 of iteration t, then lines 4-5 of iteration t+1.
template <int E, bool UCD, bool FAST>
__global__ void __launch_bounds__(kDpThreads, E >= 32 ? 2 : CDD_DP_MINB) dpso_iter_kernel(DpArgs a, int64_t t0,
                                                                                          int64_t t1) {
    using C = Chain<E, UCD>;
    constexpr int NP = C::NP;
    extern __shared__ __align__(16) uint8_t smem[];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    stage_tables<E, UCD>(smem, a.T, a.n, FAST);
    const DpTab<E, UCD> S{smem};
    const C ch{smem + DpSmem<E, UCD>::TAB + (size_t)wib * DpSmem<E, UCD>::WARP};
    uint16_t* ids = ch.id();
    uint16_t* inv = reinterpret_cast<uint16_t*>(ch.ab());  // position of each job (crossovers only)
    const int n = a.n;
  for (int64_t t = t0; t < t1; ++t) {
    const int cur = (int)(t & 1), nxt = cur ^ 1;
    if (a.trace && blockIdx.x == 0 && threadIdx.x == 0) a.trace[t] = (int64_t)(a.gkey[cur] >> 32);
    const int16_t* g = a.gperm + (size_t)cur * a.np;
    const int64_t total = (int64_t)gridDim.x * kDpWarps;
    unsigned long long wkey = ULLONG_MAX;
    // the swarm best is the same for every particle of the iteration: loaded once per warp
    uint4 qg[kDonorRounds<E>];
    load_donor<E>(g, lane, qg);
    __syncthreads();
    // first particle of a warp by its index; for long rows (E >= 32, n > 512) the rest come from a
    // work counter, so a warp is done only when the swarm is (particles / warps is rarely integral
    // and a static stride leaves the last round to a fraction of the warps): n = 1000 7.7 -> 6.9 ms
    // per 200 iterations; for short rows the atomic costs more than the imbalance (n = 100:
    // 2.5 -> 2.9 ms), so they keep the static stride
    for (int64_t i = (int64_t)blockIdx.x * kDpWarps + wib; i < a.particles;) {
        const uint64_t gid = a.offset + (uint64_t)i;
        // the personal best is issued together with the position: one round trip, not two
        uint4 qb[kDonorRounds<E>];
        load_donor<E>(a.pb + (size_t)i * a.np, lane, qb);
        // the position to shared memory (16-byte loads) and the position of every job
        {
            const int16_t* gp = a.pos + (size_t)i * a.np;
#pragma unroll
            for (int o = lane * 8; o < NP; o += 256) {
                const uint4 x = __ldg(reinterpret_cast<const uint4*>(gp + o));
                *reinterpret_cast<uint4*>(ids + o) = x;
                const uint32_t w[4] = {x.x, x.y, x.z, x.w};
#pragma unroll  // (position k >= n holds the sentinel id k: distinct entries, never read)
                for (int j = 0; j < 8; ++j)
                    inv[(j & 1) ? (w[j >> 1] >> 16) : (w[j >> 1] & 0xffffu)] = (uint16_t)(o + j);
            }
            __syncwarp();
        }
        // random words of (t, particle): lane 0 -> block 0, lane 1 -> block 1
        const uint4 wv = rng_block(a.seed, (uint32_t)t, gid, kTagDpso, (uint32_t)(lane & 1));
        const uint32_t a0 = __shfl_sync(kFull, wv.x, 0), a1 = __shfl_sync(kFull, wv.y, 0);
        const uint32_t a2 = __shfl_sync(kFull, wv.z, 0), a3 = __shfl_sync(kFull, wv.w, 0);
        const uint32_t b0 = __shfl_sync(kFull, wv.x, 1), b1 = __shfl_sync(kFull, wv.y, 1);
        const uint32_t b2 = __shfl_sync(kFull, wv.z, 1), b3 = __shfl_sync(kFull, wv.w, 1);
        const double u2 = 2.3283064365386962890625e-10;
        // lambda = w (+) F1(p): swap of two distinct positions (Floyd)
        if (__dmul_rn(__dadd_rn((double)a0, 0.5), u2) < a.w) {
            const int pa = (int)bnd(a1, (uint32_t)n - 1u);
            int qb = (int)bnd(a2, (uint32_t)n);
            if (qb == pa) qb = n - 1;
            if (lane == 0) {
                const uint16_t x = ids[pa], y = ids[qb];
                ids[pa] = y;
                ids[qb] = x;
                inv[y] = (uint16_t)pa;
                inv[x] = (uint16_t)qb;
            }
            __syncwarp();
        }
        // delta = c1 (+) F2(lambda, p^b): one-point crossover with the personal best -- lambda's
        // first c jobs stay, the others follow in personal-best order
        if (__dmul_rn(__dadd_rn((double)a3, 0.5), u2) < a.c1) {
            const int c = 1 + (int)bnd(b0, (uint32_t)n - 1u);
            fill_from<E>(ids, inv, qb, n, lane, [c](int at) { return at >= c; },
                         [c](int idx) { return c + idx; });
        }
        // p(t+1) = c2 (+) F3(delta, g): two-point crossover with the swarm best -- delta[q0..q1]
        // stays, the other positions take the remaining jobs in swarm-best order
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
            fill_from<E>(ids, inv, qg, n, lane, [q0, q1](int at) { return at < q0 || at > q1; },
                         [q0, span](int idx) { return idx < q0 ? idx : idx + span; });
        }
        // line 7: evaluate
        if constexpr (FAST)
            chain_build_fast<E>(ch, reinterpret_cast<const uint32_t*>(smem), lane);
        else
            chain_build_s<E, UCD>(ch, S, n, lane);
        const int32_t z = chain_eval<E, UCD>(ch, lane, n, a.d);
        copy_out<E, UCD>(a.pos + (size_t)i * a.np, ids, lane);
        // line 4 (iteration t+1): personal best
        const int32_t zb = a.zb[i];
        int32_t best = zb;
        if (z < zb) {
            best = z;
            copy_out<E, UCD>(a.pb + (size_t)i * a.np, ids, lane);
            if (lane == 0) a.zb[i] = z;
        }
        const unsigned long long key = ((unsigned long long)(uint32_t)best << 32) | (uint32_t)gid;
        wkey = key < wkey ? key : wkey;
        if constexpr (E >= 32) {
            unsigned int w = 0;
            if (lane == 0) w = atomicAdd(a.counter + 1 + cur, 1u);
            i = total + (int64_t)__shfl_sync(kFull, w, 0);
        } else {
            i += total;
        }
        __syncwarp();
    }
    // line 5 (iteration t+1): swarm best
    publish<E, UCD>(a, wkey, nxt, cur, true, (uint32_t)(t + 1));
    // the next iteration needs the swarm best of this one: wait for the last CTA's release
    // (the grid is co-resident: cooperative launch)
    if (t + 1 < t1) {
        if (threadIdx.x == 0) {
            uint32_t v;
            do {
                asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(a.counter + 3) : "memory");
            } while ((int32_t)(v - (uint32_t)(t + 1)) < 0);
        }
        __syncthreads();
    }
  }
}

__global__ void dpso_end_kernel(const unsigned long long* gkey, const int16_t* gperm, int n,
                                unsigned long long* best_key, int16_t* best_perm) {
    if (threadIdx.x == 0) *best_key = *gkey;
    for (int i = threadIdx.x; i < n; i += blockDim.x) best_perm[i] = gperm[i];
}

// ------------------------------------------------------------------------------- host side
constexpr size_t kAlign = 256;
inline size_t align_up(size_t x) { return (x + kAlign - 1) / kAlign * kAlign; }

struct DpWs {
    size_t pos, inv, pb, zb, gkey, gperm, counter, slots, total;
};

DpWs dp_layout(int np, int64_t N) {
    DpWs w{};
    w.pos = 0;
    w.inv = align_up(w.pos + (size_t)N * np * 2);
    w.pb = align_up(w.inv + (size_t)N * np * 2);
    w.zb = align_up(w.pb + (size_t)N * np * 2);
    w.gkey = align_up(w.zb + (size_t)N * 4);
    w.gperm = align_up(w.gkey + 16);
    w.counter = align_up(w.gperm + (size_t)2 * np * 2);
    w.slots = align_up(w.counter + 32);  // counters [4], the group publish's running keys [2]
    // one row per CTA and parity for the group layout's publish (a CTA holds >= 4 particles)
    const int64_t ctas = std::min<int64_t>(kDpsoMaxCtas, (N + 3) / 4 + 1);
    w.total = align_up(w.slots + (size_t)2 * ctas * np * 2);
    return w;
}

ChainTables dp_tables(const Instance& I, bool ucd) {
    return ucd ? ChainTables{I.tab_ab, I.tab_m, I.tab_x, I.tab_g}
               : ChainTables{I.tab_ab, I.tab_p, nullptr, nullptr, I.ab16_ok ? I.tab_ab16 : nullptr};
}

DpsoWsPtrs ws_ptrs(const Instance& I, const DpsoLaunch& p, void* ws) {
    const int np = dpso_np(I.n);
    const DpWs w = dp_layout(np, p.particles);
    uint8_t* b = static_cast<uint8_t*>(ws);
    DpsoWsPtrs r{};
    r.pos = reinterpret_cast<int16_t*>(b + w.pos);
    r.inv = reinterpret_cast<int16_t*>(b + w.inv);
    r.pb = reinterpret_cast<int16_t*>(b + w.pb);
    r.zb = reinterpret_cast<int32_t*>(b + w.zb);
    r.gkey = reinterpret_cast<unsigned long long*>(b + w.gkey);
    r.gperm = reinterpret_cast<int16_t*>(b + w.gperm);
    r.counter = reinterpret_cast<unsigned int*>(b + w.counter);
    r.slots = reinterpret_cast<int16_t*>(b + w.slots);
    r.np = np;
    return r;
}

bool use_group(const Instance& I) { return dpsog_usable(I); }

template <int E>
DpArgs make_args(const Instance& I, const DpsoLaunch& p, void* ws) {
    const DpWs w = dp_layout(dpso_np(I.n), p.particles);
    uint8_t* b = static_cast<uint8_t*>(ws);
    DpArgs a{};
    a.T = dp_tables(I, p.ucd);
    a.n = I.n;
    a.d = I.d_eff;
    a.particles = p.particles;
    a.offset = p.particle_offset;
    a.w = p.w;
    a.c1 = p.c1;
    a.c2 = p.c2;
    a.seed = p.seed;
    a.pos = reinterpret_cast<int16_t*>(b + w.pos);
    a.pb = reinterpret_cast<int16_t*>(b + w.pb);
    a.zb = reinterpret_cast<int32_t*>(b + w.zb);
    a.gkey = reinterpret_cast<unsigned long long*>(b + w.gkey);
    a.gperm = reinterpret_cast<int16_t*>(b + w.gperm);
    a.counter = reinterpret_cast<unsigned int*>(b + w.counter);
    a.err = I.err;
    if (p.peer && I.peer && I.peer->open) {
        a.pw = I.peer->world;
        a.pr = I.peer->rank;
        a.pper = p.particles;
        a.pregions = I.peer->d_regions;
    }
    a.trace = p.gbest_trace;
    a.np = dpso_np(I.n);
    return a;
}

template <class K>
int grid_for(const Instance& I, K kern, size_t smem, int64_t particles) {
    int sms = 148, occ = 1;
    resident_ctas(reinterpret_cast<const void*>(kern), I.device, kDpThreads, smem, &sms, &occ);
    int64_t need = (particles + kDpWarps - 1) / kDpWarps;
    const int64_t cap = (int64_t)sms * occ;
    if (need > cap) need = cap;
    return (int)(need < 1 ? 1 : need);
}

template <int E, bool UCD>
cudaError_t begin_e(Instance& I, const DpsoLaunch& p, void* ws, cudaStream_t s) {
    const DpArgs a = make_args<E>(I, p, ws);
    cudaError_t e = cudaMemsetAsync(a.gkey, 0xff, 2 * sizeof(unsigned long long), s);
    if (e == cudaSuccess) e = cudaMemsetAsync(a.counter, 0, 4 * sizeof(unsigned int), s);
    if (e != cudaSuccess) return e;
    const size_t smem = kDpWarps * (size_t)DpSmem<E, UCD>::BYTES;
    const int blocks = grid_for(I, dpso_init_kernel<E, UCD>, smem, p.particles);
    dpso_init_kernel<E, UCD><<<blocks, kDpThreads, smem, s>>>(a);
    return cudaGetLastError();
}

// Iterations t0..t1-1 (the grid is sized once: the attribute queries cost more host time than a
// launch).
template <int E, bool UCD>
cudaError_t iter_e(Instance& I, const DpsoLaunch& p, void* ws, int64_t t0, int64_t t1, cudaStream_t s) {
    const DpArgs a = make_args<E>(I, p, ws);
    const size_t smem = DpSmem<E, UCD>::TAB + kDpWarps * (size_t)DpSmem<E, UCD>::WARP;
    constexpr bool can_fast = !UCD && E >= 8;
    const bool fast = can_fast && I.ab16_ok;
    auto kern = fast ? dpso_iter_kernel<E, UCD, can_fast> : dpso_iter_kernel<E, UCD, false>;
    const int blocks = grid_for(I, kern, smem, p.particles);
    if (t1 <= t0) return cudaSuccess;
    // one persistent launch for iterations t0..t1-1: the CTAs wait for each other between
    // iterations (Alg. 2 lines 4-5 need the whole swarm), so they must be co-resident -- a
    // cooperative launch guarantees it (the grid is at most SMs x resident CTAs)
    void* args[] = {const_cast<DpArgs*>(&a), &t0, &t1};
    cudaError_t e = cudaLaunchCooperativeKernel(reinterpret_cast<const void*>(kern), dim3(blocks),
                                                dim3(kDpThreads), args, smem, s);
    if (e == cudaErrorCooperativeLaunchTooLarge || e == cudaErrorNotSupported) {
        // co-residency not available here: one launch per iteration (no in-kernel wait)
        (void)cudaGetLastError();
        for (int64_t t = t0; t < t1; ++t) {
            kern<<<blocks, kDpThreads, smem, s>>>(a, t, t + 1);
            const cudaError_t le = cudaGetLastError();
            if (le != cudaSuccess) return le;
        }
        return cudaSuccess;
    }
    return e;
}

template <int E>
cudaError_t begin_d(Instance& I, const DpsoLaunch& p, void* ws, cudaStream_t s) {
    return p.ucd ? begin_e<E, true>(I, p, ws, s) : begin_e<E, false>(I, p, ws, s);
}
template <int E>
cudaError_t iter_d(Instance& I, const DpsoLaunch& p, void* ws, int64_t t0, int64_t t1, cudaStream_t s) {
    return p.ucd ? iter_e<E, true>(I, p, ws, t0, t1, s) : iter_e<E, false>(I, p, ws, t0, t1, s);
}

}  // namespace

size_t dpso_peer_region_bytes(int n) { return kPeerPermOff + (size_t)2 * dpso_np(n) * sizeof(int16_t); }

size_t dpso_workspace_bytes(const Instance& I, const DpsoLaunch& p) {
    return dp_layout(dpso_np(I.n), p.particles).total;
}

cudaError_t dpso_begin(Instance& I, const DpsoLaunch& p, void* ws, cudaStream_t s) {
    if (use_group(I)) return dpsog_begin(I, p, ws_ptrs(I, p, ws), s);
    switch (sa_e_for_n(I.n)) {
        case 1: return begin_d<1>(I, p, ws, s);
        case 2: return begin_d<2>(I, p, ws, s);
        case 4: return begin_d<4>(I, p, ws, s);
        case 8: return begin_d<8>(I, p, ws, s);
        case 16: return begin_d<16>(I, p, ws, s);
        default: return begin_d<32>(I, p, ws, s);
    }
}

cudaError_t dpso_iterate(Instance& I, const DpsoLaunch& p, void* ws, int64_t t0, int64_t t1,
                         cudaStream_t s) {
    if (use_group(I)) return dpsog_iterate(I, p, ws_ptrs(I, p, ws), t0, t1, s);
    switch (sa_e_for_n(I.n)) {
        case 1: return iter_d<1>(I, p, ws, t0, t1, s);
        case 2: return iter_d<2>(I, p, ws, t0, t1, s);
        case 4: return iter_d<4>(I, p, ws, t0, t1, s);
        case 8: return iter_d<8>(I, p, ws, t0, t1, s);
        case 16: return iter_d<16>(I, p, ws, t0, t1, s);
        default: return iter_d<32>(I, p, ws, t0, t1, s);
    }
}

void dpso_gbest(const Instance& I, const DpsoLaunch& p, void* ws, int64_t t, int64_t** key,
                int16_t** perm) {
    const int np = dpso_np(I.n);
    const DpWs w = dp_layout(np, p.particles);
    uint8_t* b = static_cast<uint8_t*>(ws);
    const int par = (int)(t & 1);
    if (key) *key = reinterpret_cast<int64_t*>(b + w.gkey) + par;
    if (perm) *perm = reinterpret_cast<int16_t*>(b + w.gperm) + (size_t)par * np;
}

cudaError_t dpso_end(Instance& I, const DpsoLaunch& p, void* ws, cudaStream_t s) {
    int64_t* key = nullptr;
    int16_t* perm = nullptr;
    dpso_gbest(I, p, ws, p.iters, &key, &perm);
    dpso_end_kernel<<<1, 256, 0, s>>>(reinterpret_cast<unsigned long long*>(key), perm, I.n,
                                      I.best_key, I.best_perm);
    return cudaGetLastError();
}

}  // namespace cdd
