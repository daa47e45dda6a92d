// dpso.cu -- discrete PSO (Alg. 2) with the position update of eq. (3).
//
// One warp per particle; the particle's sequence is rebuilt in the warp's shared-memory chain
// (chain.cuh) every iteration.  Per iteration ONE kernel does lines 6-7 of iteration t (eq. (3)
// then the O(n) evaluation) and lines 4-5 of iteration t+1 (personal best, then the swarm best by a
// CTA argmin + one atomicMin per CTA on the packed (value << 32 | particle id); the last CTA to
// finish copies the winner's personal best into the double-buffered swarm-best sequence).  The
// kernel boundary is the swarm-wide barrier Alg. 2 needs between lines 5 and 6.
//
// The crossovers use a job-membership bitmap in shared memory and ballot/popc stream compaction
// over the donor sequence (personal best for F2, swarm best for F3).
#include <cuda_runtime.h>

#include <climits>

#include "chain.cuh"
#include "device_common.cuh"
#include "internal.h"

namespace cdd {
namespace {

constexpr int kDpWarps = 8;
constexpr int kDpThreads = kDpWarps * 32;

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
    unsigned int* counter;         // [1]
    int64_t* trace;
    int np;
};

template <int E, bool UCD>
struct DpSmem {
    static constexpr int NP = Chain<E, UCD>::NP;
    // chain + 32-word membership bitmap + the two donor sequences (personal / swarm best)
    static constexpr int BYTES = Chain<E, UCD>::BYTES + 128 + 2 * NP * 2;
};

__device__ __forceinline__ uint32_t lanemask_lt(int lane) { return (1u << lane) - 1u; }

// Membership bitmap of ids[lo..hi] (inclusive).
__device__ __forceinline__ void build_bitmap(uint32_t* bm, const uint16_t* ids, int lo, int hi,
                                             int lane) {
    bm[lane] = 0u;
    __syncwarp();
    for (int k = lo + lane; k <= hi; k += 32) {
        const int j = ids[k];
        atomicOr(&bm[j >> 5], 1u << (j & 31));
    }
    __syncwarp();
}

// Writes the jobs of `donor` (shared, n entries) that are not in the bitmap, in donor order, to
// the positions produced by `dst(idx)` for idx = 0, 1, ...
template <class Dst>
__device__ __forceinline__ void compact_from(uint16_t* ids, const uint32_t* bm,
                                             const int16_t* __restrict__ donor, int n, int lane,
                                             Dst&& dst) {
    int out = 0;
    for (int base = 0; base < n; base += 32) {
        const int k = base + lane;
        const int job = k < n ? (int)donor[k] : 0;
        const bool keep = k < n && !((bm[job >> 5] >> (job & 31)) & 1u);
        const uint32_t m = __ballot_sync(kFull, keep);
        if (keep) ids[dst(out + __popc(m & lanemask_lt(lane)))] = (uint16_t)job;
        out += __popc(m);
    }
    __syncwarp();
}

template <int E, bool UCD>
__device__ __forceinline__ void copy_in(uint16_t* ids, const int16_t* src, int lane) {
    constexpr int NP = Chain<E, UCD>::NP;
    for (int o = lane * 8; o < NP; o += 256)
        *reinterpret_cast<int4*>(ids + o) = *reinterpret_cast<const int4*>(src + o);
    __syncwarp();
}

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
                                       bool rearm) {
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
        if (threadIdx.x == 0) {
            if (rearm) a.gkey[cur] = ULLONG_MAX;
            *a.counter = 0u;
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

// Lines 6-7 of iteration t, then lines 4-5 of iteration t+1.
template <int E, bool UCD>
__global__ void __launch_bounds__(kDpThreads) dpso_iter_kernel(DpArgs a, int64_t t) {
    using C = Chain<E, UCD>;
    extern __shared__ __align__(16) uint8_t smem[];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    uint8_t* wbase = smem + (size_t)wib * DpSmem<E, UCD>::BYTES;
    const C ch{wbase};
    uint32_t* bm = reinterpret_cast<uint32_t*>(wbase + C::BYTES);
    int16_t* dpb = reinterpret_cast<int16_t*>(wbase + C::BYTES + 128);
    int16_t* dg = dpb + C::NP;
    uint16_t* ids = ch.id();
    const int n = a.n;
    const int cur = (int)(t & 1), nxt = cur ^ 1;
    if (a.trace && blockIdx.x == 0 && threadIdx.x == 0) a.trace[t] = (int64_t)(a.gkey[cur] >> 32);
    const int16_t* g = a.gperm + (size_t)cur * a.np;
    const int64_t total = (int64_t)gridDim.x * kDpWarps;
    unsigned long long wkey = ULLONG_MAX;
    for (int64_t i = (int64_t)blockIdx.x * kDpWarps + wib; i < a.particles; i += total) {
        const uint64_t gid = a.offset + (uint64_t)i;
        // the position and both donors (personal best, swarm best) to shared memory in one batch
        // of independent 16-byte loads, so the crossovers below never wait on global memory
        {
            constexpr int NP = C::NP;
            const int16_t* gp = a.pos + (size_t)i * a.np;
            const int16_t* gb = a.pb + (size_t)i * a.np;
            for (int o = lane * 8; o < NP; o += 256) {
                const int4 x = *reinterpret_cast<const int4*>(gp + o);
                const int4 y = *reinterpret_cast<const int4*>(gb + o);
                const int4 z = *reinterpret_cast<const int4*>(g + o);
                *reinterpret_cast<int4*>(ids + o) = x;
                *reinterpret_cast<int4*>(dpb + o) = y;
                *reinterpret_cast<int4*>(dg + o) = z;
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
                const uint16_t x = ids[pa];
                ids[pa] = ids[qb];
                ids[qb] = x;
            }
            __syncwarp();
        }
        // delta = c1 (+) F2(lambda, p^b): one-point crossover with the personal best
        if (__dmul_rn(__dadd_rn((double)a3, 0.5), u2) < a.c1) {
            const int c = 1 + (int)bnd(b0, (uint32_t)n - 1u);
            build_bitmap(bm, ids, 0, c - 1, lane);
            compact_from(ids, bm, dpb, n, lane, [c](int idx) { return c + idx; });
        }
        // p(t+1) = c2 (+) F3(delta, g): two-point crossover with the swarm best
        if (__dmul_rn(__dadd_rn((double)b1, 0.5), u2) < a.c2) {
            int q0 = (int)bnd(b2, (uint32_t)n - 1u);
            int q1 = (int)bnd(b3, (uint32_t)n);
            if (q1 == q0) q1 = n - 1;
            if (q0 > q1) {
                const int x = q0;
                q0 = q1;
                q1 = x;
            }
            build_bitmap(bm, ids, q0, q1, lane);
            const int span = q1 - q0 + 1;
            compact_from(ids, bm, dg, n, lane,
                         [q0, span](int idx) { return idx < q0 ? idx : idx + span; });
        }
        // line 7: evaluate
        chain_build<E, UCD>(ch, a.T, n, lane);
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
        __syncwarp();
    }
    // line 5 (iteration t+1): swarm best
    publish<E, UCD>(a, wkey, nxt, cur, true);
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
    size_t pos, pb, zb, gkey, gperm, counter, total;
};

DpWs dp_layout(int np, int64_t N) {
    DpWs w{};
    w.pos = 0;
    w.pb = align_up(w.pos + (size_t)N * np * 2);
    w.zb = align_up(w.pb + (size_t)N * np * 2);
    w.gkey = align_up(w.zb + (size_t)N * 4);
    w.gperm = align_up(w.gkey + 16);
    w.counter = align_up(w.gperm + (size_t)2 * np * 2);
    w.total = align_up(w.counter + 16);
    return w;
}

ChainTables dp_tables(const Instance& I, bool ucd) {
    return ucd ? ChainTables{I.tab_ab, I.tab_m, I.tab_x, I.tab_g}
               : ChainTables{I.tab_ab, I.tab_p, nullptr, nullptr};
}

template <int E>
DpArgs make_args(const Instance& I, const DpsoLaunch& p, void* ws) {
    constexpr int NP = 32 * E;
    const DpWs w = dp_layout(NP, p.particles);
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
    a.trace = p.gbest_trace;
    a.np = NP;
    return a;
}

template <class K>
int grid_for(const Instance& I, K kern, size_t smem, int64_t particles) {
    int sms = 148, occ = 1;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, I.device);
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kDpThreads, smem);
    if (occ < 1) occ = 1;
    int64_t need = (particles + kDpWarps - 1) / kDpWarps;
    const int64_t cap = (int64_t)sms * occ;
    if (need > cap) need = cap;
    return (int)(need < 1 ? 1 : need);
}

template <int E, bool UCD>
cudaError_t begin_e(Instance& I, const DpsoLaunch& p, void* ws, cudaStream_t s) {
    const DpArgs a = make_args<E>(I, p, ws);
    cudaError_t e = cudaMemsetAsync(a.gkey, 0xff, 2 * sizeof(unsigned long long), s);
    if (e == cudaSuccess) e = cudaMemsetAsync(a.counter, 0, sizeof(unsigned int), s);
    if (e != cudaSuccess) return e;
    const size_t smem = kDpWarps * (size_t)DpSmem<E, UCD>::BYTES;
    const int blocks = grid_for(I, dpso_init_kernel<E, UCD>, smem, p.particles);
    dpso_init_kernel<E, UCD><<<blocks, kDpThreads, smem, s>>>(a);
    return cudaGetLastError();
}

template <int E, bool UCD>
cudaError_t iter_e(Instance& I, const DpsoLaunch& p, void* ws, int64_t t, cudaStream_t s) {
    const DpArgs a = make_args<E>(I, p, ws);
    const size_t smem = kDpWarps * (size_t)DpSmem<E, UCD>::BYTES;
    const int blocks = grid_for(I, dpso_iter_kernel<E, UCD>, smem, p.particles);
    dpso_iter_kernel<E, UCD><<<blocks, kDpThreads, smem, s>>>(a, t);
    return cudaGetLastError();
}

template <int E>
cudaError_t begin_d(Instance& I, const DpsoLaunch& p, void* ws, cudaStream_t s) {
    return p.ucd ? begin_e<E, true>(I, p, ws, s) : begin_e<E, false>(I, p, ws, s);
}
template <int E>
cudaError_t iter_d(Instance& I, const DpsoLaunch& p, void* ws, int64_t t, cudaStream_t s) {
    return p.ucd ? iter_e<E, true>(I, p, ws, t, s) : iter_e<E, false>(I, p, ws, t, s);
}

}  // namespace

size_t dpso_workspace_bytes(const Instance& I, const DpsoLaunch& p) {
    return dp_layout(32 * sa_e_for_n(I.n), p.particles).total;
}

cudaError_t dpso_begin(Instance& I, const DpsoLaunch& p, void* ws, cudaStream_t s) {
    switch (sa_e_for_n(I.n)) {
        case 1: return begin_d<1>(I, p, ws, s);
        case 2: return begin_d<2>(I, p, ws, s);
        case 4: return begin_d<4>(I, p, ws, s);
        case 8: return begin_d<8>(I, p, ws, s);
        case 16: return begin_d<16>(I, p, ws, s);
        default: return begin_d<32>(I, p, ws, s);
    }
}

cudaError_t dpso_iterate(Instance& I, const DpsoLaunch& p, void* ws, int64_t t, cudaStream_t s) {
    switch (sa_e_for_n(I.n)) {
        case 1: return iter_d<1>(I, p, ws, t, s);
        case 2: return iter_d<2>(I, p, ws, t, s);
        case 4: return iter_d<4>(I, p, ws, t, s);
        case 8: return iter_d<8>(I, p, ws, t, s);
        case 16: return iter_d<16>(I, p, ws, t, s);
        default: return iter_d<32>(I, p, ws, t, s);
    }
}

void dpso_gbest(const Instance& I, const DpsoLaunch& p, void* ws, int64_t t, int64_t** key,
                int16_t** perm) {
    const int np = 32 * sa_e_for_n(I.n);
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
