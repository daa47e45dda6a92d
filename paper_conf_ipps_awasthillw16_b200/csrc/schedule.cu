// schedule.cu -- the optimal schedule of a sequence: what the O(n) timing
// routine finds, not just its cost.
//
// One warp per sequence, lane L owns positions [L*E, L*E+E) (E = pow2 >= ceil(n/32)); the ids
// are staged in shared memory by coalesced loads, the job data is read from tables staged per
// CTA, and the rows of C (and X) are assembled in shared memory and written out coalesced.  Same quantities as the evaluators:
//   S_k = sum_{j<k} (alpha_j + beta_j), k0 = max{k : S_k <= Btot}, C_k = sum_{j<=k} p_j;
//   CDD:    D = min(C_{k0}, d); the first job starts at s = d - D >= 0 (job k0 completes at d
//           when C_{k0} <= d, else the schedule starts at time 0), C_k <- s + C_k;
//   UCDDCP: (d >= sum P) job k0 completes at d; the weight of job k is w_k = A_{k-1} (k <= k0) or
//           B_k = sum_{j>=k} beta_j (k > k0); X_k = P_k - M_k iff w_k > gamma_k (strict),
//           p'_k = P_k - X_k, and C_k = d - (C'_{k0} - C'_k) with C' the prefix sums of p'.
// Outputs per sequence: C (int64 [n], sequence order), X (int32 [n], UCDDCP), the start time of
// the first job and the penalty of eq. (1) / (2) recomputed from that schedule.
#include <cuda_runtime.h>

#include <cstdint>

#include "device_common.cuh"
#include "internal.h"

namespace cdd {
namespace {

struct SchedArgs {
    const uint32_t* ab;  // alpha | beta << 16 by job id
    const uint8_t* p;    // P by job id
    const uint8_t* m;    // M by job id (UCDDCP)
    const uint8_t* x;    // P - M by job id (UCDDCP)
    const uint16_t* g;   // gamma by job id (UCDDCP)
    int n;
    int64_t d;
    const int16_t* perms;
    int64_t ld, batch;
    int64_t *C, *start, *pen;
    int32_t* X;
    int* err;
};

__device__ __forceinline__ int32_t warp_excl_scan(int32_t v, int lane) {
    int32_t s = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int32_t t = __shfl_up_sync(kFull, s, o);
        if (lane >= o) s += t;
    }
    return s - v;
}

__device__ __forceinline__ int64_t warp_sum64(int64_t v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
    return v;
}

// Shared-memory layout (dynamic): the instance tables by job id (ab u32, p u8 [, M | X << 8 |
// gamma << 16 u32], each array padded to 16 bytes), then per warp: the sequence's ids in lane segments
// of E positions (E = pow2 >= ceil(n/32), segments padded by 16 bytes), and the output staging
// C [and X] (int32) in lane segments padded by one element, so that the lane-contiguous compute
// writes and the coalesced copy-out reads are both (nearly) conflict free.  C is staged relative
// to a per-sequence int64 base (CDD: the start time; UCDDCP: d), |C - base| <= sum P < 2^31: half
// the shared memory of int64 staging, so more warps fit per SM.
struct SchedLayout {
    int n, E, lE;
    uint32_t tab_bytes, ids_off, c_off, x_off, warp_bytes, total;
};
__host__ __device__ inline uint32_t al16(uint32_t x) { return (x + 15u) & ~15u; }
__host__ __device__ inline SchedLayout sched_layout(int n, bool ucd, int warps) {
    SchedLayout L{};
    L.n = n;
    L.lE = 0;
    while ((32 << L.lE) < n) ++L.lE;
    L.E = 1 << L.lE;
    const uint32_t N = (uint32_t)n;
    L.tab_bytes = al16(4 * (N + 1)) + al16(N + 1) + (ucd ? al16(4 * (N + 1)) : 0u);
    L.ids_off = 0;
    L.c_off = al16(32u * (2u * L.E + 16u));
    L.x_off = L.c_off + al16(32u * 4u * (L.E + 1u));
    L.warp_bytes = L.x_off + (ucd ? al16(32u * 4u * (L.E + 1u)) : 0u);
    L.total = L.tab_bytes + (uint32_t)warps * L.warp_bytes;
    return L;
}
constexpr int kSchedWarps = 4;
#ifndef CDD_SCHED_MINB
#define CDD_SCHED_MINB 4
#endif

template <bool UCD, int E>
__global__ void __launch_bounds__(kSchedWarps * 32, UCD ? 3 : CDD_SCHED_MINB) schedule_kernel(SchedArgs a) {
    extern __shared__ __align__(16) uint8_t smem[];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const int n = a.n;
    const SchedLayout Ly = sched_layout(n, UCD, kSchedWarps);  // (its E equals the template's)
    constexpr int lE = E == 1 ? 0 : E == 2 ? 1 : E == 4 ? 2 : E == 8 ? 3 : E == 16 ? 4 : 5;
    const uint32_t N = (uint32_t)n;
    // CTA tables
    // (entry n is the zero record of the sentinel id that pads the lane segments past n: padded
    // slots add nothing to any sum, and where they pass the S <= Btot test -- only if every alpha
    // is 0 -- they repeat C_{n-1}, so no slot needs an index test)
    uint32_t* t_ab = reinterpret_cast<uint32_t*>(smem);
    uint8_t* t_p = smem + al16(4 * (N + 1));
    uint32_t* t_mxg = reinterpret_cast<uint32_t*>(t_p + al16(N + 1));  // UCDDCP: M | X << 8 | gamma << 16
    for (int j = threadIdx.x; j <= n; j += blockDim.x) {
        const bool v = j < n;
        t_ab[j] = v ? __ldg(a.ab + j) : 0u;
        t_p[j] = v ? __ldg(a.p + j) : (uint8_t)0;
        if constexpr (UCD)
            t_mxg[j] = v ? (uint32_t)__ldg(a.m + j) | ((uint32_t)__ldg(a.x + j) << 8) | ((uint32_t)__ldg(a.g + j) << 16)
                         : 0u;
    }
    uint8_t* wbase = smem + Ly.tab_bytes + (size_t)wib * Ly.warp_bytes;
    uint16_t* ids_s = reinterpret_cast<uint16_t*>(wbase + Ly.ids_off);
    int32_t* C_s = reinterpret_cast<int32_t*>(wbase + Ly.c_off);
    int32_t* X_s = reinterpret_cast<int32_t*>(wbase + Ly.x_off);
    const int IS = E + 8, CS = E + 1;  // segment strides (elements)
    const int k_lo = lane * E;
    // loops below run over all E slots of the lane's segment (unrolled); slots past n hold id n
    for (int k = n + lane; k < 32 * E; k += 32) ids_s[(k >> lE) * IS + (k & (E - 1))] = (uint16_t)n;
    __syncthreads();
    const uint16_t* myids = ids_s + lane * IS;
    int32_t* myC = C_s + lane * CS;
    int32_t* myX = X_s + lane * CS;
    const int64_t warps = (int64_t)gridDim.x * kSchedWarps;
    bool bad = false;
    uint32_t vmax = 0;                 // u16x2 maximum of the ids of whole vector chunks
    const uint32_t NN = N | (N << 16);
    // pairs of positions per store when rows of C (and X) are 16-byte aligned
    const bool pairs = E >= 2 && n % 2 == 0 && (reinterpret_cast<uintptr_t>(a.C) & 15u) == 0 &&
                       (!UCD || (reinterpret_cast<uintptr_t>(a.X) & 7u) == 0);
    // Vector path (16-byte aligned rows, ld % 8 == 0, E >= 8): a row's ids arrive as 16-byte
    // chunks of 8 (lane L takes chunks L, L + 32, ...) that are loaded one row AHEAD into registers,
    // so their latency hides behind the current row's compute; each chunk lands in one lane segment.
    constexpr int NPRE = E >= 8 ? E / 8 : 1;
    const bool vec = E >= 8 && a.ld % 8 == 0 && (reinterpret_cast<uintptr_t>(a.perms) & 15u) == 0;
    const int nch = (n + 7) / 8;
    int4 pre[NPRE];
    auto prefetch = [&](int64_t r) {
        if (r < a.batch) {
            const int4* src = reinterpret_cast<const int4*>(a.perms + r * a.ld);
#pragma unroll
            for (int t = 0; t < NPRE; ++t)
                if (lane + 32 * t < nch) pre[t] = __ldcs(src + lane + 32 * t);
        }
    };
    const int64_t row0 = (int64_t)blockIdx.x * kSchedWarps + wib;
    if (vec) prefetch(row0);
    for (int64_t row = row0; row < a.batch; row += warps) {
        const int16_t* rp = a.perms + row * a.ld;
        if (vec) {
#pragma unroll
            for (int t = 0; t < NPRE; ++t) {
                const int c = lane + 32 * t;
                if (c < nch) {
                    const uint32_t w[4] = {(uint32_t)pre[t].x, (uint32_t)pre[t].y, (uint32_t)pre[t].z,
                                           (uint32_t)pre[t].w};
                    uint32_t o[4];
                    if (8 * c + 8 <= n) {
                        // whole chunk inside the row: the maximum id (as u16: negative ids are
                        // >= 32768) raises the flag at the end; out-of-range ids read the sentinel's
                        // zero record (the row's results are unspecified, P:29-33 ids are 0..n-1)
                        vmax = __vimax3_u16x2(__vimax3_u16x2(vmax, w[0], w[1]), w[2], w[3]);
#pragma unroll
                        for (int h = 0; h < 4; ++h) o[h] = __vminu2(w[h], NN);
                    } else {
#pragma unroll
                        for (int h = 0; h < 4; ++h) {
                            uint32_t id2[2] = {w[h] & 0xffffu, w[h] >> 16};
#pragma unroll
                            for (int u = 0; u < 2; ++u) {
                                const int k = 8 * c + 2 * h + u;
                                if (k >= n) {
                                    id2[u] = N;  // the caller's padding: sentinel
                                } else if (id2[u] >= N) {  // an id outside [0, n) (incl. negative)
                                    bad = true;
                                    id2[u] = 0u;
                                }
                            }
                            o[h] = id2[0] | (id2[1] << 16);
                        }
                    }
                    const int k = 8 * c;
                    *reinterpret_cast<uint4*>(ids_s + (k >> lE) * IS + (k & (E - 1))) =
                        make_uint4(o[0], o[1], o[2], o[3]);
                }
            }
            __syncwarp();
            prefetch(row + warps);
        } else {
            // ids, coalesced, validated (an id outside [0, n) raises the flag and reads job 0)
            for (int k = lane; k < n; k += 32) {
                const int id = rp[k];
                const bool ok = id >= 0 && id < n;
                bad |= !ok;
                ids_s[(k >> lE) * IS + (k & (E - 1))] = (uint16_t)(ok ? id : 0);
            }
            __syncwarp();
        }
        // lane totals, then exclusive bases; the alpha|beta records stay in registers for the later
        // passes (the compiler cannot keep them across the shared-memory stores of C otherwise)
        constexpr int PQ = UCD ? 1 : (E + 3) / 4;
        uint32_t rr[E], pq[PQ];
        #pragma unroll
        for (int i = 0; i < PQ; ++i) pq[i] = 0u;
        int32_t tP = 0, tA = 0, tB = 0;
        #pragma unroll
        for (int i = 0; i < E; ++i) {
            const int j = myids[i];
            const uint32_t r = t_ab[j];
            rr[i] = r;
            if constexpr (!UCD) {
                const uint32_t pj = t_p[j];
                pq[i / 4] |= pj << (8 * (i % 4));
                tP += (int32_t)pj;
            }
            tA += (int32_t)(r & 0xffffu);
            tB += (int32_t)(r >> 16);
        }
        auto rec_r = [&](int i) { return rr[i]; };
        auto rec_p = [&](int i) {
            if constexpr (UCD) return 0;  // (C_{k0} is the CDD's; the UCDDCP uses the prefix of p')
            else return (int32_t)((pq[i / 4] >> (8 * (i % 4))) & 0xffu);
        };
        const int32_t Pb = warp_excl_scan(tP, lane), Ab = warp_excl_scan(tA, lane),
                      Bb = warp_excl_scan(tB, lane);
        const int32_t Btot = __shfl_sync(kFull, Bb + tB, 31);
        // k0 and C_{k0}: the last position with S_excl <= Btot (S is nondecreasing)
        int k0 = -1;
        int32_t Ck0 = 0;
        {
            int32_t c = Pb, s = Ab + Bb;
            #pragma unroll
        for (int i = 0; i < E; ++i) {
                const uint32_t r = rec_r(i);
                c += rec_p(i);
                if (s <= Btot) {
                    k0 = k_lo + i;
                    Ck0 = c;
                }
                s += (int32_t)(r & 0xffffu) + (int32_t)(r >> 16);
            }
        }
        const uint32_t has = __ballot_sync(kFull, k0 >= 0);
        const int owner = 31 - __clz(has);  // lane 0 always has k = 0 (S_0 = 0 <= Btot)
        k0 = __shfl_sync(kFull, k0, owner);
        Ck0 = __shfl_sync(kFull, Ck0, owner);
        int64_t pen = 0;
        int64_t st = 0;
        if constexpr (!UCD) {
            const int64_t D = min((int64_t)Ck0, a.d);
            st = a.d - D;  // start of the first job
            // C_k = st + c_k with c_k the prefix from time 0; D - c_k compares against the due date
            int32_t c = Pb;
            const int32_t Dl = (int32_t)D;  // D <= C_{k0} <= sum P
            #pragma unroll
        for (int i = 0; i < E; ++i) {
                const uint32_t r = rec_r(i);
                c += rec_p(i);
                myC[i] = c;
                pen += (int64_t)(r & 0xffffu) * max(0, Dl - c) + (int64_t)(r >> 16) * max(0, c - Dl);
            }
        } else {
            // compression decisions (Property 2: X_k = P_k - M_k iff the weight of position k
            // exceeds gamma_k), p' = P - X_k staged next to X, the lane totals of p', the prefix
            // of p' through k0 on its lane, and the gamma part of the penalty
            int32_t tQ = 0, qk = 0, pg = 0;  // pg <= E * 255 * 65535 < 2^31
            {
                int32_t A = Ab, B = Bb;  // exclusive prefixes
                #pragma unroll
                for (int i = 0; i < E; ++i) {
                    const uint32_t r = rr[i];
                    const uint32_t mxg = t_mxg[myids[i]];
                    const int32_t g = (int32_t)(mxg >> 16), xj = (int32_t)((mxg >> 8) & 0xffu);
                    const bool early = k_lo + i <= k0;
                    const int32_t w = early ? A : Btot - B;
                    const int32_t xk = w > g ? xj : 0;
                    const int32_t q = (int32_t)(mxg & 0xffu) + xj - xk;
                    reinterpret_cast<uint32_t*>(myX)[i] = (uint32_t)xk | ((uint32_t)q << 16);
                    tQ += q;
                    qk += early ? q : 0;
                    pg += g * xk;
                    A += (int32_t)(r & 0xffffu);
                    B += (int32_t)(r >> 16);
                }
            }
            const int32_t Qb = warp_excl_scan(tQ, lane);
            // C'_{k0}: inclusive prefix of p' at k0 (on the lane holding k0)
            const int32_t Qk0 = __shfl_sync(kFull, Qb + qk, owner);
            st = a.d - Qk0;
            int32_t q = Qb;
            #pragma unroll
            for (int i = 0; i < E; ++i) {
                const uint32_t r = rr[i];
                q += (int32_t)(reinterpret_cast<const uint32_t*>(myX)[i] >> 16);
                const int32_t c = q - Qk0;  // C_k - d
                myC[i] = c;
                pen += (int64_t)(r & 0xffffu) * max(0, -c) + (int64_t)(r >> 16) * max(0, c);
            }
            pen += pg;
        }
        pen = warp_sum64(pen);
        if (lane == 0) {
            a.start[row] = st;
            a.pen[row] = pen;
        }
        __syncwarp();
        // coalesced copy-out of the staged rows (the int64 base added here)
        int64_t* Crow = a.C + row * (int64_t)n;
        const int64_t cb = UCD ? a.d : st;
        if (pairs) {  // 16-byte streaming stores of position pairs (same lane segment: E even)
            if constexpr (E <= 64) {
                // 64 positions per step = 64/E whole segments: the staged index advances by a constant
                int idx = ((2 * lane) >> lE) * CS + ((2 * lane) & (E - 1));
                longlong2* dst = reinterpret_cast<longlong2*>(Crow) + lane;
                for (int k = 2 * lane; k < n; k += 64, idx += (64 / E) * CS, dst += 32)
                    __stcs(dst, make_longlong2(cb + C_s[idx], cb + C_s[idx + 1]));
            } else {
                for (int k = 2 * lane; k < n; k += 64) {
                    const int idx = (k >> lE) * CS + (k & (E - 1));
                    __stcs(reinterpret_cast<longlong2*>(Crow + k), make_longlong2(cb + C_s[idx], cb + C_s[idx + 1]));
                }
            }
        } else {
            for (int k = lane; k < n; k += 32) Crow[k] = cb + C_s[(k >> lE) * CS + (k & (E - 1))];
        }
        if constexpr (UCD) {
            int32_t* Xrow = a.X + row * (int64_t)n;
            if (pairs) {
                for (int k = 2 * lane; k < n; k += 64) {
                    const int idx = (k >> lE) * CS + (k & (E - 1));
                    __stcs(reinterpret_cast<int2*>(Xrow + k), make_int2(X_s[idx] & 0xffff, X_s[idx + 1] & 0xffff));
                }
            } else {
                for (int k = lane; k < n; k += 32) Xrow[k] = X_s[(k >> lE) * CS + (k & (E - 1))] & 0xffff;
            }
        }
        __syncwarp();
    }
    if (bad || (vmax & 0xffffu) >= N || (vmax >> 16) >= N) atomicOr(a.err, 1);
}

}  // namespace

cudaError_t launch_schedule(const Instance& I, bool ucd, const int16_t* perms, int64_t ld,
                            int64_t batch, int64_t* C, int32_t* X, int64_t* start, int64_t* pen,
                            cudaStream_t s) {
    if (batch == 0) return cudaSuccess;
    SchedArgs a{I.tab_ab, I.tab_p, I.tab_m, I.tab_x, I.tab_g, I.n, I.d, perms, ld, batch,
                C, start, pen, X, I.err};
    const SchedLayout Ly = sched_layout(I.n, ucd, kSchedWarps);
    void (*kern)(SchedArgs) = nullptr;
    switch (Ly.E) {
        case 1: kern = ucd ? schedule_kernel<true, 1> : schedule_kernel<false, 1>; break;
        case 2: kern = ucd ? schedule_kernel<true, 2> : schedule_kernel<false, 2>; break;
        case 4: kern = ucd ? schedule_kernel<true, 4> : schedule_kernel<false, 4>; break;
        case 8: kern = ucd ? schedule_kernel<true, 8> : schedule_kernel<false, 8>; break;
        case 16: kern = ucd ? schedule_kernel<true, 16> : schedule_kernel<false, 16>; break;
        default: kern = ucd ? schedule_kernel<true, 32> : schedule_kernel<false, 32>; break;
    }
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Ly.total);
    if (e != cudaSuccess) return e;
    int sms = 148, occ = 1;
    e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, I.device);
    if (e != cudaSuccess) return e;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kSchedWarps * 32, Ly.total);
    if (e != cudaSuccess) return e;
    const int64_t want = (batch + kSchedWarps - 1) / kSchedWarps;
    const int64_t cap = (int64_t)sms * (occ < 1 ? 1 : occ);
    const int blocks = (int)(want < cap ? want : cap);
    kern<<<blocks, kSchedWarps * 32, Ly.total, s>>>(a);
    return cudaGetLastError();
}

}  // namespace cdd
