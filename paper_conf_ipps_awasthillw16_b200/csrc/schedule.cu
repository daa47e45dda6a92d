// schedule.cu -- the optimal schedule of a sequence: what the O(n) timing
// routine finds, not just its cost.
//
// One warp per sequence, lane L owns positions [L*E, L*E+E) (E = ceil(n/32)); the job data is read
// through the id tables (global, L1-resident).  Same quantities as the evaluators:
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

template <bool UCD>
__global__ void __launch_bounds__(128) schedule_kernel(SchedArgs a) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
    const int n = a.n, E = (n + 31) / 32, k_lo = lane * E, k_hi = min(n, k_lo + E);
    bool bad = false;
    for (int64_t row = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); row < a.batch;
         row += warps) {
        const int16_t* rp = a.perms + row * a.ld;
        auto job = [&](int k) -> int {
            const int id = rp[k];
            const bool ok = id >= 0 && id < n;
            bad |= !ok;
            return ok ? id : 0;
        };
        // lane totals, then exclusive bases
        int32_t tP = 0, tA = 0, tB = 0;
        for (int k = k_lo; k < k_hi; ++k) {
            const int j = job(k);
            const uint32_t r = __ldg(a.ab + j);
            tP += __ldg(a.p + j);
            tA += (int32_t)(r & 0xffffu);
            tB += (int32_t)(r >> 16);
        }
        const int32_t Pb = warp_excl_scan(tP, lane), Ab = warp_excl_scan(tA, lane),
                      Bb = warp_excl_scan(tB, lane);
        const int32_t Btot = __shfl_sync(kFull, Bb + tB, 31);
        // k0 and C_{k0}: the last position with S_excl <= Btot (S is nondecreasing)
        int k0 = -1;
        int32_t Ck0 = 0;
        {
            int32_t c = Pb, s = Ab + Bb;
            for (int k = k_lo; k < k_hi; ++k) {
                const int j = job(k);
                const uint32_t r = __ldg(a.ab + j);
                c += __ldg(a.p + j);
                if (s <= Btot) {
                    k0 = k;
                    Ck0 = c;
                }
                s += (int32_t)(r & 0xffffu) + (int32_t)(r >> 16);
            }
        }
        const uint32_t has = __ballot_sync(kFull, k0 >= 0);
        const int owner = 31 - __clz(has);  // lane 0 always has k = 0 (S_0 = 0 <= Btot)
        k0 = __shfl_sync(kFull, k0, owner);
        Ck0 = __shfl_sync(kFull, Ck0, owner);
        int64_t* Crow = a.C + row * (int64_t)n;
        int64_t pen = 0;
        if constexpr (!UCD) {
            const int64_t D = min((int64_t)Ck0, a.d);
            const int64_t s0 = a.d - D;  // start of the first job
            int64_t c = s0 + Pb;
            for (int k = k_lo; k < k_hi; ++k) {
                const int j = job(k);
                const uint32_t r = __ldg(a.ab + j);
                c += __ldg(a.p + j);
                Crow[k] = c;
                pen += (int64_t)(r & 0xffffu) * max((int64_t)0, a.d - c) +
                       (int64_t)(r >> 16) * max((int64_t)0, c - a.d);
            }
            pen = warp_sum64(pen);
            if (lane == 0) {
                a.start[row] = s0;
                a.pen[row] = pen;
            }
        } else {
            int32_t* Xrow = a.X + row * (int64_t)n;
            // compression decisions and the lane totals of p'
            int32_t tQ = 0;
            {
                int32_t A = Ab, B = Bb;  // exclusive prefixes
                for (int k = k_lo; k < k_hi; ++k) {
                    const int j = job(k);
                    const uint32_t r = __ldg(a.ab + j);
                    const int32_t w = k <= k0 ? A : Btot - B;
                    const int32_t xk = w > (int32_t)__ldg(a.g + j) ? (int32_t)__ldg(a.x + j) : 0;
                    Xrow[k] = xk;
                    tQ += (int32_t)__ldg(a.m + j) + (int32_t)__ldg(a.x + j) - xk;
                    A += (int32_t)(r & 0xffffu);
                    B += (int32_t)(r >> 16);
                }
            }
            const int32_t Qb = warp_excl_scan(tQ, lane);
            // C'_{k0}: inclusive prefix of p' at k0
            int32_t Qk0 = 0;
            {
                int32_t q = Qb;
                for (int k = k_lo; k < k_hi; ++k) {
                    const int j = job(k);
                    q += (int32_t)__ldg(a.m + j) + (int32_t)__ldg(a.x + j) - Xrow[k];
                    if (k == k0) Qk0 = q;
                }
            }
            Qk0 = __shfl_sync(kFull, Qk0, owner);
            int32_t q = Qb;
            for (int k = k_lo; k < k_hi; ++k) {
                const int j = job(k);
                const uint32_t r = __ldg(a.ab + j);
                const int32_t xk = Xrow[k];
                q += (int32_t)__ldg(a.m + j) + (int32_t)__ldg(a.x + j) - xk;
                const int64_t c = a.d - (int64_t)(Qk0 - q);
                Crow[k] = c;
                pen += (int64_t)(r & 0xffffu) * max((int64_t)0, a.d - c) +
                       (int64_t)(r >> 16) * max((int64_t)0, c - a.d) +
                       (int64_t)__ldg(a.g + j) * xk;
            }
            pen = warp_sum64(pen);
            if (lane == 0) {
                a.start[row] = a.d - Qk0;
                a.pen[row] = pen;
            }
        }
    }
    if (bad) atomicOr(a.err, 1);
}

}  // namespace

cudaError_t launch_schedule(const Instance& I, bool ucd, const int16_t* perms, int64_t ld,
                            int64_t batch, int64_t* C, int32_t* X, int64_t* start, int64_t* pen,
                            cudaStream_t s) {
    if (batch == 0) return cudaSuccess;
    SchedArgs a{I.tab_ab, I.tab_p, I.tab_m, I.tab_x, I.tab_g, I.n, I.d, perms, ld, batch,
                C, start, pen, X, I.err};
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, I.device);
    const int64_t want = (batch + 3) / 4;
    const int blocks = (int)(want < (int64_t)sms * 16 ? want : (int64_t)sms * 16);
    if (ucd) schedule_kernel<true><<<blocks, 128, 0, s>>>(a);
    else schedule_kernel<false><<<blocks, 128, 0, s>>>(a);
    return cudaGetLastError();
}

}  // namespace cdd
