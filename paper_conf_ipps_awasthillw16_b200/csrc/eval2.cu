// eval2.cu -- batched CDD evaluation, several sequences per warp (cdd_eval_batch, S§8 A2-A7).
//
// G lanes evaluate one sequence (32/G sequences per warp), lane l owns the E contiguous positions
// [l*E, l*E+E).  Per warp, the job ids of the next group of sequences are copied from HBM to a
// double-buffered shared-memory stage with cp.async (16-byte chunks, fully coalesced, no register
// staging; chunk c of lane segment S lands in slot c ^ f(S) so that the lane-contiguous LDS.128
// reads of a segment are bank-conflict free) while the current group is evaluated.  (A TMA bulk
// copy per lane segment was measured slower: the copy takes uniform operands, so 32 per-lane
// copies serialise into an ELECT/R2UR loop.)  The records are gathered from a
// bank-partitioned table (8 copies, aligned to its size so a gather address is SHF + LOP3) into
// registers as 16-bit alpha|beta<<8 pairs and p bytes, and the evaluation is the group kernel's
// (sa_group.cuh): two scans, ballots, a boundary-row spread (re-gathered through the staged ids)
// and the PRMT/IMAD/IDP.2A/IDP.4A pass -- 2 instructions per position.
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>

#include "device_common.cuh"
#include "internal.h"

namespace cdd {
namespace {

// Table copies KC: lane L reads copy L % KC; 16 copies (2-way-at-worst bank conflicts between
// lanes L and L+16) when shared memory allows, else 8 (4 lanes per copy, ~2.9 wavefronts/gather).
constexpr int kE2MaxSmem = 227 * 1024;

// Shared-memory layout: the table (KC copies x npow2 words) must sit at an address aligned to its
// size (a gather address is then SHF + LOP3); the per-warp stages fill the gap below it first
// (the dynamic window starts above a reserved 1 KB), the rest go above it.
struct E2Layout {
    uint32_t tab_off, nb, total;  // offsets from the dynamic base; nb = warps placed below
};
__host__ __device__ inline E2Layout e2_layout(uint32_t sbase, uint32_t tbytes, uint32_t wbytes, int W) {
    const uint32_t tab = (sbase + tbytes - 1u) / tbytes * tbytes;
    uint32_t nb = (tab - sbase) / wbytes;
    if (nb > (uint32_t)W) nb = (uint32_t)W;
    return {tab - sbase, nb, tab + tbytes + ((uint32_t)W - nb) * wbytes - sbase};
}

__device__ __forceinline__ uint32_t lds32(uint32_t addr) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr));
    return v;
}

// Table gather: with TOFF != 0 the table sits at the start of the dynamic window (shared address
// TOFF, the probed base) and the base rides in the load's immediate offset, so the table need not
// be aligned to its size (room for 32 conflict-free copies at n = 1000).
template <uint32_t TOFF>
__device__ __forceinline__ uint32_t ldtab(uint32_t addr) {
    uint32_t v;
    if constexpr (TOFF == 0)
        asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr));
    else
        asm volatile("ld.shared.u32 %0, [%1+%2];" : "=r"(v) : "r"(addr), "n"(TOFF));
    return v;
}

template <uint32_t TOFF>
__device__ __forceinline__ uint2 ldtab64(uint32_t addr) {
    uint2 v;
    if constexpr (TOFF == 0)
        asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(addr));
    else
        asm volatile("ld.shared.v2.u32 {%0,%1}, [%2+%3];" : "=r"(v.x), "=r"(v.y) : "r"(addr), "n"(TOFF));
    return v;
}

__device__ __forceinline__ uint4 lds128(uint32_t addr) {
    uint4 v;
    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr));
    return v;
}

__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait1() { asm volatile("cp.async.wait_group 1;" ::: "memory"); }

template <int G>
__device__ __forceinline__ uint32_t gsum2(uint32_t v) {
#pragma unroll
    for (int off = G / 2; off > 0; off >>= 1) v += __shfl_xor_sync(kFull, v, off, G);
    return v;
}

template <int G, int E>
struct E2 {
    static constexpr int CPW = 32 / G;        // sequences per warp
    static constexpr int CPS = E / 8;         // 16-byte chunks per lane segment
    static constexpr int ROWB = G * E * 2;    // staged bytes per sequence
    static constexpr int STAGE = CPW * ROWB;
    static constexpr int SPR = E / G;         // boundary-row positions per lane
    static constexpr int T = (G * CPS + 31) / 32;  // chunks of one sequence per lane (at most)
    // swizzle of lane segment S (numbered over the warp's sequences)
    static __device__ __forceinline__ uint32_t sw(int S) { return (uint32_t)((S * CPS / 8) % CPS); }
};

// Job ids of positions e0 .. e0+SPR-1 of the staged lane segment at bseg (swizzle bsw), as
// 16-bit pairs.
template <int G, int E, int SPR>
__device__ __forceinline__ void e2_row_ids(uint32_t bseg, uint32_t bsw, int e0, uint32_t (&idw)[(SPR + 1) / 2]) {
    if constexpr (SPR >= 8) {
#pragma unroll
        for (int v = 0; v < SPR / 8; ++v) {
            const uint4 q = lds128(bseg + ((((uint32_t)(e0 / 8 + v)) ^ bsw) << 4));
            idw[4 * v] = q.x; idw[4 * v + 1] = q.y; idw[4 * v + 2] = q.z; idw[4 * v + 3] = q.w;
        }
    } else {
        const uint32_t a = bseg + ((((uint32_t)(e0 / 8)) ^ bsw) << 4) + (uint32_t)((e0 % 8) * 2);
        if constexpr (SPR == 4) {
            uint32_t x0, x1;
            asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(x0), "=r"(x1) : "r"(a));
            idw[0] = x0; idw[1] = x1;
        } else if constexpr (SPR == 2) {
            idw[0] = lds32(a);
        } else {
            uint32_t x;
            asm volatile("ld.shared.u16 %0, [%1];" : "=r"(x) : "r"(a));
            idw[0] = x;
        }
    }
}

// One group of 32/G sequences per warp and stage.
template <int G, int E, int W, uint32_t TOFF, bool TAIL, bool UCD>
__global__ void __launch_bounds__(W * 32, 1) eval2_kernel(
    const uint16_t* __restrict__ tab_ab16, const uint8_t* __restrict__ tab_p,
    const uint8_t* __restrict__ tab_m, const uint8_t* __restrict__ tab_x,
    const uint16_t* __restrict__ tab_g, int n, int npow2,
    int kc_log2, int32_t d, const int16_t* __restrict__ perms, int64_t ld, int64_t batch,
    int64_t* __restrict__ out, int* __restrict__ err, bool quad) {
    using X = E2<G, E>;
    constexpr int CPW = X::CPW, CPS = X::CPS, SPR = X::SPR;
    extern __shared__ __align__(16) uint8_t smem[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int grp = lane / G, l = lane % G, gbase = grp * G;
    const int KC = 1 << kc_log2;
    const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(smem);
    constexpr uint32_t RB = UCD ? 8u : 4u;  // bytes per table entry
    const uint32_t tbytes = (uint32_t)npow2 * RB * (uint32_t)KC;
    const E2Layout Ly = TOFF ? E2Layout{0u, 0u, tbytes + (uint32_t)W * 2u * X::STAGE}
                             : e2_layout(sbase, tbytes, 2u * X::STAGE, W);
    const uint32_t tab = TOFF ? 0u : sbase + Ly.tab_off;
    const uint32_t stage0 = sbase + ((uint32_t)warp < Ly.nb ? (uint32_t)warp * 2u * X::STAGE
                                                              : Ly.tab_off + tbytes + ((uint32_t)warp - Ly.nb) * 2u * X::STAGE);
    if constexpr (UCD) {
        // alpha | beta << 8 | gamma << 16,  M | X << 8
        uint2* s_tab = reinterpret_cast<uint2*>(smem + Ly.tab_off);
        for (int i = threadIdx.x; i < npow2 * KC; i += blockDim.x) {
            const int id = i >> kc_log2;
            s_tab[i] = id < n ? make_uint2((uint32_t)__ldg(tab_ab16 + id) | ((uint32_t)__ldg(tab_g + id) << 16),
                                           (uint32_t)__ldg(tab_m + id) | ((uint32_t)__ldg(tab_x + id) << 8))
                              : make_uint2(0u, 0u);
        }
    } else {
        uint32_t* s_tab = reinterpret_cast<uint32_t*>(smem + Ly.tab_off);
        for (int i = threadIdx.x; i < npow2 * KC; i += blockDim.x) {
            const int id = i >> kc_log2;
            s_tab[i] = id < n ? (uint32_t)__ldg(tab_ab16 + id) | ((uint32_t)__ldg(tab_p + id) << 16) : 0u;
        }
    }
    __syncthreads();
    const int SH = (UCD ? 3 : 2) + kc_log2;  // log2(RB bytes * KC copies)
    const uint32_t amask = tbytes - RB * (uint32_t)KC;
    const uint32_t tabc = tab | (uint32_t)(lane & (KC - 1)) * RB;

    const int cpr = (n + 7) / 8;  // 16-byte chunks of real ids per sequence (ld % 8 == 0)
    const uint32_t S = (uint32_t)npow2 - 1u;  // sentinel id: >= n, zero record
    const int64_t ngroups = (batch + CPW - 1) / CPW;
    const int64_t gstep = (int64_t)gridDim.x * W;
    // this lane copies chunks cg = lane + 32 t of every sequence of a group (its stage slot
    // depends on the group only through nothing: the offsets are loop invariants)
    // When the swizzle of a segment does not depend on the row within the group (G % 8 == 0), the
    // stage offsets of this lane's chunks and their "before n" predicates are loop invariants.
    constexpr bool kRowFree = G % 8 == 0;
    uint32_t soff[X::T];
    uint32_t pmask = 0;
#pragma unroll
    for (int t = 0; t < X::T; ++t) {
        const int cg = lane + 32 * t, seg = cg / CPS, c = cg % CPS;
        soff[t] = 16u * ((uint32_t)(seg * CPS) + ((uint32_t)c ^ X::sw(seg)));
        if (cg < cpr) pmask |= 1u << t;
    }
    auto issue = [&](int64_t rg, int st) {
        const uint32_t sdst = stage0 + (uint32_t)(st * X::STAGE);
#pragma unroll
        for (int r = 0; r < CPW; ++r) {
            const int64_t row = rg * CPW + r;
            if (rg < ngroups && row < batch) {  // warp-uniform
                const char* src = reinterpret_cast<const char*>(perms + row * ld) + lane * 16;
                if constexpr (X::T > 1)  // one 64-bit address per row, not re-formed under each predicate
                    asm("" : "+l"(src));
#pragma unroll
                for (int t = 0; t < X::T; ++t) {
                    if constexpr (kRowFree) {
                        if ((pmask >> t) & 1u) cp_async16(sdst + (uint32_t)(r * X::ROWB) + soff[t], src + 512 * t);
                    } else {
                        const int cg = lane + 32 * t, seg = cg / CPS, c = cg % CPS;
                        const uint32_t slot = (uint32_t)(seg * CPS) + ((uint32_t)c ^ X::sw(r * G + seg));
                        if (cg < cpr) cp_async16(sdst + (uint32_t)(r * X::ROWB) + 16u * slot, src + 512 * t);
                    }
                }
            }
        }
        cp_async_commit();
    };

    // Slots past the sequence's last real chunk are never copied: fill them once with the sentinel
    // id S = npow2 - 1 (>= n, a zero record); ids there are excluded from the validity check.
    {
        const uint4 s4 = make_uint4(S * 0x10001u, S * 0x10001u, S * 0x10001u, S * 0x10001u);
        for (int st = 0; st < 2; ++st)
#pragma unroll
            for (int r = 0; r < CPW; ++r)
                for (int cg = cpr + lane; cg < G * CPS; cg += 32) {
                    const int seg = cg / CPS, c = cg % CPS;
                    const uint32_t slot = (uint32_t)(seg * CPS) + ((uint32_t)c ^ X::sw(r * G + seg));
                    const uint32_t a = stage0 + (uint32_t)(st * X::STAGE + r * X::ROWB) + 16u * slot;
                    asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(a), "r"(s4.x), "r"(s4.y),
                                 "r"(s4.z), "r"(s4.w) : "memory");
                }
        __syncwarp();
    }
    const int64_t rg0 = (int64_t)blockIdx.x * W + warp;
    issue(rg0, 0);
    issue(rg0 + gstep, 1);
    uint32_t vmax = 0;
    bool bad = false;
    const uint32_t sw_own = X::sw(grp * G + l);
    const int kown = min(E, max(0, n - l * E));  // positions of own segment before n
    const int nfull_lane = kown / 8;
    const int cstr = (kown % 8) ? kown / 8 : -1;  // chunk straddling n (n % 8 != 0 only)
    const int kstr = kown % 8;  // real ids in that chunk
    int it = 0;
    for (int64_t rg = rg0; rg < ngroups; rg += gstep, ++it) {
        const int st = it & 1;
        cp_async_wait1();
        __syncwarp();
        const uint32_t srow = stage0 + (uint32_t)(st * X::STAGE) + (uint32_t)(grp * X::ROWB);
        const int64_t row = rg * CPW + grp;
        const bool rv = row < batch;
        const uint32_t seg_addr = srow + (uint32_t)(l * CPS * 16);
        const int nfull = rv ? nfull_lane : 0;  // chunks of own segment wholly before n
        if constexpr (TAIL) {
            // n % 8 != 0: the lane owning the chunk that straddles n checks its real ids and
            // overwrites the rest (the caller's padding) with the sentinel, in place
            if (cstr >= 0) {
                const uint32_t a = seg_addr + (((uint32_t)cstr ^ sw_own) << 4);
                const uint4 q = lds128(a);
                uint32_t ws[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    uint32_t lo = ws[j] & 0xffffu, hi = ws[j] >> 16;
                    if (2 * j < kstr) bad |= rv && lo >= (uint32_t)n; else lo = S;
                    if (2 * j + 1 < kstr) bad |= rv && hi >= (uint32_t)n; else hi = S;
                    ws[j] = lo | (hi << 16);
                }
                asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(a), "r"(ws[0]), "r"(ws[1]),
                             "r"(ws[2]), "r"(ws[3]) : "memory");
            }
            __syncwarp();
        }
        if constexpr (UCD) {
            // ---- gather: 16-bit alpha|beta<<8 pairs, gamma pairs, M and X bytes, lane totals
            uint32_t abp[E / 2], gp[E / 2], mx[E / 2];
            uint32_t tA = 0, tB = 0;
#pragma unroll
            for (int c = 0; c < CPS; ++c) {
                uint4 q = lds128(seg_addr + (((uint32_t)c ^ sw_own) << 4));
                if (c < nfull) vmax = __vimax3_u16x2(__vimax3_u16x2(vmax, q.x, q.y), q.z, q.w);
                const uint32_t wv[4] = {q.x, q.y, q.z, q.w};
                uint2 r[8];
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    r[2 * j] = ldtab64<TOFF>(((wv[j] << SH) & amask) | tabc);
                    r[2 * j + 1] = ldtab64<TOFF>(((wv[j] >> (16 - SH)) & amask) | tabc);
                }
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const uint32_t a = __byte_perm(r[2 * j].x, r[2 * j + 1].x, 0x5410u);
                    abp[4 * c + j] = a;
                    gp[4 * c + j] = __byte_perm(r[2 * j].x, r[2 * j + 1].x, 0x7632u);
                    tA = __dp4a(a, 0x00010001u, tA);
                    tB = __dp4a(a, 0x01000100u, tB);
                }
#pragma unroll
                for (int j = 0; j < 4; ++j)  // (M_{2j}, M_{2j+1}, X_{2j}, X_{2j+1}): the pass's two IDP.2A
                    mx[4 * c + j] = __byte_perm(r[2 * j].y, r[2 * j + 1].y, 0x5140u);
            }
            // ---- scan, boundary lane Lk (d >= sum P: the due date sits at C_{k0}; as gchain_eval_ucddcp)
            const uint32_t tAB = tA | (tB << 16);
            const uint32_t iAB = group_incl_scan<G>(tAB, 0);
            const uint32_t ABb = iAB - tAB;
            const int32_t Ab = (int32_t)(ABb & 0xffffu), Bb = (int32_t)(ABb >> 16);
            const int32_t Btot = (int32_t)(__shfl_sync(kFull, iAB, G - 1, G) >> 16);
            const bool lane_valid = l * E < n;
            const int Lk = max(0, hibit(group_ballot<G>(lane_valid && (Ab + Bb <= Btot), gbase)));
            const uint32_t ABbS = __shfl_sync(kFull, ABb, Lk, G);
            const int e0 = l * SPR;
            uint32_t idw[(SPR + 1) / 2];
            e2_row_ids<G, E, SPR>(srow + (uint32_t)(Lk * CPS * 16), X::sw(grp * G + Lk), e0, idw);
            const int kb = Lk * E + e0;
            uint32_t rvw[SPR], mv[SPR], xv[SPR], gv[SPR];
            uint32_t lsum = 0;
#pragma unroll
            for (int i = 0; i < SPR; ++i) {
                const uint32_t id = (i & 1) ? (idw[i >> 1] >> 16) : (idw[i >> 1] & 0xffffu);
                const uint2 rec = (rv && kb + i < n) ? ldtab64<TOFF>(((id << SH) & amask) | tabc) : make_uint2(0u, 0u);
                rvw[i] = __byte_perm(rec.x, 0u, 0x4140u);  // alpha | beta << 16
                gv[i] = rec.x >> 16;
                mv[i] = rec.y & 0xffu;
                xv[i] = (rec.y >> 8) & 0xffu;
                lsum += rvw[i];
            }
            uint32_t ex = group_incl_scan<G>(lsum, 0) - lsum;
            // elements of row Lk at or before k0 (A_excl + B_excl <= Btot, a prefix of the row)
            // switch from the tardy weight to the early weight
            int32_t corr = 0;
#pragma unroll
            for (int i = 0; i < SPR; ++i) {
                const int32_t wA = (int32_t)(ABbS & 0xffffu) + (int32_t)(ex & 0xffffu);
                const int32_t Bex = (int32_t)(ABbS >> 16) + (int32_t)(ex >> 16);
                const int32_t wB = Btot - Bex;
                const int32_t g = (int32_t)gv[i];
                const int32_t cc = (int32_t)mv[i] * (wA - wB) + (int32_t)xv[i] * (min(wA, g) - min(wB, g));
                corr += (wA + Bex <= Btot) ? cc : 0;
                ex += rvw[i];
            }
            __syncwarp();  // every lane is done with the stage: refill it two groups ahead
            issue(rg + 2 * gstep, st);
            // ---- pass: pairs of weights in 16-bit halves, w2 = base2 +- f2 (Property 2: X_j
            // compressed iff its weight exceeds gamma_j, so the X part costs min(w, gamma))
            const bool amode = l < Lk;
            const uint32_t wbase = (uint32_t)(amode ? Ab : (Btot - Bb));
            const uint32_t base2 = wbase | (wbase << 16);
            const uint32_t sgn = amode ? 1u : 0xffffffffu;
            const uint32_t psel = amode ? 0x4044u : 0x4144u;
            const uint32_t wsum = amode ? 0x00010001u : 0x01000100u;
            uint32_t s = 0, acc = 0;
#pragma unroll
            for (int j = 0; j < E / 2; ++j) {
                const uint32_t f2 = s * 0x10001u + __byte_perm(abp[j], 0u, psel);
                const uint32_t w2 = f2 * sgn + base2;
                const uint32_t mn2 = __vminu2(w2, gp[j]);
                acc = __dp2a_lo(w2, mx[j], acc);
                acc = __dp2a_hi(mn2, mx[j], acc);
                s = __dp4a(abp[j], wsum, s);
            }
            const int32_t Z = (int32_t)gsum2<G>(acc + (uint32_t)corr);
            if (rv && l == 0) out[row] = (int64_t)Z;
        } else {
            // ---- gather: 16-bit alpha|beta<<8 pairs and p bytes, lane totals
            uint32_t abp[E / 2], pw[E / 4];
            uint32_t tA = 0, tB = 0, tP = 0;
#pragma unroll
            for (int c = 0; c < CPS; ++c) {
                uint4 q = lds128(seg_addr + (((uint32_t)c ^ sw_own) << 4));
                // chunks wholly past n hold the sentinel (written once, never copied over)
                if (c < nfull) vmax = __vimax3_u16x2(__vimax3_u16x2(vmax, q.x, q.y), q.z, q.w);
                const uint32_t wv[4] = {q.x, q.y, q.z, q.w};
                uint32_t r[8];
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    r[2 * j] = ldtab<TOFF>(((wv[j] << SH) & amask) | tabc);
                    r[2 * j + 1] = ldtab<TOFF>(((wv[j] >> (16 - SH)) & amask) | tabc);
                }
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const uint32_t a = __byte_perm(r[2 * j], r[2 * j + 1], 0x5410u);
                    abp[4 * c + j] = a;
                    tA = __dp4a(a, 0x00010001u, tA);
                    tB = __dp4a(a, 0x01000100u, tB);
                }
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    const uint32_t p01 = __byte_perm(r[4 * h], r[4 * h + 1], 0x0062u);
                    const uint32_t p23 = __byte_perm(r[4 * h + 2], r[4 * h + 3], 0x0062u);
                    const uint32_t p4 = __byte_perm(p01, p23, 0x5410u);
                    pw[2 * c + h] = p4;
                    tP = __dp4a(p4, 0x01010101u, tP);
                }
            }
            // ---- scans, boundary lanes (as gchain_eval_cdd)
            const uint32_t tAB = tA | (tB << 16);
            const uint32_t iP = group_incl_scan<G>(tP, 0);
            const uint32_t iAB = group_incl_scan<G>(tAB, 0);
            const int32_t Pb = (int32_t)(iP - tP);
            const uint32_t ABb = iAB - tAB;
            const int32_t Ab = (int32_t)(ABb & 0xffffu), Bb = (int32_t)(ABb >> 16);
            const int32_t Btot = (int32_t)(__shfl_sync(kFull, iAB, G - 1, G) >> 16);
            const bool lane_valid = l * E < n;
            const int Lk = hibit(group_ballot<G>(lane_valid && (Ab + Bb <= Btot), gbase));
            const int Lt = hibit(group_ballot<G>(lane_valid && (Pb <= d), gbase));
            const int Ls = max(0, min(Lk, Lt));
            const int32_t PbS = __shfl_sync(kFull, Pb, Ls, G);
            const uint32_t ABbS = __shfl_sync(kFull, ABb, Ls, G);
            const int32_t thr = Btot - (int32_t)(ABbS & 0xffffu) - (int32_t)(ABbS >> 16);
            const uint32_t key = ((uint32_t)min(thr, 0xffff) << 16) | 0xffffu;
            // boundary row Ls: SPR consecutive positions per lane, re-gathered through the staged ids
            const int e0 = l * SPR;
            uint32_t idw[(SPR + 1) / 2];
            e2_row_ids<G, E, SPR>(srow + (uint32_t)(Ls * CPS * 16), X::sw(grp * G + Ls), e0, idw);
            uint32_t v[SPR];
            uint32_t lsum = 0;
            const int kb = Ls * E + e0;  // sequence position of this lane's first boundary element
#pragma unroll
            for (int i = 0; i < SPR; ++i) {
                const uint32_t id = (i & 1) ? (idw[i >> 1] >> 16) : (idw[i >> 1] & 0xffffu);
                const uint32_t rec = (rv && kb + i < n) ? ldtab<TOFF>(((id << SH) & amask) | tabc) : 0u;
                // p | (alpha + beta) << 16
                v[i] = __byte_perm(rec, 0u, 0x4442u) + (__dp4a(rec, 0x00000101u, 0u) << 16);
                lsum += v[i];
            }
            const uint32_t ex = group_incl_scan<G>(lsum, 0) - lsum;
            // C_{k0} matters only when the boundary row is k0's (Ls == Lk; else C_{k0} > d, D = d)
            int32_t Dr = d - PbS;
            if (__any_sync(kFull, Ls == Lk)) {
                uint32_t run = ex, cinc = 0;
                const bool sat0 = ex <= key;
#pragma unroll
                for (int i = 0; i < SPR; ++i) {
                    const bool sat = run <= key;
                    run += v[i];
                    cinc = sat ? run : cinc;
                }
                const int own = max(0, hibit(group_ballot<G>(sat0, gbase)));
                const int32_t Ck0 = PbS + (int32_t)(__shfl_sync(kFull, cinc, own, G) & 0xffffu);
                if (Ls == Lk) Dr = min(Ck0, d) - PbS;
            }
            int32_t corr = 0;
            uint32_t run = ex;
#pragma unroll
            for (int i = 0; i < SPR; ++i) {
                const int32_t ci = (int32_t)(run & 0xffffu), si = (int32_t)(run >> 16);
                corr += (si - thr) * min((int32_t)(v[i] & 0xffu), max(0, Dr - ci));
                run += v[i];
            }
            __syncwarp();  // every lane is done with the stage: refill it two groups ahead
            issue(rg + 2 * gstep, st);
            // ---- F(C_m'): early weights left of lane Ls, tardy weights from it on
            const bool amode = l < Ls;
            uint32_t s = 0, acc = 0;
            if (quad) {
                // max(alpha, beta) <= 85: the weight bytes of four positions as one word (PRMT
                // from two pair words), their byte-wise exclusive prefixes by one IMAD, dotted with
                // the P quad by IDP.4A (as the SA kernels' quad pass)
                const uint32_t xsel = amode ? 0x6420u : 0x7531u;
#pragma unroll
                for (int q = 0; q < E / 4; ++q) {
                    const uint32_t x = __byte_perm(abp[2 * q], abp[2 * q + 1], xsel);
                    acc = __dp4a(x * 0x01010100u, pw[q], acc);
                    acc += s * __dp4a(pw[q], 0x01010101u, 0u);
                    s = __dp4a(x, 0x01010101u, s);
                }
            } else {
                const uint32_t psel = amode ? 0x4044u : 0x4144u;
                const uint32_t wsum = amode ? 0x00010001u : 0x01000100u;
#pragma unroll
                for (int j = 0; j < E / 2; ++j) {
                    const uint32_t f2 = s * 0x10001u + __byte_perm(abp[j], 0u, psel);
                    acc = (j & 1) ? __dp2a_hi(f2, pw[j >> 1], acc) : __dp2a_lo(f2, pw[j >> 1], acc);
                    s = __dp4a(abp[j], wsum, s);
                }
            }
            const int32_t base = amode ? Ab : (Btot - Bb);
            const int32_t contrib = base * (int32_t)tP + (amode ? (int32_t)acc : -(int32_t)acc) + corr;
            const int32_t Z = (int32_t)gsum2<G>((uint32_t)contrib);
            if (rv && l == 0) out[row] = (int64_t)Z;
        }
    }
    asm volatile("cp.async.wait_all;" ::: "memory");
    if (bad || (vmax & 0xffffu) >= (uint32_t)n || (vmax >> 16) >= (uint32_t)n) atomicOr(err, 1);
}

// kc_log2 = log2 of the table copies (5: conflict free, 4, 3); W warps per CTA; TOFF != 0 puts the
// table at the window start (needs the probed base to equal TOFF).  cudaErrorNotSupported if the
// layout does not fit.
template <int G, int E, int W, uint32_t TOFF, bool UCD = false>
cudaError_t launch2(const Instance& I, const int16_t* perms, int64_t ld, int64_t batch,
                    int64_t* out, cudaStream_t s, int kc_log2) {
    using X = E2<G, E>;
    if (TOFF != 0 && I.smem_base != TOFF) return cudaErrorNotSupported;
    int npow2 = 1;
    while (npow2 <= I.n) npow2 <<= 1;
    const uint32_t tbytes = (uint32_t)npow2 * (UCD ? 8u : 4u) << kc_log2;
    const uint32_t total = TOFF ? tbytes + (uint32_t)W * 2u * X::STAGE
                                : e2_layout(I.smem_base, tbytes, 2u * X::STAGE, W).total;
    if (total > (uint32_t)kE2MaxSmem) return cudaErrorNotSupported;
    auto kern = (I.n % 8) ? eval2_kernel<G, E, W, TOFF, true, UCD> : eval2_kernel<G, E, W, TOFF, false, UCD>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)total);
    if (e != cudaSuccess) return e;
    int sms = 148;
    e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, I.device);
    if (e != cudaSuccess) return e;
    const int64_t groups = (batch + X::CPW - 1) / X::CPW;
    int64_t blocks = (groups + W - 1) / W;
    if (blocks > sms) blocks = sms;
    if (blocks < 1) blocks = 1;
    kern<<<(unsigned)blocks, W * 32, total, s>>>(I.tab_ab16, I.tab_p, I.tab_m, I.tab_x, I.tab_g, I.n,
                                                 npow2, kc_log2, I.d_eff, perms, ld, batch, out, I.err,
                                                 !UCD && I.ab85_ok && !getenv("CDD_EVAL2_NO_QUAD"));
    return cudaGetLastError();
}

// Most copies that fit (32, 16, 8), W = 16 warps.  UCDDCP (8-byte entries) first tries the table
// at the window start (no alignment gap: 16 copies fit at n = 1000), then aligned to its size.
template <int G, int E, bool UCD = false>
cudaError_t launch2_auto(const Instance& I, const int16_t* perms, int64_t ld, int64_t batch,
                         int64_t* out, cudaStream_t s) {
    for (int kc = 5; kc >= 3; --kc) {
        if constexpr (UCD) {
            const cudaError_t e = launch2<G, E, 16, 1024, true>(I, perms, ld, batch, out, s, kc);
            if (e != cudaErrorNotSupported) return e;
        }
        const cudaError_t e = launch2<G, E, 16, 0, UCD>(I, perms, ld, batch, out, s, kc);
        if (e != cudaErrorNotSupported) return e;
    }
    return cudaErrorNotSupported;
}

__global__ void smem_base_probe(uint32_t* out) {
    extern __shared__ __align__(16) uint8_t smem[];
    *out = (uint32_t)__cvta_generic_to_shared(smem);
}

}  // namespace

cudaError_t probe_smem_base(uint32_t* base) {
    uint32_t* d = nullptr;
    cudaError_t e = cudaMalloc(&d, sizeof(uint32_t));
    if (e != cudaSuccess) return e;
    smem_base_probe<<<1, 1, 16>>>(d);
    e = cudaMemcpy(base, d, sizeof(uint32_t), cudaMemcpyDeviceToHost);
    cudaFree(d);
    return e;
}

// Returns cudaErrorNotSupported when the layout does not apply (the caller falls back).
cudaError_t launch_eval2_cdd(const Instance& I, const int16_t* perms, int64_t ld, int64_t batch,
                             int64_t* out, cudaStream_t s) {
    if (!I.ab16_ok || ld % 8 != 0 || (reinterpret_cast<uintptr_t>(perms) & 15) != 0)
        return cudaErrorNotSupported;
    const int n = I.n;
    if (n <= 16) return cudaErrorNotSupported;  // one-warp-per-many-rows kernel of eval.cu is faster
    if (const char* cfg = getenv("CDD_EVAL2_CFG"); cfg && n > 512) {  // layout experiments
        int w = 16, flat = 0, kc = 4;
        sscanf(cfg, "%d:%d:%d", &w, &flat, &kc);
        if (w == 8) return flat ? launch2<16, 64, 8, 1024>(I, perms, ld, batch, out, s, kc)
                                : launch2<16, 64, 8, 0>(I, perms, ld, batch, out, s, kc);
        if (w == 12) return flat ? launch2<16, 64, 12, 1024>(I, perms, ld, batch, out, s, kc)
                                 : launch2<16, 64, 12, 0>(I, perms, ld, batch, out, s, kc);
        return flat ? launch2<16, 64, 16, 1024>(I, perms, ld, batch, out, s, kc)
                    : launch2<16, 64, 16, 0>(I, perms, ld, batch, out, s, kc);
    }
    if (const char* cfg = getenv("CDD_EVAL2_GE")) {  // layout experiments: "G:E"
        int g = 0, e = 0;
        sscanf(cfg, "%d:%d", &g, &e);
        if (g * e >= n) {
            switch (g * 1000 + e) {
                case 4016: return launch2_auto<4, 16>(I, perms, ld, batch, out, s);
                case 4032: return launch2_auto<4, 32>(I, perms, ld, batch, out, s);
                case 8016: return launch2_auto<8, 16>(I, perms, ld, batch, out, s);
                case 8032: return launch2_auto<8, 32>(I, perms, ld, batch, out, s);
                case 8064: return launch2_auto<8, 64>(I, perms, ld, batch, out, s);
                case 16016: return launch2_auto<16, 16>(I, perms, ld, batch, out, s);
                case 16032: return launch2_auto<16, 32>(I, perms, ld, batch, out, s);
                case 16064: return launch2_auto<16, 64>(I, perms, ld, batch, out, s);
                default: break;
            }
        }
    }
    if (n <= 64) return launch2_auto<4, 16>(I, perms, ld, batch, out, s);
    if (n <= 128) return launch2_auto<4, 32>(I, perms, ld, batch, out, s);
    if (n <= 256) return launch2_auto<8, 32>(I, perms, ld, batch, out, s);
    if (n <= 512) return launch2_auto<8, 64>(I, perms, ld, batch, out, s);
    return launch2_auto<16, 64>(I, perms, ld, batch, out, s);
}

// UCDDCP: at most 32 positions per lane (four register arrays: alpha|beta pairs, gamma pairs,
// M and X bytes).
cudaError_t launch_eval2_ucddcp(const Instance& I, const int16_t* perms, int64_t ld, int64_t batch,
                                int64_t* out, cudaStream_t s) {
    if (!I.ab16_ok || !I.has_ucd || ld % 8 != 0 || (reinterpret_cast<uintptr_t>(perms) & 15) != 0)
        return cudaErrorNotSupported;
    const int n = I.n;
    if (n <= 16 || getenv("CDD_EVAL2_NO_UCD")) return cudaErrorNotSupported;
    if (const char* cfg = getenv("CDD_EVAL2_UCD_GE")) {  // layout experiments: "G:E"
        int g = 0, e = 0;
        sscanf(cfg, "%d:%d", &g, &e);
        const int ge = g * 1000 + e;
        if (g * e >= n) {
            if (ge == 8016) return launch2_auto<8, 16, true>(I, perms, ld, batch, out, s);
            if (ge == 16016) return launch2_auto<16, 16, true>(I, perms, ld, batch, out, s);
            if (ge == 8032) return launch2_auto<8, 32, true>(I, perms, ld, batch, out, s);
            if (ge == 16032) return launch2_auto<16, 32, true>(I, perms, ld, batch, out, s);
            if (ge == 32032) return launch2_auto<32, 32, true>(I, perms, ld, batch, out, s);
            if (ge == 16064) return launch2_auto<16, 64, true>(I, perms, ld, batch, out, s);
        }
    }
    if (n <= 64) return launch2_auto<4, 16, true>(I, perms, ld, batch, out, s);
    if (n <= 128) return launch2_auto<8, 16, true>(I, perms, ld, batch, out, s);
    if (n <= 256) return launch2_auto<8, 32, true>(I, perms, ld, batch, out, s);
    if (n <= 512) return launch2_auto<16, 32, true>(I, perms, ld, batch, out, s);
    return launch2_auto<32, 32, true>(I, perms, ld, batch, out, s);
}

}  // namespace cdd
