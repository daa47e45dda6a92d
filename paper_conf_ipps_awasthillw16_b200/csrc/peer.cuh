// peer.cuh -- one exchange of a packed (value << 32 | global id) key and its sequence across the
// ranks of a peer-memory exchange (dpso_peer_* / Instance::peer), run by one whole CTA per rank.
// Used by the DPSO iteration kernels (Alg. 2 line 5 over the global swarm, every iteration) and
// by the synchronous-SA level finalisation (s^min of P:184-186 over all chains, every level).
//
// Regions (internal.h): u64 key[3] and u32 arrivals (rank 0's are the global ones), then int16
// perm[2][np] per rank.  Exchange e, parity par:
//  1. the local best sequence goes to this rank's perm[par];
//  2. system-scope atomicMin of the key into rank 0's slot e % 3, then an arrival on rank 0's
//     counter; wait until all `world` ranks have arrived at exchange e (acquire, system scope);
//  3. the global key's id decides the owner (id / per_rank); the other ranks copy its perm[par].
// Slot reuse without resets: rank 0 re-arms slot (e+1) % 3 before it arrives at e (that slot was
// last read at e-2, before every rank arrived at e-1; no rank uses it for e+1 before rank 0 has
// arrived at e).  perm[par] is rewritten at e+2, after every reader has arrived at e+1.
#pragma once
#include <cuda_runtime.h>

#include <climits>
#include <cstdint>

#include "internal.h"

namespace cdd {

__device__ __forceinline__ unsigned int peer_ld_acquire(const unsigned int* p) {
    unsigned int v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long peer_ld_acquire64(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

// Whole CTA; `seq` (len entries, global memory) holds this rank's best sequence on entry and the
// global best's on exit.  Returns the global key (every thread).
// A rank that never arrives (its process died) must not hang the others: after kPeerTimeoutNs
// the wait gives up, raises bit 2 of the instance's error flag (cdd_check reports it), and this
// and every later exchange of the run keep the LOCAL key and sequence (no peer memory is read
// once the exchange is broken: the winner could be the dead rank, or its slot already re-armed).
constexpr unsigned long long kPeerTimeoutNs = 30ull * 1000 * 1000 * 1000;
__device__ __forceinline__ unsigned long long peer_globaltimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ unsigned long long peer_exchange_block(uint8_t* const* regions, int world,
                                                                  int rank, int64_t per_rank, int np,
                                                                  uint32_t e, int par,
                                                                  unsigned long long local_key,
                                                                  int16_t* seq, int len, int* err) {
    __shared__ unsigned long long s_gk;
    __shared__ int s_owner;
    uint8_t* root = regions[0];
    unsigned long long* rkey = reinterpret_cast<unsigned long long*>(root + kPeerKeyOff);
    unsigned int* rarr = reinterpret_cast<unsigned int*>(root + kPeerArriveOff);
    int16_t* mine = reinterpret_cast<int16_t*>(regions[rank] + kPeerPermOff) + (size_t)par * np;
    for (int i = threadIdx.x; i < len; i += blockDim.x) mine[i] = seq[i];
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence_system();
        if (rank == 0) {
            rkey[(e + 1) % 3] = ULLONG_MAX;
            __threadfence_system();
        }
        atomicMin_system(&rkey[e % 3], local_key);
        __threadfence_system();
        atomicAdd_system(rarr, 1u);
        const unsigned int target = (unsigned int)world * (e + 1u);
        const unsigned long long t0 = peer_globaltimer();
        // after one timeout the exchange is broken for the rest of the run: no more waiting
        while (!(*(volatile int*)err & 2) && (int)(peer_ld_acquire(rarr) - target) < 0) {
            __nanosleep(64);
            if (peer_globaltimer() - t0 > kPeerTimeoutNs) {
                atomicOr(err, 2);
                break;
            }
        }
        unsigned long long gk = peer_ld_acquire64(&rkey[e % 3]);
        // validate before any peer read: a broken exchange, an empty key or an owner outside the
        // world fall back to this rank's own best
        const unsigned long long own = gk == ULLONG_MAX ? ~0ull : (gk & 0xffffffffull) / (unsigned long long)per_rank;
        const bool ok = !(*(volatile int*)err & 2) && gk != ULLONG_MAX && own < (unsigned long long)world &&
                        gk <= local_key;
        s_gk = ok ? gk : local_key;
        s_owner = ok ? (int)own : rank;
    }
    __syncthreads();
    const unsigned long long gk = s_gk;
    const int owner = s_owner;
    if (owner != rank) {
        const volatile int16_t* src = reinterpret_cast<const int16_t*>(regions[owner] + kPeerPermOff) + (size_t)par * np;
        for (int i = threadIdx.x; i < len; i += blockDim.x) seq[i] = src[i];
    }
    __threadfence();
    __syncthreads();
    return gk;
}

}  // namespace cdd
