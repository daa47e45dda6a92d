/*
 * cdd.h -- C-ABI of libcdd, the B200 (sm_100a) hot path of Awasthi, Lässig, Leuschner & Weise,
 * "GPGPU-based Parallel Algorithms for Scheduling Against Due Date" (IPDPSW 2016).
 *
 * Citations: P:<line> = /root/reference/PAPER.md line (section / equation / algorithm / table).
 *
 * The path: many asynchronous SA chains (Alg. 1) or a DPSO swarm (Alg. 2, eq. (3),
 * P:236-257) whose inner step is the O(n) optimal-timing routine for a fixed job sequence
 * (CDD: P:94-122; UCDDCP: P:137-166), followed by a reduction to the best sequence.
 *
 * Conventions (all entry points):
 *   - every call returns a cdd_status; nothing throws across the ABI; cdd_last_error() returns a
 *     thread-local message for the last non-OK status;
 *   - argument errors are detected synchronously and nothing is launched;
 *   - "device" pointers are CUDA device pointers on the instance's device (e.g. torch tensors);
 *     "host" pointers are ordinary host memory; the caller keeps ownership of both;
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream); calls marked
 *     ASYNC only enqueue work on it; CUDA errors surface as CDD_ECUDA at the call that sees them;
 *   - const pointers are never written; the library frees nothing it did not allocate.
 * Job sequences are int16 rows: row b holds a permutation of job ids 0..n-1 in positions 0..n-1 of
 * a row of stride ld >= n elements (ld % 8 == 0 and a 16-byte aligned base enable vector loads).
 */
#ifndef CDD_H
#define CDD_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define CDD_ABI_VERSION 5

#if defined(__GNUC__)
#define CDD_API __attribute__((visibility("default")))
#else
#define CDD_API
#endif

typedef enum {
    CDD_OK = 0,
    CDD_EINVAL = -1, /* bad argument (null pointer, size, problem/instance mismatch)          */
    CDD_ERANGE = -2, /* instance outside the supported value ranges (see cdd_instance_create)  */
    CDD_ENOMEM = -3, /* device allocation failed / workspace too small                         */
    CDD_ECUDA = -4,  /* CUDA runtime error (message in cdd_last_error)                          */
    CDD_ESTATE = -5, /* no result available yet (best_get before any run)                       */
    CDD_EDATA = -6   /* a sequence contained a job id outside [0, n) (reported by cdd_check)    */
} cdd_status;

typedef enum { CDD_PROBLEM_CDD = 0, CDD_PROBLEM_UCDDCP = 1 } cdd_problem;

/* SA neighbourhood (readings R11, R11b, R11c):
 *   CDD_MOVE_PERT_FY  the paper's move: Pert jobs at random positions (Floyd sample)
 *                     shuffled by Fisher-Yates over their slots;
 *   CDD_MOVE_SWAP     two random positions exchanged;
 *   CDD_MOVE_INSERT   the job at a random position `from` is re-inserted at a random position
 *                     `to` != from, the jobs in between move one place towards `from`
 *                     ((from, to) uniform over ordered pairs; BASELINE "swap/insertion move");
 *   CDD_MOVE_WINDOW   the contiguous sub-sequence of Pert positions at a random start shuffled by
 *                     Fisher-Yates ("A sub-sequence of size Pert=4 is selected"). */
typedef enum { CDD_MOVE_PERT_FY = 0, CDD_MOVE_SWAP = 1, CDD_MOVE_INSERT = 2, CDD_MOVE_WINDOW = 3 } cdd_move;

typedef struct cdd_instance cdd_instance; /* opaque, library-owned, bound to one device */

/* ------------------------------------------------------------------------------------------ */
/* Instances (problem data)                                                           */
/* ------------------------------------------------------------------------------------------ */
/* Copies the host arrays p, alpha, beta (and m, gamma for UCDDCP; both NULL = CDD only), all
 * indexed by job id, to device `device`.  The problem data of P:29-49 are general non-negative
 * integers.  Checks (CDD_EINVAL): 1 <= n <= 32767 (int16 job ids), p_i >= 1, alpha_i, beta_i >= 0,
 * 0 <= m_i <= p_i, gamma_i >= 0, d >= 0.  CDD_ERANGE only if a penalty could leave the exact
 * int64 range of the outputs: (sum alpha + sum beta) * sum p + sum gamma * sum (p - m) >= 2^62.
 *
 * Fast and generic paths (chosen here, reported by cdd_instance_query flags bit2):
 *   fast    -- n <= 1024, p <= 255, sum alpha, sum beta < 2^16, (sum alpha + sum beta) * sum p
 *              < 2^31, 32 * max(alpha, beta) < 2^16 (and for UCDDCP data gamma < 2^16, p - m <=
 *              255, the packed UCDDCP record fits 32 bits): packed 8/16-bit job records, int32
 *              arithmetic, the tuned kernels (every Biskup-Feldmann instance, p <= 20, alpha <= 10,
 *              beta <= 15, at n <= 1000).  The group SA kernels also need alpha, beta <= 255.
 *              An instance whose CDD data fit but whose UCDDCP record does not runs the CDD on the
 *              fast path and the UCDDCP on the generic one.
 *   generic -- everything else: int32 fields per job, int64 arithmetic, a warp (n <= 2048) or a
 *              CTA per sequence.  Serves the batched evaluators, the schedules, asynchronous SA
 *              (every move) and T0; synchronous SA and DPSO return CDD_EINVAL; the best result is
 *              read with best_get / best_device_ptrs_wide (best_device_ptrs: CDD_EINVAL).
 * Both paths compute the same penalties (the closed form of DESIGN.md §4) and draw the same
 * random numbers, so an instance's results do not depend on the path.  Synchronous.  *out
 * receives the instance. */
CDD_API int cdd_instance_create(int32_t n, const int32_t *p, const int32_t *alpha, const int32_t *beta,
                        const int32_t *m, const int32_t *gamma, int64_t d, int device,
                        cdd_instance **out);
CDD_API int cdd_instance_destroy(cdd_instance *inst);
/* n, d, sum of p, and flags (bit0: UCDDCP data present, bit1: d >= sum p, bit2: the CDD runs on
 * the generic path, bit3: the UCDDCP runs on the generic path -- its packed record does not fit
 * even where the CDD's does, bit4: the CDD's asynchronous SA at 8 threads x 128 positions per
 * chain (n in (512, 1024]) uses the small-weight layout -- alpha, beta <= 15 and
 * max(p) * max(alpha, beta) * 120 < 2^16: 4-bit weights and cached sub-block summaries, same
 * results).  Any out may be NULL. */
CDD_API int cdd_instance_query(const cdd_instance *inst, int32_t *n, int64_t *d, int64_t *sum_p,
                       int32_t *flags);

/* ------------------------------------------------------------------------------------------ */
/* Batched sequence evaluation: layer (ii) of the two-layered approach               */
/* ------------------------------------------------------------------------------------------ */
/* ASYNC.  out[b] (device int64) = optimal eq. (1) penalty of sequence row b for the CDD with the
 * instance's d (restrictive or not) -- the value the linear algorithm of P:94-122 finds.
 * perms: device int16 [batch][ld].  A job id outside [0,n) raises the instance's data-error flag
 * (see cdd_check) and makes that row's penalty unspecified; nothing is read out of bounds.
 * Duplicates are not detected. */
CDD_API int cdd_eval_batch(cdd_instance *inst, const int16_t *perms, int64_t ld, int64_t batch,
                   int64_t *out, void *stream);
/* ASYNC.  As above for the UCDDCP objective eq. (2).  CDD_EINVAL if the instance has
 * no m/gamma or d < sum p (the paper defines the algorithm for the unrestricted case). */
CDD_API int ucddcp_eval_batch(cdd_instance *inst, const int16_t *perms, int64_t ld, int64_t batch,
                      int64_t *out, void *stream);
/* SYNCHRONOUS end-to-end variant with HOST buffers: copies perms_host (int16 [batch][ld]) to the
 * device in chunks, evaluates, copies the penalties to out_host (int64 [batch]), synchronises. */
CDD_API int cdd_eval_batch_host(cdd_instance *inst, cdd_problem problem, const int16_t *perms_host,
                        int64_t ld, int64_t batch, int64_t *out_host, void *stream);
/* ASYNC.  The optimal schedule of each row (what the O(n) routine finds: P:94-122 for the CDD,
 * P:137-166 for the UCDDCP), for inspection or for materialising the best sequence of a run.
 *   C       device int64 [batch][n]: completion time of the job at each position;
 *   X       device int32 [batch][n]: UCDDCP compressions (NULL for the CDD);
 *   start   device int64 [batch]: start time of the first job;
 *   penalty device int64 [batch]: eq. (1) / (2) of this schedule, equal to the *_eval_batch value.
 * With k0 = max{k : S_k <= sum beta} (S_k = sum of alpha + beta before position k), job k0 completes
 * at d when C_{k0} <= d, else the schedule starts at 0 (CDD); UCDDCP: job k0 completes at d and job
 * k is compressed fully iff its weight (A_{k-1} for k <= k0, else B_k) exceeds gamma_k.  When the
 * cost has a flat optimum the schedule is one of the optimal ones (the penalty is unique).  Ids
 * outside [0, n) raise the data-error flag as in cdd_eval_batch. */
CDD_API int cdd_schedule_batch(cdd_instance *inst, cdd_problem problem, const int16_t *perms,
                               int64_t ld, int64_t batch, int64_t *C, int32_t *X, int64_t *start,
                               int64_t *penalty, void *stream);
/* Synchronises `stream`; returns CDD_EDATA (and clears the flag) if any evaluated sequence held
 * a job id outside [0, n) since the last check, else CDD_OK. */
CDD_API int cdd_check(cdd_instance *inst, void *stream);

/* ------------------------------------------------------------------------------------------ */
/* Asynchronous parallel SA (Alg. 1)                                                */
/* ------------------------------------------------------------------------------------------ */
typedef struct {
    cdd_problem problem;
    int64_t chains;        /* chains on this device                                            */
    int64_t steps;         /* Alg. 1 #Iterations (1000 / 5000)                       */
    double mu;             /* exponential cooling factor (0.88)                          */
    double T0;             /* > 0: initial temperature; <= 0: T0 = std of t0_samples random    */
                           /* sequences, computed on the device                          */
    int64_t t0_samples;    /* 5000 (used when T0 <= 0)                                   */
    int32_t pert;          /* perturbation size (4); 1 <= pert <= 4                      */
    cdd_move move;
    uint64_t seed;         /* Philox key                                                        */
    uint64_t chain_offset; /* global id of local chain 0 (multi-GPU: rank * chains);            */
                           /* chain_offset + chains <= 2^32                                     */
    int64_t *trace;        /* optional device int64 [chains][steps]: (E_new << 1) | accepted    */
    int64_t *chain_best;   /* optional device int64 [chains]: best penalty of each chain        */
    int64_t *chain_final;  /* optional device int64 [chains]: final penalty of each chain       */
    double *T0_out;        /* optional device double [1]: the T0 used                            */
    const double *T0_in;   /* optional device double [1]: T0 read on the device (e.g. from sa_t0); */
                           /* overrides T0 / t0_samples when non-NULL                             */
    int32_t lanes;         /* threads per chain: 0 = automatic (by n and chains), 32 = one warp  */
                           /* per chain (the only layout of the generic path),                   */
                           /* per chain, 4 / 8 / 16 = 8 / 4 / 2 chains per warp (16-bit records: */
                           /* needs alpha, beta <= 255, else CDD_EINVAL); results do not depend  */
                           /* on it (bit-identical), only the speed does                          */
    const int16_t *init;   /* optional device int16: Alg. 1 line 1's s0 given by the caller (P:205 */
                           /* "the initial job sequences are copied to the GPU"): chain c (local) */
                           /* starts from init + c * init_ld; init_ld = 0: every chain from the   */
                           /* same sequence; init_ld >= n otherwise.  NULL: each chain's own      */
                           /* Philox random sequence (reading R13).  Rows must be permutations of */
                           /* 0..n-1; an id outside [0, n) raises the data-error flag (cdd_check) */
                           /* and is replaced by 0.  Added in ABI version 3.                      */
    int64_t init_ld;
} sa_params;

/* Bytes of device workspace sa_run needs for these parameters (caller allocates, e.g. torch). */
CDD_API size_t sa_workspace_size(const cdd_instance *inst, const sa_params *params);
/* ASYNC.  Runs params->chains independent chains to completion in one persistent kernel, then
 * reduces min (best penalty, global chain id) into the instance's best buffers. */
CDD_API int sa_run(cdd_instance *inst, const sa_params *params, void *workspace, size_t workspace_bytes,
           void *stream);
/* The thread layout sa_run would use for these parameters: *lanes threads per chain (32: one
 * warp per chain; 4 / 8 / 16: 8 / 4 / 2 chains per warp) holding *positions_per_lane sequence
 * positions each (lanes x positions >= n).  Host-only, synchronous; either out may be NULL. */
CDD_API int sa_layout(const cdd_instance *inst, const sa_params *params, int32_t *lanes,
                      int32_t *positions_per_lane);
/* ASYNC.  Only the T0 rule: *T0_dev = population std of the penalties of `samples`
 * Philox-random sequences.  Workspace: sa_workspace_size() of an sa_params with T0 <= 0. */
CDD_API int sa_t0(cdd_instance *inst, cdd_problem problem, uint64_t seed, int64_t samples, double *T0_dev,
          void *workspace, size_t workspace_bytes, void *stream);

/* ------------------------------------------------------------------------------------------ */
/* Synchronous SA (Fig. 8; reading R18)                                   */
/* ------------------------------------------------------------------------------------------ */
/* Every chain starts from its own random state; at temperature level j = 0..levels-1 every chain
 * runs a Markov chain of markov_len (M) moves at the constant temperature T_j (T_0 from T0 /
 * t0_samples / T0_in as in sa_params, T_{j+1} = T_j * mu); the final state of minimal penalty over
 * all chains (ties: lowest global id) is the initial state of every chain at level j+1.  Move m of
 * level j uses the Philox counters of step j*M + m.  The instance's best buffers receive the
 * best-ever state (within a level min (penalty, chain id); a later level only if strictly better).
 * Runs on the group layout (lanes 0 = automatic, 4, 8, 16; needs alpha, beta <= 255). */
typedef struct {
    cdd_problem problem;
    int64_t chains;        /* chains on this device                                            */
    int64_t markov_len;    /* M: moves per chain per temperature level (>= 1)                  */
    int64_t levels;        /* temperature levels (>= 1); levels * M < 2^32                      */
    double mu;             /* cooling factor between levels                                      */
    double T0;             /* > 0: initial temperature; <= 0: from t0_samples             */
    int64_t t0_samples;
    int32_t pert;          /* 1 <= pert <= 4                                                     */
    cdd_move move;
    uint64_t seed;
    uint64_t chain_offset; /* global id of local chain 0 (multi-GPU: rank * chains)              */
    int32_t lanes;         /* threads per chain: 0 automatic, 4, 8 or 16                         */
    double *T0_out;        /* optional device double [1]: T_0                                    */
    const double *T0_in;   /* optional device double [1]: T_0 read on the device                */
    int64_t *level_min;    /* optional device int64 [levels]: penalty of s^min_j (device-local)  */
} sa_sync_params;
CDD_API size_t sa_sync_workspace_size(const cdd_instance *inst, const sa_sync_params *params);
/* ASYNC.  All levels on this device (the swarm of chains is this device's). */
CDD_API int sa_sync_run(cdd_instance *inst, const sa_sync_params *params, void *workspace,
                        size_t workspace_bytes, void *stream);
/* Stepping interface for chains spread over several GPUs.  ASYNC.  sa_sync_level(j) runs level j
 * (call j = 0, 1, ..., levels-1 in order with the same workspace); afterwards sa_sync_ptrs gives
 * the level's packed key (final penalty << 32 | global id, int64) and the int16 [n] state s^min_j
 * that level j+1 starts from -- MIN-all-reduce the key and broadcast the state from the owning
 * rank between levels; the best-ever buffers stay device-local (reduce them with the async-SA
 * helpers at the end). */
CDD_API int sa_sync_level(cdd_instance *inst, const sa_sync_params *params, void *workspace,
                          size_t workspace_bytes, int64_t j, void *stream);
CDD_API int sa_sync_ptrs(const cdd_instance *inst, const sa_sync_params *params, void *workspace,
                         int64_t **key_dev, int16_t **perm_dev);

/* ------------------------------------------------------------------------------------------ */
/* Discrete PSO (Alg. 2, eq. (3))                                                   */
/* ------------------------------------------------------------------------------------------ */
/* Operators (reading R15): F1 swaps two Floyd-sampled positions; F2 keeps the first
 * c positions (c uniform in [1, n-1]) and appends the other jobs in personal-best order; F3 keeps
 * the segment [q0, q1] and fills the other positions left to right with the remaining jobs in
 * swarm-best order.  x' = c (+) f(x) applies f iff rand(0,1) < c. */
typedef struct {
    cdd_problem problem;
    int64_t particles;        /* particles on this device (one warp each)                        */
    int64_t iters;            /* Alg. 2 #Iterations                                              */
    double w, c1, c2;         /* probabilities of F1 / F2 / F3 in eq. (3) (silent in the paper)    */
    uint64_t seed;
    uint64_t particle_offset; /* global id of local particle 0 (multi-GPU swarm: rank * particles) */
    int64_t *gbest_trace;     /* optional device int64 [iters]: swarm best value at line 5 of     */
                              /* iteration t (device-local unless the caller reduces across GPUs) */
} dpso_params;
CDD_API size_t dpso_workspace_size(const cdd_instance *inst, const dpso_params *params);
/* ASYNC.  Whole run on one device (the swarm is this device's particles): lines 1-2, then
 * `iters` x lines 4-7, then the final best particle into the instance's best buffers.
 * CDD_EINVAL if n < 2 (F1-F3 need two positions), particles outside [1, 2^31), or the global
 * particle ids do not fit 32 bits; iters = 0 returns the best initial particle. */
CDD_API int dpso_run(cdd_instance *inst, const dpso_params *params, void *workspace,
             size_t workspace_bytes, void *stream);
/* Stepping interface for a swarm spread over several GPUs.  ASYNC each.
 *   dpso_begin:   lines 1-2 plus the personal/swarm best of iteration 0 (device-local);
 *   dpso_gbest_ptrs(t): the packed swarm-best key (int64, (value << 32) | global id) and its
 *                 int16 [n] sequence that iteration t reads -- all-reduce the key (MIN) and
 *                 broadcast the sequence from the owning rank between dpso_begin / dpso_iterate;
 *   dpso_iterate(t): lines 6-7 of iteration t and lines 4-5 of iteration t+1;
 *   dpso_end:     copies the (reduced) swarm best after `iters` iterations to the best buffers. */
CDD_API int dpso_begin(cdd_instance *inst, const dpso_params *params, void *workspace,
               size_t workspace_bytes, void *stream);
CDD_API int dpso_iterate(cdd_instance *inst, const dpso_params *params, void *workspace,
                 size_t workspace_bytes, int64_t t, void *stream);
CDD_API int dpso_gbest_ptrs(const cdd_instance *inst, const dpso_params *params, void *workspace,
                    int64_t t, int64_t **key_dev, int16_t **perm_dev);
CDD_API int dpso_end(cdd_instance *inst, const dpso_params *params, void *workspace,
             size_t workspace_bytes, void *stream);

/* Fused swarm-best exchange over peer memory (one process per GPU; NVLink / NVSwitch P2P).
 * Alg. 2 line 5 takes the swarm best over ALL particles every iteration (reading R16).
 * Instead of two collectives between launches (dpso_gbest_ptrs + NCCL), dpso_run_peer does the
 * exchange inside its kernels: each rank's last CTA publishes its device-local best sequence in
 * its own region, MIN-reduces the packed key into rank 0's region with a system-scope atomic,
 * arrives on rank 0's counter, waits for every rank, and copies the owner's sequence with peer
 * loads.  Protocol:
 *   dpso_peer_create(world, rank, handle): allocates this rank's region (library-owned, one
 *       device allocation of 64 + 4 * 32 * ceil-pow2(n / 32) bytes) and returns its CUDA IPC handle
 *       (CDD_IPC_HANDLE_BYTES bytes, written to `ipc_handle`);
 *   the caller exchanges the handles (e.g. torch.distributed all_gather) so every rank holds all
 *       of them in rank order;
 *   dpso_peer_open(handles [world * CDD_IPC_HANDLE_BYTES]): maps every other rank's region;
 *   dpso_peer_reset(stream): re-arms this rank's region -- before EVERY run, followed by a
 *       cross-process barrier after the stream has completed (no rank may start before rank 0's
 *       region is re-armed); a fused run without a reset since the previous one returns
 *       CDD_ESTATE;
 *   dpso_run_peer(params): the whole run (as dpso_run) with particle_offset = rank * particles
 *       (equal shares); every rank must call it (the kernels wait for each other: all ranks'
 *       kernels must be able to run concurrently -- one GPU per rank, or time-sliced processes);
 *   dpso_peer_destroy: unmaps and frees (also done by cdd_instance_destroy).
 * Results are identical to one GPU running all particles (same Philox streams, same ties).
 * A rank that never arrives at an exchange (its process died) does not hang the others: after 30 s
 * the wait gives up, cdd_check reports CDD_EDATA ("a peer rank never reached ..."), and from then
 * on every rank continues with its own device-local swarm best (no peer memory is read).
 * CDD_ESTATE on a wrong order of calls; CDD_ECUDA if IPC is unavailable. */
#define CDD_IPC_HANDLE_BYTES 64
CDD_API int dpso_peer_create(cdd_instance *inst, int world, int rank, uint8_t *ipc_handle);
CDD_API int dpso_peer_open(cdd_instance *inst, const uint8_t *handles);
CDD_API int dpso_peer_reset(cdd_instance *inst, void *stream);
CDD_API int dpso_peer_destroy(cdd_instance *inst);
CDD_API int dpso_run_peer(cdd_instance *inst, const dpso_params *params, void *workspace,
                  size_t workspace_bytes, void *stream);
/* Synchronous SA over all ranks with the same peer exchange (after dpso_peer_open and a
 * dpso_peer_reset + barrier per run): every level's s^min is the minimum over the
 * chains of ALL ranks, exchanged inside the level's finalisation kernel; chain_offset must be
 * rank * chains.  The best-ever state stays device-local (reduce it once with best_device_ptrs).
 * Results equal one device running all chains (R18: the chain holding a tied best may differ). */
CDD_API int sa_sync_run_peer(cdd_instance *inst, const sa_sync_params *params, void *workspace,
                     size_t workspace_bytes, void *stream);

/* ------------------------------------------------------------------------------------------ */
/* Best result of the last run (SA or DPSO) on this instance                                   */
/* ------------------------------------------------------------------------------------------ */
/* Library-owned device buffers: packed int64 key = (penalty << 32) | global id (min = best,
 * ties to the lowest id) and int16 [n] sequence.  Valid until the next run or destroy.  The
 * caller may all-reduce the key (MIN) and broadcast the sequence across GPUs in place. */
CDD_API int best_device_ptrs(cdd_instance *inst, int64_t **packed_dev, int16_t **perm_dev);
/* Generic-path instances (flags bit2): device int64 [2] = {penalty, global id} and the int16 [n]
 * sequence (the penalty may exceed the packed key's 32 bits).  Across GPUs: MIN-reduce the
 * penalty, then the id among the ranks holding that penalty, then broadcast the owner's sequence.
 * CDD_EINVAL for fast-path instances (use best_device_ptrs).  Added in ABI version 5. */
CDD_API int best_device_ptrs_wide(cdd_instance *inst, int64_t **pen_id_dev, int16_t **perm_dev);
/* SYNCHRONOUS: penalty, sequence (host int16 [n], may be NULL) and global chain/particle id. */
CDD_API int best_get(cdd_instance *inst, int64_t *penalty, int16_t *perm_host, uint64_t *id, void *stream);

CDD_API const char *cdd_last_error(void);
CDD_API int cdd_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* CDD_H */
