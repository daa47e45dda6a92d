/*
 * oracle.h -- CPU ORACLE, TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct C implementation of what the hot path computes, written from
 * the paper (/root/reference/PAPER.md, cited as P:<line>) and the readings recorded in DESIGN.md.
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may load
 * it.  It shares NO code with paper_conf_ipps_awasthillw16_b200/csrc (the CUDA path) and neither
 * includes the other.  Random numbers the method draws come from this file's own Philox4x32-10.
 *
 * Parity status per function:
 *   or_philox4x32_10        pinned: Random123/cuRAND known-answer vectors
 *   or_det_exp              pinned: vs libm exp (rel err < 1e-15) + exact special points
 *   or_cdd_eval             pinned: Table I worked example (every intermediate value),
 *                                    shift brute force, n! brute force, V-shape, Theorem 1
 *   or_ucddcp_eval          pinned: Table I worked example (penalty 77), integer-LP brute force,
 *                                    Properties 1-2
 *   or_perm_fy / neighbour  pinned: uniformity (chi-square) on tiny n, FY definition [14];
 *                           insert: permutation + one-segment rotation + uniform (from, to);
 *                           window: contiguous positions, uniform start, uniform slot shuffle
 *   or_t0                   pinned: vs numpy population std of independently evaluated samples
 *   or_sa_chain / run       pinned: invariants (greedy at T0=0, best==eval(best perm), n=10 reaches the
 *                                    10! optimum); trajectory "parity unpinned" vs the paper
 *   or_dpso_*               pinned: operator invariants (F1/F2/F3 keep permutations, kept segments),
 *                                    w=c1=c2=0 reduces to best-of-initial; trajectory "parity unpinned"
 */
#ifndef CDD_ORACLE_H
#define CDD_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Problem data.  Arrays are indexed by job id 0..n-1.  M and gamma may be NULL (CDD). */
typedef struct {
    int32_t n;
    const int32_t *P;      /* processing times P_i >= 1                     */
    const int32_t *M;      /* minimum processing times M_i <= P_i (UCDDCP)  */
    const int32_t *alpha;  /* earliness penalty per time unit               */
    const int32_t *beta;   /* tardiness penalty per time unit               */
    const int32_t *gamma;  /* compression penalty per time unit (UCDDCP)    */
    int64_t d;             /* common due date                               */
} or_instance;

enum { OR_CDD = 0, OR_UCDDCP = 1 };

/* Trace of the literal CDD walk.  All indices 1-based as in the paper. */
#define OR_WALK_MAX 64
typedef struct {
    int32_t tau;                 /* max i with DT_i = C_i - d <= 0, 0 if none            */
    int64_t pe0, pl0;            /* sum alpha_{1..tau}, sum beta_{tau+1..n} at t=0 start  */
    int64_t first_shift;         /* DT shift placing job tau at d (0 if not taken)        */
    int32_t nsteps;              /* walk iterations (<= OR_WALK_MAX recorded)             */
    int64_t pe[OR_WALK_MAX];     /* pe after the update of iteration i                    */
    int64_t pl[OR_WALK_MAX];     /* pl after the update of iteration i                    */
    int32_t r;                   /* job position completing at d, 0 if schedule starts at 0 */
    int64_t s;                   /* start time of the first job (total right shift)       */
} or_walk;

/* ---- random numbers (cuRAND, normalised to [0,1]) -------------------------------- */
void     or_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
uint32_t or_bnd(uint32_t w, uint32_t m);           /* floor(w*m / 2^32), uniform on [0,m)   */
double   or_u01(uint32_t w);                        /* (w + 0.5) * 2^-32, in (0,1)           */
double   or_det_exp(double x);                      /* deterministic exp, spec in DESIGN.md  */

/* Counter-layout tags. */
#define OR_TAG_SA_INIT   0x11u
#define OR_TAG_SA        0x12u
#define OR_TAG_T0        0x13u
#define OR_TAG_DPSO_INIT 0x21u
#define OR_TAG_DPSO      0x22u

/* Fisher-Yates shuffle of the identity [14] driven by Philox (key=seed, ctr=(b, id_lo, id_hi, tag<<16)). */
void or_perm_fy(int32_t n, uint64_t seed, uint32_t tag, uint64_t id, int16_t *J);

/* ---- sequence evaluators (layer (ii) of the two-layered approach) --------------- */
int64_t or_cdd_eval(const or_instance *I, const int16_t *J, or_walk *w, int64_t *C_out);
/* returns INT64_MIN if d < sum P (the UCDDCP algorithm is defined for d >= sum P only) */
int64_t or_ucddcp_eval(const or_instance *I, const int16_t *J, int32_t *X_out, int64_t *C_out);
void    or_eval_batch(const or_instance *I, int problem, const int16_t *perms, int64_t ld,
                      int64_t batch, int64_t *out);

/* ---- Simulated annealing (Alg. 1; asynchronous chains P:172-179) -------------- */
/* Neighbour moves (R11, R11b, R11c): PERT_FY = Pert distinct random positions shuffled by
 * Fisher-Yates; SWAP = two random positions exchanged; INSERT = the job at a random position
 * `from` re-inserted at a random position `to` (BASELINE north_star "swap/insertion move");
 * WINDOW = a contiguous sub-sequence of Pert positions shuffled by Fisher-Yates. */
enum { OR_MOVE_PERT_FY = 0, OR_MOVE_SWAP = 1, OR_MOVE_INSERT = 2, OR_MOVE_WINDOW = 3 };
typedef struct {
    int32_t  problem;       /* OR_CDD / OR_UCDDCP                         */
    int64_t  chains;
    int64_t  steps;         /* #Iterations                                */
    double   mu;            /* cooling factor, 0.88               */
    int32_t  pert;          /* perturbation size, 4        */
    int32_t  move;          /* OR_MOVE_*                                  */
    uint64_t seed;
    uint64_t chain_offset;  /* global id of local chain 0                 */
    /* Initial sequences ("the initial job sequences are copied to the GPU"): NULL = the
     * chain's own random sequence (R13); else chain c = g - chain_offset starts from
     * init + c * init_ld (init_ld = 0: every chain from the same sequence). */
    const int16_t *init;
    int64_t  init_ld;
} or_sa_params;

/* The neighbour move of SA step k of chain g: Pert distinct positions q[0..P-1] (ascending),
 * sigma = FY permutation of the P slots (slot i receives the old job of slot sigma[i]), u = rand(0,1).
 * INSERT: q = (from, to) in draw order, sigma = identity.  WINDOW: q consecutive. */
int32_t or_sa_move(int32_t n, int32_t pert, int32_t move, uint64_t seed, uint64_t g, uint64_t k,
                   int32_t q[4], int32_t sigma[4], double *u);
/* Alg. 1 line 5: s_new = Neighbour(s) for the move drawn by or_sa_move. */
void or_sa_neighbour(int32_t n, int32_t move, int32_t P, const int32_t q[4], const int32_t sigma[4],
                     const int16_t *s, int16_t *s_new);
/* T0 = population standard deviation of the fitness of `samples` random sequences. */
double  or_t0(const or_instance *I, int32_t problem, uint64_t seed, int64_t samples);
/* One chain. Returns E_best; best_J (n) = best sequence; final_E/final_J optional; trace optional:
 * trace[k] = (E_new << 1) | accepted for k = 0..steps-1. */
int64_t or_sa_chain(const or_instance *I, const or_sa_params *p, double T0, uint64_t g,
                    int16_t *best_J, int64_t *final_E, int16_t *final_J, int64_t *trace);
/* All chains; the reduction returns min (E_best, g) lexicographically. */
void    or_sa_run(const or_instance *I, const or_sa_params *p, double T0, int64_t *best_E,
                  uint64_t *best_g, int16_t *best_J, int64_t *chain_best);

/* Synchronous SA (Fig. 8; reading R18).  Every chain starts from its own random
 * state (the SA_INIT sequence of its global id).  Temperature level j = 0..levels-1: every chain
 * runs a Markov chain of p->steps (= M) moves at the constant temperature T_j (T_0 = T0,
 * T_{j+1} = T_j * mu); move m of level j uses the counters of step k = j*M + m.  The final state of
 * minimal cost over all chains (ties: lowest global id) is s^min_j, the initial state of every chain
 * at level j+1.  Outputs: best-ever penalty / chain / level / sequence (the minimum of (E_best, g)
 * over all levels and chains; an exact tie keeps the earlier level), level_min_E[j] =
 * E(s^min_j) and level_min_g[j] (either may be NULL). */
void or_sa_sync(const or_instance *I, const or_sa_params *p, double T0, int64_t levels,
                int64_t *best_E, uint64_t *best_g, int64_t *best_level, int16_t *best_J,
                int64_t *level_min_E, uint64_t *level_min_g);

/* ---- Discrete PSO (Alg. 2; update eq. (3)) --------------------------- */
typedef struct {
    int32_t  problem;
    int64_t  particles;       /* swarm size                                   */
    int64_t  iters;           /* #Iterations                                  */
    double   w, c1, c2;       /* operator probabilities (silent in the paper) */
    uint64_t seed;
} or_dpso_params;
void or_dpso_f1(int32_t n, const int16_t *p, uint32_t w1, uint32_t w2, int16_t *out);
void or_dpso_f2(int32_t n, const int16_t *lam, const int16_t *pb, uint32_t wcut, int16_t *out);
void or_dpso_f3(int32_t n, const int16_t *delta, const int16_t *g, uint32_t w1, uint32_t w2,
                int16_t *out);
/* Runs the whole swarm; returns the final gbest (value, particle id, sequence).  Optional
 * gbest_trace[t] = gbest value found at line 5 of iteration t. */
void or_dpso_run(const or_instance *I, const or_dpso_params *p, int64_t *best_E, uint64_t *best_id,
                 int16_t *best_J, int64_t *gbest_trace);

#ifdef __cplusplus
}
#endif
#endif
