// internal.h -- host/device shared declarations of libcdd (not part of the public ABI).
#pragma once
#include <cuda_runtime.h>

#include <cstddef>
#include <cstdint>
#include <cstdlib>
#include <vector>

namespace cdd {

// Packed 32-bit job record.  CDD: p | a << sa | b << sb (b is the top field).  UCDDCP:
// a | b << sb | M << sm | X << sx | gamma << sg (gamma top).  Field widths are sized so that
// the sum of 32 records (one lane's chunk) never carries out of the p, a, b fields, which lets a
// single integer add form the prefix sums of all three at once.
struct RecLayout {
    int32_t sa, sb, sm, sx, sg;
    uint32_t pmask, amask, bmask, mmask, xmask;
};

constexpr uint32_t kTagSaInit = 0x11u, kTagSa = 0x12u, kTagT0 = 0x13u, kTagDpsoInit = 0x21u,
                   kTagDpso = 0x22u;

// Fused DPSO swarm-best exchange over peer memory (dpso_peer_*): every rank owns one region,
// exported by CUDA IPC and mapped by every other rank (NVLink / NVSwitch P2P between GPUs).
// Region layout: u64 key[3] (MIN slots, rank 0's are the global ones), u32 arrivals (rank 0's
// counts the ranks through every exchange), then int16 perm[2][np] (this rank's swarm best per
// iteration parity, read by the others when this rank owns the global best).
constexpr size_t kPeerKeyOff = 0, kPeerArriveOff = 24, kPeerPermOff = 64;
struct DpsoPeer {
    int world = 0, rank = 0, np = 0;
    uint8_t* region = nullptr;       // own region (cudaMalloc)
    std::vector<uint8_t*> mapped;    // peers' regions opened in this process (own slot: nullptr)
    uint8_t** d_regions = nullptr;   // device [world]: region of every rank (own included)
    bool open = false;
    bool armed = false;  // dpso_peer_reset since the last fused run (host-side call-order check)
};

struct Instance {
    int device = 0;
    int32_t n = 0;
    int64_t d = 0;
    int64_t sum_p = 0;
    int32_t d_eff = 0;  // min(d, sum p): CDD penalties do not depend on d beyond sum p
    bool has_ucd = false;
    RecLayout lay_cdd{}, lay_ucd{};
    uint32_t* rec_cdd = nullptr;  // device [n] records by job id
    uint32_t* rec_ucd = nullptr;
    // warp-per-chain (SA / T0 / DPSO) tables by job id: ab = alpha | beta << 16, p (u8);
    // UCDDCP: m = M (u8), x = P - M (u8), g = gamma (u16)
    uint32_t* tab_ab = nullptr;
    uint16_t* tab_ab16 = nullptr;  // alpha | beta << 8 (only when both <= 255: ab16_ok)
    bool ab16_ok = false;
    bool ab85_ok = false;  // max(alpha, beta) <= 85: the CDD evaluator's quad pass (sa_group.cuh)
    bool s85_ok = false;   // also max(alpha + beta) <= 85: quad pass of the boundary row's level 1
    // alpha, beta <= 15 and pmax * max(alpha, beta) * 120 < 2^16: the SA nibble layout with
    // sub-block summaries (sa_nib.cuh) for n in (512, 1024]
    bool nib_ok = false;
    // quad level of the group evaluators: 0 pairs, 1 quad pass, 2 also the quad boundary level 1
    // (CDD_SA_NO_QUAD / CDD_SA_NO_QUAD2 cap it for experiments)
    int quad_level() const {
        if (!ab85_ok || std::getenv("CDD_SA_NO_QUAD")) return 0;
        return (s85_ok && !std::getenv("CDD_SA_NO_QUAD2")) ? 2 : 1;
    }
    uint32_t smem_base = 1024;  // shared-window address of dynamic shared memory (probed at create)
    uint8_t* tab_p = nullptr;
    uint8_t* tab_m = nullptr;
    uint8_t* tab_x = nullptr;
    uint16_t* tab_g = nullptr;
    // generic ("wide") path (wide.cu): instances outside the packed record ranges
    bool wide = false;      // the CDD uses the generic kernels
    bool ucd_wide = false;  // the UCDDCP uses the generic kernels (its packed record does not fit)
    int64_t penalty_bound = 0;  // (sum a + sum b) * sum p + sum gamma * sum (P - M) (< 2^62)
    int4* tab_w0 = nullptr;  // {P, alpha, beta, gamma} by job id
    int2* tab_w1 = nullptr;  // {M, P - M} by job id (UCDDCP)
    long long* best_wide = nullptr;  // device {penalty, global id} of the last run (wide instances)
    int* err = nullptr;                    // device data-error flag
    unsigned long long* best_key = nullptr;  // device packed (penalty << 32 | id)
    int16_t* best_perm = nullptr;          // device [n]
    bool has_best = false;
    DpsoPeer* peer = nullptr;  // dpso_peer_create / open
    // host e2e staging
    int16_t* stage_perm = nullptr;
    int64_t* stage_out = nullptr;
    size_t stage_rows = 0;
};

// Resident CTAs per SM of `kern` with `threads` threads and `smem` dynamic shared memory (the
// dynamic-smem attribute is raised to `smem` first), and the device's SM count; memoised per
// (kernel, device, threads, smem) -- the runtime queries cost more host time than a launch.
void resident_ctas(const void* kern, int device, int threads, size_t smem, int* sms, int* occ);

// ---- launchers (eval.cu) ----
cudaError_t launch_eval_batch(const Instance& I, bool ucd, const int16_t* perms, int64_t ld,
                              int64_t batch, int64_t* out, cudaStream_t s);

// ---- launchers (eval2.cu): CDD, several sequences per warp; cudaErrorNotSupported if the
// layout does not apply (alpha or beta > 255, ld % 8 != 0, rows not 16-byte aligned)
cudaError_t launch_eval2_cdd(const Instance& I, const int16_t* perms, int64_t ld, int64_t batch,
                             int64_t* out, cudaStream_t s);
cudaError_t launch_eval2_ucddcp(const Instance& I, const int16_t* perms, int64_t ld, int64_t batch,
                                int64_t* out, cudaStream_t s);
cudaError_t probe_smem_base(uint32_t* base);

// ---- launchers (schedule.cu) ----
cudaError_t launch_schedule(const Instance& I, bool ucd, const int16_t* perms, int64_t ld,
                            int64_t batch, int64_t* C, int32_t* X, int64_t* start, int64_t* pen,
                            cudaStream_t s);

// ---- launchers (sa.cu) ----
struct SaLaunch {
    bool ucd;
    int64_t chains, steps;
    double mu;
    double T0;  // <= 0: computed into workspace
    int64_t t0_samples;
    int32_t pert, move;
    uint64_t seed, chain_offset;
    int64_t *trace, *chain_best, *chain_final;
    double* T0_out;
    const double* T0_in;
    int32_t lanes;  // 0 automatic, 32 warp per chain, 4 / 8 / 16 group kernel
    const int16_t* init = nullptr;  // caller's initial sequences (chain c: init + c * init_ld)
    int64_t init_ld = 0;
    bool peer = false;  // synchronous SA: s^min exchanged through Instance::peer in the finalisation
};
size_t sa_workspace_bytes(const Instance& I, const SaLaunch& p);
cudaError_t launch_t0(const Instance& I, bool ucd, uint64_t seed, int64_t samples, double* T0_dev,
                      void* ws, cudaStream_t s);
cudaError_t launch_sa(Instance& I, const SaLaunch& p, void* ws, cudaStream_t s);
void sa_layout(const Instance& I, const SaLaunch& p, int32_t* lanes, int32_t* per_lane);
// synchronous SA (p.steps = Markov-chain length M); 0 bytes if the instance has no 16-bit records
size_t sa_sync_workspace_bytes(const Instance& I, const SaLaunch& p);
cudaError_t launch_sa_sync_level(Instance& I, const SaLaunch& p, int64_t j, int64_t* level_min,
                                 void* ws, cudaStream_t s);
void sa_sync_ptrs(const Instance& I, const SaLaunch& p, void* ws, unsigned long long** key,
                  int16_t** perm);

// ---- launchers (dpso.cu) ----
struct DpsoLaunch {
    bool ucd;
    int64_t particles, iters;
    double w, c1, c2;
    uint64_t seed, particle_offset;
    int64_t* gbest_trace;
    bool peer = false;  // exchange the swarm best through Instance::peer inside the kernels
};
size_t dpso_peer_region_bytes(int n);
int dpso_np(int n);  // row stride of the DPSO workspace and of the peer regions
// workspace of a DPSO run (dpso.cu dp_layout), shared by both kernel layouts
struct DpsoWsPtrs {
    int16_t *pos, *inv, *pb;
    int32_t* zb;
    unsigned long long* gkey;
    int16_t* gperm;
    unsigned int* counter;
    int16_t* slots;  // [2][kDpsoMaxCtas or fewer][np]: each CTA's best personal-best row (group publish)
    int np;
};
constexpr int kDpsoMaxCtas = 8192;
// group-layout DPSO (dpso_group.cu): 8 lanes per particle; needs the 16-bit records (ab16_ok)
bool dpsog_usable(const Instance& I);
cudaError_t dpsog_begin(Instance& I, const DpsoLaunch& p, const DpsoWsPtrs& w, cudaStream_t s);
cudaError_t dpsog_iterate(Instance& I, const DpsoLaunch& p, const DpsoWsPtrs& w, int64_t t0, int64_t t1,
                          cudaStream_t s);
size_t dpso_workspace_bytes(const Instance& I, const DpsoLaunch& p);
cudaError_t dpso_begin(Instance& I, const DpsoLaunch& p, void* ws, cudaStream_t s);
// iterations t0..t1-1 of Alg. 2 (one kernel launch each)
cudaError_t dpso_iterate(Instance& I, const DpsoLaunch& p, void* ws, int64_t t0, int64_t t1,
                         cudaStream_t s);
void dpso_gbest(const Instance& I, const DpsoLaunch& p, void* ws, int64_t t, int64_t** key,
                int16_t** perm);
cudaError_t dpso_end(Instance& I, const DpsoLaunch& p, void* ws, cudaStream_t s);

// ---- launchers (wide.cu): the generic path (int64, n <= 32767, no packing)
cudaError_t launch_wide_eval(const Instance& I, bool ucd, const int16_t* perms, int64_t ld, int64_t batch,
                             int64_t* out, cudaStream_t s);
cudaError_t launch_wide_schedule(const Instance& I, bool ucd, const int16_t* perms, int64_t ld, int64_t batch,
                                 int64_t* C, int32_t* X, int64_t* start, int64_t* pen, cudaStream_t s);
size_t wide_sa_workspace_bytes(const Instance& I, const SaLaunch& p);
cudaError_t launch_wide_t0(const Instance& I, bool ucd, uint64_t seed, int64_t samples, double* T0_dev, void* ws,
                           cudaStream_t s);
cudaError_t launch_wide_sa(Instance& I, const SaLaunch& p, void* ws, cudaStream_t s);

int sa_e_for_n(int n);  // elements per lane of the warp-per-chain kernels

// ---- group-kernel SA variants (sag_*.cu: one translation unit per problem / trace / move class)
struct GroupCfg {
    int G, E;  // G = 0: warp-per-chain kernel
};
#define CDD_SAG_DECL(NAME)                                                                      \
    size_t NAME##_ws(const Instance& I, const SaLaunch& p, GroupCfg cfg);                      \
    cudaError_t NAME##_run(Instance& I, const SaLaunch& p, GroupCfg cfg, void* ws, cudaStream_t s);
#define CDD_SAG_SYNC_DECL(NAME)                                                                 \
    size_t NAME##_sync_ws(const Instance& I, const SaLaunch& p, GroupCfg cfg);                 \
    cudaError_t NAME##_sync_level(Instance& I, const SaLaunch& p, GroupCfg cfg, int64_t j,     \
                                  int64_t* level_min, void* ws, cudaStream_t s);               \
    void NAME##_sync_ptrs(const Instance& I, const SaLaunch& p, GroupCfg cfg, void* ws,        \
                          unsigned long long** key, int16_t** perm);
CDD_SAG_DECL(sag_cdd)
CDD_SAG_DECL(sag_cdd_tr)
CDD_SAG_DECL(sag_cdd_nib)
CDD_SAG_SYNC_DECL(sag_cdd_nib)
CDD_SAG_DECL(sag_cdd_nib_tr)
CDD_SAG_DECL(sag_ucd)
CDD_SAG_DECL(sag_ucd_tr)
CDD_SAG_DECL(sag_cdd_ins)
CDD_SAG_DECL(sag_cdd_ins_tr)
CDD_SAG_DECL(sag_ucd_ins)
CDD_SAG_DECL(sag_ucd_ins_tr)
CDD_SAG_SYNC_DECL(sag_cdd)
CDD_SAG_SYNC_DECL(sag_ucd)
CDD_SAG_SYNC_DECL(sag_cdd_ins)
CDD_SAG_SYNC_DECL(sag_ucd_ins)
cudaError_t sag_cdd_t0(const Instance& I, GroupCfg cfg, uint64_t seed, int64_t samples, double* T0_dev,
                       void* ws, cudaStream_t s);
cudaError_t sag_ucd_t0(const Instance& I, GroupCfg cfg, uint64_t seed, int64_t samples, double* T0_dev,
                       void* ws, cudaStream_t s);

}  // namespace cdd
