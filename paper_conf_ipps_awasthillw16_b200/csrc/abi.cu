// abi.cu -- the C-ABI of libcdd (include/cdd.h): argument checks, instance management, packed
// record construction, and the launch of the kernels in eval.cu / sa.cu / dpso.cu.
#include <cuda_runtime.h>

#include <algorithm>
#include <map>
#include <mutex>
#include <tuple>
#include <climits>
#include <cmath>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/cdd.h"
#include "internal.h"

using cdd::Instance;

struct cdd_instance : Instance {};

namespace cdd {
void resident_ctas(const void* kern, int device, int threads, size_t smem, int* sms, int* occ) {
    static std::mutex mu;
    static std::map<std::tuple<const void*, int, int, size_t>, std::pair<int, int>> memo;
    const auto key = std::make_tuple(kern, device, threads, smem);
    {
        std::lock_guard<std::mutex> lk(mu);
        const auto it = memo.find(key);
        if (it != memo.end()) {
            *sms = it->second.first;
            *occ = it->second.second;
            return;
        }
    }
    int s = 148, o = 1;
    cudaDeviceGetAttribute(&s, cudaDevAttrMultiProcessorCount, device);
    {
        // the dynamic-smem attribute only ever grows: a launch shape memoised earlier must stay valid
        static std::map<std::pair<const void*, int>, size_t> attr;
        std::lock_guard<std::mutex> lk(mu);
        size_t& cur = attr[std::make_pair(kern, device)];
        if (smem > cur) {
            cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            cur = smem;
        }
    }
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, kern, threads, smem);
    if (o < 1) o = 1;
    *sms = s;
    *occ = o;
    std::lock_guard<std::mutex> lk(mu);
    memo[key] = {s, o};
}
}  // namespace cdd

namespace {

thread_local std::string g_err;

int fail(int code, const std::string& msg) {
    g_err = msg;
    return code;
}

int cuda_fail(cudaError_t e, const char* where) {
    g_err = std::string(where) + ": " + cudaGetErrorString(e);
    return CDD_ECUDA;
}

struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int d) {
        cudaGetDevice(&prev);
        if (prev != d) cudaSetDevice(d);
    }
    ~DeviceGuard() {
        int cur = -1;
        cudaGetDevice(&cur);
        if (prev >= 0 && cur != prev) cudaSetDevice(prev);
    }
};

int bits_for(uint64_t v) {
    int b = 0;
    while (v) {
        ++b;
        v >>= 1;
    }
    return b < 1 ? 1 : b;
}

uint32_t mask_of(int w) { return w >= 32 ? 0xffffffffu : ((1u << w) - 1u); }

cudaStream_t as_stream(void* s) { return reinterpret_cast<cudaStream_t>(s); }

void free_instance(cdd_instance* I) {
    if (!I) return;
    DeviceGuard g(I->device);
    cudaFree(I->rec_cdd);
    cudaFree(I->rec_ucd);
    cudaFree(I->tab_ab);
    cudaFree(I->tab_ab16);
    cudaFree(I->tab_p);
    cudaFree(I->tab_m);
    cudaFree(I->tab_x);
    cudaFree(I->tab_g);
    cudaFree(I->tab_w0);
    cudaFree(I->tab_w1);
    cudaFree(I->best_wide);
    cudaFree(I->err);
    cudaFree(I->best_key);
    cudaFree(I->best_perm);
    cudaFree(I->stage_perm);
    cudaFree(I->stage_out);
    if (I->peer) {
        for (uint8_t* m : I->peer->mapped)
            if (m) cudaIpcCloseMemHandle(m);
        cudaFree(I->peer->d_regions);
        cudaFree(I->peer->region);
        delete I->peer;
    }
    delete I;
}

}  // namespace

extern "C" {

const char* cdd_last_error(void) { return g_err.c_str(); }
int cdd_abi_version(void) { return CDD_ABI_VERSION; }



// The generic path (wide.cu): every array as plain int32 fields by job id, int64 arithmetic.
static int create_wide(cdd_instance* I, int32_t n, const int32_t* p, const int32_t* alpha,
                       const int32_t* beta, const int32_t* m, const int32_t* gamma) {
    std::vector<int4> w0(n);
    std::vector<int2> w1(m ? n : 0);
    for (int i = 0; i < n; ++i) {
        w0[i] = make_int4(p[i], alpha[i], beta[i], gamma ? gamma[i] : 0);
        if (m) w1[i] = make_int2(m[i], p[i] - m[i]);
    }
    cudaError_t e = cudaMalloc(&I->tab_w0, sizeof(int4) * n);
    if (e == cudaSuccess && m) e = cudaMalloc(&I->tab_w1, sizeof(int2) * n);
    if (e == cudaSuccess) e = cudaMalloc(&I->best_wide, 2 * sizeof(long long));
    if (e == cudaSuccess) e = cudaMemcpy(I->tab_w0, w0.data(), sizeof(int4) * n, cudaMemcpyHostToDevice);
    if (e == cudaSuccess && m) e = cudaMemcpy(I->tab_w1, w1.data(), sizeof(int2) * n, cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = cudaMemset(I->best_wide, 0xff, 2 * sizeof(long long));
    return e == cudaSuccess ? CDD_OK : cuda_fail(e, "cdd_instance_create (generic path)");
}

int cdd_instance_create(int32_t n, const int32_t* p, const int32_t* alpha, const int32_t* beta,
                        const int32_t* m, const int32_t* gamma, int64_t d, int device,
                        cdd_instance** out) {
    if (!out) return fail(CDD_EINVAL, "out is NULL");
    *out = nullptr;
    if (n < 1 || n > 32767) return fail(CDD_EINVAL, "n must be in [1, 32767] (int16 job ids)");
    if (!p || !alpha || !beta) return fail(CDD_EINVAL, "p, alpha, beta must be non-NULL");
    if ((m == nullptr) != (gamma == nullptr)) return fail(CDD_EINVAL, "m and gamma must both be given or both NULL");
    if (d < 0) return fail(CDD_EINVAL, "d must be >= 0");
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev)
        return fail(CDD_EINVAL, "invalid CUDA device");
    int64_t sp = 0, sa = 0, sb = 0, sg = 0, sx = 0;
    int32_t pmax = 0, amax = 0, bmax = 0, mmax = 0, xmax = 0, gmax = 0;
    int64_t smax = 0;  // max(alpha_i + beta_i)
    for (int i = 0; i < n; ++i) {
        if (p[i] < 1) return fail(CDD_EINVAL, "p_i must be >= 1");
        if (alpha[i] < 0 || beta[i] < 0) return fail(CDD_EINVAL, "alpha_i, beta_i must be >= 0");
        sp += p[i];
        sa += alpha[i];
        sb += beta[i];
        pmax = std::max(pmax, p[i]);
        amax = std::max(amax, alpha[i]);
        bmax = std::max(bmax, beta[i]);
        smax = std::max(smax, (int64_t)alpha[i] + beta[i]);
        if (m) {
            if (m[i] < 0 || m[i] > p[i]) return fail(CDD_EINVAL, "need 0 <= m_i <= p_i");
            if (gamma[i] < 0) return fail(CDD_EINVAL, "gamma_i must be >= 0");
            mmax = std::max(mmax, m[i]);
            xmax = std::max(xmax, p[i] - m[i]);
            gmax = std::max(gmax, gamma[i]);
            sg += gamma[i];
            sx += p[i] - m[i];
        }
    }
    // every penalty of eq. (1) / (2) is at most (sum a + sum b) * sum p (+ sum gamma * sum (p - m));
    // the outputs are exact int64 below 2^62 (the SA trace packs (E << 1) | accepted)
    const unsigned __int128 bound = (unsigned __int128)(sa + sb) * (unsigned __int128)sp +
                                    (unsigned __int128)sg * (unsigned __int128)sx;
    if (bound >= ((unsigned __int128)1 << 62))
        return fail(CDD_ERANGE, "penalties could reach 2^62: (sum alpha + sum beta) * sum p + sum gamma * sum (p - m) must be < 2^62");
    // fast path: packed records (CDD: p | a | b fields wide enough for 32-record lane sums; SA tables:
    // p, M, P-M bytes, alpha, beta, gamma 16-bit halves) and int32 penalties
    const int wp = bits_for(32ull * (uint64_t)pmax), wa = bits_for(32ull * (uint64_t)amax),
              wb = bits_for(32ull * (uint64_t)bmax);
    const bool packed = n <= 1024 && sa < 65536 && sb < 65536 && (sa + sb) * sp < (int64_t)INT32_MAX &&
                        wp + wa + wb <= 32 && pmax <= 255 && 32 * amax < 65536 && 32 * bmax < 65536;
    int ua = 0, ub = 0, um = 0, ux = 0, ug = 0;
    bool ucd_packed = false;
    if (m) {
        ua = bits_for(32ull * (uint64_t)amax);
        ub = bits_for(32ull * (uint64_t)bmax);
        um = bits_for((uint64_t)mmax);
        ux = bits_for((uint64_t)xmax);
        ug = bits_for((uint64_t)gmax);
        ucd_packed = packed && gmax < 65536 && xmax <= 255 && ua + ub + um + ux + ug <= 32;
    }
    auto* I = new cdd_instance();
    I->device = device;
    I->n = n;
    I->d = d;
    I->sum_p = sp;
    I->d_eff = (int32_t)std::min<int64_t>(d, sp);
    I->penalty_bound = (int64_t)bound;
    DeviceGuard g(device);
    cudaError_t e = cudaSuccess;
    auto chk = [&](cudaError_t x) {
        if (e == cudaSuccess) e = x;
    };
    chk(cudaMalloc(&I->err, sizeof(int)));
    chk(cudaMalloc(&I->best_key, sizeof(unsigned long long)));
    chk(cudaMalloc(&I->best_perm, sizeof(int16_t) * n));
    if (e == cudaSuccess) {
        chk(cudaMemset(I->err, 0, sizeof(int)));
        chk(cudaMemset(I->best_key, 0xff, sizeof(unsigned long long)));
        chk(cudaMemset(I->best_perm, 0, sizeof(int16_t) * n));
    }
    if (e != cudaSuccess) {
        free_instance(I);
        return cuda_fail(e, "cdd_instance_create");
    }
    // the generic tables serve the CDD when the packed records do not fit, the UCDDCP when its own
    // packed record does not (the CDD side of such an instance stays on the fast path)
    I->has_ucd = m != nullptr;
    I->wide = !packed;
    I->ucd_wide = m != nullptr && !ucd_packed;
    if (I->wide || I->ucd_wide) {
        const int rc = create_wide(I, n, p, alpha, beta, m, gamma);
        if (rc != CDD_OK) {
            free_instance(I);
            return rc;
        }
    }
    if (!packed) {
        *out = I;
        return CDD_OK;
    }
    I->lay_cdd.sa = wp;
    I->lay_cdd.sb = wp + wa;
    I->lay_cdd.pmask = mask_of(wp);
    I->lay_cdd.amask = mask_of(wa);
    I->lay_cdd.bmask = mask_of(32 - wp - wa);
    std::vector<uint32_t> rc(n), ru;
    for (int i = 0; i < n; ++i)
        rc[i] = (uint32_t)p[i] | ((uint32_t)alpha[i] << I->lay_cdd.sa) | ((uint32_t)beta[i] << I->lay_cdd.sb);
    if (ucd_packed) {
        auto& L = I->lay_ucd;
        L.amask = mask_of(ua);
        L.sb = ua;
        L.bmask = mask_of(ub);
        L.sm = ua + ub;
        L.mmask = mask_of(um);
        L.sx = L.sm + um;
        L.xmask = mask_of(ux);
        L.sg = L.sx + ux;
        ru.resize(n);
        for (int i = 0; i < n; ++i)
            ru[i] = (uint32_t)alpha[i] | ((uint32_t)beta[i] << L.sb) | ((uint32_t)m[i] << L.sm) |
                    ((uint32_t)(p[i] - m[i]) << L.sx) | ((uint32_t)gamma[i] << L.sg);
    }
    chk(cudaMalloc(&I->rec_cdd, sizeof(uint32_t) * n));
    if (ucd_packed) chk(cudaMalloc(&I->rec_ucd, sizeof(uint32_t) * n));
    std::vector<uint32_t> tab(n);
    std::vector<uint8_t> tp(n), tm(n), tx(n);
    std::vector<uint16_t> tg(n);
    for (int i = 0; i < n; ++i) {
        tab[i] = (uint32_t)alpha[i] | ((uint32_t)beta[i] << 16);
        tp[i] = (uint8_t)p[i];
        if (ucd_packed) {
            tm[i] = (uint8_t)m[i];
            tx[i] = (uint8_t)(p[i] - m[i]);
            tg[i] = (uint16_t)gamma[i];
        }
    }
    chk(cudaMalloc(&I->tab_ab, sizeof(uint32_t) * n));
    chk(cudaMalloc(&I->tab_p, n));
    I->ab16_ok = amax <= 255 && bmax <= 255;
    I->ab85_ok = amax <= 85 && bmax <= 85;
    I->s85_ok = I->ab85_ok && smax <= 85;
    I->nib_ok = amax <= 15 && bmax <= 15 && (int64_t)pmax * std::max(amax, bmax) * 120 < 65536;
    std::vector<uint16_t> tab16(n);
    for (int i = 0; i < n; ++i) tab16[i] = (uint16_t)((alpha[i] & 0xff) | ((beta[i] & 0xff) << 8));
    chk(cudaMalloc(&I->tab_ab16, sizeof(uint16_t) * n));
    if (e == cudaSuccess)
        chk(cudaMemcpy(I->tab_ab16, tab16.data(), sizeof(uint16_t) * n, cudaMemcpyHostToDevice));
    if (ucd_packed) {
        chk(cudaMalloc(&I->tab_m, n));
        chk(cudaMalloc(&I->tab_x, n));
        chk(cudaMalloc(&I->tab_g, sizeof(uint16_t) * n));
    }
    if (e == cudaSuccess) {
        chk(cudaMemcpy(I->tab_ab, tab.data(), sizeof(uint32_t) * n, cudaMemcpyHostToDevice));
        chk(cudaMemcpy(I->tab_p, tp.data(), n, cudaMemcpyHostToDevice));
        if (ucd_packed) {
            chk(cudaMemcpy(I->tab_m, tm.data(), n, cudaMemcpyHostToDevice));
            chk(cudaMemcpy(I->tab_x, tx.data(), n, cudaMemcpyHostToDevice));
            chk(cudaMemcpy(I->tab_g, tg.data(), sizeof(uint16_t) * n, cudaMemcpyHostToDevice));
        }
    }
    if (e == cudaSuccess) {
        chk(cudaMemcpy(I->rec_cdd, rc.data(), sizeof(uint32_t) * n, cudaMemcpyHostToDevice));
        if (ucd_packed) chk(cudaMemcpy(I->rec_ucd, ru.data(), sizeof(uint32_t) * n, cudaMemcpyHostToDevice));
        chk(cdd::probe_smem_base(&I->smem_base));
    }
    if (e != cudaSuccess) {
        free_instance(I);
        return cuda_fail(e, "cdd_instance_create");
    }
    *out = I;
    return CDD_OK;
}

int cdd_instance_destroy(cdd_instance* inst) {
    if (!inst) return fail(CDD_EINVAL, "instance is NULL");
    free_instance(inst);
    return CDD_OK;
}

int cdd_instance_query(const cdd_instance* I, int32_t* n, int64_t* d, int64_t* sum_p, int32_t* flags) {
    if (!I) return fail(CDD_EINVAL, "instance is NULL");
    if (n) *n = I->n;
    if (d) *d = I->d;
    if (sum_p) *sum_p = I->sum_p;
    if (flags) *flags = (I->has_ucd ? 1 : 0) | (I->d >= I->sum_p ? 2 : 0) | (I->wide ? 4 : 0) | (I->ucd_wide ? 8 : 0) |
                          (I->nib_ok && !I->wide ? 16 : 0);
    return CDD_OK;
}

static int check_batch_args(const cdd_instance* I, const int16_t* perms, int64_t ld, int64_t batch,
                            const int64_t* out) {
    if (!I) return fail(CDD_EINVAL, "instance is NULL");
    if (batch < 0) return fail(CDD_EINVAL, "batch must be >= 0");
    if (batch > 0 && (!perms || !out)) return fail(CDD_EINVAL, "perms/out must be non-NULL");
    if (ld < I->n) return fail(CDD_EINVAL, "ld must be >= n");
    return CDD_OK;
}

// fast (packed) or generic (wide) evaluator
// the generic kernels serve this problem on this instance
static bool generic(const cdd_instance& I, bool ucd) { return ucd ? I.ucd_wide : I.wide; }

static cudaError_t any_eval(const cdd_instance& I, bool ucd, const int16_t* perms, int64_t ld, int64_t batch,
                            int64_t* out, cudaStream_t s) {
    return generic(I, ucd) ? cdd::launch_wide_eval(I, ucd, perms, ld, batch, out, s)
                           : cdd::launch_eval_batch(I, ucd, perms, ld, batch, out, s);
}

static int eval_common(cdd_instance* I, bool ucd, const int16_t* perms, int64_t ld, int64_t batch,
                       int64_t* out, void* stream) {
    int rc = check_batch_args(I, perms, ld, batch, out);
    if (rc != CDD_OK) return rc;
    if (ucd && !I->has_ucd) return fail(CDD_EINVAL, "instance has no UCDDCP data (m/gamma not given)");
    if (ucd && I->d < I->sum_p) return fail(CDD_EINVAL, "UCDDCP needs d >= sum p (unrestricted case, P:126)");
    DeviceGuard g(I->device);
    cudaError_t e = any_eval(*I, ucd, perms, ld, batch, out, as_stream(stream));
    return e == cudaSuccess ? CDD_OK : cuda_fail(e, ucd ? "ucddcp_eval_batch" : "cdd_eval_batch");
}

int cdd_eval_batch(cdd_instance* I, const int16_t* perms, int64_t ld, int64_t batch, int64_t* out,
                   void* stream) {
    return eval_common(I, false, perms, ld, batch, out, stream);
}

int ucddcp_eval_batch(cdd_instance* I, const int16_t* perms, int64_t ld, int64_t batch, int64_t* out,
                      void* stream) {
    return eval_common(I, true, perms, ld, batch, out, stream);
}

int cdd_schedule_batch(cdd_instance* I, cdd_problem problem, const int16_t* perms, int64_t ld,
                       int64_t batch, int64_t* C, int32_t* X, int64_t* start, int64_t* penalty,
                       void* stream) {
    int rc = check_batch_args(I, perms, ld, batch, penalty);
    if (rc != CDD_OK) return rc;
    if (problem != CDD_PROBLEM_CDD && problem != CDD_PROBLEM_UCDDCP) return fail(CDD_EINVAL, "bad problem");
    const bool ucd = problem == CDD_PROBLEM_UCDDCP;
    if (batch > 0 && (!C || !start || (ucd && !X))) return fail(CDD_EINVAL, "C/start (and X for UCDDCP) must be non-NULL");
    if (ucd && (!I->has_ucd || I->d < I->sum_p)) return fail(CDD_EINVAL, "instance not usable for UCDDCP (no m/gamma, or d < sum p)");
    DeviceGuard g(I->device);
    cudaError_t e = generic(*I, ucd) ? cdd::launch_wide_schedule(*I, ucd, perms, ld, batch, C, X, start, penalty, as_stream(stream))
                            : cdd::launch_schedule(*I, ucd, perms, ld, batch, C, X, start, penalty, as_stream(stream));
    return e == cudaSuccess ? CDD_OK : cuda_fail(e, "cdd_schedule_batch");
}

int cdd_eval_batch_host(cdd_instance* I, cdd_problem problem, const int16_t* perms_host, int64_t ld,
                        int64_t batch, int64_t* out_host, void* stream) {
    int rc = check_batch_args(I, perms_host, ld, batch, out_host);
    if (rc != CDD_OK) return rc;
    if (problem != CDD_PROBLEM_CDD && problem != CDD_PROBLEM_UCDDCP) return fail(CDD_EINVAL, "bad problem");
    const bool ucd = problem == CDD_PROBLEM_UCDDCP;
    if (ucd && (!I->has_ucd || I->d < I->sum_p)) return fail(CDD_EINVAL, "instance not usable for UCDDCP (no m/gamma, or d < sum p)");
    DeviceGuard g(I->device);
    cudaStream_t s = as_stream(stream);
    const int64_t chunk = std::max<int64_t>(1, std::min<int64_t>(batch, (int64_t)(256ll << 20) / (ld * 2)));
    if (I->stage_rows < (size_t)chunk * ld) {
        cudaFree(I->stage_perm);
        cudaFree(I->stage_out);
        I->stage_perm = nullptr;
        I->stage_out = nullptr;
        I->stage_rows = 0;
        cudaError_t e = cudaMalloc(&I->stage_perm, sizeof(int16_t) * (size_t)chunk * ld);
        if (e == cudaSuccess) e = cudaMalloc(&I->stage_out, sizeof(int64_t) * (size_t)chunk);
        if (e != cudaSuccess) return cuda_fail(e, "cdd_eval_batch_host staging");
        I->stage_rows = (size_t)chunk * ld;
    }
    for (int64_t a = 0; a < batch; a += chunk) {
        const int64_t rows = std::min(chunk, batch - a);
        cudaError_t e = cudaMemcpyAsync(I->stage_perm, perms_host + a * ld, sizeof(int16_t) * rows * ld,
                                        cudaMemcpyHostToDevice, s);
        if (e == cudaSuccess) e = any_eval(*I, ucd, I->stage_perm, ld, rows, I->stage_out, s);
        if (e == cudaSuccess)
            e = cudaMemcpyAsync(out_host + a, I->stage_out, sizeof(int64_t) * rows, cudaMemcpyDeviceToHost, s);
        if (e != cudaSuccess) return cuda_fail(e, "cdd_eval_batch_host");
    }
    cudaError_t e = cudaStreamSynchronize(s);
    return e == cudaSuccess ? CDD_OK : cuda_fail(e, "cdd_eval_batch_host sync");
}

int cdd_check(cdd_instance* I, void* stream) {
    if (!I) return fail(CDD_EINVAL, "instance is NULL");
    DeviceGuard g(I->device);
    cudaStream_t s = as_stream(stream);
    int flag = 0;
    cudaError_t e = cudaMemcpyAsync(&flag, I->err, sizeof(int), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return cuda_fail(e, "cdd_check");
    if (flag) {
        cudaMemsetAsync(I->err, 0, sizeof(int), s);
        cudaStreamSynchronize(s);
        return fail(CDD_EDATA, (flag & 2) ? "a peer rank never reached a swarm-best exchange (timed out)"
                                          : "a sequence contained a job id outside [0, n)");
    }
    return CDD_OK;
}

static int sa_validate(const cdd_instance* I, const sa_params* p, cdd::SaLaunch* L) {
    if (!I || !p) return fail(CDD_EINVAL, "instance/params is NULL");
    if (p->problem != CDD_PROBLEM_CDD && p->problem != CDD_PROBLEM_UCDDCP) return fail(CDD_EINVAL, "bad problem");
    const bool ucd = p->problem == CDD_PROBLEM_UCDDCP;
    if (ucd && (!I->has_ucd || I->d < I->sum_p)) return fail(CDD_EINVAL, "instance not usable for UCDDCP (no m/gamma, or d < sum p)");
    if (p->chains < 1) return fail(CDD_EINVAL, "chains must be >= 1");
    if (p->steps < 0 || p->steps >= (int64_t)UINT32_MAX) return fail(CDD_EINVAL, "steps must be in [0, 2^32)");
    if (p->chain_offset + (uint64_t)p->chains > (1ull << 32)) return fail(CDD_EINVAL, "chain ids must fit 32 bits");
    if (p->pert < 1 || p->pert > 4) return fail(CDD_EINVAL, "pert must be in [1, 4]");
    if (p->move != CDD_MOVE_PERT_FY && p->move != CDD_MOVE_SWAP && p->move != CDD_MOVE_INSERT &&
        p->move != CDD_MOVE_WINDOW)
        return fail(CDD_EINVAL, "bad move");
    if (!std::isfinite(p->mu) || p->mu < 0) return fail(CDD_EINVAL, "mu must be finite and >= 0");
    if (!(p->T0 > 0) && !p->T0_in && p->t0_samples < 1) return fail(CDD_EINVAL, "T0 <= 0 needs t0_samples >= 1");
    if (std::isnan(p->T0)) return fail(CDD_EINVAL, "T0 is NaN");
    if (p->lanes != 0 && p->lanes != 4 && p->lanes != 8 && p->lanes != 16 && p->lanes != 32)
        return fail(CDD_EINVAL, "lanes must be 0, 4, 8, 16 or 32");
    if (p->lanes >= 4 && p->lanes <= 16 && (!I->ab16_ok || generic(*I, ucd)))
        return fail(CDD_EINVAL, "lanes 4/8/16 need the fast path with alpha, beta <= 255 (16-bit records)");
    if (generic(*I, ucd) && !(p->T0 > 0) && !p->T0_in &&
        (unsigned __int128)p->t0_samples * (unsigned __int128)(uint64_t)I->penalty_bound >= ((unsigned __int128)1 << 65))
        return fail(CDD_EINVAL, "T0 from samples: t0_samples * penalty bound must be < 2^65 (exact 128-bit moments); give T0");
    if (p->lanes == 4 && I->n > 256) return fail(CDD_EINVAL, "lanes = 4 supports n <= 256");
    if (p->init && p->init_ld != 0 && p->init_ld < I->n) return fail(CDD_EINVAL, "init_ld must be 0 or >= n");
    L->ucd = ucd;
    L->lanes = p->lanes;
    L->chains = p->chains;
    L->steps = p->steps;
    L->mu = p->mu;
    L->T0 = p->T0_in ? 1.0 : p->T0;
    L->t0_samples = (p->T0 > 0 || p->T0_in) ? 0 : p->t0_samples;
    L->T0_in = p->T0_in;
    L->pert = p->pert;
    L->move = (int32_t)p->move;
    L->seed = p->seed;
    L->chain_offset = p->chain_offset;
    L->trace = p->trace;
    L->chain_best = p->chain_best;
    L->chain_final = p->chain_final;
    L->T0_out = p->T0_out;
    L->init = p->init;
    L->init_ld = p->init ? p->init_ld : 0;
    return CDD_OK;
}

size_t sa_workspace_size(const cdd_instance* I, const sa_params* p) {
    cdd::SaLaunch L{};
    if (sa_validate(I, p, &L) != CDD_OK) return 0;
    DeviceGuard g(I->device);
    return generic(*I, L.ucd) ? cdd::wide_sa_workspace_bytes(*I, L) : cdd::sa_workspace_bytes(*I, L);
}

static int sync_validate(const cdd_instance* I, const sa_sync_params* q, cdd::SaLaunch* L) {
    if (!I || !q) return fail(CDD_EINVAL, "instance/params is NULL");
    if (q->markov_len < 1 || q->levels < 1) return fail(CDD_EINVAL, "markov_len and levels must be >= 1");
    if ((double)q->markov_len * (double)q->levels >= 4294967296.0)
        return fail(CDD_EINVAL, "levels * markov_len must be < 2^32");
    if (q->lanes != 0 && q->lanes != 4 && q->lanes != 8 && q->lanes != 16)
        return fail(CDD_EINVAL, "synchronous SA runs on lanes 0, 4, 8 or 16");
    if (!I->ab16_ok || generic(*I, q->problem == CDD_PROBLEM_UCDDCP))
        return fail(CDD_EINVAL, "synchronous SA needs the fast path (packed records, alpha, beta <= 255)");
    sa_params p{};
    p.problem = q->problem;
    p.chains = q->chains;
    p.steps = q->markov_len;
    p.mu = q->mu;
    p.T0 = q->T0;
    p.t0_samples = q->t0_samples;
    p.pert = q->pert;
    p.move = q->move;
    p.seed = q->seed;
    p.chain_offset = q->chain_offset;
    p.T0_out = q->T0_out;
    p.T0_in = q->T0_in;
    p.lanes = q->lanes;
    return sa_validate(I, &p, L);
}

size_t sa_sync_workspace_size(const cdd_instance* I, const sa_sync_params* q) {
    cdd::SaLaunch L{};
    if (sync_validate(I, q, &L) != CDD_OK) return 0;
    DeviceGuard g(I->device);
    return cdd::sa_sync_workspace_bytes(*I, L);
}

int sa_sync_level(cdd_instance* I, const sa_sync_params* q, void* ws, size_t ws_bytes, int64_t j,
                  void* stream) {
    cdd::SaLaunch L{};
    const int rc = sync_validate(I, q, &L);
    if (rc != CDD_OK) return rc;
    if (j < 0 || j >= q->levels) return fail(CDD_EINVAL, "level j out of range");
    DeviceGuard g(I->device);
    const size_t need = cdd::sa_sync_workspace_bytes(*I, L);
    if (!ws || ws_bytes < need)
        return fail(CDD_ENOMEM, "workspace too small: need " + std::to_string(need) + " bytes");
    cudaError_t e = cdd::launch_sa_sync_level(*I, L, j, q->level_min, ws, as_stream(stream));
    if (e != cudaSuccess) return cuda_fail(e, "sa_sync_level");
    I->has_best = true;
    return CDD_OK;
}

int sa_sync_run_peer(cdd_instance* I, const sa_sync_params* q, void* ws, size_t ws_bytes, void* stream) {
    cdd::SaLaunch L{};
    const int rc = sync_validate(I, q, &L);
    if (rc != CDD_OK) return rc;
    cdd::DpsoPeer* P = I->peer;
    if (!P || !P->open) return fail(CDD_ESTATE, "peer exchange not open (dpso_peer_create / dpso_peer_open)");
    if (q->chain_offset != (uint64_t)P->rank * (uint64_t)q->chains)
        return fail(CDD_EINVAL, "chain_offset must be rank * chains (equal shares)");
    if (!P->armed) return fail(CDD_ESTATE, "peer exchange not re-armed: dpso_peer_reset (+ a barrier) before every fused run");
    DeviceGuard g(I->device);
    const size_t need = cdd::sa_sync_workspace_bytes(*I, L);
    if (!ws || ws_bytes < need)
        return fail(CDD_ENOMEM, "workspace too small: need " + std::to_string(need) + " bytes");
    L.peer = true;
    P->armed = false;
    for (int64_t j = 0; j < q->levels; ++j) {
        const cudaError_t e = cdd::launch_sa_sync_level(*I, L, j, q->level_min, ws, as_stream(stream));
        if (e != cudaSuccess) return cuda_fail(e, "sa_sync_run_peer");
    }
    I->has_best = true;
    return CDD_OK;
}

int sa_sync_run(cdd_instance* I, const sa_sync_params* q, void* ws, size_t ws_bytes, void* stream) {
    for (int64_t j = 0; q && j < q->levels; ++j) {
        const int rc = sa_sync_level(I, q, ws, ws_bytes, j, stream);
        if (rc != CDD_OK) return rc;
    }
    return q ? CDD_OK : fail(CDD_EINVAL, "params is NULL");
}

int sa_sync_ptrs(const cdd_instance* I, const sa_sync_params* q, void* ws, int64_t** key_dev,
                 int16_t** perm_dev) {
    cdd::SaLaunch L{};
    const int rc = sync_validate(I, q, &L);
    if (rc != CDD_OK) return rc;
    if (!ws) return fail(CDD_EINVAL, "workspace is NULL");
    unsigned long long* k = nullptr;
    int16_t* pp = nullptr;
    cdd::sa_sync_ptrs(*I, L, ws, &k, &pp);
    if (key_dev) *key_dev = reinterpret_cast<int64_t*>(k);
    if (perm_dev) *perm_dev = pp;
    return CDD_OK;
}

int sa_layout(const cdd_instance* I, const sa_params* p, int32_t* lanes, int32_t* positions_per_lane) {
    cdd::SaLaunch L{};
    const int rc = sa_validate(I, p, &L);
    if (rc != CDD_OK) return rc;
    int32_t g = 0, e = 0;
    cdd::sa_layout(*I, L, &g, &e);
    if (lanes) *lanes = g;
    if (positions_per_lane) *positions_per_lane = e;
    return CDD_OK;
}

int sa_run(cdd_instance* I, const sa_params* p, void* ws, size_t ws_bytes, void* stream) {
    cdd::SaLaunch L{};
    int rc = sa_validate(I, p, &L);
    if (rc != CDD_OK) return rc;
    DeviceGuard g(I->device);
    const size_t need = generic(*I, L.ucd) ? cdd::wide_sa_workspace_bytes(*I, L) : cdd::sa_workspace_bytes(*I, L);
    if (!ws || ws_bytes < need)
        return fail(CDD_ENOMEM, "workspace too small: need " + std::to_string(need) + " bytes");
    cudaError_t e = generic(*I, L.ucd) ? cdd::launch_wide_sa(*I, L, ws, as_stream(stream))
                                       : cdd::launch_sa(*I, L, ws, as_stream(stream));
    if (e != cudaSuccess) return cuda_fail(e, "sa_run");
    I->has_best = true;
    return CDD_OK;
}

int sa_t0(cdd_instance* I, cdd_problem problem, uint64_t seed, int64_t samples, double* T0_dev,
          void* ws, size_t ws_bytes, void* stream) {
    if (!I || !T0_dev) return fail(CDD_EINVAL, "instance/T0_dev is NULL");
    if (samples < 1) return fail(CDD_EINVAL, "samples must be >= 1");
    sa_params p{};
    p.problem = problem;
    p.chains = 1;
    p.steps = 0;
    p.mu = 0.88;
    p.T0 = 0;
    p.t0_samples = samples;
    p.pert = 4;
    cdd::SaLaunch L{};
    int rc = sa_validate(I, &p, &L);
    if (rc != CDD_OK) return rc;
    DeviceGuard g(I->device);
    const size_t need = generic(*I, L.ucd) ? cdd::wide_sa_workspace_bytes(*I, L) : cdd::sa_workspace_bytes(*I, L);
    if (!ws || ws_bytes < need)
        return fail(CDD_ENOMEM, "workspace too small: need " + std::to_string(need) + " bytes");
    cudaError_t e = generic(*I, L.ucd) ? cdd::launch_wide_t0(*I, L.ucd, seed, samples, T0_dev, ws, as_stream(stream))
                            : cdd::launch_t0(*I, L.ucd, seed, samples, T0_dev, ws, as_stream(stream));
    return e == cudaSuccess ? CDD_OK : cuda_fail(e, "sa_t0");
}

static int dpso_validate(const cdd_instance* I, const dpso_params* p, cdd::DpsoLaunch* L) {
    if (!I || !p) return fail(CDD_EINVAL, "instance/params is NULL");
    if (p->problem != CDD_PROBLEM_CDD && p->problem != CDD_PROBLEM_UCDDCP) return fail(CDD_EINVAL, "bad problem");
    const bool ucd = p->problem == CDD_PROBLEM_UCDDCP;
    if (ucd && (!I->has_ucd || I->d < I->sum_p)) return fail(CDD_EINVAL, "instance not usable for UCDDCP (no m/gamma, or d < sum p)");
    if (I->n < 2) return fail(CDD_EINVAL, "DPSO needs n >= 2");
    if (generic(*I, ucd)) return fail(CDD_EINVAL, "DPSO runs on the fast path only (packed records: n <= 1024, p <= 255, ...)");
    if (p->particles < 1 || p->particles >= (1ll << 31)) return fail(CDD_EINVAL, "particles must be in [1, 2^31)");
    if (p->iters < 0 || p->iters >= (int64_t)UINT32_MAX) return fail(CDD_EINVAL, "iters must be in [0, 2^32)");
    if (p->particle_offset + (uint64_t)p->particles > (1ull << 32)) return fail(CDD_EINVAL, "particle ids must fit 32 bits");
    if (!(p->w >= 0 && p->w <= 1 && p->c1 >= 0 && p->c1 <= 1 && p->c2 >= 0 && p->c2 <= 1))
        return fail(CDD_EINVAL, "w, c1, c2 must be probabilities");
    L->ucd = ucd;
    L->particles = p->particles;
    L->iters = p->iters;
    L->w = p->w;
    L->c1 = p->c1;
    L->c2 = p->c2;
    L->seed = p->seed;
    L->particle_offset = p->particle_offset;
    L->gbest_trace = p->gbest_trace;
    return CDD_OK;
}

size_t dpso_workspace_size(const cdd_instance* I, const dpso_params* p) {
    cdd::DpsoLaunch L{};
    if (dpso_validate(I, p, &L) != CDD_OK) return 0;
    return cdd::dpso_workspace_bytes(*I, L);
}

static int dpso_prepare(cdd_instance* I, const dpso_params* p, void* ws, size_t ws_bytes,
                        cdd::DpsoLaunch* L) {
    int rc = dpso_validate(I, p, L);
    if (rc != CDD_OK) return rc;
    const size_t need = cdd::dpso_workspace_bytes(*I, *L);
    if (!ws || ws_bytes < need)
        return fail(CDD_ENOMEM, "workspace too small: need " + std::to_string(need) + " bytes");
    return CDD_OK;
}

int dpso_run(cdd_instance* I, const dpso_params* p, void* ws, size_t ws_bytes, void* stream) {
    cdd::DpsoLaunch L{};
    int rc = dpso_prepare(I, p, ws, ws_bytes, &L);
    if (rc != CDD_OK) return rc;
    DeviceGuard g(I->device);
    cudaStream_t s = as_stream(stream);
    cudaError_t e = cdd::dpso_begin(*I, L, ws, s);
    if (e == cudaSuccess) e = cdd::dpso_iterate(*I, L, ws, 0, L.iters, s);
    if (e == cudaSuccess) e = cdd::dpso_end(*I, L, ws, s);
    if (e != cudaSuccess) return cuda_fail(e, "dpso_run");
    I->has_best = true;
    return CDD_OK;
}

int dpso_begin(cdd_instance* I, const dpso_params* p, void* ws, size_t ws_bytes, void* stream) {
    cdd::DpsoLaunch L{};
    int rc = dpso_prepare(I, p, ws, ws_bytes, &L);
    if (rc != CDD_OK) return rc;
    DeviceGuard g(I->device);
    cudaError_t e = cdd::dpso_begin(*I, L, ws, as_stream(stream));
    return e == cudaSuccess ? CDD_OK : cuda_fail(e, "dpso_begin");
}

int dpso_iterate(cdd_instance* I, const dpso_params* p, void* ws, size_t ws_bytes, int64_t t,
                 void* stream) {
    cdd::DpsoLaunch L{};
    int rc = dpso_prepare(I, p, ws, ws_bytes, &L);
    if (rc != CDD_OK) return rc;
    if (t < 0 || t >= L.iters) return fail(CDD_EINVAL, "t must be in [0, iters)");
    DeviceGuard g(I->device);
    cudaError_t e = cdd::dpso_iterate(*I, L, ws, t, t + 1, as_stream(stream));
    return e == cudaSuccess ? CDD_OK : cuda_fail(e, "dpso_iterate");
}

int dpso_gbest_ptrs(const cdd_instance* I, const dpso_params* p, void* ws, int64_t t,
                    int64_t** key_dev, int16_t** perm_dev) {
    cdd::DpsoLaunch L{};
    int rc = dpso_validate(I, p, &L);
    if (rc != CDD_OK) return rc;
    if (!ws) return fail(CDD_EINVAL, "workspace is NULL");
    if (t < 0 || t > L.iters) return fail(CDD_EINVAL, "t must be in [0, iters]");
    cdd::dpso_gbest(*I, L, ws, t, key_dev, perm_dev);
    return CDD_OK;
}

int dpso_end(cdd_instance* I, const dpso_params* p, void* ws, size_t ws_bytes, void* stream) {
    cdd::DpsoLaunch L{};
    int rc = dpso_prepare(I, p, ws, ws_bytes, &L);
    if (rc != CDD_OK) return rc;
    DeviceGuard g(I->device);
    cudaError_t e = cdd::dpso_end(*I, L, ws, as_stream(stream));
    if (e != cudaSuccess) return cuda_fail(e, "dpso_end");
    I->has_best = true;
    return CDD_OK;
}

// ---- fused DPSO swarm-best exchange over peer memory
int dpso_peer_create(cdd_instance* I, int world, int rank, uint8_t* ipc_handle) {
    if (!I || !ipc_handle) return fail(CDD_EINVAL, "instance/ipc_handle is NULL");
    if (world < 1 || rank < 0 || rank >= world) return fail(CDD_EINVAL, "need 0 <= rank < world");
    if (I->peer) return fail(CDD_ESTATE, "a peer exchange exists on this instance (dpso_peer_destroy first)");
    DeviceGuard g(I->device);
    auto* P = new cdd::DpsoPeer();
    P->world = world;
    P->rank = rank;
    P->np = cdd::dpso_np(I->n);
    const size_t bytes = cdd::dpso_peer_region_bytes(I->n);
    cudaError_t e = cudaMalloc(&P->region, bytes);
    if (e == cudaSuccess) e = cudaMemset(P->region, 0, bytes);
    cudaIpcMemHandle_t h{};
    if (e == cudaSuccess) e = cudaIpcGetMemHandle(&h, P->region);
    if (e != cudaSuccess) {
        cudaFree(P->region);
        delete P;
        return cuda_fail(e, "dpso_peer_create");
    }
    static_assert(sizeof(cudaIpcMemHandle_t) == CDD_IPC_HANDLE_BYTES, "IPC handle size");
    std::memcpy(ipc_handle, &h, sizeof(h));
    P->mapped.assign((size_t)world, nullptr);
    I->peer = P;
    return CDD_OK;
}

int dpso_peer_open(cdd_instance* I, const uint8_t* handles) {
    if (!I || !handles) return fail(CDD_EINVAL, "instance/handles is NULL");
    cdd::DpsoPeer* P = I->peer;
    if (!P) return fail(CDD_ESTATE, "no peer exchange (dpso_peer_create first)");
    if (P->open) return fail(CDD_ESTATE, "peer exchange already open");
    DeviceGuard g(I->device);
    std::vector<uint8_t*> regions((size_t)P->world, nullptr);
    cudaError_t e = cudaSuccess;
    for (int r = 0; r < P->world && e == cudaSuccess; ++r) {
        if (r == P->rank) {
            regions[r] = P->region;
            continue;
        }
        cudaIpcMemHandle_t h{};
        std::memcpy(&h, handles + (size_t)r * CDD_IPC_HANDLE_BYTES, sizeof(h));
        void* ptr = nullptr;
        e = cudaIpcOpenMemHandle(&ptr, h, cudaIpcMemLazyEnablePeerAccess);
        P->mapped[r] = static_cast<uint8_t*>(ptr);
        regions[r] = P->mapped[r];
    }
    if (e == cudaSuccess) e = cudaMalloc(&P->d_regions, sizeof(uint8_t*) * (size_t)P->world);
    if (e == cudaSuccess)
        e = cudaMemcpy(P->d_regions, regions.data(), sizeof(uint8_t*) * (size_t)P->world, cudaMemcpyHostToDevice);
    if (e != cudaSuccess) {
        for (uint8_t*& m : P->mapped)
            if (m) cudaIpcCloseMemHandle(m), m = nullptr;
        cudaFree(P->d_regions);
        P->d_regions = nullptr;
        return cuda_fail(e, "dpso_peer_open");
    }
    P->open = true;
    return CDD_OK;
}

__global__ void peer_reset_kernel(uint8_t* region, int* err) {
    if (threadIdx.x < 3) reinterpret_cast<unsigned long long*>(region + cdd::kPeerKeyOff)[threadIdx.x] = ULLONG_MAX;
    if (threadIdx.x == 3) *reinterpret_cast<unsigned int*>(region + cdd::kPeerArriveOff) = 0u;
    if (threadIdx.x == 4) atomicAnd(err, ~2);  // a previous run's exchange timeout
}

int dpso_peer_reset(cdd_instance* I, void* stream) {
    if (!I) return fail(CDD_EINVAL, "instance is NULL");
    if (!I->peer) return fail(CDD_ESTATE, "no peer exchange (dpso_peer_create first)");
    DeviceGuard g(I->device);
    peer_reset_kernel<<<1, 32, 0, as_stream(stream)>>>(I->peer->region, I->err);
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(e, "dpso_peer_reset");
    I->peer->armed = true;
    return CDD_OK;
}

int dpso_peer_destroy(cdd_instance* I) {
    if (!I) return fail(CDD_EINVAL, "instance is NULL");
    if (!I->peer) return CDD_OK;
    DeviceGuard g(I->device);
    cudaDeviceSynchronize();
    for (uint8_t* m : I->peer->mapped)
        if (m) cudaIpcCloseMemHandle(m);
    cudaFree(I->peer->d_regions);
    cudaFree(I->peer->region);
    delete I->peer;
    I->peer = nullptr;
    return CDD_OK;
}

int dpso_run_peer(cdd_instance* I, const dpso_params* p, void* ws, size_t ws_bytes, void* stream) {
    cdd::DpsoLaunch L{};
    int rc = dpso_prepare(I, p, ws, ws_bytes, &L);
    if (rc != CDD_OK) return rc;
    cdd::DpsoPeer* P = I->peer;
    if (!P || !P->open) return fail(CDD_ESTATE, "peer exchange not open (dpso_peer_create / dpso_peer_open)");
    if (p->particle_offset != (uint64_t)P->rank * (uint64_t)p->particles)
        return fail(CDD_EINVAL, "particle_offset must be rank * particles (equal shares)");
    if ((uint64_t)p->particles * (uint64_t)P->world > (1ull << 32))
        return fail(CDD_EINVAL, "global particle ids must fit 32 bits");
    if (!P->armed) return fail(CDD_ESTATE, "peer exchange not re-armed: dpso_peer_reset (+ a barrier) before every fused run");
    L.peer = true;
    P->armed = false;
    DeviceGuard g(I->device);
    cudaStream_t s = as_stream(stream);
    cudaError_t e = cdd::dpso_begin(*I, L, ws, s);
    if (e == cudaSuccess) e = cdd::dpso_iterate(*I, L, ws, 0, L.iters, s);
    if (e == cudaSuccess) e = cdd::dpso_end(*I, L, ws, s);
    if (e != cudaSuccess) return cuda_fail(e, "dpso_run_peer");
    I->has_best = true;
    return CDD_OK;
}

int best_device_ptrs(cdd_instance* I, int64_t** packed_dev, int16_t** perm_dev) {
    if (!I) return fail(CDD_EINVAL, "instance is NULL");
    if (I->wide) return fail(CDD_EINVAL, "generic-path instance: penalties may exceed the packed key, use best_device_ptrs_wide");
    if (packed_dev) *packed_dev = reinterpret_cast<int64_t*>(I->best_key);
    if (perm_dev) *perm_dev = I->best_perm;
    return CDD_OK;
}

int best_device_ptrs_wide(cdd_instance* I, int64_t** pen_id_dev, int16_t** perm_dev) {
    if (!I) return fail(CDD_EINVAL, "instance is NULL");
    if (!I->wide) return fail(CDD_EINVAL, "fast-path instance: use best_device_ptrs (packed key)");
    if (pen_id_dev) *pen_id_dev = reinterpret_cast<int64_t*>(I->best_wide);
    if (perm_dev) *perm_dev = I->best_perm;
    return CDD_OK;
}

int best_get(cdd_instance* I, int64_t* penalty, int16_t* perm_host, uint64_t* id, void* stream) {
    if (!I) return fail(CDD_EINVAL, "instance is NULL");
    if (!I->has_best) return fail(CDD_ESTATE, "no run has completed on this instance");
    DeviceGuard g(I->device);
    cudaStream_t s = as_stream(stream);
    unsigned long long key = 0;
    long long pw[2] = {-1, -1};
    cudaError_t e = I->wide ? cudaMemcpyAsync(pw, I->best_wide, sizeof pw, cudaMemcpyDeviceToHost, s)
                            : cudaMemcpyAsync(&key, I->best_key, sizeof key, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess && perm_host)
        e = cudaMemcpyAsync(perm_host, I->best_perm, sizeof(int16_t) * I->n, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) return cuda_fail(e, "best_get");
    if (I->wide) {
        if (pw[0] < 0 || pw[0] == LLONG_MAX) return fail(CDD_ESTATE, "no result");
        if (penalty) *penalty = pw[0];
        if (id) *id = (uint64_t)pw[1];
        return CDD_OK;
    }
    if (key == ULLONG_MAX) return fail(CDD_ESTATE, "no result");
    if (penalty) *penalty = (int64_t)(key >> 32);
    if (id) *id = key & 0xffffffffull;
    return CDD_OK;
}

}  // extern "C"
