// sg_api.cu — the C ABI (include/sg.h): validation, plans/workspace, orchestration of the kernels.
#include "sg_internal.cuh"
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <cmath>
#include <vector>
#include <mutex>
#include <atomic>

using namespace sg;

struct sg_plan {
    cudaStream_t s = nullptr;
    bool poisoned = false;
    int64_t rb = 0, re = 0, nr = 0, thr = 0, p = 0, m = 0;
    int dt = 0;
    int64_t* w = nullptr;
    int8_t* cls = nullptr;
    int32_t* lists = nullptr;
    int64_t* u = nullptr;
    int64_t* dbin = nullptr;  // [0..NBINS) counts, [NBINS] nlong, [NBINS+1 .. 2NBINS+1) cursors
    int64_t bin_cnt[NBINS] = {0};
    int64_t bin_off[NBINS + 1] = {0};
    int64_t nheavy = 0;
    int32_t* heavy = nullptr;       // heavy rows (local ids), heaviest first
    int64_t* range_bounds = nullptr;
    int64_t* range_off = nullptr;
    int32_t* nranges = nullptr;
    RangeRec* ranges = nullptr;
    int64_t nslots = 0, amax = 0;
    int64_t nbig = 0;               // heavy rows [0, nbig) with w >= 2^20 (1024-thread symbolic kernel)
    int64_t ndw = 0;                // heavy[0, ndw): dense-window rows (w >= 2^dw_log2), sg_dense.cu
    int32_t* dtc = nullptr;         // their per-tile output counts (ndw x T), from the symbolic pass
    int4* ditems = nullptr;         // dense-window work items (row, window range)
    int64_t* ditem_off = nullptr;   // exclusive prefix of items per dense row; [ndw] = item count
    int64_t nskew = 0;              // light rows on the sorted path (column-skewed; sg_light.cu)
    int dw_log2 = 0;
    int2* span = nullptr;           // light rows: [cmin, cmax] of the output columns
    uint32_t* lkeys = nullptr;      // sorted light bins: each row's sorted column keys (symbolic -> numeric)
    int64_t lkey_off[NBIN_LIGHT] = {0};
    int4* gscr = nullptr;           // heavy rows with more than KC entries: per-k cursor scratch
    void* pscr = nullptr;           // dense2: per-CTA part scratch for rows with many k entries
    int64_t pscr_cap = 0;
    int variant = 0;
    int32_t* long_id = nullptr;
    uint32_t* tp = nullptr;
    int64_t nlong = 0;
    int64_t nlong_tp = 0;           // nlong if the tile-pointer table is built, else 0 (over SG_OPT_TP_MAX_BYTES)
    int T = 0;
    unsigned long long* counter = nullptr;
    const int64_t* C_rp = nullptr;
    int64_t nnz_c = 0;
    std::vector<void*> allocs;
};

namespace {

std::once_flag g_pool_once;

void init_pool() {
    std::call_once(g_pool_once, [] {
        int dev = 0;
        if (cudaGetDevice(&dev) != cudaSuccess) return;
        cudaMemPool_t pool;
        if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
            uint64_t thr = UINT64_MAX;
            cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
        }
    });
}

// stream-ordered scratch owned by a scope (non-plan calls)
struct Scratch {
    cudaStream_t s;
    std::vector<void*> ptrs;
    explicit Scratch(cudaStream_t st) : s(st) {}
    void* get(size_t bytes) {
        void* p = nullptr;
        if (bytes == 0) bytes = 16;
        if (cudaMallocAsync(&p, bytes, s) != cudaSuccess) return nullptr;
        ptrs.push_back(p);
        return p;
    }
    ~Scratch() { for (void* p : ptrs) cudaFreeAsync(p, s); }
};

void* palloc(sg_plan* pl, size_t bytes) {
    void* p = nullptr;
    if (bytes == 0) bytes = 16;
    if (cudaMallocAsync(&p, bytes, pl->s) != cudaSuccess) return nullptr;
    pl->allocs.push_back(p);
    return p;
}

#define CK(x) do { cudaError_t _e = (x); if (_e != cudaSuccess) { cudaGetLastError(); return SG_ERR_CUDA; } } while (0)
#define CKP(pl, x) do { cudaError_t _e = (x); if (_e != cudaSuccess) { cudaGetLastError(); (pl)->poisoned = true; return SG_ERR_CUDA; } } while (0)

Mat mat_of(const sg_csr_view* v) {
    Mat m;
    m.nrows = v->nrows; m.ncols = v->ncols; m.nnz = v->nnz;
    m.rp = v->row_ptr; m.col = v->col_idx; m.val = v->val; m.dt = (int)v->dtype;
    return m;
}

// Process-wide options (sg_set_option). The environment seeds them ONCE, at the first call
// (SG_VALIDATE=1, SG_DW_LOG2=m); no call reads the environment afterwards.
std::once_flag g_opt_once;
std::atomic<int64_t> g_opt[SG_OPT_COUNT];

void init_options() {
    std::call_once(g_opt_once, [] {
        g_opt[SG_OPT_VALIDATE] = 0;
        g_opt[SG_OPT_DENSE_LOG2] = -1;
        g_opt[SG_OPT_VARIANT] = 0;
        const char* e = getenv("SG_VALIDATE");
        if (e && e[0] == '1') g_opt[SG_OPT_VALIDATE] = 1;
        e = getenv("SG_DW_LOG2");
        if (e && *e) g_opt[SG_OPT_DENSE_LOG2] = atoll(e);
        g_opt[SG_OPT_L2_PERSIST] = 0;
        g_opt[SG_OPT_TP_MAX_BYTES] = -1;
        e = getenv("SG_L2_PERSIST");
        if (e && *e) g_opt[SG_OPT_L2_PERSIST] = atoll(e);
    });
}

// B.col in the persisting L2 carve-out for the launches of one call (SG_OPT_L2_PERSIST): every heavy
// product gathers a column index of B, and B (193 MB on C3: 64 MB of columns, 129 MB of values) exceeds
// the 126 MB L2, so without it the C stream and the value gathers evict the columns. The window is set on
// the caller's stream for this call's launches only and cleared on exit.
struct L2Window {
    cudaStream_t s;
    bool on = false;
    L2Window(cudaStream_t st, const void* ptr, size_t bytes) : s(st) {
        init_options();
        const int64_t opt = g_opt[SG_OPT_L2_PERSIST].load();
        if (opt == 0 || bytes == 0 || !ptr) return;
        static size_t maxp = 0, maxwin = 0;
        static std::once_flag once;
        std::call_once(once, [] {
            int dev = 0, a = 0, b = 0;
            if (cudaGetDevice(&dev) != cudaSuccess) return;
            if (cudaDeviceGetAttribute(&a, cudaDevAttrMaxPersistingL2CacheSize, dev) != cudaSuccess) a = 0;
            if (cudaDeviceGetAttribute(&b, cudaDevAttrMaxAccessPolicyWindowSize, dev) != cudaSuccess) b = 0;
            maxp = (size_t)a;
            maxwin = (size_t)b;
            cudaGetLastError();
        });
        if (maxp == 0 || maxwin == 0) return;
        size_t want = opt > 0 && (size_t)opt < bytes ? (size_t)opt : bytes;
        if (want > maxp) want = maxp;
        size_t cur = 0;
        if (cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize) == cudaSuccess && cur < want)
            cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, want);
        cudaStreamAttrValue v = {};
        v.accessPolicyWindow.base_ptr = const_cast<void*>(ptr);
        v.accessPolicyWindow.num_bytes = bytes < maxwin ? bytes : maxwin;
        const double hr = (double)want / (double)v.accessPolicyWindow.num_bytes;
        v.accessPolicyWindow.hitRatio = (float)(hr < 1.0 ? hr : 1.0);
        v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        on = cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &v) == cudaSuccess;
        cudaGetLastError();
    }
    ~L2Window() {
        if (!on) return;
        cudaStreamAttrValue v = {};
        v.accessPolicyWindow.num_bytes = 0;
        cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &v);
        cudaGetLastError();
    }
};

int variant_bits() {
    init_options();
    return (int)g_opt[SG_OPT_VARIANT].load();
}

bool env_validate() {
    init_options();
    return g_opt[SG_OPT_VALIDATE].load() != 0;
}

__global__ void k_validate(Mat M, int* bad) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M.nrows; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t s = M.rp[i], e = M.rp[i + 1];
        if (e < s) { atomicOr(bad, 1); continue; }
        for (int64_t q = s; q < e; ++q) {
            int c = M.col[q];
            if (c < 0 || c >= M.ncols || (q > s && M.col[q - 1] >= c)) { atomicOr(bad, 1); break; }
        }
    }
}

sg_status validate_one(const sg_csr_view* v, cudaStream_t s) {
    if (!v) return SG_ERR_INVALID_ARG;
    if (v->nrows < 0 || v->ncols < 0 || v->nnz < 0) return SG_ERR_INVALID_ARG;
    if (v->ncols > INT32_MAX || v->nrows > INT32_MAX) return SG_ERR_OVERFLOW;
    if (v->dtype != SG_F64 && v->dtype != SG_F32) return SG_ERR_DTYPE;
    if (!v->row_ptr) return SG_ERR_INVALID_ARG;
    if (v->nnz > 0 && (!v->col_idx || !v->val)) return SG_ERR_INVALID_ARG;
    if (env_validate()) {
        Scratch sc(s);
        int* bad = (int*)sc.get(sizeof(int));
        if (!bad) return SG_ERR_OOM;
        CK(cudaMemsetAsync(bad, 0, sizeof(int), s));
        Mat m = mat_of(v);
        if (m.nrows > 0) SG_LAUNCH("k_validate", s, k_validate<<<(unsigned)((m.nrows + 255) / 256 < 4096 ? (m.nrows + 255) / 256 : 4096), 256, 0, s>>>(m, bad));
        CK(cudaGetLastError());
        int h = 0;
        CK(cudaMemcpyAsync(&h, bad, sizeof(int), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (h) return SG_ERR_NOT_CANONICAL;
    }
    return SG_OK;
}

sg_status validate_pair(const sg_csr_view* A, const sg_csr_view* B, cudaStream_t s) {
    sg_status st;
    if ((st = validate_one(A, s)) != SG_OK) return st;
    if ((st = validate_one(B, s)) != SG_OK) return st;
    if (A->ncols != B->nrows) return SG_ERR_SHAPE;
    if (A->dtype != B->dtype) return SG_ERR_DTYPE;
    return SG_OK;
}

CostModelD cm_of(const sg_cost_model* c) {
    CostModelD d;
    d.kL = c->kappa_L; d.lL = c->lambda_L; d.sL = c->sigma_L; d.rL = c->rho_L;
    d.kH = c->kappa_H; d.lH = c->lambda_H; d.tH = c->tau_H; d.mH = c->mu_H;
    d.tiles_fixed = c->tiles_fixed; d.capu = c->capu; d.cap_L = c->cap_L;
    return d;
}

// Default model: calibrated from the measured kernels (profiles/).
// Refitted for the round-2 final kernels (warp-tile rank kernel, sorted light path) by tools/sweep.py:
// non-negative least squares of the per-class kernel times over the threshold grids of ER 2^18, R-MAT 18,
// un-permuted R-MAT 18 and R-MAT 20 (C3) together, with R(u)'s floor tiles_fixed = ceil(p / 131072) per
// matrix (profiles/r02g_sweep_precal2.json + r02g_sweep_precal_c3.json, joint fit in
// profiles/r02g_costmodel_fit.txt), in ps of SM time. tiles_fixed here is the p <= 131072 value; calls with
// cm == NULL use default_range_floor(B.ncols). (Earlier fits: round-2 mid 0, 9315, 0, 0, 5016705, 0, 74786,
// 1854; round 1: 33399, 7915, 0, 0, 17907513, 1102, 68338, 209 with R(u) = max(1, ceil(u/12288)).)
constexpr int64_t kTileMinRows = 4096;  // rank rows below which the warp-tile kernel is not used

const sg_cost_model kDefaultModel = {
    /*kappa_L*/ 0, /*lambda_L*/ 7079, /*sigma_L*/ 0, /*rho_L*/ 0,
    /*kappa_H*/ 3723548, /*lambda_H*/ 0, /*tau_H*/ 46855, /*mu_H*/ 2169,
    /*tiles_fixed*/ 1, /*capu*/ 12288, /*cap_L*/ SG_CAP_L_MAX};

// The heavy path's minimum number of column ranges per row: a row whose columns span [0, p) needs at
// least ceil(p / (RW_TILES * TW)) rank-kernel ranges (and dense windows in proportion), whatever its u.
// The default model takes it as R(u)'s floor (tiles_fixed) for the B at hand.
int64_t default_range_floor(int64_t p) {
    const int64_t span = (int64_t)RW_TILES * TW;
    const int64_t r = (p + span - 1) / span;
    return r < 1 ? 1 : r;
}

// Partition model (reading R19): fitted by tools/fit_partition_model.py to 88 measured
// shard times (R-MAT 20 and 18, permuted and un-permuted, G = 2..16; profiles/r01s4_partition_model_fit.json):
// a light row costs rho_L per output, a heavy row lambda_H per product (ps of SM time).
const sg_cost_model kPartitionModel = {
    /*kappa_L*/ 0, /*lambda_L*/ 0, /*sigma_L*/ 0, /*rho_L*/ 22705,
    /*kappa_H*/ 0, /*lambda_H*/ 2064, /*tau_H*/ 0, /*mu_H*/ 0,
    /*tiles_fixed*/ 1, /*capu*/ 0, /*cap_L*/ SG_CAP_L_MAX};

// Identify over a row list (rows == nullptr: rows [0, nr)). Computes w, a, u of those rows on the
// device (exact sample-symbolic at routing threshold cap_L), then the cost histogram.
struct RowStats {
    int64_t* w = nullptr;
    int64_t* a = nullptr;
    int64_t* u = nullptr;
};

sg_status row_stats(const Mat& A, const Mat& B, const int64_t* rows, int64_t nr, int64_t cap, Scratch& sc,
                    RowStats& rs, cudaStream_t s) {
    rs.w = (int64_t*)sc.get(sizeof(int64_t) * (size_t)nr);
    rs.a = (int64_t*)sc.get(sizeof(int64_t) * (size_t)nr);
    rs.u = (int64_t*)sc.get(sizeof(int64_t) * (size_t)nr);
    int32_t* lists = (int32_t*)sc.get(sizeof(int32_t) * (size_t)nr);
    int64_t* dbin = (int64_t*)sc.get(sizeof(int64_t) * (2 * NBINS + 1));
    int64_t* all_rows = nullptr;
    if (!rs.w || !rs.a || !rs.u || !lists || !dbin) return SG_ERR_OOM;
    if (!rows) {
        all_rows = (int64_t*)sc.get(sizeof(int64_t) * (size_t)nr);
        if (!all_rows) return SG_ERR_OOM;
        // rows [0, nr): use the identity row map through sample-select with f = 1
        size_t tb = sample_tmp_bytes(nr);
        void* tmp = sc.get(tb);
        int64_t* dcount = (int64_t*)sc.get(sizeof(int64_t));
        if (!tmp || !dcount) return SG_ERR_OOM;
        CK(launch_sample_select(0, nr, 0, 0, true, all_rows, dcount, tmp, tb, s));
        rows = all_rows;
    }
    CK(launch_row_work_list(A, B, rows, nr, rs.w, rs.a, s));
    CK(cudaMemsetAsync(rs.u, 0, sizeof(int64_t) * (size_t)nr, s));
    CK(cudaMemsetAsync(dbin, 0, sizeof(int64_t) * (2 * NBINS + 1), s));
    CK(launch_bin_count(rs.w, nr, cap, dbin, nullptr, s));
    // largest a over the listed rows (part scratch of the lean symbolic, sg_sym2.cu), read back with the
    // bin counts in ONE copy + sync
    CK(launch_max_i64(rs.a, nr, (unsigned long long*)(dbin + NBINS), s));
    int64_t cnt[NBINS + 1];
    CK(cudaMemcpyAsync(cnt, dbin, sizeof(cnt), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    const int64_t amax = cnt[NBINS];
    int64_t off[NBINS + 1];
    off[0] = 0;
    for (int b = 0; b < NBINS; ++b) off[b + 1] = off[b] + cnt[b];
    CK(cudaMemcpyAsync(dbin + NBINS, off, sizeof(int64_t) * NBINS, cudaMemcpyHostToDevice, s));
    CK(launch_bin_scatter(rs.w, nr, cap, dbin + NBINS, lists, s));
    for (int b = 0; b < NBIN_LIGHT; ++b)
        CK(launch_sym_light(b, A, B, lists + off[b], cnt[b], rows, 0, rs.u, nullptr, nullptr, s));
    unsigned long long* counter = (unsigned long long*)sc.get(2 * sizeof(unsigned long long));
    if (!counter) return SG_ERR_OOM;
    if (cnt[BIN_HEAVY] == 0) return SG_OK;
    if (variant_bits() & 2) {
        CK(launch_sym_heavy(A, B, lists + off[BIN_HEAVY], cnt[BIN_HEAVY], rows, 0, rs.u, nullptr, nullptr, nullptr,
                            0, nullptr, nullptr, nullptr, 0, counter, s, cnt[BIN_HEAVY]));
        return SG_OK;
    }
    const int64_t np = sym2_scratch_parts(amax);
    void* pscr = np > 0 ? sc.get(part_bytes() * (size_t)np) : nullptr;
    if (np > 0 && !pscr) return SG_ERR_OOM;
    CK(launch_sym_heavy2(A, B, lists + off[BIN_HEAVY], cnt[BIN_HEAVY], rows, 0, rs.w, rs.u, nullptr, nullptr, nullptr,
                         0, nullptr, nullptr, nullptr, 0, counter, s, cnt[BIN_HEAVY], pscr, amax));
    return SG_OK;
}

// SG_ERR_OVERFLOW when sum_i (c_L(i) + c_H(i)) could leave int64 (kCostLimit = 2^62 in fp64)
sg_status check_cost_bound(const CostModelD& cm, const RowStats& rs, int64_t nr, Scratch& sc, cudaStream_t s) {
    double* dm = (double*)sc.get(sizeof(double));
    if (!dm) return SG_ERR_OOM;
    CK(launch_cost_mag(cm, rs.w, rs.a, rs.u, nr, dm, s));
    double hm = 0.0;
    CK(cudaMemcpyAsync(&hm, dm, sizeof(double), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    return hm >= kCostLimit ? SG_ERR_OVERFLOW : SG_OK;
}

sg_status identify(const Mat& A, const Mat& B, const int64_t* rows, int64_t nr, const sg_cost_model* c,
                   ThrResult* res, cudaStream_t s) {
    Scratch sc(s);
    RowStats rs;
    sg_status st = row_stats(A, B, rows, nr, c->cap_L, sc, rs, s);
    if (st != SG_OK) return st;
    CostModelD cm = cm_of(c);
    size_t hb = sizeof(long long) * (size_t)(c->cap_L + 1);
    long long* hd = (long long*)sc.get(hb);
    long long* hc = (long long*)sc.get(hb);
    long long* hw = (long long*)sc.get(hb);
    long long* sums = (long long*)sc.get(4 * sizeof(long long));
    ThrResult* dres = (ThrResult*)sc.get(sizeof(ThrResult));
    // overflow bound (fp64 sum of c_L + c_H) and the per-class sums of u at the chosen threshold (the
    // sample's compression, used by the cost-weighted split, R19): read back together with the
    // threshold in one copy + sync
    double* dm = (double*)sc.get(sizeof(double));
    unsigned long long* us = (unsigned long long*)sc.get(2 * sizeof(unsigned long long));
    if (!hd || !hc || !hw || !sums || !dres || !dm || !us) return SG_ERR_OOM;
    CK(launch_cost_mag(cm, rs.w, rs.a, rs.u, nr, dm, s));
    CK(launch_cost_hist(cm, rs.w, rs.a, rs.u, nr, hd, hc, hw, sums, s));
    CK(launch_argmin(cm, hd, hc, hw, sums, dres, s));
    CK(launch_class_usum_dev(rs.w, rs.u, nr, &dres->thr, us, s));
    double hm = 0.0;
    unsigned long long hu[2] = {0, 0};
    CK(cudaMemcpyAsync(res, dres, sizeof(ThrResult), cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(&hm, dm, sizeof(double), cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(hu, us, sizeof(hu), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (hm >= kCostLimit) return SG_ERR_OVERFLOW;
    res->U_L = (long long)hu[0];
    res->U_H = (long long)hu[1];
    return SG_OK;
}

sg_status check_model(const sg_cost_model* c) {
    if (c->cap_L < 0 || c->cap_L > SG_CAP_L_MAX) return SG_ERR_INVALID_ARG;
    const int64_t co[] = {c->kappa_L, c->lambda_L, c->sigma_L, c->rho_L, c->kappa_H, c->lambda_H, c->tau_H, c->mu_H,
                          c->tiles_fixed, c->capu};
    for (int64_t x : co)
        if (x < 0) return SG_ERR_INVALID_ARG;
    return SG_OK;
}

}  // namespace

extern "C" {

const char* sg_status_string(sg_status st) {
    switch (st) {
        case SG_OK: return "SG_OK";
        case SG_ERR_INVALID_ARG: return "SG_ERR_INVALID_ARG";
        case SG_ERR_SHAPE: return "SG_ERR_SHAPE";
        case SG_ERR_DTYPE: return "SG_ERR_DTYPE";
        case SG_ERR_NOT_CANONICAL: return "SG_ERR_NOT_CANONICAL";
        case SG_ERR_EMPTY_SAMPLE: return "SG_ERR_EMPTY_SAMPLE";
        case SG_ERR_OOM: return "SG_ERR_OOM";
        case SG_ERR_CUDA: return "SG_ERR_CUDA";
        case SG_ERR_NCCL: return "SG_ERR_NCCL";
        case SG_ERR_OVERFLOW: return "SG_ERR_OVERFLOW";
    }
    return "SG_ERR_UNKNOWN";
}

const char* sg_version(void) { return "sg 0.1.0 sm_100a"; }

sg_status sg_set_option(int key, int64_t value) {
    init_options();
    if (key < 0 || key >= SG_OPT_COUNT) return SG_ERR_INVALID_ARG;
    if (key == SG_OPT_VALIDATE && value != 0 && value != 1) return SG_ERR_INVALID_ARG;
    if (key == SG_OPT_DENSE_LOG2 && (value < -1 || value > 62)) return SG_ERR_INVALID_ARG;
    if (key == SG_OPT_VARIANT && (value < 0 || value > 63)) return SG_ERR_INVALID_ARG;
    if (key == SG_OPT_L2_PERSIST && value < -1) return SG_ERR_INVALID_ARG;
    if (key == SG_OPT_TP_MAX_BYTES && value < -1) return SG_ERR_INVALID_ARG;
    g_opt[key] = value;
    return SG_OK;
}

int64_t sg_get_option(int key) {
    init_options();
    if (key < 0 || key >= SG_OPT_COUNT) return INT64_MIN;
    return g_opt[key].load();
}

void sg_default_cost_model(sg_cost_model* out) {
    if (out) *out = kDefaultModel;
}

void sg_default_cost_model_for(int64_t p, sg_cost_model* out) {
    if (!out) return;
    *out = kDefaultModel;
    out->tiles_fixed = default_range_floor(p);
}

void sg_default_partition_model(sg_cost_model* out) {
    if (out) *out = kPartitionModel;
}

sg_status sg_row_work(const sg_csr_view* A, const sg_csr_view* B, int64_t row_begin, int64_t row_end, int64_t* w_out,
                      int64_t* total_out, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    init_pool();
    sg_status st = validate_pair(A, B, s);
    if (st != SG_OK) return st;
    if (row_begin < 0 || row_end < row_begin || row_end > A->nrows) return SG_ERR_INVALID_ARG;
    if (!w_out && row_end > row_begin) return SG_ERR_INVALID_ARG;
    Mat a = mat_of(A), b = mat_of(B);
    CK(launch_row_work(a, b, row_begin, row_end, w_out, s));
    if (total_out) {
        Scratch sc(s);
        int64_t n = row_end - row_begin;
        int64_t* P = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(n + 1));
        void* tmp = sc.get(scan_tmp_bytes(n));
        if (!P || !tmp) return SG_ERR_OOM;
        CK(scan_exclusive(w_out, P, n, tmp, s));
        CK(cudaMemcpyAsync(total_out, P + n, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
    }
    return SG_OK;
}

sg_status sg_sample_rows(int64_t row_begin, int64_t row_end, double f, uint64_t seed, int64_t* rows_out,
                         int64_t rows_cap, int64_t* count_out, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    init_pool();
    if (!(f > 0.0 && f <= 1.0) || row_begin < 0 || row_end < row_begin || !count_out) return SG_ERR_INVALID_ARG;
    int64_t n = row_end - row_begin;
    Scratch sc(s);
    int64_t* rows = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    int64_t* dcount = (int64_t*)sc.get(sizeof(int64_t));
    size_t tb = sample_tmp_bytes(n);
    void* tmp = sc.get(tb);
    if (!rows || !dcount || !tmp) return SG_ERR_OOM;
    bool all = f >= 1.0;
    uint64_t Tf = all ? 0 : (uint64_t)std::ldexp(f, 64);
    CK(launch_sample_select(row_begin, row_end, seed, Tf, all, rows, dcount, tmp, tb, s));
    int64_t c = 0;
    CK(cudaMemcpyAsync(&c, dcount, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    *count_out = c;
    if (rows_out && c > 0) {
        if (rows_cap < c) return SG_ERR_SHAPE;
        CK(cudaMemcpyAsync(rows_out, rows, sizeof(int64_t) * (size_t)c, cudaMemcpyDeviceToDevice, s));
        CK(cudaStreamSynchronize(s));
    }
    return SG_OK;
}

sg_status sg_sample_threshold(const sg_csr_view* A, const sg_csr_view* B, double sample_frac, uint64_t seed,
                              const sg_cost_model* cm, int64_t* thr_out, sg_sample_report* rep, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    init_pool();
    if (!thr_out) return SG_ERR_INVALID_ARG;
    if (!(sample_frac > 0.0 && sample_frac <= 1.0)) return SG_ERR_INVALID_ARG;
    sg_status st = validate_pair(A, B, s);
    if (st != SG_OK) return st;
    sg_cost_model dflt = kDefaultModel;
    dflt.tiles_fixed = default_range_floor(B->ncols);
    const sg_cost_model* c = cm ? cm : &dflt;
    if ((st = check_model(c)) != SG_OK) return st;
    Mat a = mat_of(A), b = mat_of(B);
    const int64_t n = A->nrows;
    // Sample: S = { i : h(seed, SAMPLE, i) < floor(f 2^64) }  (R4)
    Scratch sc(s);
    int64_t* S = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    int64_t* dcount = (int64_t*)sc.get(sizeof(int64_t));
    size_t tb = sample_tmp_bytes(n);
    void* tmp = sc.get(tb);
    if (!S || !dcount || !tmp) return SG_ERR_OOM;
    bool all = sample_frac >= 1.0;
    uint64_t Tf = all ? 0 : (uint64_t)std::ldexp(sample_frac, 64);
    CK(launch_sample_select(0, n, seed, Tf, all, S, dcount, tmp, tb, s));
    int64_t ns = 0;
    CK(cudaMemcpyAsync(&ns, dcount, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (ns == 0) return SG_ERR_EMPTY_SAMPLE;
    // Identify on S (exact per-row w, a, u; integer J histogram; smallest argmin)
    ThrResult r;
    st = identify(a, b, S, ns, c, &r, s);
    if (st != SG_OK) return st;
    if (r.nonempty == 0) return SG_ERR_EMPTY_SAMPLE;
    // Extrapolate: identity (r = r')
    *thr_out = r.thr;
    if (rep) {
        rep->sample_rows = ns;
        rep->sample_nonempty = r.nonempty;
        rep->thr = r.thr;
        rep->W_est_L = r.W_L;
        rep->W_est_H = r.W_all - r.W_L;
        rep->J_min = r.Jmin;
        rep->U_est_L = r.U_L;
        rep->U_est_H = r.U_H;
    }
    return SG_OK;
}

sg_status sg_threshold_on_rows(const sg_csr_view* A, const sg_csr_view* B, const int64_t* rows, int64_t nrows,
                               const sg_cost_model* cm, int64_t* thr_out, sg_sample_report* rep, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    init_pool();
    if (!thr_out || nrows < 0 || (nrows > 0 && !rows)) return SG_ERR_INVALID_ARG;
    sg_status st = validate_pair(A, B, s);
    if (st != SG_OK) return st;
    sg_cost_model dflt = kDefaultModel;
    dflt.tiles_fixed = default_range_floor(B->ncols);
    const sg_cost_model* c = cm ? cm : &dflt;
    if ((st = check_model(c)) != SG_OK) return st;
    if (nrows == 0) return SG_ERR_EMPTY_SAMPLE;
    {
        Scratch sc(s);
        unsigned long long* bad = (unsigned long long*)sc.get(sizeof(unsigned long long));
        if (!bad) return SG_ERR_OOM;
        unsigned long long hb = 0;
        CK(cudaMemsetAsync(bad, 0, sizeof(unsigned long long), s));
        CK(launch_check_rows(rows, nrows, A->nrows, bad, s));
        CK(cudaMemcpyAsync(&hb, bad, sizeof(hb), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (hb) return SG_ERR_INVALID_ARG;
    }
    ThrResult r;
    st = identify(mat_of(A), mat_of(B), rows, nrows, c, &r, s);
    if (st != SG_OK) return st;
    if (r.nonempty == 0) return SG_ERR_EMPTY_SAMPLE;
    *thr_out = r.thr;
    if (rep) {
        rep->sample_rows = nrows;
        rep->sample_nonempty = r.nonempty;
        rep->thr = r.thr;
        rep->W_est_L = r.W_L;
        rep->W_est_H = r.W_all - r.W_L;
        rep->J_min = r.Jmin;
        rep->U_est_L = r.U_L;
        rep->U_est_H = r.U_H;
    }
    return SG_OK;
}

sg_status sg_exhaustive_threshold(const sg_csr_view* A, const sg_csr_view* B, const sg_cost_model* cm,
                                  int64_t* thr_out, int64_t* J_min_out, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    init_pool();
    if (!thr_out) return SG_ERR_INVALID_ARG;
    sg_status st = validate_pair(A, B, s);
    if (st != SG_OK) return st;
    sg_cost_model dflt = kDefaultModel;
    dflt.tiles_fixed = default_range_floor(B->ncols);
    const sg_cost_model* c = cm ? cm : &dflt;
    if ((st = check_model(c)) != SG_OK) return st;
    ThrResult r;
    st = identify(mat_of(A), mat_of(B), nullptr, A->nrows, c, &r, s);
    if (st != SG_OK) return st;
    *thr_out = r.thr;
    if (J_min_out) *J_min_out = r.Jmin;
    return SG_OK;
}

sg_status sg_cost_curve(const sg_csr_view* A, const sg_csr_view* B, const sg_cost_model* cm, int64_t nt,
                        const int64_t* t_host, int64_t* J_host, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    init_pool();
    if (nt < 0 || (nt > 0 && (!t_host || !J_host))) return SG_ERR_INVALID_ARG;
    sg_status st = validate_pair(A, B, s);
    if (st != SG_OK) return st;
    sg_cost_model dflt = kDefaultModel;
    dflt.tiles_fixed = default_range_floor(B->ncols);
    const sg_cost_model* c = cm ? cm : &dflt;
    if ((st = check_model(c)) != SG_OK) return st;
    Scratch sc(s);
    RowStats rs;
    Mat a = mat_of(A), b = mat_of(B);
    st = row_stats(a, b, nullptr, A->nrows, c->cap_L, sc, rs, s);
    if (st != SG_OK) return st;
    if ((st = check_cost_bound(cm_of(c), rs, A->nrows, sc, s)) != SG_OK) return st;
    int64_t* dt = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(nt > 0 ? nt : 1));
    long long* dJ = (long long*)sc.get(sizeof(long long) * (size_t)(nt > 0 ? nt : 1));
    if (!dt || !dJ) return SG_ERR_OOM;
    if (nt > 0) {
        CK(cudaMemcpyAsync(dt, t_host, sizeof(int64_t) * (size_t)nt, cudaMemcpyHostToDevice, s));
        CK(launch_cost_curve(cm_of(c), rs.w, rs.a, rs.u, A->nrows, dt, (int)nt, dJ, s));
        CK(cudaMemcpyAsync(J_host, dJ, sizeof(long long) * (size_t)nt, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
    }
    return SG_OK;
}

sg_status sg_partition(const sg_csr_view* A, const sg_csr_view* B, int nparts, int64_t* cuts_out, int64_t* flops_out,
                       void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    init_pool();
    if (nparts < 1 || !cuts_out) return SG_ERR_INVALID_ARG;
    sg_status st = validate_pair(A, B, s);
    if (st != SG_OK) return st;
    const int64_t n = A->nrows;
    Scratch sc(s);
    int64_t* w = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    int64_t* P = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(n + 1));
    void* tmp = sc.get(scan_tmp_bytes(n));
    int64_t* dcuts = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(nparts + 1));
    if (!w || !P || !tmp || !dcuts) return SG_ERR_OOM;
    Mat a = mat_of(A), b = mat_of(B);
    CK(launch_row_work(a, b, 0, n, w, s));
    CK(scan_exclusive(w, P, n, tmp, s));
    CK(launch_cuts(P, n, nparts, dcuts, s));
    CK(cudaMemcpyAsync(cuts_out, dcuts, sizeof(int64_t) * (size_t)(nparts + 1), cudaMemcpyDeviceToHost, s));
    int64_t W = 0;
    CK(cudaMemcpyAsync(&W, P + n, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (flops_out) *flops_out = W;
    return SG_OK;
}

sg_status sg_partition_cost(const sg_csr_view* A, const sg_csr_view* B, int nparts, int64_t thr,
                            const sg_cost_model* cm, const int64_t* comp, int64_t* cuts_out, int64_t* cost_out,
                            void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    init_pool();
    if (nparts < 1 || !cuts_out || !comp || thr < 0) return SG_ERR_INVALID_ARG;
    for (int q = 0; q < 4; ++q)
        if (comp[q] < 0) return SG_ERR_INVALID_ARG;
    sg_status st = validate_pair(A, B, s);
    if (st != SG_OK) return st;
    const sg_cost_model* c = cm ? cm : &kPartitionModel;
    if ((st = check_model(c)) != SG_OK) return st;
    const int64_t n = A->nrows;
    Scratch sc(s);
    int64_t* w = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    int64_t* cost = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    int64_t* P = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(n + 1));
    void* tmp = sc.get(scan_tmp_bytes(n));
    int64_t* dcuts = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(nparts + 1));
    double* dm = (double*)sc.get(sizeof(double));
    if (!w || !cost || !P || !tmp || !dcuts || !dm) return SG_ERR_OOM;
    Mat a = mat_of(A), b = mat_of(B);
    CK(launch_row_work(a, b, 0, n, w, s));
    CK(launch_row_cost(cm_of(c), thr, comp, A->row_ptr, w, n, cost, dm, s));
    {
        double hm = 0.0;
        CK(cudaMemcpyAsync(&hm, dm, sizeof(double), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (hm >= kCostLimit) return SG_ERR_OVERFLOW;
    }
    CK(scan_exclusive(cost, P, n, tmp, s));
    CK(launch_cuts(P, n, nparts, dcuts, s));
    CK(cudaMemcpyAsync(cuts_out, dcuts, sizeof(int64_t) * (size_t)(nparts + 1), cudaMemcpyDeviceToHost, s));
    int64_t tot = 0;
    CK(cudaMemcpyAsync(&tot, P + n, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (cost_out) *cost_out = tot;
    return SG_OK;
}

sg_status sg_symbolic(const sg_csr_view* A, const sg_csr_view* B, int64_t thr, int64_t row_begin, int64_t row_end,
                      int64_t* C_row_ptr, int64_t* nnz_c_out, sg_plan** plan_out, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    init_pool();
    if (!C_row_ptr || !nnz_c_out || !plan_out) return SG_ERR_INVALID_ARG;
    if (thr < 0 || thr > SG_CAP_L_MAX) return SG_ERR_INVALID_ARG;
    sg_status st = validate_pair(A, B, s);
    if (st != SG_OK) return st;
    if (row_begin < 0 || row_end < row_begin || row_end > A->nrows) return SG_ERR_INVALID_ARG;
    sg_plan* pl = new sg_plan();
    pl->s = s;
    pl->variant = variant_bits();
    pl->rb = row_begin; pl->re = row_end; pl->nr = row_end - row_begin; pl->thr = thr;
    pl->p = B->ncols; pl->m = B->nrows; pl->dt = (int)A->dtype;
    pl->C_rp = C_row_ptr;
    const int64_t nr = pl->nr;
    Mat a = mat_of(A), b = mat_of(B);
    L2Window l2w(s, b.col, 4 * (size_t)b.nnz);
    auto fail = [&](sg_status e) { pl->poisoned = true; sg_plan_destroy(pl); return e; };
    size_t nrb = (size_t)(nr > 0 ? nr : 1);
    pl->w = (int64_t*)palloc(pl, 8 * nrb);
    pl->cls = (int8_t*)palloc(pl, nrb);
    pl->lists = (int32_t*)palloc(pl, 4 * nrb);
    pl->u = (int64_t*)palloc(pl, 8 * nrb);
    pl->dbin = (int64_t*)palloc(pl, sizeof(int64_t) * (2 * NBINS + 2));
    pl->long_id = (int32_t*)palloc(pl, 4 * (size_t)(pl->m > 0 ? pl->m : 1));
    pl->counter = (unsigned long long*)palloc(pl, sizeof(unsigned long long) * 2);
    pl->span = (int2*)palloc(pl, sizeof(int2) * nrb);
    void* stmp = palloc(pl, scan_tmp_bytes(nr + 1));
    if (!pl->w || !pl->cls || !pl->lists || !pl->u || !pl->dbin || !pl->long_id || !pl->counter || !pl->span || !stmp)
        return fail(SG_ERR_OOM);
    if (B->nnz >= INT32_MAX) return fail(SG_ERR_OVERFLOW);  // heavy cursors hold B positions in int32
    pl->T = (int)((pl->p + TW - 1) / TW);
    if (pl->T < 1) pl->T = 1;
#define CKF(x) do { if ((x) != cudaSuccess) { cudaGetLastError(); return fail(SG_ERR_CUDA); } } while (0)
    // a1 row work, a5 classes + bin counts, long rows of B
    CKF(launch_row_work(a, b, row_begin, row_end, pl->w, s));
    CKF(cudaMemsetAsync(pl->dbin, 0, sizeof(int64_t) * (2 * NBINS + 2), s));
    CKF(cudaMemsetAsync(pl->u, 0, 8 * nrb, s));
    CKF(launch_bin_count(pl->w, nr, thr, pl->dbin, pl->cls, s));
    CKF(launch_long_rows(b, pl->long_id, pl->dbin + NBINS, s));
    int64_t hc[NBINS + 1];
    CKF(cudaMemcpyAsync(hc, pl->dbin, sizeof(hc), cudaMemcpyDeviceToHost, s));
    CKF(cudaStreamSynchronize(s));
    pl->bin_off[0] = 0;
    for (int k = 0; k < NBINS; ++k) { pl->bin_cnt[k] = hc[k]; pl->bin_off[k + 1] = pl->bin_off[k] + hc[k]; }
    pl->nlong = hc[NBINS];
    CKF(cudaMemcpyAsync(pl->dbin + NBINS + 1, pl->bin_off, sizeof(int64_t) * NBINS, cudaMemcpyHostToDevice, s));
    CKF(launch_bin_scatter(pl->w, nr, thr, pl->dbin + NBINS + 1, pl->lists, s));
    // heavy rows heaviest-first, range-slot bounds -> offsets, B tile pointers
    pl->nheavy = pl->bin_cnt[BIN_HEAVY];
    if (pl->nheavy > 0) {
        pl->heavy = (int32_t*)palloc(pl, 4 * (size_t)pl->nheavy);
        unsigned int* hist = (unsigned int*)palloc(pl, 128 * sizeof(unsigned int));
        pl->range_bounds = (int64_t*)palloc(pl, 8 * (size_t)pl->nheavy);
        pl->range_off = (int64_t*)palloc(pl, 8 * (size_t)(pl->nheavy + 1));
        pl->nranges = (int32_t*)palloc(pl, 4 * (size_t)pl->nheavy);
        void* t2 = palloc(pl, scan_tmp_bytes(pl->nheavy));
        if (!pl->heavy || !hist || !pl->range_bounds || !pl->range_off || !pl->nranges || !t2) return fail(SG_ERR_OOM);
        CKF(launch_heavy_order(pl->lists + pl->bin_off[BIN_HEAVY], pl->nheavy, pl->w, hist, pl->heavy, s));
        // dense-window rows: w >= 2^dw_log2, a prefix of the heaviest-first order
        init_options();
        pl->dw_log2 = dense_window_log2(pl->p, g_opt[SG_OPT_DENSE_LOG2].load());
        const int64_t dw_min_w = pl->dw_log2 >= 62 ? INT64_MAX : ((int64_t)1 << pl->dw_log2);
        CKF(launch_range_bounds(pl->heavy, pl->nheavy, pl->w, pl->p, dw_min_w, pl->range_bounds, s));
        CKF(scan_exclusive(pl->range_bounds, pl->range_off, pl->nheavy, t2, s));
        CKF(cudaMemsetAsync(pl->counter + 1, 0, sizeof(unsigned long long), s));
        CKF(launch_max_a(a, pl->heavy, pl->nheavy, row_begin, pl->counter + 1, s));
        int64_t hb[2];
        unsigned int hh[64];
        CKF(cudaMemcpyAsync(&hb[0], pl->range_off + pl->nheavy, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        CKF(cudaMemcpyAsync(&hb[1], pl->counter + 1, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        CKF(cudaMemcpyAsync(hh, hist, sizeof(hh), cudaMemcpyDeviceToHost, s));
        CKF(cudaStreamSynchronize(s));
        // heavy order bucket b = 62 - floor(log2 w) (ascending = heaviest first): w >= 2^m <=> b <= 62 - m
        pl->ndw = 0;
        for (int hb2 = 0; hb2 <= 62 - pl->dw_log2 && hb2 < 64; ++hb2) pl->ndw += hh[hb2];
        // rows with w >= 2^20 take the 1024-thread symbolic kernel (one such row must not be a tail)
        pl->nbig = 0;
        for (int hb2 = 0; hb2 <= 62 - 20; ++hb2) pl->nbig += hh[hb2];
        if (pl->ndw > 0) {
            pl->dtc = (int32_t*)palloc(pl, sizeof(int32_t) * (size_t)pl->ndw * (size_t)pl->T);
            pl->ditems = (int4*)palloc(pl, sizeof(int4) * (size_t)dense_items_bound(pl->ndw, pl->p));
            pl->ditem_off = (int64_t*)palloc(pl, sizeof(int64_t) * (size_t)(pl->ndw + 1));
            int64_t* dcnt = (int64_t*)palloc(pl, sizeof(int64_t) * (size_t)pl->ndw);
            void* t3 = palloc(pl, scan_tmp_bytes(pl->ndw));
            if (!pl->dtc || !pl->ditems || !pl->ditem_off || !dcnt || !t3) return fail(SG_ERR_OOM);
            if (pl->variant & 4)  // round-1 items: row chunks of <= 2^19 products, row-major
                CKF(launch_dense_items(pl->heavy, pl->ndw, pl->w, pl->p, dcnt, pl->ditem_off, t3, pl->ditems, s));
            else  // window-major blocks (sg_dense.cu); the item count goes where the kernels read it
                CKF(launch_dense_items_wm(pl->ndw, pl->p, pl->ditems, pl->ditem_off + pl->ndw, s));
        }
        pl->nslots = hb[0];
        pl->amax = hb[1];
        pl->ranges = (RangeRec*)palloc(pl, sizeof(RangeRec) * (size_t)(pl->nslots > 0 ? pl->nslots : 1));
        // the tile-pointer table grows with (long B rows) x (tiles): over its budget the heavy kernels binary-search
        // (the round-1 dense / symbolic kernels of SG_OPT_VARIANT bits 0-1 need the table: built regardless)
        {
            const int64_t opt = g_opt[SG_OPT_TP_MAX_BYTES].load();
            const double budget = opt < 0 ? 8.0 * (1 << 30) : (double)opt;
            const double need = 4.0 * (double)pl->nlong * (double)(pl->T + 1);
            // ... and a table for a handful of heavy rows costs more than their binary searches (C2 at t = 512:
            // 97 heavy rows, 262 K long B rows): build it when the heavy rows' tile lookups (~ nheavy x T)
            // are at least a quarter of the long rows it covers
            const bool few = (double)pl->nheavy * (double)pl->T < 0.25 * (double)pl->nlong;
            if ((need > budget || few) && !(pl->variant & 3)) pl->nlong_tp = 0;
            else pl->nlong_tp = pl->nlong;
        }
        pl->tp = (uint32_t*)palloc(pl, 4 * (size_t)(pl->nlong_tp > 0 ? pl->nlong_tp : 1) * (size_t)(pl->T + 1));
        if (!pl->ranges || !pl->tp) return fail(SG_ERR_OOM);
        // unused range slots read as row -1 (the tile kernel walks every slot)
        CKF(cudaMemsetAsync(pl->ranges, 0xff, sizeof(RangeRec) * (size_t)(pl->nslots > 0 ? pl->nslots : 1), s));
        if (pl->ndw > 0 && pl->amax + 32 > dense2_pcap()) {
            pl->pscr_cap = pl->amax + 32;
            pl->pscr = palloc(pl, dense2_part_bytes() * (size_t)pl->pscr_cap * 148);
            if (!pl->pscr) return fail(SG_ERR_OOM);
        }
        if (pl->amax > heavy_kc() || pl->amax > dense_kc()) {
            pl->gscr = (int4*)palloc(pl, sizeof(int4) * (size_t)(heavy_grid() > dense_grid() ? heavy_grid() : dense_grid()) * (size_t)pl->amax);
            if (!pl->gscr) return fail(SG_ERR_OOM);
        }
        if (pl->nlong_tp > 0) CKF(launch_build_tp(b, pl->long_id, pl->T, pl->tp, s));
    }
    // a6 symbolic. Light bins on the sorted path sort their rows' column keys here and keep them for the
    // numeric pass (one slot of light_sort_width(b) keys per row, bin by bin); the others count with a hash set.
    {
        int64_t nkeys = 0;
        for (int k = 0; k < NBIN_LIGHT; ++k) {
            pl->lkey_off[k] = nkeys;
            if (light_sorted(k, pl->p, pl->variant)) nkeys += pl->bin_cnt[k] * (int64_t)light_sort_width(k);
        }
        if (nkeys > 0) {
            pl->lkeys = (uint32_t*)palloc(pl, 4 * (size_t)nkeys);
            if (!pl->lkeys) return fail(SG_ERR_OOM);
        }
    }
    for (int k = 0; k < NBIN_LIGHT; ++k) {
        if (light_sorted(k, pl->p, pl->variant))
            CKF(launch_sym_light_sort(k, a, b, pl->lists + pl->bin_off[k], pl->bin_cnt[k], row_begin,
                                      pl->lkeys + pl->lkey_off[k], pl->u, s));
        else
            CKF(launch_sym_light(k, a, b, pl->lists + pl->bin_off[k], pl->bin_cnt[k], nullptr, row_begin, pl->u, pl->span,
                                 (unsigned long long*)(pl->dbin + 2 * NBINS + 1), s));
    }
    if (pl->variant & 2) {
        CKF(launch_sym_heavy(a, b, pl->heavy, pl->nheavy, nullptr, row_begin, pl->u, pl->range_off, pl->ranges,
                             pl->nranges, pl->ndw, pl->dtc, pl->long_id, pl->nlong_tp > 0 ? pl->tp : nullptr, pl->T,
                             pl->counter, s, pl->nbig));
    } else if (pl->nheavy > 0) {
        const int64_t np = sym2_scratch_parts(pl->amax);
        void* pscr = np > 0 ? palloc(pl, part_bytes() * (size_t)np) : nullptr;
        if (np > 0 && !pscr) return fail(SG_ERR_OOM);
        CKF(launch_sym_heavy2(a, b, pl->heavy, pl->nheavy, nullptr, row_begin, pl->w, pl->u, pl->range_off, pl->ranges,
                              pl->nranges, pl->ndw, pl->dtc, pl->long_id, pl->nlong_tp > 0 ? pl->tp : nullptr, pl->T,
                              pl->counter, s, pl->nbig, pscr, pl->amax));
    }
    CKF(scan_exclusive(pl->u, C_row_ptr, nr, stmp, s));
    CKF(cudaMemcpyAsync(&pl->nnz_c, C_row_ptr + nr, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CKF(cudaMemcpyAsync(&pl->nskew, pl->dbin + 2 * NBINS + 1, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CKF(cudaStreamSynchronize(s));
#undef CKF
    *nnz_c_out = pl->nnz_c;
    *plan_out = pl;
    return SG_OK;
}

sg_status sg_numeric(sg_plan* pl, const sg_csr_view* A, const sg_csr_view* B, int32_t* C_col, void* C_val,
                     void* stream) {
    if (!pl) return SG_ERR_INVALID_ARG;
    if (pl->poisoned) return SG_ERR_CUDA;
    cudaStream_t s = (cudaStream_t)stream;
    if (!A || !B) return SG_ERR_INVALID_ARG;
    if (A->nrows < pl->re || B->ncols != pl->p || B->nrows != pl->m) return SG_ERR_SHAPE;
    if ((int)A->dtype != pl->dt || (int)B->dtype != pl->dt) return SG_ERR_DTYPE;
    if (pl->nnz_c > 0 && (!C_col || !C_val)) return SG_ERR_INVALID_ARG;
    if (((uintptr_t)C_col & 3u) || ((uintptr_t)C_val & (pl->dt == 0 ? 7u : 3u))) return SG_ERR_INVALID_ARG;
    if (pl->nnz_c == 0) return SG_OK;
    Mat a = mat_of(A), b = mat_of(B);
    L2Window l2w(s, b.col, 4 * (size_t)b.nnz);
    for (int k = 0; k < NBIN_LIGHT; ++k) {
        if (light_sorted(k, pl->p, pl->variant))
            CKP(pl, launch_num_light_keys(k, a, b, pl->lists + pl->bin_off[k], pl->bin_cnt[k], pl->rb,
                                          pl->lkeys + pl->lkey_off[k], pl->C_rp, C_col, C_val, s));
        else
            CKP(pl, launch_num_light(k, a, b, pl->lists + pl->bin_off[k], pl->bin_cnt[k], pl->rb, pl->span, pl->C_rp,
                                     C_col, C_val, s));
    }
    if (pl->nheavy > 0) {
        if (pl->variant & 1)
            CKP(pl, launch_num_dense(a, b, pl->heavy, pl->ndw, pl->rb, pl->long_id, pl->nlong_tp > 0 ? pl->tp : nullptr, pl->T, pl->C_rp, C_col,
                                     C_val, pl->counter, pl->gscr, pl->amax, pl->dtc, pl->ditems, pl->ditem_off + pl->ndw, s));
        else
            CKP(pl, launch_num_dense2(a, b, pl->heavy, pl->ndw, pl->rb, pl->w, pl->long_id, pl->nlong_tp > 0 ? pl->tp : nullptr, pl->T, pl->C_rp, C_col,
                                      C_val, pl->counter, pl->pscr, pl->pscr_cap, pl->dtc, pl->ditems,
                                      pl->ditem_off + pl->ndw, s));
        // rank rows: the CTA rank kernel takes the rows with more than tile_kreg() k entries, the warp-tile
        // kernel the rest (SG_OPT_VARIANT bit 3: the CTA kernel takes all of them)
        // (a few rank rows: the CTA kernel for all of them, its 16 warps per range shorten the latency tail
        // of a warp walking a range's tiles alone)
        const bool tile = !(pl->variant & 8) && (pl->nheavy - pl->ndw >= kTileMinRows || (pl->variant & 32));
        CKP(pl, launch_num_heavy(a, b, pl->heavy, pl->ndw, pl->nheavy, pl->rb, pl->range_off, pl->nranges, pl->ranges,
                                 pl->long_id, pl->nlong_tp > 0 ? pl->tp : nullptr, pl->T, pl->C_rp, C_col, C_val,
                                 pl->counter, pl->gscr, pl->amax,
                                 tile ? (int)tile_kreg() : 0, s));
        if (tile && pl->nheavy > pl->ndw)
            CKP(pl, launch_num_tile(a, b, pl->ranges, pl->nslots, pl->rb, pl->long_id, pl->nlong_tp > 0 ? pl->tp : nullptr,
                                    pl->T, pl->C_rp, C_col, C_val, pl->counter, s));
    }
    if (s != pl->s) {  // the plan's workspace frees (on pl->s) wait for this call's kernels
        cudaEvent_t ev;
        CKP(pl, cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
        CKP(pl, cudaEventRecord(ev, s));
        CKP(pl, cudaStreamWaitEvent(pl->s, ev, 0));
        cudaEventDestroy(ev);
    }
    return SG_OK;
}

sg_status sg_plan_get_info(const sg_plan* pl, sg_plan_info* out) {
    if (!pl || !out) return SG_ERR_INVALID_ARG;
    if (pl->poisoned) return SG_ERR_CUDA;
    memset(out, 0, sizeof(*out));
    out->row_begin = pl->rb; out->row_end = pl->re; out->thr = pl->thr;
    out->n_empty = pl->bin_cnt[BIN_EMPTY];
    out->n_heavy = pl->bin_cnt[BIN_HEAVY];
    for (int k = 0; k < NBIN_LIGHT; ++k) { out->light_bins[k] = pl->bin_cnt[k]; out->n_light += pl->bin_cnt[k]; }
    out->nnz_c = pl->nnz_c;
    out->n_ranges = pl->nslots;
    out->n_dense = pl->ndw;
    out->n_light_sorted = pl->nskew;
    out->dense_log2 = pl->dw_log2;
    // flops on demand
    if (pl->nr > 0) {
        cudaStream_t s = pl->s;
        Scratch sc(s);
        int64_t* P = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(pl->nr + 1));
        void* tmp = sc.get(scan_tmp_bytes(pl->nr));
        if (!P || !tmp) return SG_ERR_OOM;
        CK(scan_exclusive(pl->w, P, pl->nr, tmp, s));
        CK(cudaMemcpyAsync(&out->flops, P + pl->nr, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
    }
    return SG_OK;
}

sg_status sg_plan_get_classes(const sg_plan* pl, int8_t* cls_out, void* stream) {
    if (!pl || (!cls_out && pl->nr > 0)) return SG_ERR_INVALID_ARG;
    if (pl->poisoned) return SG_ERR_CUDA;
    if (pl->nr > 0)
        CK(cudaMemcpyAsync(cls_out, pl->cls, (size_t)pl->nr, cudaMemcpyDeviceToDevice, (cudaStream_t)stream));
    return SG_OK;
}

sg_status sg_plan_get_work(const sg_plan* pl, int64_t* w_out, void* stream) {
    if (!pl || (!w_out && pl->nr > 0)) return SG_ERR_INVALID_ARG;
    if (pl->poisoned) return SG_ERR_CUDA;
    if (pl->nr > 0)
        CK(cudaMemcpyAsync(w_out, pl->w, 8 * (size_t)pl->nr, cudaMemcpyDeviceToDevice, (cudaStream_t)stream));
    return SG_OK;
}

// ---- NEXT #4: HH-CPU four blocks (PAPER Alg. 3, Section V-A; sg_hh.cu) --------
sg_status sg_hh_filter(const sg_csr_view* M, int64_t t, int high, int64_t* rp_out, int32_t* col_out, void* val_out,
                       int64_t* nnz_out, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    init_pool();
    sg_status st = validate_one(M, s);
    if (st != SG_OK) return st;
    if (!rp_out || !nnz_out || (M->nnz > 0 && (!col_out || !val_out))) return SG_ERR_INVALID_ARG;
    Mat m = mat_of(M);
    const int64_t n = M->nrows;
    Scratch sc(s);
    int64_t* len = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    void* tmp = sc.get(scan_tmp_bytes(n));
    if (!len || !tmp) return SG_ERR_OOM;
    CK(launch_hh_len(m, t, high, len, s));
    CK(scan_exclusive(len, rp_out, n, tmp, s));
    CK(launch_hh_copy(m, rp_out, col_out, val_out, s));
    int64_t nnz = 0;
    CK(cudaMemcpyAsync(&nnz, rp_out + n, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    *nnz_out = nnz;
    return SG_OK;
}

sg_status sg_hh_hstack(const sg_csr_view* P, const sg_csr_view* Q, int64_t* rp_out, int32_t* col_out, void* val_out,
                       void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    init_pool();
    sg_status st;
    if ((st = validate_one(P, s)) != SG_OK || (st = validate_one(Q, s)) != SG_OK) return st;
    if (P->nrows != Q->nrows) return SG_ERR_SHAPE;
    if (P->dtype != Q->dtype) return SG_ERR_DTYPE;
    if (P->ncols + Q->ncols > INT32_MAX) return SG_ERR_OVERFLOW;
    if (!rp_out || (P->nnz + Q->nnz > 0 && (!col_out || !val_out))) return SG_ERR_INVALID_ARG;
    Mat mp = mat_of(P), mq = mat_of(Q);
    const int64_t n = P->nrows;
    Scratch sc(s);
    int64_t* len = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    void* tmp = sc.get(scan_tmp_bytes(n));
    if (!len || !tmp) return SG_ERR_OOM;
    CK(launch_hh_hstack(mp, mq, len, nullptr, nullptr, 0, s));
    CK(scan_exclusive(len, rp_out, n, tmp, s));
    CK(launch_hh_hstack(mp, mq, rp_out, col_out, val_out, 1, s));
    return SG_OK;
}

sg_status sg_hh_identity2(int64_t p, sg_dtype dtype, int64_t* rp_out, int32_t* col_out, void* val_out, void* stream) {
    if (p < 0 || 2 * p > INT32_MAX || !rp_out || (p > 0 && (!col_out || !val_out))) return SG_ERR_INVALID_ARG;
    if (dtype != SG_F64 && dtype != SG_F32) return SG_ERR_DTYPE;
    init_pool();
    CK(launch_hh_identity2(p, (int)dtype, rp_out, col_out, val_out, (cudaStream_t)stream));
    return SG_OK;
}

sg_status sg_hh_sample(const sg_csr_view* A, uint64_t seed, double f, int64_t* rows_out, int64_t* rp_out,
                       int32_t* col_out, int64_t* pos_out, void* val_out, int64_t* s_out, int64_t* nnz_out, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    init_pool();
    sg_status st = validate_one(A, s);
    if (st != SG_OK) return st;
    if (A->nrows != A->ncols) return SG_ERR_SHAPE;  // a principal sub-matrix needs a square A
    if (!(f > 0.0 && f <= 1.0) || !rows_out || !rp_out || !s_out || !nnz_out ||
        (A->nnz > 0 && (!col_out || !pos_out)))
        return SG_ERR_INVALID_ARG;
    Mat m = mat_of(A);
    const int64_t n = A->nrows;
    Scratch sc(s);
    int64_t* keep = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    int64_t* rank = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(n + 1));
    int64_t* cnt = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    void* tmp = sc.get(scan_tmp_bytes(n));
    if (!keep || !rank || !cnt || !tmp) return SG_ERR_OOM;
    const bool all = f >= 1.0;
    const uint64_t Tf = all ? 0 : (uint64_t)std::ldexp(f, 64);
    CK(launch_hh_mask(n, seed, Tf, all ? 1 : 0, keep, s));
    CK(scan_exclusive(keep, rank, n, tmp, s));
    int64_t sr = 0;
    CK(cudaMemcpyAsync(&sr, rank + n, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    CK(launch_hh_rows_of_rank(n, keep, rank, rows_out, s));
    CK(launch_hh_sub(m, keep, rank, rows_out, sr, cnt, nullptr, nullptr, nullptr, 0, s));
    CK(scan_exclusive(cnt, rp_out, sr, tmp, s));
    CK(launch_hh_sub(m, keep, rank, rows_out, sr, rp_out, col_out, pos_out, val_out, 1, s));
    int64_t nz = 0;
    CK(cudaMemcpyAsync(&nz, rp_out + sr, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    *s_out = sr;
    *nnz_out = nz;
    return SG_OK;
}

sg_status sg_gather_rows(const sg_csr_view* A, const int64_t* rows, int64_t nrows, int64_t* rp_out, int32_t* col_out,
                         void* val_out, int64_t cap, int64_t* nnz_out, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    init_pool();
    sg_status st = validate_one(A, s);
    if (st != SG_OK) return st;
    if (nrows < 0 || cap < 0 || !rp_out || !nnz_out || (nrows > 0 && !rows)) return SG_ERR_INVALID_ARG;
    Mat m = mat_of(A);
    {
        Scratch sc(s);  // row ids in range (one flag read back)
        unsigned long long* bad = (unsigned long long*)sc.get(sizeof(unsigned long long));
        if (!bad) return SG_ERR_OOM;
        unsigned long long hb = 0;
        CK(cudaMemsetAsync(bad, 0, sizeof(unsigned long long), s));
        CK(launch_check_rows(rows, nrows, A->nrows, bad, s));
        CK(cudaMemcpyAsync(&hb, bad, sizeof(hb), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (hb) return SG_ERR_INVALID_ARG;
    }
    Scratch sc(s);
    int64_t* len = (int64_t*)sc.get(sizeof(int64_t) * (size_t)(nrows > 0 ? nrows : 1));
    void* tmp = sc.get(scan_tmp_bytes(nrows));
    if (!len || !tmp) return SG_ERR_OOM;
    CK(launch_rows_len(m, rows, nrows, len, s));
    CK(scan_exclusive(len, rp_out, nrows, tmp, s));
    int64_t nz = 0;
    CK(cudaMemcpyAsync(&nz, rp_out + nrows, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    *nnz_out = nz;
    if (nz > cap) return SG_ERR_SHAPE;
    if (nz > 0 && (!col_out || !val_out)) return SG_ERR_INVALID_ARG;
    CK(launch_rows_copy(m, rows, nrows, rp_out, col_out, val_out, s));
    return SG_OK;
}

sg_status sg_copy_device(void* dst, const void* src, int64_t bytes, void* stream) {
    if (bytes < 0 || (bytes > 0 && (!dst || !src))) return SG_ERR_INVALID_ARG;
    if (bytes == 0) return SG_OK;
    CK(cudaMemcpyAsync(dst, src, (size_t)bytes, cudaMemcpyDeviceToDevice, (cudaStream_t)stream));
    return SG_OK;
}

void sg_plan_destroy(sg_plan* pl) {
    if (!pl) return;
    for (void* p : pl->allocs) cudaFreeAsync(p, pl->s);
    pl->allocs.clear();
    delete pl;
}

// internal accessors for sg_gather.cu
int64_t sg_internal_plan_rows(const sg_plan* pl, int64_t* rb, int64_t* re) {
    *rb = pl->rb; *re = pl->re;
    return pl->nnz_c;
}
int sg_internal_plan_dtype(const sg_plan* pl) { return pl->dt; }
bool sg_internal_plan_poisoned(const sg_plan* pl) { return pl->poisoned; }
void sg_internal_plan_poison(sg_plan* pl) { pl->poisoned = true; }

}  // extern "C"
