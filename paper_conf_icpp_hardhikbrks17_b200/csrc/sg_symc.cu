// sg_symc.cu — NEXT #3: assembly of the row-distributed C (Alg. 2 l.7: "Transfer
// results ... and add that to CPU's results") through NCCL 2.28 symmetric memory instead of collectives.
//
// The assembled C (row_ptr, col, val) lives in NCCL symmetric windows (ncclMemAlloc +
// ncclCommWindowRegister(NCCL_WIN_COLL_SYMMETRIC)) on every rank of the communicator. After the
// symbolic phase each rank learns where its rows go (one ncclAllGather of (row_begin, row_end, nnz));
// its sg_numeric then writes its rows STRAIGHT INTO ITS OWN WINDOW at that offset (the numeric epilogue
// is the local half of the transfer), and one kernel (k_symc_push) stores the rank's rows into every
// LSA peer's window over NVLink with plain st.global through the peer pointers ncclGetLsaPointer gives
// (row_ptr entries get the rank's global offset added on the way), closed by an LSA barrier so that all
// ranks' stores are complete when the kernel is. No NCCL collective moves C.
#include "sg_internal.cuh"
#include <nccl.h>
#include <nccl_device.h>
#include <vector>

extern "C" {
int64_t sg_internal_plan_rows(const sg_plan* pl, int64_t* rb, int64_t* re);
int sg_internal_plan_dtype(const sg_plan* pl);
bool sg_internal_plan_poisoned(const sg_plan* pl);
}

struct sg_sym_c {
    ncclComm_t comm = nullptr;
    int nranks = 0, rank = 0, dt = 0;
    int64_t n = 0, cap = 0;
    void* buf[3] = {nullptr, nullptr, nullptr};    // row_ptr int64[n+1], col int32[cap], val dtype[cap]
    size_t bytes[3] = {0, 0, 0};
    ncclWindow_t win[3] = {nullptr, nullptr, nullptr};
    ncclDevComm dev{};
    bool dev_ok = false;
    int64_t off = -1, total = -1;                  // this rank's first global C entry; nnz of the assembled C
    int64_t rb = 0, re = 0, nnz = 0;
};

namespace {

constexpr int SYMC_BLOCKS = 148;   // CTAs of the push kernel = LSA barriers requested
constexpr int SYMC_T = 512;

__global__ void __launch_bounds__(SYMC_T) k_symc_push(ncclDevComm dev, ncclWindow_t wrp, ncclWindow_t wcol,
                                                       ncclWindow_t wval, const int64_t* __restrict__ local_rp,
                                                       int64_t rb, int64_t nrows, int64_t off, int64_t nnz, int vsize,
                                                       int last, int64_t n_global) {
    const ncclTeam lsa = ncclTeamLsa(dev);
    const int me = lsa.rank;
    // this rank's slice of col / val already sits in its own window at [off, off + nnz); row_ptr still local
    const int32_t* mycol = (const int32_t*)ncclGetLsaPointer(wcol, (size_t)off * 4, me);
    const char* myval = (const char*)ncclGetLsaPointer(wval, (size_t)off * vsize, me);
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x, nth = (int64_t)gridDim.x * blockDim.x;
    for (int pr = 0; pr < lsa.nRanks; ++pr) {
        int64_t* rp = (int64_t*)ncclGetLsaPointer(wrp, (size_t)rb * 8, pr);
        for (int64_t i = tid; i < nrows; i += nth) rp[i] = local_rp[i] + off;
        if (last && tid == 0) rp[nrows] = off + nnz;  // row_ptr[n] = total (written by the last rank)
        if (pr == me) continue;                       // col / val are in place in the own window
        int32_t* col = (int32_t*)ncclGetLsaPointer(wcol, (size_t)off * 4, pr);
        for (int64_t e = tid; e < nnz; e += nth) col[e] = mycol[e];
        if (vsize == 8) {
            double* v = (double*)ncclGetLsaPointer(wval, (size_t)off * 8, pr);
            for (int64_t e = tid; e < nnz; e += nth) v[e] = ((const double*)myval)[e];
        } else {
            float* v = (float*)ncclGetLsaPointer(wval, (size_t)off * 4, pr);
            for (int64_t e = tid; e < nnz; e += nth) v[e] = ((const float*)myval)[e];
        }
    }
    (void)n_global;
    // every rank's CTA b has stored its share into every window before any CTA b passes
    ncclLsaBarrierSession<ncclCoopCta> bar(ncclCoopCta(), dev, ncclTeamTagLsa(), blockIdx.x);
    bar.sync(ncclCoopCta(), cuda::memory_order_acq_rel);
}

}  // namespace

extern "C" {

sg_status sg_sym_c_create(void* nccl_comm, int64_t n_rows, int64_t nnz_cap, sg_dtype dtype, sg_sym_c** out) {
    if (!nccl_comm || !out || n_rows < 0 || nnz_cap < 0 || (dtype != SG_F64 && dtype != SG_F32)) return SG_ERR_INVALID_ARG;
    sg_sym_c* S = new sg_sym_c();
    S->comm = (ncclComm_t)nccl_comm;
    S->n = n_rows;
    S->cap = nnz_cap;
    S->dt = (int)dtype;
    auto fail = [&](sg_status e) { sg_sym_c_destroy(S); return e; };
    if (ncclCommCount(S->comm, &S->nranks) != ncclSuccess || ncclCommUserRank(S->comm, &S->rank) != ncclSuccess)
        return fail(SG_ERR_NCCL);
    const size_t vs = dtype == SG_F64 ? 8 : 4;
    S->bytes[0] = 8 * (size_t)(n_rows + 1);
    S->bytes[1] = 4 * (size_t)(nnz_cap > 0 ? nnz_cap : 1);
    S->bytes[2] = vs * (size_t)(nnz_cap > 0 ? nnz_cap : 1);
    for (int q = 0; q < 3; ++q) {
        if (ncclMemAlloc(&S->buf[q], S->bytes[q]) != ncclSuccess) return fail(SG_ERR_OOM);
        if (ncclCommWindowRegister(S->comm, S->buf[q], S->bytes[q], &S->win[q], NCCL_WIN_COLL_SYMMETRIC) != ncclSuccess)
            return fail(SG_ERR_NCCL);
    }
    ncclDevCommRequirements reqs{};
    reqs.lsaBarrierCount = SYMC_BLOCKS;
    if (ncclDevCommCreate(S->comm, &reqs, &S->dev) != ncclSuccess) return fail(SG_ERR_NCCL);
    S->dev_ok = true;
    *out = S;
    return SG_OK;
}

sg_status sg_sym_c_buffers(const sg_sym_c* S, int64_t** row_ptr, int32_t** col, void** val) {
    if (!S) return SG_ERR_INVALID_ARG;
    if (row_ptr) *row_ptr = (int64_t*)S->buf[0];
    if (col) *col = (int32_t*)S->buf[1];
    if (val) *val = S->buf[2];
    return SG_OK;
}

sg_status sg_sym_c_layout(sg_sym_c* S, sg_plan* plan, int64_t* c_offset_out, int64_t* nnz_total_out, void* stream) {
    if (!S || !plan || !c_offset_out) return SG_ERR_INVALID_ARG;
    if (sg_internal_plan_poisoned(plan)) return SG_ERR_CUDA;
    if (sg_internal_plan_dtype(plan) != S->dt) return SG_ERR_DTYPE;
    cudaStream_t s = (cudaStream_t)stream;
    int64_t rb = 0, re = 0;
    const int64_t nnz = sg_internal_plan_rows(plan, &rb, &re);
    int64_t* d = nullptr;
    if (cudaMallocAsync(&d, sizeof(int64_t) * 3 * (size_t)(S->nranks + 1), s) != cudaSuccess) return SG_ERR_OOM;
    const int64_t mine[3] = {rb, re, nnz};
    std::vector<int64_t> lay(3 * (size_t)S->nranks), begin(S->nranks), off(S->nranks + 1);
    int64_t n = 0, total = 0;
    sg_status st = SG_OK;
    if (cudaMemcpyAsync(d, mine, sizeof(mine), cudaMemcpyHostToDevice, s) != cudaSuccess) st = SG_ERR_CUDA;
    else if (ncclAllGather(d, d + 3, 3, ncclInt64, S->comm, s) != ncclSuccess) st = SG_ERR_NCCL;
    else if (cudaMemcpyAsync(lay.data(), d + 3, sizeof(int64_t) * lay.size(), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
             cudaStreamSynchronize(s) != cudaSuccess) st = SG_ERR_CUDA;
    cudaFreeAsync(d, s);
    if (st != SG_OK) return st;
    if ((st = sg_gather_layout(lay.data(), S->nranks, begin.data(), off.data(), &n, &total)) != SG_OK) return st;
    if (n != S->n || total > S->cap) return SG_ERR_SHAPE;  // identical on every rank
    S->off = off[S->rank];
    S->total = total;
    S->rb = rb;
    S->re = re;
    S->nnz = nnz;
    *c_offset_out = S->off;
    if (nnz_total_out) *nnz_total_out = total;
    return SG_OK;
}

sg_status sg_sym_c_assemble(sg_sym_c* S, sg_plan* plan, const int64_t* local_row_ptr, void* stream) {
    if (!S || !plan || !local_row_ptr) return SG_ERR_INVALID_ARG;
    if (S->off < 0) return SG_ERR_INVALID_ARG;  // sg_sym_c_layout first
    int64_t rb = 0, re = 0;
    sg_internal_plan_rows(plan, &rb, &re);
    if (rb != S->rb || re != S->re) return SG_ERR_SHAPE;
    cudaStream_t s = (cudaStream_t)stream;
    const int last = S->re == S->n ? 1 : 0;
    SG_LAUNCH("k_symc_push", s, k_symc_push<<<SYMC_BLOCKS, SYMC_T, 0, s>>>(S->dev, S->win[0], S->win[1], S->win[2], local_row_ptr,
                                                                         S->rb, S->re - S->rb, S->off, S->nnz,
                                                                         S->dt == 0 ? 8 : 4, last, S->n));
    if (cudaGetLastError() != cudaSuccess || cudaStreamSynchronize(s) != cudaSuccess) return SG_ERR_CUDA;
    return SG_OK;
}

void sg_sym_c_destroy(sg_sym_c* S) {
    if (!S) return;
    if (S->dev_ok) ncclDevCommDestroy(S->comm, &S->dev);
    for (int q = 0; q < 3; ++q) {
        if (S->win[q]) ncclCommWindowDeregister(S->comm, S->win[q]);
        if (S->buf[q]) ncclMemFree(S->buf[q]);
    }
    delete S;
}

}  // extern "C"
