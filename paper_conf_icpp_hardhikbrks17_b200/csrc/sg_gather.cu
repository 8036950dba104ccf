// sg_gather.cu — assembly of the row-distributed C over NCCL (Alg. 2 l.7: "Transfer
// results of GPU to CPU and add that to CPU's results"), generalised to G GPUs of one NVSwitch box.
//
//   1. ncclAllGather of (row_begin, row_end, nnz) per rank        -> every rank knows the layout
//   2. allgatherv of the local row_ptr prefixes                     -> grouped ncclBroadcast per root
//      (NCCL has no native allgatherv; G broadcasts inside one ncclGroup run concurrently)
//   3. offset fix-up kernel: rank r's slice += sum_{q<r} nnz_q      -> the global row_ptr
//   4. optional allgatherv of C_col / C_val (only where the full C fits on every GPU)
#include "sg_internal.cuh"
#include <nccl.h>
#include <vector>

using namespace sg;

extern "C" {
int64_t sg_internal_plan_rows(const sg_plan* pl, int64_t* rb, int64_t* re);
int sg_internal_plan_dtype(const sg_plan* pl);
bool sg_internal_plan_poisoned(const sg_plan* pl);
void sg_internal_plan_poison(sg_plan* pl);
}

namespace {
__global__ void k_fix_offsets(int64_t* rp, const int64_t* __restrict__ seg_begin, const int64_t* __restrict__ seg_off,
                              int nseg, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        // segment of row i: largest r with seg_begin[r] <= i (nseg small: linear scan)
        int r = 0;
        for (int q = 1; q < nseg; ++q) if (seg_begin[q] <= i) r = q;
        rp[i] += seg_off[r];
    }
}
}  // namespace

// Host-only assembly arithmetic (no CUDA, no NCCL): validates that the per-rank row blocks are
// contiguous in rank order from row 0, and derives each rank's first row and first C entry.
extern "C" sg_status sg_gather_layout(const int64_t* lay, int nranks, int64_t* begin, int64_t* off, int64_t* n_out,
                                      int64_t* total_out) {
    if (!lay || nranks < 1 || !begin || !off || !n_out || !total_out) return SG_ERR_INVALID_ARG;
    if (lay[0] != 0) return SG_ERR_SHAPE;
    off[0] = 0;
    for (int r = 0; r < nranks; ++r) {
        if (lay[3 * r + 1] < lay[3 * r] || lay[3 * r + 2] < 0) return SG_ERR_SHAPE;
        if (r > 0 && lay[3 * r] != lay[3 * (r - 1) + 1]) return SG_ERR_SHAPE;
        begin[r] = lay[3 * r];
        off[r + 1] = off[r] + lay[3 * r + 2];
    }
    *n_out = lay[3 * (nranks - 1) + 1];
    *total_out = off[nranks];
    return SG_OK;
}

extern "C" sg_status sg_gather(sg_plan* plan, void* nccl_comm, int gather_values, const int64_t* local_row_ptr,
                               const int32_t* local_col, const void* local_val, int64_t* C_row_ptr_global,
                               int64_t row_ptr_cap, int32_t* C_col_global, void* C_val_global, int64_t nnz_cap,
                               int64_t* nnz_total_out, void* stream) {
    if (!plan || !nccl_comm || !local_row_ptr || !C_row_ptr_global || !nnz_total_out) return SG_ERR_INVALID_ARG;
    if (row_ptr_cap < 0 || nnz_cap < 0) return SG_ERR_INVALID_ARG;
    if (sg_internal_plan_poisoned(plan)) return SG_ERR_CUDA;
    cudaStream_t s = (cudaStream_t)stream;
    ncclComm_t comm = (ncclComm_t)nccl_comm;
    int nranks = 0, rank = 0;
    if (ncclCommCount(comm, &nranks) != ncclSuccess || ncclCommUserRank(comm, &rank) != ncclSuccess) return SG_ERR_NCCL;
    int64_t rb = 0, re = 0;
    const int64_t nnz = sg_internal_plan_rows(plan, &rb, &re);
    const int dt = sg_internal_plan_dtype(plan);
    if (gather_values && (!C_col_global || !C_val_global || (nnz > 0 && (!local_col || !local_val))))
        return SG_ERR_INVALID_ARG;
    // 1. layout allgather
    int64_t* dlay = nullptr;
    // every rank publishes (row_begin, row_end, nnz, row_ptr_cap, nnz_cap): the capacity check below is
    // then evaluated on identical data by every rank, so all of them skip (or run) the broadcasts together
    constexpr int NL = 5;
    if (cudaMallocAsync(&dlay, sizeof(int64_t) * NL * (size_t)(nranks + 1) * 2, s) != cudaSuccess) return SG_ERR_OOM;
    int64_t mine[NL] = {rb, re, nnz, row_ptr_cap, gather_values ? nnz_cap : INT64_MAX};
    std::vector<int64_t> lay5(NL * (size_t)nranks), lay(3 * (size_t)nranks);
    sg_status st = SG_OK;
    do {
        if (cudaMemcpyAsync(dlay, mine, sizeof(mine), cudaMemcpyHostToDevice, s) != cudaSuccess) { st = SG_ERR_CUDA; break; }
        if (ncclAllGather(dlay, dlay + NL, NL, ncclInt64, comm, s) != ncclSuccess) { st = SG_ERR_NCCL; break; }
        if (cudaMemcpyAsync(lay5.data(), dlay + NL, sizeof(int64_t) * NL * nranks, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaStreamSynchronize(s) != cudaSuccess) { st = SG_ERR_CUDA; break; }
        for (int r = 0; r < nranks; ++r)
            for (int q = 0; q < 3; ++q) lay[3 * r + q] = lay5[NL * r + q];
        // contiguity: rank order, covering [0, n); entry offsets of every rank's C rows
        std::vector<int64_t> off(nranks + 1, 0), begin(nranks);
        int64_t n = 0, total = 0;
        if ((st = sg_gather_layout(lay.data(), nranks, begin.data(), off.data(), &n, &total)) != SG_OK) break;
        // capacities of EVERY rank's outputs (identical decision on all ranks; nothing written yet)
        for (int r = 0; r < nranks; ++r)
            if (lay5[NL * r + 3] < n + 1 || lay5[NL * r + 4] < total) st = SG_ERR_SHAPE;
        if (st != SG_OK) break;
        // 2. allgatherv of the local prefixes (rows_r entries each, excluding the trailing total)
        if (ncclGroupStart() != ncclSuccess) { st = SG_ERR_NCCL; break; }
        for (int r = 0; r < nranks; ++r) {
            const int64_t cnt = lay[3 * r + 1] - lay[3 * r];
            if (cnt <= 0) continue;
            if (ncclBroadcast(r == rank ? (const void*)local_row_ptr : (const void*)(C_row_ptr_global + begin[r]),
                              C_row_ptr_global + begin[r], (size_t)cnt, ncclInt64, r, comm, s) != ncclSuccess) {
                st = SG_ERR_NCCL;
            }
        }
        if (gather_values) {
            const ncclDataType_t vt = dt == 0 ? ncclFloat64 : ncclFloat32;
            const size_t vs = dt == 0 ? 8 : 4;
            for (int r = 0; r < nranks; ++r) {
                const int64_t cnt = lay[3 * r + 2];
                if (cnt <= 0) continue;
                int32_t* cdst = C_col_global + off[r];
                char* vdst = (char*)C_val_global + vs * (size_t)off[r];
                if (ncclBroadcast(r == rank ? (const void*)local_col : (const void*)cdst, cdst, (size_t)cnt, ncclInt32, r,
                                  comm, s) != ncclSuccess ||
                    ncclBroadcast(r == rank ? local_val : (const void*)vdst, vdst, (size_t)cnt, vt, r, comm, s) != ncclSuccess)
                    st = SG_ERR_NCCL;
            }
        }
        if (ncclGroupEnd() != ncclSuccess) st = SG_ERR_NCCL;
        if (st != SG_OK) break;
        // 3. offset fix-up on the received slices, trailing total
        if (cudaMemcpyAsync(dlay, begin.data(), sizeof(int64_t) * nranks, cudaMemcpyHostToDevice, s) != cudaSuccess ||
            cudaMemcpyAsync(dlay + nranks, off.data(), sizeof(int64_t) * nranks, cudaMemcpyHostToDevice, s) != cudaSuccess ||
            cudaMemcpyAsync(C_row_ptr_global + n, &total, sizeof(int64_t), cudaMemcpyHostToDevice, s) != cudaSuccess) {
            st = SG_ERR_CUDA;
            break;
        }
        if (n > 0) {
            int grid = (int)((n + 255) / 256 < 148 * 8 ? (n + 255) / 256 : 148 * 8);
            SG_LAUNCH("k_fix_offsets", s, k_fix_offsets<<<grid, 256, 0, s>>>(C_row_ptr_global, dlay, dlay + nranks, nranks, n));
        }
        if (cudaGetLastError() != cudaSuccess || cudaStreamSynchronize(s) != cudaSuccess) { st = SG_ERR_CUDA; break; }
        *nnz_total_out = total;
    } while (0);
    cudaFreeAsync(dlay, s);
    if (st == SG_ERR_CUDA) sg_internal_plan_poison(plan);
    return st;
}
