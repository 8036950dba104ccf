// sg_hh.cu — SURVEY §8(f) NEXT #4: the HH-CPU four-block variant of the paper's scale-free case study
// (PAPER Alg. 3; Section V-A), B200-native.
//
//   Phase I   a row is HIGH dense iff it has more than t non-zeros (L274): sg_hh_filter keeps the rows
//             of one class (the others emptied, row ids unchanged), giving A_H, A_L, B_H, B_L.
//   Phase II/III  the four products A_X B_Y run on the library's hot path (sg_symbolic / sg_numeric):
//             on one GPU the paper's two devices are its two kernel paths.
//   Phase IV  "combine" = the row-wise sum of two sparse matrices P + Q, computed as ONE more product of
//             the hot path: [P Q] * [I; I] (sg_hh_hstack builds [P Q], sg_hh_identity2 builds [I; I]) —
//             every row of [P Q] is a row of products with B rows of length 1, so the accumulators add
//             equal columns and emit the union sorted, with structural zeros kept (R9).
//   Sample    sg_hh_sample: the principal sub-matrix A[S, S] on a Bernoulli(f) index set S, columns
//             relabelled by rank (reading R20; f = 1/sqrt(n) gives the paper's sqrt(n) x sqrt(n) A').
#include "sg_device.cuh"

namespace sg {
namespace {

__device__ __forceinline__ uint64_t hh_sm64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

// kept length of every row: its nnz if (nnz > t) == high, else 0
__global__ void k_hh_len(Mat M, int64_t t, int high, int64_t* __restrict__ len) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < M.nrows; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t d = M.rp[i + 1] - M.rp[i];
        len[i] = ((d > t) == (high != 0)) ? d : 0;
    }
}

// copy the kept rows (warp per row): out_rp from the scan of k_hh_len
template <class VT>
__global__ void k_hh_copy(Mat M, const int64_t* __restrict__ out_rp, int32_t* __restrict__ col, VT* __restrict__ val) {
    const int lane = threadIdx.x & 31;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < M.nrows;
         i += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int64_t o = out_rp[i], n = out_rp[i + 1] - o, s = M.rp[i];
        for (int64_t q = lane; q < n; q += 32) {
            col[o + q] = __ldg(M.col + s + q);
            val[o + q] = __ldg(reinterpret_cast<const VT*>(M.val) + s + q);
        }
    }
}

// [P Q]: row i = P_i followed by Q_i with columns shifted by P.ncols (warp per row)
template <class VT>
__global__ void k_hh_hstack(Mat P, Mat Q, int64_t* __restrict__ rp, int32_t* __restrict__ col, VT* __restrict__ val,
                            int pass) {
    const int lane = threadIdx.x & 31;
    for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < P.nrows;
         i += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int64_t p0 = P.rp[i], pn = P.rp[i + 1] - p0, q0 = Q.rp[i], qn = Q.rp[i + 1] - q0;
        if (pass == 0) {
            if (lane == 0) rp[i] = pn + qn;  // lengths; the caller scans them
            continue;
        }
        const int64_t o = rp[i];
        for (int64_t q = lane; q < pn; q += 32) {
            col[o + q] = __ldg(P.col + p0 + q);
            val[o + q] = __ldg(reinterpret_cast<const VT*>(P.val) + p0 + q);
        }
        for (int64_t q = lane; q < qn; q += 32) {
            col[o + pn + q] = (int32_t)(__ldg(Q.col + q0 + q) + P.ncols);
            val[o + pn + q] = __ldg(reinterpret_cast<const VT*>(Q.val) + q0 + q);
        }
    }
}

// [I; I] (2p x p): row k has the single entry (k mod p, 1)
template <class VT>
__global__ void k_hh_identity2(int64_t p, int64_t* __restrict__ rp, int32_t* __restrict__ col, VT* __restrict__ val) {
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k <= 2 * p; k += (int64_t)gridDim.x * blockDim.x) {
        rp[k] = k;
        if (k < 2 * p) {
            col[k] = (int32_t)(k < p ? k : k - p);
            val[k] = (VT)1;
        }
    }
}

// sample mask: keep[i] = h(seed, SAMPLE, i) < Tf (all rows when all != 0)
__global__ void k_hh_mask(int64_t n, uint64_t seed, uint64_t Tf, int all, int64_t* __restrict__ keep) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        keep[i] = (all || hh_sm64(seed ^ hh_sm64(TAG_SAMPLE ^ hh_sm64((uint64_t)i))) < Tf) ? 1 : 0;
}

// per kept row: number of entries whose column is a kept index (pass 0), then the relabelled copy (pass 1)
template <class VT>
__global__ void k_hh_sub(Mat M, const int64_t* __restrict__ keep, const int64_t* __restrict__ rank,
                         const int64_t* __restrict__ rows_of_rank, int64_t s, int64_t* __restrict__ cnt_or_rp,
                         int32_t* __restrict__ col, int64_t* __restrict__ pos, VT* __restrict__ val, int pass) {
    const int lane = threadIdx.x & 31;
    for (int64_t r = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; r < s; r += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int64_t i = rows_of_rank[r];
        const int64_t q0 = M.rp[i], q1 = M.rp[i + 1];
        int64_t o = pass ? cnt_or_rp[r] : 0;
        for (int64_t b = q0; b < q1; b += 32) {
            const int64_t q = b + lane;
            int32_t j = -1;
            bool in = false;
            if (q < q1) {
                j = __ldg(M.col + q);
                in = j < M.nrows && keep[j] != 0;
            }
            const unsigned m = __ballot_sync(0xffffffffu, in);
            if (pass && in) {
                const int64_t at = o + __popc(m & ((1u << lane) - 1u));
                col[at] = (int32_t)rank[j];
                pos[at] = q;
                if (val) val[at] = __ldg(reinterpret_cast<const VT*>(M.val) + q);
            }
            o += __popc(m);
        }
        if (!pass && lane == 0) cnt_or_rp[r] = o;
    }
}

__global__ void k_hh_rows_of_rank(int64_t n, const int64_t* __restrict__ keep, const int64_t* __restrict__ rank,
                                  int64_t* __restrict__ rows_of_rank) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        if (keep[i]) rows_of_rank[rank[i]] = i;
}

// A[S, :] (the row sample of the measured Identify): lengths of the listed rows, then a warp-per-row copy
__global__ void k_rows_len(Mat M, const int64_t* __restrict__ rows, int64_t nr, int64_t* __restrict__ len) {
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nr; j += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = rows[j];
        len[j] = M.rp[i + 1] - M.rp[i];
    }
}

template <class VT>
__global__ void k_rows_copy(Mat M, const int64_t* __restrict__ rows, int64_t nr, const int64_t* __restrict__ out_rp,
                            int32_t* __restrict__ col, VT* __restrict__ val) {
    const int lane = threadIdx.x & 31;
    for (int64_t j = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; j < nr;
         j += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int64_t o = out_rp[j], n = out_rp[j + 1] - o, s = M.rp[rows[j]];
        for (int64_t q = lane; q < n; q += 32) {
            col[o + q] = __ldg(M.col + s + q);
            val[o + q] = __ldg(reinterpret_cast<const VT*>(M.val) + s + q);
        }
    }
}

}  // namespace

cudaError_t launch_rows_len(const Mat& M, const int64_t* rows, int64_t nr, int64_t* len, cudaStream_t s) {
    if (nr <= 0) return cudaSuccess;
    SG_LAUNCH("k_rows_len", s, (k_rows_len<<<grid_for(nr, 256, 148 * 8), 256, 0, s>>>(M, rows, nr, len)));
    return cudaGetLastError();
}

cudaError_t launch_rows_copy(const Mat& M, const int64_t* rows, int64_t nr, const int64_t* out_rp, int32_t* col, void* val,
                             cudaStream_t s) {
    if (nr <= 0) return cudaSuccess;
    const int g = grid_for(nr, 8, 148 * 16);
    if (M.dt == 0) SG_LAUNCH("k_rows_copy", s, (k_rows_copy<double><<<g, 256, 0, s>>>(M, rows, nr, out_rp, col, (double*)val)));
    else SG_LAUNCH("k_rows_copy", s, (k_rows_copy<float><<<g, 256, 0, s>>>(M, rows, nr, out_rp, col, (float*)val)));
    return cudaGetLastError();
}

cudaError_t launch_hh_len(const Mat& M, int64_t t, int high, int64_t* len, cudaStream_t s) {
    if (M.nrows <= 0) return cudaSuccess;
    SG_LAUNCH("k_hh_len", s, (k_hh_len<<<grid_for(M.nrows, 256, 148 * 8), 256, 0, s>>>(M, t, high, len)));
    return cudaGetLastError();
}

cudaError_t launch_hh_copy(const Mat& M, const int64_t* out_rp, int32_t* col, void* val, cudaStream_t s) {
    if (M.nrows <= 0) return cudaSuccess;
    const int g = grid_for(M.nrows, 8, 148 * 16);
    if (M.dt == 0) SG_LAUNCH("k_hh_copy", s, (k_hh_copy<double><<<g, 256, 0, s>>>(M, out_rp, col, (double*)val)));
    else SG_LAUNCH("k_hh_copy", s, (k_hh_copy<float><<<g, 256, 0, s>>>(M, out_rp, col, (float*)val)));
    return cudaGetLastError();
}

cudaError_t launch_hh_hstack(const Mat& P, const Mat& Q, int64_t* rp, int32_t* col, void* val, int pass, cudaStream_t s) {
    if (P.nrows <= 0) return cudaSuccess;
    const int g = grid_for(P.nrows, 8, 148 * 16);
    if (P.dt == 0) SG_LAUNCH("k_hh_hstack", s, (k_hh_hstack<double><<<g, 256, 0, s>>>(P, Q, rp, col, (double*)val, pass)));
    else SG_LAUNCH("k_hh_hstack", s, (k_hh_hstack<float><<<g, 256, 0, s>>>(P, Q, rp, col, (float*)val, pass)));
    return cudaGetLastError();
}

cudaError_t launch_hh_identity2(int64_t p, int dt, int64_t* rp, int32_t* col, void* val, cudaStream_t s) {
    const int g = grid_for(2 * p + 1, 256, 148 * 8);
    if (dt == 0) SG_LAUNCH("k_hh_identity2", s, (k_hh_identity2<double><<<g, 256, 0, s>>>(p, rp, col, (double*)val)));
    else SG_LAUNCH("k_hh_identity2", s, (k_hh_identity2<float><<<g, 256, 0, s>>>(p, rp, col, (float*)val)));
    return cudaGetLastError();
}

cudaError_t launch_hh_mask(int64_t n, uint64_t seed, uint64_t Tf, int all, int64_t* keep, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    SG_LAUNCH("k_hh_mask", s, (k_hh_mask<<<grid_for(n, 256, 148 * 8), 256, 0, s>>>(n, seed, Tf, all, keep)));
    return cudaGetLastError();
}

cudaError_t launch_hh_rows_of_rank(int64_t n, const int64_t* keep, const int64_t* rank, int64_t* rows_of_rank,
                                   cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    SG_LAUNCH("k_hh_rows_of_rank", s, (k_hh_rows_of_rank<<<grid_for(n, 256, 148 * 8), 256, 0, s>>>(n, keep, rank, rows_of_rank)));
    return cudaGetLastError();
}

cudaError_t launch_hh_sub(const Mat& M, const int64_t* keep, const int64_t* rank, const int64_t* rows_of_rank, int64_t s_rows,
                          int64_t* cnt_or_rp, int32_t* col, int64_t* pos, void* val, int pass, cudaStream_t s) {
    if (s_rows <= 0) return cudaSuccess;
    const int g = grid_for(s_rows, 8, 148 * 16);
    if (M.dt == 0)
        SG_LAUNCH("k_hh_sub", s, (k_hh_sub<double><<<g, 256, 0, s>>>(M, keep, rank, rows_of_rank, s_rows, cnt_or_rp, col, pos,
                                                                     (double*)val, pass)));
    else
        SG_LAUNCH("k_hh_sub", s, (k_hh_sub<float><<<g, 256, 0, s>>>(M, keep, rank, rows_of_rank, s_rows, cnt_or_rp, col, pos,
                                                                    (float*)val, pass)));
    return cudaGetLastError();
}

}  // namespace sg
