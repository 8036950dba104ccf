// sg_light.cu — the LIGHT path (0 < w_i <= thr, "less than t nonzeros"): rows
// binned by U = 2^ceil(log2 w_i); a shared-memory table sized from U (u_i <= w_i <= U).
// Symbolic: keys-only hash set -> exact u_i, plus the row's output column span.
// Numeric: order-preserving hash accumulator over that span; emission places every entry at
// (#occupied slots before its run) + (rank inside its run) -> sorted row, no sort pass.
//
// Bins U <= 512: one WARP per row, several rows per block, products flattened over the warp (one k
// per lane). Bins U >= 1024: one BLOCK per row, products flattened over the block (packed k
// entries, one contiguous slice per warp; sg_device.cuh) — such rows often have few k with long B
// rows, which per-warp k chunks would leave to one warp.
#include "sg_device.cuh"

namespace sg {

// warp-level bins: (b, U, R rows per block of 32*R threads)
#define SG_LIGHT_WARP_BINS(X) \
    X(0, 1, 8)                \
    X(1, 2, 8)                \
    X(2, 4, 8)                \
    X(3, 8, 8)                \
    X(4, 16, 8)               \
    X(5, 32, 8)               \
    X(6, 64, 8)               \
    X(7, 128, 8)              \
    X(8, 256, 8)              \
    X(9, 512, 4)
// block-level bins: (b, U, NT threads per block = per row)
#define SG_LIGHT_BLOCK_BINS(X) \
    X(10, 1024, 256)           \
    X(11, 2048, 512)           \
    X(12, 4096, 1024)

// the keys-only hash set insert of the symbolic pass (any hash; order is irrelevant there)
template <int P, int LOGP>
__device__ __forceinline__ int set_insert(int32_t* T, int32_t c) {
    uint32_t h = ((uint32_t)c * 0x9E3779B1u) >> (32 - LOGP);
    while (true) {
        int32_t old = T[h];
        if (old == c) return 0;
        if (old == EMPTY_KEY) {
            old = atomicCAS(&T[h], EMPTY_KEY, c);
            if (old == EMPTY_KEY) return 1;
            if (old == c) return 0;
        }
        h = (h + 1) & (P - 1);
    }
}

// ------------------------------------------------------------------------------------------------
// symbolic, warp per row: u_i = |union of cols(B_k)| and the span [cmin, cmax] of those columns
// ------------------------------------------------------------------------------------------------
template <int U, int R>
__global__ void __launch_bounds__(32 * R) k_sym_light(Mat A, Mat B, const int32_t* __restrict__ list, int64_t cnt,
                                                      const int64_t* __restrict__ rowmap, int64_t rb,
                                                      int64_t* __restrict__ u, int2* __restrict__ span) {
    constexpr int P = 2 * U < 64 ? 64 : 2 * U;  // power of two, load <= 1/2
    constexpr int LOGP = __builtin_ctz(P);
    __shared__ int32_t tab[R * P];
    const int g = threadIdx.x / 32, lane = threadIdx.x & 31;
    int32_t* T = tab + g * P;
    for (int s = lane; s < P; s += 32) T[s] = EMPTY_KEY;
    __syncwarp();
    for (int64_t j = (int64_t)blockIdx.x * R + g; j < cnt; j += (int64_t)gridDim.x * R) {
        const int64_t li = list[j];
        const int64_t row = rowmap ? rowmap[li] : rb + li;
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        int ins = 0, cmn = INT_MAX, cmx = -1;
        for (int64_t pb = s0; pb < s1; pb += 32) {
            chunk_products<false, double, 2>(A, B, pb, min(pb + 32, s1), [](int, int64_t&, int&) {},
                                             [&](int32_t c, double) {
                                                 cmn = min(cmn, c);
                                                 cmx = max(cmx, c);
                                                 ins += set_insert<P, LOGP>(T, c);
                                             });
        }
        ins = warp_sum(ins);
        cmn = warp_min(cmn);
        cmx = warp_max(cmx);
        if (lane == 0) {
            u[li] = ins;
            if (span) span[li] = make_int2(cmn, cmx);
        }
        __syncwarp();
        for (int s = lane; s < P; s += 32) T[s] = EMPTY_KEY;
        __syncwarp();
    }
}

// symbolic, block per row (U >= 1024)
template <int U, int NT>
__global__ void __launch_bounds__(NT) k_sym_light_blk(Mat A, Mat B, const int32_t* __restrict__ list, int64_t cnt,
                                                      const int64_t* __restrict__ rowmap, int64_t rb,
                                                      int64_t* __restrict__ u, int2* __restrict__ span) {
    constexpr int P = 2 * U;
    constexpr int LOGP = __builtin_ctz(P);
    __shared__ int32_t T[P];
    __shared__ int64_t s_beg[NT];
    __shared__ int s_off[NT];
    __shared__ long long wsll[33];
    __shared__ int red[3][NT / 32];
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    for (int s = tid; s < P; s += NT) T[s] = EMPTY_KEY;
    __syncthreads();
    for (int64_t j = blockIdx.x; j < cnt; j += gridDim.x) {
        const int64_t li = list[j];
        const int64_t row = rowmap ? rowmap[li] : rb + li;
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        int ins = 0, cmn = INT_MAX, cmx = -1;
        for (int64_t c0 = s0; c0 < s1; c0 += NT) {
            const int64_t i = c0 + tid;
            int len = 0;
            int64_t beg = 0;
            if (i < s1) {
                const int k = __ldg(A.col + i);
                beg = __ldg(B.rp + k);
                len = (int)(__ldg(B.rp + k + 1) - beg);
            }
            int nk;
            const int tot = chunk_compact<NT, int64_t>(len, beg, 0.0, s_beg, s_off, nullptr, &nk, wsll);
            warp_slice<NT, false, double, int64_t>(s_beg, s_off, nullptr, nk, tot, B, [&](int32_t c, double) {
                if (c < 0) return;
                cmn = min(cmn, c);
                cmx = max(cmx, c);
                ins += set_insert<P, LOGP>(T, c);
            });
            __syncthreads();
        }
        ins = warp_sum(ins);
        cmn = warp_min(cmn);
        cmx = warp_max(cmx);
        if (lane == 0) { red[0][wid] = ins; red[1][wid] = cmn; red[2][wid] = cmx; }
        __syncthreads();
        if (tid == 0) {
            int a = 0, mn = INT_MAX, mx = -1;
            for (int q = 0; q < NT / 32; ++q) { a += red[0][q]; mn = min(mn, red[1][q]); mx = max(mx, red[2][q]); }
            u[li] = a;
            if (span) span[li] = make_int2(mn, mx);
        }
        for (int s = tid; s < P; s += NT) T[s] = EMPTY_KEY;
        __syncthreads();
    }
}

cudaError_t launch_sym_light(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt,
                             const int64_t* rowmap, int64_t rb, int64_t* u, int2* span, cudaStream_t s) {
    if (cnt <= 0) return cudaSuccess;
    switch (b) {
#define X(B_, U_, R_)                                                                                     \
    case B_:                                                                                              \
        SG_LAUNCH("k_sym_light", s, (k_sym_light<U_, R_><<<grid_for(cnt, R_, 148 * 32), 32 * R_, 0, s>>>( \
                                        A, B, list, cnt, rowmap, rb, u, span)));                           \
        break;
        SG_LIGHT_WARP_BINS(X)
#undef X
#define X(B_, U_, NT_)                                                                                       \
    case B_:                                                                                                 \
        SG_LAUNCH("k_sym_light", s, (k_sym_light_blk<U_, NT_><<<grid_for(cnt, 1, 148 * 8), NT_, 0, s>>>(     \
                                        A, B, list, cnt, rowmap, rb, u, span)));                              \
        break;
        SG_LIGHT_BLOCK_BINS(X)
#undef X
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// numeric: order-preserving hash over [cmin, cmax] -> ascending row without a sort pass
// ------------------------------------------------------------------------------------------------
template <int U>
struct LightTable {
    static constexpr int H = 2 * U;  // home range (load <= 1/2)
    static constexpr int P = H + U;  // + overflow room: probing never passes the end (u <= U)
};

template <int U, int R, class VT>
__global__ void __launch_bounds__(32 * R) k_num_light(Mat A, Mat B, const int32_t* __restrict__ list, int64_t cnt,
                                                      int64_t rb, const int2* __restrict__ span,
                                                      const int64_t* __restrict__ C_rp, int32_t* __restrict__ C_col,
                                                      VT* __restrict__ C_val) {
    constexpr int H = LightTable<U>::H, P = LightTable<U>::P;
    extern __shared__ double smem_d[];
    const int g = threadIdx.x / 32, lane = threadIdx.x & 31;
    double* vals = smem_d + g * P;
    int32_t* keys = reinterpret_cast<int32_t*>(smem_d + R * P) + g * P;
    for (int s = lane; s < P; s += 32) { keys[s] = EMPTY_KEY; vals[s] = 0.0; }
    __syncwarp();
    for (int64_t j = (int64_t)blockIdx.x * R + g; j < cnt; j += (int64_t)gridDim.x * R) {
        const int64_t li = list[j];
        const int64_t row = rb + li;
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        const int2 sp = span[li];
        const int64_t width = (int64_t)sp.y - sp.x + 1;
        const bool ident = width <= P;
        const uint64_t mult = ident ? 0 : (((uint64_t)H << 32) / (uint64_t)width);
        const int cmin = sp.x;
        int hmax = -1;
        for (int64_t pb = s0; pb < s1; pb += 32) {
            chunk_products<true, VT, 2>(A, B, pb, min(pb + 32, s1), [](int, int64_t&, int&) {},
                                        [&](int32_t c, double v) {
                                            int h = acc_insert(keys, vals, c, v, (uint32_t)(c - cmin), ident, mult);
                                            hmax = max(hmax, h);
                                        });
        }
        hmax = warp_max(hmax);
        __syncwarp();
        emit_slots<32, 32 * R, VT>(keys, vals, hmax + 1, C_rp[li], C_col, C_val, nullptr, !ident);
        __syncwarp();
    }
}

template <int U, int NT, class VT>
__global__ void __launch_bounds__(NT) k_num_light_blk(Mat A, Mat B, const int32_t* __restrict__ list, int64_t cnt,
                                                      int64_t rb, const int2* __restrict__ span,
                                                      const int64_t* __restrict__ C_rp, int32_t* __restrict__ C_col,
                                                      VT* __restrict__ C_val) {
    constexpr int H = LightTable<U>::H, P = LightTable<U>::P;
    extern __shared__ double smem_d[];
    __shared__ int64_t s_beg[NT];
    __shared__ int s_off[NT];
    __shared__ double s_a[NT];
    __shared__ long long wsll[33];
    __shared__ int ws[NT / 32];
    __shared__ int s_hmax;
    const int tid = threadIdx.x, lane = tid & 31;
    double* vals = smem_d;
    int32_t* keys = reinterpret_cast<int32_t*>(smem_d + P);
    for (int s = tid; s < P; s += NT) { keys[s] = EMPTY_KEY; vals[s] = 0.0; }
    if (tid == 0) s_hmax = -1;
    __syncthreads();
    for (int64_t j = blockIdx.x; j < cnt; j += gridDim.x) {
        const int64_t li = list[j];
        const int64_t row = rb + li;
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        const int2 sp = span[li];
        const int64_t width = (int64_t)sp.y - sp.x + 1;
        const bool ident = width <= P;
        const uint64_t mult = ident ? 0 : (((uint64_t)H << 32) / (uint64_t)width);
        const int cmin = sp.x;
        int hmax = -1;
        for (int64_t c0 = s0; c0 < s1; c0 += NT) {
            const int64_t i = c0 + tid;
            int len = 0;
            int64_t beg = 0;
            double a = 0.0;
            if (i < s1) {
                const int k = __ldg(A.col + i);
                beg = __ldg(B.rp + k);
                len = (int)(__ldg(B.rp + k + 1) - beg);
                a = ldv<VT>(A.val, i);
            }
            int nk;
            const int tot = chunk_compact<NT, int64_t>(len, beg, a, s_beg, s_off, s_a, &nk, wsll);
            warp_slice<NT, true, VT, int64_t>(s_beg, s_off, s_a, nk, tot, B, [&](int32_t c, double v) {
                if (c < 0) return;
                const int h = acc_insert(keys, vals, c, v, (uint32_t)(c - cmin), ident, mult);
                hmax = max(hmax, h);
            });
            __syncthreads();
        }
        hmax = warp_max(hmax);
        if (lane == 0) atomicMax(&s_hmax, hmax);
        __syncthreads();
        const int nslots = s_hmax + 1;
        __syncthreads();
        if (tid == 0) s_hmax = -1;
        emit_slots<NT, NT, VT>(keys, vals, nslots, C_rp[li], C_col, C_val, ws, !ident);
        __syncthreads();
    }
}

template <class VT>
static cudaError_t num_light_V(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, int64_t rb,
                               const int2* span, const int64_t* C_rp, int32_t* C_col, void* C_val, cudaStream_t s) {
    switch (b) {
#define X(B_, U_, R_)                                                                                         \
    case B_: {                                                                                                \
        auto kern = k_num_light<U_, R_, VT>;                                                                  \
        const int smem = R_ * LightTable<U_>::P * 12;                                                         \
        if (smem > 48 * 1024) {                                                                               \
            cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);     \
            if (e != cudaSuccess) return e;                                                                   \
        }                                                                                                     \
        SG_LAUNCH("k_num_light", s, (kern<<<grid_for(cnt, R_, 148 * 32), 32 * R_, smem, s>>>(                 \
                                        A, B, list, cnt, rb, span, C_rp, C_col, (VT*)C_val)));                 \
        break;                                                                                                \
    }
        SG_LIGHT_WARP_BINS(X)
#undef X
#define X(B_, U_, NT_)                                                                                        \
    case B_: {                                                                                                \
        auto kern = k_num_light_blk<U_, NT_, VT>;                                                             \
        const int smem = LightTable<U_>::P * 12;                                                              \
        if (smem > 48 * 1024) {                                                                               \
            cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);     \
            if (e != cudaSuccess) return e;                                                                   \
        }                                                                                                     \
        SG_LAUNCH("k_num_light", s, (kern<<<grid_for(cnt, 1, 148 * 8), NT_, smem, s>>>(                       \
                                        A, B, list, cnt, rb, span, C_rp, C_col, (VT*)C_val)));                 \
        break;                                                                                                \
    }
        SG_LIGHT_BLOCK_BINS(X)
#undef X
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

cudaError_t launch_num_light(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, int64_t rb,
                             const int2* span, const int64_t* C_rp, int32_t* C_col, void* C_val, cudaStream_t s) {
    if (cnt <= 0) return cudaSuccess;
    return A.dt == 0 ? num_light_V<double>(b, A, B, list, cnt, rb, span, C_rp, C_col, C_val, s)
                     : num_light_V<float>(b, A, B, list, cnt, rb, span, C_rp, C_col, C_val, s);
}

}  // namespace sg
