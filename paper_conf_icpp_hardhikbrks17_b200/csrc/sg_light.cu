// sg_light.cu — the LIGHT path (0 < w_i <= thr, "less than t nonzeros"): rows
// binned by U = 2^ceil(log2 w_i); G threads per row with a shared-memory table sized from U
// (u_i <= w_i <= U). Symbolic: keys-only hash set -> exact u_i, plus the row's output column span.
// Numeric: order-preserving hash accumulator over that span -> sorted row, no sort pass.
#include "sg_device.cuh"

namespace sg {

// (U, G, R) per light bin: G threads per row, R rows per block (BLK = G*R)
#define SG_LIGHT_BINS(X)            \
    X(0, 1, 32, 8)                  \
    X(1, 2, 32, 8)                  \
    X(2, 4, 32, 8)                  \
    X(3, 8, 32, 8)                  \
    X(4, 16, 32, 8)                 \
    X(5, 32, 32, 8)                 \
    X(6, 64, 32, 8)                 \
    X(7, 128, 32, 8)                \
    X(8, 256, 32, 8)                \
    X(9, 512, 32, 4)                \
    X(10, 1024, 64, 2)              \
    X(11, 2048, 128, 1)             \
    X(12, 4096, 256, 1)

// ------------------------------------------------------------------------------------------------
// symbolic: u_i = |union of cols(B_k)| and the span [cmin, cmax] of those columns
// ------------------------------------------------------------------------------------------------
template <int U, int G, int R>
__global__ void __launch_bounds__(G * R) k_sym_light(Mat A, Mat B, const int32_t* __restrict__ list, int64_t cnt,
                                                     const int64_t* __restrict__ rowmap, int64_t rb,
                                                     int64_t* __restrict__ u, int2* __restrict__ span) {
    constexpr int BLK = G * R;
    constexpr int P = 2 * U < 64 ? 64 : 2 * U;  // power of two, load <= 1/2
    constexpr int LOGP = __builtin_ctz(P);
    constexpr int NW = G / 32;
    __shared__ int32_t tab[R * P];
    __shared__ int red[BLK / 32][3];
    const int g = threadIdx.x / G, t = threadIdx.x % G, lane = threadIdx.x & 31, wg = t / 32;
    int32_t* T = tab + g * P;
    for (int s = t; s < P; s += G) T[s] = EMPTY_KEY;
    group_bar<G, BLK>();
    for (int64_t j = (int64_t)blockIdx.x * R + g; j < cnt; j += (int64_t)gridDim.x * R) {
        const int64_t li = list[j];
        const int64_t row = rowmap ? rowmap[li] : rb + li;
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        int ins = 0, cmn = INT_MAX, cmx = -1;
        for (int64_t pb = s0 + 32 * wg; pb < s1; pb += 32 * NW) {
            chunk_products<false, double, 2>(
                A, B, pb, min(pb + 32, s1), [](int, int64_t&, int&) {},
                [&](int32_t c, double) {
                    cmn = min(cmn, c);
                    cmx = max(cmx, c);
                    uint32_t h = ((uint32_t)c * 0x9E3779B1u) >> (32 - LOGP);
                    while (true) {
                        int32_t old = T[h];
                        if (old == c) break;
                        if (old == EMPTY_KEY) {
                            old = atomicCAS(&T[h], EMPTY_KEY, c);
                            if (old == EMPTY_KEY) { ++ins; break; }
                            if (old == c) break;
                        }
                        h = (h + 1) & (P - 1);
                    }
                });
        }
        ins = warp_sum(ins);
        cmn = warp_min(cmn);
        cmx = warp_max(cmx);
        if constexpr (NW > 1) {
            if (lane == 0) { red[threadIdx.x / 32][0] = ins; red[threadIdx.x / 32][1] = cmn; red[threadIdx.x / 32][2] = cmx; }
            group_bar<G, BLK>();
            const int w0 = (threadIdx.x / G) * NW;
            ins = 0; cmn = INT_MAX; cmx = -1;
            for (int q = 0; q < NW; ++q) { ins += red[w0 + q][0]; cmn = min(cmn, red[w0 + q][1]); cmx = max(cmx, red[w0 + q][2]); }
        }
        if (t == 0) {
            u[li] = ins;
            if (span) span[li] = make_int2(cmn, cmx);
        }
        group_bar<G, BLK>();
        for (int s = t; s < P; s += G) T[s] = EMPTY_KEY;
        group_bar<G, BLK>();
    }
}

cudaError_t launch_sym_light(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt,
                             const int64_t* rowmap, int64_t rb, int64_t* u, int2* span, cudaStream_t s) {
    if (cnt <= 0) return cudaSuccess;
    switch (b) {
#define X(B_, U_, G_, R_)                                                                                  \
    case B_:                                                                                               \
        SG_LAUNCH("k_sym_light", s, (k_sym_light<U_, G_, R_><<<grid_for(cnt, R_, 148 * 32), G_ * R_, 0, s>>>( \
                                        A, B, list, cnt, rowmap, rb, u, span)));                            \
        break;
        SG_LIGHT_BINS(X)
#undef X
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// numeric: order-preserving hash over [cmin, cmax] -> ascending row without a sort pass
// ------------------------------------------------------------------------------------------------
template <int U, int G, int R, class VT>
__global__ void __launch_bounds__(G * R) k_num_light(Mat A, Mat B, const int32_t* __restrict__ list, int64_t cnt,
                                                     int64_t rb, const int2* __restrict__ span,
                                                     const int64_t* __restrict__ C_rp, int32_t* __restrict__ C_col,
                                                     VT* __restrict__ C_val) {
    constexpr int BLK = G * R;
    constexpr int H = 2 * U;          // home range (load <= 1/2)
    constexpr int P = H + U;          // + overflow room: probing never passes the end (u <= U)
    constexpr int NW = G / 32;
    extern __shared__ double smem_d[];
    __shared__ int ws[BLK / 32];
    const int g = threadIdx.x / G, t = threadIdx.x % G, lane = threadIdx.x & 31, wg = t / 32;
    double* vals = smem_d + g * P;
    int32_t* keys = reinterpret_cast<int32_t*>(smem_d + R * P) + g * P;
    int* gws = ws + g * NW;
    for (int s = t; s < P; s += G) { keys[s] = EMPTY_KEY; vals[s] = 0.0; }
    group_bar<G, BLK>();
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
        for (int64_t pb = s0 + 32 * wg; pb < s1; pb += 32 * NW) {
            chunk_products<true, VT, 2>(A, B, pb, min(pb + 32, s1), [](int, int64_t&, int&) {},
                                        [&](int32_t c, double v) {
                                            int h = acc_insert(keys, vals, c, v, (uint32_t)(c - cmin), ident, mult);
                                            hmax = max(hmax, h);
                                        });
        }
        hmax = warp_max(hmax);
        if constexpr (NW > 1) {
            if (lane == 0) gws[wg] = hmax;
            group_bar<G, BLK>();
            for (int q = 0; q < NW; ++q) hmax = max(hmax, gws[q]);
        }
        group_bar<G, BLK>();
        const int nslots = hmax + 1;
        emit_slots<G, BLK, VT>(keys, vals, nslots, C_rp[li], C_col, C_val, gws, !ident);
        group_bar<G, BLK>();
    }
}

template <class VT>
static cudaError_t num_light_V(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, int64_t rb,
                               const int2* span, const int64_t* C_rp, int32_t* C_col, void* C_val, cudaStream_t s) {
    switch (b) {
#define X(B_, U_, G_, R_)                                                                                     \
    case B_: {                                                                                                \
        auto kern = k_num_light<U_, G_, R_, VT>;                                                              \
        const int smem = R_ * 3 * U_ * 12;                                                                    \
        if (smem > 48 * 1024) {                                                                               \
            cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);     \
            if (e != cudaSuccess) return e;                                                                   \
        }                                                                                                     \
        SG_LAUNCH("k_num_light", s, (kern<<<grid_for(cnt, R_, 148 * 32), G_ * R_, smem, s>>>(                 \
                                        A, B, list, cnt, rb, span, C_rp, C_col, (VT*)C_val)));                 \
        break;                                                                                                \
    }
        SG_LIGHT_BINS(X)
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
