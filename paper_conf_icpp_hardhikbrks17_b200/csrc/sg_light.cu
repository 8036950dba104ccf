// sg_light.cu — the LIGHT path (0 < w_i <= thr, "less than t nonzeros"): rows
// binned by U = 2^ceil(log2 w_i); a shared-memory table sized from U (u_i <= w_i <= U).
// Symbolic: keys-only hash set -> exact u_i, plus the row's output column span.
// Numeric: order-preserving hash accumulator over that span; emission places every entry at
// (#occupied slots before its run) + (rank inside its run) -> sorted row, no sort pass.
//
// Bins U <= 512 (numeric: U <= 256): one WARP per row, several rows per block, products flattened over
// the warp (one k per lane). Larger bins: one BLOCK per row, products flattened over the block (packed k
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
// The NUMERIC pass puts U = 512 rows on 4-warp blocks instead: a warp-per-row table of 3U slots
// (18 KB) allowed only 12 warps per SM; one 4-warp block per row keeps 48 (C2: light numeric
// 3.17 -> 2.59 ms). The symbolic pass (2U keys only) keeps the warp layout, which is faster there.
#define SG_NUM_LIGHT_WARP_BINS(X) \
    X(0, 1, 8) X(1, 2, 8) X(2, 4, 8) X(3, 8, 8) X(4, 16, 8) X(5, 32, 8) X(6, 64, 8) X(7, 128, 8) X(8, 256, 8)
#define SG_NUM_LIGHT_BLOCK_BINS(X) X(9, 512, 128) X(10, 1024, 256) X(11, 2048, 512) X(12, 4096, 1024)

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

// ---- column-skew detection for the numeric pass's order-preserving hash -------------------------
// The numeric pass homes column c at floor((c - cmin) * 2U / width). When a row's columns cluster far
// below that resolution (R-MAT without the label permutation: hubs at low ids) the keys crowd some
// stretches of homes and the probe runs grow with u. Rows with u > 64 keys in which some bucket of
// 32 consecutive homes receives more than SKEW_BUCKET keys (local load > 1.25; a uniform row has
// 16 on average) are flagged (span.x = -1 - cmin) and the numeric pass takes the SORTED path for
// them: uniform hash, then a bitonic sort of the row's entries in shared memory.
__device__ __forceinline__ uint32_t light_home(int32_t c, int cmin, uint64_t mult) {
    return (uint32_t)(((uint64_t)(uint32_t)(c - cmin) * mult) >> 32);
}
template <int U> __device__ __forceinline__ uint64_t light_mult(int64_t width) {
    return (((uint64_t)(2 * U)) << 32) / (uint64_t)width;
}
constexpr int SKEW_MIN_U = 64;
#ifndef SG_SYM_UNR
#define SG_SYM_UNR 4
#endif
constexpr int SYM_UNR = SG_SYM_UNR;  // warp symbolic: gather batches in flight
constexpr int SKEW_BUCKET = 40;

// ------------------------------------------------------------------------------------------------
// symbolic, warp per row: u_i = |union of cols(B_k)| and the span [cmin, cmax] of those columns
// ------------------------------------------------------------------------------------------------
template <int U, int R>
__global__ void __launch_bounds__(32 * R) k_sym_light(Mat A, Mat B, const int32_t* __restrict__ list, int64_t cnt,
                                                      const int64_t* __restrict__ rowmap, int64_t rb,
                                                      int64_t* __restrict__ u, int2* __restrict__ span,
                                                      unsigned long long* nskew) {
    constexpr int P = 2 * U < 64 ? 64 : 2 * U;  // power of two, load <= 1/2
    constexpr int LOGP = __builtin_ctz(P);
    constexpr int HBW = (2 * U + 31) / 32;      // key counts per 32 homes (skew detection)
    __shared__ int32_t tab[R * P];
    __shared__ uint32_t hbits[R * HBW];
    const int g = threadIdx.x / 32, lane = threadIdx.x & 31;
    int32_t* T = tab + g * P;
    uint32_t* hb = hbits + g * HBW;
    for (int s = lane; s < P; s += 32) T[s] = EMPTY_KEY;
    for (int s = lane; s < HBW; s += 32) hb[s] = 0u;
    __syncwarp();
    for (int64_t j = (int64_t)blockIdx.x * R + g; j < cnt; j += (int64_t)gridDim.x * R) {
        const int64_t li = list[j];
        const int64_t row = rowmap ? rowmap[li] : rb + li;
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        int ins = 0, cmn = INT_MAX, cmx = -1;
        for (int64_t pb = s0; pb < s1; pb += 32) {
            chunk_products<false, double, SYM_UNR>(A, B, pb, min(pb + 32, s1), [](int, int64_t&, int&) {},
                                             [&](int32_t c, double) {
                                                 cmn = min(cmn, c);
                                                 cmx = max(cmx, c);
                                                 ins += set_insert<P, LOGP>(T, c);
                                             });
        }
        ins = warp_sum(ins);
        cmn = warp_min(cmn);
        cmx = warp_max(cmx);
        bool skew = false;
        if (span && U > SKEW_MIN_U && ins > SKEW_MIN_U && (int64_t)cmx - cmn + 1 > 3 * U) {
            __syncwarp();
            const uint64_t mult = light_mult<U>((int64_t)cmx - cmn + 1);
            for (int s = lane; s < P; s += 32) {
                const int32_t c = T[s];
                if (c != EMPTY_KEY) atomicAdd(&hb[light_home(c, cmn, mult) >> 5], 1u);  // keys per 32 homes
            }
            __syncwarp();
            int d = 0;
            for (int q = lane; q < HBW; q += 32) { d = max(d, (int)hb[q]); hb[q] = 0u; }
            skew = warp_max(d) > SKEW_BUCKET;
        }
        if (lane == 0) {
            u[li] = ins;
            if (span) span[li] = make_int2(skew ? -1 - cmn : cmn, cmx);
            if (skew && nskew) atomicAdd(nskew, 1ull);
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
                                                      int64_t* __restrict__ u, int2* __restrict__ span,
                                                      unsigned long long* nskew) {
    constexpr int P = 2 * U;
    constexpr int LOGP = __builtin_ctz(P);
    constexpr int HBW = 2 * U / 32;
    __shared__ int32_t T[P];
    __shared__ uint32_t hb[HBW];
    __shared__ int s_d;
    __shared__ int64_t s_beg[NT];
    __shared__ int s_off[NT];
    __shared__ long long wsll[33];
    __shared__ int red[3][NT / 32];
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    for (int s = tid; s < P; s += NT) T[s] = EMPTY_KEY;
    for (int s = tid; s < HBW; s += NT) hb[s] = 0u;
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
        int a_ = 0, mn = INT_MAX, mx = -1;
        for (int q = 0; q < NT / 32; ++q) { a_ += red[0][q]; mn = min(mn, red[1][q]); mx = max(mx, red[2][q]); }
        bool skew = false;
        if (span && a_ > SKEW_MIN_U && (int64_t)mx - mn + 1 > 3 * U) {  // block-uniform
            const uint64_t mult = light_mult<U>((int64_t)mx - mn + 1);
            for (int s = tid; s < P; s += NT) {
                const int32_t c = T[s];
                if (c != EMPTY_KEY) atomicAdd(&hb[light_home(c, mn, mult) >> 5], 1u);  // keys per 32 homes
            }
            if (tid == 0) s_d = 0;
            __syncthreads();
            int d = 0;
            for (int q = tid; q < HBW; q += NT) { d = max(d, (int)hb[q]); hb[q] = 0u; }
            d = warp_max(d);
            if (lane == 0 && d) atomicMax(&s_d, d);
            __syncthreads();
            skew = s_d > SKEW_BUCKET;
        }
        if (tid == 0) {
            u[li] = a_;
            if (span) span[li] = make_int2(skew ? -1 - mn : mn, mx);
            if (skew && nskew) atomicAdd(nskew, 1ull);
        }
        __syncthreads();  // red[] and s_d read by everyone before the next row rewrites them
        for (int s = tid; s < P; s += NT) T[s] = EMPTY_KEY;
        __syncthreads();
    }
}

cudaError_t launch_sym_light(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt,
                             const int64_t* rowmap, int64_t rb, int64_t* u, int2* span, unsigned long long* nskew,
                             cudaStream_t s) {
    if (cnt <= 0) return cudaSuccess;
    switch (b) {
#define X(B_, U_, R_)                                                                                     \
    case B_:                                                                                              \
        SG_LAUNCH("k_sym_light", s, (k_sym_light<U_, R_><<<grid_for(cnt, R_, 148 * 32), 32 * R_, 0, s>>>( \
                                        A, B, list, cnt, rowmap, rb, u, span, nskew)));                    \
        break;
        SG_LIGHT_WARP_BINS(X)
#undef X
#define X(B_, U_, NT_)                                                                                       \
    case B_:                                                                                                 \
        SG_LAUNCH("k_sym_light", s, (k_sym_light_blk<U_, NT_><<<grid_for(cnt, 1, 148 * 8), NT_, 0, s>>>(     \
                                        A, B, list, cnt, rowmap, rb, u, span, nskew)));                       \
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
// ---- the SORTED path of column-skewed rows: uniform hash over [0, H), then the row's entries are
// gathered into [H, H + u) (order irrelevant), bitonic-sorted by column and written out ----
template <int H>
__device__ __forceinline__ void uni_insert(int32_t* keys, double* vals, int32_t c, double v) {
    constexpr int LOGH = __builtin_ctz(H);
    uint32_t h = ((uint32_t)c * 0x9E3779B1u) >> (32 - LOGH);
    while (true) {
        int32_t old = keys[h];
        if (old == c) break;
        if (old == EMPTY_KEY) {
            old = atomicCAS(&keys[h], EMPTY_KEY, c);
            if (old == EMPTY_KEY || old == c) break;
        }
        h = (h + 1) & (H - 1);
    }
    atomicAdd(&vals[h], v);
}

// bitonic sort of n (a power of two) (key, value) pairs by key by the G threads of a group
template <int G, int BLK>
__device__ __forceinline__ void bitonic_pairs(int32_t* k, double* v, int n) {
    const int t = threadIdx.x % G;
    for (int kk = 2; kk <= n; kk <<= 1)
        for (int j = kk >> 1; j > 0; j >>= 1) {
            for (int i = t; i < n / 2; i += G) {
                const int ix = ((i & ~(j - 1)) << 1) | (i & (j - 1));
                const int iy = ix + j;
                const int32_t a = k[ix], b = k[iy];
                if ((a > b) == ((ix & kk) == 0)) {
                    k[ix] = b;
                    k[iy] = a;
                    const double x = v[ix];
                    v[ix] = v[iy];
                    v[iy] = x;
                }
            }
            group_bar<G, BLK>();
        }
}

// Gather the occupied slots of [0, H) into [H, H + u), clearing [0, H); sort; emit; clear [H, H + n).
// cnt: a group-private shared counter (0 on entry; left at 0).
template <int G, int BLK, int H, class VT>
__device__ __forceinline__ void sorted_emit(int32_t* keys, double* vals, int* cnt, int64_t base,
                                            int32_t* __restrict__ C_col, VT* __restrict__ C_val) {
    const int t = threadIdx.x % G;
    for (int s = t; s < H; s += G) {
        const int32_t c = keys[s];
        if (c != EMPTY_KEY) {
            const int at = H + atomicAdd(cnt, 1);
            keys[at] = c;
            vals[at] = vals[s];
            keys[s] = EMPTY_KEY;
            vals[s] = 0.0;
        }
    }
    group_bar<G, BLK>();
    const int u = *cnt;
    int n = 1;
    while (n < u) n <<= 1;
    for (int s = u + t; s < n; s += G) keys[H + s] = INT_MAX;  // pads sort last
    group_bar<G, BLK>();
    bitonic_pairs<G, BLK>(keys + H, vals + H, n);
    for (int i = t; i < u; i += G) {
        st_out(C_col + base + i, keys[H + i]);
        st_out(C_val + base + i, (VT)vals[H + i]);
    }
    group_bar<G, BLK>();
    for (int s = t; s < n; s += G) { keys[H + s] = EMPTY_KEY; vals[H + s] = 0.0; }
    if (t == 0) *cnt = 0;
    group_bar<G, BLK>();
}

#ifndef SG_LIGHT_OCC
#define SG_LIGHT_OCC 1  // emission driven by an occupancy bitmap (0: scan every slot)
#endif
template <int U>
struct LightTable {
    static constexpr int H = 2 * U;  // home range (load <= 1/2)
    static constexpr int P = H + U;  // + overflow room: probing never passes the end (u <= U)
    static constexpr int OW = (P + 31) / 32;  // occupancy words
    // per-row shared memory: vals, keys, occupancy bits, word prefix (+1)
    static constexpr int BYTES = P * 12 + (SG_LIGHT_OCC ? (OW * 4 + (OW + 1) * 4) : 0);
};

template <int U, int R, class VT>
__global__ void __launch_bounds__(32 * R) k_num_light(Mat A, Mat B, const int32_t* __restrict__ list, int64_t cnt,
                                                      int64_t rb, const int2* __restrict__ span,
                                                      const int64_t* __restrict__ C_rp, int32_t* __restrict__ C_col,
                                                      VT* __restrict__ C_val) {
    constexpr int H = LightTable<U>::H, P = LightTable<U>::P, OW = LightTable<U>::OW;
    extern __shared__ double smem_d[];
    __shared__ int s_cnt[R];
    const int g = threadIdx.x / 32, lane = threadIdx.x & 31;
    double* vals = smem_d + g * P;
    int32_t* keys = reinterpret_cast<int32_t*>(smem_d + R * P) + g * P;
    uint32_t* occ = reinterpret_cast<uint32_t*>(reinterpret_cast<int32_t*>(smem_d + R * P) + R * P) + g * OW;
    int* wp = reinterpret_cast<int*>(reinterpret_cast<uint32_t*>(reinterpret_cast<int32_t*>(smem_d + R * P) + R * P) + R * OW) +
              g * (OW + 1);
    for (int s = lane; s < P; s += 32) { keys[s] = EMPTY_KEY; vals[s] = 0.0; }
    if (SG_LIGHT_OCC)
        for (int s = lane; s < OW; s += 32) occ[s] = 0u;
    if (lane == 0) s_cnt[g] = 0;
    __syncwarp();
    for (int64_t j = (int64_t)blockIdx.x * R + g; j < cnt; j += (int64_t)gridDim.x * R) {
        const int64_t li = list[j];
        const int64_t row = rb + li;
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        const int2 sp = span[li];
        if constexpr (U > SKEW_MIN_U) {
            if (sp.x < 0) {  // column-skewed row: sorted path
                for (int64_t pb = s0; pb < s1; pb += 32)
                    chunk_products<true, VT, 2>(A, B, pb, min(pb + 32, s1), [](int, int64_t&, int&) {},
                                                [&](int32_t c, double v) { uni_insert<H>(keys, vals, c, v); });
                __syncwarp();
                sorted_emit<32, 32 * R, H, VT>(keys, vals, &s_cnt[g], C_rp[li], C_col, C_val);
                continue;
            }
        }
        const int64_t width = (int64_t)sp.y - sp.x + 1;
        const bool ident = width <= P;
        const uint64_t mult = ident ? 0 : (((uint64_t)H << 32) / (uint64_t)width);
        const int cmin = sp.x;
        int hmax = -1;
        for (int64_t pb = s0; pb < s1; pb += 32) {
            chunk_products<true, VT, 2>(A, B, pb, min(pb + 32, s1), [](int, int64_t&, int&) {},
                                        [&](int32_t c, double v) {
                                            const int h = SG_LIGHT_OCC
                                                ? acc_insert_occ(keys, vals, occ, c, v, (uint32_t)(c - cmin), ident, mult)
                                                : acc_insert(keys, vals, c, v, (uint32_t)(c - cmin), ident, mult);
                                            hmax = max(hmax, h);
                                        });
        }
        hmax = warp_max(hmax);
        __syncwarp();
        if (SG_LIGHT_OCC) emit_occ<32, 32 * R, VT>(keys, vals, occ, wp, hmax + 1, C_rp[li], C_col, C_val, nullptr, !ident);
        else emit_slots<32, 32 * R, VT>(keys, vals, hmax + 1, C_rp[li], C_col, C_val, nullptr, !ident);
        __syncwarp();
    }
}

template <int U, int NT, class VT>
__global__ void __launch_bounds__(NT) k_num_light_blk(Mat A, Mat B, const int32_t* __restrict__ list, int64_t cnt,
                                                      int64_t rb, const int2* __restrict__ span,
                                                      const int64_t* __restrict__ C_rp, int32_t* __restrict__ C_col,
                                                      VT* __restrict__ C_val) {
    constexpr int H = LightTable<U>::H, P = LightTable<U>::P, OW = LightTable<U>::OW;
    static_assert(!SG_LIGHT_OCC || OW <= NT, "emit_occ: one occupancy word per thread");
    extern __shared__ double smem_d[];
    __shared__ int64_t s_beg[NT];
    __shared__ int s_off[NT];
    __shared__ double s_a[NT];
    __shared__ long long wsll[33];
    __shared__ int ws[NT / 32];
    __shared__ int s_hmax, s_cnt;
    const int tid = threadIdx.x, lane = tid & 31;
    double* vals = smem_d;
    int32_t* keys = reinterpret_cast<int32_t*>(smem_d + P);
    uint32_t* occ = reinterpret_cast<uint32_t*>(keys + P);
    int* wp = reinterpret_cast<int*>(occ + OW);
    for (int s = tid; s < P; s += NT) { keys[s] = EMPTY_KEY; vals[s] = 0.0; }
    if (SG_LIGHT_OCC)
        for (int s = tid; s < OW; s += NT) occ[s] = 0u;
    if (tid == 0) { s_hmax = -1; s_cnt = 0; }
    __syncthreads();
    for (int64_t j = blockIdx.x; j < cnt; j += gridDim.x) {
        const int64_t li = list[j];
        const int64_t row = rb + li;
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        const int2 sp = span[li];
        if (sp.x < 0) {  // column-skewed row (block-uniform): sorted path
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
                    if (c >= 0) uni_insert<H>(keys, vals, c, v);
                });
                __syncthreads();
            }
            sorted_emit<NT, NT, H, VT>(keys, vals, &s_cnt, C_rp[li], C_col, C_val);
            continue;
        }
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
                const int h = SG_LIGHT_OCC ? acc_insert_occ(keys, vals, occ, c, v, (uint32_t)(c - cmin), ident, mult)
                                           : acc_insert(keys, vals, c, v, (uint32_t)(c - cmin), ident, mult);
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
        if (SG_LIGHT_OCC) emit_occ<NT, NT, VT>(keys, vals, occ, wp, nslots, C_rp[li], C_col, C_val, ws, !ident);
        else emit_slots<NT, NT, VT>(keys, vals, nslots, C_rp[li], C_col, C_val, ws, !ident);
        __syncthreads();
    }
}

// ---- numeric, SORTED warp path (rows with w <= 512 when the column fits in 32 - log2 U bits) -----------
// One warp per row: the row's w <= U products are gathered (flattened over its k entries) as 32-bit keys
// (c << log2 U) | j, j = the product's index in the row, with a_ik * b_kj staged in shared memory at j;
// the U keys (padded with all-ones) are bitonic-sorted in registers (U/32 per lane, blocked layout: lane
// exchanges by shuffle, in-lane ones by min/max); then, in striped order, the first key of every column
// run emits the column and the sum of its run's values (summed in product order) at the position given
// by a ballot prefix of the run heads. No hashing and no shared-memory atomics: the light rows of ER or
// permuted R-MAT have almost no duplicate columns (C2: nnz(C) / W = 0.9995), so a probe-and-CAS table
// spends its atomics on entries that never meet.
#ifndef SG_SORT_UNR
#define SG_SORT_UNR 4
#endif
constexpr int SORT_UNR = SG_SORT_UNR;  // gather batches in flight per round

template <int N>
__device__ __forceinline__ void bitonic_warp_blocked(uint32_t (&x)[N / 32]) {
    constexpr int E = N / 32;
    const int lane = threadIdx.x & 31;
    #pragma unroll
    for (int k = 2; k <= N; k <<= 1) {
        #pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
            if (j >= E) {  // partner in lane ^ (j / E), same register
                const int lx = j / E;
                const bool lower = (lane & lx) == 0;
                #pragma unroll
                for (int r = 0; r < E; ++r) {
                    const bool asc = (((lane * E + r) & k) == 0);
                    const uint32_t y = __shfl_xor_sync(FULL, x[r], lx);
                    x[r] = (lower == asc) ? min(x[r], y) : max(x[r], y);
                }
            } else {  // partner in the same lane, register r ^ j
                #pragma unroll
                for (int r = 0; r < E; ++r) {
                    if (r & j) continue;
                    const bool asc = (((lane * E + r) & k) == 0);
                    const uint32_t a = x[r], b = x[r | j];
                    const uint32_t lo = min(a, b), hi = max(a, b);
                    x[r] = asc ? lo : hi;
                    x[r | j] = asc ? hi : lo;
                }
            }
        }
    }
}

// The sorted path is split between the two passes: the SYMBOLIC pass gathers the row's columns, sorts the
// keys and keeps them (the row's slot of U keys in a plan buffer; u_i = the number of column runs); the
// NUMERIC pass gathers only the values, in the same product order j, and emits from the stored keys.
// MODE 1: symbolic (columns -> sorted keys, u_i); MODE 2: numeric (values + stored keys -> C).
template <int U, int R, class VT, int MODE>
__global__ void __launch_bounds__(32 * R, 1024 / (32 * R)) k_light_sort(Mat A, Mat B, const int32_t* __restrict__ list,
                                                                     int64_t cnt, int64_t rb, uint32_t* __restrict__ keys,
                                                                     int64_t* __restrict__ u, const int64_t* __restrict__ C_rp,
                                                                     int32_t* __restrict__ C_col, VT* __restrict__ C_val) {
    static_assert(U >= 32 && (U & (U - 1)) == 0, "U: a power of two >= 32");
    constexpr int E = U / 32, LOGU = __builtin_ctz(U);
    constexpr bool VALS = MODE == 2;
    __shared__ __align__(16) uint32_t skeys[R][U];
    __shared__ double svals[R][VALS ? U : 1];
    const int g = threadIdx.x >> 5, lane = threadIdx.x & 31;
    uint32_t* sk = skeys[g];
    double* sv = svals[g];
    for (int64_t jr = (int64_t)blockIdx.x * R + g; jr < cnt; jr += (int64_t)gridDim.x * R) {
        const int64_t li = list[jr];
        const int64_t row = rb + li;
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        uint32_t* rk = keys + jr * U;  // the row's key slot
        // ---- gather: product j -> key (c << LOGU) | j (symbolic) or value a_ik b_kj at sv[j] (numeric) ----
        int jb = 0;
        for (int64_t pb = s0; pb < s1; pb += 32) {
            const int64_t pa = pb + lane;
            int len = 0;
            int64_t q0 = 0;
            double a = 0.0;
            if (pa < s1) {
                const int k = __ldg(A.col + pa);
                q0 = __ldg(B.rp + k);
                len = (int)(__ldg(B.rp + k + 1) - q0);
                if (VALS) a = ldv<VT>(A.val, pa);
            }
            const int inc = warp_incl_scan(len);
            const int off = inc - len;
            const int tot = __shfl_sync(FULL, inc, 31);
            for (int j0 = 0; j0 < tot; j0 += 32 * SORT_UNR) {
                int c[SORT_UNR];
                double v[SORT_UNR];
                #pragma unroll
                for (int r = 0; r < SORT_UNR; ++r) {
                    const int j = j0 + 32 * r + lane;
                    int sl = 0;
                    #pragma unroll
                    for (int bb = 16; bb; bb >>= 1) {
                        const int o = __shfl_sync(FULL, off, sl + bb);
                        if (o <= j) sl += bb;
                    }
                    const int64_t q = __shfl_sync(FULL, q0, sl) + (j - __shfl_sync(FULL, off, sl));
                    const double as = VALS ? __shfl_sync(FULL, a, sl) : 0.0;
                    c[r] = -1;
                    if (j < tot) {
                        if (VALS) { c[r] = 0; v[r] = as * ldv<VT>(B.val, q); }
                        else c[r] = __ldg(B.col + q);
                    }
                }
                #pragma unroll
                for (int r = 0; r < SORT_UNR; ++r)
                    if (c[r] >= 0) {
                        const int jj = jb + j0 + 32 * r + lane;
                        if (VALS) sv[jj] = v[r];
                        else sk[jj] = ((uint32_t)c[r] << LOGU) | (uint32_t)jj;
                    }
            }
            jb += tot;
        }
        const int w = jb;  // <= U (the bin bound)
        SG_BOUND(w <= U);
        if constexpr (MODE == 1) {
            for (int j = w + lane; j < U; j += 32) sk[j] = 0xFFFFFFFFu;
            __syncwarp();
            // ---- sort (blocked: lane holds keys [lane E, lane E + E)); keep; count the column runs ----
            uint32_t x[E];
            #pragma unroll
            for (int r = 0; r < E; ++r) x[r] = sk[lane * E + r];
            bitonic_warp_blocked<U>(x);
            if constexpr (E % 4 == 0) {
                #pragma unroll
                for (int r = 0; r < E; r += 4)
                    *reinterpret_cast<uint4*>(rk + lane * E + r) = make_uint4(x[r], x[r + 1], x[r + 2], x[r + 3]);
            } else {
                #pragma unroll
                for (int r = 0; r < E; ++r) rk[lane * E + r] = x[r];
            }
            const uint32_t prev_last = __shfl_up_sync(FULL, x[E - 1], 1);
            int heads = 0;
            #pragma unroll
            for (int r = 0; r < E; ++r) {
                const int i = lane * E + r;
                const uint32_t prev = r > 0 ? x[r - 1] : prev_last;
                heads += (i < w && (i == 0 || (prev >> LOGU) != (x[r] >> LOGU))) ? 1 : 0;
            }
            heads = warp_sum(heads);
            if (lane == 0) u[li] = heads;
            __syncwarp();  // sk reused by the next row
        } else {
            // ---- the stored keys; runs of equal columns -> one entry each, in order ----
            for (int e = lane; e < w; e += 32) sk[e] = rk[e];
            __syncwarp();
            const int64_t base = C_rp[li];
            int pos0 = 0;
            for (int e0 = 0; e0 < w; e0 += 32) {
                const int e = e0 + lane;
                const uint32_t key = e < w ? sk[e] : 0xFFFFFFFFu;
                const uint32_t col = key >> LOGU;
                const bool head = e < w && (e == 0 || (sk[e - 1] >> LOGU) != col);
                const unsigned m = __ballot_sync(FULL, head);
                if (head) {
                    double sum = sv[key & (U - 1)];
                    for (int t = e + 1; t < w; ++t) {
                        const uint32_t kt = sk[t];
                        if ((kt >> LOGU) != col) break;
                        sum += sv[kt & (U - 1)];
                    }
                    const int64_t o = base + pos0 + __popc(m & lanemask_lt());
                    st_out(C_col + o, (int32_t)col);
                    st_out(C_val + o, (VT)sum);
                }
                pos0 += __popc(m);
            }
            SG_BOUND(base + pos0 == C_rp[li + 1]);  // exactly the symbolic pass's u_i entries
            __syncwarp();  // sk / sv reused by the next row
        }
    }
}

// key-slot width of bin b on the sorted path (keys per row)
int light_sort_width(int b) { return b < 5 ? 32 : (1 << b); }

template <class VT, int MODE>
static cudaError_t light_sort_V(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, int64_t rb,
                                uint32_t* keys, int64_t* u, const int64_t* C_rp, int32_t* C_col, void* C_val,
                                cudaStream_t s) {
    const char* nm = MODE == 1 ? "k_sym_light_sort" : "k_num_light_sort";
#define SG_SORT_CASE(U_, R_)                                                                                   \
    SG_LAUNCH(nm, s, (k_light_sort<U_, R_, VT, MODE><<<grid_for(cnt, R_, 148 * 32), 32 * R_, 0, s>>>(            \
                         A, B, list, cnt, rb, keys, u, C_rp, C_col, (VT*)C_val)));                             \
    break;
    switch (b) {
        case 0: case 1: case 2: case 3: case 4: case 5: SG_SORT_CASE(32, 8)
        case 6: SG_SORT_CASE(64, 8)
        case 7: SG_SORT_CASE(128, 8)
        case 8: SG_SORT_CASE(256, 8)
        case 9: SG_SORT_CASE(512, 4)
        default: return cudaErrorInvalidValue;
    }
#undef SG_SORT_CASE
    return cudaGetLastError();
}

cudaError_t launch_sym_light_sort(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, int64_t rb,
                                  uint32_t* keys, int64_t* u, cudaStream_t s) {
    if (cnt <= 0) return cudaSuccess;
    return light_sort_V<double, 1>(b, A, B, list, cnt, rb, keys, u, nullptr, nullptr, nullptr, s);
}

cudaError_t launch_num_light_keys(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, int64_t rb,
                                  const uint32_t* keys, const int64_t* C_rp, int32_t* C_col, void* C_val, cudaStream_t s) {
    if (cnt <= 0) return cudaSuccess;
    uint32_t* k = const_cast<uint32_t*>(keys);
    return A.dt == 0 ? light_sort_V<double, 2>(b, A, B, list, cnt, rb, k, nullptr, C_rp, C_col, C_val, s)
                     : light_sort_V<float, 2>(b, A, B, list, cnt, rb, k, nullptr, C_rp, C_col, C_val, s);
}

// the sorted warp path applies to bin b (U = 2^b) when its keys fit: c < 2^(32 - log2 max(U, 32))
#ifndef SG_LIGHT_SORT
#define SG_LIGHT_SORT 1
#endif
bool light_sorted(int b, int64_t p, int variant) {
    const int lu = b < 5 ? 5 : b;
    return SG_LIGHT_SORT && !(variant & 16) && b <= 9 && p <= ((int64_t)1 << (32 - lu));
}

template <class VT>
static cudaError_t num_light_V(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, int64_t rb,
                               const int2* span, const int64_t* C_rp, int32_t* C_col, void* C_val, cudaStream_t s) {
    switch (b) {
#define X(B_, U_, R_)                                                                                         \
    case B_: {                                                                                                \
        auto kern = k_num_light<U_, R_, VT>;                                                                  \
        const int smem = R_ * LightTable<U_>::BYTES;                                                          \
        if (smem > 48 * 1024) {                                                                               \
            cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);     \
            if (e != cudaSuccess) return e;                                                                   \
        }                                                                                                     \
        SG_LAUNCH("k_num_light", s, (kern<<<grid_for(cnt, R_, 148 * 32), 32 * R_, smem, s>>>(                 \
                                        A, B, list, cnt, rb, span, C_rp, C_col, (VT*)C_val)));                 \
        break;                                                                                                \
    }
        SG_NUM_LIGHT_WARP_BINS(X)
#undef X
#define X(B_, U_, NT_)                                                                                        \
    case B_: {                                                                                                \
        auto kern = k_num_light_blk<U_, NT_, VT>;                                                             \
        const int smem = LightTable<U_>::BYTES;                                                               \
        if (smem > 48 * 1024) {                                                                               \
            cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);     \
            if (e != cudaSuccess) return e;                                                                   \
        }                                                                                                     \
        SG_LAUNCH("k_num_light", s, (kern<<<grid_for(cnt, 1, 148 * 16), NT_, smem, s>>>(                      \
                                        A, B, list, cnt, rb, span, C_rp, C_col, (VT*)C_val)));                 \
        break;                                                                                                \
    }
        SG_NUM_LIGHT_BLOCK_BINS(X)
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
