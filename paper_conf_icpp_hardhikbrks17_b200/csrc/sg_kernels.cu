// sg_kernels.cu — the sm_100a kernels of the hot path.
//
//   a1 k_row_work        w_i = sum_{k in A_i} nnz(B_k)
//   a2 k_scan_*          exclusive prefix (P of w; C.row_ptr of u)          PAPER L217 (V_L)
//   a3 k_samp_*          Bernoulli row sample S by SplitMix64
//      k_cost_hist/k_argmin  J(t;S) histogram + smallest argmin
//   a4 k_cuts            closest-prefix row cuts
//   a5 k_bin_*           EMPTY / LIGHT(2^b bins) / HEAVY by thr
//   a6 k_sym_light / k_sym_heavy   u_i = nnz(C_i) (+ heavy range plan)
//   a7+a8 k_num_light / k_num_heavy  c_ij = sum_k a_ik b_kj, sorted CSR out
//
// Accumulator: an ORDER-PRESERVING linear-probing hash in shared memory. The home slot of column
// c is monotone in c, so occupied runs ("clusters") are mutually ordered; sorting each short
// cluster in place and compacting occupied slots in slot order yields the row in ascending column
// order without a sort of the whole row. When the row's (or range's) column span
// fits the table, the map is the identity (a dense accumulator, no probing).
#include "sg_internal.cuh"
#include <climits>

namespace sg {

// ------------------------------------------------------------------------------------------------
// small helpers
// ------------------------------------------------------------------------------------------------
__device__ __forceinline__ uint64_t sm64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}
__device__ __forceinline__ uint64_t h3(uint64_t seed, uint64_t tag, uint64_t j) {
    return sm64(seed ^ sm64(tag ^ sm64(j)));
}

template <class T> __device__ __forceinline__ T warp_sum(T v) {
    #pragma unroll
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}
__device__ __forceinline__ int warp_min(int v) {
    #pragma unroll
    for (int o = 16; o; o >>= 1) v = min(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}
__device__ __forceinline__ int warp_max(int v) {
    #pragma unroll
    for (int o = 16; o; o >>= 1) v = max(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}
template <class T> __device__ __forceinline__ T warp_incl_scan(T v) {
    int lane = threadIdx.x & 31;
    #pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T y = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o) v += y;
    }
    return v;
}

template <class VT> __device__ __forceinline__ double ldv(const void* v, int64_t q) {
    return (double)__ldg(reinterpret_cast<const VT*>(v) + q);
}

static inline int grid_for(int64_t work, int per_block, int max_blocks) {
    int64_t g = (work + per_block - 1) / per_block;
    if (g < 1) g = 1;
    if (g > max_blocks) g = max_blocks;
    return (int)g;
}

// ------------------------------------------------------------------------------------------------
// a1: row work
// ------------------------------------------------------------------------------------------------
__global__ void k_row_work(Mat A, Mat B, int64_t rb, int64_t re, int64_t* __restrict__ w) {
    const int lane = threadIdx.x & 31;
    int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t i = rb + warp; i < re; i += nw) {
        int64_t s = A.rp[i], e = A.rp[i + 1];
        long long acc = 0;
        for (int64_t p = s + lane; p < e; p += 32) {
            int k = __ldg(A.col + p);
            acc += __ldg(B.rp + k + 1) - __ldg(B.rp + k);
        }
        acc = warp_sum(acc);
        if (lane == 0) w[i - rb] = acc;
    }
}

cudaError_t launch_row_work(const Mat& A, const Mat& B, int64_t rb, int64_t re, int64_t* w, cudaStream_t s) {
    if (re <= rb) return cudaSuccess;
    k_row_work<<<grid_for(re - rb, 8, 148 * 32), 256, 0, s>>>(A, B, rb, re, w);
    return cudaGetLastError();
}

__global__ void k_row_work_list(Mat A, Mat B, const int64_t* __restrict__ rows, int64_t nr, int64_t* __restrict__ w,
                                int64_t* __restrict__ a) {
    const int lane = threadIdx.x & 31;
    int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t j = warp; j < nr; j += nw) {
        int64_t i = rows[j];
        int64_t s = A.rp[i], e = A.rp[i + 1];
        long long acc = 0;
        for (int64_t p = s + lane; p < e; p += 32) {
            int k = __ldg(A.col + p);
            acc += __ldg(B.rp + k + 1) - __ldg(B.rp + k);
        }
        acc = warp_sum(acc);
        if (lane == 0) { w[j] = acc; a[j] = e - s; }
    }
}

cudaError_t launch_row_work_list(const Mat& A, const Mat& B, const int64_t* rows, int64_t nr, int64_t* w,
                                 int64_t* a, cudaStream_t s) {
    if (nr <= 0) return cudaSuccess;
    k_row_work_list<<<grid_for(nr, 8, 148 * 32), 256, 0, s>>>(A, B, rows, nr, w, a);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// a2: exclusive scan (int64), three kernels per level, recursive over block sums
// ------------------------------------------------------------------------------------------------
constexpr int SCAN_T = 256, SCAN_I = 8, SCAN_TILE = SCAN_T * SCAN_I;

__device__ __forceinline__ long long block_excl_scan(long long v, long long* total) {
    __shared__ long long ws[SCAN_T / 32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    long long inc = warp_incl_scan(v);
    if (lane == 31) ws[wid] = inc;
    __syncthreads();
    if (wid == 0) {
        long long x = lane < SCAN_T / 32 ? ws[lane] : 0;
        long long xi = warp_incl_scan(x);
        if (lane < SCAN_T / 32) ws[lane] = xi - x;
        if (lane == 31) *total = xi;
    }
    __syncthreads();
    long long r = ws[wid] + inc - v;
    __syncthreads();
    return r;
}

__global__ void __launch_bounds__(SCAN_T) k_scan_tile(const int64_t* __restrict__ in, int64_t* __restrict__ out,
                                                      int64_t n, int64_t* __restrict__ bsum) {
    __shared__ long long tot;
    int64_t base = (int64_t)blockIdx.x * SCAN_TILE + threadIdx.x * SCAN_I;
    long long v[SCAN_I];
    long long t = 0;
    #pragma unroll
    for (int i = 0; i < SCAN_I; ++i) { v[i] = base + i < n ? in[base + i] : 0; t += v[i]; }
    long long ex = block_excl_scan(t, &tot);
    #pragma unroll
    for (int i = 0; i < SCAN_I; ++i) {
        if (base + i < n) out[base + i] = ex;
        ex += v[i];
    }
    if (threadIdx.x == 0) bsum[blockIdx.x] = tot;
}

__global__ void k_scan_add(int64_t* __restrict__ out, int64_t n, const int64_t* __restrict__ bscan, int64_t nb) {
    int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (j < n) out[j] += bscan[j / SCAN_TILE];
    if (j == n) out[n] = bscan[nb];
}

size_t scan_tmp_bytes(int64_t n) {
    if (n <= SCAN_TILE) return 2 * sizeof(int64_t) * 2;
    int64_t nb = (n + SCAN_TILE - 1) / SCAN_TILE;
    return sizeof(int64_t) * (size_t)(2 * nb + 1) + scan_tmp_bytes(nb);
}

cudaError_t scan_exclusive(const int64_t* in, int64_t* out, int64_t n, void* tmp, cudaStream_t s) {
    if (n <= 0) return cudaMemsetAsync(out, 0, sizeof(int64_t), s);
    int64_t nb = (n + SCAN_TILE - 1) / SCAN_TILE;
    int64_t* bsum = (int64_t*)tmp;
    int64_t* bscan = bsum + nb;
    k_scan_tile<<<(unsigned)nb, SCAN_T, 0, s>>>(in, out, n, bsum);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    if (nb == 1) {
        // bscan = [0, total]
        e = cudaMemsetAsync(bscan, 0, sizeof(int64_t), s);
        if (e != cudaSuccess) return e;
        e = cudaMemcpyAsync(bscan + 1, bsum, sizeof(int64_t), cudaMemcpyDeviceToDevice, s);
    } else {
        e = scan_exclusive(bsum, bscan, nb, bscan + nb + 1, s);
    }
    if (e != cudaSuccess) return e;
    k_scan_add<<<(unsigned)((n + 1 + 255) / 256), 256, 0, s>>>(out, n, bscan, nb);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// a3: Bernoulli(f) row sample, stable (ascending) selection
// ------------------------------------------------------------------------------------------------
__device__ __forceinline__ bool sampled(int64_t i, uint64_t seed, uint64_t Tf, bool all) {
    return all || h3(seed, TAG_SAMPLE, (uint64_t)i) < Tf;
}

__global__ void __launch_bounds__(SCAN_T) k_samp_count(int64_t rb, int64_t re, uint64_t seed, uint64_t Tf, bool all,
                                                       int64_t* __restrict__ bsum) {
    __shared__ long long tot;
    int64_t base = rb + (int64_t)blockIdx.x * SCAN_TILE + threadIdx.x * SCAN_I;
    long long c = 0;
    for (int i = 0; i < SCAN_I; ++i)
        if (base + i < re && sampled(base + i, seed, Tf, all)) ++c;
    block_excl_scan(c, &tot);
    if (threadIdx.x == 0) bsum[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(SCAN_T) k_samp_write(int64_t rb, int64_t re, uint64_t seed, uint64_t Tf, bool all,
                                                       const int64_t* __restrict__ bscan, int64_t* __restrict__ out,
                                                       int64_t nb, int64_t* __restrict__ d_count) {
    __shared__ long long tot;
    int64_t base = rb + (int64_t)blockIdx.x * SCAN_TILE + threadIdx.x * SCAN_I;
    bool f[SCAN_I];
    long long c = 0;
    for (int i = 0; i < SCAN_I; ++i) { f[i] = base + i < re && sampled(base + i, seed, Tf, all); c += f[i]; }
    long long ex = block_excl_scan(c, &tot) + bscan[blockIdx.x];
    for (int i = 0; i < SCAN_I; ++i)
        if (f[i]) out[ex++] = base + i;
    if (blockIdx.x == 0 && threadIdx.x == 0) *d_count = bscan[nb];
}

size_t sample_tmp_bytes(int64_t n) {
    int64_t nb = (n + SCAN_TILE - 1) / SCAN_TILE;
    if (nb < 1) nb = 1;
    return sizeof(int64_t) * (size_t)(2 * nb + 1) + scan_tmp_bytes(nb);
}

cudaError_t launch_sample_select(int64_t rb, int64_t re, uint64_t seed, uint64_t Tf, bool all, int64_t* out_rows,
                                 int64_t* d_count, void* tmp, size_t, cudaStream_t s) {
    int64_t n = re - rb;
    if (n <= 0) return cudaMemsetAsync(d_count, 0, sizeof(int64_t), s);
    int64_t nb = (n + SCAN_TILE - 1) / SCAN_TILE;
    int64_t* bsum = (int64_t*)tmp;
    int64_t* bscan = bsum + nb;
    k_samp_count<<<(unsigned)nb, SCAN_T, 0, s>>>(rb, re, seed, Tf, all, bsum);
    cudaError_t e = scan_exclusive(bsum, bscan, nb, bscan + nb + 1, s);
    if (e != cudaSuccess) return e;
    k_samp_write<<<(unsigned)nb, SCAN_T, 0, s>>>(rb, re, seed, Tf, all, bscan, out_rows, nb, d_count);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// a5: binning (EMPTY / LIGHT bins by ceil(log2 w) / HEAVY)
// ------------------------------------------------------------------------------------------------
__device__ __forceinline__ int bin_of(int64_t w, int64_t thr) {
    if (w == 0) return BIN_EMPTY;
    if (w > thr) return BIN_HEAVY;
    return w <= 1 ? 0 : 64 - __clzll((unsigned long long)(w - 1));
}

__global__ void k_bin_count(const int64_t* __restrict__ w, int64_t nr, int64_t thr, unsigned long long* cnt,
                            int8_t* cls) {
    __shared__ unsigned int sc[NBINS];
    if (threadIdx.x < NBINS) sc[threadIdx.x] = 0;
    __syncthreads();
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nr; j += (int64_t)gridDim.x * blockDim.x) {
        int b = bin_of(w[j], thr);
        atomicAdd(&sc[b], 1u);
        if (cls) cls[j] = b == BIN_EMPTY ? 0 : (b == BIN_HEAVY ? 2 : 1);
    }
    __syncthreads();
    if (threadIdx.x < NBINS && sc[threadIdx.x]) atomicAdd(&cnt[threadIdx.x], (unsigned long long)sc[threadIdx.x]);
}

cudaError_t launch_bin_count(const int64_t* w, int64_t nr, int64_t thr, int64_t* d_cnt, int8_t* cls, cudaStream_t s) {
    if (nr <= 0) return cudaSuccess;
    k_bin_count<<<grid_for(nr, 1024, 148 * 8), 256, 0, s>>>(w, nr, thr, (unsigned long long*)d_cnt, cls);
    return cudaGetLastError();
}

__global__ void k_bin_scatter(const int64_t* __restrict__ w, int64_t nr, int64_t thr, unsigned long long* cursor,
                              int32_t* __restrict__ lists) {
    __shared__ unsigned int sc[NBINS];
    __shared__ unsigned long long sb[NBINS];
    const int64_t per = 1024;
    for (int64_t c0 = (int64_t)blockIdx.x * per; c0 < nr; c0 += (int64_t)gridDim.x * per) {
        if (threadIdx.x < NBINS) sc[threadIdx.x] = 0;
        __syncthreads();
        int b[4];
        unsigned r[4];
        #pragma unroll
        for (int i = 0; i < 4; ++i) {
            int64_t j = c0 + threadIdx.x + i * 256;
            b[i] = -1;
            if (j < nr) { b[i] = bin_of(w[j], thr); r[i] = atomicAdd(&sc[b[i]], 1u); }
        }
        __syncthreads();
        if (threadIdx.x < NBINS) sb[threadIdx.x] = sc[threadIdx.x] ? atomicAdd(&cursor[threadIdx.x], (unsigned long long)sc[threadIdx.x]) : 0;
        __syncthreads();
        #pragma unroll
        for (int i = 0; i < 4; ++i) {
            int64_t j = c0 + threadIdx.x + i * 256;
            if (b[i] >= 0) lists[sb[b[i]] + r[i]] = (int32_t)j;
        }
        __syncthreads();
    }
}

cudaError_t launch_bin_scatter(const int64_t* w, int64_t nr, int64_t thr, int64_t* d_cursor, int32_t* lists,
                               cudaStream_t s) {
    if (nr <= 0) return cudaSuccess;
    k_bin_scatter<<<grid_for(nr, 1024, 148 * 8), 256, 0, s>>>(w, nr, thr, (unsigned long long*)d_cursor, lists);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// group synchronisation: G == 32 -> one warp per row; otherwise one block per row (G == BLK)
// ------------------------------------------------------------------------------------------------
template <int G> __device__ __forceinline__ void gsync() {
    if constexpr (G == 32) __syncwarp(); else __syncthreads();
}
// exclusive prefix of a per-thread count within the group + group total
template <int G> __device__ __forceinline__ int gscan(int c, int* total, int* ws /*>= G/32 ints*/) {
    const int lane = threadIdx.x & 31;
    int inc = warp_incl_scan(c);
    if constexpr (G == 32) {
        *total = __shfl_sync(0xffffffffu, inc, 31);
        return inc - c;
    } else {
        const int wid = threadIdx.x >> 5;
        if (lane == 31) ws[wid] = inc;
        __syncthreads();
        int before = 0, tot = 0;
        #pragma unroll 4
        for (int q = 0; q < G / 32; ++q) { int x = ws[q]; tot += x; if (q < wid) before += x; }
        __syncthreads();
        *total = tot;
        return before + inc - c;
    }
}
template <int G> __device__ __forceinline__ long long gsum(long long v, long long* ws) {
    v = warp_sum(v);
    if constexpr (G == 32) return v;
    else {
        const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
        if (lane == 0) ws[wid] = v;
        __syncthreads();
        long long t = 0;
        for (int q = 0; q < G / 32; ++q) t += ws[q];
        __syncthreads();
        return t;
    }
}
template <int G> __device__ __forceinline__ void gminmax(int& mn, int& mx, int* ws) {
    mn = warp_min(mn);
    mx = warp_max(mx);
    if constexpr (G != 32) {
        const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
        if (lane == 0) { ws[2 * wid] = mn; ws[2 * wid + 1] = mx; }
        __syncthreads();
        mn = INT_MAX; mx = -1;
        for (int q = 0; q < G / 32; ++q) { mn = min(mn, ws[2 * q]); mx = max(mx, ws[2 * q + 1]); }
        __syncthreads();
    }
}

// ------------------------------------------------------------------------------------------------
// a6 light: exact u_i with a keys-only hash set per row (any hash: order is irrelevant here)
// ------------------------------------------------------------------------------------------------
template <int U, int G, int BLK>
__global__ void __launch_bounds__(BLK) k_sym_light(Mat A, Mat B, const int32_t* __restrict__ list, int64_t cnt,
                                                   const int64_t* __restrict__ rowmap, int64_t rb,
                                                   int64_t* __restrict__ u) {
    constexpr int P = 2 * U < 32 ? 32 : 2 * U;   // power of two
    constexpr int LOGP = __builtin_ctz(P);
    constexpr int R = BLK / G;
    __shared__ int32_t tab[R * P];
    __shared__ long long ws[BLK / 32 > 0 ? BLK / 32 : 1];
    const int g = threadIdx.x / G, t = threadIdx.x % G;
    int32_t* T = tab + g * P;
    for (int s = t; s < P; s += G) T[s] = EMPTY_KEY;
    gsync<G>();
    for (int64_t j = (int64_t)blockIdx.x * R + g; j < cnt; j += (int64_t)gridDim.x * R) {
        int64_t li = list[j];
        int64_t row = rowmap ? rowmap[li] : rb + li;
        int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        long long ins = 0;
        for (int64_t pa = s0; pa < s1; ++pa) {
            int k = __ldg(A.col + pa);
            int64_t q0 = __ldg(B.rp + k), q1 = __ldg(B.rp + k + 1);
            for (int64_t q = q0 + t; q < q1; q += G) {
                int32_t c = __ldg(B.col + q);
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
            }
        }
        long long tot = gsum<G>(ins, ws);
        if (t == 0) u[li] = tot;
        gsync<G>();
        for (int s = t; s < P; s += G) T[s] = EMPTY_KEY;
        gsync<G>();
    }
}

template <int U, int G, int BLK>
static cudaError_t sym_light_T(const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, const int64_t* rowmap,
                               int64_t rb, int64_t* u, cudaStream_t s) {
    constexpr int R = BLK / G;
    int grid = grid_for(cnt, R, 148 * 16);
    k_sym_light<U, G, BLK><<<grid, BLK, 0, s>>>(A, B, list, cnt, rowmap, rb, u);
    return cudaGetLastError();
}

cudaError_t launch_sym_light(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt,
                             const int64_t* rowmap, int64_t rb, int64_t* u, cudaStream_t s) {
    if (cnt <= 0) return cudaSuccess;
    switch (b) {
        case 0: return sym_light_T<1, 32, 256>(A, B, list, cnt, rowmap, rb, u, s);
        case 1: return sym_light_T<2, 32, 256>(A, B, list, cnt, rowmap, rb, u, s);
        case 2: return sym_light_T<4, 32, 256>(A, B, list, cnt, rowmap, rb, u, s);
        case 3: return sym_light_T<8, 32, 256>(A, B, list, cnt, rowmap, rb, u, s);
        case 4: return sym_light_T<16, 32, 256>(A, B, list, cnt, rowmap, rb, u, s);
        case 5: return sym_light_T<32, 32, 256>(A, B, list, cnt, rowmap, rb, u, s);
        case 6: return sym_light_T<64, 32, 256>(A, B, list, cnt, rowmap, rb, u, s);
        case 7: return sym_light_T<128, 32, 256>(A, B, list, cnt, rowmap, rb, u, s);
        case 8: return sym_light_T<256, 32, 256>(A, B, list, cnt, rowmap, rb, u, s);
        case 9: return sym_light_T<512, 64, 64>(A, B, list, cnt, rowmap, rb, u, s);
        case 10: return sym_light_T<1024, 128, 128>(A, B, list, cnt, rowmap, rb, u, s);
        case 11: return sym_light_T<2048, 256, 256>(A, B, list, cnt, rowmap, rb, u, s);
        case 12: return sym_light_T<4096, 512, 512>(A, B, list, cnt, rowmap, rb, u, s);
        default: return cudaErrorInvalidValue;
    }
}

// ------------------------------------------------------------------------------------------------
// a6 heavy: bitmap over a column window, per-tile popcounts, greedy range plan
// ------------------------------------------------------------------------------------------------
__device__ __forceinline__ int64_t lower_bound_col(const int32_t* __restrict__ col, int64_t lo, int64_t hi, int64_t x) {
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if ((int64_t)__ldg(col + mid) < x) lo = mid + 1; else hi = mid;
    }
    return lo;
}

__global__ void __launch_bounds__(HEAVY_THREADS, 1) k_sym_heavy(Mat A, Mat B, const int32_t* __restrict__ list,
                                                                 int64_t cnt, const int64_t* __restrict__ rowmap,
                                                                 int64_t rb, int64_t* __restrict__ u,
                                                                 const int64_t* __restrict__ range_off,
                                                                 RangeRec* __restrict__ ranges) {
    extern __shared__ uint32_t bm[];                 // WIN/32 words
    __shared__ int32_t tcnt[WIN / TW];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nwarps = HEAVY_THREADS / 32;
    const int64_t p = B.ncols;
    const int64_t nwin = (p + WIN - 1) / WIN;
    for (int64_t j = blockIdx.x; j < cnt; j += gridDim.x) {
        int64_t li = list[j];
        int64_t row = rowmap ? rowmap[li] : rb + li;
        int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        long long utot = 0;
        int nr = 0, off = 0;
        for (int64_t win = 0; win < nwin; ++win) {
            const int64_t wlo = win * WIN, whi = min(p, wlo + WIN);
            const int nwords = (int)((whi - wlo + 31) / 32);
            for (int q = threadIdx.x; q < nwords; q += HEAVY_THREADS) bm[q] = 0u;
            __syncthreads();
            for (int64_t pa = s0 + wid; pa < s1; pa += nwarps) {
                int k = __ldg(A.col + pa);
                int64_t q0 = __ldg(B.rp + k), q1 = __ldg(B.rp + k + 1);
                if (nwin > 1) {
                    int64_t a = 0, b = 0;
                    if (lane == 0) { a = lower_bound_col(B.col, q0, q1, wlo); b = lower_bound_col(B.col, a, q1, whi); }
                    q0 = __shfl_sync(0xffffffffu, a, 0);
                    q1 = __shfl_sync(0xffffffffu, b, 0);
                }
                for (int64_t q = q0 + lane; q < q1; q += 32) {
                    uint32_t c = (uint32_t)(__ldg(B.col + q) - wlo);
                    atomicOr(&bm[c >> 5], 1u << (c & 31));
                }
            }
            __syncthreads();
            const int nt = (int)((whi - wlo + TW - 1) / TW);
            for (int tt = wid; tt < nt; tt += nwarps) {
                int a = tt * (TW / 32), b = min(nwords, a + TW / 32);
                int c = 0;
                for (int q = a + lane; q < b; q += 32) c += __popc(bm[q]);
                c = warp_sum(c);
                if (lane == 0) tcnt[tt] = c;
            }
            __syncthreads();
            if (threadIdx.x == 0) {
                const int tg0 = (int)(wlo / TW);
                bool open = false;
                int t0 = 0, t1 = 0, cur = 0;
                auto emit = [&](int a, int b, int c) {
                    if (c > 0) {
                        if (ranges) {
                            RangeRec r;
                            r.row = (int32_t)li; r.t0 = a; r.t1 = b; r.cnt = c; r.off = off; r.pad = 0;
                            ranges[range_off[j] + nr] = r;
                        }
                        off += c;
                        ++nr;
                    }
                };
                for (int tt = 0; tt < nt; ++tt) {
                    int c = tcnt[tt];
                    utot += c;
                    if (open && cur + c <= CAPU) { cur += c; t1 = tg0 + tt + 1; continue; }
                    if (open) emit(t0, t1, cur);
                    open = true; t0 = tg0 + tt; t1 = t0 + 1; cur = c;
                    if (cur > CAPU) { emit(t0, t1, cur); open = false; }
                }
                if (open) emit(t0, t1, cur);
            }
            __syncthreads();
        }
        if (threadIdx.x == 0) u[li] = utot;
    }
}

cudaError_t launch_sym_heavy(const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, const int64_t* rowmap,
                             int64_t rb, const int64_t*, int64_t* u, const int64_t* range_off, RangeRec* ranges,
                             cudaStream_t s) {
    if (cnt <= 0) return cudaSuccess;
    const int smem = (WIN / 32) * 4;
    static bool attr = false;
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(k_sym_heavy, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
        attr = true;
    }
    int grid = (int)(cnt < 148 * 4 ? cnt : 148 * 4);
    k_sym_heavy<<<grid, HEAVY_THREADS, smem, s>>>(A, B, list, cnt, rowmap, rb, u, range_off, ranges);
    return cudaGetLastError();
}

// per heavy row: an upper bound on its range count
__global__ void k_range_bounds(const int32_t* __restrict__ heavy, int64_t nh, const int64_t* __restrict__ w,
                               int64_t p, int64_t* __restrict__ bounds) {
    int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (j >= nh) return;
    int64_t wi = w[heavy[j]];
    int64_t mu = wi < p ? wi : p;
    int64_t T = (p + TW - 1) / TW;
    int64_t nwin = (p + WIN - 1) / WIN;
    int64_t b = 2 * mu / CAPU + nwin + 1;
    bounds[j] = b < T ? b : T;
}

cudaError_t launch_range_bounds(const int32_t* heavy, int64_t nh, const int64_t* w, int64_t p, int64_t* bounds,
                                cudaStream_t s) {
    if (nh <= 0) return cudaSuccess;
    k_range_bounds<<<(unsigned)((nh + 255) / 256), 256, 0, s>>>(heavy, nh, w, p, bounds);
    return cudaGetLastError();
}

__global__ void k_fill_unused(RangeRec* r, int64_t n) {
    int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (j < n) { RangeRec x; x.row = -1; x.t0 = x.t1 = x.cnt = x.off = x.pad = 0; r[j] = x; }
}

cudaError_t launch_fill_ranges_unused(RangeRec* r, int64_t n, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    k_fill_unused<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(r, n);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// B tile pointers: for B rows longer than LONG_ROW, tp[id][t] = #entries with col < t*TW
// ------------------------------------------------------------------------------------------------
__global__ void k_long_rows(Mat B, int32_t* __restrict__ long_id, unsigned long long* nlong) {
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < B.nrows; k += (int64_t)gridDim.x * blockDim.x) {
        int64_t len = B.rp[k + 1] - B.rp[k];
        long_id[k] = len > LONG_ROW ? (int32_t)atomicAdd(nlong, 1ull) : -1;
    }
}

cudaError_t launch_long_rows(const Mat& B, int32_t* long_id, int64_t* d_nlong, cudaStream_t s) {
    if (B.nrows <= 0) return cudaSuccess;
    k_long_rows<<<grid_for(B.nrows, 256, 148 * 8), 256, 0, s>>>(B, long_id, (unsigned long long*)d_nlong);
    return cudaGetLastError();
}

__global__ void k_build_tp(Mat B, const int32_t* __restrict__ long_id, int T, uint32_t* __restrict__ tp) {
    const int lane = threadIdx.x & 31;
    int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t k = warp; k < B.nrows; k += nw) {
        int id = long_id[k];
        if (id < 0) continue;
        int64_t q0 = B.rp[k], q1 = B.rp[k + 1];
        uint32_t* row = tp + (int64_t)id * (T + 1);
        for (int t = lane; t <= T; t += 32)
            row[t] = (uint32_t)(lower_bound_col(B.col, q0, q1, (int64_t)t * TW) - q0);
    }
}

cudaError_t launch_build_tp(const Mat& B, const int32_t* long_id, int T, uint32_t* tp, cudaStream_t s) {
    if (B.nrows <= 0) return cudaSuccess;
    k_build_tp<<<grid_for(B.nrows, 8, 148 * 16), 256, 0, s>>>(B, long_id, T, tp);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// a7 + a8: numeric with the order-preserving hash accumulator
// ------------------------------------------------------------------------------------------------
// insert (c, v): identity map when `ident`, else linear probing from the monotone home slot
__device__ __forceinline__ void acc_insert(int32_t* keys, double* vals, int32_t c, double v, uint32_t d,
                                           bool ident, uint64_t mult) {
    uint32_t h;
    if (ident) {
        h = d;
        if (keys[h] != c) keys[h] = c;           // idempotent: every writer stores the same key
    } else {
        h = (uint32_t)(((uint64_t)d * mult) >> 32);
        while (true) {
            int32_t old = keys[h];
            if (old == c) break;
            if (old == EMPTY_KEY) {
                old = atomicCAS(&keys[h], EMPTY_KEY, c);
                if (old == EMPTY_KEY || old == c) break;
            }
            ++h;
        }
    }
    atomicAdd(&vals[h], v);
}

// sort the occupied run starting at slot s (insertion sort; runs are short at load <= 0.5)
__device__ __forceinline__ void sort_run(int32_t* keys, double* vals, int s, int P) {
    int e = s + 1;
    while (e < P && keys[e] != EMPTY_KEY) ++e;
    for (int i = s + 1; i < e; ++i) {
        int32_t k = keys[i];
        double v = vals[i];
        int q = i - 1;
        while (q >= s && keys[q] > k) { keys[q + 1] = keys[q]; vals[q + 1] = vals[q]; --q; }
        keys[q + 1] = k;
        vals[q + 1] = v;
    }
}

// group-wide: sort clusters (hash mode), then compact slots [0, nslots) in order into C at `base`,
// clearing every slot it empties.
template <int G, class VT>
__device__ __forceinline__ void emit_sorted(int32_t* keys, double* vals, int nslots, bool ident, int64_t base,
                                            int32_t* __restrict__ C_col, VT* __restrict__ C_val, int* ws) {
    const int t = threadIdx.x % G;
    if (!ident) {
        for (int s = t; s < nslots; s += G)
            if (keys[s] != EMPTY_KEY && (s == 0 || keys[s - 1] == EMPTY_KEY)) sort_run(keys, vals, s, nslots);
        gsync<G>();
    }
    int64_t pos = base;
    for (int s0 = 0; s0 < nslots; s0 += G) {
        int s = s0 + t;
        int32_t k = s < nslots ? keys[s] : EMPTY_KEY;
        int occ = k != EMPTY_KEY;
        int tot;
        int ex = gscan<G>(occ, &tot, ws);
        if (occ) {
            C_col[pos + ex] = k;
            C_val[pos + ex] = (VT)vals[s];
            keys[s] = EMPTY_KEY;
            vals[s] = 0.0;
        }
        pos += tot;
    }
}

template <int U, int G, int BLK, class VT>
__global__ void __launch_bounds__(BLK) k_num_light(Mat A, Mat B, const int32_t* __restrict__ list, int64_t cnt,
                                                   int64_t rb, const int64_t* __restrict__ C_rp,
                                                   int32_t* __restrict__ C_col, VT* __restrict__ C_val) {
    constexpr int P = 3 * U < 4 ? 4 : 3 * U;
    constexpr int H = 2 * U;
    constexpr int R = BLK / G;
    extern __shared__ double smem_d[];
    double* vals_all = smem_d;
    int32_t* keys_all = reinterpret_cast<int32_t*>(vals_all + R * P);
    __shared__ int ws[2 * (BLK / 32 > 0 ? BLK / 32 : 1)];
    const int g = threadIdx.x / G, t = threadIdx.x % G;
    double* vals = vals_all + g * P;
    int32_t* keys = keys_all + g * P;
    for (int s = t; s < P; s += G) { keys[s] = EMPTY_KEY; vals[s] = 0.0; }
    gsync<G>();
    for (int64_t j = (int64_t)blockIdx.x * R + g; j < cnt; j += (int64_t)gridDim.x * R) {
        int64_t li = list[j];
        int64_t row = rb + li;
        int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        // column span of the row's output: min first / max last column of the B_k rows
        int cmin = INT_MAX, cmax = -1;
        for (int64_t pa = s0 + t; pa < s1; pa += G) {
            int k = __ldg(A.col + pa);
            int64_t q0 = __ldg(B.rp + k), q1 = __ldg(B.rp + k + 1);
            if (q1 > q0) { cmin = min(cmin, __ldg(B.col + q0)); cmax = max(cmax, __ldg(B.col + q1 - 1)); }
        }
        gminmax<G>(cmin, cmax, ws);
        const int64_t span = (int64_t)cmax - cmin + 1;
        const bool ident = span <= P;
        const uint64_t mult = ident ? 0 : (((uint64_t)H << 32) / (uint64_t)span);
        for (int64_t pa = s0; pa < s1; ++pa) {
            int k = __ldg(A.col + pa);
            double a = ldv<VT>(A.val, pa);
            int64_t q0 = __ldg(B.rp + k), q1 = __ldg(B.rp + k + 1);
            for (int64_t q = q0 + t; q < q1; q += G) {
                int32_t c = __ldg(B.col + q);
                acc_insert(keys, vals, c, a * ldv<VT>(B.val, q), (uint32_t)(c - cmin), ident, mult);
            }
        }
        gsync<G>();
        emit_sorted<G, VT>(keys, vals, ident ? (int)span : P, ident, C_rp[li], C_col, C_val, ws);
        gsync<G>();
    }
}

template <int U, int G, int BLK, class VT>
static cudaError_t num_light_T(const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, int64_t rb,
                               const int64_t* C_rp, int32_t* C_col, void* C_val, cudaStream_t s) {
    constexpr int P = 3 * U < 4 ? 4 : 3 * U;
    constexpr int R = BLK / G;
    const int smem = R * P * (8 + 4);
    auto kern = k_num_light<U, G, BLK, VT>;
    if (smem > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
    }
    int grid = grid_for(cnt, R, 148 * 16);
    kern<<<grid, BLK, smem, s>>>(A, B, list, cnt, rb, C_rp, C_col, (VT*)C_val);
    return cudaGetLastError();
}

template <class VT>
static cudaError_t num_light_V(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, int64_t rb,
                               const int64_t* C_rp, int32_t* C_col, void* C_val, cudaStream_t s) {
    switch (b) {
        case 0: return num_light_T<1, 32, 256, VT>(A, B, list, cnt, rb, C_rp, C_col, C_val, s);
        case 1: return num_light_T<2, 32, 256, VT>(A, B, list, cnt, rb, C_rp, C_col, C_val, s);
        case 2: return num_light_T<4, 32, 256, VT>(A, B, list, cnt, rb, C_rp, C_col, C_val, s);
        case 3: return num_light_T<8, 32, 256, VT>(A, B, list, cnt, rb, C_rp, C_col, C_val, s);
        case 4: return num_light_T<16, 32, 256, VT>(A, B, list, cnt, rb, C_rp, C_col, C_val, s);
        case 5: return num_light_T<32, 32, 256, VT>(A, B, list, cnt, rb, C_rp, C_col, C_val, s);
        case 6: return num_light_T<64, 32, 256, VT>(A, B, list, cnt, rb, C_rp, C_col, C_val, s);
        case 7: return num_light_T<128, 32, 256, VT>(A, B, list, cnt, rb, C_rp, C_col, C_val, s);
        case 8: return num_light_T<256, 32, 256, VT>(A, B, list, cnt, rb, C_rp, C_col, C_val, s);
        case 9: return num_light_T<512, 64, 64, VT>(A, B, list, cnt, rb, C_rp, C_col, C_val, s);
        case 10: return num_light_T<1024, 128, 128, VT>(A, B, list, cnt, rb, C_rp, C_col, C_val, s);
        case 11: return num_light_T<2048, 256, 256, VT>(A, B, list, cnt, rb, C_rp, C_col, C_val, s);
        case 12: return num_light_T<4096, 512, 512, VT>(A, B, list, cnt, rb, C_rp, C_col, C_val, s);
        default: return cudaErrorInvalidValue;
    }
}

cudaError_t launch_num_light(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, int64_t rb,
                             const int64_t* C_rp, int32_t* C_col, void* C_val, cudaStream_t s) {
    if (cnt <= 0) return cudaSuccess;
    return A.dt == 0 ? num_light_V<double>(b, A, B, list, cnt, rb, C_rp, C_col, C_val, s)
                     : num_light_V<float>(b, A, B, list, cnt, rb, C_rp, C_col, C_val, s);
}

template <class VT>
__global__ void __launch_bounds__(HEAVY_THREADS, 1) k_num_heavy(Mat A, Mat B, const RangeRec* __restrict__ ranges,
                                                                 int64_t nslots, int64_t rb,
                                                                 const int32_t* __restrict__ long_id,
                                                                 const uint32_t* __restrict__ tp, int T,
                                                                 const int64_t* __restrict__ C_rp,
                                                                 int32_t* __restrict__ C_col, VT* __restrict__ C_val,
                                                                 unsigned long long* counter) {
    extern __shared__ double smem_d[];
    double* vals = smem_d;
    int32_t* keys = reinterpret_cast<int32_t*>(vals + PH);
    __shared__ int ws[HEAVY_THREADS / 32];
    __shared__ long long s_j;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nwarps = HEAVY_THREADS / 32;
    const int64_t p = B.ncols;
    for (int s = threadIdx.x; s < PH; s += HEAVY_THREADS) { keys[s] = EMPTY_KEY; vals[s] = 0.0; }
    while (true) {
        __syncthreads();
        if (threadIdx.x == 0) s_j = (long long)atomicAdd(counter, 1ull);
        __syncthreads();
        const int64_t j = s_j;
        if (j >= nslots) break;
        const RangeRec r = ranges[j];
        if (r.row < 0 || r.cnt == 0) continue;
        const int64_t row = rb + r.row;
        const int64_t lo = (int64_t)r.t0 * TW;
        const int64_t hi = min(p, (int64_t)r.t1 * TW);
        const int64_t span = hi - lo;
        const bool ident = span <= PH;
        const uint64_t mult = ident ? 0 : (((uint64_t)HH << 32) / (uint64_t)span);
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        for (int64_t pa = s0 + wid; pa < s1; pa += nwarps) {
            const int k = __ldg(A.col + pa);
            const double a = ldv<VT>(A.val, pa);
            const int64_t q0 = __ldg(B.rp + k), q1 = __ldg(B.rp + k + 1);
            const int64_t len = q1 - q0;
            if (len <= LONG_ROW) {
                if (lane < len) {
                    int32_t c = __ldg(B.col + q0 + lane);
                    if (c >= lo && c < hi)
                        acc_insert(keys, vals, c, a * ldv<VT>(B.val, q0 + lane), (uint32_t)(c - lo), ident, mult);
                }
            } else {
                const uint32_t* tr = tp + (int64_t)__ldg(long_id + k) * (T + 1);
                const int64_t qs = q0 + __ldg(tr + r.t0), qe = q0 + __ldg(tr + r.t1);
                for (int64_t q = qs + lane; q < qe; q += 32) {
                    int32_t c = __ldg(B.col + q);
                    acc_insert(keys, vals, c, a * ldv<VT>(B.val, q), (uint32_t)(c - lo), ident, mult);
                }
            }
        }
        __syncthreads();
        emit_sorted<HEAVY_THREADS, VT>(keys, vals, ident ? (int)span : PH, ident, C_rp[r.row] + r.off, C_col, C_val,
                                       ws);
    }
}

cudaError_t launch_num_heavy(const Mat& A, const Mat& B, const RangeRec* ranges, int64_t nslots, int64_t rb,
                             const int32_t* long_id, const uint32_t* tp, int T, const int64_t* C_rp, int32_t* C_col,
                             void* C_val, unsigned long long* d_counter, cudaStream_t s) {
    if (nslots <= 0) return cudaSuccess;
    const int smem = PH * (8 + 4);
    cudaError_t e = cudaMemsetAsync(d_counter, 0, sizeof(unsigned long long), s);
    if (e != cudaSuccess) return e;
    int grid = (int)(nslots < 148 ? nslots : 148);
    if (A.dt == 0) {
        e = cudaFuncSetAttribute(k_num_heavy<double>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
        k_num_heavy<double><<<grid, HEAVY_THREADS, smem, s>>>(A, B, ranges, nslots, rb, long_id, tp, T, C_rp, C_col,
                                                               (double*)C_val, d_counter);
    } else {
        e = cudaFuncSetAttribute(k_num_heavy<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
        k_num_heavy<float><<<grid, HEAVY_THREADS, smem, s>>>(A, B, ranges, nslots, rb, long_id, tp, T, C_rp, C_col,
                                                              (float*)C_val, d_counter);
    }
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// a3 Identify: cost histogram over the (sampled) rows and the smallest argmin over t
// ------------------------------------------------------------------------------------------------
__device__ __forceinline__ long long ceil_log2_max2(long long u) {
    long long x = u < 2 ? 2 : u;
    return 64 - __clzll((unsigned long long)(x - 1));
}
__device__ __forceinline__ long long costL(const CostModelD& cm, long long w, long long a, long long u) {
    (void)a;
    return cm.kL + cm.lL * w + cm.sL * u * ceil_log2_max2(u) + cm.rL * u;
}
__device__ __forceinline__ long long costH(const CostModelD& cm, long long w, long long a, long long u) {
    long long R = cm.capu == 0 ? cm.tiles_fixed : ((u + cm.capu - 1) / cm.capu > 1 ? (u + cm.capu - 1) / cm.capu : 1);
    return cm.kH + cm.lH * w + cm.tH * a * R + cm.mH * u;
}

__global__ void k_cost_hist(CostModelD cm, const int64_t* __restrict__ w, const int64_t* __restrict__ a,
                            const int64_t* __restrict__ u, int64_t nr, unsigned long long* hd, unsigned long long* hc,
                            unsigned long long* hw, unsigned long long* sums) {
    long long base = 0, W = 0, ne = 0;
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nr; j += (int64_t)gridDim.x * blockDim.x) {
        long long wj = w[j];
        if (wj == 0) continue;
        long long cH = costH(cm, wj, a[j], u[j]);
        base += cH;
        W += wj;
        ne += 1;
        if (wj <= cm.cap_L) {
            long long cL = costL(cm, wj, a[j], u[j]);
            atomicAdd(&hd[wj], (unsigned long long)(cL - cH));
            atomicAdd(&hc[wj], 1ull);
            atomicAdd(&hw[wj], (unsigned long long)wj);
        }
    }
    base = warp_sum(base); W = warp_sum(W); ne = warp_sum(ne);
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(&sums[0], (unsigned long long)base);
        atomicAdd(&sums[1], (unsigned long long)W);
        atomicAdd(&sums[2], (unsigned long long)ne);
    }
}

cudaError_t launch_cost_hist(const CostModelD& cm, const int64_t* w, const int64_t* a, const int64_t* u, int64_t nr,
                             long long* hd, long long* hc, long long* hw, long long* sums, cudaStream_t s) {
    cudaError_t e;
    size_t hb = sizeof(long long) * (size_t)(cm.cap_L + 1);
    if ((e = cudaMemsetAsync(hd, 0, hb, s)) != cudaSuccess) return e;
    if ((e = cudaMemsetAsync(hc, 0, hb, s)) != cudaSuccess) return e;
    if ((e = cudaMemsetAsync(hw, 0, hb, s)) != cudaSuccess) return e;
    if ((e = cudaMemsetAsync(sums, 0, 4 * sizeof(long long), s)) != cudaSuccess) return e;
    if (nr <= 0) return cudaSuccess;
    k_cost_hist<<<grid_for(nr, 1024, 148 * 8), 256, 0, s>>>(cm, w, a, u, nr, (unsigned long long*)hd,
                                                            (unsigned long long*)hc, (unsigned long long*)hw,
                                                            (unsigned long long*)sums);
    return cudaGetLastError();
}

__global__ void __launch_bounds__(1024) k_argmin(CostModelD cm, const long long* __restrict__ hd,
                                                 const long long* __restrict__ hc, const long long* __restrict__ hw,
                                                 const long long* __restrict__ sums, ThrResult* out) {
    __shared__ long long ws[32];
    __shared__ long long bJ[32], bT[32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const long long n = cm.cap_L + 1;
    const long long per = (n + 1023) / 1024;
    const long long a0 = threadIdx.x * per, a1 = min(n, a0 + per);
    long long loc = 0;
    for (long long t = a0; t < a1; ++t) loc += hd[t];
    long long inc = warp_incl_scan(loc);
    if (lane == 31) ws[wid] = inc;
    __syncthreads();
    if (wid == 0) { long long x = ws[lane]; long long xi = warp_incl_scan(x); ws[lane] = xi - x; }
    __syncthreads();
    long long pre = ws[wid] + inc - loc;  // sum of hd over t < a0
    const long long base = sums[0];
    long long bestJ = LLONG_MAX, bestT = LLONG_MAX;
    for (long long t = a0; t < a1; ++t) {
        pre += hd[t];
        if (t == 0 || hc[t] > 0) {
            long long J = base + pre;
            if (J < bestJ) { bestJ = J; bestT = t; }
        }
    }
    // reduce (min J, then min t)
    for (int o = 16; o; o >>= 1) {
        long long oj = __shfl_xor_sync(0xffffffffu, bestJ, o), ot = __shfl_xor_sync(0xffffffffu, bestT, o);
        if (oj < bestJ || (oj == bestJ && ot < bestT)) { bestJ = oj; bestT = ot; }
    }
    if (lane == 0) { bJ[wid] = bestJ; bT[wid] = bestT; }
    __syncthreads();
    if (wid == 0) {
        bestJ = bJ[lane]; bestT = bT[lane];
        for (int o = 16; o; o >>= 1) {
            long long oj = __shfl_xor_sync(0xffffffffu, bestJ, o), ot = __shfl_xor_sync(0xffffffffu, bestT, o);
            if (oj < bestJ || (oj == bestJ && ot < bestT)) { bestJ = oj; bestT = ot; }
        }
        if (lane == 0) { bJ[0] = bestJ; bT[0] = bestT; }
    }
    __syncthreads();
    const long long thr = bT[0];
    long long wl = 0;
    for (long long t = threadIdx.x; t <= thr && t < n; t += 1024) wl += hw[t];
    wl = warp_sum(wl);
    if (lane == 0) ws[wid] = wl;
    __syncthreads();
    if (threadIdx.x == 0) {
        long long s = 0;
        for (int q = 0; q < 32; ++q) s += ws[q];
        out->thr = thr; out->Jmin = bJ[0]; out->base = base; out->W_L = s; out->W_all = sums[1];
        out->nonempty = sums[2];
    }
}

cudaError_t launch_argmin(const CostModelD& cm, const long long* hd, const long long* hc, const long long* hw,
                          const long long* sums, ThrResult* out, cudaStream_t s) {
    k_argmin<<<1, 1024, 0, s>>>(cm, hd, hc, hw, sums, out);
    return cudaGetLastError();
}

__global__ void k_cost_curve(CostModelD cm, const int64_t* __restrict__ w, const int64_t* __restrict__ a,
                             const int64_t* __restrict__ u, int64_t nr, const int64_t* __restrict__ ts, int nt,
                             unsigned long long* J) {
    for (int q = 0; q < nt; ++q) {
        const long long t = ts[q];
        long long acc = 0;
        for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nr; j += (int64_t)gridDim.x * blockDim.x) {
            long long wj = w[j];
            if (wj == 0) continue;
            acc += wj <= t ? costL(cm, wj, a[j], u[j]) : costH(cm, wj, a[j], u[j]);
        }
        acc = warp_sum(acc);
        if ((threadIdx.x & 31) == 0) atomicAdd(&J[q], (unsigned long long)acc);
    }
}

cudaError_t launch_cost_curve(const CostModelD& cm, const int64_t* w, const int64_t* a, const int64_t* u, int64_t nr,
                              const int64_t* t, int nt, long long* J, cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(J, 0, sizeof(long long) * nt, s);
    if (e != cudaSuccess || nr <= 0 || nt <= 0) return e;
    k_cost_curve<<<grid_for(nr, 2048, 148 * 4), 256, 0, s>>>(cm, w, a, u, nr, t, nt, (unsigned long long*)J);
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// a4: closest-prefix cuts (one thread; G is small)
// ------------------------------------------------------------------------------------------------
__device__ int64_t lb_i64(const int64_t* P, int64_t lo, int64_t hi, long long x) {  // first j in [lo,hi) with P[j] >= x
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if (P[mid] < x) lo = mid + 1; else hi = mid;
    }
    return lo;
}

__global__ void k_cuts(const int64_t* __restrict__ P, int64_t n, int G, int64_t* __restrict__ cuts) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    const long long W = P[n];
    cuts[0] = 0;
    int64_t prev = 0;
    for (int g = 1; g < G; ++g) {
        long long target = (long long)(((__int128)W * g) / G);
        int64_t j2 = lb_i64(P, 0, n + 1, target);  // smallest j with P[j] >= target
        int64_t best = j2;
        if (j2 > n || P[j2] != target) {
            if (j2 > 0) {
                int64_t j1 = lb_i64(P, 0, n + 1, P[j2 - 1]);  // first index of the plateau below target
                long long d1 = target - P[j1];
                long long d2 = j2 <= n ? P[j2] - target : LLONG_MAX;
                best = d1 <= d2 ? j1 : j2;
            }
        }
        if (best > n) best = n;
        if (best < prev) best = prev;
        cuts[g] = best;
        prev = best;
    }
    cuts[G] = n;
}

cudaError_t launch_cuts(const int64_t* P, int64_t n, int G, int64_t* cuts, cudaStream_t s) {
    k_cuts<<<1, 32, 0, s>>>(P, n, G, cuts);
    return cudaGetLastError();
}

__global__ void k_gather_rows(const int64_t* __restrict__ src, const int64_t* __restrict__ rows, int64_t nr,
                              int64_t* __restrict__ dst) {
    int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (j < nr) dst[j] = src[rows[j]];
}

cudaError_t launch_gather_rows(const int64_t* src, const int64_t* rows, int64_t nr, int64_t* dst, cudaStream_t s) {
    if (nr <= 0) return cudaSuccess;
    k_gather_rows<<<(unsigned)((nr + 255) / 256), 256, 0, s>>>(src, rows, nr, dst);
    return cudaGetLastError();
}

__global__ void k_add_offset(int64_t* x, int64_t n, int64_t off) {
    int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (j < n) x[j] += off;
}

cudaError_t launch_add_offset(int64_t* x, int64_t n, int64_t off, cudaStream_t s) {
    if (n <= 0 || off == 0) return cudaSuccess;
    k_add_offset<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(x, n, off);
    return cudaGetLastError();
}

}  // namespace sg
