// sg_kernels.cu — the sm_100a kernels of the hot path.
//
//   a1 k_row_work        w_i = sum_{k in A_i} nnz(B_k)
//   a2 k_scan_*          exclusive prefix (P of w; C.row_ptr of u)          PAPER L217 (V_L)
//   a3 k_samp_*          Bernoulli row sample S by SplitMix64
//      k_cost_hist/k_argmin  J(t;S) histogram + smallest argmin
//   a4 k_cuts            closest-prefix row cuts
//   a5 k_bin_*           EMPTY / LIGHT(2^b bins) / HEAVY by thr
//   a6-a8 light path: sg_light.cu; heavy path: sg_heavy.cu
#include "sg_device.cuh"

namespace sg {

// ------------------------------------------------------------------------------------------------
// counter hash of the row sampler (R4; the oracle carries its own copy)
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
    SG_LAUNCH("k_row_work", s, k_row_work<<<grid_for(re - rb, 8, 148 * 32), 256, 0, s>>>(A, B, rb, re, w));
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
    SG_LAUNCH("k_row_work_list", s, k_row_work_list<<<grid_for(nr, 8, 148 * 32), 256, 0, s>>>(A, B, rows, nr, w, a));
    return cudaGetLastError();
}

// max of x[0..n) (non-negative values) into *out (zeroed by the caller)
__global__ void k_max_i64(const int64_t* __restrict__ x, int64_t n, unsigned long long* out) {
    unsigned long long m = 0;
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
        const unsigned long long v = (unsigned long long)x[j];
        m = v > m ? v : m;
    }
    #pragma unroll
    for (int o = 16; o; o >>= 1) { const unsigned long long y = __shfl_xor_sync(FULL, m, o); m = y > m ? y : m; }
    if ((threadIdx.x & 31) == 0 && m) atomicMax(out, m);
}

cudaError_t launch_max_i64(const int64_t* x, int64_t n, unsigned long long* out, cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(out, 0, sizeof(unsigned long long), s);
    if (e != cudaSuccess || n <= 0) return e;
    SG_LAUNCH("k_max_i64", s, k_max_i64<<<grid_for(n, 1024, 148 * 4), 256, 0, s>>>(x, n, out));
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
    SG_LAUNCH("k_scan_tile", s, k_scan_tile<<<(unsigned)nb, SCAN_T, 0, s>>>(in, out, n, bsum));
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
    SG_LAUNCH("k_scan_add", s, k_scan_add<<<(unsigned)((n + 1 + 255) / 256), 256, 0, s>>>(out, n, bscan, nb));
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
    SG_LAUNCH("k_samp_count", s, k_samp_count<<<(unsigned)nb, SCAN_T, 0, s>>>(rb, re, seed, Tf, all, bsum));
    cudaError_t e = scan_exclusive(bsum, bscan, nb, bscan + nb + 1, s);
    if (e != cudaSuccess) return e;
    SG_LAUNCH("k_samp_write", s, k_samp_write<<<(unsigned)nb, SCAN_T, 0, s>>>(rb, re, seed, Tf, all, bscan, out_rows, nb, d_count));
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
    SG_LAUNCH("k_bin_count", s, k_bin_count<<<grid_for(nr, 1024, 148 * 8), 256, 0, s>>>(w, nr, thr, (unsigned long long*)d_cnt, cls));
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
    SG_LAUNCH("k_bin_scatter", s, k_bin_scatter<<<grid_for(nr, 1024, 148 * 8), 256, 0, s>>>(w, nr, thr, (unsigned long long*)d_cursor, lists));
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
    long long R = cm.tiles_fixed;  // R(u) = tiles_fixed (capu == 0) or max(1, tiles_fixed, ceil(u / capu))
    if (cm.capu != 0) {
        const long long q = (u + cm.capu - 1) / cm.capu, lo = cm.tiles_fixed > 1 ? cm.tiles_fixed : 1;
        R = q > lo ? q : lo;
    }
    return cm.kH + cm.lH * w + cm.tH * a * R + cm.mH * u;
}

// Overflow guard (include/sg.h SG_ERR_OVERFLOW): the same per-row costs evaluated in fp64. Every
// coefficient is non-negative (check_model), so sum over rows of c_L + c_H bounds |J|, every prefix
// of the histogram and every cut target; the host rejects the model when that bound reaches 2^62.
__device__ __forceinline__ double cost_mag(const CostModelD& cm, double w, double a, double u) {
    const double lg = (double)ceil_log2_max2((long long)u);
    const double R = cm.capu == 0 ? (double)cm.tiles_fixed
                                  : fmax(fmax(1.0, (double)cm.tiles_fixed), ceil(u / (double)cm.capu));
    const double cl = (double)cm.kL + (double)cm.lL * w + (double)cm.sL * u * lg + (double)cm.rL * u;
    const double ch = (double)cm.kH + (double)cm.lH * w + (double)cm.tH * a * R + (double)cm.mH * u;
    return cl + ch;
}

__global__ void k_cost_mag(CostModelD cm, const int64_t* __restrict__ w, const int64_t* __restrict__ a,
                           const int64_t* __restrict__ u, int64_t nr, double* out) {
    double m = 0.0;
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nr; j += (int64_t)gridDim.x * blockDim.x) {
        const long long wj = w[j];
        if (wj > 0) m += cost_mag(cm, (double)wj, (double)a[j], (double)u[j]);
    }
    m = warp_sum(m);
    if ((threadIdx.x & 31) == 0 && m != 0.0) atomicAdd(out, m);
}

cudaError_t launch_cost_mag(const CostModelD& cm, const int64_t* w, const int64_t* a, const int64_t* u, int64_t nr,
                            double* out, cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(out, 0, sizeof(double), s);
    if (e != cudaSuccess || nr <= 0) return e;
    SG_LAUNCH("k_cost_mag", s, k_cost_mag<<<grid_for(nr, 1024, 148 * 8), 256, 0, s>>>(cm, w, a, u, nr, out));
    return cudaGetLastError();
}

// ---- NEXT #2: modeled per-row cost for the cost-weighted split (R19) -----------------
// c_i = 0 (w = 0), c_L(w, a, uh) (w <= thr), c_H(w, a, uh) (w > thr); uh = min(w, ceil(w U_c / W_c)).
__global__ void k_row_cost(CostModelD cm, long long thr, long long UL, long long WL, long long UH, long long WH,
                           const int64_t* __restrict__ arp, const int64_t* __restrict__ w, int64_t n,
                           int64_t* __restrict__ cost, double* __restrict__ mag) {
    double m = 0.0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const long long wi = w[i];
        if (wi == 0) { cost[i] = 0; continue; }
        const long long ai = arp[i + 1] - arp[i];
        const bool light = wi <= thr;
        const long long U = light ? UL : UH, Wc = light ? WL : WH;
        long long uh = wi;
        if (Wc > 0) {
            const __int128 q = ((__int128)wi * U + Wc - 1) / Wc;
            if (q < (__int128)uh) uh = (long long)q;
        }
        cost[i] = light ? costL(cm, wi, ai, uh) : costH(cm, wi, ai, uh);
        m += cost_mag(cm, (double)wi, (double)ai, (double)uh);
    }
    m = warp_sum(m);
    if ((threadIdx.x & 31) == 0 && m != 0.0) atomicAdd(mag, m);
}

cudaError_t launch_row_cost(const CostModelD& cm, int64_t thr, const int64_t* comp, const int64_t* arp,
                            const int64_t* w, int64_t n, int64_t* cost, double* mag, cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(mag, 0, sizeof(double), s);
    if (e != cudaSuccess || n <= 0) return e;
    SG_LAUNCH("k_row_cost", s, k_row_cost<<<grid_for(n, 256, 148 * 8), 256, 0, s>>>(cm, thr, comp[0], comp[1], comp[2],
                                                                                       comp[3], arp, w, n, cost, mag));
    return cudaGetLastError();
}

// per-class sums of u over a row list at a known threshold: out[0] = sum u (0 < w <= thr),
// out[1] = sum u (w > thr)
__global__ void k_class_usum(const int64_t* __restrict__ w, const int64_t* __restrict__ u, int64_t nr, long long thr,
                             unsigned long long* out) {
    unsigned long long sl = 0, sh = 0;
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nr; j += (int64_t)gridDim.x * blockDim.x) {
        const long long wj = w[j];
        if (wj == 0) continue;
        if (wj <= thr) sl += (unsigned long long)u[j]; else sh += (unsigned long long)u[j];
    }
    sl = warp_sum(sl);
    sh = warp_sum(sh);
    if ((threadIdx.x & 31) == 0) {
        if (sl) atomicAdd(&out[0], sl);
        if (sh) atomicAdd(&out[1], sh);
    }
}

// the same with the threshold read from device memory (k_argmin's result; no host round trip)
__global__ void k_class_usum_dev(const int64_t* __restrict__ w, const int64_t* __restrict__ u, int64_t nr,
                                 const long long* __restrict__ thr_dev, unsigned long long* out) {
    const long long thr = *thr_dev;
    unsigned long long sl = 0, sh = 0;
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nr; j += (int64_t)gridDim.x * blockDim.x) {
        const long long wj = w[j];
        if (wj == 0) continue;
        if (wj <= thr) sl += (unsigned long long)u[j]; else sh += (unsigned long long)u[j];
    }
    sl = warp_sum(sl);
    sh = warp_sum(sh);
    if ((threadIdx.x & 31) == 0) {
        if (sl) atomicAdd(&out[0], sl);
        if (sh) atomicAdd(&out[1], sh);
    }
}

cudaError_t launch_class_usum_dev(const int64_t* w, const int64_t* u, int64_t nr, const long long* thr_dev,
                                  unsigned long long* out, cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(out, 0, 2 * sizeof(unsigned long long), s);
    if (e != cudaSuccess || nr <= 0) return e;
    SG_LAUNCH("k_class_usum", s, k_class_usum_dev<<<grid_for(nr, 256, 148 * 4), 256, 0, s>>>(w, u, nr, thr_dev, out));
    return cudaGetLastError();
}

cudaError_t launch_class_usum(const int64_t* w, const int64_t* u, int64_t nr, int64_t thr, unsigned long long* out,
                              cudaStream_t s) {
    cudaError_t e = cudaMemsetAsync(out, 0, 2 * sizeof(unsigned long long), s);
    if (e != cudaSuccess || nr <= 0) return e;
    SG_LAUNCH("k_class_usum", s, k_class_usum<<<grid_for(nr, 256, 148 * 4), 256, 0, s>>>(w, u, nr, thr, out));
    return cudaGetLastError();
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
    SG_LAUNCH("k_cost_hist", s, k_cost_hist<<<grid_for(nr, 1024, 148 * 8), 256, 0, s>>>(cm, w, a, u, nr, (unsigned long long*)hd,
                                                            (unsigned long long*)hc, (unsigned long long*)hw,
                                                            (unsigned long long*)sums));
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
    SG_LAUNCH("k_argmin", s, k_argmin<<<1, 1024, 0, s>>>(cm, hd, hc, hw, sums, out));
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
    SG_LAUNCH("k_cost_curve", s, k_cost_curve<<<grid_for(nr, 2048, 148 * 4), 256, 0, s>>>(cm, w, a, u, nr, t, nt, (unsigned long long*)J));
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
    SG_LAUNCH("k_cuts", s, k_cuts<<<1, 32, 0, s>>>(P, n, G, cuts));
    return cudaGetLastError();
}

__global__ void k_gather_rows(const int64_t* __restrict__ src, const int64_t* __restrict__ rows, int64_t nr,
                              int64_t* __restrict__ dst) {
    int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (j < nr) dst[j] = src[rows[j]];
}

cudaError_t launch_gather_rows(const int64_t* src, const int64_t* rows, int64_t nr, int64_t* dst, cudaStream_t s) {
    if (nr <= 0) return cudaSuccess;
    SG_LAUNCH("k_gather_rows", s, k_gather_rows<<<(unsigned)((nr + 255) / 256), 256, 0, s>>>(src, rows, nr, dst));
    return cudaGetLastError();
}

// count of row ids outside [0, n) (argument check of sg_threshold_on_rows)
__global__ void k_check_rows(const int64_t* __restrict__ rows, int64_t nr, int64_t n, unsigned long long* bad) {
    int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (j < nr && (rows[j] < 0 || rows[j] >= n)) atomicAdd(bad, 1ull);
}

cudaError_t launch_check_rows(const int64_t* rows, int64_t nr, int64_t n, unsigned long long* bad, cudaStream_t s) {
    if (nr <= 0) return cudaSuccess;
    SG_LAUNCH("k_check_rows", s, k_check_rows<<<(unsigned)((nr + 255) / 256), 256, 0, s>>>(rows, nr, n, bad));
    return cudaGetLastError();
}

__global__ void k_add_offset(int64_t* x, int64_t n, int64_t off) {
    int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (j < n) x[j] += off;
}

cudaError_t launch_add_offset(int64_t* x, int64_t n, int64_t off, cudaStream_t s) {
    if (n <= 0 || off == 0) return cudaSuccess;
    SG_LAUNCH("k_add_offset", s, k_add_offset<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(x, n, off));
    return cudaGetLastError();
}

}  // namespace sg
