// sg_heavy.cu — the HEAVY path (w_i > thr, "more than t"): one CTA per heavy row
// (symbolic: 256 threads, six CTAs per SM, 2^18-column bitmap windows; numeric: 512 threads, two CTAs
// per SM — several CTAs per SM so that one CTA's barriers and serial phases overlap the others'
// products), rows taken heaviest-first from a dynamic counter.
//
// Symbolic: the row's products set bits of a shared-memory bitmap over a WIN-column window (a window's
// segment of each B row from the tile pointers);
// per-8192-column-tile popcounts give u_i and a plan of column RANGES, each holding at most
// RCAP = 8192 output entries and spanning at most RW_TILES tiles (the numeric accumulator).
//
// Numeric, per range [lo, hi): pass 1 rebuilds the range's bitmap, a block scan turns word
// popcounts into a rank prefix, pass 2 accumulates every product into a COMPACT fp64 array at
// rank(c) = prefix[word] + popc(word & below) — a rank-indexed dense accumulator: no hashing, no
// probing, and the output is sorted by construction: C.col[rank] is written by the product that
// finds the accumulator at 0.0 (the first arrival), C.val by a coalesced copy of the array.
// Products are flattened over the whole block (one k per thread, block scan of segment lengths,
// per-product binary search), so rows with few k (median 9 on R-MAT) still use every warp.
// Per-k cursors advance monotonically across ranges; B rows longer than LONG_ROW locate their
// segment through the tile-pointer table tp (one load), short rows by a bounded scan.
#include "sg_device.cuh"
#include <cstdio>

namespace sg {

#ifndef SG_INREG
#define SG_INREG 1
#endif
constexpr int KC = NUM_T;             // numeric k entries per chunk: one per thread
constexpr int RW_WORDS = RW_TILES * TW / 32;   // = 256 words per warp in the rank prefix
static_assert(TW <= RCAP, "a single full tile must fit the numeric accumulator");

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
    SG_LAUNCH("k_long_rows", s, (k_long_rows<<<grid_for(B.nrows, 256, 148 * 8), 256, 0, s>>>(B, long_id, (unsigned long long*)d_nlong)));
    return cudaGetLastError();
}

__global__ void k_build_tp(Mat B, const int32_t* __restrict__ long_id, int T, uint32_t* __restrict__ tp) {
    const int lane = threadIdx.x & 31;
    int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t k = warp; k < B.nrows; k += nw) {
        int id = long_id[k];
        if (id < 0) continue;
        const int64_t q0 = B.rp[k], q1 = B.rp[k + 1];
        const int len = (int)(q1 - q0);
        uint32_t* row = tp + (int64_t)id * (T + 1);
        // entry q with tile t_q starts every tile in (t_{q-1}, t_q]: one pass over the entries
        int tprev_chunk = -1;
        for (int b0 = 0; b0 < len; b0 += 32) {
            const int q = b0 + lane;
            const int tq = q < len ? (int)(__ldg(B.col + q0 + q) / TW) : T + 1;
            int tp_prev = __shfl_up_sync(FULL, tq, 1);
            if (lane == 0) tp_prev = tprev_chunk;
            if (q < len)
                for (int t = tp_prev + 1; t <= tq; ++t) row[t] = (uint32_t)q;
            tprev_chunk = __shfl_sync(FULL, tq, 31);
        }
        const int tlast = len > 0 ? (int)(__ldg(B.col + q1 - 1) / TW) : -1;
        for (int t = tlast + 1 + lane; t <= T; t += 32) row[t] = (uint32_t)len;
    }
}

cudaError_t launch_build_tp(const Mat& B, const int32_t* long_id, int T, uint32_t* tp, cudaStream_t s) {
    if (B.nrows <= 0) return cudaSuccess;
    SG_LAUNCH("k_build_tp", s, (k_build_tp<<<grid_for(B.nrows, 8, 148 * 16), 256, 0, s>>>(B, long_id, T, tp)));
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// heavy rows heaviest-first: counting sort of the heavy list by descending ceil(log2 w)
// ------------------------------------------------------------------------------------------------
__global__ void k_heavy_hist(const int32_t* __restrict__ heavy, int64_t nh, const int64_t* __restrict__ w,
                             unsigned int* hist) {
    __shared__ unsigned int sh[64];
    if (threadIdx.x < 64) sh[threadIdx.x] = 0;
    __syncthreads();
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nh; j += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(&sh[63 - (64 - __clzll((unsigned long long)w[heavy[j]]))], 1u);  // descending log2
    __syncthreads();
    if (threadIdx.x < 64 && sh[threadIdx.x]) atomicAdd(&hist[threadIdx.x], sh[threadIdx.x]);
}

__global__ void k_heavy_scatter(const int32_t* __restrict__ heavy, int64_t nh, const int64_t* __restrict__ w,
                                unsigned int* hist /*64 counts -> cursors*/, int32_t* __restrict__ out) {
    __shared__ unsigned int base[64];
    if (threadIdx.x == 0) {
        // every block recomputes the exclusive offsets from the counts in hist[0..64)
        unsigned int a = 0;
        for (int b = 0; b < 64; ++b) { base[b] = a; a += hist[b]; }
    }
    __syncthreads();
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nh; j += (int64_t)gridDim.x * blockDim.x) {
        int b = 63 - (64 - __clzll((unsigned long long)w[heavy[j]]));
        unsigned int pos = atomicAdd(&hist[64 + b], 1u);
        out[base[b] + pos] = heavy[j];
    }
}

cudaError_t launch_heavy_order(const int32_t* heavy, int64_t nh, const int64_t* w, unsigned int* hist128,
                               int32_t* out, cudaStream_t s) {
    if (nh <= 0) return cudaSuccess;
    cudaError_t e = cudaMemsetAsync(hist128, 0, 128 * sizeof(unsigned int), s);
    if (e != cudaSuccess) return e;
    int g = grid_for(nh, 1024, 148 * 4);
    SG_LAUNCH("k_heavy_hist", s, (k_heavy_hist<<<g, 256, 0, s>>>(heavy, nh, w, hist128)));
    SG_LAUNCH("k_heavy_scatter", s, (k_heavy_scatter<<<g, 256, 0, s>>>(heavy, nh, w, hist128, out)));
    return cudaGetLastError();
}

// per heavy row: an upper bound on its range count
__global__ void k_range_bounds(const int32_t* __restrict__ heavy, int64_t nh, const int64_t* __restrict__ w,
                               int64_t p, int64_t dw_min_w, int64_t* __restrict__ bounds) {
    int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (j >= nh) return;
    int64_t wi = w[heavy[j]];
    if (wi >= dw_min_w) { bounds[j] = 0; return; }  // dense-window row (sg_dense.cu): no range plan
    int64_t mu = wi < p ? wi : p;
    int64_t T = (p + TW - 1) / TW;
    int64_t nwin = (p + WIN - 1) / WIN;
    // distinct keys per window <= u_win / RHALF + 1 + (tiles per window / RW_TILES); each big tile
    // (> RHALF entries, at most u / RHALF of them) adds at most two more range starts
    int64_t b = 3 * (mu / RHALF) + nwin * (1 + (WIN / TW) / RW_TILES) + 1;
    bounds[j] = b < T ? b : T;
}

cudaError_t launch_range_bounds(const int32_t* heavy, int64_t nh, const int64_t* w, int64_t p, int64_t dw_min_w,
                                int64_t* bounds, cudaStream_t s) {
    if (nh <= 0) return cudaSuccess;
    SG_LAUNCH("k_range_bounds", s, (k_range_bounds<<<(unsigned)((nh + 255) / 256), 256, 0, s>>>(heavy, nh, w, p, dw_min_w, bounds)));
    return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// a6 heavy symbolic
// ------------------------------------------------------------------------------------------------
template <int ST, int SOCC, int SWIN>
__global__ void __launch_bounds__(ST, SOCC) k_sym_heavy(Mat A, Mat B, const int32_t* __restrict__ list, int64_t j0,
                                                                 int64_t cnt, const int64_t* __restrict__ rowmap,
                                                                 int64_t rb, int64_t* __restrict__ u,
                                                                 const int64_t* __restrict__ range_off,
                                                                 RangeRec* __restrict__ ranges,
                                                                 int32_t* __restrict__ nranges, int64_t ndw,
                                                                 int32_t* __restrict__ dtc, const int32_t* __restrict__ long_id,
                                                                 const uint32_t* __restrict__ tp, int T,
                                                                 unsigned long long* counter) {
    extern __shared__ uint32_t bm[];  // SWIN/32 words
    __shared__ int64_t s_beg[ST];
    __shared__ int s_off[ST];
    __shared__ int tcnt[SWIN / TW];
    __shared__ int Ps[SWIN / TW];
    __shared__ unsigned char st[SWIN / TW];
    __shared__ long long wsll[33];
    __shared__ long long s_j;
    __shared__ int s_nr, s_u;
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5, nwarps = ST / 32;
    const int64_t p = B.ncols;
    const int64_t nwin = (p + SWIN - 1) / SWIN;
    while (true) {
        if (tid == 0) s_j = j0 + (long long)atomicAdd(counter, 1ull);
        __syncthreads();
        const int64_t j = s_j;
        __syncthreads();
        if (j >= cnt) break;
        const int64_t li = list[j];
        const int64_t row = rowmap ? rowmap[li] : rb + li;
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        int utot = 0, nr = 0;
        for (int64_t win = 0; win < nwin; ++win) {
            const int64_t wlo = win * SWIN, whi = min(p, wlo + SWIN);
            const int nwords = (int)((whi - wlo + 31) / 32);
            for (int q = tid; q < nwords; q += ST) bm[q] = 0u;
            for (int64_t c0 = s0; c0 < s1; c0 += ST) {
                const int64_t i = c0 + tid;
                int len = 0;
                int64_t beg = 0;
                if (i < s1) {
                    const int k = __ldg(A.col + i);
                    int64_t q0 = __ldg(B.rp + k), q1 = __ldg(B.rp + k + 1);
                    if (nwin > 1) {
                        if (tp && q1 - q0 > LONG_ROW) {  // the window's segment from the B tile pointers
                            const uint32_t* tr = tp + (int64_t)__ldg(long_id + k) * (T + 1);
                            const int64_t b0 = q0;
                            q0 = b0 + __ldg(tr + wlo / TW);
                            q1 = b0 + __ldg(tr + (whi == p ? T : (int)(whi / TW)));
                        } else if (tp) {  // short row: count its entries below the window bounds
                            int n0 = 0, n1 = 0;
                            #pragma unroll
                            for (int q = 0; q < LONG_ROW; ++q)
                                if (q0 + q < q1) {
                                    const int c = __ldg(B.col + q0 + q);
                                    n0 += c < wlo;
                                    n1 += c < whi;
                                }
                            q1 = q0 + n1;
                            q0 = q0 + n0;
                        } else {
                            q0 = lower_bound_col(B.col, q0, q1, wlo);
                            q1 = lower_bound_col(B.col, q0, q1, whi);
                        }
                    }
                    beg = q0;
                    len = (int)(q1 - q0);
                }
                int nk;
                const int tot = chunk_compact<ST, int64_t>(len, beg, 0.0, s_beg, s_off, nullptr, &nk, wsll);
                const uint32_t bb = opaque_u32(smem_addr(bm) - 4u * ((uint32_t)wlo >> 5));  // wlo: multiple of 32
                warp_slice<ST, false, double, int64_t>(s_beg, s_off, nullptr, nk, tot, B, [&](int32_t c, double) {
                    if (c >= 0) red_or_s(bb + 4u * ((uint32_t)c >> 5), 1u << (c & 31));
                });
                __syncthreads();
            }
            // per-tile popcounts
            const int nt = (int)((whi - wlo + TW - 1) / TW);
            for (int tt = wid; tt < nt; tt += nwarps) {
                const int a = tt * (TW / 32), b = min(nwords, a + TW / 32);
                int c = 0;
                for (int q = a + lane; q < b; q += 32) c += __popc(bm[q]);
                c = warp_sum(c);
                if (lane == 0) tcnt[tt] = c;
            }
            __syncthreads();
            // range plan (warp 0): key(t) = (ceil(P_t / RHALF) - 1, t / RW_TILES); a range is a run of
            // equal keys, and a BIG tile (more than RHALF entries) is a range of its own -> a range without
            // a big tile holds <= RHALF + cnt(first tile) <= 2 RHALF = RCAP entries, a big tile alone
            // <= TW <= RCAP; width <= RW_TILES tiles.
            if (wid == 0 && j < ndw) {  // dense-window row (sg_dense.cu): u and its tile counts, no range plan
                int c = 0;
                const int64_t Tall = (p + TW - 1) / TW;
                for (int t = lane; t < nt; t += 32) {
                    c += tcnt[t];
                    if (dtc) dtc[j * Tall + wlo / TW + t] = tcnt[t];
                }
                c = warp_sum(c);
                if (lane == 0) { s_nr = nr; s_u = utot + c; }
            } else if (wid == 0) {
                int c4[4], loc = 0;
                #pragma unroll
                for (int q = 0; q < 4; ++q) { const int t = 4 * lane + q; c4[q] = t < nt ? tcnt[t] : 0; loc += c4[q]; }
                int pre = warp_incl_scan(loc) - loc;
                int key[4];
                #pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int t = 4 * lane + q;
                    pre += c4[q];
                    key[q] = ((pre + RHALF - 1) / RHALF - 1) * (SWIN / TW / RW_TILES) + t / RW_TILES;
                    if (t < nt) Ps[t] = pre;
                }
                const int prevkey = __shfl_up_sync(FULL, key[3], 1);
                const bool prevbig = __shfl_up_sync(FULL, c4[3], 1) > RHALF;
                #pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int t = 4 * lane + q;
                    const int kp = q == 0 ? prevkey : key[q - 1];
                    const bool bigp = q == 0 ? prevbig : c4[q - 1] > RHALF;
                    if (t < nt) st[t] = (t == 0 || key[q] != kp || c4[q] > RHALF || bigp) ? 1 : 0;
                }
                __syncwarp();
                for (int t0 = 0; t0 < nt; t0 += 32) {
                    const int t = t0 + lane;
                    int e = t + 1, cntr = 0;
                    bool valid = false;
                    if (t < nt && st[t]) {
                        while (e < nt && !st[e]) ++e;
                        cntr = Ps[e - 1] - (t > 0 ? Ps[t - 1] : 0);
                        valid = cntr > 0;
                    }
                    const unsigned m = __ballot_sync(FULL, valid);
                    if (valid && ranges) {
                        RangeRec r;
                        r.row = (int32_t)li;
                        r.t0 = (int32_t)(wlo / TW) + t;
                        r.t1 = (int32_t)(wlo / TW) + e;
                        r.cnt = cntr;
                        r.off = utot + (t > 0 ? Ps[t - 1] : 0);
                        r.pad = 0;
                        ranges[range_off[j] + nr + __popc(m & lanemask_lt())] = r;
                    }
                    nr += __popc(m);
                }
                if (lane == 0) { s_nr = nr; s_u = utot + Ps[nt - 1]; }
            }
            __syncthreads();
            nr = s_nr;
            utot = s_u;
            __syncthreads();
        }
        if (tid == 0) {
            u[li] = utot;
            if (nranges) nranges[j] = nr;
        }
    }
}

template <int ST, int SOCC, int SWIN>
static cudaError_t sym_heavy_part(const Mat& A, const Mat& B, const int32_t* list, int64_t j0, int64_t cnt,
                                  const int64_t* rowmap, int64_t rb, int64_t* u, const int64_t* range_off,
                                  RangeRec* ranges, int32_t* nranges, int64_t ndw, int32_t* dtc, const int32_t* long_id,
                                  const uint32_t* tp, int T, unsigned long long* counter, cudaStream_t s) {
    if (cnt - j0 <= 0) return cudaSuccess;
    const int smem = (SWIN / 32) * 4;
    cudaError_t e = cudaFuncSetAttribute(k_sym_heavy<ST, SOCC, SWIN>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    if ((e = cudaMemsetAsync(counter, 0, sizeof(unsigned long long), s)) != cudaSuccess) return e;
    const int64_t n = cnt - j0;
    const int grid = (int)(n < 148 * SOCC ? n : 148 * SOCC);
    SG_LAUNCH("k_sym_heavy", s, (k_sym_heavy<ST, SOCC, SWIN><<<grid, ST, smem, s>>>(A, B, list, j0, cnt, rowmap, rb, u,
                                                                                     range_off, ranges, nranges, ndw, dtc,
                                                                                     long_id, tp, T, counter)));
    return cudaGetLastError();
}

// Heavy rows [0, nbig) of the heaviest-first list (the ones whose single-CTA time could be a tail)
// run on 1024-thread CTAs over 2^20-column windows; the rest on SYM_OCC smaller CTAs per SM over
// WIN-column windows (segments from the tile pointers), whose barriers overlap each other.
cudaError_t launch_sym_heavy(const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, const int64_t* rowmap,
                             int64_t rb, int64_t* u, const int64_t* range_off, RangeRec* ranges, int32_t* nranges,
                             int64_t ndw, int32_t* dtc, const int32_t* long_id, const uint32_t* tp, int T,
                             unsigned long long* counter, cudaStream_t s, int64_t nbig) {
    if (cnt <= 0) return cudaSuccess;
    if (nbig > cnt) nbig = cnt;
    cudaError_t e = sym_heavy_part<1024, 1, (1 << 20)>(A, B, list, 0, nbig, rowmap, rb, u, range_off, ranges, nranges, ndw,
                                                        dtc, long_id, tp, T, counter, s);
    if (e != cudaSuccess) return e;
    return sym_heavy_part<HEAVY_THREADS, SYM_OCC, WIN>(A, B, list, nbig, cnt, rowmap, rb, u, range_off, ranges, nranges,
                                                       ndw, dtc, long_id, tp, T, counter, s);
}

// ------------------------------------------------------------------------------------------------
// a7 + a8 heavy numeric: rank-indexed compact accumulator per range
// ------------------------------------------------------------------------------------------------
struct HeavySmem {
    uint32_t bm[RW_WORDS];       // 32 KB  range bitmap
    double vals[RCAP + 2];       // 64 KB compact accumulator: rank r at vals[r + sh], sh = C offset parity
    uint16_t pref[RW_WORDS];     // 16 KB  rank prefix per bitmap word
    int32_t s_beg[KC];           // packed chunk entries: segment begin (B position)
    int32_t s_off[KC];           //                       exclusive prefix of segment lengths
    double s_a[KC];              //                       a_ik
    int32_t c_cur[KC];           // single-chunk rows, per k: cursor (B position)
    int32_t c_end[KC];           //   end of the B row
    int32_t c_q0[KC];            //   start of the B row
    int32_t c_lid[KC];           //   long-row id or -1 (short row: <= LONG_ROW entries)
    double c_a[KC];              //   a_ik
    long long wsll[33];
    int ws[33];
};

// fp64 values leave shared memory by a bulk async copy (TMA engine, no LSU traffic)
__device__ __forceinline__ void bulk_s2g(void* gdst, const void* ssrc, uint32_t bytes) {
    const uint32_t sa = (uint32_t)__cvta_generic_to_shared(ssrc);
#if SG_STCS
    uint64_t pol;  // C values: evict-first in L2 (see st_out)
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(gdst), "r"(sa),
                 "r"(bytes), "l"(pol) : "memory");
#else
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gdst), "r"(sa), "r"(bytes) : "memory");
#endif
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

#if defined(SG_HV_EXP) && SG_HV_EXP == 8  // timing experiment: per-phase cycle counters (lane 0 of each warp)
__device__ unsigned long long g_hv_phase[10];
#define HV_MARK(k) do { if ((threadIdx.x & 31) == 0) { long long _t = clock64(); hph[k] += _t - hv_last; hv_last = _t; } } while (0)
#elif defined(SG_HV_EXP) && SG_HV_EXP == 9
#define HV_MARK(k) HV_MARK9_##k
#define HV_MARK9_0 do { } while (0)
#define HV_MARK9_6 do { } while (0)
#define HV_MARK9_1 do { if (tid == 0) hv_ts[1] = clock64(); } while (0)
#define HV_MARK9_2 do { if (tid == 0) hv_ts[2] = clock64(); } while (0)
#define HV_MARK9_3 do { if (tid == 0) hv_ts[3] = clock64(); } while (0)
#define HV_MARK9_4 do { if (tid == 0) hv_ts[4] = clock64(); } while (0)
#define HV_MARK9_5 do { if (tid == 0) hv_ts[5] = clock64(); } while (0)
#else
#define HV_MARK(k) do { } while (0)
#endif
#if defined(SG_HV_EXP) && SG_HV_EXP == 9  // timing experiment: per-range cycles (and per phase) binned by log2(products)
__device__ unsigned long long g_hv_rng[24][4];
__device__ unsigned long long g_hv_ph[24][5];
#endif

// seg_end that also serves long B rows when the plan has no tile pointers (table over its memory budget,
// SG_OPT_TP_MAX_BYTES): a binary search of the row's remaining entries
__device__ __forceinline__ int seg_end_any(const Mat& B, int cur, int e1, int q0, bool is_long, uint32_t tpv, int64_t hi) {
    if (!is_long && e1 - cur > LONG_ROW) return (int)lower_bound_col(B.col, cur, e1, hi);
    return seg_end(B, cur, e1, q0, is_long, tpv, hi);
}

template <class VT>
__global__ void __launch_bounds__(NUM_T, NUM_OCC) k_num_heavy(
    Mat A, Mat B, const int32_t* __restrict__ heavy, int64_t h0, int64_t nheavy, int64_t rb, const int64_t* __restrict__ range_off,
    const int32_t* __restrict__ nranges, const RangeRec* __restrict__ ranges, const int32_t* __restrict__ long_id,
    const uint32_t* __restrict__ tp, int T, const int64_t* __restrict__ C_rp, int32_t* __restrict__ C_col,
    VT* __restrict__ C_val, unsigned long long* counter, int4* __restrict__ gscr, int64_t amax, int amin) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    HeavySmem& S = *reinterpret_cast<HeavySmem*>(smem_raw);
    __shared__ long long s_j;
    const int tid = threadIdx.x;
    const int64_t p = B.ncols;
    int4* gs = gscr + (int64_t)blockIdx.x * amax;  // multi-chunk rows: per-k (cur, -, beg, len)
    for (int q = tid; q < RW_WORDS; q += NUM_T) S.bm[q] = 0u;
    for (int q = tid; q < RCAP + 2; q += NUM_T) S.vals[q] = 0.0;
    const uint32_t a_bm = smem_addr(S.bm);
    const uint32_t a_pref = a_bm + (uint32_t)((const char*)S.pref - (const char*)S.bm);
    const uint32_t a_vals = a_bm + (uint32_t)((const char*)S.vals - (const char*)S.bm);
#ifndef SG_BULK
#define SG_BULK 1
#endif
    constexpr bool kBulk = SG_BULK && sizeof(VT) == 8;  // fp64 output: accumulator copied out by bulk async copy
    int clear_n = 0;                          // accumulator entries still to be cleared (bulk path)
#if defined(SG_HV_EXP) && SG_HV_EXP == 8
    unsigned long long hph[10] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
    long long hv_last = clock64();
#endif
    while (true) {
        if (tid == 0) s_j = h0 + (long long)atomicAdd(counter, 1ull);
        __syncthreads();
        const int64_t h = s_j;
        __syncthreads();
        if (h >= nheavy) break;
        HV_MARK(6);
        const int64_t li = heavy[h];
        const int64_t row = rb + li;
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        const int na = (int)(s1 - s0);
        if (na <= amin) continue;  // a sparse rank row: the warp-tile kernel's (sg_tile.cu)
        const bool single = na <= KC;
        const int nr = nranges[h];
        const RangeRec* rr = ranges + range_off[h];
        const int64_t crow = C_rp[li];
        // per-k cursor state; single-chunk rows keep it in shared memory, one k per thread
        uint32_t tpv = 0;  // prefetched tile pointer of this thread's k for the next range
        for (int i = tid; i < na; i += NUM_T) {
            const int k = __ldg(A.col + s0 + i);
            const int32_t q0 = (int32_t)__ldg(B.rp + k), q1 = (int32_t)__ldg(B.rp + k + 1);
            if (single) {
                const int lid = tp && q1 - q0 > LONG_ROW ? __ldg(long_id + k) : -1;
                S.c_cur[i] = q0; S.c_end[i] = q1; S.c_q0[i] = q0; S.c_lid[i] = lid;
                S.c_a[i] = ldv<VT>(A.val, s0 + i);
                if (lid >= 0 && nr > 0) tpv = __ldg(tp + (int64_t)lid * (T + 1) + rr[0].t1);
            } else {
                gs[i] = make_int4(q0, 0, 0, 0);
            }
        }
        __syncthreads();
        HV_MARK(0);
#if defined(SG_HV_EXP) && SG_HV_EXP == 8
        if (threadIdx.x == 0) { hph[8] += nr; }
#endif
        RangeRec Rn;  // next range's record, loaded one range ahead
        if (nr > 0) Rn = rr[0];
        for (int ri = 0; ri < nr; ++ri) {
            const RangeRec R = Rn;
            if (ri + 1 < nr) Rn = rr[ri + 1];
#if defined(SG_HV_EXP) && SG_HV_EXP == 9
            const long long hv_t0 = clock64();
            long long hv_ts[6];
            hv_ts[0] = hv_t0;
#endif
            const int64_t lo = (int64_t)R.t0 * TW, hi = min(p, (int64_t)R.t1 * TW);
            int tot1 = 0, nk1 = 0;
            bool inreg = false;
            int i0_rest = 0;
            int rc[4];
            double rv[4];
            // ---- pass 1: segments (advance cursors) + bitmap of the range ----
            for (int c0 = 0; c0 < na; c0 += KC) {
                const int i = c0 + tid;
                int len = 0, beg = 0;
                double a = 0.0;
                if (i < na) {
                    if (single) {
                        const int cur = S.c_cur[i], lid = S.c_lid[i];
                        const int end = seg_end_any(B, cur, S.c_end[i], S.c_q0[i], lid >= 0, tpv, hi);
                        beg = cur; len = end - cur; a = S.c_a[i];
                        S.c_cur[i] = end;
                    } else {
                        const int4 g = gs[i];
                        const int k = __ldg(A.col + s0 + i);
                        const int32_t q0 = (int32_t)__ldg(B.rp + k), e1 = (int32_t)__ldg(B.rp + k + 1);
                        const bool lng = tp && e1 - q0 > LONG_ROW;
                        const uint32_t tv = lng ? __ldg(tp + (int64_t)__ldg(long_id + k) * (T + 1) + R.t1) : 0u;
                        const int end = seg_end_any(B, g.x, e1, q0, lng, tv, hi);
                        beg = g.x; len = end - g.x;
                        gs[i] = make_int4(end, 0, beg, len);
                    }
                }
                int nk;
                const int ctot = chunk_compact<NUM_T, int32_t>(len, beg, a, S.s_beg, S.s_off, S.s_a, &nk, S.wsll);
                HV_MARK(1);
#if defined(SG_HV_EXP) && SG_HV_EXP == 8
                if (threadIdx.x == 0) hph[9] += ctot;
#endif
                const uint32_t bb = opaque_u32(a_bm - 4u * ((uint32_t)lo >> 5));  // &bm[(c - lo) >> 5] = bb + 4(c >> 5)
                auto setbit = [&](int32_t c, double) {
                    if (c >= 0) red_or_s(bb + 4u * ((uint32_t)c >> 5), 1u << (c & 31));
                };
                // single-chunk rows: each warp's first four batches stay in registers from pass 1 to pass 2
                // (B read once for ranges of up to 4 * NUM_T products), only the rest is re-read in pass 2
                inreg = SG_INREG && single;
                if (inreg) {
                    i0_rest = warp_slice_head<NUM_T, VT, int32_t>(S.s_beg, S.s_off, S.s_a, nk, ctot, B, rc, rv);
                    #pragma unroll
                    for (int r = 0; r < 4; ++r) setbit(rc[r], 0.0);
                    warp_slice_rest<false, NUM_T, VT, int32_t>(S.s_beg, S.s_off, S.s_a, nk, ctot, i0_rest, B, setbit);
                } else {
                    warp_slice<NUM_T, false, VT, int32_t>(S.s_beg, S.s_off, nullptr, nk, ctot, B, setbit);
                }
                // prefetch the next range's tile pointer (its latency hides behind this range; issued
                // after pass 1 so that the next range record Rn has arrived)
                if (single && i < na && ri + 1 < nr) {
                    const int lid = S.c_lid[i];
                    if (lid >= 0) tpv = __ldg(tp + (int64_t)lid * (T + 1) + Rn.t1);
                }
                tot1 = ctot;
                nk1 = nk;
                if (!single) __syncthreads();
            }
            __syncthreads();
            HV_MARK(2);
            // ---- rank prefix over the range's words: thread t owns words [8t, 8t+8) (two 128-bit
            // loads, a sequential local prefix, one block scan, one 128-bit store of 8 uint16) ----
            {
                static_assert(RW_WORDS == 8 * NUM_T, "prefix layout: 8 words per thread");
                const uint4 q0 = reinterpret_cast<const uint4*>(S.bm)[2 * tid];
                const uint4 q1 = reinterpret_cast<const uint4*>(S.bm)[2 * tid + 1];
                const int c0 = __popc(q0.x), c1 = __popc(q0.y), c2 = __popc(q0.z), c3 = __popc(q0.w);
                const int c4 = __popc(q1.x), c5 = __popc(q1.y), c6 = __popc(q1.z), c7 = __popc(q1.w);
                int t2;
                if (kBulk && tid == 0) bulk_wait_read();  // previous range's values have left shared memory
                const int p0 = block_scan<NUM_T>(c0 + c1 + c2 + c3 + c4 + c5 + c6 + c7, &t2, S.ws);
                SG_BOUND(t2 == R.cnt);  // the range's bitmap holds exactly the plan's entries
                if (kBulk) {
                    for (int e = tid; e < clear_n; e += NUM_T) S.vals[e] = 0.0;
                    clear_n = 0;
                }
                const int p1 = p0 + c0, p2 = p1 + c1, p3 = p2 + c2, p4 = p3 + c3, p5 = p4 + c4, p6 = p5 + c5,
                          p7 = p6 + c6;
                uint4 o;
                o.x = (uint32_t)p0 | ((uint32_t)p1 << 16);
                o.y = (uint32_t)p2 | ((uint32_t)p3 << 16);
                o.z = (uint32_t)p4 | ((uint32_t)p5 << 16);
                o.w = (uint32_t)p6 | ((uint32_t)p7 << 16);
                reinterpret_cast<uint4*>(S.pref)[tid] = o;  // words >= nwords are zero: harmless prefixes
            }
            __syncthreads();
            HV_MARK(3);
            // ---- pass 2: every product accumulated at rank(c); the column is written on first arrival ----
            const int64_t base = crow + R.off;
            // vals[e + sh] and C_val[base + e] share 16 B alignment: sh from the ADDRESS (C_val is 8 B aligned,
            // sg_numeric checks; the caller's buffer itself need not be 16 B aligned)
            const int sh = kBulk ? (int)(((uintptr_t)(C_val + base) >> 3) & 1u) : 0;
            // lo is a multiple of 32: word (c - lo) >> 5 = (c >> 5) - (lo >> 5), bit c & 31
            const uint32_t bw = opaque_u32(a_bm - 4u * ((uint32_t)lo >> 5));
            const uint32_t pw = a_pref - 2u * ((uint32_t)lo >> 5);
            const uint32_t vb = a_vals + 8u * (uint32_t)sh;
            auto acc = [&](int32_t c, double v) {
                if (c < 0) return;
                const uint32_t cw = (uint32_t)c >> 5;
                const uint32_t wv = ld_u32_s(bw + 4u * cw);
                const int rank = (int)ld_u16_s(bw + (pw - bw) + 2u * cw) + __popc(wv & ((1u << (c & 31)) - 1u));
                // the product that finds the accumulator at exactly 0.0 writes the column: the first
                // product of every column does (accumulators start at 0.0); a later one only when the
                // partial sum is exactly 0.0, rewriting the same value
#if defined(SG_HV_EXP) && SG_HV_EXP == 3  // timing experiment: per-warp rotated ranks, no cross-warp same-address collisions (wrong C)
                const uint32_t rr2 = ((uint32_t)rank + 97u * (threadIdx.x >> 5)) % (uint32_t)RCAP;
                if (atom_add_f64_s(bw + (vb - bw) + 8u * rr2, v) == 0.0) st_out(C_col + base + rank, c);
#else
                if (atom_add_f64_s(bw + (vb - bw) + 8u * (uint32_t)rank, v) == 0.0) st_out(C_col + base + rank, c);
#endif
            };
            if (inreg) {
                #pragma unroll
                for (int r = 0; r < 4; ++r) acc(rc[r], rv[r]);
                warp_slice_rest<true, NUM_T, VT, int32_t>(S.s_beg, S.s_off, S.s_a, nk1, tot1, i0_rest, B, acc);
            } else if (single) {
                warp_slice<NUM_T, true, VT, int32_t>(S.s_beg, S.s_off, S.s_a, nk1, tot1, B, acc);  // pass-1 packing kept
            } else {
                for (int c0 = 0; c0 < na; c0 += KC) {
                    const int i = c0 + tid;
                    int len = 0, beg = 0;
                    double a = 0.0;
                    if (i < na) {
                        const int4 g = gs[i];
                        beg = g.z; len = g.w;
                        if (len > 0) a = ldv<VT>(A.val, s0 + i);
                    }
                    int nk;
                    const int ctot = chunk_compact<NUM_T, int32_t>(len, beg, a, S.s_beg, S.s_off, S.s_a, &nk, S.wsll);
                    warp_slice<NUM_T, true, VT, int32_t>(S.s_beg, S.s_off, S.s_a, nk, ctot, B, acc);
                    __syncthreads();
                }
            }
            if (kBulk) fence_proxy_async_smem();  // accumulator writes visible to the bulk copy
            __syncthreads();
            HV_MARK(4);
            // ---- values by rank; bitmap cleared for the next range ----
            const int cnt = R.cnt;
            if constexpr (kBulk) {
                // one bulk copy of the 16 B-aligned body; head / tail doubles by plain stores. The
                // accumulator is cleared in the next range's prefix phase, after the copy has read it.
                const int e0 = sh, n2 = (cnt - e0) & ~1;
                if (tid == 0 && n2 > 0) bulk_s2g(C_val + base + e0, &S.vals[e0 + sh], (uint32_t)n2 * 8u);
                if (tid == 32) {
                    if (sh && cnt > 0) st_out(C_val + base, (VT)S.vals[sh]);
                    if (e0 + n2 < cnt) st_out(C_val + base + e0 + n2, (VT)S.vals[e0 + n2 + sh]);
                }
                clear_n = cnt + 1;
            } else {
                for (int e = tid; e < cnt; e += NUM_T) {
                    st_out(C_val + base + e, (VT)S.vals[e]);
                    S.vals[e] = 0.0;
                }
            }
            {
                uint4* bm4 = reinterpret_cast<uint4*>(S.bm);
                bm4[2 * tid] = make_uint4(0, 0, 0, 0);
                bm4[2 * tid + 1] = make_uint4(0, 0, 0, 0);
            }
            HV_MARK(5);
#if defined(SG_HV_EXP) && SG_HV_EXP == 9
            if (tid == 0) {
                const int bn = 32 - __clz(tot1 | 1);
                atomicAdd(&g_hv_rng[bn][0], 1ull);
                atomicAdd(&g_hv_rng[bn][1], (unsigned long long)(clock64() - hv_t0));
                atomicAdd(&g_hv_rng[bn][2], (unsigned long long)tot1);
                atomicAdd(&g_hv_rng[bn][3], (unsigned long long)R.cnt);
                for (int k = 0; k < 5; ++k) atomicAdd(&g_hv_ph[bn][k], (unsigned long long)(hv_ts[k + 1] - hv_ts[k]));
            }
#endif
            // no barrier here: the next range's first reads of the cleared bitmap / accumulator and its
            // rewrite of the packed chunk arrays all come after chunk_compact's barriers
        }
    }
    if (kBulk && tid == 0) bulk_wait_all();
#if defined(SG_HV_EXP) && SG_HV_EXP == 8
    if ((threadIdx.x & 31) == 0)
        for (int k = 0; k < 10; ++k) atomicAdd(&g_hv_phase[k], hph[k]);
#endif
}

cudaError_t launch_num_heavy(const Mat& A, const Mat& B, const int32_t* heavy, int64_t h0, int64_t nheavy, int64_t rb,
                             const int64_t* range_off, const int32_t* nranges, const RangeRec* ranges,
                             const int32_t* long_id, const uint32_t* tp, int T, const int64_t* C_rp, int32_t* C_col,
                             void* C_val, unsigned long long* counter, int4* gscr, int64_t amax, int amin, cudaStream_t s) {
    if (nheavy - h0 <= 0) return cudaSuccess;
    const int smem = (int)sizeof(HeavySmem);
    cudaError_t e = cudaMemsetAsync(counter, 0, sizeof(unsigned long long), s);
    if (e != cudaSuccess) return e;
    const int64_t nh = nheavy - h0;
    const int grid = (int)(nh < NUM_OCC * 148 ? nh : NUM_OCC * 148);
    if (A.dt == 0) {
        if ((e = cudaFuncSetAttribute(k_num_heavy<double>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
        SG_LAUNCH("k_num_heavy", s, (k_num_heavy<double><<<grid, NUM_T, smem, s>>>(
                                        A, B, heavy, h0, nheavy, rb, range_off, nranges, ranges, long_id, tp, T, C_rp, C_col,
                                        (double*)C_val, counter, gscr, amax, amin)));
    } else {
        if ((e = cudaFuncSetAttribute(k_num_heavy<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
        SG_LAUNCH("k_num_heavy", s, (k_num_heavy<float><<<grid, NUM_T, smem, s>>>(
                                        A, B, heavy, h0, nheavy, rb, range_off, nranges, ranges, long_id, tp, T, C_rp, C_col,
                                        (float*)C_val, counter, gscr, amax, amin)));
    }
#if defined(SG_HV_EXP) && SG_HV_EXP == 8
    {
        unsigned long long hh[10] = {0};
        cudaStreamSynchronize(s);
        cudaMemcpyFromSymbol(hh, g_hv_phase, sizeof(hh));
        fprintf(stderr, "[rank phases, Gcycles summed over warps] row-setup %.2f seg+compact %.2f pass1 %.2f prefix %.2f "
                "pass2 %.2f emit %.2f fetch %.2f | ranges %llu products %llu (thread-0 counts)\n",
                hh[0] / 1e9, hh[1] / 1e9, hh[2] / 1e9, hh[3] / 1e9, hh[4] / 1e9, hh[5] / 1e9, hh[6] / 1e9,
                hh[8], hh[9]);
        unsigned long long z[10] = {0};
        cudaMemcpyToSymbol(g_hv_phase, z, sizeof(z));
    }
#endif
#if defined(SG_HV_EXP) && SG_HV_EXP == 9
    {
        unsigned long long hh[24][4] = {{0}}, ph[24][5] = {{0}};
        cudaStreamSynchronize(s);
        cudaMemcpyFromSymbol(hh, g_hv_rng, sizeof(hh));
        cudaMemcpyFromSymbol(ph, g_hv_ph, sizeof(ph));
        for (int b = 0; b < 24; ++b)
            if (hh[b][0])
                fprintf(stderr, "[rank ranges] products<2^%d: ranges %llu  cycles/range %.0f  products/range %.0f  out/range %.0f"
                        " | seg+compact %.0f pass1 %.0f prefix %.0f pass2 %.0f emit %.0f\n",
                        b, hh[b][0], (double)hh[b][1] / hh[b][0], (double)hh[b][2] / hh[b][0], (double)hh[b][3] / hh[b][0],
                        (double)ph[b][0] / hh[b][0], (double)ph[b][1] / hh[b][0], (double)ph[b][2] / hh[b][0],
                        (double)ph[b][3] / hh[b][0], (double)ph[b][4] / hh[b][0]);
        unsigned long long z[24][4] = {{0}}, z5[24][5] = {{0}};
        cudaMemcpyToSymbol(g_hv_rng, z, sizeof(z));
        cudaMemcpyToSymbol(g_hv_ph, z5, sizeof(z5));
    }
#endif
    return cudaGetLastError();
}

int heavy_kc() { return KC; }
int heavy_grid() { return NUM_OCC * 148; }

}  // namespace sg

namespace sg {
__global__ void k_max_a(Mat A, const int32_t* __restrict__ list, int64_t cnt, int64_t rb, unsigned long long* out) {
    unsigned long long m = 0;
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < cnt; j += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = rb + list[j];
        const unsigned long long a = (unsigned long long)(A.rp[r + 1] - A.rp[r]);
        m = a > m ? a : m;
    }
    #pragma unroll
    for (int o = 16; o; o >>= 1) { unsigned long long y = __shfl_xor_sync(FULL, m, o); m = y > m ? y : m; }
    if ((threadIdx.x & 31) == 0 && m) atomicMax(out, m);
}

cudaError_t launch_max_a(const Mat& A, const int32_t* list, int64_t cnt, int64_t rb, unsigned long long* out,
                         cudaStream_t s) {
    if (cnt <= 0) return cudaSuccess;
    SG_LAUNCH("k_max_a", s, (k_max_a<<<grid_for(cnt, 1024, 148 * 4), 256, 0, s>>>(A, list, cnt, rb, out)));
    return cudaGetLastError();
}
}  // namespace sg
