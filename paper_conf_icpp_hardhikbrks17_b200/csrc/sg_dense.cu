// sg_dense.cu — the densest HEAVY rows (w_i >= 2^dw_log2 > thr; PAPER L272-L274 routes them to the
// heavy path): a single-pass DENSE-WINDOW numeric.
//
// One CTA (1024 threads) per row, rows heaviest-first from a dynamic counter. The row's column
// space is swept in windows of WD = 24576 columns (three tiles); the accumulator is a dense fp64
// array indexed by column (vals[c - lo]): no bitmap pre-pass and no rank lookup per product (the
// rank-mode kernel in sg_heavy.cu needs both). The product that finds vals[c - lo] at exactly 0.0
// (the first arrival) marks bit (c - lo) of a 768-word occupancy bitmap; the window's entries are
// then emitted in column order (sorted by construction): one block scan of per-thread popcounts
// (24 columns each), each thread writing its own set bits; only the emitted slots are cleared.
//
// Work items are (row, window range): a row with w_i products is cut into ceil(w_i / DW_CHUNK_W)
// chunks of consecutive windows (each chunk's output offset from the symbolic pass's tile counts),
// taken heaviest-first from a dynamic counter, so the heaviest row (9.7M products at R-MAT 20) is
// spread over many SMs instead of being one CTA's serial tail.
// Per-k cursors advance window by window: B rows longer than LONG_ROW read their end from the
// tile-pointer table tp (prefetched one window ahead), short rows count their entries below the
// window end (cached in shared memory when two-tile windows leave room for it).
#include "sg_device.cuh"

namespace sg {

#ifndef SG_DW_T
#define SG_DW_T 1024
#endif
#ifndef SG_DW_OCC
#define SG_DW_OCC 1
#endif
#ifndef SG_DW_TILES
#define SG_DW_TILES 3
#endif
constexpr int DW_T = SG_DW_T;           // threads per CTA
constexpr int DW_OCC = SG_DW_OCC;       // CTAs per SM (while one CTA waits at a window barrier, another accumulates)
constexpr int DW_TILES = SG_DW_TILES;   // TW tiles per window
constexpr int WD = DW_TILES * TW;       // 24576 columns per window (192 KB fp64 accumulator)
constexpr int DW_WORDS = WD / 32;       // 768 occupancy words
constexpr int CPT = WD / DW_T;          // columns per thread in the emission
constexpr bool kShortCache = DW_TILES == 2;  // smem left for the short-row column cache
constexpr int DKC = DW_T;               // k entries per chunk (one per thread)
static_assert(CPT * DW_T == WD && CPT <= 32, "emission: CPT columns per thread");

struct DenseSmem {
    double vals[WD];                // dense accumulator of the window
    uint32_t bm[DW_WORDS + 1];      // occupancy (set by the first arrival); +1 pad word
    int32_t s_beg[DKC];             // packed chunk entries: segment begin (B position)
    int32_t s_off[DKC];             //                       exclusive prefix of segment lengths
    double s_a[DKC];                //                       a_ik
    int32_t sc[kShortCache ? LONG_ROW : 1][DKC];  // short B rows of single-chunk rows: their columns ([q][k], INT_MAX pad)
    long long wsll[33];
    int ws[33];
};

template <class VT>
__global__ void __launch_bounds__(DW_T, DW_OCC) k_num_dense(
    Mat A, Mat B, const int32_t* __restrict__ heavy, int64_t ndw, int64_t rb, const int32_t* __restrict__ long_id,
    const uint32_t* __restrict__ tp, int T, const int64_t* __restrict__ C_rp, int32_t* __restrict__ C_col,
    VT* __restrict__ C_val, unsigned long long* counter, int4* __restrict__ gscr, int64_t amax,
    const int32_t* __restrict__ dtc, const int4* __restrict__ items, const int64_t* __restrict__ nitems) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    DenseSmem& S = *reinterpret_cast<DenseSmem*>(smem_raw);
    __shared__ long long s_j;
    const int tid = threadIdx.x;
    const int64_t p = B.ncols;
    int4* gs = gscr + (int64_t)blockIdx.x * amax;  // multi-chunk rows: per-k cursor
    const uint32_t a_vals = smem_addr(S.vals), a_bm = smem_addr(S.bm);
    for (int q = tid; q < WD; q += DW_T) S.vals[q] = 0.0;
    for (int q = tid; q < DW_WORDS + 1; q += DW_T) S.bm[q] = 0u;
    const int64_t n_items = *nitems;
    while (true) {
        if (tid == 0) s_j = (long long)atomicAdd(counter, 1ull);
        __syncthreads();
        const int64_t it = s_j;
        __syncthreads();
        if (it >= n_items) break;
        // work item: windows [ta, tb) of dense row h (a row with w_i products is cut into
        // ceil(w_i / DW_CHUNK_W) chunks of consecutive windows, so no single row is a tail)
        const int4 item = items[it];
        const int64_t h = item.x;
        const int ta = item.y, tb = item.z;
        const int64_t li = heavy[h];
        const int64_t row = rb + li;
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        const int na = (int)(s1 - s0);
        const bool single = na <= DKC;
        const int t0 = ta;
        const int64_t lo0 = (int64_t)t0 * WD;
        // output offset of window t0 inside the row: the row's tile counts below tile t0*DW_TILES
        int64_t off0 = 0;
        if (t0 > 0) {
            long long c = 0;
            const int te = min(t0 * DW_TILES, T);
            for (int q = tid; q < te; q += DW_T) c += dtc[h * (int64_t)T + q];
            long long tot;
            block_scan_ll<DW_T>(c, &tot, S.wsll);
            off0 = tot;
            __syncthreads();  // every warp has read wsll before chunk_compact rewrites it
        }
        const int64_t rowbase = C_rp[li];
        int64_t pos = rowbase + off0;
        // per-k state of single-chunk rows: thread tid owns k entry tid; cursor at column lo0
        int cur = 0, q0 = 0, lid = -1, e1r = 0;
        uint32_t tpv = 0;
        double a = 0.0;
        if (single) {
            if (tid < na) {
                const int k = __ldg(A.col + s0 + tid);
                q0 = (int)__ldg(B.rp + k);
                const int len = (int)(__ldg(B.rp + k + 1) - q0);
                a = ldv<VT>(A.val, s0 + tid);
                if (len > LONG_ROW) {
                    lid = __ldg(long_id + k);
                    const uint32_t* tr = tp + (int64_t)lid * (T + 1);
                    cur = q0 + (int)__ldg(tr + min(t0 * DW_TILES, T));
                    tpv = __ldg(tr + min((t0 + 1) * DW_TILES, T));
                } else if constexpr (kShortCache) {
                    int n0 = 0;
                    #pragma unroll
                    for (int q = 0; q < LONG_ROW; ++q) {
                        const int c = q < len ? __ldg(B.col + q0 + q) : INT_MAX;
                        S.sc[q][tid] = c;
                        n0 += c < lo0;
                    }
                    cur = q0 + n0;
                } else {
                    e1r = q0 + len;
                    cur = t0 > 0 ? seg_end(B, q0, e1r, q0, false, 0u, lo0) : q0;
                }
            }
        } else {
            for (int i = tid; i < na; i += DW_T) {
                const int k = __ldg(A.col + s0 + i);
                const int32_t kq0 = (int32_t)__ldg(B.rp + k), e1 = (int32_t)__ldg(B.rp + k + 1);
                int c0 = kq0;
                if (t0 > 0) {
                    const bool lng = e1 - kq0 > LONG_ROW;
                    const uint32_t tv = lng ? __ldg(tp + (int64_t)__ldg(long_id + k) * (T + 1) + min(t0 * DW_TILES, T)) : 0u;
                    c0 = seg_end(B, kq0, e1, kq0, lng, tv, lo0);
                }
                gs[i] = make_int4(c0, 0, 0, 0);
            }
        }
#ifndef SG_DW_PIPE
#define SG_DW_PIPE 1
#endif
        if (SG_DW_PIPE && single) {
            // Single-chunk rows, software-pipelined: window t+1's segments are found while window t is
            // emitted, and ONE block scan (block_scan2) places both window t's output entries and window
            // t+1's packed chunk entries: 3 barriers per window instead of 4.
            auto seg_next = [&](int tw, int& len, int& beg) {  // segment of this thread's k in window tw
                len = 0;
                beg = cur;
                if (tid < na && tw < tb) {
                    const int64_t whi = min(p, (int64_t)(tw + 1) * WD);
                    int end;
                    if (lid >= 0) {
                        end = q0 + (int)tpv;
                        if (tw + 1 < tb) tpv = __ldg(tp + (int64_t)lid * (T + 1) + min((tw + 2) * DW_TILES, T));
                    } else if constexpr (kShortCache) {
                        int n = 0;
                        #pragma unroll
                        for (int q = 0; q < LONG_ROW; ++q) n += S.sc[q][tid] < whi;
                        end = q0 + n;
                    } else {
                        end = seg_end(B, cur, e1r, q0, false, 0u, whi);
                    }
                    len = end - cur;
                    cur = end;
                }
            };
            int nk, any;
            {
                int len, beg;
                seg_next(ta, len, beg);
                any = chunk_compact<DW_T, int32_t>(len, beg, a, S.s_beg, S.s_off, S.s_a, &nk, S.wsll);
            }
            for (int t = ta; t < tb; ++t) {
                const int64_t lo = (int64_t)t * WD;
                const uint32_t vb = opaque_u32(a_vals - 8u * (uint32_t)lo);
                const uint32_t bb = opaque_u32(a_bm - 4u * ((uint32_t)lo >> 5));
                if (any > 0)
                    warp_slice<DW_T, true, VT, int32_t>(S.s_beg, S.s_off, S.s_a, nk, any, B, [&](int32_t c, double v) {
                        if (c < 0) return;
                        if (atom_add_f64_s(vb + 8u * (uint32_t)c, v) == 0.0)
                            red_or_s(bb + 4u * ((uint32_t)c >> 5), 1u << (c & 31));
                    });
                __syncthreads();  // window t accumulated; the packed chunk arrays are free
                uint32_t hw;
                {
                    const int b0 = CPT * tid, w0 = b0 >> 5, shv = b0 & 31;
                    const unsigned long long two = ((unsigned long long)S.bm[w0 + 1] << 32) | S.bm[w0];
                    hw = (uint32_t)(two >> shv) & (CPT == 32 ? 0xFFFFFFFFu : ((1u << CPT) - 1u));
                }
                int len, beg;
                seg_next(t + 1, len, beg);
                int ex, wtot;
                long long exc, totc;
                block_scan2<DW_T>(__popc(hw), ((long long)len << 16) | (len > 0 ? 1 : 0), &ex, &wtot, &exc, &totc, S.ws,
                                  S.wsll);
                for (int q = tid; q < DW_WORDS; q += DW_T) S.bm[q] = 0u;  // every bitmap read preceded the scan
                {
                    uint32_t m = hw;
                    int64_t at = pos + ex;
                    const int ebase = tid * CPT;
                    while (m) {
                        const int e = ebase + __ffs(m) - 1;
                        m &= m - 1u;
                        st_out(C_col + at, (int32_t)(lo + e));
                        st_out(C_val + at, (VT)S.vals[e]);
                        S.vals[e] = 0.0;
                        ++at;
                    }
                }
                pos += wtot;
                if (len > 0) {
                    const int ci = (int)(exc & 0xFFFF);
                    S.s_beg[ci] = beg;
                    S.s_off[ci] = (int)(exc >> 16);
                    S.s_a[ci] = a;
                    mark_slice_starts<DW_T>(ci, (int)(exc >> 16), len, (int)(totc >> 16));
                }
                nk = (int)(totc & 0xFFFF);
                any = (int)(totc >> 16);
                __syncthreads();  // chunk arrays of window t+1 published; clears ordered before its products
            }
            continue;
        }
        for (int t = ta; t < tb; ++t) {
            const int tn = t + 1;  // next window
            const int64_t lo = (int64_t)t * WD, hi = min(p, lo + WD);
            const int th = min((t + 1) * DW_TILES, T);  // tile index of hi
            // window-relative shared addresses folded into one base each (lo is a multiple of 32):
            // &vals[c - lo] = vb + 8c, &bm[(c - lo) >> 5] = bb + 4(c >> 5)  (mod 2^32)
            const uint32_t vb = opaque_u32(a_vals - 8u * (uint32_t)lo);
            const uint32_t bb = opaque_u32(a_bm - 4u * ((uint32_t)lo >> 5));
            auto acc = [&](int32_t c, double v) {
                if (c < 0) return;
                // first arrival (accumulator at exactly 0.0) marks the column; a later product that finds
                // an exact 0.0 partial sum re-marks it (idempotent)
                if (atom_add_f64_s(vb + 8u * (uint32_t)c, v) == 0.0) red_or_s(bb + 4u * ((uint32_t)c >> 5), 1u << (c & 31));
            };
            int any = 0;
            if (single) {
                int len = 0;
                const int beg = cur;
                if (tid < na) {
                    int end;
                    if (lid >= 0) {
                        end = q0 + (int)tpv;
                        if (tn < tb) tpv = __ldg(tp + (int64_t)lid * (T + 1) + min((tn + 1) * DW_TILES, T));
                    } else if constexpr (kShortCache) {
                        int n = 0;
                        #pragma unroll
                        for (int q = 0; q < LONG_ROW; ++q) n += S.sc[q][tid] < hi;
                        end = q0 + n;
                    } else {
                        end = seg_end(B, cur, e1r, q0, false, 0u, hi);
                    }
                    len = end - cur;
                    cur = end;
                }
                int nk;
                any = chunk_compact<DW_T, int32_t>(len, beg, a, S.s_beg, S.s_off, S.s_a, &nk, S.wsll);
                if (any == 0) continue;  // block-uniform: nothing in this window
                warp_slice<DW_T, true, VT, int32_t>(S.s_beg, S.s_off, S.s_a, nk, any, B, acc);
            } else {
                for (int c0 = 0; c0 < na; c0 += DKC) {
                    const int i = c0 + tid;
                    int len = 0, beg = 0;
                    double ai = 0.0;
                    if (i < na) {
                        const int4 g = gs[i];
                        const int k = __ldg(A.col + s0 + i);
                        const int32_t kq0 = (int32_t)__ldg(B.rp + k), e1 = (int32_t)__ldg(B.rp + k + 1);
                        const bool lng = e1 - kq0 > LONG_ROW;
                        const uint32_t tv = lng ? __ldg(tp + (int64_t)__ldg(long_id + k) * (T + 1) + th) : 0u;
                        const int end = seg_end(B, g.x, e1, kq0, lng, tv, hi);
                        beg = g.x;
                        len = end - g.x;
                        if (len > 0) ai = ldv<VT>(A.val, s0 + i);
                        gs[i] = make_int4(end, 0, 0, 0);
                    }
                    int nk;
                    const int ctot = chunk_compact<DW_T, int32_t>(len, beg, ai, S.s_beg, S.s_off, S.s_a, &nk, S.wsll);
                    if (ctot > 0) warp_slice<DW_T, true, VT, int32_t>(S.s_beg, S.s_off, S.s_a, nk, ctot, B, acc);
                    any += ctot;
                }
                if (any == 0) continue;
            }
            __syncthreads();  // every product of the window accumulated
            // ---- emission: thread tid owns columns [CPT*tid, CPT*tid + CPT) of the window; one block
            // scan of their popcounts places every run; each thread writes its set bits in order ----
            uint32_t hw;
            {
                const int b0 = CPT * tid, w0 = b0 >> 5, shv = b0 & 31;
                const unsigned long long two = ((unsigned long long)S.bm[w0 + 1] << 32) | S.bm[w0];
                hw = (uint32_t)(two >> shv) & (CPT == 32 ? 0xFFFFFFFFu : ((1u << CPT) - 1u));
            }
            int wtot;
            const int ex = block_scan1<DW_T, int>(__popc(hw), &wtot, S.ws);
            for (int q = tid; q < DW_WORDS; q += DW_T) S.bm[q] = 0u;  // all reads preceded the scan's barrier
            {
                uint32_t m = hw;
                int64_t at = pos + ex;
                const int ebase = tid * CPT;
                while (m) {
                    const int e = ebase + __ffs(m) - 1;
                    m &= m - 1u;
                    st_out(C_col + at, (int32_t)(lo + e));
                    st_out(C_val + at, (VT)S.vals[e]);
                    S.vals[e] = 0.0;
                    ++at;
                }
            }
            pos += wtot;
            // the next window's chunk_compact barriers order these clears before its products
        }
    }
}

// ---- work items: chunks of consecutive windows per dense row ------------------------------------
constexpr int64_t DW_CHUNK_W = 1 << 19;  // products per work item (about 1/20 of the heaviest R-MAT 20 row)

__device__ __forceinline__ int64_t dense_nchunk(int64_t w, int nwin) {
    int64_t c = (w + DW_CHUNK_W - 1) / DW_CHUNK_W;
    return c < 1 ? 1 : (c > nwin ? nwin : c);
}

__global__ void k_dense_nchunk(const int32_t* __restrict__ heavy, int64_t ndw, const int64_t* __restrict__ w, int nwin,
                               int64_t* __restrict__ cnt) {
    const int64_t h = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (h < ndw) cnt[h] = dense_nchunk(w[heavy[h]], nwin);
}

__global__ void k_dense_items(const int32_t* __restrict__ heavy, int64_t ndw, const int64_t* __restrict__ w, int nwin,
                              const int64_t* __restrict__ off, int4* __restrict__ items) {
    const int64_t h = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (h >= ndw) return;
    const int64_t nc = dense_nchunk(w[heavy[h]], nwin);
    for (int64_t c = 0; c < nc; ++c)
        items[off[h] + c] = make_int4((int)h, (int)(c * nwin / nc), (int)((c + 1) * nwin / nc), 0);
}

// Window-major items [r2]: every dense row is cut into blocks of DW_BLOCK consecutive windows and the
// items are ordered block by block (item blk * ndw + h = row h's block blk; rows heaviest first inside a
// block). The persistent CTAs take items in that order, so at any time they all sweep the same one or
// two window blocks: the slab of B they gather (~193 MB / 43 windows per window at C3) stays L2-resident
// instead of every CTA streaming its own part of B through L2 (round 1: dense-kernel DRAM traffic ~4x
// its algorithmic bytes, profiles/r02f_ncu_traffic.txt).
constexpr int DW_BLOCK = 3;

__global__ void k_dense_items_wm(int64_t ndw, int nwin, int nblk, int4* __restrict__ items, int64_t* __restrict__ nitems) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i == 0) *nitems = ndw * nblk;
    if (i >= ndw * nblk) return;
    const int blk = (int)(i / ndw);
    const int64_t h = i % ndw;
    items[i] = make_int4((int)h, blk * DW_BLOCK, min(nwin, (blk + 1) * DW_BLOCK), 0);
}

cudaError_t launch_dense_items_wm(int64_t ndw, int64_t p, int4* items, int64_t* nitems, cudaStream_t s) {
    if (ndw <= 0) return cudaSuccess;
    const int nwin = (int)((p + WD - 1) / WD);
    const int nblk = (nwin + DW_BLOCK - 1) / DW_BLOCK;
    const int64_t n = ndw * nblk;
    SG_LAUNCH("k_dense_items", s, (k_dense_items_wm<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(ndw, nwin, nblk, items, nitems)));
    return cudaGetLastError();
}

int64_t dense_items_bound(int64_t ndw, int64_t p) {
    const int64_t nwin = (p + WD - 1) / WD;
    return ndw * (nwin < 1 ? 1 : nwin);
}

cudaError_t launch_dense_items(const int32_t* heavy, int64_t ndw, const int64_t* w, int64_t p, int64_t* cnt,
                               int64_t* off, void* scan_tmp, int4* items, cudaStream_t s) {
    if (ndw <= 0) return cudaSuccess;
    const int nwin = (int)((p + WD - 1) / WD);
    const unsigned g = (unsigned)((ndw + 255) / 256);
    SG_LAUNCH("k_dense_nchunk", s, (k_dense_nchunk<<<g, 256, 0, s>>>(heavy, ndw, w, nwin, cnt)));
    cudaError_t e = scan_exclusive(cnt, off, ndw, scan_tmp, s);  // off[ndw] = number of items
    if (e != cudaSuccess) return e;
    SG_LAUNCH("k_dense_items", s, (k_dense_items<<<g, 256, 0, s>>>(heavy, ndw, w, nwin, off, items)));
    return cudaGetLastError();
}

cudaError_t launch_num_dense(const Mat& A, const Mat& B, const int32_t* heavy, int64_t ndw, int64_t rb,
                             const int32_t* long_id, const uint32_t* tp, int T, const int64_t* C_rp, int32_t* C_col,
                             void* C_val, unsigned long long* counter, int4* gscr, int64_t amax,
                             const int32_t* dtc, const int4* items, const int64_t* nitems, cudaStream_t s) {
    if (ndw <= 0) return cudaSuccess;
    const int smem = (int)sizeof(DenseSmem);
    cudaError_t e = cudaMemsetAsync(counter, 0, sizeof(unsigned long long), s);  // item counter
    if (e != cudaSuccess) return e;
    const int grid = 148 * DW_OCC;  // persistent; CTAs beyond the item count exit at once
    if (A.dt == 0) {
        if ((e = cudaFuncSetAttribute(k_num_dense<double>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
        SG_LAUNCH("k_num_dense", s, (k_num_dense<double><<<grid, DW_T, smem, s>>>(A, B, heavy, ndw, rb, long_id, tp, T, C_rp,
                                                                                  C_col, (double*)C_val, counter, gscr, amax, dtc, items, nitems)));
    } else {
        if ((e = cudaFuncSetAttribute(k_num_dense<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
        SG_LAUNCH("k_num_dense", s, (k_num_dense<float><<<grid, DW_T, smem, s>>>(A, B, heavy, ndw, rb, long_id, tp, T, C_rp,
                                                                                 C_col, (float*)C_val, counter, gscr, amax, dtc, items, nitems)));
    }
    return cudaGetLastError();
}

int dense_window_cols() { return WD; }
int dense_grid() { return 148 * DW_OCC; }
int dense_kc() { return DKC; }

}  // namespace sg

namespace sg {
// Rows with w >= 2^m take the dense-window kernel. Its fixed cost grows with the number of windows
// (p / WD) while its saving over the rank kernel grows with w, so m tracks log2 p: 2^19 at p = 2^20
// (C3: 283.5 vs 284.6 ms/step at 2^18), 2^17 at p = 2^18 (R-MAT 18: 35.2 vs 35.6 ms).
int dense_window_log2(int64_t p, int64_t opt) {
    if (opt >= 0) return (int)(opt > 62 ? 62 : opt);  // sg_set_option(SG_OPT_DENSE_LOG2); 62 disables the path
    int lp = 0;
    while (lp < 62 && ((int64_t)1 << lp) < p) ++lp;
    const int m = lp - 1;
    return m < 4 ? 4 : m;
}
}  // namespace sg
