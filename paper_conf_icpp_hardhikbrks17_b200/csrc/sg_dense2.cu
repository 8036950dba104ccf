// sg_dense2.cu — dense-window HEAVY numeric with a lean product walk.
//
// Same accumulator as sg_dense.cu (a dense fp64 window of WD columns, first-arrival occupancy bits,
// emission in column order), different product enumeration. ncu (profiles/r02_*) put 60-70 % of that
// kernel's instructions in the per-window block packing (chunk_compact) and the per-batch shuffle search
// over the packed entries (SliceCursor), against ~15 % in the accumulate itself. Here:
//
//  * once per work item the row's products [0, w_i) are cut into 32 equal, contiguous slices, one per
//    warp: a warp's slice is a list of PARTS (k, sub-range of B_k), a k that straddles a slice boundary
//    being split (so no warp is left with a whole hub row of B). Part state (cursor, end, a_ik) lives in
//    shared memory (global scratch for rows with more than D2_PCAP - 32 k entries);
//  * per window, each warp walks only its own parts, 32 at a time: one cursor step per part (the B
//    tile pointer for long B rows, a bounded scan for short ones), then LONG segments (>= 32 products)
//    are swept lane-strided with four batches in flight and no search, SHORT ones flattened by one warp
//    scan plus a 5-step shuffle search per batch. No block barrier until the window is complete.
#include "sg_device.cuh"
#include <cstdio>

namespace sg {

constexpr int D2_T = 1024;                 // threads per CTA (one CTA per SM)
constexpr int D2_NW = D2_T / 32;           // warps = product slices per work item
constexpr int D2_TILES = 3;                // TW-column tiles per window
constexpr int D2_WD = D2_TILES * TW;       // 24576 columns per window (192 KB fp64 accumulator)
constexpr int D2_WORDS = D2_WD / 32;       // occupancy words
constexpr int D2_CPT = D2_WD / D2_T;       // columns per thread in the emission
constexpr int D2_PCAP = 1216;              // parts held in shared memory
static_assert(D2_CPT * D2_T == D2_WD && D2_CPT <= 32, "emission: D2_CPT columns per thread");

using D2Part = Part;

struct D2Smem {
    double vals[D2_WD];
    uint32_t bm[D2_WORDS + 1];  // +1 pad word for the two-word emission read
    D2Part parts[D2_PCAP];
    int32_t wpart[D2_NW + 1];   // warp w owns parts [wpart[w], wpart[w+1])
    long long wsll[33];
    int ws[33];
};
static_assert(sizeof(D2Smem) + 64 <= 232448, "dense2 shared memory exceeds the sm_100a per-block limit");

size_t dense2_part_bytes() { return sizeof(D2Part); }
int dense2_pcap() { return D2_PCAP; }


#if defined(SG_D2_EXP) && SG_D2_EXP == 8  // timing experiment: per-phase cycle counters (lane 0 of each warp)
__device__ unsigned long long g_d2_phase[8];
#define D2_MARK(k) do { if (lane == 0) { long long _t = clock64(); ph[k] += _t - t_last; t_last = _t; } } while (0)
#else
#define D2_MARK(k) do { } while (0)
#endif

template <class VT>
__global__ void __launch_bounds__(D2_T, 1) k_num_dense2(
    Mat A, Mat B, const int32_t* __restrict__ heavy, int64_t rb, const int64_t* __restrict__ wrow,
    const int32_t* __restrict__ long_id, const uint32_t* __restrict__ tp, int T, const int64_t* __restrict__ C_rp,
    int32_t* __restrict__ C_col, VT* __restrict__ C_val, unsigned long long* counter, D2Part* __restrict__ pscr,
    int64_t pscr_cap, const int32_t* __restrict__ dtc, const int4* __restrict__ items,
    const int64_t* __restrict__ nitems) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    D2Smem& S = *reinterpret_cast<D2Smem*>(smem_raw);
    __shared__ long long s_j;
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int64_t p = B.ncols;
    const uint32_t a_vals = smem_addr(S.vals), a_bm = smem_addr(S.bm);
    for (int q = tid; q < D2_WD; q += D2_T) S.vals[q] = 0.0;
    for (int q = tid; q < D2_WORDS + 1; q += D2_T) S.bm[q] = 0u;
    const int64_t n_items = *nitems;
#if defined(SG_D2_EXP) && SG_D2_EXP == 8
    unsigned long long ph[6] = {0, 0, 0, 0, 0, 0};
    long long t_last = clock64();
#endif
    while (true) {
        if (tid == 0) s_j = (long long)atomicAdd(counter, 1ull);
        __syncthreads();
        const int64_t it = s_j;
        if (it >= n_items) break;
        D2_MARK(5);
        const int4 item = items[it];
        const int64_t h = item.x;
        const int ta = item.y, tb = item.z;
        const int64_t li = heavy[h];
        const int64_t row = rb + li;
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        const int na = (int)(s1 - s0);
        const long long L = wrow[li];  // products of the row = sum of its B row lengths (> 0: heavy)
        D2Part* P = na + D2_NW <= D2_PCAP ? S.parts : pscr + (int64_t)blockIdx.x * pscr_cap;
        const int64_t lo0 = (int64_t)ta * D2_WD;
        const int tlo = min(ta * D2_TILES, T);
        // output offset of window ta inside the row: the row's tile counts below tile ta*D2_TILES
        long long off0 = 0;
        if (ta > 0) {
            long long c = 0;
            for (int q = tid; q < tlo; q += D2_T) c += dtc[h * (int64_t)T + q];
            block_scan_ll<D2_T>(c, &off0, S.wsll);
            __syncthreads();  // wsll read by every warp before the part scans rewrite it
        }
        // ---- parts: the row's products cut into D2_NW equal slices (k entries split at boundaries) ----
        build_parts<D2_T, VT, true>(A, B, s0, na, L, long_id, tp, T, tlo, lo0, P, S.wpart, S.wsll, S.ws);
        D2_MARK(0);
        const int pw0 = S.wpart[wid], pw1 = S.wpart[wid + 1];
        int64_t pos = C_rp[li] + off0;
        // the first 32 parts of the warp read their window-end tile pointer one window ahead
        uint32_t tpn = 0;
        int lid0 = -1;
        if (pw0 + lane < pw1) {
            lid0 = P[pw0 + lane].lid;
            if (lid0 >= 0) tpn = __ldg(tp + (int64_t)lid0 * (T + 1) + min((ta + 1) * D2_TILES, T));
        }
        for (int t = ta; t < tb; ++t) {
            const int64_t lo = (int64_t)t * D2_WD, hi = min(p, lo + D2_WD);
            const int th = min((t + 1) * D2_TILES, T);
            const uint32_t vb = opaque_u32(a_vals - 8u * (uint32_t)lo);
            const uint32_t bb = opaque_u32(a_bm - 4u * ((uint32_t)lo >> 5));
            auto acc = [&](int32_t c, double v) {
                // first arrival (accumulator at exactly 0.0) marks the column; a later product that finds
                // an exact 0.0 partial sum re-marks it (idempotent)
#ifndef SG_D2_EXP
#define SG_D2_EXP 0
#endif
#if SG_D2_EXP == 1 || SG_D2_EXP == 5  // timing experiment: products gathered, not accumulated (wrong C)
                if (v == 1234.5) red_or_s_nc(bb + 4u * ((uint32_t)c >> 5), 1u);
#elif SG_D2_EXP == 2  // timing experiment: plain shared RMW instead of the CAS (wrong C)
                const uint32_t ad = vb + 8u * (uint32_t)c;
                const double o = ld_f64_s(ad);
                asm volatile("st.shared.f64 [%0], %1;" ::"r"(ad), "d"(o + v));
                if (o == 0.0) red_or_s_nc(bb + 4u * ((uint32_t)c >> 5), 1u << (c & 31));
#elif SG_D2_EXP == 3  // timing experiment: per-warp rotated addresses (no cross-warp collisions; wrong C)
                const uint32_t cc = (uint32_t)(c - (int)lo + 97 * (int)(threadIdx.x >> 5)) % (uint32_t)D2_WD;
                if (atom_add_f64_s_nc(a_vals + 8u * cc, v) == 0.0) red_or_s_nc(bb + 4u * ((uint32_t)c >> 5), 1u << (c & 31));
#else
                if (atom_add_f64_s(vb + 8u * (uint32_t)c, v) == 0.0) red_or_s(bb + 4u * ((uint32_t)c >> 5), 1u << (c & 31));
#endif
            };
            for (int g = pw0; g < pw1; g += 32) {
                const int j = g + lane;
                int beg = 0, len = 0;
                double a = 0.0;
                if (j < pw1) {
                    const int cur = P[j].cur, end = P[j].end;
                    if (cur < end) {
                        const int lid = P[j].lid;
                        int e;
                        if (lid >= 0) {
                            const uint32_t tv = g == pw0 ? tpn : __ldg(tp + (int64_t)lid * (T + 1) + th);
                            // a part may start past this window's end (its slice begins mid-row)
                            e = max(cur, min(end, P[j].q0 + (int)tv));
                        } else {
                            e = cur;
                            while (e < end && __ldg(B.col + e) < hi) ++e;  // <= LONG_ROW entries
                        }
                        beg = cur;
                        len = e - cur;
                        a = P[j].a;
                        P[j].cur = e;
                    }
                }
                if (g == pw0 && lid0 >= 0 && t + 1 < tb)
                    tpn = __ldg(tp + (int64_t)lid0 * (T + 1) + min((t + 2) * D2_TILES, T));
                seg_walk<true, VT>(B, beg, len, a, acc);
            }
            D2_MARK(1);
            __syncthreads();  // window t accumulated
            D2_MARK(2);
#ifndef SG_D2_EMIT
#define SG_D2_EMIT 1
#endif
#if SG_D2_EMIT
            // ---- emission, coalesced: warp w owns bitmap words [24w, 24w + 24) (768 columns); a warp scan
            // of their popcounts and one exchange of warp totals place its entries; then output positions
            // p = 32 r + lane are written by lane (word found by a 5-step shuffle search, bit by a popc
            // bisection), so every store instruction covers 32 consecutive C entries (ncu: the
            // per-thread scattered emission was 25 % of the kernel, profiles/r02_dense2_phases.txt) ----
            static_assert(D2_WORDS == 24 * D2_NW, "emission: 24 bitmap words per warp");
            const int wbase = 24 * wid;
            const uint32_t wv = lane < 24 ? S.bm[wbase + lane] : 0u;
            const int pcw = __popc(wv);
            const int incl = warp_incl_scan(pcw);
            const int excl = incl - pcw;
            const int wt = __shfl_sync(FULL, incl, 31);
            if (lane == 0) S.ws[wid] = wt;
            __syncthreads();  // warp totals published; every bitmap word read
            const int xw = S.ws[lane];
            const int xi = warp_incl_scan(xw);
            const int woff = __shfl_sync(FULL, xi - xw, wid);
            const int wtot = __shfl_sync(FULL, xi, 31);
            if (lane < 24) S.bm[wbase + lane] = 0u;
            for (int p0 = 0; p0 < wt; p0 += 32) {
                const int pp = p0 + lane;
                int sw = 0;  // largest word index with excl <= pp (lanes >= 24 hold excl = wt > pp)
                #pragma unroll
                for (int b = 16; b; b >>= 1) {
                    const int e2 = __shfl_sync(FULL, excl, sw + b);
                    if (e2 <= pp) sw += b;
                }
                uint32_t x = __shfl_sync(FULL, wv, sw);
                int k = pp - __shfl_sync(FULL, excl, sw);
                if (pp < wt) {
                    int bit = 0, c;  // k-th set bit of x (0-based)
                    c = __popc(x & 0xFFFFu); if (k >= c) { k -= c; bit += 16; x >>= 16; }
                    c = __popc(x & 0xFFu);   if (k >= c) { k -= c; bit += 8;  x >>= 8; }
                    c = __popc(x & 0xFu);    if (k >= c) { k -= c; bit += 4;  x >>= 4; }
                    c = __popc(x & 0x3u);    if (k >= c) { k -= c; bit += 2;  x >>= 2; }
                    if (k >= (int)(x & 1u)) bit += 1;
                    const int e = 32 * (wbase + sw) + bit;
                    const int64_t at = pos + woff + pp;
#if SG_D2_EXP == 4 || SG_D2_EXP == 5  // timing experiment: emission without the global stores (wrong C)
                    if (S.vals[e] == 1234.5) st_out(C_col + at, (int32_t)(lo + e));
#else
                    st_out(C_col + at, (int32_t)(lo + e));
                    st_out(C_val + at, (VT)S.vals[e]);
#endif
                    S.vals[e] = 0.0;
                }
            }
#else
            // ---- emission: thread tid owns columns [D2_CPT*tid, +D2_CPT) of the window; one block scan of
            // their popcounts places every run; each thread writes its set bits in column order ----
            uint32_t hwb;
            {
                const int b0 = D2_CPT * tid, w0 = b0 >> 5, shv = b0 & 31;
                const unsigned long long two = ((unsigned long long)S.bm[w0 + 1] << 32) | S.bm[w0];
                hwb = (uint32_t)(two >> shv) & (D2_CPT == 32 ? 0xFFFFFFFFu : ((1u << D2_CPT) - 1u));
            }
            int wtot;
            const int ex = block_scan1<D2_T, int>(__popc(hwb), &wtot, S.ws);
            for (int q = tid; q < D2_WORDS; q += D2_T) S.bm[q] = 0u;  // every read preceded the scan's barrier
            {
                uint32_t m = hwb;
                int64_t at = pos + ex;
                const int ebase = tid * D2_CPT;
                while (m) {
                    const int e = ebase + __ffs(m) - 1;
                    m &= m - 1u;
                    st_out(C_col + at, (int32_t)(lo + e));
                    st_out(C_val + at, (VT)S.vals[e]);
                    S.vals[e] = 0.0;
                    ++at;
                }
            }
#endif
            pos += wtot;
            D2_MARK(3);
            __syncthreads();  // clears (and ws) ordered before the next window's products / scans
            D2_MARK(4);
        }
    }
#if defined(SG_D2_EXP) && SG_D2_EXP == 8
    if (lane == 0)
        for (int k = 0; k < 6; ++k) atomicAdd(&g_d2_phase[k], ph[k]);
#endif
}

cudaError_t launch_num_dense2(const Mat& A, const Mat& B, const int32_t* heavy, int64_t ndw, int64_t rb,
                              const int64_t* w, const int32_t* long_id, const uint32_t* tp, int T, const int64_t* C_rp,
                              int32_t* C_col, void* C_val, unsigned long long* counter, void* pscr, int64_t pscr_cap,
                              const int32_t* dtc, const int4* items, const int64_t* nitems, cudaStream_t s) {
    if (ndw <= 0) return cudaSuccess;
    const int smem = (int)sizeof(D2Smem);
    cudaError_t e = cudaMemsetAsync(counter, 0, sizeof(unsigned long long), s);  // item counter
    if (e != cudaSuccess) return e;
    const int grid = 148;  // persistent; CTAs beyond the item count exit at once
    if (A.dt == 0) {
        if ((e = cudaFuncSetAttribute(k_num_dense2<double>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
        SG_LAUNCH("k_num_dense", s, (k_num_dense2<double><<<grid, D2_T, smem, s>>>(A, B, heavy, rb, w, long_id, tp, T, C_rp, C_col,
                                                                                 (double*)C_val, counter, (D2Part*)pscr,
                                                                                 pscr_cap, dtc, items, nitems)));
    } else {
        if ((e = cudaFuncSetAttribute(k_num_dense2<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
        SG_LAUNCH("k_num_dense", s, (k_num_dense2<float><<<grid, D2_T, smem, s>>>(A, B, heavy, rb, w, long_id, tp, T, C_rp, C_col,
                                                                                (float*)C_val, counter, (D2Part*)pscr,
                                                                                pscr_cap, dtc, items, nitems)));
    }
#if defined(SG_D2_EXP) && SG_D2_EXP == 8
    {
        unsigned long long h[8] = {0};
        cudaStreamSynchronize(s);
        cudaMemcpyFromSymbol(h, g_d2_phase, sizeof(h));
        fprintf(stderr, "[d2 phases, Gcycles summed over warps] setup %.2f products %.2f barrier1 %.2f emission %.2f barrier2 %.2f item-fetch %.2f\n",
                h[0] / 1e9, h[1] / 1e9, h[2] / 1e9, h[3] / 1e9, h[4] / 1e9, h[5] / 1e9);
        unsigned long long z[8] = {0};
        cudaMemcpyToSymbol(g_d2_phase, z, sizeof(z));
    }
#endif
    return cudaGetLastError();
}

}  // namespace sg
