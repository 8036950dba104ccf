// sg_tile.cu — warp-owned column tiles for the SPARSE rank rows: heavy rows below the dense-window cut
// with at most KREG = 64 k entries ("more than t"; the row-row Gustavson product of
// L74 / Alg. 2 l.5-6, L222-L223). Rank rows with more k entries stay on the CTA rank kernel
// (sg_heavy.cu), whose block-wide flattening keeps all 16 warps busy on them.
//
// Same work items as the CTA rank kernel: the symbolic range plan, a range = one heavy row x a run of
// <= RW_TILES column tiles of TW columns. Here a range is ONE WARP's work item and the warp walks its
// tiles in order, owning everything it touches: the tile's TW-bit bitmap, its rank prefix and a
// CAPW-entry fp64 accumulator in the warp's private shared-memory slab. No two warps share an
// accumulator, so there are no block barriers between the phases (the CTA kernel pays ~6 K cycles of
// barrier-separated latency per range, DESIGN.md §7.1 — most of the cost of these rows' ranges, which
// hold only ~100-500 products) and the fp64 accumulate meets only intra-warp collisions.
//
// Per tile t: each lane holds the segments of up to two k entries (B rows) inside the tile, from carried
// cursors and the next tile's end prefetched one tile ahead (the tile pointer tp[id][t+1] of a long B row,
// the column at the cursor of a short one). The tile's products are flattened lane-major across the warp;
// the first round (NB batches of 32) is gathered WITH values and kept in registers, so tiles of at most
// 32*NB products read B once. Pass 1 ORs the columns into the bitmap; a warp scan of the 256 word
// popcounts gives the rank prefix and u_t; pass 2 accumulates a_ik*b_kj at rank(c) (the first arrival
// writes C.col[rank]); the accumulator leaves by coalesced stores. A tile with u_t > CAPW is accumulated
// in rank windows of CAPW (pass 2 repeated, products outside the window skipped).
#include "sg_device.cuh"
#include <cstdio>

namespace sg {

#ifndef SG_TT_WARPS
#define SG_TT_WARPS 4
#endif
#ifndef SG_TT_OCC
#define SG_TT_OCC 8
#endif
#ifndef SG_CAPW
#define SG_CAPW 512
#endif
#ifndef SG_TT_CHUNK
#define SG_TT_CHUNK 1
#endif
#ifndef SG_TT_NB
#define SG_TT_NB 3
#endif
constexpr int TT_WARPS = SG_TT_WARPS;  // warps per CTA (independent; the CTA only shares the launch)
constexpr int TT_T = 32 * TT_WARPS;
constexpr int TT_OCC = SG_TT_OCC;      // CTAs per SM (shared-memory bound)
constexpr int CAPW = SG_CAPW;          // accumulator entries per warp
constexpr int TT_CHUNK = SG_TT_CHUNK;  // range slots taken per counter increment
constexpr int NB = SG_TT_NB;           // batches of 32 products per round (the first round stays in registers)
#ifndef SG_KREG
#define SG_KREG 64
#endif
constexpr int KREG = SG_KREG;          // rows with at most KREG (<= 64) k entries (up to two per lane)
static_assert(KREG <= 64, "two k entries per lane at most");
constexpr int TWW = TW / 32;           // bitmap words per tile
static_assert(TWW == 8 * 32, "prefix layout: 8 words per lane");

#if defined(SG_TT_EXP)  // timing experiment: per-phase cycles summed over warps (lane 0)
__device__ unsigned long long g_tt[10];
#define TT_MARK(k) do { if (lane == 0) { const long long _t = clock64(); tph[k] += _t - tt_last; tt_last = _t; } } while (0)
#else
#define TT_MARK(k) do { } while (0)
#endif

struct __align__(16) TileWarp {
    double acc[CAPW];
    double av[KREG];      // a_ik of the range's row
    uint32_t bm[TWW];
    uint16_t pref[TWW];
};

// one k entry's cursor: B positions [cur, q1) still to come; q0 = start of the B row; lid = tile-pointer id
// (-1: short row); nx = the prefetched end information for the NEXT tile (long: tp[lid][t+1] of that tile;
// short: the column at cur, INT_MAX past the row end)
struct KCur {
    int cur, q0, q1, lid, nx;
};

__device__ __forceinline__ void kcur_init(const Mat& A, const Mat& B, int64_t s0, int i, int na, int t0,
                                          const int32_t* __restrict__ long_id, const uint32_t* __restrict__ tp,
                                          int T, KCur& k) {
    k.cur = k.q0 = k.q1 = 0;
    k.lid = -1;
    k.nx = INT_MAX;
    if (i >= na) return;
    const int kk = __ldg(A.col + s0 + i);
    k.q0 = (int)__ldg(B.rp + kk);
    k.q1 = (int)__ldg(B.rp + kk + 1);
    if (tp && k.q1 - k.q0 > LONG_ROW) k.lid = __ldg(long_id + kk);
    if (k.lid >= 0) {
        const uint32_t* tr = tp + (int64_t)k.lid * (T + 1);
        k.cur = k.q0 + (int)__ldg(tr + t0);
        k.nx = (int)__ldg(tr + t0 + 1);
    } else {
        k.cur = t0 == 0 ? k.q0 : (int)lower_bound_col(B.col, k.q0, k.q1, (int64_t)t0 * TW);
        k.nx = k.cur < k.q1 ? __ldg(B.col + k.cur) : INT_MAX;
    }
}

// end of the entry's segment in tile t (columns < hi); prefetches the next tile's information
__device__ __forceinline__ int kcur_end(const Mat& B, KCur& k, const uint32_t* __restrict__ tp, int T, int t,
                                        int64_t hi) {
    if (k.lid >= 0) {
        const int e = k.q0 + k.nx;
        if (t + 2 <= T) k.nx = (int)__ldg(tp + (int64_t)k.lid * (T + 1) + t + 2);
        return e;
    }
    int e = k.cur, c = k.nx;
    while (c < hi) {  // short row (<= LONG_ROW entries; or any row when B has no tile pointers)
        ++e;
        c = e < k.q1 ? __ldg(B.col + e) : INT_MAX;
    }
    k.nx = c;
    return e;
}

// Product j of the tile (0 <= j < tot): lane s holds products [off_s, off_s + l0_s + l1_s), the first l0_s
// from its k entry s (B positions b0_s..), the rest from its entry s + 32 (b1_s..). Returns the B position
// and the entry index (for a_ik).
template <bool TWO>
__device__ __forceinline__ int tile_pos(int j, int off, int b0, int l0, int b1, int& ki) {
    int s = 0;
    #pragma unroll
    for (int bb = 16; bb; bb >>= 1) {
        const int o = __shfl_sync(FULL, off, s + bb);
        if (o <= j) s += bb;
    }
    const int r = j - __shfl_sync(FULL, off, s);
    const int B0 = __shfl_sync(FULL, b0, s);
    if constexpr (!TWO) {
        ki = s;
        return B0 + r;
    } else {
        const int L0 = __shfl_sync(FULL, l0, s), B1 = __shfl_sync(FULL, b1, s);
        ki = r < L0 ? s : s + 32;
        return r < L0 ? B0 + r : B1 + (r - L0);
    }
}

// one round: batches [j0, j0 + 32 NB) -> c[r] (SEG_NONE past tot), v[r] = b_kj and ki[r] = the entry of a_ik
// if VAL (the product a_ik * b_kj is formed at the accumulation, so no instruction here waits on the loads)
template <bool TWO, bool VAL, class VT>
__device__ __forceinline__ void tile_round(const Mat& B, int j0, int tot, int off, int b0, int l0, int b1,
                                           int (&c)[NB], double (&v)[NB], int (&kix)[NB]) {
    const int lane = threadIdx.x & 31;
    const int32_t* __restrict__ bcol = B.col;
    const VT* __restrict__ bval = reinterpret_cast<const VT*>(B.val);
    #pragma unroll
    for (int r = 0; r < NB; ++r) {
        const int j = j0 + 32 * r + lane;
        int ki;
        const int q = tile_pos<TWO>(j, off, b0, l0, b1, ki);
        c[r] = SEG_NONE;
        v[r] = 0.0;
        kix[r] = ki;
        if (j < tot) {
            c[r] = __ldg(bcol + q);
            if (VAL) v[r] = (double)__ldg(bval + q);
        }
    }
}

template <class VT>
__global__ void __launch_bounds__(TT_T, TT_OCC) k_num_tile(
    Mat A, Mat B, const RangeRec* __restrict__ ranges, int64_t nslots, int64_t rb, const int32_t* __restrict__ long_id,
    const uint32_t* __restrict__ tp, int T, const int64_t* __restrict__ C_rp, int32_t* __restrict__ C_col,
    VT* __restrict__ C_val, unsigned long long* counter) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    TileWarp& S = reinterpret_cast<TileWarp*>(smem_raw)[wid];
    for (int q = lane; q < CAPW; q += 32) S.acc[q] = 0.0;
    for (int q = lane; q < TWW; q += 32) S.bm[q] = 0u;
    __syncwarp();
    const uint32_t a_acc = smem_addr(S.acc), a_bm = smem_addr(S.bm), a_pref = smem_addr(S.pref);
    const int64_t p = B.ncols;
#if defined(SG_TT_EXP)
    unsigned long long tph[10] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
    long long tt_last = clock64();
#endif
    while (true) {
        unsigned long long j0 = 0;
        if (lane == 0) j0 = atomicAdd(counter, (unsigned long long)TT_CHUNK);
        j0 = __shfl_sync(FULL, j0, 0);
        if ((int64_t)j0 >= nslots) break;
        for (int jj = 0; jj < TT_CHUNK; ++jj) {
            const int64_t slot = (int64_t)j0 + jj;
            if (slot >= nslots) break;
            const RangeRec R = ranges[slot];
            if (R.row < 0) continue;  // unused slot of the per-row bound
            const int64_t row = rb + R.row;
            const int64_t s0 = __ldg(A.rp + row);
            const int na = (int)(__ldg(A.rp + row + 1) - s0);
            if (na > KREG) continue;  // the CTA rank kernel's row
            int64_t out = C_rp[R.row] + R.off;
            TT_MARK(0);
            KCur k0, k1;
            kcur_init(A, B, s0, lane, na, R.t0, long_id, tp, T, k0);
            if (na > 32) kcur_init(A, B, s0, lane + 32, na, R.t0, long_id, tp, T, k1);
            else k1.cur = k1.q0 = k1.q1 = 0, k1.lid = -1, k1.nx = INT_MAX;
            S.av[lane] = lane < na ? ldv<VT>(A.val, s0 + lane) : 0.0;
            S.av[lane + 32] = lane + 32 < na ? ldv<VT>(A.val, s0 + lane + 32) : 0.0;
            __syncwarp();
            TT_MARK(1);
            // tile layout: lane segments (b0, l0), (b1, l1) and the lane-major flattening (off, tot)
            struct Lay { int b0, l0, b1, l1, off, tot; };
            auto layout = [&](int t) {
                const int64_t hi = min(p, (int64_t)(t + 1) * TW);
                Lay L;
                L.b0 = k0.cur;
                const int e0 = kcur_end(B, k0, tp, T, t, hi);
                L.l0 = e0 - k0.cur;
                k0.cur = e0;
                L.b1 = k1.cur;
                L.l1 = 0;
                if (na > 32) {
                    const int e1 = kcur_end(B, k1, tp, T, t, hi);
                    L.l1 = e1 - k1.cur;
                    k1.cur = e1;
                }
                SG_BOUND(L.l0 >= 0 && L.l1 >= 0 && k0.cur <= k0.q1 && k1.cur <= k1.q1);
                const int len = L.l0 + L.l1;
                const int inc = warp_incl_scan(len);
                L.tot = __shfl_sync(FULL, inc, 31);
                L.off = inc - len;
                return L;
            };
            auto round = [&](const Lay& L, int j0r, bool val, int (&c)[NB], double (&v)[NB], int (&kx)[NB]) {
                if (val) {
                    if (na > 32) tile_round<true, true, VT>(B, j0r, L.tot, L.off, L.b0, L.l0, L.b1, c, v, kx);
                    else tile_round<false, true, VT>(B, j0r, L.tot, L.off, L.b0, L.l0, L.b1, c, v, kx);
                } else {
                    if (na > 32) tile_round<true, false, VT>(B, j0r, L.tot, L.off, L.b0, L.l0, L.b1, c, v, kx);
                    else tile_round<false, false, VT>(B, j0r, L.tot, L.off, L.b0, L.l0, L.b1, c, v, kx);
                }
            };
            for (int t = R.t0; t < R.t1; ++t) {
                const Lay L = layout(t);
                int rc[NB], rk[NB];
                double rv[NB];
                round(L, 0, true, rc, rv, rk);
                const int64_t tlo = (int64_t)t * TW;
                // tlo is a multiple of 32: word (c - tlo) >> 5 = (c >> 5) - (tlo >> 5)
                const uint32_t bw = opaque_u32(a_bm - 4u * ((uint32_t)tlo >> 5));
                const uint32_t pw = opaque_u32(a_pref - 2u * ((uint32_t)tlo >> 5));
                auto setbit = [&](int32_t c) { red_or_s(bw + 4u * ((uint32_t)c >> 5), 1u << (c & 31)); };
                TT_MARK(2);
                // ---- pass 1: bitmap (the first round is in registers, later rounds gather columns only) ----
                #pragma unroll
                for (int r = 0; r < NB; ++r)
                    if (rc[r] != SEG_NONE) setbit(rc[r]);
                for (int j0r = 32 * NB; j0r < L.tot; j0r += 32 * NB) {
                    int c[NB], kx[NB];
                    double v[NB];
                    round(L, j0r, false, c, v, kx);
                    #pragma unroll
                    for (int r = 0; r < NB; ++r)
                        if (c[r] != SEG_NONE) setbit(c[r]);
                }
                __syncwarp();
                TT_MARK(3);
                // ---- rank prefix: lane owns words [4 lane, 4 lane + 4) and [128 + 4 lane, 128 + 4 lane + 4) (unit-stride
                // 16-byte accesses: no bank conflicts); one warp scan per half ----
                int ut;
                {
                    const uint4 w0 = reinterpret_cast<const uint4*>(S.bm)[lane];
                    const uint4 w1 = reinterpret_cast<const uint4*>(S.bm)[32 + lane];
                    const int c0 = __popc(w0.x), c1 = __popc(w0.y), c2 = __popc(w0.z), c3 = __popc(w0.w);
                    const int c4 = __popc(w1.x), c5 = __popc(w1.y), c6 = __popc(w1.z), c7 = __popc(w1.w);
                    const int s1 = c0 + c1 + c2 + c3, s2 = c4 + c5 + c6 + c7;
                    const int i1 = warp_incl_scan(s1), i2 = warp_incl_scan(s2);
                    const int t1 = __shfl_sync(FULL, i1, 31);
                    ut = t1 + __shfl_sync(FULL, i2, 31);
                    const int p0 = i1 - s1, p1 = p0 + c0, p2 = p1 + c1, p3 = p2 + c2;
                    const int p4 = t1 + i2 - s2, p5 = p4 + c4, p6 = p5 + c5, p7 = p6 + c6;
                    uint2* pr = reinterpret_cast<uint2*>(S.pref);
                    pr[lane] = make_uint2((uint32_t)p0 | ((uint32_t)p1 << 16), (uint32_t)p2 | ((uint32_t)p3 << 16));
                    pr[32 + lane] = make_uint2((uint32_t)p4 | ((uint32_t)p5 << 16), (uint32_t)p6 | ((uint32_t)p7 << 16));
                }
                SG_BOUND(out + ut <= C_rp[R.row + 1]);
                __syncwarp();
                TT_MARK(4);
                // ---- pass 2 (per rank window of CAPW): accumulate at rank(c); values out; clear ----
                for (int r0 = 0; r0 < ut; r0 += CAPW) {
                    const int64_t ob = out + r0;
                    auto acc = [&](int32_t c, double b, int ki) {
                        const double v = S.av[ki] * b;
                        const uint32_t cw = (uint32_t)c >> 5, bit = 1u << (c & 31);
                        const uint32_t wv = ld_u32_s(bw + 4u * cw);
                        const int rk = (int)ld_u16_s(pw + 2u * cw) + __popc(wv & (bit - 1u)) - r0;
                        if ((unsigned)rk < (unsigned)CAPW) {
                            // the first product of a column finds 0.0 and writes the column (a later one
                            // only if the partial sum is exactly 0.0: the same column again)
                            if (atom_add_f64_s(a_acc + 8u * (uint32_t)rk, v) == 0.0) st_out(C_col + ob + rk, c);
                        }
                    };
                    #pragma unroll
                    for (int r = 0; r < NB; ++r)
                        if (rc[r] != SEG_NONE) acc(rc[r], rv[r], rk[r]);
                    for (int j0r = 32 * NB; j0r < L.tot; j0r += 32 * NB) {
                        int c[NB], kx[NB];
                        double v[NB];
                        round(L, j0r, true, c, v, kx);
                        #pragma unroll
                        for (int r = 0; r < NB; ++r)
                            if (c[r] != SEG_NONE) acc(c[r], v[r], kx[r]);
                    }
                    __syncwarp();
                    TT_MARK(5);
                    const int n = min(CAPW, ut - r0);
                    for (int q = lane; q < n; q += 32) {
                        st_out(C_val + ob + q, (VT)S.acc[q]);
                        S.acc[q] = 0.0;
                    }
                    __syncwarp();
                }
                {
                    uint4* bm4 = reinterpret_cast<uint4*>(S.bm);
                    bm4[lane] = make_uint4(0, 0, 0, 0);
                    bm4[32 + lane] = make_uint4(0, 0, 0, 0);
                }
                out += ut;
                __syncwarp();
                TT_MARK(6);
#if defined(SG_TT_EXP)
                if (lane == 0) { tph[8] += ut; tph[9] += 1; }
#endif
            }
            SG_BOUND(out == C_rp[R.row] + R.off + R.cnt);  // the range holds exactly the plan's entries
#if defined(SG_TT_EXP)
            if (lane == 0) tph[7] += 1;
#endif
        }
    }
#if defined(SG_TT_EXP)
    if (lane == 0)
        for (int q = 0; q < 10; ++q) atomicAdd(&g_tt[q], tph[q]);
#endif
}

cudaError_t launch_num_tile(const Mat& A, const Mat& B, const RangeRec* ranges, int64_t nslots, int64_t rb,
                            const int32_t* long_id, const uint32_t* tp, int T, const int64_t* C_rp, int32_t* C_col,
                            void* C_val, unsigned long long* counter, cudaStream_t s) {
    if (nslots <= 0) return cudaSuccess;
    const int smem = (int)sizeof(TileWarp) * TT_WARPS;
    cudaError_t e = cudaMemsetAsync(counter, 0, sizeof(unsigned long long), s);
    if (e != cudaSuccess) return e;
    const int grid = TT_OCC * 148;
    if (A.dt == 0) {
        if ((e = cudaFuncSetAttribute(k_num_tile<double>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
        SG_LAUNCH("k_num_tile", s, (k_num_tile<double><<<grid, TT_T, smem, s>>>(A, B, ranges, nslots, rb, long_id, tp, T, C_rp,
                                                                             C_col, (double*)C_val, counter)));
    } else {
        if ((e = cudaFuncSetAttribute(k_num_tile<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
        SG_LAUNCH("k_num_tile", s, (k_num_tile<float><<<grid, TT_T, smem, s>>>(A, B, ranges, nslots, rb, long_id, tp, T, C_rp,
                                                                            C_col, (float*)C_val, counter)));
    }
#if defined(SG_TT_EXP)
    {
        unsigned long long h[10];
        cudaStreamSynchronize(s);
        cudaMemcpyFromSymbol(h, g_tt, sizeof(h));
        fprintf(stderr, "[tile phases, Gcycles over warps] fetch %.2f kinit %.2f | kend+scan %.2f pass1 %.2f prefix %.2f pass2 %.2f"
                " emit %.2f | ranges %llu outputs %llu tiles %llu\n",
                h[0] / 1e9, h[1] / 1e9, h[2] / 1e9, h[3] / 1e9, h[4] / 1e9, h[5] / 1e9, h[6] / 1e9, h[7], h[8], h[9]);
        unsigned long long z[10] = {0};
        cudaMemcpyToSymbol(g_tt, z, sizeof(z));
    }
#endif
    return cudaGetLastError();
}

int64_t tile_kreg() { return KREG; }

}  // namespace sg
