// sg_device.cuh — device helpers shared by the libsg kernels: warp primitives, group barriers,
// the flattened product iterator and the order-preserving hash accumulator.
#pragma once
#include "sg_internal.cuh"
#include <climits>

// Bounds assertions of a debug build (-DSG_DEBUG_BOUNDS, tools/ab_builds / the GPU tests with SG_LIB_PATH):
// every kernel's output count per row / range against the symbolic plan, cursor and rank ranges. A failed
// assert traps the kernel, so the call returns SG_ERR_CUDA and the test fails. Compiled out by default.
#if defined(SG_DEBUG_BOUNDS)
#include <cassert>
#define SG_BOUND(cond) assert(cond)
#else
#define SG_BOUND(cond) do { } while (0)
#endif

namespace sg {

constexpr unsigned FULL = 0xffffffffu;

template <class T> __device__ __forceinline__ T warp_sum(T v) {
    #pragma unroll
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
    return v;
}
__device__ __forceinline__ int warp_min(int v) {
    #pragma unroll
    for (int o = 16; o; o >>= 1) v = min(v, __shfl_xor_sync(FULL, v, o));
    return v;
}
__device__ __forceinline__ int warp_max(int v) {
    #pragma unroll
    for (int o = 16; o; o >>= 1) v = max(v, __shfl_xor_sync(FULL, v, o));
    return v;
}
template <class T> __device__ __forceinline__ T warp_incl_scan(T v) {
    const int lane = threadIdx.x & 31;
    #pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T y = __shfl_up_sync(FULL, v, o);
        if (lane >= o) v += y;
    }
    return v;
}
__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// C is written once and never re-read by the kernels: streaming stores (st.global.cs, evict-first
// in L2) keep the 116 GB output stream from evicting B, the operand every product gathers.
#ifndef SG_STCS
#define SG_STCS 1
#endif
template <class T> __device__ __forceinline__ void st_out(T* p, T v) {
#if SG_STCS
    __stcs(p, v);
#else
    *p = v;
#endif
}

// ---- 32-bit shared-window addressing for the hot accumulators --------------------------------------
// Taking &S.x[i] of dynamic shared memory yields a GENERIC pointer; under the 64-register cap of
// 1024-thread CTAs the compiler then re-derives the shared window base (S2R SR_CgaCtaId + LEA) at every
// product. A 32-bit .shared address computed once keeps the accumulate at LDS/ATOMS [reg].
__device__ __forceinline__ uint32_t opaque_u32(uint32_t x) {
    uint32_t a;
    asm volatile("mov.b32 %0, %1;" : "=r"(a) : "r"(x));
    return a;
}
__device__ __forceinline__ uint32_t smem_addr(const void* p) {
    // opaque to the optimizer: held in a register instead of being re-derived from SR_CgaCtaId per use
    uint32_t a;
    asm volatile("mov.b32 %0, %1;" : "=r"(a) : "r"((uint32_t)__cvta_generic_to_shared(p)));
    return a;
}
__device__ __forceinline__ double atom_add_f64_s(uint32_t a, double v) {
    double old;
    asm volatile("atom.shared.add.f64 %0, [%1], %2;" : "=d"(old) : "r"(a), "d"(v) : "memory");
    return old;
}
// The same two accumulator atomics WITHOUT a compiler memory clobber: global loads may be scheduled
// across them (software pipelining of the B gathers). Only for accumulators whose plain shared reads
// and writes are all separated from the atomics by __syncthreads().
__device__ __forceinline__ double atom_add_f64_s_nc(uint32_t a, double v) {
    double old;
    asm volatile("atom.shared.add.f64 %0, [%1], %2;" : "=d"(old) : "r"(a), "d"(v));
    return old;
}
__device__ __forceinline__ void red_or_s_nc(uint32_t a, uint32_t v) {
    asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(a), "r"(v));
}
__device__ __forceinline__ void red_or_s(uint32_t a, uint32_t v) {
    asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_u32_s(uint32_t a) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
    return v;
}
__device__ __forceinline__ double ld_f64_s(uint32_t a) {
    double v;
    asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a) : "memory");
    return v;
}
__device__ __forceinline__ uint32_t ld_u16_s(uint32_t a) {
    uint16_t v;
    asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a) : "memory");
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

// ---- groups: G threads own one row (G = 32: a warp; G = BLK: the block; else named barriers) ----
template <int G, int BLK> __device__ __forceinline__ void group_bar() {
    if constexpr (G == 32) __syncwarp();
    else if constexpr (G == BLK) __syncthreads();
    else {
        const int g = threadIdx.x / G;
        asm volatile("bar.sync %0, %1;" ::"r"(1 + g), "r"(G) : "memory");
    }
}

// ---- flattened products of up to 32 consecutive A entries [pa0, pa1) of one row -------------------
// Lane l loads k_l = A.col[pa0 + l] and its B-row segment; an exclusive scan of the segment lengths
// flattens the products so that every lane gathers an independent (col, val) per round, UNR rounds
// in flight (memory-level parallelism instead of one dependent chain per k).
// seg(k, q0, len) may narrow the segment (heavy ranges); f(c, v) consumes a product.
template <bool VAL, class VT, int UNR, class SEG, class F>
__device__ __forceinline__ void chunk_products(const Mat& A, const Mat& B, int64_t pa0, int64_t pa1, SEG&& seg,
                                               F&& f) {
    const int lane = threadIdx.x & 31;
    const int64_t pa = pa0 + lane;
    int len = 0;
    int64_t q0 = 0;
    double a = 0.0;
    if (pa < pa1) {
        const int k = __ldg(A.col + pa);
        q0 = __ldg(B.rp + k);
        len = (int)(__ldg(B.rp + k + 1) - q0);
        if (VAL) a = ldv<VT>(A.val, pa);
        seg(k, q0, len);
    }
    const int inc = warp_incl_scan(len);
    const int off = inc - len;
    const int tot = __shfl_sync(FULL, inc, 31);
    for (int j0 = 0; j0 < tot; j0 += 32 * UNR) {
        int c[UNR];
        double v[UNR];
        #pragma unroll
        for (int r = 0; r < UNR; ++r) {
            const int j = j0 + 32 * r + lane;
            int s = 0;
            #pragma unroll
            for (int b = 16; b; b >>= 1) {
                const int o = __shfl_sync(FULL, off, s + b);
                if (o <= j) s += b;
            }
            const int64_t q = __shfl_sync(FULL, q0, s) + (j - __shfl_sync(FULL, off, s));
            const double as = VAL ? __shfl_sync(FULL, a, s) : 0.0;
            c[r] = -1;
            if (j < tot) {
                c[r] = __ldg(B.col + q);
                if (VAL) v[r] = as * ldv<VT>(B.val, q);
            }
        }
        #pragma unroll
        for (int r = 0; r < UNR; ++r)
            if (c[r] >= 0) f(c[r], VAL ? v[r] : 0.0);
    }
}

// ---- the order-preserving hash accumulator -----------------------------------------------------
// home(c) = identity (c - lo) when the span fits the table, else floor((c - lo) * mult / 2^32),
// monotone in c; linear probing moves forward only, never wraps (overflow room >= capacity).
// Returns the slot used.
__device__ __forceinline__ int acc_insert(int32_t* keys, double* vals, int32_t c, double v, uint32_t d, bool ident,
                                          uint64_t mult) {
    uint32_t h;
    if (ident) {
        h = d;
        // every writer of slot d stores the same key c into a slot that starts at EMPTY_KEY (-1, all bits
        // set): an atomic AND installs it race-free (a native shared atomic; compute-sanitizer racecheck
        // flagged the earlier plain idempotent store, profiles/r02_sanitizer_racecheck.log)
        atomicAnd(&keys[h], c);
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
    return (int)h;
}

// Group-wide emission of slots [0, nslots) in slot order into C at `base`, clearing each slot.
// Each warp of the group owns a contiguous chunk of slots; one group-level exclusive scan of the
// per-warp counts places the chunks (ws: >= G/32 ints of shared memory per group).
template <int G, int BLK, class VT>
__device__ __forceinline__ void emit_slots(int32_t* keys, double* vals, int nslots, int64_t base,
                                           int32_t* __restrict__ C_col, VT* __restrict__ C_val, int* ws,
                                           bool ranked) {
    constexpr int NW = G / 32;
    const int lane = threadIdx.x & 31;
    const int w = (threadIdx.x % G) / 32;
    const int chunk = ((nslots + NW - 1) / NW + 31) & ~31;
    const int s_lo = w * chunk, s_hi = min(nslots, s_lo + chunk);
    int64_t pos = base;
    if constexpr (NW > 1) {
        int cnt = 0;
        for (int s0 = s_lo; s0 < s_hi; s0 += 32) {
            const int s = s0 + lane;
            cnt += __popc(__ballot_sync(FULL, s < s_hi && keys[s] != EMPTY_KEY));
        }
        if (lane == 0) ws[w] = cnt;
        group_bar<G, BLK>();
        for (int q = 0; q < w; ++q) pos += ws[q];
        group_bar<G, BLK>();
    }
    if (!ranked) {  // slot order is column order (identity map or runs already sorted)
        for (int s0 = s_lo; s0 < s_hi; s0 += 32) {
            const int s = s0 + lane;
            const int32_t k = s < s_hi ? keys[s] : EMPTY_KEY;
            const unsigned m = __ballot_sync(FULL, k != EMPTY_KEY);
            if (k != EMPTY_KEY) {
                const int64_t o = pos + __popc(m & lanemask_lt());
                st_out(C_col + o, k);
                st_out(C_val + o, (VT)vals[s]);
                keys[s] = EMPTY_KEY;
                vals[s] = 0.0;
            }
            pos += __popc(m);
        }
        return;
    }
    // Order-preserving hash: runs (maximal occupied stretches) are mutually ordered but not sorted
    // inside. The entry in slot s goes to (#occupied slots before its run) + (its rank inside the
    // run): found from the occupancy ballot plus a short scan of the run's keys — no data movement.
    for (int s0 = s_lo; s0 < s_hi; s0 += 32) {
        const int s = s0 + lane;
        const int32_t k = s < s_hi ? keys[s] : EMPTY_KEY;
        const unsigned m = __ballot_sync(FULL, k != EMPTY_KEY);
        if (k != EMPTY_KEY) {
            const unsigned below = ~m & lanemask_lt();
            int rs;
            if (below) rs = s0 + 31 - __clz(below) + 1;
            else { rs = s0; while (rs > 0 && keys[rs - 1] != EMPTY_KEY) --rs; }
            const unsigned above = lane == 31 ? 0u : (~m & (~0u << (lane + 1)));
            int re;
            if (above) re = s0 + __ffs(above) - 1;
            else { re = s0 + 32; while (re < nslots && keys[re] != EMPTY_KEY) ++re; }
            int rank = 0;
            for (int j = rs; j < re; ++j) rank += keys[j] < k;
            const int64_t o = pos + __popc(m & lanemask_lt()) - (s - rs) + rank;
            st_out(C_col + o, k);
            st_out(C_val + o, (VT)vals[s]);
        }
        pos += __popc(m);
    }
    group_bar<G, BLK>();  // every rank computed before any slot is cleared
    for (int s = s_lo + lane; s < s_hi; s += 32)
        if (keys[s] != EMPTY_KEY) { keys[s] = EMPTY_KEY; vals[s] = 0.0; }
}

// ---- occupancy-driven emission of the light accumulator ------------------------------------------
// acc_insert with an occupancy bitmap: the product that installs a key in an empty slot also sets the
// slot's bit (one native 32-bit shared atomic per distinct column), so that emission visits the
// occupied slots only instead of scanning every slot of the table.
__device__ __forceinline__ int acc_insert_occ(int32_t* keys, double* vals, uint32_t* occ, int32_t c, double v, uint32_t d,
                                              bool ident, uint64_t mult) {
    uint32_t h;
    if (ident) {
        h = d;
        if (atomicAnd(&keys[h], c) == EMPTY_KEY) atomicOr(&occ[h >> 5], 1u << (h & 31));  // see acc_insert
    } else {
        h = (uint32_t)(((uint64_t)d * mult) >> 32);
        while (true) {
            int32_t old = keys[h];
            if (old == c) break;
            if (old == EMPTY_KEY) {
                old = atomicCAS(&keys[h], EMPTY_KEY, c);
                if (old == EMPTY_KEY) { atomicOr(&occ[h >> 5], 1u << (h & 31)); break; }
                if (old == c) break;
            }
            ++h;
        }
    }
    atomicAdd(&vals[h], v);
    return (int)h;
}

// index of the r-th (0-based) set bit of m (r < popc(m)), by popcount bisection
__device__ __forceinline__ int select_bit(uint32_t m, int r) {
    int pos = 0;
    #pragma unroll
    for (int sh = 16; sh; sh >>= 1) {
        const int c = __popc(m & ((1u << sh) - 1u));
        if (r >= c) { r -= c; m >>= sh; pos += sh; }
    }
    return pos;
}

// ---- block-level product flattening (heavy path; light rows with U >= 1024) ----------------------
__device__ __forceinline__ int64_t lower_bound_col(const int32_t* __restrict__ col, int64_t lo, int64_t hi, int64_t x) {
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if ((int64_t)__ldg(col + mid) < x) lo = mid + 1; else hi = mid;
    }
    return lo;
}

// exclusive scan of one int per thread over a 1024-thread block; *total for everyone
// Exclusive scan of one value per thread over an NT-thread block with ONE barrier: warp totals go
// to ws, then every warp re-scans the (<= 32) warp totals itself. ws must not be rewritten until
// the caller has passed another __syncthreads (call sites alternate between distinct ws arrays).
template <int NT, class T>
__device__ __forceinline__ T block_scan1(T v, T* total, T* ws) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const T inc = warp_incl_scan(v);
    if (lane == 31) ws[wid] = inc;
    __syncthreads();
    const T x = lane < NT / 32 ? ws[lane] : T(0);
    const T xi = warp_incl_scan(x);
    *total = __shfl_sync(FULL, xi, 31);
    return __shfl_sync(FULL, xi - x, wid) + inc - v;
}
template <int NT>
__device__ __forceinline__ int block_scan(int v, int* total, int* ws) { return block_scan1<NT, int>(v, total, ws); }

// Two exclusive scans (an int and a long long per thread) sharing ONE barrier (same ws rule as
// block_scan1 for both ws arrays).
template <int NT>
__device__ __forceinline__ void block_scan2(int v1, long long v2, int* ex1, int* tot1, long long* ex2, long long* tot2,
                                            int* ws1, long long* ws2) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int i1 = warp_incl_scan(v1);
    const long long i2 = warp_incl_scan(v2);
    if (lane == 31) { ws1[wid] = i1; ws2[wid] = i2; }
    __syncthreads();
    const int x1 = lane < NT / 32 ? ws1[lane] : 0;
    const long long x2 = lane < NT / 32 ? ws2[lane] : 0LL;
    const int y1 = warp_incl_scan(x1);
    const long long y2 = warp_incl_scan(x2);
    *tot1 = __shfl_sync(FULL, y1, 31);
    *tot2 = __shfl_sync(FULL, y2, 31);
    *ex1 = __shfl_sync(FULL, y1 - x1, wid) + i1 - v1;
    *ex2 = __shfl_sync(FULL, y2 - x2, wid) + i2 - v2;
}

// largest i in [0, nk) with off[i] <= j (that entry has len > 0)
__device__ __forceinline__ int find_k(const int* off, int nk, int j) {
    int lo = 0, hi = nk - 1;
    while (lo < hi) {
        int mid = (lo + hi + 1) >> 1;
        if (off[mid] <= j) lo = mid; else hi = mid - 1;
    }
    return lo;
}

template <int NT>
__device__ __forceinline__ long long block_scan_ll(long long v, long long* total, long long* ws) {
    return block_scan1<NT, long long>(v, total, ws);
}

// Group-wide emission of the occupied slots of [0, nslots) (bits of occ) in slot order into C at
// `base`; clears the slots and the bits. wp: >= ceil(nslots/32) + 1 ints of group-private shared
// memory (word prefix), ws: >= G/32 ints (block scan). Entry e (the e-th occupied slot, s) goes to
// e when slot order is column order (identity map), else (ranked: order-preserving hash, runs mutually
// ordered but not sorted inside) to e - (s - run start) + (its rank inside the run).
template <int G, int BLK, class VT>
__device__ __forceinline__ void emit_occ(int32_t* keys, double* vals, uint32_t* occ, int* wp, int nslots, int64_t base,
                                         int32_t* __restrict__ C_col, VT* __restrict__ C_val, int* ws, bool ranked) {
    const int t = threadIdx.x % G, lane = threadIdx.x & 31;
    const int W = (nslots + 31) >> 5;
    int u;
    if constexpr (G == 32) {
        int carry = 0;
        for (int w0 = 0; w0 < W; w0 += 32) {
            const int w = w0 + lane;
            const int c = w < W ? __popc(occ[w]) : 0;
            const int inc = warp_incl_scan(c);
            if (w < W) wp[w] = carry + inc - c;
            carry += __shfl_sync(FULL, inc, 31);
        }
        u = carry;
        if (lane == 0) wp[W] = u;
        __syncwarp();
    } else {
        // W <= G: one word per thread (P / 32 <= G for the block bins)
        const int c = t < W ? __popc(occ[t]) : 0;
        int tot;
        const int ex = block_scan<G>(c, &tot, ws);
        if (t < W) wp[t] = ex;
        if (t == 0) wp[W] = tot;
        u = tot;
        group_bar<G, BLK>();
    }
    for (int e0 = t - lane; e0 < u; e0 += G) {
        const int e = e0 + lane;
        if (e < u) {
            int lo = 0, hi = W - 1;  // largest w with wp[w] <= e (that word holds entry e)
            while (lo < hi) {
                const int mid = (lo + hi + 1) >> 1;
                if (wp[mid] <= e) lo = mid; else hi = mid - 1;
            }
            const uint32_t m = occ[lo];
            const int bit = select_bit(m, e - wp[lo]);
            const int s = 32 * lo + bit;
            const int32_t k = keys[s];
            int o = e;
            if (ranked) {
                int rs, re;
                const uint32_t below = ~m & ((1u << bit) - 1u);
                if (below) rs = 32 * lo + (31 - __clz(below)) + 1;
                else {
                    int ww = lo - 1;
                    while (ww >= 0 && occ[ww] == 0xFFFFFFFFu) --ww;
                    rs = ww < 0 ? 0 : 32 * ww + (31 - __clz(~occ[ww])) + 1;
                }
                const uint32_t above = bit == 31 ? 0u : (~m & (~0u << (bit + 1)));
                if (above) re = 32 * lo + __ffs(above) - 1;
                else {
                    int ww = lo + 1;
                    while (ww < W && occ[ww] == 0xFFFFFFFFu) ++ww;
                    re = ww >= W ? 32 * W : 32 * ww + __ffs(~occ[ww]) - 1;
                }
                if (re - rs > 1) {
                    int rank = 0;
                    for (int j = rs; j < re; ++j) rank += keys[j] < k;
                    o = e - (s - rs) + rank;
                }
            }
            st_out(C_col + base + o, k);
            st_out(C_val + base + o, (VT)vals[s]);
        }
    }
    group_bar<G, BLK>();  // every rank computed before any slot is cleared
    for (int w = t; w < W; w += G) {
        uint32_t m = occ[w];
        while (m) {
            const int b = __ffs(m) - 1;
            m &= m - 1u;
            keys[32 * w + b] = EMPTY_KEY;
            vals[32 * w + b] = 0.0;
        }
        occ[w] = 0u;
    }
}

// First packed entry of every warp's product slice (see SliceCursor): written by the entry whose
// product range contains the slice start, so no warp binary-searches the packed offsets.
__shared__ int sg_wstart[32];

// slice length per warp for tot products over NW warps (a multiple of 32; SliceCursor uses the same)
__device__ __forceinline__ int slice_per(int tot, int NW) { return (((tot + NW - 1) / NW) + 31) & ~31; }

// entry ci holds products [o, o + len) of a packing with tot products: mark the slices starting inside
template <int NT>
__device__ __forceinline__ void mark_slice_starts(int ci, int o, int len, int tot) {
    constexpr int NW = NT / 32;
    const int per = slice_per(tot, NW);
    if (len <= 0 || per <= 0) return;
    for (int w = (o + per - 1) / per; w < NW && w * per < o + len; ++w) sg_wstart[w] = ci;
}

// One chunk of k entries (one per thread): pack the entries with len > 0, in order, into
// s_beg / s_off (exclusive prefix of len) / s_a; returns the chunk's product count, *nk = packed.
template <int NT, class BEG>
__device__ __forceinline__ int chunk_compact(int len, BEG beg, double a, BEG* s_beg, int* s_off, double* s_a, int* nk,
                                             long long* wsll) {
    long long tot;
    const long long ex = block_scan_ll<NT>(((long long)len << 16) | (len > 0 ? 1 : 0), &tot, wsll);
    if (len > 0) {
        const int ci = (int)(ex & 0xFFFF);
        s_beg[ci] = beg;
        s_off[ci] = (int)(ex >> 16);
        if (s_a) s_a[ci] = a;
        mark_slice_starts<NT>(ci, (int)(ex >> 16), len, (int)(tot >> 16));
    }
    *nk = (int)(tot & 0xFFFF);
    __syncthreads();
    return (int)(tot >> 16);
}

// Products [0, tot) of a packed chunk, split into one contiguous slice per warp (a multiple of 32).
// Within a slice a batch of 32 consecutive products lies in at most 32 consecutive packed entries
// (each has len >= 1), so every lane finds its entry with a 5-step shuffle search (or none: the
// fast path when the batch lies inside one long B segment).
template <int NT, bool VAL, class VT, class BEG>
struct SliceCursor {
    static_assert(sizeof(BEG) == 4 || sizeof(BEG) == 8, "segment begin: int32 or int64");
    // 32-bit shared addresses of the packed chunk arrays (see smem_addr)
    // one opaque base register; the other arrays sit at constant byte distances from it
    uint32_t a_beg, d_off, d_a;
    int nk, tot, j_lo, j_hi, i0;
    __device__ __forceinline__ BEG beg_at(int i) const {
        if constexpr (sizeof(BEG) == 4) return (BEG)(int32_t)ld_u32_s(a_beg + 4u * (uint32_t)i);
        else {
            int64_t v;
            asm volatile("ld.shared.s64 %0, [%1];" : "=l"(v) : "r"(a_beg + 8u * (uint32_t)i) : "memory");
            return (BEG)v;
        }
    }
    __device__ __forceinline__ int off_at(int i) const { return (int)ld_u32_s(a_beg + d_off + 4u * (uint32_t)i); }
    __device__ __forceinline__ double a_at(int i) const { return ld_f64_s(a_beg + d_a + 8u * (uint32_t)i); }
    __device__ __forceinline__ SliceCursor(const BEG* sb, const int* so, const double* sa, int nk_, int tot_)
        : nk(nk_), tot(tot_) {
        constexpr int NW = NT / 32;
        a_beg = smem_addr(sb);
        d_off = (uint32_t)((const char*)so - (const char*)sb);
        d_a = sa ? (uint32_t)((const char*)sa - (const char*)sb) : 0u;
        const int wid = threadIdx.x >> 5;
        const int per = slice_per(tot, NW);
        j_lo = wid * per;
        j_hi = min(tot, j_lo + per);
        i0 = j_lo < j_hi ? sg_wstart[wid] : 0;  // written by the packing (chunk_compact)
    }
    // batch [j0, j0 + 32): lane's (column, a_ik * b_kj), c = -1 beyond the slice
    __device__ __forceinline__ void fetch(const Mat& B, int j0, int& c, double& v) { fetchv<VAL>(B, j0, c, v); }
    template <bool V>
    __device__ __forceinline__ void fetchv(const Mat& B, int j0, int& c, double& v) {
        const int lane = threadIdx.x & 31;
        const int e0 = i0 + 1 < nk ? off_at(i0 + 1) : tot;
        if (j0 + 31 < e0) {  // fast path: the whole batch lies inside entry i0 (hub rows of B)
            const int j = j0 + lane;
            c = -1;
            v = 0.0;
            if (j < j_hi) {
                const int64_t q = (int64_t)beg_at(i0) + (j - off_at(i0));
                c = __ldg(B.col + q);
                if (V) v = a_at(i0) * ldv<VT>(B.val, q);
            }
            return;
        }
        const int ii = i0 + lane;
        const int o = ii < nk ? off_at(ii) : INT_MAX;
        const int j = j0 + lane;
        int s = 0;
        #pragma unroll
        for (int b = 16; b; b >>= 1) {
            const int ob = __shfl_sync(FULL, o, s + b);
            if (ob <= j) s += b;
        }
        const int kk = i0 + s;
        const int os = __shfl_sync(FULL, o, s);
        c = -1;
        v = 0.0;
        if (j < j_hi) {
            const int64_t q = (int64_t)beg_at(kk) + (j - os);
            c = __ldg(B.col + q);
            if (V) v = a_at(kk) * ldv<VT>(B.val, q);
        }
        i0 = __shfl_sync(FULL, kk, 31);
    }
};

// Streams the warp's slice from product j_start on (sc.i0 = the packed entry holding j_start) through
// f, four batches in flight (fetch(j + 96) is issued before batch j is consumed). f is called by every
// lane (c < 0: no product) so it may use warp collectives. V: fetch values too.
template <bool V, int NT, bool VAL, class VT, class BEG, class F>
__device__ __forceinline__ void warp_slice_from(SliceCursor<NT, VAL, VT, BEG>& sc, int j_start, const Mat& B, F&& f) {
    const int j_hi = sc.j_hi;
    if (j_start >= j_hi) return;
    int c0, c1, c2, c3;
    double v0, v1, v2, v3;
    sc.template fetchv<V>(B, j_start, c0, v0);
    sc.template fetchv<V>(B, j_start + 32, c1, v1);
    sc.template fetchv<V>(B, j_start + 64, c2, v2);
    for (int j0 = j_start; j0 < j_hi; j0 += 128) {
        sc.template fetchv<V>(B, j0 + 96, c3, v3);
        f(c0, v0);
        if (j0 + 128 >= j_hi) { f(c1, v1); f(c2, v2); f(c3, v3); break; }
        sc.template fetchv<V>(B, j0 + 128, c0, v0);
        f(c1, v1);
        sc.template fetchv<V>(B, j0 + 160, c1, v1);
        f(c2, v2);
        sc.template fetchv<V>(B, j0 + 192, c2, v2);
        f(c3, v3);
    }
}
template <int NT, bool VAL, class VT, class BEG, class F>
__device__ __forceinline__ void warp_slice(const BEG* s_beg, const int* s_off, const double* s_a, int nk, int tot,
                                           const Mat& B, F&& f) {
    SliceCursor<NT, VAL, VT, BEG> sc(s_beg, s_off, s_a, nk, tot);
    warp_slice_from<VAL>(sc, sc.j_lo, B, f);
}

// The first four batches of the warp's slice fetched into registers (columns AND values) — a two-pass
// consumer (bitmap, then rank accumulation) then re-reads B only for the rest of its slice, from the
// returned cursor entry on (see warp_slice_rest).
template <int NT, class VT, class BEG>
__device__ __forceinline__ int warp_slice_head(const BEG* s_beg, const int* s_off, const double* s_a, int nk, int tot,
                                               const Mat& B, int (&c)[4], double (&v)[4]) {
    SliceCursor<NT, true, VT, BEG> sc(s_beg, s_off, s_a, nk, tot);
    #pragma unroll
    for (int r = 0; r < 4; ++r) {
        c[r] = -1;
        v[r] = 0.0;
        if (sc.j_lo + 32 * r < sc.j_hi) sc.fetch(B, sc.j_lo + 32 * r, c[r], v[r]);
    }
    return sc.i0;
}
// Products [j_lo + 128, j_hi) of the warp's slice (after warp_slice_head; i0 = its return value).
template <bool V, int NT, class VT, class BEG, class F>
__device__ __forceinline__ void warp_slice_rest(const BEG* s_beg, const int* s_off, const double* s_a, int nk, int tot,
                                                int i0, const Mat& B, F&& f) {
    SliceCursor<NT, V, VT, BEG> sc(s_beg, s_off, s_a, nk, tot);
    sc.i0 = i0;
    warp_slice_from<V>(sc, sc.j_lo + 128, B, f);
}

// Segment of one k entry for tiles [.., t1) starting at its cursor: long B rows read the tile
// pointer (prefetched `tpv`), short rows (<= LONG_ROW entries) count their entries below hi with
// independent loads. Returns the new cursor.
__device__ __forceinline__ int seg_end(const Mat& B, int cur, int e1, int q0, bool is_long, uint32_t tpv, int64_t hi) {
    if (is_long) return q0 + (int)tpv;
    int n = 0;
    #pragma unroll
    for (int q = 0; q < LONG_ROW; ++q)
        if (cur + q < e1 && __ldg(B.col + cur + q) < hi) ++n;
    return cur + n;
}


// ---- per-warp product slices ("parts"; sg_dense2.cu, sg_sym2.cu) --------------------------------
// A row's products [0, L) (L = w_i = sum of its B row lengths, in A-column order) are cut into NW
// equal contiguous slices, one per warp; warp w owns products [bw(w), bw(w+1)), bw(w) = floor(L w/NW).
// A PART is one warp's share of one k entry: B_k[cur .. end). Parts are ordered by (k, warp), so each
// warp's parts are contiguous; wpart[w] = first part of warp w, wpart[NW] = number of parts (<= na + NW).
struct Part {
    int32_t cur, end;  // B positions still to come
    int32_t q0, lid;   // start of the B row; its tile-pointer id (-1: short row, <= LONG_ROW entries)
    double a;          // a_ik (0 for structure-only walks)
};

template <int NW> __device__ __forceinline__ int part_warp_of(long long x, long long L) {
    int w = (int)((x * NW) / L);
    while (w < NW - 1 && (L * (w + 1)) / NW <= x) ++w;  // one step unless L < NW
    return w;
}

// Block-wide (NT threads): builds the parts of row (s0, na) into P / wpart. Cursors start at the
// first entry with column >= lo0 (tile tlo = lo0 / TW of the tile pointers; lo0 = 0 for a whole row).
template <int NT, class VT, bool WITH_A>
__device__ __forceinline__ void build_parts(const Mat& A, const Mat& B, int64_t s0, int na, long long L,
                                            const int32_t* __restrict__ long_id, const uint32_t* __restrict__ tp,
                                            int T, int tlo, int64_t lo0, Part* P, int32_t* wpart, long long* wsll,
                                            int* ws) {
    constexpr int NW = NT / 32;
    const int tid = threadIdx.x;
    for (int w = tid; w <= NW; w += NT) wpart[w] = -1;
    long long carry_p = 0;
    int carry_n = 0;
    for (int c0 = 0; c0 < na; c0 += NT) {
        const int i = c0 + tid;
        int len = 0, q0 = 0, lid = -1;
        double a = 0.0;
        if (i < na) {
            const int k = __ldg(A.col + s0 + i);
            q0 = (int)__ldg(B.rp + k);
            len = (int)(__ldg(B.rp + k + 1) - q0);
            if (WITH_A) a = ldv<VT>(A.val, s0 + i);
            if (len > LONG_ROW && tp) lid = __ldg(long_id + k);
        }
        long long tot;
        const long long ex = block_scan_ll<NT>((long long)len, &tot, wsll) + carry_p;  // (barrier inside)
        int wf = 0, wl = -1;
        if (len > 0) {
            wf = part_warp_of<NW>(ex, L);
            wl = part_warp_of<NW>(ex + len - 1, L);
        }
        int ntot;
        const int po = block_scan1<NT, int>(wl - wf + 1, &ntot, ws) + carry_n;
        if (len > 0) {
            int first = q0;  // first entry at or after column lo0 (all parts of this k share it)
            if (lo0 > 0) {
                if (lid >= 0) {
                    first = q0 + (int)__ldg(tp + (int64_t)lid * (T + 1) + tlo);
                } else {
                    first = (int)lower_bound_col(B.col, q0, q0 + len, lo0);
                }
            }
            for (int w = wf; w <= wl; ++w) {
                const long long bw = (L * w) / NW, bw1 = (L * (w + 1)) / NW;
                const int lo = (int)(max(ex, bw) - ex), hi = (int)(min(ex + len, bw1) - ex);
                Part pt;
                pt.cur = max(q0 + lo, first);
                pt.end = q0 + hi;
                pt.q0 = q0;
                pt.lid = lid;
                pt.a = a;
                P[po + (w - wf)] = pt;
                if (bw >= ex) wpart[w] = po + (w - wf);  // the part holding product bw(w) starts warp w
            }
        }
        carry_p += tot;
        carry_n += ntot;
        __syncthreads();  // ws / wsll free for the next chunk's scans
    }
    if (tid == 0) {  // warps without products (only when L < NW) start where the next one does
        wpart[NW] = carry_n;
        for (int w = NW - 1; w >= 0; --w)
            if (wpart[w] < 0) wpart[w] = wpart[w + 1];
    }
    __syncthreads();
}

// The end (exclusive B position) of part P's products below column hi: the tile pointer of tile th
// (hi = th * TW, or p) for long B rows (tv = tp[lid][th], possibly prefetched), a bounded scan for short
// ones; never before the cursor (a part may start past this window: its slice begins mid-row).
__device__ __forceinline__ int part_seg_end(const Mat& B, const Part& pt, uint32_t tv, int64_t hi) {
    if (pt.lid >= 0) return max(pt.cur, min(pt.end, pt.q0 + (int)tv));
    if (pt.end - pt.cur > LONG_ROW) return (int)lower_bound_col(B.col, pt.cur, pt.end, hi);  // no tile pointers
    int e = pt.cur;
    while (e < pt.end && __ldg(B.col + e) < hi) ++e;  // <= LONG_ROW entries
    return e;
}

// Streams one warp's 32 lane-held segments (beg, len, a) through acc(c, v) (v = a * b_kj if VAL). Segments of >= SEG_LONG
// products are swept lane-strided, 4 batches in flight, no search; all shorter ones are flattened
// (one warp scan of their lengths, a 5-step shuffle search per batch) and streamed SEG_UNR batches at a
// time. (sg_dense2.cu; a software-pipelined variant that gathers the next SEG_UNR batches during the accumulation of
// the current ones measured slower: 33.4 vs 31.7 ms on C3 rows/2, profiles/r02_dense2_ab.txt.)
constexpr int SEG_LONG = 128;
constexpr int32_t SEG_NONE = INT_MAX;  // no product (a column is < INT32_MAX; tagged columns are negative)
constexpr int SEG_UNR = 4;
template <bool VAL, class VT, class F>
__device__ __forceinline__ void seg_walk(const Mat& B, int beg, int len, double a, F&& acc) {
    const int lane = threadIdx.x & 31;
    const int32_t* __restrict__ bcol = B.col;
    const VT* __restrict__ bval = reinterpret_cast<const VT*>(B.val);
    unsigned lm = __ballot_sync(FULL, len >= SEG_LONG);
    while (lm) {
        const int L = __ffs(lm) - 1;
        lm &= lm - 1u;
        const int b = __shfl_sync(FULL, beg, L), n = __shfl_sync(FULL, len, L);
        const double av = __shfl_sync(FULL, a, L);
        for (int j = lane; j < n; j += 128) {
            int c[4];
            double v[4];
            #pragma unroll
            for (int r = 0; r < 4; ++r) {
                const int jj = j + 32 * r;
                c[r] = SEG_NONE;
                v[r] = 0.0;
                if (jj < n) {
                    c[r] = __ldg(bcol + b + jj);
                    if (VAL) v[r] = av * (double)__ldg(bval + b + jj);
                }
            }
            #pragma unroll
            for (int r = 0; r < 4; ++r)
                if (c[r] != SEG_NONE) acc(c[r], v[r]);
        }
    }
    const int sl = len < SEG_LONG ? len : 0;
    const int inc = warp_incl_scan(sl);
    const int tot = __shfl_sync(FULL, inc, 31);
    const int off = inc - sl;
    for (int j0 = 0; j0 < tot; j0 += 32 * SEG_UNR) {
        int c[SEG_UNR];
        double v[SEG_UNR];
        #pragma unroll
        for (int r = 0; r < SEG_UNR; ++r) {
            const int j = j0 + 32 * r + lane;
            int s = 0;
            #pragma unroll
            for (int bb = 16; bb; bb >>= 1) {
                const int o = __shfl_sync(FULL, off, s + bb);
                if (o <= j) s += bb;
            }
            const int q = __shfl_sync(FULL, beg, s) + (j - __shfl_sync(FULL, off, s));
            const double as = __shfl_sync(FULL, a, s);
            c[r] = SEG_NONE;
            v[r] = 0.0;
            if (j < tot) {
                c[r] = __ldg(bcol + q);
                if (VAL) v[r] = as * (double)__ldg(bval + q);
            }
        }
        #pragma unroll
        for (int r = 0; r < SEG_UNR; ++r)
            if (c[r] != SEG_NONE) acc(c[r], v[r]);
    }
}

}  // namespace sg
