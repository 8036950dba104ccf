// sg_rank2.cu — HEAVY numeric, rank-indexed compact accumulator per column range,
// with per-warp product slices instead of per-range block packing.
//
// Same algorithm and outputs as k_num_heavy (sg_heavy.cu): for every range of the symbolic plan
// (<= RCAP entries, <= RW_TILES column tiles) pass 1 builds the range's bitmap, a block scan turns word
// popcounts into a uint16 rank prefix, pass 2 adds every product into a compact fp64 array at
// rank(c) = prefix[word] + popc(word & below) and the first arrival writes C.col; the values leave by one
// bulk async copy. What changes is the enumeration: the row's products are cut ONCE into one contiguous
// slice per warp (Part lists, sg_device.cuh), and per range each warp advances only its own parts (one
// tile-pointer step per part) and walks their segments — in pass 1 and again in pass 2 — with the
// lean lane-strided / flattened walker; the per-range block scan + packing of every k entry
// (chunk_compact) and the per-batch search over it (SliceCursor) are gone (profiles/r02_*: 13 % of the
// rank kernel's warp time went to segments + compaction alone).
#include "sg_device.cuh"

namespace sg {

constexpr int R2_NW = NUM_T / 32;
constexpr int R2_PCAP = 704;  // parts in shared memory (rows with more k entries use global scratch)

struct Rank2Smem {
    uint32_t bm[RW_TILES * TW / 32];  // range bitmap
    double vals[RCAP + 2];            // compact accumulator: rank r at vals[r + sh]
    uint16_t pref[RW_TILES * TW / 32];// rank prefix per bitmap word
    Part parts[R2_PCAP];
    int32_t pbeg[R2_PCAP];            // each part's first position in the current range (pass 2 re-walk)
    int32_t wpart[R2_NW + 1];
    long long wsll[33];
    int ws[33];
};
static_assert(RW_TILES * TW / 32 == 8 * NUM_T, "prefix layout: 8 words per thread");
static_assert(2 * (sizeof(Rank2Smem) + 1024) <= 233472 || NUM_OCC == 1, "rank2: two CTAs per SM must fit");

__device__ __forceinline__ void r2_bulk_s2g(void* gdst, const void* ssrc, uint32_t bytes) {
    const uint32_t sa = (uint32_t)__cvta_generic_to_shared(ssrc);
    uint64_t pol;  // C values: evict-first in L2
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(gdst), "r"(sa),
                 "r"(bytes), "l"(pol) : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}

template <class VT>
__global__ void __launch_bounds__(NUM_T, NUM_OCC) k_num_rank2(
    Mat A, Mat B, const int32_t* __restrict__ heavy, int64_t h0, int64_t nheavy, int64_t rb, const int64_t* __restrict__ wrow,
    const int64_t* __restrict__ range_off, const int32_t* __restrict__ nranges, const RangeRec* __restrict__ ranges,
    const int32_t* __restrict__ long_id, const uint32_t* __restrict__ tp, int T, const int64_t* __restrict__ C_rp,
    int32_t* __restrict__ C_col, VT* __restrict__ C_val, unsigned long long* counter, Part* __restrict__ pscr,
    int32_t* __restrict__ bscr, int64_t pscr_cap) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    Rank2Smem& S = *reinterpret_cast<Rank2Smem*>(smem_raw);
    __shared__ long long s_j;
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int64_t p = B.ncols;
    constexpr int RWW = RW_TILES * TW / 32;
    for (int q = tid; q < RWW; q += NUM_T) S.bm[q] = 0u;
    for (int q = tid; q < RCAP + 2; q += NUM_T) S.vals[q] = 0.0;
    const uint32_t a_bm = smem_addr(S.bm);
    const uint32_t a_pref = a_bm + (uint32_t)((const char*)S.pref - (const char*)S.bm);
    const uint32_t a_vals = a_bm + (uint32_t)((const char*)S.vals - (const char*)S.bm);
    constexpr bool kBulk = sizeof(VT) == 8;  // fp64 output: accumulator copied out by a bulk async copy
    int clear_n = 0;                          // accumulator entries still to be cleared (bulk path)
    while (true) {
        if (tid == 0) s_j = h0 + (long long)atomicAdd(counter, 1ull);
        __syncthreads();
        const int64_t h = s_j;
        if (h >= nheavy) break;
        const int64_t li = heavy[h];
        const int64_t row = rb + li;
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        const int na = (int)(s1 - s0);
        const int nr = nranges[h];
        const RangeRec* rr = ranges + range_off[h];
        const int64_t crow = C_rp[li];
        const bool in_smem = na + R2_NW <= R2_PCAP;
        Part* P = in_smem ? S.parts : pscr + (int64_t)blockIdx.x * pscr_cap;
        int32_t* PB = in_smem ? S.pbeg : bscr + (int64_t)blockIdx.x * pscr_cap;  // range begins of parts >= 32
        build_parts<NUM_T, VT, true>(A, B, s0, na, (long long)wrow[li], long_id, tp, T, 0, 0, P, S.wpart, S.wsll, S.ws);
        const int pw0 = S.wpart[wid], pw1 = S.wpart[wid + 1];
        RangeRec Rn;
        if (nr > 0) Rn = rr[0];
        // group-0 tile pointer of the next range, prefetched one range ahead
        uint32_t tvn = 0;
        int lid0 = -1;
        if (pw0 + lane < pw1) {
            lid0 = P[pw0 + lane].lid;
            if (lid0 >= 0 && nr > 0) tvn = __ldg(tp + (int64_t)lid0 * (T + 1) + Rn.t1);
        }
        for (int ri = 0; ri < nr; ++ri) {
            const RangeRec R = Rn;
            if (ri + 1 < nr) Rn = rr[ri + 1];
            const int64_t lo = (int64_t)R.t0 * TW, hi = min(p, (int64_t)R.t1 * TW);
            // ---- pass 1: this warp's segments of the range (cursor steps) + the range bitmap ----
            const uint32_t bb = opaque_u32(a_bm - 4u * ((uint32_t)lo >> 5));  // &bm[(c - lo) >> 5] = bb + 4(c >> 5)
            auto setbit = [&](int32_t c, double) { red_or_s(bb + 4u * ((uint32_t)c >> 5), 1u << (c & 31)); };
            int beg0 = 0, len0 = 0;
            double a0 = 0.0;
            for (int g = pw0; g < pw1; g += 32) {
                const int j = g + lane;
                int beg = 0, len = 0;
                double a = 0.0;
                if (j < pw1) {
                    const Part pt = P[j];
                    beg = pt.cur;
                    if (pt.cur < pt.end) {
                        const uint32_t tv = g == pw0 ? tvn : (pt.lid >= 0 ? __ldg(tp + (int64_t)pt.lid * (T + 1) + R.t1) : 0u);
                        const int e = part_seg_end(B, pt, tv, hi);
                        len = e - pt.cur;
                        a = pt.a;
                        P[j].cur = e;
                    }
                    if (g != pw0) PB[j] = beg;  // warps with more than 32 parts re-walk these in pass 2
                }
                if (g == pw0) {
                    beg0 = beg; len0 = len; a0 = a;
                    if (lid0 >= 0 && ri + 1 < nr) tvn = __ldg(tp + (int64_t)lid0 * (T + 1) + Rn.t1);
                }
                seg_walk<false, VT>(B, beg, len, 0.0, setbit);
            }
            __syncthreads();
            // ---- rank prefix over the range's words: thread t owns words [8t, 8t+8) ----
            {
                const uint4 q0 = reinterpret_cast<const uint4*>(S.bm)[2 * tid];
                const uint4 q1 = reinterpret_cast<const uint4*>(S.bm)[2 * tid + 1];
                const int c0 = __popc(q0.x), c1 = __popc(q0.y), c2 = __popc(q0.z), c3 = __popc(q0.w);
                const int c4 = __popc(q1.x), c5 = __popc(q1.y), c6 = __popc(q1.z), c7 = __popc(q1.w);
                int t2;
                if (kBulk && tid == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
                const int p0 = block_scan<NUM_T>(c0 + c1 + c2 + c3 + c4 + c5 + c6 + c7, &t2, S.ws);
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
                reinterpret_cast<uint4*>(S.pref)[tid] = o;
            }
            __syncthreads();
            // ---- pass 2: every product accumulated at rank(c); the column is written on first arrival ----
            const int64_t base = crow + R.off;
            const int sh = kBulk ? (int)(((uintptr_t)(C_val + base) >> 3) & 1u) : 0;
            const uint32_t bw = opaque_u32(a_bm - 4u * ((uint32_t)lo >> 5));
            const uint32_t pw = a_pref - 2u * ((uint32_t)lo >> 5);
            const uint32_t vb = a_vals + 8u * (uint32_t)sh;
            auto acc = [&](int32_t c, double v) {
                const uint32_t cw = (uint32_t)c >> 5;
                const uint32_t wv = ld_u32_s(bw + 4u * cw);
                const int rank = (int)ld_u16_s(bw + (pw - bw) + 2u * cw) + __popc(wv & ((1u << (c & 31)) - 1u));
                if (atom_add_f64_s(bw + (vb - bw) + 8u * (uint32_t)rank, v) == 0.0) st_out(C_col + base + rank, c);
            };
            seg_walk<true, VT>(B, beg0, len0, a0, acc);
            for (int g = pw0 + 32; g < pw1; g += 32) {
                const int j = g + lane;
                int beg = 0, len = 0;
                double a = 0.0;
                if (j < pw1) {
                    beg = PB[j];
                    len = P[j].cur - beg;
                    a = P[j].a;
                }
                seg_walk<true, VT>(B, beg, len, a, acc);
            }
            if (kBulk) asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // accumulator -> bulk copy
            __syncthreads();
            // ---- values by rank (bulk copy); bitmap cleared for the next range ----
            const int cnt = R.cnt;
            if constexpr (kBulk) {
                const int e0 = sh, n2 = (cnt - e0) & ~1;
                if (tid == 0 && n2 > 0) r2_bulk_s2g(C_val + base + e0, &S.vals[e0 + sh], (uint32_t)n2 * 8u);
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
            __syncthreads();  // bitmap clear (and vals reads) before the next range's pass 1
        }
    }
    if (kBulk && tid == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

// global scratch for rows of more than R2_PCAP - R2_NW k entries: per CTA (amax + R2_NW) Part records
// followed (after all CTAs' parts) by as many int32 range begins; in bytes
size_t rank2_scratch_bytes(int64_t amax) {
    if (amax + R2_NW <= R2_PCAP) return 0;
    return (size_t)NUM_OCC * 148 * (size_t)(amax + R2_NW) * (sizeof(Part) + sizeof(int32_t));
}

cudaError_t launch_num_rank2(const Mat& A, const Mat& B, const int32_t* heavy, int64_t h0, int64_t nheavy, int64_t rb,
                             const int64_t* w, const int64_t* range_off, const int32_t* nranges, const RangeRec* ranges,
                             const int32_t* long_id, const uint32_t* tp, int T, const int64_t* C_rp, int32_t* C_col,
                             void* C_val, unsigned long long* counter, void* pscr, int64_t amax, cudaStream_t s) {
    if (nheavy - h0 <= 0) return cudaSuccess;
    const int smem = (int)sizeof(Rank2Smem);
    cudaError_t e = cudaMemsetAsync(counter, 0, sizeof(unsigned long long), s);
    if (e != cudaSuccess) return e;
    const int64_t nh = nheavy - h0;
    const int grid = (int)(nh < NUM_OCC * 148 ? nh : NUM_OCC * 148);
    const int64_t cap = amax + R2_NW;
    Part* ps = (Part*)pscr;
    int32_t* bs = pscr ? reinterpret_cast<int32_t*>(ps + (int64_t)NUM_OCC * 148 * cap) : nullptr;
    if (A.dt == 0) {
        if ((e = cudaFuncSetAttribute(k_num_rank2<double>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
        SG_LAUNCH("k_num_heavy", s, (k_num_rank2<double><<<grid, NUM_T, smem, s>>>(A, B, heavy, h0, nheavy, rb, w, range_off,
                                                                                  nranges, ranges, long_id, tp, T, C_rp, C_col,
                                                                                  (double*)C_val, counter, ps, bs, cap)));
    } else {
        if ((e = cudaFuncSetAttribute(k_num_rank2<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem)) != cudaSuccess) return e;
        SG_LAUNCH("k_num_heavy", s, (k_num_rank2<float><<<grid, NUM_T, smem, s>>>(A, B, heavy, h0, nheavy, rb, w, range_off,
                                                                                 nranges, ranges, long_id, tp, T, C_rp, C_col,
                                                                                 (float*)C_val, counter, ps, bs, cap)));
    }
    return cudaGetLastError();
}

}  // namespace sg
