// sg_sym2.cu — heavy SYMBOLIC (u_i = nnz(C_i), per-tile counts, the numeric range plan; PAPER L204,
// L223: the two-phase row-row product) with per-warp product slices.
//
// Same outputs as k_sym_heavy (sg_heavy.cu), different product enumeration: once per row the products
// are cut into one contiguous slice per warp (Part lists, sg_device.cuh build_parts); per 2^SWIN-column
// bitmap window each warp walks only its own parts (one cursor step per part: the B tile pointer of the
// window end, or a bounded scan) and ORs their columns into the shared bitmap — no per-window block
// packing of the k entries (chunk_compact) and no per-batch search over them (SliceCursor), which ncu
// put at most of k_sym_heavy's instructions (it issued on 82 % of cycles, profiles/r01s4_*).
#include "sg_device.cuh"

namespace sg {

template <int ST> struct Sym2Cfg;
template <> struct Sym2Cfg<256> { static constexpr int PCS = 160; };    // six CTAs per SM (32 KB bitmaps)
template <> struct Sym2Cfg<1024> { static constexpr int PCS = 4000; };  // one CTA per SM (128 KB bitmap)

template <int ST, int SWIN> constexpr int sym2_smem() { return (SWIN / 32) * 4 + Sym2Cfg<ST>::PCS * (int)sizeof(Part); }

template <int ST, int SOCC, int SWIN>
__global__ void __launch_bounds__(ST, SOCC) k_sym2(Mat A, Mat B, const int32_t* __restrict__ list, int64_t j0, int64_t cnt,
                                                   const int64_t* __restrict__ rowmap, int64_t rb,
                                                   const int64_t* __restrict__ wrow, int64_t* __restrict__ u,
                                                   const int64_t* __restrict__ range_off, RangeRec* __restrict__ ranges,
                                                   int32_t* __restrict__ nranges, int64_t ndw, int32_t* __restrict__ dtc,
                                                   const int32_t* __restrict__ long_id, const uint32_t* __restrict__ tp,
                                                   int T, unsigned long long* counter, Part* __restrict__ pscr,
                                                   int64_t pscr_cap) {
    extern __shared__ __align__(16) uint32_t bm[];  // SWIN/32 words, then PCS parts
    constexpr int NW = ST / 32;
    constexpr int PCS = Sym2Cfg<ST>::PCS;
    Part* sparts = reinterpret_cast<Part*>(bm + SWIN / 32);
    __shared__ int32_t wpart[NW + 1];
    __shared__ int tcnt[SWIN / TW];
    __shared__ int Ps[SWIN / TW];
    __shared__ unsigned char st[SWIN / TW];
    __shared__ long long wsll[33];
    __shared__ int ws[33];
    __shared__ long long s_j;
    __shared__ int s_nr, s_u;
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int64_t p = B.ncols;
    const int64_t nwin = (p + SWIN - 1) / SWIN;
    const uint32_t a_bm = smem_addr(bm);
    while (true) {
        if (tid == 0) s_j = j0 + (long long)atomicAdd(counter, 1ull);
        __syncthreads();
        const int64_t j = s_j;
        __syncthreads();
        if (j >= cnt) break;
        const int64_t li = list[j];
        const int64_t row = rowmap ? rowmap[li] : rb + li;
        const int64_t s0 = __ldg(A.rp + row), s1 = __ldg(A.rp + row + 1);
        const int na = (int)(s1 - s0);
        Part* P = na + NW <= PCS ? sparts : pscr + (int64_t)blockIdx.x * pscr_cap;
        build_parts<ST, double, false>(A, B, s0, na, (long long)wrow[li], long_id, tp, T, 0, 0, P, wpart, wsll, ws);
        const int pw0 = wpart[wid], pw1 = wpart[wid + 1];
        int utot = 0, nr = 0;
        for (int64_t win = 0; win < nwin; ++win) {
            const int64_t wlo = win * SWIN, whi = min(p, wlo + SWIN);
            const int th = whi == p ? T : (int)(whi / TW);
            const int nwords = (int)((whi - wlo + 31) / 32);
            for (int q = tid; q < nwords; q += ST) bm[q] = 0u;
            __syncthreads();  // cleared before any warp sets bits
            const uint32_t bb = opaque_u32(a_bm - 4u * ((uint32_t)wlo >> 5));  // wlo: multiple of 32
            auto setbit = [&](int32_t c, double) { red_or_s(bb + 4u * ((uint32_t)c >> 5), 1u << (c & 31)); };
            for (int g = pw0; g < pw1; g += 32) {
                const int jj = g + lane;
                int beg = 0, len = 0;
                if (jj < pw1) {
                    const Part pt = P[jj];
                    if (pt.cur < pt.end) {
                        const uint32_t tv = pt.lid >= 0 ? __ldg(tp + (int64_t)pt.lid * (T + 1) + th) : 0u;
                        const int e = part_seg_end(B, pt, tv, whi);
                        beg = pt.cur;
                        len = e - pt.cur;
                        P[jj].cur = e;
                    }
                }
                seg_walk<false, double>(B, beg, len, 0.0, setbit);
            }
            __syncthreads();
            // per-tile popcounts
            const int nt = (int)((whi - wlo + TW - 1) / TW);
            for (int tt = wid; tt < nt; tt += NW) {
                const int a = tt * (TW / 32), b = min(nwords, a + TW / 32);
                int c = 0;
                for (int q = a + lane; q < b; q += 32) c += __popc(bm[q]);
                c = warp_sum(c);
                if (lane == 0) tcnt[tt] = c;
            }
            __syncthreads();
            // range plan (warp 0): identical to k_sym_heavy (sg_heavy.cu)
            if (wid == 0 && j < ndw) {  // dense-window row: u and its tile counts, no range plan
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
static cudaError_t sym2_part(const Mat& A, const Mat& B, const int32_t* list, int64_t j0, int64_t cnt, const int64_t* rowmap,
                             int64_t rb, const int64_t* w, int64_t* u, const int64_t* range_off, RangeRec* ranges,
                             int32_t* nranges, int64_t ndw, int32_t* dtc, const int32_t* long_id, const uint32_t* tp, int T,
                             unsigned long long* counter, Part* pscr, int64_t pscr_cap, cudaStream_t s) {
    if (cnt - j0 <= 0) return cudaSuccess;
    constexpr int smem = sym2_smem<ST, SWIN>();
    cudaError_t e = cudaFuncSetAttribute(k_sym2<ST, SOCC, SWIN>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    if ((e = cudaMemsetAsync(counter, 0, sizeof(unsigned long long), s)) != cudaSuccess) return e;
    const int64_t n = cnt - j0;
    const int grid = (int)(n < 148 * SOCC ? n : 148 * SOCC);
    SG_LAUNCH("k_sym_heavy", s, (k_sym2<ST, SOCC, SWIN><<<grid, ST, smem, s>>>(A, B, list, j0, cnt, rowmap, rb, w, u, range_off,
                                                                             ranges, nranges, ndw, dtc, long_id, tp, T,
                                                                             counter, pscr, pscr_cap)));
    return cudaGetLastError();
}

// Part scratch (in Part records) that launch_sym_heavy2 needs for rows of at most amax k entries.
size_t part_bytes() { return sizeof(Part); }

int64_t sym2_scratch_parts(int64_t amax) {
    const int64_t small = amax + 8 > Sym2Cfg<256>::PCS ? (int64_t)148 * SYM_OCC * (amax + 8) : 0;
    const int64_t big = amax + 32 > Sym2Cfg<1024>::PCS ? (int64_t)148 * (amax + 32) : 0;
    return small > big ? small : big;
}

cudaError_t launch_sym_heavy2(const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, const int64_t* rowmap,
                              int64_t rb, const int64_t* w, int64_t* u, const int64_t* range_off, RangeRec* ranges,
                              int32_t* nranges, int64_t ndw, int32_t* dtc, const int32_t* long_id, const uint32_t* tp, int T,
                              unsigned long long* counter, cudaStream_t s, int64_t nbig, void* pscr, int64_t amax) {
    if (cnt <= 0) return cudaSuccess;
    if (nbig > cnt) nbig = cnt;
    static_assert(HEAVY_THREADS == 256 && WIN == (1 << 18), "sym2: the small-CTA geometry of k_sym_heavy");
    cudaError_t e = sym2_part<1024, 1, (1 << 20)>(A, B, list, 0, nbig, rowmap, rb, w, u, range_off, ranges, nranges, ndw,
                                                  dtc, long_id, tp, T, counter, (Part*)pscr, amax + 32, s);
    if (e != cudaSuccess) return e;
    return sym2_part<256, SYM_OCC, WIN>(A, B, list, nbig, cnt, rowmap, rb, w, u, range_off, ranges, nranges, ndw, dtc,
                                        long_id, tp, T, counter, (Part*)pscr, amax + 8, s);
}

}  // namespace sg
