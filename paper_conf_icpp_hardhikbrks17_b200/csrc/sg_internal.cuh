// sg_internal.cuh — internal declarations shared by the libsg translation units (CUDA side only;
// nothing here is shared with oracle/). Layout and kernel design: DESIGN.md §6-§7.
#pragma once
#include <cuda_runtime.h>
#include <cstdint>
#include <cstddef>
#include "sg.h"

namespace sg {

// ---- launch accounting / optional per-launch CUDA-event timing (sg_profile.cu) ------------------
struct Prof {
    Prof(const char* name, cudaStream_t s);
    ~Prof();
    cudaStream_t s;
    long long idx;
};
#define SG_LAUNCH(name, stream, ...) do { ::sg::Prof _sg_prof(name, stream); __VA_ARGS__; } while (0)

// ---- routing classes and bins (heavy iff w > t; R13: w == t light) --
constexpr int NBIN_LIGHT = 13;   // light bin b holds 2^(b-1) < w <= 2^b  (b = 0: w == 1); U_b = 2^b
constexpr int BIN_EMPTY = 13;    // w == 0 (R7)
constexpr int BIN_HEAVY = 14;    // w > thr
constexpr int NBINS = 15;

// ---- heavy path geometry ---------------------------------------------------
constexpr int TW = 8192;          // column tile width of the heavy path (tile = unit of range planning)
constexpr int LONG_ROW = 8;       // B rows longer than this get per-tile pointers
#ifndef SG_SYM_WIN_LOG2
#define SG_SYM_WIN_LOG2 18
#endif
#ifndef SG_SYM_T
#define SG_SYM_T 256
#endif
#ifndef SG_SYM_OCC
#define SG_SYM_OCC 6
#endif
// rank-kernel (heavy numeric, sg_heavy.cu) geometry; the symbolic range plan depends on it
#ifndef SG_NUM_T
#define SG_NUM_T 512
#endif
#ifndef SG_NUM_OCC
#define SG_NUM_OCC 2
#endif
#ifndef SG_RCAP
#define SG_RCAP 8192
#endif
constexpr int NUM_T = SG_NUM_T;       // rank numeric: threads per CTA
constexpr int NUM_OCC = SG_NUM_OCC;   // rank numeric CTAs per SM (smem-bound)
constexpr int RW_TILES = NUM_T / 32;  // max tiles per numeric range (16 -> 128K columns, 16 KB bitmap)
constexpr int RCAP = SG_RCAP;         // max entries per numeric range (fp64 accumulator 64 KB)
constexpr int RHALF = RCAP / 2;       // range key granularity (a range = run of tiles with equal key)
constexpr int WIN = 1 << SG_SYM_WIN_LOG2;  // heavy symbolic bitmap window (columns); WIN/8 bytes of smem
constexpr int HEAVY_THREADS = SG_SYM_T;    // heavy symbolic threads per CTA
constexpr int SYM_OCC = SG_SYM_OCC;        // heavy symbolic CTAs per SM

constexpr int32_t EMPTY_KEY = -1;
constexpr uint64_t TAG_SAMPLE = 0x53414d504c450001ULL;  // DESIGN.md R4 (stream tag of the row sampler)

struct RangeRec {  // one heavy numeric work item: row x tiles [t0, t1)
    int32_t row;   // local row index (row - row_begin); -1 = unused slot
    int32_t t0, t1;
    int32_t cnt;   // exact number of C entries in the range
    int32_t off;   // offset of the range's first entry within the row
    int32_t pad;
};

struct Mat {  // device CSR view
    int64_t nrows, ncols, nnz;
    const int64_t* rp;
    const int32_t* col;
    const void* val;
    int dt;  // 0 f64, 1 f32
};

struct CostModelD {
    int64_t kL, lL, sL, rL, kH, lH, tH, mH, tiles_fixed, capu, cap_L;
};

// ---- launchers (sg_kernels.cu) ------------------------------------------------------------------
cudaError_t launch_row_work(const Mat& A, const Mat& B, int64_t rb, int64_t re, int64_t* w, cudaStream_t s);
cudaError_t launch_row_work_list(const Mat& A, const Mat& B, const int64_t* rows, int64_t nr, int64_t* w_rows,
                                 int64_t* a_rows, cudaStream_t s);
// exclusive scan in[0..n) -> out[0..n] (out[0] = 0, out[n] = total); tmp: scan_tmp_bytes(n) bytes
size_t scan_tmp_bytes(int64_t n);
cudaError_t scan_exclusive(const int64_t* in, int64_t* out, int64_t n, void* tmp, cudaStream_t s);
// stable selection of sampled rows: count then write
cudaError_t launch_sample_select(int64_t rb, int64_t re, uint64_t seed, uint64_t Tf, bool all,
                                 int64_t* out_rows, int64_t* d_count, void* tmp, size_t tmp_bytes, cudaStream_t s);
size_t sample_tmp_bytes(int64_t n);
// binning: w of nr rows (rows = list or rb + j); bins by thr; cls optional
cudaError_t launch_bin_count(const int64_t* w, int64_t nr, int64_t thr, int64_t* d_cnt /*NBINS*/, int8_t* cls,
                             cudaStream_t s);
cudaError_t launch_bin_scatter(const int64_t* w, int64_t nr, int64_t thr, int64_t* d_cursor /*NBINS*/,
                               int32_t* lists, cudaStream_t s);
// light path (sg_light.cu): bin b, rows = list entries (local index li); global row = rowmap ? rowmap[li] : rb + li
cudaError_t launch_sym_light(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt,
                             const int64_t* rowmap, int64_t rb, int64_t* u, int2* span /*nullable*/,
                             unsigned long long* nskew /*nullable: count of column-skewed rows*/, cudaStream_t s);
// light bin b takes the sorted warp path of the numeric pass for B with p columns (no span / skew
// information needed from the symbolic pass then); SG_OPT_VARIANT bit 4 keeps the order-preserving hash
bool light_sorted(int b, int64_t p, int variant);
// the sorted light path, split over the passes: the symbolic pass sorts each row's column keys into the row's
// slot of light_sort_width(b) keys (keys + list position x width) and writes u_i; the numeric pass gathers
// the values and emits C from the stored keys
int light_sort_width(int b);
cudaError_t launch_sym_light_sort(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, int64_t rb,
                                  uint32_t* keys, int64_t* u, cudaStream_t s);
cudaError_t launch_num_light_keys(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, int64_t rb,
                                  const uint32_t* keys, const int64_t* C_rp, int32_t* C_col, void* C_val, cudaStream_t s);
cudaError_t launch_num_light(int b, const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, int64_t rb,
                             const int2* span, const int64_t* C_rp, int32_t* C_col, void* C_val, cudaStream_t s);
// heavy path (sg_heavy.cu)
cudaError_t launch_long_rows(const Mat& B, int32_t* long_id, int64_t* d_nlong, cudaStream_t s);
cudaError_t launch_build_tp(const Mat& B, const int32_t* long_id, int T, uint32_t* tp, cudaStream_t s);
cudaError_t launch_heavy_order(const int32_t* heavy, int64_t nh, const int64_t* w, unsigned int* hist128,
                               int32_t* out, cudaStream_t s);
cudaError_t launch_range_bounds(const int32_t* heavy_list, int64_t nheavy, const int64_t* w, int64_t p,
                                int64_t dw_min_w, int64_t* bounds, cudaStream_t s);
cudaError_t launch_sym_heavy(const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, const int64_t* rowmap,
                             int64_t rb, int64_t* u, const int64_t* range_off, RangeRec* ranges, int32_t* nranges,
                             int64_t ndw, int32_t* dtc /*ndw x T tile counts, nullable*/, const int32_t* long_id /*nullable*/,
                             const uint32_t* tp /*nullable: binary search*/, int T, unsigned long long* counter,
                             cudaStream_t s, int64_t nbig /*rows [0, nbig) on the 1024-thread kernel*/);
// lean heavy symbolic (sg_sym2.cu): same outputs as launch_sym_heavy; w = row work indexed like u;
// pscr: sym2_scratch_parts(amax) Part records for rows of more than a few hundred k entries
cudaError_t launch_sym_heavy2(const Mat& A, const Mat& B, const int32_t* list, int64_t cnt, const int64_t* rowmap,
                              int64_t rb, const int64_t* w, int64_t* u, const int64_t* range_off, RangeRec* ranges,
                              int32_t* nranges, int64_t ndw, int32_t* dtc, const int32_t* long_id, const uint32_t* tp, int T,
                              unsigned long long* counter, cudaStream_t s, int64_t nbig, void* pscr, int64_t amax);
int64_t sym2_scratch_parts(int64_t amax);
size_t part_bytes();
cudaError_t launch_num_heavy(const Mat& A, const Mat& B, const int32_t* heavy, int64_t h0, int64_t nheavy, int64_t rb,
                             const int64_t* range_off, const int32_t* nranges, const RangeRec* ranges,
                             const int32_t* long_id, const uint32_t* tp, int T, const int64_t* C_rp, int32_t* C_col,
                             void* C_val, unsigned long long* counter, int4* gscr, int64_t amax, int amin /*skip rows with <= amin k entries*/, cudaStream_t s);
cudaError_t launch_max_i64(const int64_t* x, int64_t n, unsigned long long* out /*zeroed here*/, cudaStream_t s);
cudaError_t launch_max_a(const Mat& A, const int32_t* list, int64_t cnt, int64_t rb, unsigned long long* out,
                         cudaStream_t s);
// dense-window heavy rows (sg_dense.cu): heavy[0, ndw), all with w >= 2^dense_window_log2(p)
cudaError_t launch_num_dense(const Mat& A, const Mat& B, const int32_t* heavy, int64_t ndw, int64_t rb,
                             const int32_t* long_id, const uint32_t* tp, int T, const int64_t* C_rp, int32_t* C_col,
                             void* C_val, unsigned long long* counter, int4* gscr, int64_t amax,
                             const int32_t* dtc, const int4* items, const int64_t* nitems, cudaStream_t s);
// dense-window rows, lean product walk (sg_dense2.cu); pscr: per-CTA part scratch (pscr_cap parts) for
// rows with more than dense2_pcap() - 32 k entries
cudaError_t launch_num_dense2(const Mat& A, const Mat& B, const int32_t* heavy, int64_t ndw, int64_t rb,
                              const int64_t* w, const int32_t* long_id, const uint32_t* tp, int T, const int64_t* C_rp,
                              int32_t* C_col, void* C_val, unsigned long long* counter, void* pscr, int64_t pscr_cap,
                              const int32_t* dtc, const int4* items, const int64_t* nitems, cudaStream_t s);
size_t dense2_part_bytes();
int dense2_pcap();
// dense-window work items (row, window range): at most dense_items_bound(ndw, p); off[ndw] = count
int64_t dense_items_bound(int64_t ndw, int64_t p);
// window-major items (blocks of consecutive windows, ordered block by block); *nitems (device) = count
cudaError_t launch_dense_items_wm(int64_t ndw, int64_t p, int4* items, int64_t* nitems, cudaStream_t s);
cudaError_t launch_dense_items(const int32_t* heavy, int64_t ndw, const int64_t* w, int64_t p, int64_t* cnt,
                               int64_t* off, void* scan_tmp, int4* items, cudaStream_t s);
int dense_window_cols();
int dense_window_log2(int64_t p, int64_t opt);  // opt >= 0 overrides (sg_set_option; 62 disables the path)
int heavy_kc();
// warp-owned tile numeric for the rank rows (sg_tile.cu): range slots [0, nslots) (row < 0 = unused);
// only rows with at most tile_kreg() k entries (the rest: launch_num_heavy with amin = tile_kreg())
cudaError_t launch_num_tile(const Mat& A, const Mat& B, const RangeRec* ranges, int64_t nslots, int64_t rb,
                            const int32_t* long_id, const uint32_t* tp, int T, const int64_t* C_rp, int32_t* C_col,
                            void* C_val, unsigned long long* counter, cudaStream_t s);
int64_t tile_kreg();
int heavy_grid();
int dense_grid();
int dense_kc();
// threshold: cost histogram over rows then argmin over t in [0, cap_L]
struct ThrResult { long long thr, Jmin, base, W_L, W_all, nonempty, U_L, U_H; };
cudaError_t launch_cost_hist(const CostModelD& cm, const int64_t* w, const int64_t* a, const int64_t* u, int64_t nr,
                             long long* hist_d /*cap_L+1*/, long long* hist_c /*cap_L+1*/, long long* hist_w,
                             long long* sums /*4*/, cudaStream_t s);
cudaError_t launch_argmin(const CostModelD& cm, const long long* hist_d, const long long* hist_c,
                          const long long* hist_w, const long long* sums, ThrResult* out, cudaStream_t s);
cudaError_t launch_cost_curve(const CostModelD& cm, const int64_t* w, const int64_t* a, const int64_t* u, int64_t nr,
                              const int64_t* t, int nt, long long* J, cudaStream_t s);
cudaError_t launch_cuts(const int64_t* P, int64_t n, int G, int64_t* cuts, cudaStream_t s);
cudaError_t launch_row_cost(const CostModelD& cm, int64_t thr, const int64_t* comp /*host, 4*/, const int64_t* arp,
                            const int64_t* w, int64_t n, int64_t* cost, double* mag /*sum of c_L + c_H in fp64*/,
                            cudaStream_t s);
// sum over rows with w > 0 of c_L + c_H in fp64 (the overflow bound; sg_kernels.cu)
cudaError_t launch_cost_mag(const CostModelD& cm, const int64_t* w, const int64_t* a, const int64_t* u, int64_t nr,
                            double* out, cudaStream_t s);
constexpr double kCostLimit = 4611686018427387904.0;  // 2^62: a cost bound at or above it -> SG_ERR_OVERFLOW
cudaError_t launch_class_usum(const int64_t* w, const int64_t* u, int64_t nr, int64_t thr, unsigned long long* out,
                              cudaStream_t s);
cudaError_t launch_class_usum_dev(const int64_t* w, const int64_t* u, int64_t nr, const long long* thr_dev,
                                  unsigned long long* out, cudaStream_t s);
// HH four-block variant (sg_hh.cu)
cudaError_t launch_hh_len(const Mat& M, int64_t t, int high, int64_t* len, cudaStream_t s);
cudaError_t launch_rows_len(const Mat& M, const int64_t* rows, int64_t nr, int64_t* len, cudaStream_t s);
cudaError_t launch_rows_copy(const Mat& M, const int64_t* rows, int64_t nr, const int64_t* out_rp, int32_t* col, void* val,
                             cudaStream_t s);
cudaError_t launch_hh_copy(const Mat& M, const int64_t* out_rp, int32_t* col, void* val, cudaStream_t s);
cudaError_t launch_hh_hstack(const Mat& P, const Mat& Q, int64_t* rp, int32_t* col, void* val, int pass, cudaStream_t s);
cudaError_t launch_hh_identity2(int64_t p, int dt, int64_t* rp, int32_t* col, void* val, cudaStream_t s);
cudaError_t launch_hh_mask(int64_t n, uint64_t seed, uint64_t Tf, int all, int64_t* keep, cudaStream_t s);
cudaError_t launch_hh_rows_of_rank(int64_t n, const int64_t* keep, const int64_t* rank, int64_t* rows_of_rank,
                                   cudaStream_t s);
cudaError_t launch_hh_sub(const Mat& M, const int64_t* keep, const int64_t* rank, const int64_t* rows_of_rank, int64_t s_rows,
                          int64_t* cnt_or_rp, int32_t* col, int64_t* pos, void* val /*nullable*/, int pass, cudaStream_t s);
cudaError_t launch_gather_rows(const int64_t* src, const int64_t* rows, int64_t nr, int64_t* dst, cudaStream_t s);
cudaError_t launch_add_offset(int64_t* x, int64_t n, int64_t off, cudaStream_t s);
cudaError_t launch_check_rows(const int64_t* rows, int64_t nr, int64_t n, unsigned long long* bad, cudaStream_t s);

}  // namespace sg
