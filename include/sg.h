/*
 * sg.h — C ABI of libsg, the B200 (sm_100a) sampled-threshold Gustavson SpGEMM.
 *
 * The operation is C = A·B on CSR inputs, "A with n rows and m columns, B with m rows and k
 * columns ... Resultant Matrix C with n rows and k columns" (Alg. 2), computed
 * row by row (Gustavson; Alg. 2 l.5-6, L222-L223). Rows are routed between a light
 * and a heavy kernel path by a threshold t on the per-row work volume w_i = L_AB[i],
 * heavy iff w_i > t, and t is chosen by the paper's Sample -> Identify ->
 * Extrapolate procedure (Fig. 2). Row ranges for several GPUs are cut on the work
 * prefix (Alg. 2 l.1-4, L215-L218; threshold vector, L106). "PAPER Lnnn" is line nnn of the paper
 * text; DESIGN.md lists every reading taken where it is ambiguous.
 *
 * Conventions shared by every entry point
 *  - Matrices are canonical CSR: row_ptr int64[nrows+1] (row_ptr[0] == 0), col_idx int32[nnz]
 *    strictly ascending within each row, values fp64 or fp32[nnz]. A and B must have the same
 *    value dtype; C gets that dtype. Inputs are BORROWED device pointers, never freed by sg.
 *  - Pointers are DEVICE pointers unless marked (host). Scalars marked (host) are written by the
 *    call before it returns (the call synchronises the stream for them).
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream). Work is
 *    stream-ordered; the only host synchronisations are the documented host outputs.
 *  - Every call returns a status and never throws across the ABI. On error, caller-owned outputs
 *    are left untouched where possible and a plan involved in the failure is poisoned (every later
 *    call with it returns SG_ERR_CUDA); destroy it with sg_plan_destroy.
 *  - Structural semantics: C has an entry wherever some product a_ik*b_kj exists, even if the
 *    values cancel to zero (reading R9). Columns of each C row are ascending.
 */
#ifndef SG_H
#define SG_H

#include <stdint.h>
#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    SG_OK = 0,
    SG_ERR_INVALID_ARG = 1,   /* null pointer, sample_frac outside (0,1], thr outside [0,cap_L], bad row range */
    SG_ERR_SHAPE = 2,         /* A.ncols != B.nrows, or a buffer shape mismatch */
    SG_ERR_DTYPE = 3,         /* A and B value dtypes differ, or unknown dtype */
    SG_ERR_NOT_CANONICAL = 4, /* only with SG_OPT_VALIDATE = 1: unsorted/duplicate/out-of-range columns, bad row_ptr */
    SG_ERR_EMPTY_SAMPLE = 5,  /* the sample holds no non-empty row */
    SG_ERR_OOM = 6,           /* device workspace allocation failed */
    SG_ERR_CUDA = 7,          /* a CUDA runtime error (or a poisoned plan) */
    SG_ERR_NCCL = 8,          /* an NCCL error in sg_gather */
    SG_ERR_OVERFLOW = 9       /* a dimension exceeds INT32_MAX, B.nnz >= INT32_MAX, or sum_i (c_L(i) + c_H(i)) over the
                                 rows a cost-model call sees, evaluated in fp64, reaches 2^62 (so no int64 sum can wrap) */
} sg_status;

typedef enum { SG_F64 = 0, SG_F32 = 1 } sg_dtype;

/* A borrowed view of a device CSR matrix. */
typedef struct {
    int64_t nrows, ncols, nnz;
    const int64_t* row_ptr;   /* device, nrows+1 */
    const int32_t* col_idx;   /* device, nnz */
    const void* val;          /* device, nnz of dtype */
    sg_dtype dtype;
} sg_csr_view;

/* Per-row path costs in integer picoseconds (the "offline relation" of PAPER L94):
 *   c_L(i) = kappa_L + lambda_L*w_i + sigma_L*u_i*ceil(log2 max(u_i,2)) + rho_L*u_i
 *   c_H(i) = kappa_H + lambda_H*w_i + tau_H*a_i*R(u_i) + mu_H*u_i
 *   R(u)   = tiles_fixed if capu == 0, else max(1, tiles_fixed, ceil(u/capu))
 * with a_i = nnz(A_i), w_i = L_AB[i], u_i = nnz(C_i). cap_L is the largest admissible
 * threshold (the light path's table capacity); it must be <= SG_CAP_L_MAX. Every coefficient must be
 * >= 0 (INVALID_ARG otherwise): costs are then non-negative and every cost prefix is monotone. */
typedef struct {
    int64_t kappa_L, lambda_L, sigma_L, rho_L;
    int64_t kappa_H, lambda_H, tau_H, mu_H;
    int64_t tiles_fixed, capu, cap_L;
} sg_cost_model;

#define SG_CAP_L_MAX 4096

/* What sg_sample_threshold saw (host struct). */
typedef struct {
    int64_t sample_rows;      /* |S| (Binomial(n, f)) */
    int64_t sample_nonempty;  /* rows of S with w > 0 */
    int64_t thr;              /* the returned threshold */
    int64_t W_est_L, W_est_H; /* sum of w over sampled light / heavy rows at thr */
    int64_t J_min;            /* min_t J(t; S) in ps (unscaled: the n/|S| factor cancels in the argmin) */
    int64_t U_est_L, U_est_H; /* sum of u = nnz(C_i) over sampled light / heavy rows at thr (the sample's
                                 per-class compression, input of sg_partition_cost) */
} sg_sample_report;

/* Per-class counts of a plan (host struct). */
typedef struct {
    int64_t row_begin, row_end, thr;
    int64_t n_empty, n_light, n_heavy;
    int64_t nnz_c;            /* sum of u_i over the plan's rows */
    int64_t flops;            /* W = sum of w_i over the plan's rows (multiply-adds) */
    int64_t n_ranges;         /* heavy column ranges (numeric work items of the heavy path) */
    int64_t light_bins[13];   /* light rows per bin b: 2^(b-1) < w <= 2^b (b = 0: w == 1) */
    int64_t n_dense;          /* heavy rows on the dense-window kernel (w >= 2^dense_log2) */
    int64_t dense_log2;       /* that row-work bound (SG_OPT_DENSE_LOG2 overrides; 62: path disabled) */
    int64_t n_light_sorted;   /* light rows whose columns cluster (hash homes crowded): uniform hash + sort */
} sg_plan_info;

typedef struct sg_plan sg_plan;   /* opaque; owns only its workspace */

/* Process-wide options, read by every later call (not per plan; set them before sg_symbolic).
 *   SG_OPT_VALIDATE    0/1: check canonical CSR inputs on every call (SG_ERR_NOT_CANONICAL).
 *   SG_OPT_DENSE_LOG2  -1 (default) = automatic; m in [0, 62]: heavy rows with w >= 2^m take the
 *                      dense-window numeric kernel; 62 disables that path.
 *   SG_OPT_VARIANT     kernel variant bits for A/B measurements (0 = the default kernels; bit 0: the
 *                      previous dense-window kernel, sg_dense.cu; bit 1: the previous heavy symbolic
 *                      kernel, k_sym_heavy in sg_heavy.cu; bit 2: row-major dense-window work items
 *                      instead of window-major ones; bit 3: the CTA rank kernel for every rank row instead of
 *                      the warp-tile kernel for rows of <= 64 k entries; bit 4: the order-preserving hash for
 *                      every light bin instead of the sorted warp path for w <= 512; bit 5: the warp-tile
 *                      kernel even when a plan has fewer than 4096 rank rows). Every variant computes the same C.
 *   SG_OPT_L2_PERSIST  bytes of B.col kept in the persisting L2 carve-out during sg_symbolic / sg_numeric
 *                      (every heavy product gathers a column of B): -1 = all of B.col up to the device's
 *                      maximum carve-out, 0 (default) = off (measured no gain on C3: 239.9 vs 235.1 ms). The calls set the stream's access-policy window
 *                      for their own launches and clear it before returning; the device's persisting-L2 limit
 *                      is raised once (a process-wide setting).
 *   SG_OPT_TP_MAX_BYTES  memory budget of the plan's B tile-pointer table (4 bytes x (long B rows) x (p/8192 + 1);
 *                      it grows with rows x columns, not nnz): -1 (default) = 8 GiB; above the budget the
 *                      heavy kernels locate B-row segments by binary search instead (same C, slower).
 * The environment seeds them once, at the library's first call (SG_VALIDATE=1, SG_DW_LOG2=m, SG_L2_PERSIST=b).
 * Errors: INVALID_ARG (unknown key or value out of range). sg_get_option: INT64_MIN if unknown. */
typedef enum { SG_OPT_VALIDATE = 0, SG_OPT_DENSE_LOG2 = 1, SG_OPT_VARIANT = 2, SG_OPT_L2_PERSIST = 3, SG_OPT_TP_MAX_BYTES = 4,
               SG_OPT_COUNT = 5 } sg_option;
sg_status sg_set_option(int key, int64_t value);
int64_t sg_get_option(int key);

/* Human-readable status name (static storage). */
const char* sg_status_string(sg_status st);
/* Library version string, e.g. "sg 0.1.0 sm_100a". */
const char* sg_version(void);
/* The calibrated default cost model, with tiles_fixed = 1. Calls given cm == NULL use it
 * with tiles_fixed = ceil(B.ncols / 131072), the heavy path's minimum number of column ranges per row
 * (R(u)'s floor): exactly the model sg_default_cost_model_for(B.ncols) returns. */
void sg_default_cost_model(sg_cost_model* out /*host*/);
void sg_default_cost_model_for(int64_t p, sg_cost_model* out /*host*/);
/* The default model of sg_partition_cost: fitted to measured per-shard times. */
void sg_default_partition_model(sg_cost_model* out /*host*/);

/* Row work volume w_i = sum_{k in A_i} nnz(B_k) = L_AB[i] (Alg. 2 l.1 L215) for rows
 * [row_begin, row_end) into w_out[0 .. row_end-row_begin) (device, caller-owned). If total_out is
 * non-NULL the sum W is written there (host; synchronises). */
sg_status sg_row_work(const sg_csr_view* A, const sg_csr_view* B, int64_t row_begin, int64_t row_end,
                      int64_t* w_out, int64_t* total_out /*host, nullable*/, void* stream);

/* Sample -> Identify -> Extrapolate: draws the Bernoulli(sample_frac) row sample
 * S = { i : h(seed, SAMPLE, i) < floor(sample_frac*2^64) } (uniform sampling, L92; R4),
 * computes (w_i, a_i, u_i) for i in S on the device (u_i by an exact sample-symbolic pass), and
 * returns thr = the smallest minimiser of J(t;S) = sum_{i in S, 0<w_i<=t} c_L(i) + sum_{i in S,
 * w_i>t} c_H(i) over t in {0} u {w_i : i in S, 0 < w_i <= cap_L} (Identify, L87-L89). Extrapolation
 * is the identity (r = r', L236). cm == NULL uses sg_default_cost_model. Synchronises.
 * Errors: INVALID_ARG (sample_frac outside (0,1]), EMPTY_SAMPLE, SHAPE, DTYPE. */
sg_status sg_sample_threshold(const sg_csr_view* A, const sg_csr_view* B, double sample_frac, uint64_t seed,
                              const sg_cost_model* cm, int64_t* thr_out /*host*/,
                              sg_sample_report* rep /*host, nullable*/, void* stream);

/* Identify on an EXPLICIT row sample (PAPER L87-L89 with a caller-chosen I_s): rows (device int64,
 * nrows entries, each in [0, A.nrows); duplicates count twice) -> thr = the smallest minimiser of
 * J(t; rows), exactly as sg_sample_threshold computes it on its Bernoulli sample. For the paper's
 * sample-shape experiments: a predetermined sub-matrix vs a random one (L250, Fig. 7), sqrt(n) rows
 * (L139, L287). Synchronises. Errors: INVALID_ARG (row id out of range), EMPTY_SAMPLE, SHAPE, DTYPE. */
sg_status sg_threshold_on_rows(const sg_csr_view* A, const sg_csr_view* B, const int64_t* rows, int64_t nrows,
                               const sg_cost_model* cm, int64_t* thr_out /*host*/, sg_sample_report* rep /*host, nullable*/,
                               void* stream);

/* The exhaustive threshold thr* = thr over ALL rows (needs u_i for every row, i.e. a full
 * symbolic pass — what the paper calls "not practical", L198, L246). Used for the gap report. */
sg_status sg_exhaustive_threshold(const sg_csr_view* A, const sg_csr_view* B, const sg_cost_model* cm,
                                  int64_t* thr_out /*host*/, int64_t* J_min_out /*host, nullable*/, void* stream);

/* J(t; all rows) for an explicit list of thresholds (host arrays of length nt), for the gap report.
 * Needs a full symbolic pass, like sg_exhaustive_threshold. Synchronises. */
sg_status sg_cost_curve(const sg_csr_view* A, const sg_csr_view* B, const sg_cost_model* cm,
                        int64_t nt, const int64_t* t_host, int64_t* J_host /*host, nt*/, void* stream);

/* Work-balanced contiguous row blocks for nparts GPUs (Alg. 2 l.2-4, L216-L218, as a vector L106):
 * cuts_out[0] = 0, cuts_out[nparts] = A.nrows, and cuts_out[g] (0<g<nparts) is the boundary j whose
 * work prefix P[j] = sum_{i<j} w_i is closest to floor(g*W/nparts), ties to the smaller j, made
 * monotone. Part g owns rows [cuts_out[g], cuts_out[g+1]). flops_out = W. Synchronises. */
sg_status sg_partition(const sg_csr_view* A, const sg_csr_view* B, int nparts,
                       int64_t* cuts_out /*host, nparts+1*/, int64_t* flops_out /*host, nullable*/, void* stream);

/* Cost-weighted contiguous row blocks (reading R19): the rule of
 * sg_partition applied to the prefix of each row's MODELED path cost at the routing threshold thr
 * instead of its flops — Alg. 2's split (L216-L218) as a per-device vector (L106) that balances
 * predicted time. Row i costs 0 if w_i = 0, c_L(w_i, a_i, uh_i) if w_i <= thr, else c_H(w_i, a_i,
 * uh_i) (the cost model above; cm == NULL: sg_default_partition_model), where uh_i = min(w_i, ceil(w_i*U_c/W_c))
 * estimates u_i from the sample's per-class compression comp = {U_L, W_L, U_H, W_H} (host, 4;
 * sg_sample_report's U_est_L, W_est_L, U_est_H, W_est_H; uh_i = w_i where W_c = 0).
 * cuts_out (host, nparts+1); cost_out (host, nullable) = total modeled cost in ps. Synchronises.
 * Errors: INVALID_ARG (nparts < 1, thr < 0, negative comp, bad model), SHAPE, DTYPE. */
sg_status sg_partition_cost(const sg_csr_view* A, const sg_csr_view* B, int nparts, int64_t thr,
                            const sg_cost_model* cm, const int64_t* comp /*host, 4*/,
                            int64_t* cuts_out /*host, nparts+1*/, int64_t* cost_out /*host, nullable*/, void* stream);

/* Symbolic phase for rows [row_begin, row_end) at threshold thr (0 <= thr <= SG_CAP_L_MAX):
 * classifies rows (EMPTY w=0, LIGHT 0<w<=thr, HEAVY w>thr; L272-L274), computes u_i = nnz(C_i)
 * exactly and writes the local exclusive prefix C_row_ptr[0..row_end-row_begin] (device,
 * caller-owned; C_row_ptr[0] = 0). nnz_c_out (host) = C_row_ptr[last]; synchronises so the caller
 * can allocate C. *plan_out receives a plan owning the routing workspace for sg_numeric. */
sg_status sg_symbolic(const sg_csr_view* A, const sg_csr_view* B, int64_t thr, int64_t row_begin, int64_t row_end,
                      int64_t* C_row_ptr, int64_t* nnz_c_out /*host*/, sg_plan** plan_out /*host*/, void* stream);

/* Numeric phase: writes C_col (int32[nnz_c]) and C_val (dtype[nnz_c]) for the plan's rows, each
 * row at [C_row_ptr[i], C_row_ptr[i+1]) with ascending columns; c_ij = sum_k a_ik*b_kj accumulated
 * in fp64 (stored in the input dtype). A and B must be the views given to sg_symbolic. C_col must
 * be 4-byte aligned and C_val aligned to its element size (INVALID_ARG otherwise); no larger
 * alignment is assumed. `stream` may differ from the plan's stream: the plan's later frees are
 * ordered after this call's work. A plan is not thread-safe: do not run two sg_numeric calls on one
 * plan concurrently (they share its work counters). */
sg_status sg_numeric(sg_plan* plan, const sg_csr_view* A, const sg_csr_view* B,
                     int32_t* C_col, void* C_val, void* stream);

/* Assembly of the row-distributed C (Alg. 2 l.7, L224) over NCCL: rank r of the communicator owns
 * the plan rows [row_begin_r, row_end_r) (contiguous, in rank order, covering [0, n)). Gathers the
 * per-rank layout (allgather), writes the GLOBAL row_ptr (n+1, device) on every rank (allgatherv of
 * the local prefixes + offset fix-up) and, if gather_values != 0, the full C_col / C_val (nnz_total,
 * device) on every rank. nccl_comm is an ncclComm_t (e.g. ProcessGroupNCCL._comm_ptr()).
 * local_row_ptr / local_col / local_val are this rank's sg_symbolic / sg_numeric outputs.
 * row_ptr_cap = entries of C_row_ptr_global, nnz_cap = entries of C_col_global / C_val_global
 * (ignored when gather_values == 0): every rank's capacities are exchanged with the layout and the
 * call returns SHAPE on EVERY rank, before any output is written, if some rank's buffers are smaller
 * than n+1 / nnz_total. nnz_total_out (host). Synchronises. Errors: NCCL, SHAPE (ranges not
 * contiguous, or a capacity too small), INVALID_ARG. */
sg_status sg_gather(sg_plan* plan, void* nccl_comm, int gather_values,
                    const int64_t* local_row_ptr, const int32_t* local_col, const void* local_val,
                    int64_t* C_row_ptr_global, int64_t row_ptr_cap,
                    int32_t* C_col_global /*nullable*/, void* C_val_global /*nullable*/, int64_t nnz_cap,
                    int64_t* nnz_total_out /*host*/, void* stream);

/* ---- assembly through NCCL symmetric memory (Alg. 2 l.7) --------
 * The assembled C lives in NCCL symmetric windows on every rank (ncclMemAlloc + ncclCommWindowRegister,
 * NCCL_WIN_COLL_SYMMETRIC; NCCL >= 2.28 device API). Flow per rank: sg_symbolic -> sg_sym_c_layout
 * (where this rank's rows go) -> sg_numeric with C_col / C_val = the window buffers + that offset (the
 * numeric kernels write the rank's rows straight into its own window) -> sg_sym_c_assemble (one kernel
 * stores the rank's rows into every LSA peer's window over NVLink through ncclGetLsaPointer, then an
 * LSA barrier). No NCCL collective moves C. */
typedef struct sg_sym_c sg_sym_c;
/* Collective over nccl_comm: every rank passes the same n_rows (rows of the global C) and nnz_cap
 * (capacity of col / val). Errors: INVALID_ARG, OOM (ncclMemAlloc), NCCL. */
sg_status sg_sym_c_create(void* nccl_comm, int64_t n_rows, int64_t nnz_cap, sg_dtype dtype, sg_sym_c** out /*host*/);
/* This rank's copy of the assembled C: row_ptr int64[n_rows+1], col int32[nnz_cap], val dtype[nnz_cap]
 * (device; owned by the sg_sym_c, valid until sg_sym_c_destroy). Any output pointer may be NULL. */
sg_status sg_sym_c_buffers(const sg_sym_c* S, int64_t** row_ptr, int32_t** col, void** val);
/* Collective (one ncclAllGather of (row_begin, row_end, nnz) per rank; synchronises): this rank's first
 * global C entry (host) and the total nnz (host, nullable). Errors: SHAPE (blocks not contiguous from row
 * 0, rows != n_rows, or total > nnz_cap; the same on every rank), DTYPE, NCCL. */
sg_status sg_sym_c_layout(sg_sym_c* S, sg_plan* plan, int64_t* c_offset_out /*host*/, int64_t* nnz_total_out /*host*/,
                          void* stream);
/* Collective: pushes this rank's rows (local_row_ptr = the plan's sg_symbolic prefix, plus the global
 * offset; col / val from its window at the offset, written there by sg_numeric) into every LSA peer's
 * window, then an LSA barrier; on return every rank's buffers hold the whole C. Synchronises. */
sg_status sg_sym_c_assemble(sg_sym_c* S, sg_plan* plan, const int64_t* local_row_ptr, void* stream);
void sg_sym_c_destroy(sg_sym_c* S);
/* Stream-ordered device-to-device copy of `bytes` bytes (plumbing for bindings that hold raw device
 * pointers, e.g. copying out of a sg_sym_c window). Errors: INVALID_ARG, CUDA. */
sg_status sg_copy_device(void* dst, const void* src, int64_t bytes, void* stream);

/* ---- the HH-CPU four-block variant (PAPER Alg. 3, Section V-A) ------
 * A row is HIGH dense iff it has more than t non-zeros (L274). C = A_H B_H + A_H B_L + A_L B_H + A_L B_L:
 * the four products run on the hot path (sg_symbolic / sg_numeric); Phase IV adds two results P + Q as
 * the product [P Q] * [I; I] (the accumulators add equal columns, structural zeros kept). The Python
 * binding's spgemm_hh() / hh_threshold() drive the whole algorithm. */
/* Phase I: keeps the rows of M with (nnz > t) == (high != 0), empties the others (row ids unchanged).
 * rp_out int64[nrows+1]; col_out / val_out capacity M.nnz (device, caller-owned); nnz_out (host).
 * Synchronises. Errors: INVALID_ARG, DTYPE, OVERFLOW. */
sg_status sg_hh_filter(const sg_csr_view* M, int64_t t, int high, int64_t* rp_out, int32_t* col_out, void* val_out,
                       int64_t* nnz_out /*host*/, void* stream);
/* [P Q]: nrows x (P.ncols + Q.ncols), row i = P_i then Q_i with columns shifted by P.ncols. Outputs:
 * rp_out int64[nrows+1], col_out / val_out capacity P.nnz + Q.nnz. Errors: SHAPE (row counts), DTYPE,
 * OVERFLOW (P.ncols + Q.ncols > INT32_MAX). */
sg_status sg_hh_hstack(const sg_csr_view* P, const sg_csr_view* Q, int64_t* rp_out, int32_t* col_out, void* val_out,
                       void* stream);
/* [I; I] (2p x p): row k holds (k mod p, 1). rp_out int64[2p+1], col_out int32[2p], val_out dtype[2p]. */
sg_status sg_hh_identity2(int64_t p, sg_dtype dtype, int64_t* rp_out, int32_t* col_out, void* val_out, void* stream);
/* Phase I Sample (L285-L287; reading R20): the principal sub-matrix A' = A[S, S] of a square A on
 * S = { i : h(seed, SAMPLE, i) < floor(f 2^64) } (f = 1/sqrt(n): the paper's sqrt(n) x sqrt(n) sample),
 * columns relabelled by rank. Outputs (device, capacity n / n+1 / A.nnz): rows_out = S ascending, rp_out
 * (s+1), col_out (relabelled), pos_out (each entry's position in A), val_out (its value; nullable);
 * s_out, nnz_out (host). Synchronises. Errors: SHAPE (A not square), INVALID_ARG. */
sg_status sg_hh_sample(const sg_csr_view* A, uint64_t seed, double f, int64_t* rows_out, int64_t* rp_out,
                       int32_t* col_out, int64_t* pos_out, void* val_out /*nullable*/, int64_t* s_out /*host*/,
                       int64_t* nnz_out /*host*/, void* stream);

/* Sample ("a smaller instance"; R3): A_S = the rows `rows` (device int64[nrows], any
 * order, each in [0, A.nrows)) of A as a CSR with all of A's columns (B stays whole). Outputs (device):
 * rp_out int64[nrows+1], col_out / val_out of capacity `cap` entries; *nnz_out (host) = nnz(A_S), written
 * even when it exceeds cap. Synchronises (the row-id check and nnz read back). Errors: INVALID_ARG (a row id
 * out of range, null pointers), SHAPE (nnz(A_S) > cap: nothing copied; call again with the returned size).
 * The measured-mode Identify of the Python binding (measured_threshold) times the hot path on A_S B. */
sg_status sg_gather_rows(const sg_csr_view* A, const int64_t* rows, int64_t nrows, int64_t* rp_out, int32_t* col_out,
                         void* val_out, int64_t cap, int64_t* nnz_out /*host*/, void* stream);

/* The host-only arithmetic of sg_gather (no device work, usable without a GPU): lay holds the
 * per-rank (row_begin, row_end, nnz) triples in rank order. Checks that the blocks are contiguous
 * from row 0 (SHAPE otherwise) and writes begin[r] (first row of rank r, nranks entries), off[r]
 * (first C entry of rank r; nranks+1 entries, off[nranks] = total), the row count n and the total. */
sg_status sg_gather_layout(const int64_t* lay /*host, 3*nranks*/, int nranks, int64_t* begin /*host*/,
                           int64_t* off /*host*/, int64_t* n_out /*host*/, int64_t* total_out /*host*/);

/* Plan introspection for tests and reports. */
sg_status sg_plan_get_info(const sg_plan* plan, sg_plan_info* out /*host*/);
/* Row classes of the plan's rows: 0 EMPTY, 1 LIGHT, 2 HEAVY (device int8, row_end-row_begin). */
sg_status sg_plan_get_classes(const sg_plan* plan, int8_t* cls_out, void* stream);
/* The plan's w_i (device int64, row_end-row_begin). */
sg_status sg_plan_get_work(const sg_plan* plan, int64_t* w_out, void* stream);

/* Destroys a plan (NULL is allowed). Frees its workspace stream-ordered on the plan's stream. */
void sg_plan_destroy(sg_plan* plan);

/* The sample set S itself (device int64 row ids in ascending order, capacity rows_cap) and its
 * size (host), for parity tests of the sampler. Rows in [row_begin, row_end). */
sg_status sg_sample_rows(int64_t row_begin, int64_t row_end, double sample_frac, uint64_t seed,
                         int64_t* rows_out, int64_t rows_cap, int64_t* count_out /*host*/, void* stream);

/* ---- instrumentation (bench.py's measured kernel durations) -------------------
 * Every kernel launch is counted. With profiling enabled, a CUDA event pair is recorded on the
 * launching stream around each launch; sg_profile_read (after the stream is synchronised) copies
 * up to max records: names as 32-byte NUL-terminated strings, durations in ms. */
void sg_profile_enable(int on);
int64_t sg_launch_count(void);
int64_t sg_profile_count(void);
int64_t sg_profile_read(char* names /*host, 32*max bytes, nullable*/, double* ms /*host, max, nullable*/, int64_t max);
void sg_profile_reset(void);

#ifdef __cplusplus
}
#endif
#endif /* SG_H */
