/*
 * oracle/oracle.cpp — TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct CPU implementation of what the hot path computes, written
 * from the paper (Mallipeddi et al., "Nearly Balanced Work Partitioning for Heterogeneous
 * Algorithms", ICPP 2017; /root/reference/PAPER.md, cited as "PAPER Lnnn") and the readings
 * recorded in DESIGN.md §2. Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library. It shares no code, header, table or helper
 * with the CUDA path (paper_conf_icpp_hardhikbrks17_b200/), and neither includes the other.
 *
 * Every function follows the plain definition of the quantity it computes — no blocking,
 * fusion or reordering — so it can be checked against the paper by eye:
 *
 *   O1 oracle_spgemm_count / oracle_spgemm_fill
 *        Gustavson row-row SpGEMM, C_i = sum_{k in A_i} a_ik * B_k, with a sorted-map
 *        (std::map<int32, double>) accumulator per row. PAPER L74 (Gustavson [13]), Alg. 2
 *        l.5-6 (L222-L223). Structural semantics: an entry exists iff some product exists,
 *        even if its value sums to zero (reading R9). Accumulation in fp64 from the
 *        (possibly fp32) inputs.
 *        oracle_spgemm_moments: the same accumulator, reporting per row u_i and the sums of c, c^2,
 *        c^3 over its columns (mod 2^64) — a structure digest for C that does not fit in host memory.
 *   O2 oracle_row_work
 *        L_AB = A x V_B with V_B[k] = nnz(B_k): w_i = sum_{k in A_i} nnz(B_k), the work volume
 *        of row i (Alg. 2 l.1 L215).
 *   O3 oracle_partition
 *        Alg. 2 l.2-4 (L216-L218) generalised to G parts (L106 "threshold vector"): cut_g is
 *        the row boundary j whose prefix P[j] = sum_{i<j} w_i is closest to floor(g*W/G),
 *        ties to the smaller j, forced monotone; part g owns rows [cut_g, cut_{g+1}).
 *   Sampler  oracle_sample_rows
 *        Uniform sampling ("we limit ourselves to uniform sampling"), Bernoulli(f)
 *        per row through a counter-based SplitMix64 hash (reading R4). This file
 *        carries its own copy of the generator, independent of the CUDA side's copy.
 *   O4 oracle_cost_L / oracle_cost_H / oracle_J / oracle_threshold
 *        "Identify": evaluate candidate thresholds on the (sampled) rows and
 *        keep the best. Cost J(t;R) = sum_{i in R, 0<w_i<=t} c_L(i) + sum_{i in R, w_i>t} c_H(i)
 *        (heavy iff "more than t", L272-L274; equality -> light, reading R13), candidates
 *        {0} u {w_i > 0} clipped to t <= cap_L, thr = smallest minimiser. "Extrapolate" is the
 *        identity (L236 r = r'; whole rows sampled, reading R3).
 *   HH oracle_hh_block_count / oracle_hh_block_fill / oracle_hh_sample / oracle_hh_extrapolate
 *        The HH-CPU four-block decomposition (Alg. 3): C = sum over (X, Y) in {H, L}^2 of
 *        A_X B_Y, high iff more than t non-zeros (L274); the sqrt(n)-row sampler with relabelled columns
 *        (L285-L287; reading R20) and the extrapolation t_A = t_s^2 (L291).
 *   O6 oracle_heavy_share
 *        r(t) = 100 * sum_{w_i > t} w_i / W, the split percentage of Alg. 2 (L204, L208).
 */
#include <cstdint>
#include <cstring>
#include <cmath>
#include <map>
#include <vector>
#include <algorithm>
#ifdef _OPENMP
#include <omp.h>
#endif

typedef __int128 i128;

namespace {

// ---- the oracle's own SplitMix64 (reading R4) ----------------------------------
inline uint64_t splitmix64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}
inline uint64_t hash3(uint64_t seed, uint64_t tag, uint64_t j) {
    return splitmix64(seed ^ splitmix64(tag ^ splitmix64(j)));
}
const uint64_t TAG_SAMPLE = 0x53414d504c450001ULL;

inline double load_val(const void* v, int is_f32, int64_t q) {
    return is_f32 ? (double)((const float*)v)[q] : ((const double*)v)[q];
}

}  // namespace

extern "C" {

int oracle_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

uint64_t oracle_hash(uint64_t seed, uint64_t tag, uint64_t j) { return hash3(seed, tag, j); }
uint64_t oracle_tag_sample(void) { return TAG_SAMPLE; }

// ---- O2: w_i = sum_{k in A_i} nnz(B_k) --------------------------------------
void oracle_row_work(int64_t n, const int64_t* Arp, const int32_t* Acol, const int64_t* Brp, int64_t* w) {
    #pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t i = 0; i < n; ++i) {
        int64_t s = 0;
        for (int64_t p = Arp[i]; p < Arp[i + 1]; ++p) {
            int32_t k = Acol[p];
            s += Brp[k + 1] - Brp[k];
        }
        w[i] = s;
    }
}

// ---- O1: Gustavson with a sorted-map accumulator -----------------
// Counts u_i = |union_{k in A_i} cols(B_k)| for each listed row.
void oracle_spgemm_count(const int64_t* Arp, const int32_t* Acol,
                         const int64_t* Brp, const int32_t* Bcol,
                         int64_t nsel, const int64_t* rows, int64_t* u) {
    #pragma omp parallel for schedule(dynamic, 1)
    for (int64_t s = 0; s < nsel; ++s) {
        int64_t i = rows[s];
        std::map<int32_t, double> acc;
        for (int64_t p = Arp[i]; p < Arp[i + 1]; ++p) {
            int32_t k = Acol[p];
            for (int64_t q = Brp[k]; q < Brp[k + 1]; ++q) acc[Bcol[q]] += 0.0;
        }
        u[s] = (int64_t)acc.size();
    }
}

// Structure moments of the listed rows (for parity at sizes whose C does not fit host memory):
// m[4s..4s+3] = (u_i, sum c, sum c^2, sum c^3) over the columns c of C_i = the keys of the same
// sorted-map accumulator, sums modulo 2^64 (unsigned wrap-around).
void oracle_spgemm_moments(const int64_t* Arp, const int32_t* Acol, const int64_t* Brp, const int32_t* Bcol,
                           int64_t nsel, const int64_t* rows, uint64_t* m) {
    #pragma omp parallel for schedule(dynamic, 1)
    for (int64_t s = 0; s < nsel; ++s) {
        int64_t i = rows[s];
        std::map<int32_t, double> acc;
        for (int64_t p = Arp[i]; p < Arp[i + 1]; ++p) {
            int32_t k = Acol[p];
            for (int64_t q = Brp[k]; q < Brp[k + 1]; ++q) acc[Bcol[q]] += 0.0;
        }
        uint64_t s1 = 0, s2 = 0, s3 = 0;
        for (const auto& kv : acc) {
            uint64_t c = (uint64_t)(uint32_t)kv.first;
            s1 += c;
            s2 += c * c;
            s3 += c * c * c;
        }
        m[4 * s] = (uint64_t)acc.size();
        m[4 * s + 1] = s1;
        m[4 * s + 2] = s2;
        m[4 * s + 3] = s3;
    }
}

// Fills the listed rows: row s is written at [out_ptr[s], out_ptr[s+1]) with ascending columns.
void oracle_spgemm_fill(const int64_t* Arp, const int32_t* Acol, const void* Aval, int A_f32,
                        const int64_t* Brp, const int32_t* Bcol, const void* Bval, int B_f32,
                        int64_t nsel, const int64_t* rows, const int64_t* out_ptr,
                        int32_t* col_out, double* val_out, double* absmag_out /*nullable*/) {
    #pragma omp parallel for schedule(dynamic, 1)
    for (int64_t s = 0; s < nsel; ++s) {
        int64_t i = rows[s];
        std::map<int32_t, double> acc;
        std::map<int32_t, double> mag;  // sum_k |a_ik b_kj|, the tolerance scale (R16)
        for (int64_t p = Arp[i]; p < Arp[i + 1]; ++p) {
            int32_t k = Acol[p];
            double a = load_val(Aval, A_f32, p);
            for (int64_t q = Brp[k]; q < Brp[k + 1]; ++q) {
                double b = load_val(Bval, B_f32, q);
                acc[Bcol[q]] += a * b;
                if (absmag_out) mag[Bcol[q]] += std::fabs(a * b);
            }
        }
        int64_t o = out_ptr[s];
        for (const auto& kv : acc) {
            col_out[o] = kv.first;
            val_out[o] = kv.second;
            if (absmag_out) absmag_out[o] = mag[kv.first];
            ++o;
        }
    }
}

// ---- Sampler: S = { i : h(seed, SAMPLE, i) < T_f }  (reading R4) -------------
// T_f = floor(f * 2^64) computed here from f; f >= 1 selects every row. Returns |S|.
int64_t oracle_sample_rows(int64_t row_begin, int64_t row_end, uint64_t seed, double f, int64_t* rows_out) {
    int64_t c = 0;
    bool all = f >= 1.0;
    uint64_t Tf = all ? 0 : (uint64_t)std::ldexp(f, 64);
    for (int64_t i = row_begin; i < row_end; ++i)
        if (all || hash3(seed, TAG_SAMPLE, (uint64_t)i) < Tf) rows_out[c++] = i;
    return c;
}

// ---- O4: per-row path costs in integer picoseconds (DESIGN.md §4 cost model) -------------
typedef struct {
    int64_t kappa_L, lambda_L, sigma_L, rho_L;      // light: kappa + lambda*w + sigma*u*ceil(log2 max(u,2)) + rho*u
    int64_t kappa_H, lambda_H, tau_H, mu_H;         // heavy: kappa + lambda*w + tau*a*R(u) + mu*u
    int64_t tiles_fixed;                            // R(u) = tiles_fixed if capu == 0
    int64_t capu;                                   // else R(u) = max(1, tiles_fixed, ceil(u / capu))
    int64_t cap_L;                                  // largest admissible threshold (light capacity)
} oracle_cost_model;

static int64_t ceil_log2_max2(int64_t u) {
    int64_t x = u < 2 ? 2 : u;
    int64_t l = 0;
    while (((int64_t)1 << l) < x) ++l;
    return l;
}

int64_t oracle_cost_L(const oracle_cost_model* cm, int64_t w, int64_t a, int64_t u) {
    (void)a;
    return cm->kappa_L + cm->lambda_L * w + cm->sigma_L * u * ceil_log2_max2(u) + cm->rho_L * u;
}

int64_t oracle_cost_H(const oracle_cost_model* cm, int64_t w, int64_t a, int64_t u) {
    int64_t R = cm->capu == 0 ? cm->tiles_fixed
                              : std::max<int64_t>(std::max<int64_t>(1, cm->tiles_fixed), (u + cm->capu - 1) / cm->capu);
    return cm->kappa_H + cm->lambda_H * w + cm->tau_H * a * R + cm->mu_H * u;
}

// J(t; R) by its definition, one candidate at a time: rows with w == 0 are EMPTY (cost 0,
// reading R7), 0 < w <= t LIGHT, w > t HEAVY. Result as a 128-bit integer (hi, lo).
void oracle_J(const oracle_cost_model* cm, int64_t nrows, const int64_t* w, const int64_t* a, const int64_t* u,
              int64_t t, int64_t* J_hi, uint64_t* J_lo) {
    i128 J = 0;
    for (int64_t r = 0; r < nrows; ++r) {
        if (w[r] == 0) continue;
        if (w[r] <= t) J += oracle_cost_L(cm, w[r], a[r], u[r]);
        else J += oracle_cost_H(cm, w[r], a[r], u[r]);
    }
    *J_hi = (int64_t)(J >> 64);
    *J_lo = (uint64_t)J;
}

// thr(R) = min { t in cands : J(t;R) = min J }, cands = {0} u {w_r > 0 : w_r <= cap_L}.
// Evaluated in ascending-w order: J(t) = sum_{w>0} c_H + sum_{0<w_r<=t} (c_L - c_H).
int64_t oracle_threshold(const oracle_cost_model* cm, int64_t nrows, const int64_t* w, const int64_t* a,
                         const int64_t* u, int64_t* Jmin_hi, uint64_t* Jmin_lo) {
    std::vector<int64_t> idx;
    idx.reserve(nrows);
    i128 base = 0;
    for (int64_t r = 0; r < nrows; ++r) {
        if (w[r] == 0) continue;
        base += oracle_cost_H(cm, w[r], a[r], u[r]);
        idx.push_back(r);
    }
    std::sort(idx.begin(), idx.end(), [&](int64_t x, int64_t y) { return w[x] < w[y]; });
    i128 best = base;  // t = 0: every non-empty row heavy
    int64_t best_t = 0;
    i128 J = base;
    size_t k = 0;
    while (k < idx.size()) {
        int64_t t = w[idx[k]];
        if (t > cm->cap_L) break;
        while (k < idx.size() && w[idx[k]] == t) {  // all rows with w == t turn light together
            int64_t r = idx[k];
            J += (i128)oracle_cost_L(cm, w[r], a[r], u[r]) - (i128)oracle_cost_H(cm, w[r], a[r], u[r]);
            ++k;
        }
        if (J < best) { best = J; best_t = t; }
    }
    if (Jmin_hi) *Jmin_hi = (int64_t)(best >> 64);
    if (Jmin_lo) *Jmin_lo = (uint64_t)best;
    return best_t;
}

// ---- O3: work-prefix partition into G contiguous parts -----------
void oracle_partition(int64_t n, const int64_t* w, int G, int64_t* cuts) {
    std::vector<int64_t> P(n + 1, 0);
    for (int64_t i = 0; i < n; ++i) P[i + 1] = P[i] + w[i];
    i128 W = P[n];
    cuts[0] = 0;
    for (int g = 1; g < G; ++g) {
        int64_t target = (int64_t)((W * g) / G);
        // closest prefix, ties -> smaller index (linear scan: the plain definition)
        int64_t bestj = 0;
        i128 bestd = -1;
        for (int64_t j = 0; j <= n; ++j) {
            i128 d = (i128)P[j] - target;
            if (d < 0) d = -d;
            if (bestd < 0 || d < bestd) { bestd = d; bestj = j; }
        }
        cuts[g] = std::max(bestj, cuts[g - 1]);
    }
    cuts[G] = n;
}

// ---- O3': cost-weighted partition (reading R19) -----------
// Alg. 2 balances L_AB, i.e. flops (L215-L218); the paper's "threshold vector" (L106) splits by
// what each device will SPEND. Here each row's modeled cost is the path cost of O4 at the routing
// threshold thr: c(i) = 0 if w_i = 0, c_L(w_i, a_i, uh_i) if w_i <= thr, else c_H(w_i, a_i, uh_i),
// with u_i (unknown before the symbolic pass) estimated from the sample by its class's compression:
// uh_i = min(w_i, ceil(w_i * U_c / W_c)) for (U_c, W_c) = (sum u, sum w) over the SAMPLED rows of
// class c (uh_i = w_i when W_c = 0). Cuts: the O3 rule on the prefix of c.
int64_t oracle_row_cost(const oracle_cost_model* cm, int64_t thr, const int64_t* comp /*U_L, W_L, U_H, W_H*/,
                        int64_t w, int64_t a) {
    if (w == 0) return 0;
    const bool light = w <= thr;
    const int64_t U = light ? comp[0] : comp[2], Wc = light ? comp[1] : comp[3];
    int64_t uh = w;
    if (Wc > 0) {
        i128 q = ((i128)w * U + Wc - 1) / Wc;
        if (q < uh) uh = (int64_t)q;
    }
    return light ? oracle_cost_L(cm, w, a, uh) : oracle_cost_H(cm, w, a, uh);
}

void oracle_partition_cost(const oracle_cost_model* cm, int64_t thr, const int64_t* comp, int64_t n,
                           const int64_t* w, const int64_t* a, int G, int64_t* cuts, int64_t* cost_total) {
    std::vector<int64_t> c(n);
    i128 tot = 0;
    for (int64_t i = 0; i < n; ++i) { c[i] = oracle_row_cost(cm, thr, comp, w[i], a[i]); tot += c[i]; }
    oracle_partition(n, c.data(), G, cuts);
    if (cost_total) *cost_total = (int64_t)tot;
}

// ---- HH (Alg. 3 "HH-CPU") ---------------------------------
// A row is HIGH dense iff it has MORE than t non-zeros (L274). With A_H / A_L the high / low rows of A
// and B_H / B_L those of B, C = A B = A_H B_H + A_H B_L + A_L B_H + A_L B_L where X_Y (X, Y in {H, L})
// restricts row i to class X and its k entries to B rows of class Y (Alg. 3 Phases II-III), and Phase IV
// adds the blocks. oracle_hh_block_fill writes block (xa, yb) (0 = L, 1 = H) of the listed rows with
// the same sorted-map accumulator as O1: rows of the other class, and k entries of the other class,
// contribute nothing (an empty row stays empty).
void oracle_hh_block_count(const int64_t* Arp, const int32_t* Acol, const int64_t* Brp, const int32_t* Bcol,
                           int64_t t, int xa, int yb, int64_t nsel, const int64_t* rows, int64_t* u) {
    #pragma omp parallel for schedule(dynamic, 1)
    for (int64_t s = 0; s < nsel; ++s) {
        int64_t i = rows[s];
        std::map<int32_t, double> acc;
        if (((Arp[i + 1] - Arp[i]) > t) == (xa == 1)) {
            for (int64_t p = Arp[i]; p < Arp[i + 1]; ++p) {
                int32_t k = Acol[p];
                if (((Brp[k + 1] - Brp[k]) > t) != (yb == 1)) continue;
                for (int64_t q = Brp[k]; q < Brp[k + 1]; ++q) acc[Bcol[q]] += 0.0;
            }
        }
        u[s] = (int64_t)acc.size();
    }
}

void oracle_hh_block_fill(const int64_t* Arp, const int32_t* Acol, const void* Aval, int A_f32,
                          const int64_t* Brp, const int32_t* Bcol, const void* Bval, int B_f32,
                          int64_t t, int xa, int yb, int64_t nsel, const int64_t* rows, const int64_t* out_ptr,
                          int32_t* col_out, double* val_out) {
    #pragma omp parallel for schedule(dynamic, 1)
    for (int64_t s = 0; s < nsel; ++s) {
        int64_t i = rows[s];
        std::map<int32_t, double> acc;
        if (((Arp[i + 1] - Arp[i]) > t) == (xa == 1)) {
            for (int64_t p = Arp[i]; p < Arp[i + 1]; ++p) {
                int32_t k = Acol[p];
                if (((Brp[k + 1] - Brp[k]) > t) != (yb == 1)) continue;
                double a = load_val(Aval, A_f32, p);
                for (int64_t q = Brp[k]; q < Brp[k + 1]; ++q) acc[Bcol[q]] += a * load_val(Bval, B_f32, q);
            }
        }
        int64_t o = out_ptr[s];
        for (const auto& kv : acc) { col_out[o] = kv.first; val_out[o] = kv.second; ++o; }
    }
}

// Phase I Sample of Section V-A (L285-L287): A' keeps ~sqrt(n) rows of A chosen uniformly at random
// (Bernoulli(1/sqrt(n)) per row through the sampler hash, reading R4) and, in each kept row, the
// elements whose column is itself a kept row index, relabelled by rank so that A' is s x s with
// s = |kept rows| ("column indices transformed so that the column indices are within 1 to sqrt(n)";
// DESIGN.md reading R20). Writes the kept rows' ids (rows_out, s entries) and A' (rp_out s+1; col_out,
// pos_out = source position in A, up to nnz(A) entries). Returns s.
int64_t oracle_hh_sample(int64_t n, const int64_t* Arp, const int32_t* Acol, uint64_t seed, double f,
                         int64_t* rows_out, int64_t* rp_out, int32_t* col_out, int64_t* pos_out) {
    const uint64_t Tf = f >= 1.0 ? ~0ull : (uint64_t)std::ldexp(f, 64);
    std::vector<int64_t> rank(n, -1);
    int64_t s = 0;
    for (int64_t i = 0; i < n; ++i)
        if (f >= 1.0 || hash3(seed, TAG_SAMPLE, (uint64_t)i) < Tf) { rank[i] = s; rows_out[s++] = i; }
    int64_t o = 0;
    rp_out[0] = 0;
    for (int64_t r = 0; r < s; ++r) {
        int64_t i = rows_out[r];
        for (int64_t p = Arp[i]; p < Arp[i + 1]; ++p) {
            int32_t j = Acol[p];
            if (j < n && rank[j] >= 0) { col_out[o] = (int32_t)rank[j]; pos_out[o] = p; ++o; }
        }
        rp_out[r + 1] = o;
    }
    return s;
}

// Phase I Extrapolate (L291): the off-line relation the paper found for spmm, t_A = t_s * t_s.
int64_t oracle_hh_extrapolate(int64_t t_s) { return t_s * t_s; }

// ---- O6: r(t) = 100 * sum_{w_i > t} w_i / W  (split percentage) -------
double oracle_heavy_share(int64_t n, const int64_t* w, int64_t t) {
    i128 W = 0, H = 0;
    for (int64_t i = 0; i < n; ++i) { W += w[i]; if (w[i] > t) H += w[i]; }
    if (W == 0) return 0.0;
    return 100.0 * (double)H / (double)W;
}

}  // extern "C"
