/*
 * sr_oracle.c -- fp64 CPU oracle for softmax-recomposed multi-head attention.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  It shares no code, header, table or constant
 * generator with the CUDA path in paper_conf_iiswc_choilkha22_b200/ (task rule 3).
 *
 * What it computes (PAPER.md = "Accelerating Transformer Networks through Recomposing Softmax
 * Layers", Choi et al., IISWC 2022):
 *
 *   or_attention / or_attention_rows -- the attention layer exactly as PAPER.md L51-L53 defines
 *     it: x_j = scale * <q_i, k_j> (MatMul then divide by sqrt(D_head)), masked elements set to
 *     -inf (the mask layer), safe softmax of Eq. (1):
 *         m = max_j x_j,  d = sum_j e^{x_j - m},  y_j = e^{x_j - m} / d,
 *     then the MatMul with V: o_i = sum_j y_j v_j.  Masked terms are exactly zero so they are
 *     skipped.  A row whose every element is masked outputs 0 (reading R9; the paper is
 *     silent).
 *
 *   or_recomposed -- the decomposed softmax of Eq. (2) and its three
 *     sub-layers in the paper's order and notation:
 *       LS: per sub-vector X_k of width T:  m'_k = max_i x_{k,i},  d'_k = sum_j e^{x_{k,j} - m'_k},
 *           X'_{k,i} = e^{x_{k,i} - m'_k}                     (unnormalised; reading R1)
 *       IR: m = max_k m'_k,  d = sum_k e^{m'_k - m} d'_k,  r'_k = e^{m'_k - m} / d
 *           (Eq. 2 numerator read as e^{m'_k - m}: reading R2)
 *       GS: y_{k,i} = X'_{k,i} * r'_k
 *     followed by the same MatMul with V.  A fully masked sub-vector has m'_k = -inf, d'_k = 0 and
 *     r'_k = 0 (reading R8); (-inf) - (-inf) is never evaluated.
 *
 * Masks (the "certain criteria" of PAPER.md L53; readings R7, R13, R14 in DESIGN.md):
 *   kv_len (optional, any kind): key j allowed only if j < kv_len[b]    (key-side suffix padding)
 *   causal (optional, any kind): key j allowed only if j <= i
 *   OR_MASK_NONE   dense
 *   OR_MASK_BLOCK  block-sparse: allowed iff block (i/blk, j/blk) is listed
 *                  in the CSR row of the head's layout
 *   OR_MASK_WINDOW Longformer: allowed iff |i-j| <= window/2 or i < n_global or j < n_global
 *   OR_MASK_ELEM   explicit element mask [B*H][S][S] (brute-force tests)
 *
 * Everything is plain loops in fp64 on fp64 inputs (the dtype-rounded values upcast exactly).
 * Rows are independent, so rows are split across pthreads; nothing else is reordered.
 */
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <unistd.h>

enum { OR_MASK_NONE = 0, OR_MASK_BLOCK = 1, OR_MASK_WINDOW = 2, OR_MASK_ELEM = 3 };

typedef struct {
    int kind;
    int causal;
    const int32_t* kv_len;  /* [B] or NULL */
    int block;              /* OR_MASK_BLOCK */
    int layout_heads;       /* 1 or H */
    const int32_t* row_ptr; /* [layout_heads][S/block + 1], absolute offsets into col_idx */
    const int32_t* col_idx;
    int window;             /* OR_MASK_WINDOW */
    int n_global;
    const uint8_t* elem;    /* OR_MASK_ELEM: [B*H][S][S] */
} or_mask;

typedef struct {
    const double *q, *k, *v;
    int B, H, S, D;
    double scale;
    const or_mask* m;
} or_problem;

/* The mask layer: is element (i, j) of head (b, h) kept?  PAPER.md L53. */
static int or_allowed(const or_problem* p, int b, int h, int i, int j)
{
    const or_mask* m = p->m;
    if (m->kv_len && j >= m->kv_len[b]) return 0;
    if (m->causal && j > i) return 0;
    switch (m->kind) {
    case OR_MASK_NONE:
        return 1;
    case OR_MASK_BLOCK: {
        int nb = p->S / m->block;
        int lh = (m->layout_heads == 1) ? 0 : h;
        const int32_t* rp = m->row_ptr + (size_t)lh * (nb + 1);
        int r = i / m->block, c = j / m->block;
        for (int32_t t = rp[r]; t < rp[r + 1]; ++t)
            if (m->col_idx[t] == c) return 1;
        return 0;
    }
    case OR_MASK_WINDOW:
        return abs(i - j) <= m->window / 2 || i < m->n_global || j < m->n_global;
    case OR_MASK_ELEM:
        return m->elem[(((size_t)b * p->H + h) * p->S + i) * p->S + j] != 0;
    }
    return 0;
}

/* x_j = scale * <q_i, k_j>   (MatMul of Q and K^T, divided by sqrt(D_head)) */
static double or_score(const or_problem* p, size_t bh, int i, int j)
{
    const double* qi = p->q + (bh * p->S + i) * p->D;
    const double* kj = p->k + (bh * p->S + j) * p->D;
    double s = 0.0;
    for (int c = 0; c < p->D; ++c) s += qi[c] * kj[c];
    return p->scale * s;
}

/* One output row by the textbook definition: Eq. (1) safe softmax, then y . V. */
static void or_row_textbook(const or_problem* p, size_t bh, int i, double* x, double* o)
{
    int b = (int)(bh / p->H), h = (int)(bh % p->H);
    int S = p->S, D = p->D;
    double m = -INFINITY;
    for (int j = 0; j < S; ++j) {
        if (or_allowed(p, b, h, i, j)) {
            x[j] = or_score(p, bh, i, j);
            if (x[j] > m) m = x[j];
        } else {
            x[j] = -INFINITY;
        }
    }
    for (int c = 0; c < D; ++c) o[c] = 0.0;
    if (m == -INFINITY) return; /* fully masked row -> 0 (reading R9) */
    double d = 0.0;
    for (int j = 0; j < S; ++j)
        if (x[j] != -INFINITY) d += exp(x[j] - m);
    for (int j = 0; j < S; ++j) {
        if (x[j] == -INFINITY) continue;
        double y = exp(x[j] - m) / d;
        const double* vj = p->v + (bh * S + j) * D;
        for (int c = 0; c < D; ++c) o[c] += y * vj[c];
    }
}

/* One output row by the decomposition of Eq. (2): LS, IR, GS, then y . V.
 * mp/dp/rp (optional) receive m'_k, d'_k, r'_k with stride S between sub-vectors. */
static void or_row_recomposed(const or_problem* p, size_t bh, int i, int T, double* x, double* o,
                              double* mp, double* dp, double* rp)
{
    int b = (int)(bh / p->H), h = (int)(bh % p->H);
    int S = p->S, D = p->D;
    int Nsv = (S + T - 1) / T;
    for (int j = 0; j < S; ++j)
        x[j] = or_allowed(p, b, h, i, j) ? or_score(p, bh, i, j) : -INFINITY;

    double* mk = (double*)malloc(sizeof(double) * Nsv * 3);
    double* dk = mk + Nsv;
    double* rk = dk + Nsv;
    /* LS: local max and local sum per sub-vector X_k */
    for (int k = 0; k < Nsv; ++k) {
        double m_loc = -INFINITY;
        for (int j = k * T; j < (k + 1) * T && j < S; ++j)
            if (x[j] > m_loc) m_loc = x[j];
        double d_loc = 0.0;
        if (m_loc != -INFINITY)
            for (int j = k * T; j < (k + 1) * T && j < S; ++j)
                if (x[j] != -INFINITY) d_loc += exp(x[j] - m_loc);
        mk[k] = m_loc;
        dk[k] = d_loc;
    }
    /* IR: global max, global normaliser, reconstruction factors */
    double m = -INFINITY;
    for (int k = 0; k < Nsv; ++k)
        if (mk[k] > m) m = mk[k];
    double d = 0.0;
    for (int k = 0; k < Nsv; ++k)
        if (mk[k] != -INFINITY) d += exp(mk[k] - m) * dk[k];
    for (int k = 0; k < Nsv; ++k)
        rk[k] = (mk[k] == -INFINITY || m == -INFINITY) ? 0.0 : exp(mk[k] - m) / d;
    /* GS + MatMul: y_{k,i} = X'_{k,i} * r'_k;  o = sum_j y_j v_j */
    for (int c = 0; c < D; ++c) o[c] = 0.0;
    for (int k = 0; k < Nsv; ++k) {
        if (rk[k] == 0.0) continue;
        for (int j = k * T; j < (k + 1) * T && j < S; ++j) {
            if (x[j] == -INFINITY) continue;
            double y = exp(x[j] - mk[k]) * rk[k];
            const double* vj = p->v + (bh * S + j) * D;
            for (int c = 0; c < D; ++c) o[c] += y * vj[c];
        }
    }
    if (mp)
        for (int k = 0; k < Nsv; ++k) {
            mp[(size_t)k * S] = mk[k];
            dp[(size_t)k * S] = dk[k];
            rp[(size_t)k * S] = rk[k];
        }
    free(mk);
}

/* ------------------------------------------------------------------ row-parallel driver */

typedef struct {
    const or_problem* p;
    const int64_t* rows; /* flat row ids bh*S + i, or NULL = all rows */
    int64_t n_rows, begin, end;
    double* out;         /* [n_rows][D] (rows given) or [B*H*S][D] */
    int T;               /* 0 = textbook, else recomposed with sub-vector width T */
    double *mp, *dp, *rp;/* recomposed only: [B*H][Nsv][S] or NULL */
} or_job;

static void* or_worker(void* arg)
{
    or_job* jb = (or_job*)arg;
    const or_problem* p = jb->p;
    double* x = (double*)malloc(sizeof(double) * p->S);
    int Nsv = jb->T > 0 ? (p->S + jb->T - 1) / jb->T : 0;
    for (int64_t r = jb->begin; r < jb->end; ++r) {
        int64_t flat = jb->rows ? jb->rows[r] : r;
        size_t bh = (size_t)(flat / p->S);
        int i = (int)(flat % p->S);
        double* o = jb->out + (size_t)r * p->D;
        if (jb->T <= 0) {
            or_row_textbook(p, bh, i, x, o);
        } else {
            size_t base = bh * (size_t)Nsv * p->S + i;
            or_row_recomposed(p, bh, i, jb->T, x, o, jb->mp ? jb->mp + base : NULL,
                              jb->dp ? jb->dp + base : NULL, jb->rp ? jb->rp + base : NULL);
        }
    }
    free(x);
    return NULL;
}

static int or_run(const or_problem* p, const int64_t* rows, int64_t n_rows, double* out, int T,
                  double* mp, double* dp, double* rp, int nthreads)
{
    if (nthreads <= 0) nthreads = (int)sysconf(_SC_NPROCESSORS_ONLN);
    if (nthreads < 1) nthreads = 1;
    if (nthreads > n_rows) nthreads = n_rows > 0 ? (int)n_rows : 1;
    pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * nthreads);
    or_job* jobs = (or_job*)malloc(sizeof(or_job) * nthreads);
    for (int t = 0; t < nthreads; ++t) {
        jobs[t] = (or_job){p, rows, n_rows, n_rows * t / nthreads, n_rows * (t + 1) / nthreads,
                           out, T, mp, dp, rp};
        if (nthreads == 1) or_worker(&jobs[t]);
        else pthread_create(&th[t], NULL, or_worker, &jobs[t]);
    }
    if (nthreads > 1)
        for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
    free(th);
    free(jobs);
    return nthreads;
}

/* ------------------------------------------------------------------ exported API */

/* Full layer: out[B][H][S][D] = attention(q, k, v) by the textbook definition.
 * Returns the number of threads used. */
int or_attention(const double* q, const double* k, const double* v, double* out, int B, int H,
                 int S, int D, double scale, const or_mask* m, int nthreads)
{
    or_problem p = {q, k, v, B, H, S, D, scale, m};
    return or_run(&p, NULL, (int64_t)B * H * S, out, 0, NULL, NULL, NULL, nthreads);
}

/* Selected rows only (flat ids bh*S + i); out_rows[n_rows][D].  Used to check full-size GPU runs
 * on sampled outputs and to time a bounded CPU sample. */
int or_attention_rows(const double* q, const double* k, const double* v, int B, int H, int S,
                      int D, double scale, const or_mask* m, const int64_t* rows, int64_t n_rows,
                      double* out_rows, int nthreads)
{
    or_problem p = {q, k, v, B, H, S, D, scale, m};
    return or_run(&p, rows, n_rows, out_rows, 0, NULL, NULL, NULL, nthreads);
}

/* Full layer through the decomposition of Eq. (2) with sub-vector width T.
 * mprime/dprime/rprime (optional) are [B*H][ceil(S/T)][S]. */
int or_recomposed(const double* q, const double* k, const double* v, double* out, int B, int H,
                  int S, int D, double scale, const or_mask* m, int T, double* mprime,
                  double* dprime, double* rprime, int nthreads)
{
    if (T <= 0) return -1;
    or_problem p = {q, k, v, B, H, S, D, scale, m};
    return or_run(&p, NULL, (int64_t)B * H * S, out, T, mprime, dprime, rprime, nthreads);
}

/* The mask predicate itself, exported so tests can enumerate it (e.g. count allowed elements). */
int64_t or_count_allowed(int B, int H, int S, const or_mask* m, int64_t* per_head /*[B*H] or NULL*/)
{
    or_problem p = {NULL, NULL, NULL, B, H, S, 0, 0.0, m};
    int64_t total = 0;
    for (int bh = 0; bh < B * H; ++bh) {
        int64_t c = 0;
        for (int i = 0; i < S; ++i)
            for (int j = 0; j < S; ++j) c += or_allowed(&p, bh / H, bh % H, i, j);
        if (per_head) per_head[bh] = c;
        total += c;
    }
    return total;
}
