/*
 * abacus_oracle.c -- fp64 CPU oracle for the Abacus candidate search.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load or call this
 * library.  It shares no code, header, table or helper with the CUDA path
 * (paper_conf_sc_cui0czlzsmylg21_b200/csrc); neither side includes the other.
 *
 * Plain, slow, obviously-correct: scalar loops in double precision, nested
 * recursion for enumeration, no blocking, no fusion, single thread.
 * Citations are P:<line> into the paper text (Cui et al., SC'21, PAPER.md),
 * readings c1..c20 are SURVEY.md §8(c) / DESIGN.md "Readings".
 *
 * Parity pins (tests/test_oracle_*.py): Fig. 8 literal vector, Fig. 12
 * replay, dyadic hand-computed MLP, brute-force enumeration, closed-form
 * counts, linear-predictor knapsack closed form, Eq. 2/3 worked example.
 * The bf16-emulating MLP (orc_mlp64_emu) is a secondary reference used only
 * to localise bf16 error; its rounding points are pinned by hand-rounded
 * single values, and the emulation as a whole against torch's independent
 * fp32 -> bf16 conversion (tests/test_oracle_pins.py
 * test_bf16_emulation_against_torch_rounding).  The determinism hash
 * primitives (orc_splitmix64, orc_fnv1a64) are pinned by their published
 * known answers.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORC_H 32     /* hidden width: "3 layers, whose dimension is 32" */
#define ORC_KMAX 16  /* hard upper bound on co-located slots the oracle handles */

/* -------------------------------------------------------------------------- */
/* Records                                                                     */
/* -------------------------------------------------------------------------- */

/* one present model in an operator group: (ops, ope, bs, seqlen), Fig. 8 */
typedef struct {
    int32_t model_id, ops, ope, bs, seqlen;
} orc_present_t;

/* one sweep-grid slot (same meaning as the ABI's abacus_slot_t) */
typedef struct {
    int32_t model_id, start_op, batch, seqlen, end_lo, end_hi, allow_absent;
} orc_gslot_t;

/* one active query (same meaning as the ABI's abacus_query_t) */
typedef struct {
    int32_t model_id, next_op, batch, seqlen;
    double qos_ms, t_start_ms;
} orc_query_t;

typedef struct {
    uint64_t best_key;      /* max key over feasible candidates, 0 = none     */
    uint64_t best_index;    /* t* (low 40 bits of best_key)                    */
    double best_y;          /* y(t*)                                           */
    double y0;              /* y(t = 0) if 0 in range, else NAN                */
    uint64_t feasible;      /* # candidates with y <= H                        */
    uint64_t evaluated;     /* # candidates evaluated                          */
    uint64_t hash;          /* sum_t splitmix64(t ^ fnv1a64(x(t))) mod 2^64    */
    uint64_t maxkey_strict; /* max key over y <= H - eps|H|                    */
    uint64_t maxkey_loose;  /* max key over y <= H + eps|H|                    */
    int32_t best_sum_n;     /* sum of n over t*                                */
    int32_t pad;
} orc_sweep_result_t;

typedef struct {
    int32_t status;      /* 0 OK, 1 DROP (ABI ABACUS_DECIDE_*)                */
    int32_t critical;    /* caller index of the least-headroom query          */
    int32_t order[4];    /* headroom order, caller indices                    */
    int32_t end_op[4];   /* per caller query: ope, 0 = not in the group       */
    int32_t space_used;  /* 0 GRID, 1 CHAIN                                   */
    int32_t total_ops;   /* sum n of the chosen group                         */
    uint64_t key, index, evaluated, feasible, maxkey_strict, maxkey_loose;
    double headroom_ms;  /* H = (double)(float)h_c                            */
    double pred_ms;      /* y(t*)                                             */
    double pred_critical_only_ms; /* y(0)                                     */
    double h[4];         /* per caller query headroom (Eq. 2 + Eq. 3)         */
} orc_decision_t;

/* -------------------------------------------------------------------------- */
/* Hashes: constants fixed so both sides agree          */
/* -------------------------------------------------------------------------- */
uint64_t orc_splitmix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

uint64_t orc_fnv1a64(const int16_t* x, int32_t d) {
    uint64_t h = 0xcbf29ce484222325ULL;
    for (int32_t i = 0; i < d; i++) {
        uint16_t v = (uint16_t)x[i];
        uint8_t b0 = (uint8_t)(v & 0xff), b1 = (uint8_t)(v >> 8); /* little endian */
        h ^= b0; h *= 0x100000001b3ULL;
        h ^= b1; h *= 0x100000001b3ULL;
    }
    return h;
}

/* -------------------------------------------------------------------------- */
/* Eq. 2 + Eq. 3: QoS headroom                                                 */
/*   T_h = T_QoS - (T_cur - T_start)               (Eq. 2)        */
/*   T_schedule_h = T_h - T_predict_lat            (Eq. 3)        */
/* reading c15: the in-flight prediction is subtracted from every query.      */
/* -------------------------------------------------------------------------- */
double orc_headroom(double qos_ms, double t_start_ms, double now_ms, double inflight_pred_ms) {
    double t_h = qos_ms - (now_ms - t_start_ms);
    return t_h - inflight_pred_ms;
}

/* Sort by headroom ascending; ties by model id (c10). */
void orc_order(int32_t k, const double* h, const int32_t* model_id, int32_t* order) {
    for (int32_t i = 0; i < k; i++) order[i] = i;
    for (int32_t i = 1; i < k; i++) {          /* insertion sort, stable */
        int32_t v = order[i], j = i - 1;
        while (j >= 0 && (h[order[j]] > h[v] ||
                          (h[order[j]] == h[v] && model_id[order[j]] > model_id[v]))) {
            order[j + 1] = order[j];
            j--;
        }
        order[j + 1] = v;
    }
}

/* -------------------------------------------------------------------------- */
/* Fig. 8 feature encoding                              */
/*   x[m-1] = 1 for each present model m (N-bit multi-hot, c6)                */
/*   present models in ascending model id fill slots p = 0,1,..:              */
/*   x[N+4p .. N+4p+3] = (ops, ope, bs, seqlen)   (c4, c7; seqlen 0 CV, c8)   */
/*   remaining entries 0                                                       */
/* returns 0, or -1 on invalid input (too many slots, bad/duplicate id, c9)   */
/* -------------------------------------------------------------------------- */
int32_t orc_encode(int32_t n_models, int32_t kmax, int32_t n, const orc_present_t* s, int16_t* x) {
    int32_t d = n_models + 4 * kmax;
    orc_present_t tmp[ORC_KMAX];
    if (n < 0 || n > kmax || n > ORC_KMAX) return -1;
    for (int32_t i = 0; i < d; i++) x[i] = 0;
    for (int32_t i = 0; i < n; i++) {
        if (s[i].model_id < 1 || s[i].model_id > n_models) return -1;
        for (int32_t j = 0; j < i; j++)
            if (s[j].model_id == s[i].model_id) return -1;
        tmp[i] = s[i];
    }
    for (int32_t i = 1; i < n; i++) {          /* insertion sort by model id */
        orc_present_t v = tmp[i];
        int32_t j = i - 1;
        while (j >= 0 && tmp[j].model_id > v.model_id) { tmp[j + 1] = tmp[j]; j--; }
        tmp[j + 1] = v;
    }
    for (int32_t p = 0; p < n; p++) {
        x[tmp[p].model_id - 1] = 1;
        x[n_models + 4 * p + 0] = (int16_t)tmp[p].ops;
        x[n_models + 4 * p + 1] = (int16_t)tmp[p].ope;
        x[n_models + 4 * p + 2] = (int16_t)tmp[p].bs;
        x[n_models + 4 * p + 3] = (int16_t)tmp[p].seqlen;
    }
    return 0;
}

/* batch form: groups[g][j] with model_id == 0 marking an unused slot */
int32_t orc_encode_groups(int32_t n_models, int32_t kmax, int64_t count,
                          const orc_present_t* groups, int16_t* x) {
    int32_t d = n_models + 4 * kmax;
    for (int64_t g = 0; g < count; g++) {
        orc_present_t s[ORC_KMAX];
        int32_t n = 0;
        for (int32_t j = 0; j < kmax; j++)
            if (groups[g * kmax + j].model_id != 0) s[n++] = groups[g * kmax + j];
        if (orc_encode(n_models, kmax, n, s, x + g * d) != 0) return -1;
    }
    return 0;
}

/* -------------------------------------------------------------------------- */
/* Predictor MLP (c1 ReLU hidden / identity output; c2 D->32x3->1)  */
/*   y = w4 . ReLU(W3 ReLU(W2 ReLU(W1 x + b1) + b2) + b3) + b4                 */
/* params: W1[32][d] b1[32] W2[32][32] b2[32] W3[32][32] b3[32] w4[32] b4,    */
/* row-major [out][in], fp32, promoted exactly to double.                     */
/* -------------------------------------------------------------------------- */
double orc_mlp64(const float* prm, int32_t d, const int16_t* x) {
    const float* W1 = prm;
    const float* b1 = W1 + ORC_H * d;
    const float* W2 = b1 + ORC_H;
    const float* b2 = W2 + ORC_H * ORC_H;
    const float* W3 = b2 + ORC_H;
    const float* b3 = W3 + ORC_H * ORC_H;
    const float* w4 = b3 + ORC_H;
    const float* b4 = w4 + ORC_H;
    double h1[ORC_H], h2[ORC_H], h3[ORC_H];
    for (int32_t i = 0; i < ORC_H; i++) {
        double s = 0.0;
        for (int32_t j = 0; j < d; j++) s += (double)W1[i * d + j] * (double)x[j];
        s += (double)b1[i];
        h1[i] = s > 0.0 ? s : 0.0;
    }
    for (int32_t i = 0; i < ORC_H; i++) {
        double s = 0.0;
        for (int32_t j = 0; j < ORC_H; j++) s += (double)W2[i * ORC_H + j] * h1[j];
        s += (double)b2[i];
        h2[i] = s > 0.0 ? s : 0.0;
    }
    for (int32_t i = 0; i < ORC_H; i++) {
        double s = 0.0;
        for (int32_t j = 0; j < ORC_H; j++) s += (double)W3[i * ORC_H + j] * h2[j];
        s += (double)b3[i];
        h3[i] = s > 0.0 ? s : 0.0;
    }
    double y = 0.0;
    for (int32_t j = 0; j < ORC_H; j++) y += (double)w4[j] * h3[j];
    return y + (double)b4[0];
}

void orc_mlp64_batch(const float* prm, int32_t d, const int16_t* x, int64_t count, double* y) {
    for (int64_t i = 0; i < count; i++) y[i] = orc_mlp64(prm, d, x + i * d);
}

/* round-to-nearest-even to bf16 (8 significant bits), from double */
double orc_round_bf16(double v) {
    if (v == 0.0 || !isfinite(v)) return v;
    int e;
    double m = frexp(v, &e);                 /* v = m * 2^e, 0.5 <= |m| < 1 */
    double scaled = ldexp(m, 8);             /* 8 significant bits */
    double r = nearbyint(scaled);            /* default mode: ties to even */
    return ldexp(r, e - 8);
}

/* bf16-emulating MLP, a secondary reference only.
 * flags: 1 round W1..W3,w4 to bf16; 2 round b1..b4 to bf16;
 *        4 round the input features to bf16; 8 round post-ReLU h1,h2,h3 to bf16.
 * Accumulation stays in double. */
double orc_mlp64_emu(const float* prm, int32_t d, const int16_t* x, int32_t flags) {
    const float* W1 = prm;
    const float* b1 = W1 + ORC_H * d;
    const float* W2 = b1 + ORC_H;
    const float* b2 = W2 + ORC_H * ORC_H;
    const float* W3 = b2 + ORC_H;
    const float* b3 = W3 + ORC_H * ORC_H;
    const float* w4 = b3 + ORC_H;
    const float* b4 = w4 + ORC_H;
#define RW(v) ((flags & 1) ? orc_round_bf16((double)(v)) : (double)(v))
#define RB(v) ((flags & 2) ? orc_round_bf16((double)(v)) : (double)(v))
#define RX(v) ((flags & 4) ? orc_round_bf16((double)(v)) : (double)(v))
#define RA(v) ((flags & 8) ? orc_round_bf16((double)(v)) : (double)(v))
    double h1[ORC_H], h2[ORC_H], h3[ORC_H];
    for (int32_t i = 0; i < ORC_H; i++) {
        double s = 0.0;
        for (int32_t j = 0; j < d; j++) s += RW(W1[i * d + j]) * RX(x[j]);
        s += RB(b1[i]);
        h1[i] = RA(s > 0.0 ? s : 0.0);
    }
    for (int32_t i = 0; i < ORC_H; i++) {
        double s = 0.0;
        for (int32_t j = 0; j < ORC_H; j++) s += RW(W2[i * ORC_H + j]) * h1[j];
        s += RB(b2[i]);
        h2[i] = RA(s > 0.0 ? s : 0.0);
    }
    for (int32_t i = 0; i < ORC_H; i++) {
        double s = 0.0;
        for (int32_t j = 0; j < ORC_H; j++) s += RW(W3[i * ORC_H + j]) * h2[j];
        s += RB(b3[i]);
        h3[i] = RA(s > 0.0 ? s : 0.0);
    }
    double y = 0.0;
    for (int32_t j = 0; j < ORC_H; j++) y += RW(w4[j]) * h3[j];
    return y + RB(b4[0]);
#undef RW
#undef RB
#undef RX
#undef RA
}

void orc_mlp64_emu_batch(const float* prm, int32_t d, const int16_t* x, int64_t count,
                         int32_t flags, double* y) {
    for (int64_t i = 0; i < count; i++) y[i] = orc_mlp64_emu(prm, d, x + i * d, flags);
}

/* -------------------------------------------------------------------------- */
/* Sweep over a grid: enumerate (nested recursion, last slot innermost, a      */
/* running counter -- P:1349-1355 reading c13), encode, predict, mask, key.    */
/* digit d of slot j: allow_absent ? (d == 0 -> absent, else ope = lo + d - 1) */
/*                                 : ope = lo + d                              */
/* key(t) = ((sum_n + 1) << 40) | t,  n = ope - ops + 1  (c7, c12)             */
/* feasible(t) = y(t) <= H  (inclusive, c11)                                   */
/* -------------------------------------------------------------------------- */
typedef struct {
    int32_t n_models, kmax, d, k, flags;
    const float* prm;
    const orc_gslot_t* g;
    double H, eps;
    uint64_t first, last, counter;
    uint64_t sub[ORC_KMAX];
    int32_t ope[ORC_KMAX];
    double* y_out;
    int16_t* x_out;
    int32_t* ope_out;
    orc_sweep_result_t* r;
    int32_t nsum_min;             /* orc_sweep_shell: visit only sum_n >= nsum_min */
    int32_t rest_max[ORC_KMAX + 1];
} orc_sweep_state_t;

static void orc_visit(orc_sweep_state_t* st) {
    orc_present_t pres[ORC_KMAX];
    int16_t x[64];
    int32_t n = 0, sum_n = 0;
    uint64_t t = st->counter;
    for (int32_t j = 0; j < st->k; j++) {
        if (st->ope[j] == 0) continue;
        pres[n].model_id = st->g[j].model_id;
        pres[n].ops = st->g[j].start_op;
        pres[n].ope = st->ope[j];
        pres[n].bs = st->g[j].batch;
        pres[n].seqlen = st->g[j].seqlen;
        sum_n += st->ope[j] - st->g[j].start_op + 1;
        n++;
    }
    orc_encode(st->n_models, st->kmax, n, pres, x);
    double y = st->flags ? orc_mlp64_emu(st->prm, st->d, x, st->flags) : orc_mlp64(st->prm, st->d, x);
    uint64_t off = t - st->first;
    if (st->y_out) st->y_out[off] = y;
    if (st->x_out) memcpy(st->x_out + off * (uint64_t)st->d, x, sizeof(int16_t) * (size_t)st->d);
    if (st->ope_out)
        for (int32_t j = 0; j < st->k; j++) st->ope_out[off * (uint64_t)st->k + (uint64_t)j] = st->ope[j];
    orc_sweep_result_t* r = st->r;
    r->evaluated++;
    r->hash += orc_splitmix64(t ^ orc_fnv1a64(x, st->d));
    if (t == 0) r->y0 = y;
    uint64_t key = ((uint64_t)(sum_n + 1) << 40) | t;
    double tol = st->eps * fabs(st->H);
    if (y <= st->H) {
        r->feasible++;
        if (key > r->best_key) {
            r->best_key = key;
            r->best_index = t;
            r->best_y = y;
            r->best_sum_n = sum_n;
        }
    }
    if (y <= st->H - tol && key > r->maxkey_strict) r->maxkey_strict = key;
    if (y <= st->H + tol && key > r->maxkey_loose) r->maxkey_loose = key;
}

static void orc_rec(orc_sweep_state_t* st, int32_t j) {
    if (j == st->k) {
        if (st->counter >= st->first && st->counter < st->last) orc_visit(st);
        st->counter++;
        return;
    }
    const orc_gslot_t* s = &st->g[j];
    int32_t radix = s->allow_absent + (s->end_hi - s->end_lo + 1);
    for (int32_t dgt = 0; dgt < radix; dgt++) {
        if (st->counter >= st->last) return;
        if (st->counter + st->sub[j] <= st->first) {   /* whole subtree before range */
            st->counter += st->sub[j];
            continue;
        }
        if (s->allow_absent) st->ope[j] = dgt == 0 ? 0 : s->end_lo + dgt - 1;
        else st->ope[j] = s->end_lo + dgt;
        orc_rec(st, j + 1);
    }
}

/* The same enumeration restricted to the candidates with sum_n >= nsum_min:
 * a subtree whose largest reachable sum_n (the ops taken so far plus every
 * later slot at its largest end op) is below the bound is skipped whole, its
 * indices counted.  Used to check a huge sweep's answer: every key above it
 * has a sum_n at least the answer's (reading c12), so the check needs only
 * this shell (SURVEY.md §8(c) "Large sweeps"). */
static void orc_rec_shell(orc_sweep_state_t* st, int32_t j, int32_t psum) {
    if (j == st->k) {
        orc_visit(st);
        st->counter++;
        return;
    }
    const orc_gslot_t* s = &st->g[j];
    int32_t radix = s->allow_absent + (s->end_hi - s->end_lo + 1);
    for (int32_t dgt = 0; dgt < radix; dgt++) {
        int32_t ope;
        if (s->allow_absent) ope = dgt == 0 ? 0 : s->end_lo + dgt - 1;
        else ope = s->end_lo + dgt;
        int32_t n_j = ope == 0 ? 0 : ope - s->start_op + 1;
        if (psum + n_j + st->rest_max[j + 1] < st->nsum_min) {
            st->counter += st->sub[j];
            continue;
        }
        st->ope[j] = ope;
        orc_rec_shell(st, j + 1, psum + n_j);
    }
}

int32_t orc_sweep_shell(int32_t n_models, int32_t kmax, const float* prm, int32_t k, const orc_gslot_t* g,
                        double H, int32_t nsum_min, double eps, int32_t emu_flags, orc_sweep_result_t* r) {
    orc_sweep_state_t st;
    if (k < 1 || k > kmax || k > ORC_KMAX) return -1;
    memset(&st, 0, sizeof(st));
    memset(r, 0, sizeof(*r));
    r->y0 = NAN;
    r->best_y = NAN;
    st.n_models = n_models;
    st.kmax = kmax;
    st.d = n_models + 4 * kmax;
    st.k = k;
    st.flags = emu_flags;
    st.prm = prm;
    st.g = g;
    st.H = H;
    st.eps = eps;
    st.first = 0;
    st.last = UINT64_MAX;
    st.r = r;
    st.nsum_min = nsum_min;
    st.rest_max[k] = 0;
    for (int32_t j = k - 1; j >= 0; j--) st.rest_max[j] = st.rest_max[j + 1] + (g[j].end_hi - g[j].start_op + 1);
    for (int32_t j = 0; j < k; j++) {
        uint64_t sz = 1;
        for (int32_t i = j + 1; i < k; i++)
            sz *= (uint64_t)(g[i].allow_absent + g[i].end_hi - g[i].end_lo + 1);
        st.sub[j] = sz;
    }
    orc_rec_shell(&st, 0, 0);
    return 0;
}

/* grid size T = prod radix; 0 if invalid */
uint64_t orc_grid_size(int32_t k, const orc_gslot_t* g) {
    uint64_t T = 1;
    for (int32_t j = 0; j < k; j++) {
        if (g[j].end_hi < g[j].end_lo) return 0;
        T *= (uint64_t)(g[j].allow_absent + g[j].end_hi - g[j].end_lo + 1);
    }
    return T;
}

int32_t orc_sweep(int32_t n_models, int32_t kmax, const float* prm, int32_t k, const orc_gslot_t* g,
                  double H, uint64_t first, uint64_t count, double eps, int32_t emu_flags,
                  double* y_out, int16_t* x_out, int32_t* ope_out, orc_sweep_result_t* r) {
    orc_sweep_state_t st;
    if (k < 1 || k > kmax || k > ORC_KMAX) return -1;
    memset(&st, 0, sizeof(st));
    memset(r, 0, sizeof(*r));
    r->y0 = NAN;
    r->best_y = NAN;
    st.n_models = n_models;
    st.kmax = kmax;
    st.d = n_models + 4 * kmax;
    st.k = k;
    st.flags = emu_flags;
    st.prm = prm;
    st.g = g;
    st.H = H;
    st.eps = eps;
    st.first = first;
    st.last = first + count;
    st.y_out = y_out;
    st.x_out = x_out;
    st.ope_out = ope_out;
    st.r = r;
    for (int32_t j = 0; j < k; j++) {
        uint64_t s = 1;
        for (int32_t i = j + 1; i < k; i++)
            s *= (uint64_t)(g[i].allow_absent + g[i].end_hi - g[i].end_lo + 1);
        st.sub[j] = s;
    }
    orc_rec(&st, 0);
    return 0;
}

/* -------------------------------------------------------------------------- */
/* Per-decision search (P:630-753 steps 1-2; §6.2; Eq. 2/3)        */
/* space: 0 GRID (all end-op combinations), 1 CHAIN (the paper's prefix-full + */
/* one-partial chain, c13), 2 AUTO (GRID iff T <= budget).        */
/* -------------------------------------------------------------------------- */
int32_t orc_search(int32_t n_models, int32_t kmax, const int32_t* ops_per_model, const float* prm,
                   const orc_query_t* q, int32_t k, double now_ms, double inflight_ms,
                   int32_t space, uint64_t budget, double eps, int32_t emu_flags,
                   orc_decision_t* out) {
    double h[ORC_KMAX];
    int32_t mid[ORC_KMAX], order[ORC_KMAX];
    orc_gslot_t g[ORC_KMAX];
    if (k < 1 || k > kmax || k > 4) return -1;
    memset(out, 0, sizeof(*out));
    for (int32_t i = 0; i < k; i++) {
        if (q[i].model_id < 1 || q[i].model_id > n_models) return -1;
        for (int32_t j = 0; j < i; j++)
            if (q[j].model_id == q[i].model_id) return -2;
        int32_t Lm = ops_per_model[q[i].model_id - 1];
        if (q[i].next_op < 1 || q[i].next_op > Lm) return -1;
        h[i] = orc_headroom(q[i].qos_ms, q[i].t_start_ms, now_ms, inflight_ms);
        mid[i] = q[i].model_id;
        out->h[i] = h[i];
    }
    orc_order(k, h, mid, order);
    for (int32_t j = 0; j < k; j++) out->order[j] = order[j];
    out->critical = order[0];
    double H = (double)(float)h[order[0]];          /* the fp32 threshold the GPU sees */
    out->headroom_ms = H;
    /* slots in headroom order: critical fully included */
    for (int32_t j = 0; j < k; j++) {
        const orc_query_t* qq = &q[order[j]];
        int32_t Lm = ops_per_model[qq->model_id - 1];
        g[j].model_id = qq->model_id;
        g[j].start_op = qq->next_op;
        g[j].batch = qq->batch;
        g[j].seqlen = qq->seqlen;
        g[j].end_hi = Lm;
        g[j].end_lo = j == 0 ? Lm : qq->next_op;
        g[j].allow_absent = j == 0 ? 0 : 1;
    }
    uint64_t T = orc_grid_size(k, g);
    int32_t use_chain = space == 1 || (space == 2 && T > budget);
    out->space_used = use_chain;
    int32_t ope_best[ORC_KMAX];
    for (int32_t j = 0; j < k; j++) ope_best[j] = 0;
    if (!use_chain) {
        orc_sweep_result_t r;
        orc_sweep(n_models, kmax, prm, k, g, H, 0, T, eps, emu_flags, NULL, NULL, NULL, &r);
        out->key = r.best_key;
        out->index = r.best_index;
        out->evaluated = r.evaluated;
        out->feasible = r.feasible;
        out->maxkey_strict = r.maxkey_strict;
        out->maxkey_loose = r.maxkey_loose;
        out->pred_ms = r.best_y;
        out->pred_critical_only_ms = r.y0;
        out->total_ops = r.best_key ? r.best_sum_n : 0;
        /* decode t* (mixed radix, last slot fastest) */
        uint64_t t = r.best_index;
        for (int32_t j = k - 1; j >= 0; j--) {
            uint64_t radix = (uint64_t)(g[j].allow_absent + g[j].end_hi - g[j].end_lo + 1);
            int32_t dgt = (int32_t)(t % radix);
            t /= radix;
            if (g[j].allow_absent) ope_best[j] = dgt == 0 ? 0 : g[j].end_lo + dgt - 1;
            else ope_best[j] = g[j].end_lo + dgt;
        }
    } else {
        /* CHAIN: u = 0 critical only; block j (j = 1..k-1): slots 1..j-1 full,
           slot j ope = s_j + dd - 1 for dd = 1..R_j, later slots absent. */
        uint64_t u = 0;
        double tol = eps * fabs(H);
        out->pred_critical_only_ms = NAN;
        out->pred_ms = NAN;
        for (int32_t j = 0; j < k; j++) {
            int32_t R = j == 0 ? 1 : g[j].end_hi - g[j].start_op + 1;
            for (int32_t dd = 1; dd <= R; dd++) {
                orc_present_t pres[ORC_KMAX];
                int16_t x[64];
                int32_t n = 0, sum_n = 0, ope[ORC_KMAX];
                for (int32_t i = 0; i < k; i++) {
                    if (i < j) ope[i] = g[i].end_hi;
                    else if (i == j) ope[i] = j == 0 ? g[0].end_hi : g[i].start_op + dd - 1;
                    else ope[i] = 0;
                }
                for (int32_t i = 0; i < k; i++) {
                    if (ope[i] == 0) continue;
                    pres[n].model_id = g[i].model_id;
                    pres[n].ops = g[i].start_op;
                    pres[n].ope = ope[i];
                    pres[n].bs = g[i].batch;
                    pres[n].seqlen = g[i].seqlen;
                    sum_n += ope[i] - g[i].start_op + 1;
                    n++;
                }
                orc_encode(n_models, kmax, n, pres, x);
                double y = emu_flags ? orc_mlp64_emu(prm, n_models + 4 * kmax, x, emu_flags)
                                     : orc_mlp64(prm, n_models + 4 * kmax, x);
                uint64_t key = ((uint64_t)(sum_n + 1) << 40) | u;
                out->evaluated++;
                if (u == 0) out->pred_critical_only_ms = y;
                if (y <= H) {
                    out->feasible++;
                    if (key > out->key) {
                        out->key = key;
                        out->index = u;
                        out->pred_ms = y;
                        out->total_ops = sum_n;
                        for (int32_t i = 0; i < k; i++) ope_best[i] = ope[i];
                    }
                }
                if (y <= H - tol && key > out->maxkey_strict) out->maxkey_strict = key;
                if (y <= H + tol && key > out->maxkey_loose) out->maxkey_loose = key;
                u++;
            }
        }
    }
    /* drop mechanism (c14): the critical query alone does not fit */
    if (!(out->pred_critical_only_ms <= H)) {
        out->status = 1;
        for (int32_t i = 0; i < 4; i++) out->end_op[i] = 0;
        return 0;
    }
    out->status = 0;
    for (int32_t j = 0; j < k; j++) out->end_op[order[j]] = ope_best[j];
    return 0;
}

/* -------------------------------------------------------------------------- */
/* Multi-way search over the CHAIN (§7.7) */
/* Round 1 ("between queries"): one batched call predicts u = 0 (drop test)    */
/* and every block end B_j (queries 1..j fully added); the last fitting block   */
/* end is lo, the first missing one after it is hi.  Later rounds ("among the   */
/* operators"): the open interval (lo, hi) of the next query's ops is probed    */
/* at m points p_i = lo + floor(i (hi - lo) / (m + 1)), i = 1..m (all points    */
/* when it holds <= m); lo <- last fitting probe, hi <- first missing probe     */
/* after it (reading c17).  Ends when the interval is empty.  Returns u* = lo.  */
/* -------------------------------------------------------------------------- */
typedef struct {
    int32_t status;      /* 0 OK, 1 DROP */
    int32_t rounds;      /* batched predictor calls */
    int32_t predictions; /* candidates predicted */
    int32_t total_ops;
    uint64_t u;          /* chosen chain index */
    double headroom_ms, pred_ms, pred_critical_only_ms;
    int32_t end_op[4];   /* per caller query */
    int32_t order[4];
} orc_mway_t;

static double orc_chain_y(int32_t n_models, int32_t kmax, const float* prm, int32_t emu, int32_t k,
                          const orc_gslot_t* g, const uint64_t* cum, uint64_t u, int32_t* ope_out,
                          int32_t* sum_n_out) {
    orc_present_t pres[ORC_KMAX];
    int16_t x[64];
    int32_t ope[ORC_KMAX], n = 0, sum_n = 0, blk = 0;
    for (int32_t j = 1; j < k; j++)
        if (u >= cum[j]) blk = j;
    for (int32_t i = 0; i < k; i++) {
        if (i < blk) ope[i] = g[i].end_hi;
        else if (i == blk) ope[i] = blk == 0 ? g[0].end_hi : g[i].start_op + (int32_t)(u - cum[i]);
        else ope[i] = 0;
    }
    for (int32_t i = 0; i < k; i++) {
        if (ope[i] == 0) continue;
        pres[n].model_id = g[i].model_id;
        pres[n].ops = g[i].start_op;
        pres[n].ope = ope[i];
        pres[n].bs = g[i].batch;
        pres[n].seqlen = g[i].seqlen;
        sum_n += ope[i] - g[i].start_op + 1;
        n++;
    }
    orc_encode(n_models, kmax, n, pres, x);
    if (ope_out)
        for (int32_t i = 0; i < k; i++) ope_out[i] = ope[i];
    if (sum_n_out) *sum_n_out = sum_n;
    return emu ? orc_mlp64_emu(prm, n_models + 4 * kmax, x, emu) : orc_mlp64(prm, n_models + 4 * kmax, x);
}

int32_t orc_search_mway(int32_t n_models, int32_t kmax, const int32_t* ops_per_model, const float* prm,
                        const orc_query_t* q, int32_t k, double now_ms, double inflight_ms, int32_t ways,
                        int32_t emu_flags, orc_mway_t* out) {
    double h[ORC_KMAX];
    int32_t mid[ORC_KMAX], order[ORC_KMAX];
    orc_gslot_t g[ORC_KMAX];
    uint64_t cum[ORC_KMAX + 1];
    if (k < 1 || k > kmax || k > 4 || ways < 1 || ways > 128) return -1;
    memset(out, 0, sizeof(*out));
    for (int32_t i = 0; i < k; i++) {
        if (q[i].model_id < 1 || q[i].model_id > n_models) return -1;
        for (int32_t j = 0; j < i; j++)
            if (q[j].model_id == q[i].model_id) return -2;
        h[i] = orc_headroom(q[i].qos_ms, q[i].t_start_ms, now_ms, inflight_ms);
        mid[i] = q[i].model_id;
    }
    orc_order(k, h, mid, order);
    for (int32_t j = 0; j < k; j++) out->order[j] = order[j];
    double H = (double)(float)h[order[0]];
    out->headroom_ms = H;
    for (int32_t j = 0; j < k; j++) {
        const orc_query_t* qq = &q[order[j]];
        int32_t Lm = ops_per_model[qq->model_id - 1];
        g[j].model_id = qq->model_id;
        g[j].start_op = qq->next_op;
        g[j].batch = qq->batch;
        g[j].seqlen = qq->seqlen;
        g[j].end_hi = Lm;
        g[j].end_lo = j == 0 ? Lm : qq->next_op;
        g[j].allow_absent = j == 0 ? 0 : 1;
    }
    /* chain blocks: u = 0 critical; block j covers [cum[j], cum[j] + R_j) */
    cum[0] = 0;
    cum[1] = 1;
    for (int32_t j = 1; j < k; j++) cum[j + 1] = cum[j] + (uint64_t)(g[j].end_hi - g[j].start_op + 1);
    /* round 1: u = 0 and the block ends */
    uint64_t probes[ORC_KMAX + 1];
    int32_t np = 0;
    probes[np++] = 0;
    for (int32_t j = 1; j < k; j++) probes[np++] = cum[j + 1] - 1;
    uint64_t lo = 0, hi = cum[k];
    out->rounds = 1;
    int32_t fit[ORC_KMAX + 1];
    for (int32_t i = 0; i < np; i++) {
        double y = orc_chain_y(n_models, kmax, prm, emu_flags, k, g, cum, probes[i], NULL, NULL);
        out->predictions++;
        fit[i] = y <= H;
        if (i == 0) out->pred_critical_only_ms = y;
    }
    if (!fit[0]) {
        out->status = 1;
        out->pred_ms = out->pred_critical_only_ms;
        return 0;
    }
    int32_t last = 0;
    for (int32_t i = 1; i < np; i++)
        if (fit[i]) last = i;
    lo = probes[last];
    hi = cum[k];
    for (int32_t i = last + 1; i < np; i++)
        if (!fit[i]) { hi = probes[i]; break; }
    /* later rounds: m-way among the operators of the next query */
    while (hi - lo > 1) {
        uint64_t p[128];
        int32_t n = 0;
        uint64_t span = hi - lo;
        if (span - 1 <= (uint64_t)ways) {
            for (uint64_t v = lo + 1; v < hi; v++) p[n++] = v;
        } else {
            for (int32_t i = 1; i <= ways; i++) {
                uint64_t v = lo + (span * (uint64_t)i) / (uint64_t)(ways + 1);
                if (v > lo && v < hi && (n == 0 || v > p[n - 1])) p[n++] = v;
            }
        }
        out->rounds++;
        int32_t f[128];
        for (int32_t i = 0; i < n; i++) {
            f[i] = orc_chain_y(n_models, kmax, prm, emu_flags, k, g, cum, p[i], NULL, NULL) <= H;
            out->predictions++;
        }
        int32_t lf = -1;
        for (int32_t i = 0; i < n; i++)
            if (f[i]) lf = i;
        uint64_t nlo = lf >= 0 ? p[lf] : lo, nhi = hi;
        for (int32_t i = lf + 1; i < n; i++)
            if (!f[i]) { nhi = p[i]; break; }
        lo = nlo;
        hi = nhi;
    }
    int32_t ope[ORC_KMAX], sum_n = 0;
    out->u = lo;
    out->pred_ms = orc_chain_y(n_models, kmax, prm, emu_flags, k, g, cum, lo, ope, &sum_n);
    out->total_ops = sum_n;
    out->status = 0;
    for (int32_t j = 0; j < k; j++) out->end_op[order[j]] = ope[j];
    return 0;
}
