/*
 * oracle.c — TEST INFRASTRUCTURE ONLY. The plain, slow, single-threaded CPU definition of what the
 * CUDA path computes. Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load it. It shares no code, header, table or helper with
 * paper_conf_dac_liuy25_b200/ (the product), and neither includes the other.
 *
 * What it computes (written out from PAPER.md):
 *   - Truth-table / pattern convention (§II-A): bit i of a truth table is the function
 *     value under the assignment with sum_j 2^j a_j = i, i.e. input j takes bit j of pattern i.
 *   - Global check of a pair (§III-B1): the inputs are the union of
 *     the two structural supports in increasing node id; every assignment is
 *     enumerated one at a time in ascending pattern order and the two roots compared; the first
 *     mismatching pattern is the counter-example (footnote 1 at :69). Reading Q8: the
 *     canonical CEX is the minimum pattern index in the pair's own support order, every
 *     non-support PI = 0. k > k_max -> UNDECIDED (PAPER.md:181/:183 thresholds; reading Q12).
 *   - Local check on a cut (§III-C1): inputs are the cut leaves (increasing
 *     id, reading Q15); identical local functions => EQUIVALENT; otherwise UNDECIDED, never NEQ,
 *     because a mismatch may be an SDC (reading Q13).
 *   - AND node value: v(n) = (v(f0) ^ c0) & (v(f1) ^ c1), const0 = 0.
 *
 * One byte per node, one assignment at a time, no bit-parallel tricks. The only speed-up used is
 * the one SURVEY.md §8(c) allows: pairs whose support sets are identical share one enumeration.
 * AIGER parsing is done here from scratch (ASCII "aag", combinational only).
 *
 * Pins (tests/test_oracle_*.py): the worked examples of PAPER.md:33/:35/:67/:79, the adder and
 * multiplier closed forms (a+b, a*b), invariants (self-miter, rewrites), injected bugs, and an
 * independent pure-Python brute-force enumerator on random AIGs with <= 12 PIs.
 */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#define OR_UNDECIDED 0
#define OR_EQUIVALENT 1
#define OR_NOT_EQUIVALENT 2
#define OR_BADCUT (-1)

typedef struct oaig {
    uint32_t num_pis;
    uint32_t num_ands;
    uint32_t num_pos;
    uint32_t *f0; /* fanin literal 0 of node id (index = id); valid for AND ids */
    uint32_t *f1;
    uint32_t *pos;
} oaig;

/* ------------------------------------------------------------------------------------------ */
/* AIGER ASCII reader: accepts any gate order, renumbers to PIs 1..I then ANDs in a DFS        */
/* topological order that keeps the file order when it is already topological (reading Q22).  */
/* ------------------------------------------------------------------------------------------ */

static int read_u32(FILE *f, uint32_t *out) {
    unsigned long v;
    if (fscanf(f, "%lu", &v) != 1) return -1;
    *out = (uint32_t)v;
    return 0;
}

oaig *oracle_read_aag(const char *path, char *err, int errlen) {
    FILE *f = fopen(path, "r");
    if (!f) { snprintf(err, errlen, "cannot open %s", path); return NULL; }
    char magic[8] = {0};
    uint32_t M, I, L, O, A;
    if (fscanf(f, "%7s", magic) != 1 || strcmp(magic, "aag") != 0 || read_u32(f, &M) || read_u32(f, &I) ||
        read_u32(f, &L) || read_u32(f, &O) || read_u32(f, &A)) {
        snprintf(err, errlen, "bad header"); fclose(f); return NULL;
    }
    if (L != 0) { snprintf(err, errlen, "latches not supported"); fclose(f); return NULL; }
    uint32_t *in_lit = malloc(sizeof(uint32_t) * (I + 1));
    uint32_t *out_lit = malloc(sizeof(uint32_t) * (O + 1));
    uint32_t *g_lhs = malloc(sizeof(uint32_t) * (A + 1));
    uint32_t *g_r0 = malloc(sizeof(uint32_t) * (A + 1));
    uint32_t *g_r1 = malloc(sizeof(uint32_t) * (A + 1));
    int bad = 0;
    for (uint32_t i = 0; i < I && !bad; i++) bad |= read_u32(f, &in_lit[i]);
    for (uint32_t i = 0; i < O && !bad; i++) bad |= read_u32(f, &out_lit[i]);
    for (uint32_t i = 0; i < A && !bad; i++) bad |= read_u32(f, &g_lhs[i]) | read_u32(f, &g_r0[i]) | read_u32(f, &g_r1[i]);
    fclose(f);
    if (bad) { snprintf(err, errlen, "truncated file"); goto fail; }

    /* file variable -> gate index, and file variable -> new id */
    uint32_t nv = M + 1;
    int64_t *gate_of = malloc(sizeof(int64_t) * nv);
    int64_t *new_id = malloc(sizeof(int64_t) * nv);
    uint8_t *state = calloc(nv, 1);
    for (uint32_t v = 0; v < nv; v++) { gate_of[v] = -1; new_id[v] = -1; }
    new_id[0] = 0;
    for (uint32_t i = 0; i < I; i++) {
        uint32_t v = in_lit[i] >> 1;
        if (v >= nv) { snprintf(err, errlen, "input out of range"); bad = 1; break; }
        new_id[v] = 1 + i;
    }
    for (uint32_t i = 0; i < A && !bad; i++) {
        uint32_t v = g_lhs[i] >> 1;
        if (v >= nv) { snprintf(err, errlen, "gate out of range"); bad = 1; break; }
        gate_of[v] = i;
    }
    uint32_t next = 1 + I;
    uint32_t *stack = malloc(sizeof(uint32_t) * (2 * (size_t)nv + 2));
    for (uint32_t i = 0; i < A && !bad; i++) {
        size_t sp = 0;
        stack[sp++] = g_lhs[i] >> 1;
        while (sp && !bad) {
            uint32_t v = stack[sp - 1];
            if (new_id[v] >= 0) { sp--; continue; }
            if (gate_of[v] < 0) { snprintf(err, errlen, "undefined variable %u", v); bad = 1; break; }
            uint32_t a = g_r0[gate_of[v]] >> 1, b = g_r1[gate_of[v]] >> 1;
            if (a >= nv || b >= nv) { snprintf(err, errlen, "fanin out of range"); bad = 1; break; }
            if (state[v] == 0) {
                state[v] = 1;
                if (new_id[b] < 0) stack[sp++] = b;
                if (new_id[a] < 0) stack[sp++] = a;
            } else if (new_id[a] >= 0 && new_id[b] >= 0) {
                new_id[v] = next++;
                sp--;
            } else {
                snprintf(err, errlen, "combinational cycle"); bad = 1;
            }
        }
    }
    oaig *g = NULL;
    if (!bad) {
        g = calloc(1, sizeof(oaig));
        g->num_pis = I; g->num_ands = A; g->num_pos = O;
        uint32_t N = 1 + I + A;
        g->f0 = calloc(N, sizeof(uint32_t));
        g->f1 = calloc(N, sizeof(uint32_t));
        g->pos = calloc(O + 1, sizeof(uint32_t));
        for (uint32_t i = 0; i < A; i++) {
            uint32_t id = (uint32_t)new_id[g_lhs[i] >> 1];
            g->f0[id] = 2 * (uint32_t)new_id[g_r0[i] >> 1] + (g_r0[i] & 1);
            g->f1[id] = 2 * (uint32_t)new_id[g_r1[i] >> 1] + (g_r1[i] & 1);
        }
        for (uint32_t i = 0; i < O; i++) {
            uint32_t v = out_lit[i] >> 1;
            if (v >= nv || new_id[v] < 0) { snprintf(err, errlen, "bad output"); free(g->f0); free(g->f1); free(g->pos); free(g); g = NULL; break; }
            g->pos[i] = 2 * (uint32_t)new_id[v] + (out_lit[i] & 1);
        }
    }
    free(stack); free(state); free(new_id); free(gate_of);
    free(in_lit); free(out_lit); free(g_lhs); free(g_r0); free(g_r1);
    return g;
fail:
    free(in_lit); free(out_lit); free(g_lhs); free(g_r0); free(g_r1);
    return NULL;
}

void oracle_free(oaig *g) {
    if (!g) return;
    free(g->f0); free(g->f1); free(g->pos); free(g);
}

uint32_t oracle_num_pis(const oaig *g) { return g->num_pis; }
uint32_t oracle_num_ands(const oaig *g) { return g->num_ands; }
uint32_t oracle_num_pos(const oaig *g) { return g->num_pos; }
uint32_t oracle_po(const oaig *g, uint32_t i) { return g->pos[i]; }
void oracle_fanins(const oaig *g, uint32_t id, uint32_t *l0, uint32_t *l1) { *l0 = g->f0[id]; *l1 = g->f1[id]; }

static int is_and(const oaig *g, uint32_t id) { return id > g->num_pis && id <= g->num_pis + g->num_ands; }

/* ------------------------------------------------------------------------------------------ */
/* Transitive fanin: mark every node reachable backwards from the roots, stopping */
/* at nodes flagged in `stop` (cut leaves) — with no stop set this is the whole TFI.             */
/* ------------------------------------------------------------------------------------------ */

static void mark_tfi(const oaig *g, const uint32_t *roots, int nroots, const uint8_t *stop, uint8_t *mark) {
    uint32_t N = 1 + g->num_pis + g->num_ands;
    uint32_t *stack = malloc(sizeof(uint32_t) * (N + 4));
    size_t sp = 0;
    for (int r = 0; r < nroots; r++) {
        if (!mark[roots[r]]) { mark[roots[r]] = 1; stack[sp++] = roots[r]; }
    }
    while (sp) {
        uint32_t v = stack[--sp];
        if (stop && stop[v]) continue;
        if (!is_and(g, v)) continue;
        uint32_t a = g->f0[v] >> 1, b = g->f1[v] >> 1;
        if (!mark[a]) { mark[a] = 1; stack[sp++] = a; }
        if (!mark[b]) { mark[b] = 1; stack[sp++] = b; }
    }
    free(stack);
}

/* Structural support of {var(la), var(lb)}: PIs in the TFI, increasing id.
 * Returns k (may exceed cap; only min(k,cap) ids are written). */
int oracle_support(const oaig *g, uint32_t la, uint32_t lb, uint32_t *S_out, int cap) {
    uint32_t N = 1 + g->num_pis + g->num_ands;
    uint8_t *mark = calloc(N, 1);
    uint32_t roots[2] = {la >> 1, lb >> 1};
    mark_tfi(g, roots, 2, NULL, mark);
    int k = 0;
    for (uint32_t id = 1; id <= g->num_pis; id++)
        if (mark[id]) { if (k < cap) S_out[k] = id; k++; }
    free(mark);
    return k;
}

/* ------------------------------------------------------------------------------------------ */
/* Global checks (SURVEY.md §8(c) "Global check of a pair")                                   */
/* ------------------------------------------------------------------------------------------ */

typedef struct { uint32_t idx; uint32_t k; uint32_t *S; } pair_sup;

static int cmp_sup(const void *x, const void *y) {
    const pair_sup *a = x, *b = y;
    if (a->k != b->k) return a->k < b->k ? -1 : 1;
    for (uint32_t j = 0; j < a->k; j++)
        if (a->S[j] != b->S[j]) return a->S[j] < b->S[j] ? -1 : 1;
    return a->idx < b->idx ? -1 : (a->idx > b->idx);
}

static int same_sup(const pair_sup *a, const pair_sup *b) {
    if (a->k != b->k) return 0;
    for (uint32_t j = 0; j < a->k; j++) if (a->S[j] != b->S[j]) return 0;
    return 1;
}

/*
 * For each pair p: k_out[p] = |S_p|; if k > k_max (or k > 63): verdict UNDECIDED, cex = UINT64_MAX.
 * Otherwise scan patterns i in [lo, min(hi, 2^k)) ascending; at the first i with v(la) != v(lb):
 * verdict NEQ, cex = i. If none: verdict EQ (for the full range [0, 2^k) this is the definition;
 * for a sub-range it means "no mismatch in this range" — the sharded oracle of SURVEY.md §8(c)).
 * Returns the number of node evaluations performed (for throughput reporting).
 */
uint64_t oracle_check_pairs(const oaig *g, uint32_t n, const uint32_t *la, const uint32_t *lb, uint32_t k_max,
                            uint64_t lo, uint64_t hi, int32_t *verdict, uint64_t *cex, uint32_t *k_out) {
    uint32_t N = 1 + g->num_pis + g->num_ands;
    uint64_t evals = 0;
    pair_sup *ps = calloc(n ? n : 1, sizeof(pair_sup));
    for (uint32_t p = 0; p < n; p++) {
        ps[p].idx = p;
        ps[p].S = malloc(sizeof(uint32_t) * (g->num_pis + 1));
        ps[p].k = (uint32_t)oracle_support(g, la[p], lb[p], ps[p].S, (int)g->num_pis + 1);
        k_out[p] = ps[p].k;
        verdict[p] = OR_UNDECIDED;
        cex[p] = UINT64_MAX;
    }
    qsort(ps, n, sizeof(pair_sup), cmp_sup);
    uint8_t *val = calloc(N, 1);
    uint8_t *mark = calloc(N, 1);
    uint32_t *cone = malloc(sizeof(uint32_t) * (N + 1));
    uint32_t *roots = malloc(sizeof(uint32_t) * (2 * (size_t)n + 2));
    uint8_t *done = calloc(n ? n : 1, 1);
    for (uint32_t s = 0; s < n;) {
        uint32_t e = s + 1;
        while (e < n && same_sup(&ps[s], &ps[e])) e++;
        uint32_t k = ps[s].k;
        if (k > k_max || k > 63) { s = e; continue; }
        /* cone of the group = union of the TFIs of all roots of the group, in increasing id */
        memset(mark, 0, N);
        int nr = 0;
        for (uint32_t t = s; t < e; t++) { roots[nr++] = la[ps[t].idx] >> 1; roots[nr++] = lb[ps[t].idx] >> 1; }
        mark_tfi(g, roots, nr, NULL, mark);
        uint32_t nc = 0;
        for (uint32_t id = g->num_pis + 1; id < N; id++) if (mark[id]) cone[nc++] = id;
        uint64_t total = (uint64_t)1 << k;
        uint64_t end = hi < total ? hi : total;
        uint32_t remaining = e - s;
        for (uint32_t t = s; t < e; t++) done[t] = 0;
        memset(val, 0, N); /* const0 and every PI outside S stay 0 */
        for (uint64_t i = lo; i < end && remaining; i++) {
            for (uint32_t j = 0; j < k; j++) val[ps[s].S[j]] = (uint8_t)((i >> j) & 1u);
            for (uint32_t c = 0; c < nc; c++) {
                uint32_t id = cone[c];
                uint8_t a = val[g->f0[id] >> 1] ^ (uint8_t)(g->f0[id] & 1u);
                uint8_t b = val[g->f1[id] >> 1] ^ (uint8_t)(g->f1[id] & 1u);
                val[id] = a & b;
            }
            evals += nc;
            for (uint32_t t = s; t < e; t++) {
                if (done[t]) continue;
                uint32_t p = ps[t].idx;
                uint8_t va = val[la[p] >> 1] ^ (uint8_t)(la[p] & 1u);
                uint8_t vb = val[lb[p] >> 1] ^ (uint8_t)(lb[p] & 1u);
                if (va != vb) { verdict[p] = OR_NOT_EQUIVALENT; cex[p] = i; done[t] = 1; remaining--; }
            }
        }
        for (uint32_t t = s; t < e; t++)
            if (!done[t]) verdict[ps[t].idx] = OR_EQUIVALENT;
        s = e;
    }
    for (uint32_t p = 0; p < n; p++) free(ps[p].S);
    free(ps); free(val); free(mark); free(cone); free(roots); free(done);
    return evals;
}

/* CEX vector of pattern `idx` of pair (la, lb): PI S[j] = bit j of idx, all other PIs 0
 * (SURVEY.md §8(c) step 4). out[i] is the value of PI id i+1. Returns k. */
int oracle_cex_vector(const oaig *g, uint32_t la, uint32_t lb, uint64_t idx, uint8_t *out) {
    uint32_t *S = malloc(sizeof(uint32_t) * (g->num_pis + 1));
    int k = oracle_support(g, la, lb, S, (int)g->num_pis + 1);
    memset(out, 0, g->num_pis);
    for (int j = 0; j < k && j < 64; j++) out[S[j] - 1] = (uint8_t)((idx >> j) & 1u);
    free(S);
    return k;
}

/* Evaluate one literal under a full PI assignment pis[0..I-1] (PI id i+1 = pis[i]).
 * Used by tests to confirm a CEX vector really separates the pair. */
int oracle_eval_lit(const oaig *g, uint32_t lit, const uint8_t *pis) {
    uint32_t N = 1 + g->num_pis + g->num_ands;
    uint8_t *val = calloc(N, 1);
    for (uint32_t i = 0; i < g->num_pis; i++) val[1 + i] = pis[i] & 1u;
    for (uint32_t id = g->num_pis + 1; id < N; id++)
        val[id] = (uint8_t)((val[g->f0[id] >> 1] ^ (g->f0[id] & 1u)) & (val[g->f1[id] >> 1] ^ (g->f1[id] & 1u)));
    int r = val[lit >> 1] ^ (int)(lit & 1u);
    free(val);
    return r;
}

/* Value of every node id (const 0 = 0) under one PI assignment; val_out[1 + num_pis + num_ands]. */
void oracle_eval_all(const oaig *g, const uint8_t *pis, uint8_t *val) {
    uint32_t N = 1 + g->num_pis + g->num_ands;
    val[0] = 0;
    for (uint32_t i = 0; i < g->num_pis; i++) val[1 + i] = pis[i] & 1u;
    for (uint32_t id = g->num_pis + 1; id < N; id++)
        val[id] = (uint8_t)((val[g->f0[id] >> 1] ^ (g->f0[id] & 1u)) & (val[g->f1[id] >> 1] ^ (g->f1[id] & 1u)));
}

/* ------------------------------------------------------------------------------------------ */
/* Local checks (SURVEY.md §8(c) "Local check of a pair on cut L")                             */
/* ------------------------------------------------------------------------------------------ */

/*
 * Check q uses leaves[cut_off[q] .. cut_off[q+1]) (node ids, any order; sorted here by id).
 * verdict[q] = EQUIVALENT if the local functions of both roots over the leaves are identical,
 * UNDECIDED otherwise, OR_BADCUT if the backward traversal from a root reaches a PI that is not a
 * leaf (the leaf set is not a cut). Returns the number of bad cuts.
 */
int oracle_check_local(const oaig *g, uint32_t n, const uint32_t *la, const uint32_t *lb, const uint32_t *cut_off,
                       const uint32_t *leaves, int32_t *verdict) {
    uint32_t N = 1 + g->num_pis + g->num_ands;
    uint8_t *stop = calloc(N, 1), *mark = calloc(N, 1), *val = calloc(N, 1);
    uint32_t *cone = malloc(sizeof(uint32_t) * (N + 1));
    uint32_t *L = malloc(sizeof(uint32_t) * (N + 1));
    int bad = 0;
    for (uint32_t q = 0; q < n; q++) {
        uint32_t nl = cut_off[q + 1] - cut_off[q];
        for (uint32_t j = 0; j < nl; j++) L[j] = leaves[cut_off[q] + j];
        /* increasing id (reading Q15); insertion sort keeps this obviously correct */
        for (uint32_t j = 1; j < nl; j++) {
            uint32_t x = L[j]; int t = (int)j - 1;
            while (t >= 0 && L[t] > x) { L[t + 1] = L[t]; t--; }
            L[t + 1] = x;
        }
        memset(stop, 0, N); memset(mark, 0, N);
        for (uint32_t j = 0; j < nl; j++) stop[L[j]] = 1;
        uint32_t roots[2] = {la[q] >> 1, lb[q] >> 1};
        mark_tfi(g, roots, 2, stop, mark);
        int ok = 1;
        for (uint32_t id = 1; id <= g->num_pis; id++)
            if (mark[id] && !stop[id]) ok = 0;
        if (!ok || nl > 30) { verdict[q] = OR_BADCUT; bad++; continue; }
        uint32_t nc = 0;
        for (uint32_t id = g->num_pis + 1; id < N; id++) if (mark[id] && !stop[id]) cone[nc++] = id;
        int32_t v = OR_EQUIVALENT;
        memset(val, 0, N);
        for (uint64_t i = 0; i < ((uint64_t)1 << nl); i++) {
            for (uint32_t j = 0; j < nl; j++) val[L[j]] = (uint8_t)((i >> j) & 1u);
            for (uint32_t c = 0; c < nc; c++) {
                uint32_t id = cone[c];
                uint8_t a = val[g->f0[id] >> 1] ^ (uint8_t)(g->f0[id] & 1u);
                uint8_t b = val[g->f1[id] >> 1] ^ (uint8_t)(g->f1[id] & 1u);
                val[id] = a & b;
            }
            uint8_t va = val[la[q] >> 1] ^ (uint8_t)(la[q] & 1u);
            uint8_t vb = val[lb[q] >> 1] ^ (uint8_t)(lb[q] & 1u);
            if (va != vb) { v = OR_UNDECIDED; break; }
        }
        verdict[q] = v;
    }
    free(stop); free(mark); free(val); free(cone); free(L);
    return bad;
}
