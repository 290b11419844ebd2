/*
 * oracle_cli.c — TEST INFRASTRUCTURE ONLY. Command-line front end of oracle.c that prints the
 * diffable result format of SURVEY.md §8(c):
 *   oracle check <file.aag> <pairs.txt> [k_max [lo hi]]
 *       one line per pair: "pair_idx lit_a lit_b k verdict{EQ,NEQ,UND} cex_index|-"
 *       then for NEQ pairs: "cex pair_idx <num_pis bits as hex, PI 1 = bit 0>"
 *   oracle local <file.aag> <checks.txt>
 *       one line per check: "check_idx lit_a lit_b leaves... verdict{EQ,UND,BADCUT}"
 * pairs.txt: first line P, then P lines "lit_a lit_b".
 * checks.txt: first line Q, then Q lines "lit_a lit_b n leaf_1 .. leaf_n".
 */
#include <inttypes.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

typedef struct oaig oaig;
oaig *oracle_read_aag(const char *path, char *err, int errlen);
void oracle_free(oaig *g);
uint32_t oracle_num_pis(const oaig *g);
uint64_t oracle_check_pairs(const oaig *g, uint32_t n, const uint32_t *la, const uint32_t *lb, uint32_t k_max,
                            uint64_t lo, uint64_t hi, int32_t *verdict, uint64_t *cex, uint32_t *k_out);
int oracle_cex_vector(const oaig *g, uint32_t la, uint32_t lb, uint64_t idx, uint8_t *out);
int oracle_check_local(const oaig *g, uint32_t n, const uint32_t *la, const uint32_t *lb, const uint32_t *cut_off,
                       const uint32_t *leaves, int32_t *verdict);

static const char *vname(int32_t v) {
    switch (v) {
        case 1: return "EQ";
        case 2: return "NEQ";
        case 0: return "UND";
        default: return "BADCUT";
    }
}

static void print_hex_bits(const uint8_t *bits, uint32_t n) {
    /* PI 1 = bit 0; print most significant nibble first */
    uint32_t nib = (n + 3) / 4;
    if (nib == 0) { printf("0"); return; }
    for (int32_t h = (int32_t)nib - 1; h >= 0; h--) {
        unsigned v = 0;
        for (int b = 3; b >= 0; b--) {
            uint32_t i = (uint32_t)h * 4 + (uint32_t)b;
            v = (v << 1) | (i < n ? bits[i] : 0u);
        }
        printf("%x", v);
    }
}

int main(int argc, char **argv) {
    if (argc < 4) {
        fprintf(stderr, "usage: %s check <aag> <pairs> [k_max [lo hi]] | local <aag> <checks>\n", argv[0]);
        return 2;
    }
    char err[256] = {0};
    oaig *g = oracle_read_aag(argv[2], err, sizeof err);
    if (!g) { fprintf(stderr, "oracle: %s\n", err); return 1; }
    FILE *f = fopen(argv[3], "r");
    if (!f) { fprintf(stderr, "oracle: cannot open %s\n", argv[3]); return 1; }
    unsigned long n = 0;
    if (fscanf(f, "%lu", &n) != 1) { fprintf(stderr, "oracle: bad list\n"); return 1; }
    if (strcmp(argv[1], "check") == 0) {
        uint32_t *la = malloc(4 * (n + 1)), *lb = malloc(4 * (n + 1)), *k = malloc(4 * (n + 1));
        int32_t *v = malloc(4 * (n + 1));
        uint64_t *cex = malloc(8 * (n + 1));
        for (unsigned long p = 0; p < n; p++) {
            unsigned long a, b;
            if (fscanf(f, "%lu %lu", &a, &b) != 2) { fprintf(stderr, "oracle: bad pair line\n"); return 1; }
            la[p] = (uint32_t)a; lb[p] = (uint32_t)b;
        }
        uint32_t k_max = argc > 4 ? (uint32_t)strtoul(argv[4], NULL, 10) : 32;
        uint64_t lo = argc > 6 ? strtoull(argv[5], NULL, 10) : 0;
        uint64_t hi = argc > 6 ? strtoull(argv[6], NULL, 10) : UINT64_MAX;
        oracle_check_pairs(g, (uint32_t)n, la, lb, k_max, lo, hi, v, cex, k);
        for (unsigned long p = 0; p < n; p++) {
            printf("%lu %u %u %u %s ", p, la[p], lb[p], k[p], vname(v[p]));
            if (v[p] == 2) printf("%" PRIu64 "\n", cex[p]); else printf("-\n");
        }
        uint8_t *bits = malloc(oracle_num_pis(g) + 1);
        for (unsigned long p = 0; p < n; p++) {
            if (v[p] != 2) continue;
            oracle_cex_vector(g, la[p], lb[p], cex[p], bits);
            printf("cex %lu ", p);
            print_hex_bits(bits, oracle_num_pis(g));
            printf("\n");
        }
    } else if (strcmp(argv[1], "local") == 0) {
        uint32_t *la = malloc(4 * (n + 1)), *lb = malloc(4 * (n + 1)), *off = malloc(4 * (n + 2));
        int32_t *v = malloc(4 * (n + 1));
        size_t cap = 64, used = 0;
        uint32_t *lv = malloc(4 * cap);
        off[0] = 0;
        for (unsigned long q = 0; q < n; q++) {
            unsigned long a, b, m;
            if (fscanf(f, "%lu %lu %lu", &a, &b, &m) != 3) { fprintf(stderr, "oracle: bad check line\n"); return 1; }
            la[q] = (uint32_t)a; lb[q] = (uint32_t)b;
            for (unsigned long j = 0; j < m; j++) {
                unsigned long x;
                if (fscanf(f, "%lu", &x) != 1) { fprintf(stderr, "oracle: bad leaf\n"); return 1; }
                if (used == cap) { cap *= 2; lv = realloc(lv, 4 * cap); }
                lv[used++] = (uint32_t)x;
            }
            off[q + 1] = (uint32_t)used;
        }
        oracle_check_local(g, (uint32_t)n, la, lb, off, lv, v);
        for (unsigned long q = 0; q < n; q++) {
            printf("%lu %u %u", q, la[q], lb[q]);
            for (uint32_t j = off[q]; j < off[q + 1]; j++) printf(" %u", lv[j]);
            printf(" %s\n", vname(v[q]));
        }
    } else {
        fprintf(stderr, "oracle: unknown command %s\n", argv[1]);
        return 2;
    }
    fclose(f);
    oracle_free(g);
    return 0;
}
