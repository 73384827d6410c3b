/* decision_latency.c -- per-decision latency of abacus_search through the C ABI
 * (no Python on the path).  Input file (written by tools/decision_latency.py):
 *   int32 n_models, int32 L[n_models], int32 n_params, float params[n_params],
 *   int32 precision, int32 space, uint64 budget, int32 n_dec, int32 warm,
 *   n_dec x { int32 k, double now, double inflight, k x abacus_query_t }
 * Output: one line of JSON with p50/p99/p99.9 (us) and the grid-size spread.
 * With a second argument B > 0: abacus_search_batch over consecutive batches
 * of B decisions (the first `warm` decisions warm up); reports per-call
 * latency, decisions/s and the kernel share (CUDA events around the launch).
 */
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>
#include "abacus.h"

static double now_us(void) {
    struct timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return ts.tv_sec * 1e6 + ts.tv_nsec * 1e-3;
}
static int cmpd(const void* a, const void* b) {
    double x = *(const double*)a, y = *(const double*)b;
    return x < y ? -1 : x > y;
}
static int cmpu(const void* a, const void* b) {
    const uint64_t x = *(const uint64_t*)a, y = *(const uint64_t*)b;
    return x < y ? -1 : x > y;
}
#define RD(p, n, f) do { if (fread(p, 1, n, f) != (size_t)(n)) { fprintf(stderr, "short read\n"); return 2; } } while (0)

int main(int argc, char** argv) {
    if (argc < 2) { fprintf(stderr, "usage: %s input.bin\n", argv[0]); return 2; }
    FILE* f = fopen(argv[1], "rb");
    if (!f) return 2;
    int32_t nm, np, prec, space, ndec, warm;
    uint64_t budget;
    RD(&nm, 4, f);
    int32_t* L = malloc(4 * nm);
    RD(L, 4 * nm, f);
    RD(&np, 4, f);
    float* prm = malloc(4 * np);
    RD(prm, 4 * np, f);
    RD(&prec, 4, f); RD(&space, 4, f); RD(&budget, 8, f); RD(&ndec, 4, f); RD(&warm, 4, f);
    int32_t* ks = malloc(4 * ndec);
    double* nows = malloc(8 * ndec);
    double* infl = malloc(8 * ndec);
    abacus_query_t* qs = malloc(sizeof(abacus_query_t) * 4 * ndec);
    for (int i = 0; i < ndec; i++) {
        RD(&ks[i], 4, f); RD(&nows[i], 8, f); RD(&infl[i], 8, f);
        RD(&qs[4 * i], sizeof(abacus_query_t) * ks[i], f);
    }
    fclose(f);
    abacus_ctx* ctx = NULL;
    int rc = abacus_create(0, nm, L, 4, &ctx);
    if (rc) { fprintf(stderr, "create failed %d\n", rc); return 1; }
    rc = abacus_load_predictor(ctx, prm, np, prec);
    if (rc) { fprintf(stderr, "load failed %s\n", abacus_last_error(ctx)); return 1; }
    int B = argc > 2 ? atoi(argv[2]) : 0;
    if (B > 0) {
        abacus_decision_t* out = malloc(sizeof(abacus_decision_t) * B);
        abacus_set_timing(ctx, 1);
        /* warm-up: one call of the same size (grows the ctx buffers) */
        if (ndec < B) { fprintf(stderr, "need >= B decisions\n"); return 2; }
        rc = abacus_search_batch(ctx, qs, ks, nows, infl, B, space, budget, out);
        if (rc) { fprintf(stderr, "batch failed %s\n", abacus_last_error(ctx)); return 1; }
        int calls = (ndec - warm) / B;
        double* cl = malloc(8 * calls);
        double kms = 0.0, tsum = 0.0;
        uint64_t evsum = 0;
        int ndrop = 0;
        for (int c = 0; c < calls; c++) {
            const int i0 = warm + c * B;
            double t0 = now_us();
            rc = abacus_search_batch(ctx, &qs[4 * i0], &ks[i0], &nows[i0], &infl[i0], B, space, budget, out);
            double t1 = now_us();
            if (rc) { fprintf(stderr, "batch failed %s\n", abacus_last_error(ctx)); return 1; }
            cl[c] = t1 - t0;
            tsum += cl[c];
            kms += abacus_last_kernel_ms(ctx);
            for (int i = 0; i < B; i++) { evsum += out[i].evaluated; ndrop += out[i].status == ABACUS_DECIDE_DROP; }
        }
        qsort(cl, calls, sizeof(double), cmpd);
        printf("{\"batch\": %d, \"calls\": %d, \"call_p50_us\": %.1f, \"call_p99_us\": %.1f, "
               "\"decisions_per_s\": %.1f, \"kernel_us_mean\": %.1f, \"evaluated_mean\": %.1f, "
               "\"candidates_per_s\": %.4g, \"drops\": %d}\n",
               B, calls, cl[calls / 2], cl[(int)(0.99 * calls)], (double)calls * B / (tsum * 1e-6),
               kms * 1e3 / calls, (double)evsum / ((double)calls * B), (double)evsum / (tsum * 1e-6), ndrop);
        abacus_destroy(ctx);
        return 0;
    }
    double* lat = malloc(8 * ndec);
    uint64_t* ev = malloc(8 * ndec);
    int ndrop = 0;
    for (int i = 0; i < ndec; i++) {
        abacus_decision_t d;
        double t0 = now_us();
        if (space == 3)  /* multi-way search, budget = ways */
            rc = abacus_search_mway(ctx, &qs[4 * i], ks[i], nows[i], infl[i], (int32_t)budget, &d, NULL);
        else
            rc = abacus_search(ctx, &qs[4 * i], ks[i], nows[i], infl[i], space, budget, &d);
        double t1 = now_us();
        if (rc) { fprintf(stderr, "search failed %s\n", abacus_last_error(ctx)); return 1; }
        lat[i] = t1 - t0;
        ev[i] = d.evaluated;
        ndrop += d.status == ABACUS_DECIDE_DROP;
    }
    int n = ndec - warm;
    qsort(lat + warm, n, sizeof(double), cmpd);
    uint64_t evmax = 0, evsum = 0;
    for (int i = warm; i < ndec; i++) { evmax = ev[i] > evmax ? ev[i] : evmax; evsum += ev[i]; }
    /* candidates evaluated per decision (grid / chain size): percentiles */
    qsort(ev + warm, n, sizeof(uint64_t), cmpu);
    printf("{\"decisions\": %d, \"p50_us\": %.2f, \"p90_us\": %.2f, \"p99_us\": %.2f, \"p999_us\": %.2f, "
           "\"max_us\": %.2f, \"evaluated_mean\": %.1f, \"evaluated_max\": %llu, \"evaluated_p50\": %llu, "
           "\"evaluated_p90\": %llu, \"evaluated_p99\": %llu, \"drops\": %d, \"launches\": %llu}\n",
           n, lat[warm + n / 2], lat[warm + (int)(0.9 * n)], lat[warm + (int)(0.99 * n)],
           lat[warm + (int)(0.999 * n)], lat[ndec - 1], (double)evsum / n, (unsigned long long)evmax,
           (unsigned long long)ev[warm + n / 2], (unsigned long long)ev[warm + (int)(0.9 * n)],
           (unsigned long long)ev[warm + (int)(0.99 * n)], ndrop, (unsigned long long)abacus_kernel_launches(ctx));
    abacus_destroy(ctx);
    return 0;
}
