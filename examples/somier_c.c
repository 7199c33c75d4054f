/*
 * somier_c.c -- the C ABI used from plain C (no Python, no PyTorch):
 * the paper's Listing 10 pattern -- a spread over a device list, the Somier
 * step enqueued asynchronously (nowait), a taskgroup-like sync, the "centers"
 * result, and an exit-data read-back of the owned planes.
 *
 *   gcc -O2 -I include examples/somier_c.c -L paper_conf_ipps_torresft22_b200 -lsomier \
 *       -Wl,-rpath,$PWD/paper_conf_ipps_torresft22_b200 -o somier_c
 *   ./somier_c [n] [steps] [chunk]
 */
#include <stdio.h>
#include <stdlib.h>

#include "somier.h"
#include "spread.h"

#define CHECK(call)                                                                         \
    do {                                                                                    \
        spread_status st_ = (call);                                                         \
        if (st_ != SPREAD_OK) {                                                             \
            fprintf(stderr, "%s failed: %s (%s)\n", #call, spread_last_error(),            \
                    spread_status_string(st_));                                            \
            return 1;                                                                       \
        }                                                                                   \
    } while (0)

int main(int argc, char** argv) {
    const int64_t n = argc > 1 ? atoll(argv[1]) : 64;
    const int64_t steps = argc > 2 ? atoll(argv[2]) : 20;
    const int64_t chunk = argc > 3 ? atoll(argv[3]) : 0;
    /* devices(0) range(1:n-2) spread_schedule(static, chunk) */
    const int devices[1] = {0};
    spread_t sp;
    CHECK(spread_create(devices, 1, 1, n - 2, SPREAD_SCHED_STATIC, chunk, &sp));
    int64_t nchunks;
    CHECK(spread_num_chunks(sp, &nchunks));
    for (int64_t c = 0; c < nchunks && c < 4; c++) {
        int pos, id;
        int64_t start, size, first, len;
        spread_map halo = {SPREAD_MAP_TO, 1, 1};
        CHECK(spread_get_chunk(sp, c, &pos, &id, &start, &size));
        CHECK(spread_map_extent(sp, c, halo, n, &first, &len));
        printf("chunk %lld: device %d, omp_spread_start %lld, omp_spread_size %lld, map(to: X[%lld:%lld])\n",
               (long long)c, id, (long long)start, (long long)size, (long long)first, (long long)len);
    }
    somier_params p = {{n, n, n}, 1.0, 1.0, 10.0, 1.0, 1e-3, 0.05, 42, SOMIER_K1_AUTO, SOMIER_EXCHANGE_FUSED, SOMIER_MATH_EXACT, 0};
    somier_t h;
    CHECK(somier_init(sp, &p, &h));
    CHECK(spread_destroy(sp)); /* the handle keeps its own copy */
    CHECK(somier_step(h, steps)); /* nowait */
    CHECK(somier_sync(h));        /* taskgroup */
    somier_stats_t st;
    CHECK(somier_stats(h, &st));
    printf("step %lld centre (%.17g, %.17g, %.17g) vmax %.17g nodes %lld\n", (long long)st.step, st.centre[0],
           st.centre[1], st.centre[2], st.vmax, (long long)st.nodes);
    /* the "centers" of every step: the last few from the history */
    const int64_t nh = steps < 4 ? steps : 4;
    somier_stats_t hist[4];
    CHECK(somier_stats_history(h, steps - nh + 1, nh, hist));
    for (int64_t i = 0; i < nh; i++)
        printf("history step %lld centre (%.17g, %.17g, %.17g) vmax %.17g\n", (long long)hist[i].step,
               hist[i].centre[0], hist[i].centre[1], hist[i].centre[2], hist[i].vmax);
    const size_t N = (size_t)(n * n * n);
    double* g = (double*)malloc(6 * N * sizeof(double));
    if (!g) return 1;
    CHECK(somier_read(h, g, g + N, g + 2 * N, g + 3 * N, g + 4 * N, g + 5 * N));
    const size_t mid = (size_t)((n / 2 * n + n / 2) * n + n / 2);
    printf("x[%lld,%lld,%lld] = (%.17g, %.17g, %.17g)\n", (long long)(n / 2), (long long)(n / 2), (long long)(n / 2),
           g[mid], g[N + mid], g[2 * N + mid]);
    free(g);
    CHECK(somier_destroy(h));
    return 0;
}
