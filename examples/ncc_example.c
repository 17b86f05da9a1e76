/* examples/ncc_example.c -- the C ABI without Python: template matching on a synthetic
 * frame with a planted template, end to end through ncc_match_host (host buffers).
 *
 *   gcc -O2 -I include examples/ncc_example.c -o ncc_example \
 *       -L paper_conf_ipps_moorelk13_b200 -lncc_b200 -Wl,-rpath,$PWD/paper_conf_ipps_moorelk13_b200
 *   ./ncc_example            # prints the peak; exit code 0 iff it is the planted offset
 */
#include <stdio.h>
#include <stdlib.h>

#include "ncc.h"

static unsigned int lcg(unsigned int* s) { return *s = *s * 1664525u + 1013904223u; }

int main(void) {
    const int H = 512, W = 512, h = 48, w = 40, u0 = 123, v0 = 301;
    float* img = (float*)malloc(sizeof(float) * H * W);
    float* tmpl = (float*)malloc(sizeof(float) * h * w);
    unsigned int seed = 12345u;
    for (int i = 0; i < H * W; ++i) img[i] = (float)(lcg(&seed) >> 8) / 16777216.0f;
    for (int i = 0; i < h; ++i)
        for (int j = 0; j < w; ++j) tmpl[i * w + j] = img[(u0 + i) * W + (v0 + j)];

    ncc_problem p = {0};
    p.mode = NCC_MODE_MATCH;
    p.score = NCC_SCORE_NCC;
    p.image_h = H;
    p.image_w = W;
    p.image_pitch = W;
    p.tmpl_h = h;
    p.tmpl_w = w;
    p.batch = 1;
    p.shard_count = 1;
    ncc_plan plan = NULL;
    ncc_status st = ncc_plan_create(&p, 0, &plan);
    if (st != NCC_OK) {
        fprintf(stderr, "ncc_plan_create: %s %s\n", ncc_status_string(st), ncc_last_cuda_error());
        return 2;
    }
    ncc_plan_info info;
    ncc_plan_query(plan, &info, sizeof(info));
    ncc_peak peak;
    st = ncc_match_host(plan, img, tmpl, w, NULL, &peak, NULL);
    if (st != NCC_OK) {
        fprintf(stderr, "ncc_match_host: %s %s\n", ncc_status_string(st), ncc_last_cuda_error());
        return 3;
    }
    ncc_plan_destroy(plan); /* waits for the plan's work: the peak is in host memory now */
    printf("variant %s (tier %d): peak score %.6f at (%d, %d), planted (%d, %d)\n", info.variant_name,
           info.specialized, peak.score, peak.u, peak.v, u0, v0);
    free(img);
    free(tmpl);
    return (peak.u == u0 && peak.v == v0 && peak.score > 0.9999f) ? 0 : 1;
}
