/*
 * Plain-C use of the library (include/tid.h), no Python: build an index of R synthetic references,
 * search B queries (each a noisy copy of some reference's keypoints), verify one pair.
 *
 *   gcc -O2 -I include examples/search_example.c -L paper_conf_icpp_wangzll21_b200 -ltid \
 *       -Wl,-rpath,$PWD/paper_conf_icpp_wangzll21_b200 -o /tmp/search_example && /tmp/search_example
 *
 * Host buffers throughout: the library copies to / from the GPU itself.
 */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "tid.h"

#define CHECK(call)                                                                   \
  do {                                                                                \
    tid_status s_ = (call);                                                           \
    if (s_ != TID_OK) {                                                               \
      fprintf(stderr, "%s failed (%d): %s\n", #call, (int)s_, tid_last_error());      \
      return 1;                                                                       \
    }                                                                                 \
  } while (0)

static uint32_t lcg(uint32_t* s) { return *s = *s * 1664525u + 1013904223u; }

int main(void) {
  const int32_t m = 256, n = 500, k = 5;
  const int64_t R = 1000, B = 4;
  uint32_t seed = 2021;
  uint8_t* refs = (uint8_t*)malloc((size_t)R * m * 128);
  uint8_t* qs = (uint8_t*)malloc((size_t)B * n * 128);
  for (size_t i = 0; i < (size_t)R * m * 128; ++i) refs[i] = (uint8_t)(lcg(&seed) >> 25);  /* 0..127 */
  for (int64_t b = 0; b < B; ++b) {  /* query b: 200 noisy copies of reference 17*b+3, then noise */
    const uint8_t* tgt = refs + (size_t)(17 * b + 3) * m * 128;
    for (int32_t j = 0; j < n; ++j)
      for (int t = 0; t < 128; ++t) {
        uint8_t v = (uint8_t)(lcg(&seed) >> 25);
        if (j < 200) v = (uint8_t)(tgt[(size_t)j * 128 + t] + ((lcg(&seed) >> 30) & 1));
        qs[((size_t)b * n + j) * 128 + t] = v;
      }
  }
  tid_config cfg;
  memset(&cfg, 0, sizeof cfg);
  cfg.device = 0;
  cfg.dim = 128;
  cfg.ref_kp = m;
  cfg.query_kp_max = 1024;
  cfg.ratio_num = 4;
  cfg.ratio_den = 5;
  cfg.world_size = 1;
  tid_index* idx = NULL;
  CHECK(tid_index_create(&cfg, &idx));
  int64_t first = 0;
  CHECK(tid_add_references(idx, refs, NULL, R, &first));
  int64_t ids[4 * 5];
  int32_t counts[4 * 5];
  CHECK(tid_search(idx, qs, NULL, n, B, k, ids, counts, NULL));
  for (int64_t b = 0; b < B; ++b) {
    printf("query %lld (planted %lld):", (long long)b, (long long)(17 * b + 3));
    for (int i = 0; i < k; ++i) printf(" %lld:%d", (long long)ids[b * k + i], counts[b * k + i]);
    printf("\n");
  }
  uint32_t vc = 0;
  CHECK(tid_verify(idx, qs, n, refs + (size_t)3 * m * 128, m, 1, NULL, NULL, &vc, NULL, NULL));
  printf("verify(query 0, reference 3): %u good matches\n", vc);
  CHECK(tid_index_destroy(idx));
  free(refs);
  free(qs);
  return ids[0] == 3 ? 0 : 2;
}
