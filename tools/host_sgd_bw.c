/* Host-side SGD throughput (the "bf16 H2D with host-side fp32 masters" option of SURVEY
 * §8f(3)): w32 -= lr * g16 (bf16 gradient from the device), then the bf16
 * shadow for the next H2D, over n parameters with T threads.  Prints GB/s of host DRAM
 * traffic (4 + 2 + 4 + 2 bytes per parameter) and ms per 1e9 parameters.
 *   gcc -O3 -fopenmp tools/host_sgd_bw.c -o /tmp/host_sgd_bw && /tmp/host_sgd_bw [n] */
#include <omp.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

static inline float bf2f(uint16_t h) { uint32_t u = (uint32_t)h << 16; float f; memcpy(&f, &u, 4); return f; }
static inline uint16_t f2bf(float f) { uint32_t u; memcpy(&u, &f, 4); u += 0x7fff + ((u >> 16) & 1); return (uint16_t)(u >> 16); }

int main(int argc, char** argv) {
  const size_t n = argc > 1 ? strtoull(argv[1], 0, 10) : (size_t)1 << 29;
  float* w = aligned_alloc(64, n * 4);
  uint16_t* g = aligned_alloc(64, n * 2);
  uint16_t* s = aligned_alloc(64, n * 2);
#pragma omp parallel for schedule(static)
  for (size_t i = 0; i < n; ++i) { w[i] = (float)(i % 1000) * 1e-3f; g[i] = f2bf(1e-2f); s[i] = 0; }
  const float lr = 0.01f;
  double best = 1e30;
  for (int rep = 0; rep < 5; ++rep) {
    const double t0 = omp_get_wtime();
#pragma omp parallel for schedule(static)
    for (size_t i = 0; i < n; ++i) {
      const float v = w[i] - lr * bf2f(g[i]);
      w[i] = v;
      s[i] = f2bf(v);
    }
    const double t = omp_get_wtime() - t0;
    if (t < best) best = t;
  }
  printf("threads %d  n %zu  best %.3f s  %.1f GB/s  %.1f ms per 1e9 params\n", omp_get_max_threads(), n, best,
         12.0 * n / best / 1e9, best / n * 1e12);
  return (int)(w[n / 2] > 1e9);
}
