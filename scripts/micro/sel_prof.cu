// Timing harness for select_fused_kernel variants (dev tool, not product code):
// includes the library sources into one TU so -DRA_SEL_VEC=... / -DRA_SEL_PROFILE
// builds of the kernel can be compared on one box.
//   usage: sel_prof [T0 [T1 ...]]   (LT thresholds of the chain; default 0 -2^30)
#include "../../paper_conf_ipps_wudwcyc12_b200/csrc/capi.cu"
#include "../../paper_conf_ipps_wudwcyc12_b200/csrc/select_fused.cu"
#include "../../paper_conf_ipps_wudwcyc12_b200/csrc/q1_fused.cu"
#include "../../paper_conf_ipps_wudwcyc12_b200/csrc/q1_narrow.cu"
#include "../../paper_conf_ipps_wudwcyc12_b200/csrc/gather.cu"
#include "../../paper_conf_ipps_wudwcyc12_b200/csrc/compact.cu"
#include <cstdlib>
#ifndef VARIANT
#define VARIANT "full"
#endif

__global__ void fill(int32_t* x, int64_t n, uint64_t seed) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    uint64_t z = seed + i * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; z ^= z >> 31;
    x[i] = (int32_t)(z >> 32);
  }
}

int main(int argc, char** argv) {
  int64_t n = 1ll << 28;
  int32_t *x, *out; int64_t* cnt; void* ws;
  ra_pred p[RA_MAX_PREDS];
  int k = 0;
  for (int a = 1; a < argc && k < RA_MAX_PREDS; ++a) p[k++] = {RA_LT, (int32_t)strtoll(argv[a], 0, 0)};
  if (!k) { p[0] = {RA_LT, 0}; p[1] = {RA_LT, -1073741824}; k = 2; }
  cudaMalloc(&x, n * 4); cudaMalloc(&out, n * 4); cudaMalloc(&cnt, 8);
  size_t wsb = ra_select_workspace_bytes(n, k, 1);
  cudaMalloc(&ws, wsb); cudaMemset(ws, 0, wsb);
  fill<<<1184, 256>>>(x, n, 7);
  for (int i = 0; i < 3; ++i) ra_select_chain(x, n, p, k, 1, out, n, cnt, ws, wsb, 0);
  cudaDeviceSynchronize();
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a);
  const int reps = 20;
  for (int i = 0; i < reps; ++i) ra_select_chain(x, n, p, k, 1, out, n, cnt, ws, wsb, 0);
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  ms /= reps;
  int64_t c; cudaMemcpy(&c, cnt, 8, cudaMemcpyDeviceToHost);
  printf("%-24s thr %-12d ms %.4f  GB/s %.0f  count %lld  ctas/sm %d smem %zu err=%s\n", VARIANT, p[k - 1].value, ms,
         (4.0 * n + 4.0 * c) / ms / 1e6, (long long)c, ra::sel_ctas_per_sm(), sizeof(ra::SelSmem),
         cudaGetErrorString(cudaGetLastError()));
  {  // verify the last launch's output against a host filter (dev check)
    int32_t* hx = (int32_t*)malloc(n * 4);
    int32_t* ho = (int32_t*)malloc(n * 4);
    cudaMemcpy(hx, x, n * 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(ho, out, c * 4, cudaMemcpyDeviceToHost);
    int64_t m = 0, bad = 0;
    for (int64_t i = 0; i < n; ++i) {
      bool keep = true;
      for (int j = 0; j < k; ++j) keep &= hx[i] < p[j].value;
      if (keep) { if (m < c && ho[m] != hx[i]) ++bad; ++m; }
    }
    printf("  verify: expected count %lld, mismatches %lld -> %s\n", (long long)m, (long long)bad,
           (m == c && bad == 0) ? "OK" : "FAIL");
    free(hx); free(ho);
  }
#ifdef RA_SEL_PROFILE
  unsigned long long z[16];
  cudaMemcpyFromSymbol(z, ra::g_sel_prof, sizeof(z));
  const double tiles = z[5] ? (double)z[5] : 1.0;
  printf("  per tile (cycles, summed over all launches): repolls %.3f full-wait w0 %.0f w7 %.0f | placed-wait %.0f | B1 w0 %.0f w7 %.0f | loop %.0f\n"
         "  lookback: counted-wait %.0f winfull-wait %.0f window-sum %.0f | producer: empty-wait %.0f atomic %.0f\n"
         "  windows: uncopied (too long) %.4f per tile, mean length %.1f\n",
         z[0] / tiles, z[1] / tiles, z[8] / tiles, z[2] / tiles, z[3] / tiles, z[13] / tiles, z[4] / tiles, z[9] / tiles,
         z[6] / tiles, z[7] / tiles, z[11] / tiles, z[12] / tiles, z[14] / tiles, z[15] / tiles);
#endif
  return 0;
}
