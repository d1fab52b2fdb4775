// Phase-timer harness for select_fused_kernel (built with -DRA_SEL_PROFILE).
// Not product code: includes the library sources into one TU.
#include "../../paper_conf_ipps_wudwcyc12_b200/csrc/capi.cu"
#include "../../paper_conf_ipps_wudwcyc12_b200/csrc/select_fused.cu"
#include "../../paper_conf_ipps_wudwcyc12_b200/csrc/q1_fused.cu"
#include <vector>
#ifndef VARIANT
#define VARIANT "full"
#endif
#include <cstdlib>

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
  cudaMalloc(&x, n * 4); cudaMalloc(&out, n * 4); cudaMalloc(&cnt, 8);
  size_t wsb = ra_select_workspace_bytes(n, 2, 1);
  cudaMalloc(&ws, wsb); cudaMemset(ws, 0, wsb);
  fill<<<1184, 256>>>(x, n, 7);
  ra_pred p[2] = {{RA_LT, 0}, {RA_LT, -1073741824}};
  for (int i = 0; i < 3; ++i) ra_select_chain(x, n, p, 2, 1, out, n, cnt, ws, wsb, 0);
  cudaDeviceSynchronize();
  unsigned long long* trace; cudaMalloc(&trace, 8 * ((n + 4095) / 4096));
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a);
  const int reps = 10;
  for (int i = 0; i < reps; ++i) ra_select_chain(x, n, p, 2, 1, out, n, cnt, ws, wsb, 0);
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  int64_t c; cudaMemcpy(&c, cnt, 8, cudaMemcpyDeviceToHost);
  printf("%-28s ms/call %.4f  count %lld  ctas/sm %d  err=%s\n", VARIANT, ms / reps, (long long)c, ra::sel_ctas_per_sm(),
         cudaGetErrorString(cudaGetLastError()));
#ifdef RA_SEL_PROFILE
  {
    cudaMemcpyToSymbol(ra::g_sel_trace, &trace, sizeof(trace));
    ra_select_chain(x, n, p, 2, 1, out, n, cnt, ws, wsb, 0);
    cudaDeviceSynchronize();
    int64_t nt = (n + 4095) / 4096;
    std::vector<unsigned long long> tr(nt);
    cudaMemcpy(tr.data(), trace, 8 * nt, cudaMemcpyDeviceToHost);
    int G = 296; unsigned long long t0 = ~0ull;
    for (auto v : tr) t0 = v < t0 ? v : t0;
    // per round: spread (max - min) of count times, and mean lag of CTA b vs CTA 0
    double spread = 0; int rounds = (int)(nt / G);
    double lagsum[8] = {0};
    for (int r = 0; r < rounds; ++r) {
      unsigned long long lo = ~0ull, hi = 0;
      for (int bb = 0; bb < G; ++bb) { auto v = tr[(int64_t)r * G + bb]; lo = v < lo ? v : lo; hi = v > hi ? v : hi; }
      spread += hi - lo;
      for (int q = 0; q < 8; ++q) lagsum[q] += (double)tr[(int64_t)r * G + q * 37] - (double)tr[(int64_t)r * G];
    }
    printf("rounds %d: mean round spread %.0f ns; total %.0f ns; per-round time %.0f ns\n", rounds, spread / rounds,
           (double)(tr[nt - 1] - t0), (double)(tr[nt - 1] - t0) / rounds);
    for (int q = 0; q < 8; ++q) printf("  CTA %3d mean lag vs CTA 0: %8.0f ns\n", q * 37, lagsum[q] / rounds);
  }
  unsigned long long z[8];
  cudaMemcpyFromSymbol(z, ra::g_sel_prof, sizeof(z));
  printf("per tile: repolls %.3f  wait_placed(due) %.0f cyc  wait_data %.0f cyc\n", (double)z[0] / z[3], (double)z[1] / z[3], (double)z[2] / z[3]);
#endif
  return 0;
}
