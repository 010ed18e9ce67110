// Does redux.sync with per-segment membermasks (different lanes of one converged warp naming
// different masks) give segmented reductions on sm_100a?  int add and f32 max.
#include <cstdio>
#include <cstdint>
__global__ void k(const int* vals, const float* fv, const unsigned* seg_mask, int* out_add, float* out_max, int n) {
  int w = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32;
  if (w >= n) return;
  int lane = threadIdx.x & 31;
  unsigned m = seg_mask[w * 32 + lane];
  int v = vals[w * 32 + lane];
  float f = fv[w * 32 + lane];
  int r = __reduce_add_sync(m, v);
  float mx;
  asm volatile("redux.sync.max.f32 %0, %1, %2;" : "=f"(mx) : "f"(f), "r"(m));
  out_add[w * 32 + lane] = r;
  out_max[w * 32 + lane] = mx;
}
int main() {
  const int n = 4096;
  int *v, *oa; float *f, *om; unsigned* sm;
  cudaMallocManaged(&v, n * 32 * 4); cudaMallocManaged(&oa, n * 32 * 4);
  cudaMallocManaged(&f, n * 32 * 4); cudaMallocManaged(&om, n * 32 * 4); cudaMallocManaged(&sm, n * 32 * 4);
  unsigned long long s = 12345;
  auto rnd = [&]() { s = s * 6364136223846793005ULL + 1442695040888963407ULL; return (unsigned)(s >> 33); };
  for (int w = 0; w < n; ++w) {
    int l = 0;
    while (l < 32) {
      int len = 1 + rnd() % 12; if (l + len > 32) len = 32 - l;
      unsigned mask = (len == 32) ? 0xffffffffu : (((1u << len) - 1u) << l);
      for (int j = l; j < l + len; ++j) sm[w * 32 + j] = mask;
      l += len;
    }
    for (int j = 0; j < 32; ++j) { v[w * 32 + j] = (int)(rnd() % 100000) - 50000; f[w * 32 + j] = (float)((int)(rnd() % 20001) - 10000) * 0.37f; }
  }
  k<<<n / 8, 256>>>(v, f, sm, oa, om, n);
  cudaError_t e = cudaDeviceSynchronize();
  if (e) { printf("cuda error %s\n", cudaGetErrorString(e)); return 1; }
  long bad_a = 0, bad_m = 0;
  for (int w = 0; w < n; ++w)
    for (int j = 0; j < 32; ++j) {
      unsigned mask = sm[w * 32 + j]; int sa = 0; float mx = -1e30f;
      for (int i = 0; i < 32; ++i) if (mask >> i & 1) { sa += v[w * 32 + i]; mx = fmaxf(mx, f[w * 32 + i]); }
      bad_a += sa != oa[w * 32 + j]; bad_m += mx != om[w * 32 + j];
    }
  printf("segmented redux: add mismatches %ld, f32 max mismatches %ld (of %d)\n", bad_a, bad_m, n * 32);
  return 0;
}
