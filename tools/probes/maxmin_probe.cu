// Probe: does the hardware max/min (FMNMX) order -0 < +0 and ignore NaN like the oracle's op_max/op_min?
#include <cstdio>
#include <cmath>
#include <cstring>
__global__ void k(const float* a, const float* b, float* mx, float* mn, int n) {
  int i = threadIdx.x;
  if (i < n) { mx[i] = fmaxf(a[i], b[i]); mn[i] = fminf(a[i], b[i]); }
}
int main() {
  const int n = 8;
  float a[n] = {-0.f, 0.f, -0.f, 0.f, NAN, 1.f, NAN, -1.f};
  float b[n] = {0.f, -0.f, -0.f, 0.f, 1.f, NAN, NAN, -0.f};
  float *da, *db, *dx, *dn;
  cudaMalloc(&da, 64); cudaMalloc(&db, 64); cudaMalloc(&dx, 64); cudaMalloc(&dn, 64);
  cudaMemcpy(da, a, 32, cudaMemcpyHostToDevice); cudaMemcpy(db, b, 32, cudaMemcpyHostToDevice);
  k<<<1, 32>>>(da, db, dx, dn, n);
  float x[n], m[n];
  cudaMemcpy(x, dx, 32, cudaMemcpyDeviceToHost); cudaMemcpy(m, dn, 32, cudaMemcpyDeviceToHost);
  for (int i = 0; i < n; i++) {
    unsigned ux, um; memcpy(&ux, &x[i], 4); memcpy(&um, &m[i], 4);
    printf("a=%g b=%g  max=%g (0x%08x)  min=%g (0x%08x)\n", a[i], b[i], x[i], ux, m[i], um);
  }
}
