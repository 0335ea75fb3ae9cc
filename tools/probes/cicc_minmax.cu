// CUDA 12.9 NVVM crash reproducer (SIGILL in cicc): min(min(v, r), v (op) r)
// built from fminf/fmaxf intrinsics.  nvcc -ptx -arch=sm_100a cicc_minmax.cu
// dies with "Illegal instruction"; fop_device.cuh's op_min/op_max use inline
// PTX min/max.f32 instead (same FMNMX instruction, no crash).
extern "C" __global__ void k(const float* x, float* y, int n) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  float v = x[i];
  float r = v > 0.f ? v : 0.f;
  float c = fmaxf(fmaxf(v, r), __fadd_rn(v, r));
  y[i] = c;
}
