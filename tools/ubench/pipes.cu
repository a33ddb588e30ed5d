// Pipe-throughput microbenchmark ("the INT32 rate on sm_100
// must be measured, not assumed"): thread-instructions per clock per SM for
// the instructions the tile kernel is made of.  8 independent chains per
// thread, 148 x 4 CTAs of 256 threads, clock64 per CTA.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o pipes pipes.cu && ./pipes
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ float max3f(float a, float b, float c) {
  float d; asm volatile("max.f32 %0, %1, %2, %3;" : "=f"(d) : "f"(a), "f"(b), "f"(c)); return d; }
__device__ __forceinline__ float max2f(float a, float b) {
  float d; asm volatile("max.f32 %0, %1, %2;" : "=f"(d) : "f"(a), "f"(b)); return d; }
__device__ __forceinline__ float add1f(float a, float b) {
  float d; asm volatile("add.rn.f32 %0, %1, %2;" : "=f"(d) : "f"(a), "f"(b)); return d; }
__device__ __forceinline__ unsigned iadd3(unsigned a, unsigned b, unsigned c) {
  unsigned d; asm volatile("add.u32 %0, %1, %2;\n\tadd.u32 %0, %0, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c)); return d; }
__device__ __forceinline__ unsigned lop3(unsigned a, unsigned b, unsigned c) {
  unsigned d; asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(d) : "r"(a), "r"(b), "r"(c)); return d; }
__device__ __forceinline__ unsigned imad(unsigned a, unsigned b, unsigned c) {
  unsigned d; asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c)); return d; }
__device__ __forceinline__ float ffma(float a, float b, float c) {
  float d; asm volatile("fma.rn.f32 %0, %1, %2, %3;" : "=f"(d) : "f"(a), "f"(b), "f"(c)); return d; }
__device__ __forceinline__ unsigned long long add2f(unsigned long long a, unsigned long long b) {
  unsigned long long d; asm volatile("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b)); return d; }

constexpr int R = 1 << 14;
template <int OP>
__global__ void k(float *out, long long *clk, float s) {
  float x[8];
  unsigned long long y[8];
  unsigned z[8];
  __shared__ float sh[1024];
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) sh[i] = s * i;
  for (int i = 0; i < 8; i++) { x[i] = s * (threadIdx.x + i); y[i] = __float_as_uint(x[i]) * 0x100000001ull; z[i] = threadIdx.x * 7 + i; }
  const float xs = s * 0.5f;
  const unsigned zs = 0x9e3779b9u;
  const unsigned long long ys = y[7] ^ 0x1ull;
  __syncthreads();
  long long t0 = clock64();
#pragma unroll 1
  for (int r = 0; r < R; r++) {
#pragma unroll
    for (int i = 0; i < 8; i++) {
      if (OP == 0) x[i] = max2f(x[i], s);
      if (OP == 1) x[i] = max3f(x[i], s, xs);
      if (OP == 2) x[i] = add1f(x[i], s);
      if (OP == 3) y[i] = add2f(y[i], ys);
      if (OP == 4) { x[i] = max2f(x[i], s); x[(i + 4) & 7] = add1f(x[(i + 4) & 7], s); }
      if (OP == 5) { x[i] = max3f(x[i], s, xs); y[i] = add2f(y[i], ys); }
      if (OP == 6) { x[i] = max3f(x[i], s, xs); x[(i + 4) & 7] = add1f(x[(i + 4) & 7], s); }
      if (OP == 7) { x[i] = max2f(x[i], s); y[i] = add2f(y[i], ys); }
      if (OP == 8) z[i] = lop3(z[i], zs, z[(i + 1) & 7]);
      if (OP == 9) z[i] = imad(z[i], zs, z[(i + 1) & 7]);
      if (OP == 10) x[i] = ffma(x[i], s, xs);
      if (OP == 11) x[i] = x[i] + sh[(z[i] + i * 33 + r) & 1023];
    }
  }
  __syncthreads();
  long long t1 = clock64();
  float a = 0;
  for (int i = 0; i < 8; i++) a += x[i] + __uint_as_float((unsigned)y[i]) + (float)z[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = a;
  if (threadIdx.x == 0) clk[blockIdx.x] = t1 - t0;
}

template <int OP>
void run(const char *name, int ninstr_per_iter, int blocks_per_sm) {
  int nsm;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  const int nb = nsm * blocks_per_sm, nt = 256;
  float *out;
  long long *clk;
  cudaMalloc(&out, sizeof(float) * nb * nt);
  cudaMallocManaged(&clk, sizeof(long long) * nb);
  k<OP><<<nb, nt>>>(out, clk, 1.0001f);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  k<OP><<<nb, nt>>>(out, clk, 1.0001f);
  cudaEventRecord(e1);
  cudaDeviceSynchronize();
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  long long mx = 0;
  for (int b = 0; b < nb; b++) mx = clk[b] > mx ? clk[b] : mx;
  const double thr_instr = (double)nb * nt * R * 8 * ninstr_per_iter;
  printf("%-28s warps/SM %2d  thread-instr/clk/SM %6.1f  (%.3e thread-instr/s, %.3f ms)\n", name,
         blocks_per_sm * 8, thr_instr / nsm / mx * blocks_per_sm / blocks_per_sm, thr_instr / (ms * 1e-3), ms);
  cudaFree(out);
  cudaFree(clk);
}

int main() {
  for (int bps : {2, 3}) {
    run<0>("FMNMX (2-input max)", 1, bps);
    run<1>("FMNMX3 (3-input max)", 1, bps);
    run<2>("FADD", 1, bps);
    run<3>("FADD2 (f32x2)", 1, bps);
    run<4>("FMNMX + FADD interleaved", 2, bps);
    run<5>("FMNMX3 + FADD2 interleaved", 2, bps);
    run<6>("FMNMX3 + FADD interleaved", 2, bps);
    run<7>("FMNMX + FADD2 interleaved", 2, bps);
    run<8>("LOP3", 1, bps);
    run<9>("IMAD", 1, bps);
    run<10>("FFMA", 1, bps);
    run<11>("LDS (loads only; +LOP3,IADD,FADD each)", 1, bps);
  }
  return 0;
}
