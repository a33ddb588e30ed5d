// finalize.cu -- exact Pareto filter of the search's candidates by sort +
// sweep: O(m log m) for m survivors of the staircase
// prefilter (k_pareto_prefilter), any m up to the candidate capacity.
//
// Order the survivors by (T asc, E asc, index asc) -- three stable radix
// sorts (least significant key first) of the 64-bit keys; T, E > 0, so their
// IEEE bit patterns order like the values -- then a point is on the front
// iff its E is strictly below the minimum E of every point before it
// (exclusive prefix minimum).  Equal (T, E) keep their first = lowest index
// (reading R23: one index per distinct point); the output is in T-ascending
// (= X-descending) order.  The sorts, the scan and the compaction are CUB
// device primitives (library code, like cuBLAS for a GEMM); the key
// extraction, flags and gathers are the kernels below.
#include <cuda_runtime.h>

#include <cub/cub.cuh>

#include <algorithm>
#include <limits>

#include "device_common.cuh"

namespace sched {

namespace {

__global__ void k_fin_keys(const CandRec *cand, const unsigned int *surv, int m, int which,
                           unsigned long long *key, unsigned int *val) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < m; i += gridDim.x * blockDim.x) {
    if (which == 0) val[i] = (unsigned int)i;
    const CandRec c = cand[surv[val[i]]];
    key[i] = which == 0 ? c.idx : (unsigned long long)__double_as_longlong(which == 1 ? c.e : c.t);
  }
}

__global__ void k_fin_e(const CandRec *cand, const unsigned int *surv, const unsigned int *val, int m, double *e) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < m; i += gridDim.x * blockDim.x) e[i] = cand[surv[val[i]]].e;
}

__global__ void k_fin_flag(const double *e, const double *emin, int m, unsigned char *flag) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < m; i += gridDim.x * blockDim.x)
    flag[i] = e[i] < emin[i] ? 1 : 0;
}

__global__ void k_fin_out(const DevParams p, const unsigned int *surv, const unsigned int *sel, const int *nsel,
                          int out_cap) {
  const int nf = *nsel;
  const CandRec *cand = (const CandRec *)p.cand;
  CandRec *out = (CandRec *)(p.out + sizeof(BestRec) * kMaxW);
  for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < nf && r < out_cap; r += gridDim.x * blockDim.x)
    out[r] = cand[surv[sel[r]]];
  if (blockIdx.x == 0 && threadIdx.x == 0) p.ctr[kCtrFront] = (unsigned long long)nf;
}

struct MinOp {
  __device__ __forceinline__ double operator()(double a, double b) const { return b < a ? b : a; }
};

size_t al(size_t x) { return (x + 255) / 256 * 256; }

}  // namespace

constexpr size_t kFinTemp = 16u << 20;  // CUB temporary storage reserved in the workspace

size_t finalize_bytes(uint32_t cap) {
  const size_t n = cap;
  return al(8 * n) * 2 + al(4 * n) * 2 + al(8 * n) * 2 + al(n) + al(4 * n) + al(4) + kFinTemp;
}

// m survivors (indices into the candidate buffer) at surv; writes the front
// to p.out after the best records and its size to ctr[kCtrFront]
cudaError_t finalize_front(const DevParams &p, unsigned char *fin, size_t fin_bytes, const unsigned int *surv, int m,
                           int out_cap, int nsm, cudaStream_t st, int *launches) {
  const size_t n = p.cand_cap;
  if (fin_bytes < finalize_bytes(p.cand_cap) || (size_t)m > n) return cudaErrorInvalidValue;
  unsigned char *q = fin;
  auto take = [&](size_t b) {
    unsigned char *r = q;
    q += al(b);
    return r;
  };
  unsigned long long *ka = (unsigned long long *)take(8 * n), *kb = (unsigned long long *)take(8 * n);
  unsigned int *va = (unsigned int *)take(4 * n), *vb = (unsigned int *)take(4 * n);
  double *e = (double *)take(8 * n), *emin = (double *)take(8 * n);
  unsigned char *flag = take(n);
  unsigned int *sel = (unsigned int *)take(4 * n);
  int *nsel = (int *)take(4);
  void *temp = take(kFinTemp);
  const int grid = std::max(1, std::min(4 * nsm, (m + 255) / 256));
  const CandRec *cand = (const CandRec *)p.cand;

  cub::DoubleBuffer<unsigned long long> keys(ka, kb);
  cub::DoubleBuffer<unsigned int> vals(va, vb);
  size_t need = 0, t = 0;
  cudaError_t err = cub::DeviceRadixSort::SortPairs(nullptr, need, keys, vals, m, 0, 64, st);
  if (err != cudaSuccess) return err;
  err = cub::DeviceScan::ExclusiveScan(nullptr, t, e, emin, MinOp(), std::numeric_limits<double>::infinity(), m, st);
  if (err != cudaSuccess) return err;
  need = std::max(need, t);
  err = cub::DeviceSelect::Flagged(nullptr, t, va, flag, sel, nsel, m, st);
  if (err != cudaSuccess) return err;
  need = std::max(need, t);
  if (need > kFinTemp) return cudaErrorMemoryAllocation;
  // (index), then E, then T: stable least-significant-key-first radix sorts
  for (int which = 0; which < 3; which++) {
    k_fin_keys<<<grid, 256, 0, st>>>(cand, surv, m, which, keys.Current(), vals.Current());
    if ((err = cudaGetLastError()) != cudaSuccess) return err;
    size_t tb = kFinTemp;
    err = cub::DeviceRadixSort::SortPairs(temp, tb, keys, vals, m, 0, 64, st);
    if (err != cudaSuccess) return err;
  }
  k_fin_e<<<grid, 256, 0, st>>>(cand, surv, vals.Current(), m, e);
  size_t tb = kFinTemp;
  err = cub::DeviceScan::ExclusiveScan(temp, tb, e, emin, MinOp(), std::numeric_limits<double>::infinity(), m, st);
  if (err != cudaSuccess) return err;
  k_fin_flag<<<grid, 256, 0, st>>>(e, emin, m, flag);
  tb = kFinTemp;
  err = cub::DeviceSelect::Flagged(temp, tb, vals.Current(), flag, sel, nsel, m, st);
  if (err != cudaSuccess) return err;
  k_fin_out<<<grid, 256, 0, st>>>(p, surv, sel, nsel, out_cap);
  if ((err = cudaGetLastError()) != cudaSuccess) return err;
  *launches += 6;  // this file's kernels (keys x 3, e, flag, out); CUB's sort / scan / select kernels are library launches
  return cudaSuccess;
}

}  // namespace sched
