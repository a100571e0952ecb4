// scan.cuh — exclusive prefix sums (u32 counts -> u64 offsets) on the device.
// Used for EF block payload offsets (index build) and for per-query unit /
// region offsets (query planning).  out[n] receives the total.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

namespace griffin {

constexpr int kScanThreads = 1024;
constexpr int kScanItems = 8;
constexpr uint32_t kScanTile = kScanThreads * kScanItems;

template <class T>
__device__ __forceinline__ T block_excl_scan(T v, T *warp_sums, T *total) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  T x = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    T t = __shfl_up_sync(0xffffffffu, x, d);
    if (lane >= d) x += t;
  }
  if (lane == 31) warp_sums[wid] = x;
  __syncthreads();
  if (wid == 0) {
    const int nw = blockDim.x >> 5;
    T s = lane < nw ? warp_sums[lane] : T(0);
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      T t = __shfl_up_sync(0xffffffffu, s, d);
      if (lane >= d) s += t;
    }
    if (lane < nw) warp_sums[lane] = s;  // inclusive warp prefix
    if (lane == nw - 1) *total = s;
  }
  __syncthreads();
  const T wpre = wid ? warp_sums[wid - 1] : T(0);
  const T r = wpre + x - v;
  __syncthreads();
  return r;
}

// Single-CTA scan for any n (loops over tiles); base added to everything.
template <class TIn>
__global__ void __launch_bounds__(kScanThreads) scan_single_kernel(const TIn *in, uint64_t *out,
                                                                   uint64_t n, uint64_t *total_out) {
  __shared__ uint64_t ws[32];
  __shared__ uint64_t tot;
  uint64_t carry = 0;
  for (uint64_t t0 = 0; t0 < n; t0 += kScanTile) {
    uint64_t loc[kScanItems];
    uint64_t s = 0;
#pragma unroll
    for (int i = 0; i < kScanItems; ++i) {
      uint64_t idx = t0 + (uint64_t)threadIdx.x * kScanItems + i;
      loc[i] = idx < n ? (uint64_t)in[idx] : 0;
      s += loc[i];
    }
    uint64_t pre = block_excl_scan<uint64_t>(s, ws, &tot);
    uint64_t run = carry + pre;
#pragma unroll
    for (int i = 0; i < kScanItems; ++i) {
      uint64_t idx = t0 + (uint64_t)threadIdx.x * kScanItems + i;
      if (idx < n) out[idx] = run;
      run += loc[i];
    }
    carry += tot;
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    out[n] = carry;
    if (total_out) *total_out = carry;
  }
}

template <class TIn>
__global__ void __launch_bounds__(kScanThreads) scan_tile_sums(const TIn *in, uint64_t n,
                                                               uint64_t *tsum) {
  __shared__ uint64_t ws[32];
  __shared__ uint64_t tot;
  const uint64_t t0 = (uint64_t)blockIdx.x * kScanTile;
  uint64_t s = 0;
#pragma unroll
  for (int i = 0; i < kScanItems; ++i) {
    uint64_t idx = t0 + (uint64_t)threadIdx.x * kScanItems + i;
    if (idx < n) s += (uint64_t)in[idx];
  }
  block_excl_scan<uint64_t>(s, ws, &tot);
  if (threadIdx.x == 0) tsum[blockIdx.x] = tot;
}

template <class TIn>
__global__ void __launch_bounds__(kScanThreads) scan_tile_apply(const TIn *in, uint64_t n,
                                                                const uint64_t *toff,
                                                                uint64_t *out) {
  __shared__ uint64_t ws[32];
  __shared__ uint64_t tot;
  const uint64_t t0 = (uint64_t)blockIdx.x * kScanTile;
  uint64_t loc[kScanItems];
  uint64_t s = 0;
#pragma unroll
  for (int i = 0; i < kScanItems; ++i) {
    uint64_t idx = t0 + (uint64_t)threadIdx.x * kScanItems + i;
    loc[i] = idx < n ? (uint64_t)in[idx] : 0;
    s += loc[i];
  }
  uint64_t run = toff[blockIdx.x] + block_excl_scan<uint64_t>(s, ws, &tot);
#pragma unroll
  for (int i = 0; i < kScanItems; ++i) {
    uint64_t idx = t0 + (uint64_t)threadIdx.x * kScanItems + i;
    if (idx < n) out[idx] = run;
    run += loc[i];
  }
}

// out[0..n] (n+1 entries).  `tmp` must hold ceil(n/kScanTile)+1 u64.
template <class TIn>
inline cudaError_t exclusive_scan(const TIn *in, uint64_t *out, uint64_t n, uint64_t *tmp,
                                  cudaStream_t st, uint64_t *nlaunch = nullptr) {
  const uint64_t ntiles = (n + kScanTile - 1) / kScanTile;
  if (ntiles <= 4) {
    scan_single_kernel<TIn><<<1, kScanThreads, 0, st>>>(in, out, n, nullptr);
    if (nlaunch) *nlaunch += 1;
    return cudaGetLastError();
  }
  if (nlaunch) *nlaunch += 3;
  scan_tile_sums<TIn><<<(unsigned)ntiles, kScanThreads, 0, st>>>(in, n, tmp);
  scan_single_kernel<uint64_t><<<1, kScanThreads, 0, st>>>(tmp, tmp, ntiles, nullptr);
  scan_tile_apply<TIn><<<(unsigned)ntiles, kScanThreads, 0, st>>>(in, n, tmp, out);
  // out[n] = total
  return cudaMemcpyAsync(out + n, tmp + ntiles, sizeof(uint64_t), cudaMemcpyDeviceToDevice, st);
}

}  // namespace griffin
