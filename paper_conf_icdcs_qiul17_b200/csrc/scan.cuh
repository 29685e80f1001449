// scan.cuh -- exclusive prefix sums over the fine partitions, multi-CTA.
//
// The per-partition arrays (records, K-mers, table capacities; PAPER.md
// Sec. IV-A P:L783-788 sizes the tables from them) have up to 16,777,215
// entries, far more than one CTA scans quickly, so the sums run in three
// launches: per-tile totals (one CTA per 4096 entries), one CTA scanning the
// <= 4096 tile totals in place, and per-tile block scans offset by their
// tile's prefix.  Small arrays take one single-CTA launch instead.
#pragma once
#include <cub/block/block_reduce.cuh>
#include <cub/block/block_scan.cuh>

#include <cstdint>

#include "dbg_device.cuh"

namespace dbg {

constexpr int kTileThreads = 512, kTileItems = 8, kTileSize = kTileThreads * kTileItems;
constexpr int kTileScanThreads = 1024, kTileScanItems = 4;  // <= 4096 tiles of 4096: NP*refine <= 2^24 - 1
constexpr int kSingleCtaMax = 4 * kTileSize;                 // one launch up to this many entries

__host__ __device__ inline int scan_tiles(int n) { return (n + kTileSize - 1) / kTileSize; }

// Entry i of the scanned sequence.
struct IdentityOp {
  const uint64_t* in;
  __device__ __forceinline__ unsigned long long operator()(int i) const { return in[i]; }
};

// Table capacity of partition i (table_capacity, dbg_device.cuh); with
// slots > 0, partitions built on chip (onchip_tables > 0) count 0
// (dbg_table_plan_split).
struct CapacityOp {
  const uint64_t* in;
  double ratio;
  uint64_t slots;
  uint32_t max_split;
  __device__ __forceinline__ unsigned long long operator()(int i) const {
    const uint64_t nk = in[i], cap = table_capacity(ratio, nk);
    return slots && onchip_tables(nk, cap, slots, max_split) ? 0ull : cap;
  }
};

// sums[t] = sum of op(i) over tile t.
template <class Op>
__global__ void __launch_bounds__(kTileThreads) tile_reduce_kernel(Op op, int n, unsigned long long* sums) {
  typedef cub::BlockReduce<unsigned long long, kTileThreads> Red;
  __shared__ typename Red::TempStorage tmp;
  const int base = blockIdx.x * kTileSize;
  unsigned long long s = 0;
#pragma unroll
  for (int q = 0; q < kTileItems; ++q) {
    const int i = base + q * kTileThreads + threadIdx.x;
    if (i < n) s += op(i);
  }
  s = Red(tmp).Sum(s);
  if (threadIdx.x == 0) sums[blockIdx.x] = s;
}

// In place: sums[0..n) -> exclusive prefix, sums[n] = total (one CTA, n <= 4096).
static __global__ void __launch_bounds__(kTileScanThreads) tile_scan_kernel(unsigned long long* sums, int n) {
  typedef cub::BlockScan<unsigned long long, kTileScanThreads> Scan;
  __shared__ typename Scan::TempStorage tmp;
  unsigned long long v[kTileScanItems];
#pragma unroll
  for (int q = 0; q < kTileScanItems; ++q) {
    const int i = threadIdx.x * kTileScanItems + q;
    v[q] = i < n ? sums[i] : 0ull;
  }
  unsigned long long tot;
  Scan(tmp).ExclusiveSum(v, v, tot);
#pragma unroll
  for (int q = 0; q < kTileScanItems; ++q) {
    const int i = threadIdx.x * kTileScanItems + q;
    if (i < n) sums[i] = v[q];
  }
  if (threadIdx.x == 0) sums[n] = tot;
}

// out[i] = tile prefix + exclusive block scan; out[n] = total (last tile).
template <class Op>
__global__ void __launch_bounds__(kTileThreads) tile_apply_kernel(Op op, int n, const unsigned long long* off,
                                                                  uint64_t* out) {
  typedef cub::BlockScan<unsigned long long, kTileThreads> Scan;
  __shared__ typename Scan::TempStorage tmp;
  const int base = blockIdx.x * kTileSize + threadIdx.x * kTileItems;
  unsigned long long v[kTileItems];
#pragma unroll
  for (int q = 0; q < kTileItems; ++q) v[q] = base + q < n ? op(base + q) : 0ull;
  unsigned long long tot;
  Scan(tmp).ExclusiveSum(v, v, tot);
  const unsigned long long o = off[blockIdx.x];
#pragma unroll
  for (int q = 0; q < kTileItems; ++q)
    if (base + q < n) out[base + q] = o + v[q];
  if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) out[n] = o + tot;
}

// One CTA for small n: 512 threads x 8 items per pass, carried across passes.
template <class Op>
__global__ void __launch_bounds__(kTileThreads) single_cta_scan_kernel(Op op, int n, uint64_t* out) {
  typedef cub::BlockScan<unsigned long long, kTileThreads> Scan;
  __shared__ typename Scan::TempStorage tmp;
  __shared__ unsigned long long carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (int t0 = 0; t0 < n; t0 += kTileSize) {
    const int base = t0 + threadIdx.x * kTileItems;
    unsigned long long v[kTileItems];
#pragma unroll
    for (int q = 0; q < kTileItems; ++q) v[q] = base + q < n ? op(base + q) : 0ull;
    unsigned long long tot;
    Scan(tmp).ExclusiveSum(v, v, tot);
    const unsigned long long c = carry;
#pragma unroll
    for (int q = 0; q < kTileItems; ++q)
      if (base + q < n) out[base + q] = c + v[q];
    __syncthreads();
    if (threadIdx.x == 0) carry = c + tot;
    __syncthreads();
  }
  if (threadIdx.x == 0) out[n] = carry;
}

// out[0..n] = exclusive prefix sum of op(0..n-1), out[n] = total.  scratch:
// scan_tiles(n) + 1 words, needed only when n > kSingleCtaMax.
template <class Op>
inline cudaError_t exclusive_scan(Op op, int n, uint64_t* out, unsigned long long* scratch, cudaStream_t stream) {
  if (n <= kSingleCtaMax || scratch == nullptr) {
    single_cta_scan_kernel<Op><<<1, kTileThreads, 0, stream>>>(op, n, out);
    return cudaPeekAtLastError();
  }
  const int tiles = scan_tiles(n);
  tile_reduce_kernel<Op><<<tiles, kTileThreads, 0, stream>>>(op, n, scratch);
  tile_scan_kernel<<<1, kTileScanThreads, 0, stream>>>(scratch, tiles);
  tile_apply_kernel<Op><<<tiles, kTileThreads, 0, stream>>>(op, n, scratch, out);
  return cudaPeekAtLastError();
}

}  // namespace dbg
