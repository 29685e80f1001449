// dbg_device.cuh -- device helpers shared by the sm_100a kernels of libdbg.so.
// Product code: never includes or links anything under oracle/.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "../../include/dbg.h"

namespace dbg {

constexpr int kWarp = 32;
constexpr uint32_t kFull = 0xffffffffu;
// Record header (dbg.h): n_kmers (bits 0-5, <= 63) | has_left (bit 6) | has_right (bit 7) |
// fine pid (bits 8-31): up to 2^24 - 1 fine partitions.
constexpr uint32_t kMaxPid = (1u << 24) - 1;
constexpr int kHdrPidShift = 8;
constexpr uint32_t kHdrNMask = 63u;
__host__ __device__ __forceinline__ uint32_t rec_header(uint32_t n, uint32_t hl, uint32_t hr, uint32_t pid) {
  return n | hl << 6 | hr << 7 | pid << kHdrPidShift;
}
__host__ __device__ __forceinline__ uint32_t hdr_n(uint32_t h) { return h & kHdrNMask; }
__host__ __device__ __forceinline__ uint32_t hdr_hl(uint32_t h) { return (h >> 6) & 1u; }
__host__ __device__ __forceinline__ uint32_t hdr_hr(uint32_t h) { return (h >> 7) & 1u; }
__host__ __device__ __forceinline__ uint32_t hdr_pid(uint32_t h) { return h >> kHdrPidShift; }
constexpr uint64_t kOccupied = 1ull << 63;

// Status bits (dbg_sync_status).
constexpr uint32_t kStatusTableFull = 1u;
constexpr uint32_t kStatusNoSpace = 2u;

// Record geometry (dbg.h): 4 words (48 bases) for K <= 39, 8 (112 bases) for
// K <= 63, 16 (240 bases) for K <= 127 (row f3).
__host__ __device__ inline uint32_t record_words(int k) { return k <= 39 ? 4u : (k <= 63 ? 8u : 16u); }
__host__ __device__ inline uint32_t record_max_kmers(int k) {
  // bases = 16 * (R - 1) >= has_left + n + K - 1 + has_right, and n fits the header's 6 bits
  const uint32_t n = 16u * (record_words(k) - 1u) - (uint32_t)k - 1u;
  return n < kHdrNMask ? n : kHdrNMask;
}

// Number of fine partitions the device works on (dbg.h: num_partitions * refine).
__host__ __device__ inline int fine_partitions(const dbg_params* prm) {
  return prm->num_partitions * (prm->refine > 1 ? prm->refine : 1);
}

// Minimizer length of the device's fine partitioning (dbg.h fine_p; 0 = P).
__host__ __device__ inline int partition_p(const dbg_params* prm) { return prm->fine_p ? prm->fine_p : prm->p; }

// Table capacity of a partition (Sec. IV-A): ceil(lambda/(4 alpha)
// * N^i_kmer), at least 1 when the partition is not empty.
__host__ __device__ inline uint64_t table_capacity(double ratio, uint64_t nk) {
  if (nk == 0) return 0;
  const double c = ceil(ratio * (double)nk);
  return c < 1.0 ? 1ull : (uint64_t)c;
}

// On-chip path (hash.cu): a partition's table lives in one CTA's shared memory
// ("grouped", 1) when its capacity fits the CTA table, or is split over ns >= 2
// CTA tables, ns = ceil(1.25 cap / slots) <= max_split; otherwise (0) it takes
// the global tables.  On-chip counters are 16 bits wide and a vertex's count
// never exceeds its partition's N^i_kmer, so only partitions with
// N^i_kmer <= 65535 go on chip.
constexpr uint64_t kSmemMaxKmers = 65535;
constexpr int32_t kDefaultSmemSplit = 32, kMaxSmemSplit = 64;
__host__ __device__ inline uint32_t smem_max_split(const dbg_params* prm) {
  const int32_t m = prm->smem_split == 0 ? kDefaultSmemSplit : prm->smem_split;
  return (uint32_t)(m < 1 ? 1 : (m > kMaxSmemSplit ? kMaxSmemSplit : m));
}
__host__ __device__ inline uint32_t onchip_tables(uint64_t nk, uint64_t cap, uint64_t slots, uint32_t max_split) {
  if (nk == 0 || nk > kSmemMaxKmers) return 0;
  if (cap <= slots) return 1;
  if (max_split < 2) return 0;
  const uint64_t ns = (5 * cap + 4 * slots - 1) / (4 * slots);
  return ns <= max_split ? (uint32_t)ns : 0u;
}

// MurmurHash3 64-bit finaliser: the partition function of reading I
// ("superkmer ID ... from the minimizer's hash bit value with a modulo",
// P:L455-459), and the slot hash of the tables.
__host__ __device__ __forceinline__ uint64_t fmix64(uint64_t k) {
  k ^= k >> 33;
  k *= 0xff51afd7ed558ccdULL;
  k ^= k >> 33;
  k *= 0xc4ceb9fe1a85ec53ULL;
  k ^= k >> 33;
  return k;
}

// Unsigned 64-bit division by an invariant integer (Granlund & Montgomery
// 1994, Fig. 4.1): exact x mod d for every 64-bit x, d >= 1.
struct FastMod {
  uint64_t d, m;
  int sh1, sh2;
};

inline FastMod make_fastmod(uint64_t d) {
  int l = 0;
  while (l < 64 && (1ull << l) < d) ++l;  // l = ceil(log2 d)
  FastMod f;
  f.d = d;
  const unsigned __int128 two_l = (unsigned __int128)1 << l;
  f.m = (uint64_t)((((unsigned __int128)1 << 64) * (two_l - d)) / d + 1);
  f.sh1 = l < 1 ? l : 1;
  f.sh2 = l - 1 > 0 ? l - 1 : 0;
  return f;
}

__device__ __forceinline__ uint32_t fast_mod(const FastMod& f, uint64_t x) {
  const uint64_t t1 = __umul64hi(f.m, x);
  const uint64_t q = (t1 + ((x - t1) >> f.sh1)) >> f.sh2;
  return (uint32_t)(x - q * f.d);
}

// Reverse complement of a P-mer held in the low 2P bits (reading A:
// complement = 3 - c = c ^ 3; the 2-bit groups are reversed).
__device__ __forceinline__ uint64_t revcomp64(uint64_t x, int p) {
  uint64_t y = __brevll(~x);
  y = ((y >> 1) & 0x5555555555555555ull) | ((y & 0x5555555555555555ull) << 1);
  return y >> (64 - 2 * p);
}

// 64 bases starting at base position pos of the packed stream (MSB-first),
// i.e. the bits that follow; positions past the end read as A.
__device__ __forceinline__ uint64_t window64(const uint64_t* __restrict__ words, uint64_t n_words,
                                             uint64_t pos) {
  uint64_t wi = pos >> 5;
  uint32_t sh = (uint32_t)(pos & 31) * 2;
  uint64_t hi = wi < n_words ? __ldg(words + wi) : 0;
  if (sh == 0) return hi;
  uint64_t lo = wi + 1 < n_words ? __ldg(words + wi + 1) : 0;
  return (hi << sh) | (lo >> (64 - sh));
}

// ---- shared memory, mbarriers and 1-D TMA (cp.async.bulk) on sm_100a
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* m, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(m)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* m, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(m)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* m) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(m)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* m, uint32_t parity) {
  uint32_t done;
  do {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}"
        : "=r"(done) : "r"(smem_u32(m)), "r"(parity) : "memory");
  } while (!done);
}
// 1-D TMA: bytes (multiple of 16) from global src (16-byte aligned) into shared dst.
__device__ __forceinline__ void tma_bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* m) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(m)) : "memory");
}

}  // namespace dbg
