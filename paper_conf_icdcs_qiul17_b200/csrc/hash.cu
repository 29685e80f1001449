// hash.cu -- Step 2 of ParaHash on sm_100a: per-partition subgraph construction
// (Sec. III-C; Sec. III-D), kernel (b) of the north
// star, plus extraction of the vertex records (Def. 3).
//
// Table: open addressing, linear probing, 64-B slots (two 32-B sectors):
//   K <= 31: u64 key | u32 out[4] | u32 in[4] | u32 t_out | pad
//   K <= 63: u64 key_hi | u64 key_lo | u32 out[4] | u32 in[4] | u32 t_out | pad
// Key words carry bit 63 = occupied, so a zero-filled table is EMPTY and one
// memset initialises keys and counters together.  For two-word keys the
// 2K-bit code is split 63/63 bits, so each word of a claimed key is non-zero
// and a torn 16-B read (one word still zero) is recognisable.
//
// One insertion, multiple updates: the first
// occurrence of a vertex claims an EMPTY slot with a single 64-bit (K <= 31)
// or 128-bit (K <= 63) atomicCAS -- the whole key is published atomically, so
// the paper's {empty, locked, occupied} state word and its "locked" spin
// are unnecessary; every later occurrence finds the key with a
// plain load and only issues red.global.add on its counters.
//
// Counter economy: each occurrence increments exactly one "out-side" counter
// (out[c] if it has a successor in the vertex orientation, else t_out) and at
// most one in-side counter, so count = sum(out) + t_out is derived at
// extraction and the per-occurrence count atomic of the paper's entry
// disappears: two reds per K-mer instead of three.
#include <cub/device/device_radix_sort.cuh>

#include "dbg_device.cuh"

namespace dbg {

typedef unsigned __int128 u128;

constexpr int kHashThreads = 256;
constexpr uint64_t kSlotSeed = 0x9e3779b97f4a7c15ull;

template <int KW>
struct SlotLayout;
template <>
struct SlotLayout<1> {
  typedef uint64_t Code;
  static constexpr int kOut = 2, kIn = 6, kTerm = 10;  // u32 indices within the slot
};
template <>
struct SlotLayout<2> {
  typedef u128 Code;
  static constexpr int kOut = 4, kIn = 8, kTerm = 12;
};

struct HashArgs {
  const uint32_t* records;
  const uint64_t* rec_off;
  const uint64_t* tab_off;
  uint64_t slot_base;
  char* slots;
  uint32_t* status;
  int pid_begin, pid_end;
  int k;
};

template <int R>
__device__ __forceinline__ uint32_t base_at(const uint32_t (&w)[R], int i) {
  const int q = i >> 4;
  uint32_t v = w[1];
#pragma unroll
  for (int t = 1; t < R - 1; ++t) v = (q == t) ? w[1 + t] : v;
  return (v >> (30 - 2 * (i & 15))) & 3u;
}

__device__ __forceinline__ uint64_t slot_hash(uint64_t code) { return fmix64(code ^ kSlotSeed); }
__device__ __forceinline__ uint64_t slot_hash(u128 code) {
  return fmix64((uint64_t)code ^ fmix64((uint64_t)(code >> 64) ^ kSlotSeed));
}

// Finds the slot of `code` in the table [tbase, cap), inserting it if absent.
// Returns nullptr if the probe sequence wrapped (table full, reading O).
__device__ __forceinline__ uint32_t* find_or_insert(char* tbase, uint64_t cap, uint64_t code) {
  const unsigned long long key = code | kOccupied;
  uint64_t idx = __umul64hi(slot_hash(code), cap);
  for (uint64_t pr = 0; pr < cap; ++pr) {
    unsigned long long* kp = reinterpret_cast<unsigned long long*>(tbase + idx * kSlotBytes);
    unsigned long long cur = __ldcg(kp);
    if (cur == key) return reinterpret_cast<uint32_t*>(kp);
    if (cur == 0) {
      cur = atomicCAS(kp, 0ull, key);  // one insertion per distinct vertex
      if (cur == 0 || cur == key) return reinterpret_cast<uint32_t*>(kp);
    }
    idx = idx + 1 == cap ? 0 : idx + 1;
  }
  return nullptr;
}

__device__ __forceinline__ uint32_t* find_or_insert(char* tbase, uint64_t cap, u128 code) {
  const unsigned long long khi = (unsigned long long)(code >> 63) | kOccupied;
  const unsigned long long klo = ((unsigned long long)code & ~kOccupied) | kOccupied;
  uint64_t idx = __umul64hi(slot_hash(code), cap);
  for (uint64_t pr = 0; pr < cap; ++pr) {
    ulonglong2* kp = reinterpret_cast<ulonglong2*>(tbase + idx * kSlotBytes);
    ulonglong2 cur = __ldcg(kp);
    if (cur.x == khi && cur.y == klo) return reinterpret_cast<uint32_t*>(kp);
    if (cur.x == 0 || cur.y == 0) {  // empty, or a torn read of a key being published
      ulonglong2 want;
      want.x = khi;
      want.y = klo;
      cur = atomicCAS(kp, make_ulonglong2(0ull, 0ull), want);
      if ((cur.x == 0 && cur.y == 0) || (cur.x == khi && cur.y == klo))
        return reinterpret_cast<uint32_t*>(kp);
    }
    idx = idx + 1 == cap ? 0 : idx + 1;
  }
  return nullptr;
}

__device__ __forceinline__ void red_add(uint32_t* p) {
  asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" ::"l"(p) : "memory");
}

// Binary search: the partition i in [lo, hi) with off[i] <= x < off[i+1].
__device__ __forceinline__ int find_part(const uint64_t* __restrict__ off, int lo, int hi, uint64_t x) {
  while (hi - lo > 1) {
    int mid = (lo + hi) >> 1;
    if (__ldg(off + mid) <= x) lo = mid;
    else hi = mid;
  }
  return lo;
}

// One thread per record (a superkmer piece): roll the forward and reverse
// codes over its K-mers (<kmer, edge> pair generation), then
// insert/update each canonical K-mer.
template <int KW, int R>
__global__ void __launch_bounds__(kHashThreads) hash_build_kernel(HashArgs a) {
  typedef typename SlotLayout<KW>::Code Code;
  const uint64_t r_begin = a.rec_off[a.pid_begin], r_end = a.rec_off[a.pid_end];
  const int K = a.k;
  const Code mask = (K == 32 * KW) ? ~(Code)0 : (((Code)1 << (2 * K)) - 1);
  const int top = 2 * K - 2;
  for (uint64_t rec = r_begin + (uint64_t)blockIdx.x * kHashThreads + threadIdx.x; rec < r_end;
       rec += (uint64_t)gridDim.x * kHashThreads) {
    uint32_t w[R];
    const uint4* src = reinterpret_cast<const uint4*>(a.records + rec * R);
#pragma unroll
    for (int v = 0; v < R / 4; ++v) {
      uint4 x = __ldcs(src + v);  // streamed once
      w[4 * v] = x.x;
      w[4 * v + 1] = x.y;
      w[4 * v + 2] = x.z;
      w[4 * v + 3] = x.w;
    }
    const uint32_t hdr = w[0];
    const int n = hdr & 255u;
    const int hl = (hdr >> 8) & 1u, hr = (hdr >> 9) & 1u;
    const uint32_t pid = hdr >> 10;
    const uint64_t t0 = __ldg(a.tab_off + pid);
    const uint64_t cap = __ldg(a.tab_off + pid + 1) - t0;
    char* tbase = a.slots + (t0 - a.slot_base) * kSlotBytes;
    Code fwd = 0, rc = 0;
    for (int j = 0; j < K; ++j) {
      const uint32_t b = base_at<R>(w, hl + j);
      fwd = (fwd << 2) | (Code)b;
      rc |= (Code)(3u - b) << (2 * j);
    }
    int pred = hl ? (int)base_at<R>(w, 0) : -1;
    for (int t = 0; t < n; ++t) {
      const bool has_succ = t < n - 1 || hr;
      const int succ = has_succ ? (int)base_at<R>(w, hl + t + K) : -1;
      const bool is_fwd = fwd < rc;  // odd K: never equal (reading C)
      int o_idx, i_idx;
      if (is_fwd) {  // reading J
        o_idx = succ >= 0 ? SlotLayout<KW>::kOut + succ : SlotLayout<KW>::kTerm;
        i_idx = pred >= 0 ? SlotLayout<KW>::kIn + pred : -1;
      } else {
        o_idx = pred >= 0 ? SlotLayout<KW>::kOut + 3 - pred : SlotLayout<KW>::kTerm;
        i_idx = succ >= 0 ? SlotLayout<KW>::kIn + 3 - succ : -1;
      }
      uint32_t* slot = find_or_insert(tbase, cap, is_fwd ? fwd : rc);
      if (slot) {
        red_add(slot + o_idx);
        if (i_idx >= 0) red_add(slot + i_idx);
      } else {
        atomicOr(a.status, kStatusTableFull);
      }
      if (t + 1 < n) {
        pred = (int)(uint32_t)(fwd >> top) & 3;
        fwd = ((fwd << 2) | (Code)succ) & mask;
        rc = (rc >> 2) | ((Code)(3 - succ) << top);
      }
    }
  }
}

struct ExtractArgs {
  const char* slots;
  const uint64_t* tab_off;
  uint64_t slot_base;
  int pid_begin, pid_end;
  dbg_vertex* out;
  uint64_t out_cap;
  unsigned long long* n_out;
  unsigned long long* stats;  // distinct, sum_count, sum_edges, checksum
  uint32_t* status;
};

__device__ __forceinline__ unsigned long long warp_sum(unsigned long long v) {
#pragma unroll
  for (int d = 16; d; d >>= 1) v += __shfl_xor_sync(kFull, v, d);
  return v;
}

// Compaction of occupied slots into dbg_vertex records + totals + checksum.
template <int KW>
__global__ void __launch_bounds__(256) extract_kernel(ExtractArgs a) {
  const uint64_t s_begin = a.tab_off[a.pid_begin], s_end = a.tab_off[a.pid_end];
  const int lane = threadIdx.x & 31;
  const uint64_t n_iter = (s_end - s_begin + 31) / 32 * 32;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_iter;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t s = s_begin + i;
    bool occ = false;
    dbg_vertex v;
    if (s < s_end) {
      const char* sp = a.slots + (s - a.slot_base) * kSlotBytes;
      const uint4* q = reinterpret_cast<const uint4*>(sp);
      uint4 x0 = __ldcs(q), x1 = __ldcs(q + 1), x2 = __ldcs(q + 2), x3 = __ldcs(q + 3);
      uint32_t u[16] = {x0.x, x0.y, x0.z, x0.w, x1.x, x1.y, x1.z, x1.w,
                        x2.x, x2.y, x2.z, x2.w, x3.x, x3.y, x3.z, x3.w};
      const uint64_t k0 = ((uint64_t)u[1] << 32) | u[0];
      if (k0 & kOccupied) {
        occ = true;
        int c0;
        if (KW == 1) {
          v.kmer_hi = 0;
          v.kmer_lo = k0 & ~kOccupied;
          c0 = 2;
        } else {
          const uint64_t k1 = ((uint64_t)u[3] << 32) | u[2];
          const u128 code = ((u128)(k0 & ~kOccupied) << 63) | (u128)(k1 & ~kOccupied);
          v.kmer_hi = (uint64_t)(code >> 64);
          v.kmer_lo = (uint64_t)code;
          c0 = 4;
        }
        uint32_t cnt = u[c0 + 8];  // t_out
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          v.out[c] = u[c0 + c];
          v.in[c] = u[c0 + 4 + c];
          cnt += v.out[c];
        }
        v.count = cnt;  // count = sum(out) + t_out
        v.pid = (uint32_t)find_part(a.tab_off, a.pid_begin, a.pid_end, s);
      }
    }
    const uint32_t ballot = __ballot_sync(kFull, occ);
    unsigned long long base = 0;
    if (ballot) {
      if (lane == 0) base = atomicAdd(a.n_out, (unsigned long long)__popc(ballot));
      base = __shfl_sync(kFull, base, 0);
    }
    unsigned long long st_count = 0, st_edges = 0, st_sum = 0;
    if (occ) {
      const uint64_t pos = base + __popc(ballot & ((1u << lane) - 1u));
      if (pos < a.out_cap) a.out[pos] = v;
      else atomicOr(a.status, kStatusNoSpace);
      st_count = v.count;
      uint64_t f[11] = {v.kmer_hi, v.kmer_lo, v.count, v.out[0], v.out[1], v.out[2], v.out[3],
                        v.in[0], v.in[1], v.in[2], v.in[3]};
      uint64_t h = 0;
#pragma unroll
      for (int t = 0; t < 11; ++t) {
        h = fmix64(h ^ f[t]);
        if (t >= 3) st_edges += f[t];
      }
      st_sum = h;
    }
    if (ballot) {
      st_count = warp_sum(st_count);
      st_edges = warp_sum(st_edges);
      st_sum = warp_sum(st_sum);
      if (lane == 0) {
        atomicAdd(a.stats + 0, (unsigned long long)__popc(ballot));
        atomicAdd(a.stats + 1, st_count);
        atomicAdd(a.stats + 2, st_edges);
        atomicAdd(a.stats + 3, st_sum);
      }
    }
  }
}

__global__ void sort_prepare_kernel(const dbg_vertex* __restrict__ in, uint64_t n,
                                    unsigned long long* __restrict__ key,
                                    unsigned long long* __restrict__ idx) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    key[i] = in[i].kmer_lo;
    idx[i] = i;
  }
}

__global__ void sort_gather_hi_kernel(const dbg_vertex* __restrict__ in, uint64_t n,
                                      const unsigned long long* __restrict__ idx,
                                      unsigned long long* __restrict__ key) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x)
    key[i] = in[idx[i]].kmer_hi;
}

__global__ void sort_gather_kernel(const dbg_vertex* __restrict__ in, uint64_t n,
                                   const unsigned long long* __restrict__ idx,
                                   dbg_vertex* __restrict__ out) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x)
    out[i] = in[idx[i]];
}

}  // namespace dbg

using namespace dbg;

static int sm_count_h() {
  int dev = 0, n = 148;
  if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
  return n;
}

static bool hash_params_ok(const dbg_params* prm) {
  return prm && prm->k >= 1 && prm->k <= 63 && (prm->k & 1) && prm->p >= 1 && prm->p <= prm->k &&
         prm->p <= 31 && prm->num_partitions >= 1 && (uint32_t)prm->num_partitions <= kMaxPid;
}

extern "C" dbg_status dbg_hash_build(const dbg_params* prm, const dbg_partition_set* part,
                                     int32_t pid_begin, int32_t pid_end, void* d_slots,
                                     const uint64_t* d_table_offset, uint64_t slot_base,
                                     uint32_t* d_status, cudaStream_t stream) {
  if (!hash_params_ok(prm) || !part || !part->d_records || !part->d_record_offset || !d_slots ||
      !d_table_offset || !d_status)
    return DBG_EINVAL;
  if (pid_begin < 0 || pid_end > prm->num_partitions || pid_begin > pid_end) return DBG_EINVAL;
  if (pid_begin == pid_end) return DBG_OK;
  HashArgs a;
  a.records = part->d_records;
  a.rec_off = part->d_record_offset;
  a.tab_off = d_table_offset;
  a.slot_base = slot_base;
  a.slots = static_cast<char*>(d_slots);
  a.status = d_status;
  a.pid_begin = pid_begin;
  a.pid_end = pid_end;
  a.k = prm->k;
  const int grid = sm_count_h() * 8;  // 8 CTAs x 256 threads = 64 warps per SM
  if (prm->k <= 31) hash_build_kernel<1, 4><<<grid, kHashThreads, 0, stream>>>(a);
  else if (prm->k <= 39) hash_build_kernel<2, 4><<<grid, kHashThreads, 0, stream>>>(a);
  else hash_build_kernel<2, 8><<<grid, kHashThreads, 0, stream>>>(a);
  return cudaPeekAtLastError() == cudaSuccess ? DBG_OK : DBG_ECUDA;
}

extern "C" dbg_status dbg_extract_graph(const dbg_params* prm, const void* d_slots,
                                        const uint64_t* d_table_offset, uint64_t slot_base,
                                        int32_t pid_begin, int32_t pid_end, dbg_vertex* d_out,
                                        uint64_t out_cap, uint64_t* d_n_out, dbg_stats* d_stats,
                                        uint32_t* d_status, cudaStream_t stream) {
  if (!hash_params_ok(prm) || !d_slots || !d_table_offset || !d_n_out || !d_stats || !d_status ||
      (out_cap && !d_out))
    return DBG_EINVAL;
  if (pid_begin < 0 || pid_end > prm->num_partitions || pid_begin > pid_end) return DBG_EINVAL;
  if (pid_begin == pid_end) return DBG_OK;
  ExtractArgs a;
  a.slots = static_cast<const char*>(d_slots);
  a.tab_off = d_table_offset;
  a.slot_base = slot_base;
  a.pid_begin = pid_begin;
  a.pid_end = pid_end;
  a.out = d_out;
  a.out_cap = out_cap;
  a.n_out = reinterpret_cast<unsigned long long*>(d_n_out);
  a.stats = reinterpret_cast<unsigned long long*>(d_stats);
  a.status = d_status;
  const int grid = sm_count_h() * 8;
  if (prm->k <= 31) extract_kernel<1><<<grid, 256, 0, stream>>>(a);
  else extract_kernel<2><<<grid, 256, 0, stream>>>(a);
  return cudaPeekAtLastError() == cudaSuccess ? DBG_OK : DBG_ECUDA;
}

static size_t cub_sort_bytes(uint64_t n) {
  size_t bytes = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, bytes, (unsigned long long*)nullptr,
                                  (unsigned long long*)nullptr, (unsigned long long*)nullptr,
                                  (unsigned long long*)nullptr, (int64_t)n, 0, 64);
  return bytes;
}

static uint64_t align256(uint64_t x) { return (x + 255) & ~(uint64_t)255; }

extern "C" uint64_t dbg_sort_workspace_bytes(const dbg_params* prm, uint64_t n) {
  (void)prm;
  return 4 * align256(8 * (n ? n : 1)) + align256(cub_sort_bytes(n ? n : 1));
}

extern "C" dbg_status dbg_sort_vertices(const dbg_params* prm, const dbg_vertex* d_in,
                                        dbg_vertex* d_out, uint64_t n, void* d_workspace,
                                        uint64_t workspace_bytes, cudaStream_t stream) {
  if (!hash_params_ok(prm) || (n && (!d_in || !d_out || !d_workspace)) || d_in == d_out)
    return DBG_EINVAL;
  if (n == 0) return DBG_OK;
  if (workspace_bytes < dbg_sort_workspace_bytes(prm, n)) return DBG_EINVAL;
  char* ws = static_cast<char*>(d_workspace);
  const uint64_t arr = align256(8 * n);
  unsigned long long* k0 = reinterpret_cast<unsigned long long*>(ws);
  unsigned long long* k1 = reinterpret_cast<unsigned long long*>(ws + arr);
  unsigned long long* i0 = reinterpret_cast<unsigned long long*>(ws + 2 * arr);
  unsigned long long* i1 = reinterpret_cast<unsigned long long*>(ws + 3 * arr);
  void* tmp = ws + 4 * arr;
  size_t tmp_bytes = workspace_bytes - 4 * arr;
  const int grid = sm_count_h() * 4;
  sort_prepare_kernel<<<grid, 256, 0, stream>>>(d_in, n, k0, i0);
  const int k = prm->k;
  const int lo_bits = k <= 31 ? 2 * k : 64;
  if (cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, k0, k1, i0, i1, (int64_t)n, 0, lo_bits,
                                      stream) != cudaSuccess)
    return DBG_ECUDA;
  unsigned long long* idx = i1;
  if (k > 31) {  // LSD: then a stable sort by the high word
    sort_gather_hi_kernel<<<grid, 256, 0, stream>>>(d_in, n, i1, k0);
    if (cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, k0, k1, i1, i0, (int64_t)n, 0,
                                        2 * k - 64, stream) != cudaSuccess)
      return DBG_ECUDA;
    idx = i0;
  }
  sort_gather_kernel<<<grid, 256, 0, stream>>>(d_in, n, idx, d_out);
  return cudaPeekAtLastError() == cudaSuccess ? DBG_OK : DBG_ECUDA;
}
