// wide.cu -- row f3: K-mers longer than 63 bases (K <= 127, keys of four
// 64-bit words) in the resident global tables, with the paper's state-transfer
// protocol for multi-word keys (Sec. III-C3; Fig. 4).
//
// A key of up to 254 bits cannot be published by one CAS (the 64/128-bit CAS
// of the K <= 63 tables), so an entry carries the paper's occupancy state
// {empty, locked, occupied} in the two top bits of its first word:
//   empty    word 0 == 0
//   locked   word 0 == LOCK: a thread won the CAS empty -> locked and is
//            writing the key words ("other threads trying to access the kmer
//            are blocked")
//   occupied word 0 == OCC | top code bits: the key is complete and never
//            changes again; it is read concurrently by every later
//            occurrence, which then updates the edge counters with atomic
//            increments
// The inserting thread writes words 1..3 and then publishes word 0 with a
// release store; a reader that sees OCC through an acquire load reads a
// complete key.  A reader that sees LOCK waits (the "gray" entry of Fig. 4).
//
// Entry (48 B): u64 w0 (state | code bits 192..253), w1, w2, w3 (code bits
// 128..191, 64..127, 0..63), u32 t_out, 12 B pad; then the 32-B counter
// records out[4], in[4] (count = sum(out) + t_out, as for K <= 63).
//
// Records (dbg.h) are 16 words (240 bases) for K > 63; one thread walks one
// record, rolling the forward and reverse-complement codes base by base.
#include <cub/block/block_reduce.cuh>

#include "dbg_device.cuh"

int dbg_sm_count();

namespace dbg {

constexpr int kWideThreads = 256;
constexpr uint64_t kWideOcc = 1ull << 63, kWideLock = 1ull << 62;
constexpr uint32_t kWideEntry = 48;  // then a 32-B counter record per slot

// A code of up to 256 bits, w[0] most significant.
struct W4 {
  uint64_t w[4];
};

__device__ __forceinline__ bool w4_less(const W4& a, const W4& b) {
#pragma unroll
  for (int j = 0; j < 4; ++j)
    if (a.w[j] != b.w[j]) return a.w[j] < b.w[j];
  return false;
}

// mask of the low 2K bits, per word
__device__ __forceinline__ uint64_t w4_mask(int K, int j) {
  const int lo = 64 * (3 - j), bits = 2 * K - lo;  // bits of word j inside the code
  return bits >= 64 ? ~0ull : (bits <= 0 ? 0ull : ((1ull << bits) - 1));
}

// fwd = (fwd << 2 | b) mod 4^K
__device__ __forceinline__ void w4_push_back(W4& x, uint32_t b, int K) {
#pragma unroll
  for (int j = 0; j < 3; ++j) x.w[j] = (x.w[j] << 2) | (x.w[j + 1] >> 62);
  x.w[3] = (x.w[3] << 2) | b;
#pragma unroll
  for (int j = 0; j < 4; ++j) x.w[j] &= w4_mask(K, j);
}

// rc = rc >> 2 | (3 - b) << 2(K-1)
__device__ __forceinline__ void w4_push_front(W4& x, uint32_t b, int K) {
#pragma unroll
  for (int j = 3; j > 0; --j) x.w[j] = (x.w[j] >> 2) | (x.w[j - 1] << 62);
  x.w[0] >>= 2;
  const int bit = 2 * (K - 1);
  x.w[3 - bit / 64] |= (uint64_t)(3u - b) << (bit % 64);
}

__device__ __forceinline__ uint64_t w4_hash(const W4& x) {
  uint64_t h = 0x9e3779b97f4a7c15ull;
#pragma unroll
  for (int j = 0; j < 4; ++j) h = fmix64(h ^ x.w[j]);
  return h;
}

__device__ __forceinline__ uint64_t ld_acquire64(const unsigned long long* p) {
  uint64_t v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release64(unsigned long long* p, uint64_t v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

struct WideArgs {
  const uint32_t* records;
  const uint64_t* rec_off;
  const uint64_t* tab_off;
  char* table;  // n_slots entries of 48 B, then n_slots counter records of 32 B
  int pid_begin, pid_end, k;
  uint32_t* status;
};

// Lookup / insertion / update of one occurrence (Sec. III-C).
// Returns false when the probe sequence wraps (table full, reading O).
__device__ bool wide_upsert(char* entries, uint32_t* ctrs, uint64_t cap, const W4& code, int o, int i) {
  uint64_t idx = __umul64hi(w4_hash(code), cap);
  for (uint64_t pr = 0; pr < cap; ++pr, idx = idx + 1 == cap ? 0 : idx + 1) {
    unsigned long long* e = reinterpret_cast<unsigned long long*>(entries + idx * kWideEntry);
    uint64_t s = ld_acquire64(e);
    if (s == 0) {
      const uint64_t old = atomicCAS(e, 0ull, (unsigned long long)kWideLock);  // empty -> locked
      if (old == 0) {  // this thread inserts the vertex: write the key, then publish it
        e[1] = code.w[1];
        e[2] = code.w[2];
        e[3] = code.w[3];
        st_release64(e, kWideOcc | code.w[0]);  // locked -> occupied
        s = kWideOcc | code.w[0];
      } else {
        s = old;
      }
    }
    while (!(s & kWideOcc)) {  // locked: the key is being written -- wait for it (Fig. 4, gray)
      __nanosleep(64);
      s = ld_acquire64(e);
    }
    if ((s & ~kWideOcc) == code.w[0] && __ldcg(e + 1) == code.w[1] && __ldcg(e + 2) == code.w[2] &&
        __ldcg(e + 3) == code.w[3]) {
      uint32_t* c = ctrs + idx * 8;
      if (o < 4) atomicAdd(c + o, 1u);
      else atomicAdd(reinterpret_cast<uint32_t*>(e + 4), 1u);  // t_out
      if (i >= 0) atomicAdd(c + 4 + i, 1u);
      return true;
    }
  }
  return false;
}

__global__ void __launch_bounds__(kWideThreads) wide_hash_kernel(WideArgs a) {
  constexpr int R = 16;
  const uint64_t r_begin = a.rec_off[a.pid_begin], r_end = a.rec_off[a.pid_end];
  const uint64_t s0 = a.tab_off[a.pid_begin], n_slots = a.tab_off[a.pid_end] - s0;
  uint32_t* ctr_base = reinterpret_cast<uint32_t*>(a.table + n_slots * kWideEntry);
  const int K = a.k;
  bool ok = true;
  for (uint64_t r = r_begin + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; r < r_end;
       r += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t* w = a.records + r * R;
    const uint32_t w0 = w[0];
    const int n = hdr_n(w0), hl = hdr_hl(w0), hr = hdr_hr(w0);
    const uint32_t pid = hdr_pid(w0);
    const uint64_t t0 = __ldg(a.tab_off + pid) - s0, cap = __ldg(a.tab_off + pid + 1) - __ldg(a.tab_off + pid);
    auto base = [&](int q) { return (__ldg(w + 1 + (q >> 4)) >> (30 - 2 * (q & 15))) & 3u; };
    W4 fwd = {{0, 0, 0, 0}}, rc = {{0, 0, 0, 0}};
    for (int q = hl; q < hl + K - 1; ++q) {  // the first K-1 bases of the first K-mer
      const uint32_t b = base(q);
      w4_push_back(fwd, b, K);
      w4_push_front(rc, b, K);
    }
    for (int t = 0; t < n; ++t) {
      const int bq = hl + t;  // first base of K-mer t
      const uint32_t b = base(bq + K - 1);
      w4_push_back(fwd, b, K);
      w4_push_front(rc, b, K);
      const int pred = bq > 0 ? (int)base(bq - 1) : -1;
      const int succ = (t < n - 1 || hr) ? (int)base(bq + K) : -1;
      // canonical orientation and edge indices (readings C, J)
      const bool is_fwd = w4_less(fwd, rc);
      const W4& code = is_fwd ? fwd : rc;
      const int o = is_fwd ? (succ >= 0 ? succ : 4) : (pred >= 0 ? 3 - pred : 4);
      const int i = is_fwd ? pred : (succ >= 0 ? 3 - succ : -1);
      ok &= wide_upsert(a.table + t0 * kWideEntry, ctr_base + t0 * 8, cap, code, o, i);
    }
  }
  if (!ok) atomicOr(a.status, kStatusTableFull);
}

struct WideOut {
  dbg_vertex_wide* out;
  uint64_t out_cap;
  unsigned long long* n_out;
  unsigned long long* stats;
  uint32_t* status;
  uint32_t min_count;
  FastMod np_mod;
};

// Compaction + clean-on-extract of the occupied entries (one thread per slot).
__global__ void __launch_bounds__(kWideThreads) wide_extract_kernel(WideArgs a, WideOut oa) {
  typedef cub::BlockReduce<unsigned long long, kWideThreads> Red;
  __shared__ typename Red::TempStorage tmp;
  const uint64_t s0 = a.tab_off[a.pid_begin], n_slots = a.tab_off[a.pid_end] - s0;
  uint32_t* ctr_base = reinterpret_cast<uint32_t*>(a.table + n_slots * kWideEntry);
  unsigned long long st_n = 0, st_count = 0, st_edges = 0;
  for (uint64_t s = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; s < n_slots;
       s += (uint64_t)gridDim.x * blockDim.x) {
    unsigned long long* e = reinterpret_cast<unsigned long long*>(a.table + s * kWideEntry);
    const uint64_t e0 = __ldcg(e);
    if (!(e0 & kWideOcc)) continue;
    uint4* c4 = reinterpret_cast<uint4*>(ctr_base + s * 8);
    const uint4 co = __ldcg(c4), ci = __ldcg(c4 + 1);
    const uint32_t tout = __ldcg(reinterpret_cast<const uint32_t*>(e + 4));
    dbg_vertex_wide v;
    v.kmer[0] = e0 & ~kWideOcc;
    v.kmer[1] = __ldcg(e + 1);
    v.kmer[2] = __ldcg(e + 2);
    v.kmer[3] = __ldcg(e + 3);
    v.out[0] = co.x; v.out[1] = co.y; v.out[2] = co.z; v.out[3] = co.w;
    v.in[0] = ci.x; v.in[1] = ci.y; v.in[2] = ci.z; v.in[3] = ci.w;
    v.count = co.x + co.y + co.z + co.w + tout;  // count = sum(out) + t_out
    int lo = a.pid_begin, hi = a.pid_end;        // the slot's partition
    while (hi - lo > 1) {
      const int mid = (lo + hi) >> 1;
      if (__ldg(a.tab_off + mid) <= s0 + s) lo = mid;
      else hi = mid;
    }
    v.pid = fast_mod(oa.np_mod, (uint64_t)lo);
    for (int q = 0; q < 6; ++q) __stcg(e + q, 0ull);  // clean-on-extract
    __stcg(c4, make_uint4(0, 0, 0, 0));
    __stcg(c4 + 1, make_uint4(0, 0, 0, 0));
    if (oa.min_count > 1 && v.count < oa.min_count) continue;  // row f4
    const unsigned long long pos = atomicAdd(oa.n_out, 1ull);
    if (pos < oa.out_cap) oa.out[pos] = v;
    else atomicOr(oa.status, kStatusNoSpace);
    st_n += 1;
    st_count += v.count;
    st_edges += (uint64_t)co.x + co.y + co.z + co.w + ci.x + ci.y + ci.z + ci.w;
  }
  const unsigned long long n = Red(tmp).Sum(st_n);
  __syncthreads();
  const unsigned long long c = Red(tmp).Sum(st_count);
  __syncthreads();
  const unsigned long long ed = Red(tmp).Sum(st_edges);
  if (threadIdx.x == 0 && n) {
    atomicAdd(oa.stats + 0, n);
    atomicAdd(oa.stats + 1, c);
    atomicAdd(oa.stats + 2, ed);
  }
}

}  // namespace dbg

using namespace dbg;

// Called by dbg_hash_build / dbg_extract_graph (hash.cu) for K > 63.
dbg_status dbg_wide_hash_build(const dbg_params* prm, const dbg_partition_set* part, int32_t pid_begin,
                               int32_t pid_end, void* d_table, const uint64_t* d_table_offset, uint32_t* d_status,
                               cudaStream_t stream) {
  WideArgs a;
  a.records = part->d_records;
  a.rec_off = part->d_record_offset;
  a.tab_off = d_table_offset;
  a.table = static_cast<char*>(d_table);
  a.pid_begin = pid_begin;
  a.pid_end = pid_end;
  a.k = prm->k;
  a.status = d_status;
  wide_hash_kernel<<<dbg_sm_count() * 8, kWideThreads, 0, stream>>>(a);
  return cudaPeekAtLastError() == cudaSuccess ? DBG_OK : DBG_ECUDA;
}

dbg_status dbg_wide_extract(const dbg_params* prm, void* d_table, const uint64_t* d_table_offset, int32_t pid_begin,
                            int32_t pid_end, void* d_out, uint64_t out_cap, uint64_t* d_n_out, dbg_stats* d_stats,
                            uint32_t* d_status, cudaStream_t stream) {
  WideArgs a;
  a.records = nullptr;
  a.rec_off = nullptr;
  a.tab_off = d_table_offset;
  a.table = static_cast<char*>(d_table);
  a.pid_begin = pid_begin;
  a.pid_end = pid_end;
  a.k = prm->k;
  a.status = d_status;
  WideOut oa;
  oa.out = static_cast<dbg_vertex_wide*>(d_out);
  oa.out_cap = out_cap;
  oa.n_out = reinterpret_cast<unsigned long long*>(d_n_out);
  oa.stats = reinterpret_cast<unsigned long long*>(d_stats);
  oa.status = d_status;
  oa.min_count = prm->min_count;
  oa.np_mod = make_fastmod((uint64_t)prm->num_partitions);
  wide_extract_kernel<<<dbg_sm_count() * 8, kWideThreads, 0, stream>>>(a, oa);
  return cudaPeekAtLastError() == cudaSuccess ? DBG_OK : DBG_ECUDA;
}
