// hash.cu -- Step 2 of ParaHash on sm_100a: per-partition subgraph construction
// (Sec. III-C; Sec. III-D), kernel (b) of the north
// star, plus extraction of the vertex records (Def. 3).
//
// Table of one partition with capacity n (open addressing, linear probing):
//   key entries  n x KE bytes
//     K <= 31: KE = 16  { u64 key; u32 t_out; u32 pad }
//     K <= 63: KE = 32  { u64 key_hi; u64 key_lo; u32 t_out; u32 pad[3] }
//   counters     n x 32 bytes  { u32 out[4]; u32 in[4] }
// A key word is 0 (empty) or OCC | code (bit 63 of the hi word = occupied).
//
// One insertion, multiple updates: a probe loads the
// key entry; an EMPTY slot is claimed with atomicCAS(slot, EMPTY, key) --
// 64-bit for K <= 31, 128-bit for K <= 63 -- whose return value decides:
// EMPTY means this occurrence inserted the vertex (the single insertion), the
// own key means another thread just did, anything else means probe on.  The
// whole key is published by that one CAS, so the paper's {empty, locked,
// occupied} protocol for multi-word keys (Fig. 4) collapses to
// {empty, occupied}: there is no partially written key to wait for.  Then
// red.global.add on two counters (the multiple updates).  (Probing with the
// CAS itself was measured slower: every probe then costs an L2 atomic.)
//
// Clean-on-extract: tables are all-zero before hashing (one memset when the
// buffer is allocated), and extraction writes zeros back over every occupied
// slot it reads.  So no per-partition zero-fill is needed, counters never
// need initialising by the inserting thread, and no memory fence is needed
// between the key CAS and the counter updates.
//
// Counter economy: each occurrence increments exactly one "out-side" counter
// (out[c] if it has a successor in the vertex orientation, else t_out) and at
// most one in-side counter, so count = sum(out) + t_out is derived at
// extraction: two reds per K-mer instead of the paper's three.
//
// Kernels:
//  smem_subgraph_kernel the hot path: one persistent CTA per SM builds groups of fine partitions
//                       in shared-memory tables and extracts them (dbg_build_subgraphs_smem)
//  hash_build_kernel    resident tables of partitions [b, e) (dbg_hash_build): partitions too
//                       large for one SM, and K > 63 (wide.cu)
//  extract_kernel       compaction + clean of resident tables (dbg_extract_graph)
#include <cub/block/block_reduce.cuh>
#include <cub/block/block_scan.cuh>
#include <cub/device/device_radix_sort.cuh>

#include <cstdlib>

#include "dbg_device.cuh"
#include "scan.cuh"

// Kernel variants (A/B builds: tools/build_variants.py); the defaults are the measured winners.

int dbg_sm_count();
bool dbg_params_ok(const dbg_params* prm);
// row f3 (wide.cu): K > 63 in the resident tables, with the locked-state protocol
dbg_status dbg_wide_hash_build(const dbg_params* prm, const dbg_partition_set* part, int32_t pid_begin,
                               int32_t pid_end, void* d_table, const uint64_t* d_table_offset, uint32_t* d_status,
                               cudaStream_t stream);
dbg_status dbg_wide_extract(const dbg_params* prm, void* d_table, const uint64_t* d_table_offset, int32_t pid_begin,
                            int32_t pid_end, void* d_out, uint64_t out_cap, uint64_t* d_n_out, dbg_stats* d_stats,
                            uint32_t* d_status, cudaStream_t stream);

namespace dbg {

typedef unsigned __int128 u128;

constexpr int kThreads = 256;
constexpr uint64_t kCodeMask = (1ull << 62) - 1;
constexpr uint64_t kSlotSeed = 0x9e3779b97f4a7c15ull;
constexpr int kXPer = 8;
constexpr uint32_t kExtractSlots = kThreads * kXPer;
constexpr int kJobs = 4;  // occurrences in flight per lane

__host__ __device__ inline uint32_t key_bytes(int k) { return k <= 31 ? 16u : (k <= 63 ? 32u : 48u); }
constexpr uint32_t kCtrBytes = 32;

__device__ __forceinline__ uint64_t slot_hash(uint64_t code) { return fmix64(code ^ kSlotSeed); }
__device__ __forceinline__ uint64_t slot_hash(u128 code) {
  return fmix64((uint64_t)code ^ fmix64((uint64_t)(code >> 64) ^ kSlotSeed));
}

__device__ __forceinline__ void red_add(uint32_t* p) {
  asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" ::"l"(p) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// ----- key words and the probe CAS

template <typename Code>
struct KeyOf;
template <>
struct KeyOf<uint64_t> {
  typedef unsigned long long T;
  static __device__ __forceinline__ T make(uint64_t code) { return code | kOccupied; }
  static __device__ __forceinline__ bool empty(T v) { return v == 0; }
  static __device__ __forceinline__ bool same(T a, T b) { return a == b; }
  static __device__ __forceinline__ T cas(char* kp, T want) {
    return atomicCAS(reinterpret_cast<unsigned long long*>(kp), 0ull, want);
  }
  static __device__ __forceinline__ T load(const char* kp) {
    return __ldcg(reinterpret_cast<const unsigned long long*>(kp));
  }
};
template <>
struct KeyOf<u128> {
  typedef ulonglong2 T;
  static __device__ __forceinline__ T make(u128 code) {
    T t;
    t.x = (uint64_t)(code >> 64) | kOccupied;  // hi word: <= 62 code bits + OCC
    t.y = (uint64_t)code;
    return t;
  }
  static __device__ __forceinline__ bool empty(T v) { return v.x == 0 && v.y == 0; }
  static __device__ __forceinline__ bool same(T a, T b) { return a.x == b.x && a.y == b.y; }
  static __device__ __forceinline__ T cas(char* kp, T want) {
    return atomicCAS(reinterpret_cast<ulonglong2*>(kp), make_ulonglong2(0ull, 0ull), want);
  }
  // A 16-B load is not single-copy atomic: a torn read of a key being
  // published shows one word of it and one zero word.  Such a value is
  // neither EMPTY nor a key (every claimed hi word has OCC set and claimed
  // entries never change), except the ambiguous (hi, 0) pair, which is
  // treated as EMPTY so the CAS returns the entry atomically.
  static __device__ __forceinline__ T load(const char* kp) {
    T v = __ldcg(reinterpret_cast<const ulonglong2*>(kp));
    if (v.x == 0 || v.y == 0) v = make_ulonglong2(0ull, 0ull);
    return v;
  }
};

// ----- K-mer decoding from a record held in shared memory (dbg.h layout)

// Record words may be staged with a stride (word q at w[q * stride]).
__device__ __forceinline__ uint32_t rec_word(const uint32_t* w, int q, int R, int stride = 1) {
  return q < R ? w[q * stride] : 0u;
}

__device__ __forceinline__ uint32_t rec_base(const uint32_t* w, int i, int stride = 1) {
  return (w[(1 + (i >> 4)) * stride] >> (30 - 2 * (i & 15))) & 3u;
}

// The 64 bits of the record's base string that start at base b.
__device__ __forceinline__ uint64_t rec_bits64(const uint32_t* w, int b, int R, int stride = 1) {
  const int q = 1 + (b >> 4), off = 2 * (b & 15);
  const uint64_t hi = ((uint64_t)rec_word(w, q, R, stride) << 32) | rec_word(w, q + 1, R, stride);
  if (off == 0) return hi;
  return (hi << off) | (rec_word(w, q + 2, R, stride) >> (32 - off));
}

__device__ __forceinline__ void kmer_at(const uint32_t* w, int b, int K, int R, uint64_t& fwd, uint64_t& rc,
                                        int stride = 1) {
  fwd = rec_bits64(w, b, R, stride) >> (64 - 2 * K);
  rc = revcomp64(fwd, K);
}

__device__ __forceinline__ u128 revcomp128(u128 x, int k) {
  const uint64_t lo = (uint64_t)x, hi = (uint64_t)(x >> 64);
  uint64_t a = __brevll(~lo), b = __brevll(~hi);  // reversed: the old low half becomes the high half
  a = ((a >> 1) & 0x5555555555555555ull) | ((a & 0x5555555555555555ull) << 1);
  b = ((b >> 1) & 0x5555555555555555ull) | ((b & 0x5555555555555555ull) << 1);
  return (((u128)a << 64) | (u128)b) >> (128 - 2 * k);
}

__device__ __forceinline__ void kmer_at(const uint32_t* w, int b, int K, int R, u128& fwd, u128& rc,
                                        int stride = 1) {
  const uint64_t hi = rec_bits64(w, b, R, stride), lo = rec_bits64(w, b + 32, R, stride);
  fwd = (((u128)hi << 64) | (u128)lo) >> (128 - 2 * K);
  rc = revcomp128(fwd, K);
}

// Per-warp staging of up to 32 records: words, table placement, K-mer prefix.
template <int R>
struct WarpRecs {
  uint32_t w[32][R];
  unsigned long long t0[32];   // first slot of the record's table (table-block coordinates)
  unsigned long long cap[32];  // capacity of that table
  uint32_t pre[33];            // exclusive prefix of the records' K-mer counts
};

// One occurrence: canonical key, out-side counter o (0..3, 4 = t_out), in-side
// counter i (-1..3), its table and current probe slot.
template <typename Code>
struct Job {
  typename KeyOf<Code>::T want;
  uint64_t t0, cap, idx;
  int o, i;
};

// Decodes K-mer number kid of the warp's records (the cursor r only moves
// forward): <kmer, edge> pair generation, in the canonical
// orientation of reading J.
template <typename Code, int R>
__device__ __forceinline__ Job<Code> make_job(const WarpRecs<R>& sm, uint32_t kid, int& r, int K) {
  Job<Code> jb;
  while (sm.pre[r + 1] <= kid) ++r;
  const uint32_t* w = sm.w[r];
  const uint32_t hdr = w[0];
  const int n = hdr_n(hdr), hl = hdr_hl(hdr), hr = hdr_hr(hdr);
  const int t = (int)(kid - sm.pre[r]);
  const int b = hl + t;  // first base of the K-mer in the record
  Code fwd, rc;
  kmer_at(w, b, K, R, fwd, rc);
  const int pred = (t > 0 || hl) ? (int)rec_base(w, b - 1) : -1;
  const int succ = (t < n - 1 || hr) ? (int)rec_base(w, b + K) : -1;
  Code code;
  if (fwd < rc) {  // odd K: never equal (reading C)
    code = fwd;
    jb.o = succ >= 0 ? succ : 4;
    jb.i = pred;
  } else {
    code = rc;
    jb.o = pred >= 0 ? 3 - pred : 4;
    jb.i = succ >= 0 ? 3 - succ : -1;
  }
  jb.want = KeyOf<Code>::make(code);
  jb.t0 = sm.t0[r];
  jb.cap = sm.cap[r];
  jb.idx = __umul64hi(slot_hash(code), jb.cap);
  return jb;
}

// Insert/update of every K-mer of up to 32 records per warp.
// Lane l takes a contiguous share of the warp's K-mers (balanced whatever the
// record lengths) and keeps kJobs occurrences in flight: their probe CASes
// are issued together, collisions are resolved, then the counter reds.
// table_of(pid, t0, cap) places a partition's table in the block [keys, ctr).
// Returns false if a table overflowed.
template <typename Code, int R, typename TableOf>
__device__ __forceinline__ bool hash_warp(const uint32_t* recs, int64_t n_recs, int K, char* keys, uint32_t* ctr,
                                          TableOf table_of, WarpRecs<R>& sm) {
  typedef KeyOf<Code> KO;
  constexpr uint32_t KE = sizeof(Code) == 8 ? 16 : 32;
  const int lane = threadIdx.x & 31;
  uint32_t n = 0;
  if (lane < n_recs) {
    const uint4* src = reinterpret_cast<const uint4*>(recs + (uint64_t)lane * R);
#pragma unroll
    for (int v = 0; v < R / 4; ++v) {
      const uint4 x = __ldcs(src + v);  // streamed once
      sm.w[lane][4 * v] = x.x;
      sm.w[lane][4 * v + 1] = x.y;
      sm.w[lane][4 * v + 2] = x.z;
      sm.w[lane][4 * v + 3] = x.w;
    }
    const uint32_t hdr = sm.w[lane][0];
    uint64_t t0, cap;
    table_of(hdr_pid(hdr), t0, cap);
    n = cap ? hdr_n(hdr) : 0u;  // capacity 0: the partition is built elsewhere (on chip)
    sm.t0[lane] = t0;
    sm.cap[lane] = cap;
  }
  uint32_t incl = n;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t v = __shfl_up_sync(kFull, incl, d);
    if (lane >= d) incl += v;
  }
  sm.pre[lane + 1] = incl;
  if (lane == 0) sm.pre[0] = 0;
  const uint32_t total = __shfl_sync(kFull, incl, 31);
  __syncwarp();
  const uint32_t share = (total + 31) / 32;
  const uint32_t k0 = min(total, lane * share), k1 = min(total, k0 + share);
  bool ok = true;
  int r = 0;
  for (uint32_t kid = k0; kid < k1; kid += kJobs) {
    Job<Code> jb[kJobs];
    typename KO::T cur[kJobs];
    bool live[kJobs];
#pragma unroll
    for (int q = 0; q < kJobs; ++q) {
      live[q] = kid + q < k1;
      if (live[q]) {
        jb[q] = make_job<Code, R>(sm, kid + q, r, K);
        cur[q] = KO::load(keys + (jb[q].t0 + jb[q].idx) * KE);  // all first probes in flight
      }
    }
#pragma unroll
    for (int q = 0; q < kJobs; ++q) {
      if (!live[q]) continue;
      uint64_t probes = 1;
      for (;;) {
        // a plain load finds the vertex (the common case: duplicates outnumber
        // distinct vertices ~4:1); only an EMPTY slot costs a CAS
        if (KO::empty(cur[q])) cur[q] = KO::cas(keys + (jb[q].t0 + jb[q].idx) * KE, jb[q].want);
        if (KO::empty(cur[q]) || KO::same(cur[q], jb[q].want)) break;
        if (probes++ == jb[q].cap) break;
        jb[q].idx = jb[q].idx + 1 == jb[q].cap ? 0 : jb[q].idx + 1;
        cur[q] = KO::load(keys + (jb[q].t0 + jb[q].idx) * KE);
      }
      if (!KO::empty(cur[q]) && !KO::same(cur[q], jb[q].want)) {
        ok = false;  // wrapped: table full (reading O)
        continue;
      }
      const uint64_t s = jb[q].t0 + jb[q].idx;
      uint32_t* c = ctr + s * 8;
      red_add(jb[q].o < 4 ? c + jb[q].o : reinterpret_cast<uint32_t*>(keys + s * KE + KE / 2));
      if (jb[q].i >= 0) red_add(c + 4 + jb[q].i);
    }
  }
  __syncwarp();
  return ok;
}

// --------------------------------------------------------------- extraction

struct OutArgs {
  uint32_t np_out;  // the paper's NP: dbg_vertex.pid = fine pid mod NP ...
  bool kmer_pid;    // ... or, when fine_p != P, the partition of the vertex's P-minimizer
  int k, p;
  FastMod np_mod;
  dbg_vertex* out;
  uint64_t out_cap;
  unsigned long long* n_out;
  unsigned long long* stats;  // distinct, sum_count, sum_edges, checksum
  uint32_t* status;
  uint32_t min_count;  // row f4: vertices with count < min_count are dropped (0, 1: keep all)
};

static OutArgs make_out_args(const dbg_params* prm, dbg_vertex* d_out, uint64_t out_cap, uint64_t* d_n_out,
                             dbg_stats* d_stats, uint32_t* d_status) {
  OutArgs oa;
  oa.np_out = (uint32_t)prm->num_partitions;
  oa.kmer_pid = partition_p(prm) != prm->p;
  oa.k = prm->k;
  oa.p = prm->p;
  oa.np_mod = make_fastmod((uint64_t)prm->num_partitions);
  oa.out = d_out;
  oa.out_cap = out_cap;
  oa.n_out = reinterpret_cast<unsigned long long*>(d_n_out);
  oa.stats = reinterpret_cast<unsigned long long*>(d_stats);
  oa.status = d_status;
  oa.min_count = prm->min_count;
  return oa;
}

// The paper's partition of a vertex (readings D, E, I, V): fmix64 of the
// canonical P-minimizer of its canonical K-mer (code = hi:lo, 2K bits, first
// base most significant) mod NP -- the minimizer of every superkmer that holds
// the K-mer, on either strand.  With rc the K-mer's reverse complement, the
// canonical P-mer at offset q is min(code >> 2(K-P-q), rc >> 2q) & mask: two
// funnel shifts per window, no dependence chain across windows.
template <typename PT>
__device__ __forceinline__ uint64_t kmer_minimizer64(uint64_t code, int K, int P) {
  const uint64_t rc = revcomp64(code, K);
  const PT mask = (PT)((2ull << (2 * P - 1)) - 1);
  PT m = (PT)~(PT)0;
  for (int q = 0, s = 2 * (K - P); q <= K - P; ++q, s -= 2) {
    const PT f = (PT)(code >> s) & mask, r = (PT)(rc >> (2 * q)) & mask;
    const PT c = f < r ? f : r;
    m = c < m ? c : m;
  }
  return (uint64_t)m;
}

template <typename PT>
__device__ __forceinline__ uint64_t kmer_minimizer128(u128 code, int K, int P) {
  const u128 rc = revcomp128(code, K);
  const PT mask = (PT)((2ull << (2 * P - 1)) - 1);
  PT m = (PT)~(PT)0;
  for (int q = 0, s = 2 * (K - P); q <= K - P; ++q, s -= 2) {
    const PT f = (PT)(uint64_t)(code >> s) & mask, r = (PT)(uint64_t)(rc >> (2 * q)) & mask;
    const PT c = f < r ? f : r;
    m = c < m ? c : m;
  }
  return (uint64_t)m;
}

__device__ __forceinline__ uint32_t kmer_partition(uint64_t hi, uint64_t lo, const OutArgs& oa) {
  uint64_t m;
  if (oa.k <= 31) m = oa.p <= 16 ? kmer_minimizer64<uint32_t>(lo, oa.k, oa.p) : kmer_minimizer64<uint64_t>(lo, oa.k, oa.p);
  else {
    const u128 code = ((u128)hi << 64) | lo;
    m = oa.p <= 16 ? kmer_minimizer128<uint32_t>(code, oa.k, oa.p) : kmer_minimizer128<uint64_t>(code, oa.k, oa.p);
  }
  return fast_mod(oa.np_mod, fmix64(m));
}

// kmer_partition with compile-time K <= 31 and P <= 16 (the chr14 launch: K = 31, P = 11 under a
// longer device minimizer).  Each P-mer is taken TOP-aligned in a 32-bit word -- its 2P bits
// followed by the next bases of the K-mer (or zeros) -- with one funnel shift, and the words are
// min-reduced three at a time: the top 2P bits of the minimum word are the minimum P-mer (a
// numeric minimum is decided by the leading bits first), on either strand, so no masks are needed.
// The same minimizer as kmer_minimizer64 (the vertex's P-minimizer, reading V).
template <int KC, int PC>
__device__ __forceinline__ uint32_t kmer_partition_c(uint64_t lo, const OutArgs& oa) {
  static_assert(KC <= 31 && PC >= 1 && PC <= 16, "one-word K-mer, 32-bit P-mer");
  const uint64_t rc = revcomp64(lo, KC);
  // forward P-mer q = bits [2(K-P-q), 2(K-q)) of lo; reverse one = bits [2q, 2q+2P) of rc
  const uint64_t fa = lo << (64 - 2 * KC);  // the K-mer's first base at bit 63
  uint32_t m = ~0u;
#pragma unroll
  for (int q = 0; q <= KC - PC; ++q) {
    const uint32_t f = (uint32_t)((fa << (2 * q)) >> 32);
    const uint32_t r = (uint32_t)((rc << (64 - 2 * q - 2 * PC)) >> 32);
    m = min(m, min(f, r));
  }
  return fast_mod(oa.np_mod, fmix64((uint64_t)(m >> (32 - 2 * PC))));
}

struct XShared {
  typename cub::BlockScan<uint32_t, kThreads>::TempStorage scan;
  typename cub::BlockReduce<unsigned long long, kThreads>::TempStorage red;
  unsigned long long base;
};

// Block-wide: compact the occupied entries among slots [0, n) of a contiguous
// key/counter range into records and zero them again (clean-on-extract);
// pid_of(local slot) gives the partition.  Two passes keep registers low:
// occupancy bits + block scan, then re-read (L1/L2 hits), write, clean.
template <int KW, typename PidFn>
__device__ __forceinline__ void extract_tile(char* keys, uint32_t* ctr, uint64_t n, PidFn pid_of,
                                             const OutArgs& oa, XShared& sh) {
  constexpr uint32_t KE = KW == 1 ? 16 : 32;
  uint32_t bits = 0;
#pragma unroll
  for (int q = 0; q < kXPer; ++q) {
    const uint64_t s = (uint64_t)q * kThreads + threadIdx.x;
    if (s < n && (__ldcg(reinterpret_cast<const uint64_t*>(keys + s * KE)) & kOccupied)) bits |= 1u << q;
  }
  if (oa.min_count > 1) {  // row f4: drop (and clean) the vertices with count < min_count
    uint32_t b = bits;
    while (b) {
      const int q = __ffs(b) - 1;
      b &= b - 1;
      const uint64_t s = (uint64_t)q * kThreads + threadIdx.x;
      uint4* kp4 = reinterpret_cast<uint4*>(keys + s * KE);
      uint4* cp = reinterpret_cast<uint4*>(ctr + s * 8);
      const uint32_t tout = __ldcg(reinterpret_cast<const uint32_t*>(keys + s * KE + (KW == 1 ? 8 : 16)));
      const uint4 a = __ldcg(cp);
      if (a.x + a.y + a.z + a.w + tout < oa.min_count) {
        const uint4 z = make_uint4(0, 0, 0, 0);
        __stcg(kp4, z);
        if (KW == 2) __stcg(kp4 + 1, z);
        __stcg(cp, z);
        __stcg(cp + 1, z);
        bits &= ~(1u << q);
      }
    }
  }
  const uint32_t cnt = __popc(bits);
  uint32_t excl, total;
  cub::BlockScan<uint32_t, kThreads>(sh.scan).ExclusiveSum(cnt, excl, total);
  if (threadIdx.x == 0) sh.base = total ? atomicAdd(oa.n_out, (unsigned long long)total) : 0ull;
  __syncthreads();
  uint64_t pos = sh.base + excl;
  unsigned long long st_count = 0, st_edges = 0;
  while (bits) {
    const int q = __ffs(bits) - 1;
    bits &= bits - 1;
    const uint64_t s = (uint64_t)q * kThreads + threadIdx.x;
    uint4* kp4 = reinterpret_cast<uint4*>(keys + s * KE);
    const uint4 e0 = __ldcg(kp4);
    dbg_vertex v;
    uint32_t tout;
    if (KW == 1) {
      v.kmer_hi = 0;
      v.kmer_lo = (((uint64_t)e0.y << 32) | e0.x) & kCodeMask;
      tout = e0.z;
    } else {
      v.kmer_hi = (((uint64_t)e0.y << 32) | e0.x) & kCodeMask;
      v.kmer_lo = ((uint64_t)e0.w << 32) | e0.z;
      tout = __ldcg(reinterpret_cast<const uint32_t*>(kp4 + 1));
    }
    uint4* cp = reinterpret_cast<uint4*>(ctr + s * 8);
    const uint4 a = __ldcg(cp), b = __ldcg(cp + 1);
    const uint4 z = make_uint4(0, 0, 0, 0);
    __stcg(kp4, z);  // clean-on-extract
    if (KW == 2) __stcg(kp4 + 1, z);
    __stcg(cp, z);
    __stcg(cp + 1, z);
    v.out[0] = a.x; v.out[1] = a.y; v.out[2] = a.z; v.out[3] = a.w;
    v.in[0] = b.x; v.in[1] = b.y; v.in[2] = b.z; v.in[3] = b.w;
    v.count = a.x + a.y + a.z + a.w + tout;  // count = sum(out) + t_out
    v.pid = oa.kmer_pid ? kmer_partition(v.kmer_hi, v.kmer_lo, oa) : pid_of(s) % oa.np_out;
    if (pos < oa.out_cap) oa.out[pos] = v;
    else atomicOr(oa.status, kStatusNoSpace);
    ++pos;
    st_count += v.count;
    st_edges += (uint64_t)a.x + a.y + a.z + a.w + b.x + b.y + b.z + b.w;
  }
  if (total) {  // block-uniform
    typedef cub::BlockReduce<unsigned long long, kThreads> Red;
    const unsigned long long c = Red(sh.red).Sum(st_count);
    __syncthreads();
    const unsigned long long e = Red(sh.red).Sum(st_edges);
    if (threadIdx.x == 0) {
      atomicAdd(oa.stats + 0, (unsigned long long)total);
      atomicAdd(oa.stats + 1, c);
      atomicAdd(oa.stats + 2, e);
    }
  }
  __syncthreads();
}

// Binary search: the partition i in [lo, hi) with off[i] <= x < off[i+1].
__device__ __forceinline__ int find_part(const uint64_t* __restrict__ off, int lo, int hi, uint64_t x) {
  while (hi - lo > 1) {
    const int mid = (lo + hi) >> 1;
    if (__ldg(off + mid) <= x) lo = mid;
    else hi = mid;
  }
  return lo;
}

// --------------------------------------------------------------- resident tables

struct ResidentArgs {
  const uint32_t* records;
  const uint64_t* rec_off;
  const uint64_t* tab_off;
  char* table;  // [keys of all slots of [b,e)] [counters of all slots]
  int pid_begin, pid_end, k;
  uint32_t* status;
};

template <typename Code, int R>
__global__ void __launch_bounds__(kThreads) hash_build_kernel(ResidentArgs a) {
  constexpr uint32_t KE = sizeof(Code) == 8 ? 16 : 32;
  __shared__ WarpRecs<R> sh[kThreads / 32];
  const uint64_t r_begin = a.rec_off[a.pid_begin], r_end = a.rec_off[a.pid_end];
  const uint64_t s0 = a.tab_off[a.pid_begin], n_slots = a.tab_off[a.pid_end] - s0;
  uint32_t* ctr_base = reinterpret_cast<uint32_t*>(a.table + n_slots * KE);
  const uint64_t* off = a.tab_off;
  auto table_of = [=](uint32_t pid, uint64_t& t0, uint64_t& cap) {
    t0 = __ldg(off + pid) - s0;
    cap = __ldg(off + pid + 1) - __ldg(off + pid);
  };
  const int warp = threadIdx.x >> 5;
  const uint64_t n_chunks = (r_end - r_begin + 31) / 32;
  for (uint64_t c = (uint64_t)blockIdx.x * (kThreads / 32) + warp; c < n_chunks;
       c += (uint64_t)gridDim.x * (kThreads / 32)) {
    const uint64_t r0 = r_begin + 32 * c;
    const int64_t n = (int64_t)min((uint64_t)32, r_end - r0);
    if (!hash_warp<Code, R>(a.records + r0 * R, n, a.k, a.table, ctr_base, table_of, sh[warp]))
      atomicOr(a.status, kStatusTableFull);
  }
}

// Same as hash_build_kernel for an explicit list of partitions (the oversize
// ones of the on-chip path): warp-chunks of 32 records are numbered across the
// listed partitions by chunk_prefix (exclusive prefix of ceil(records/32)).
template <typename Code, int R>
__global__ void __launch_bounds__(kThreads) hash_build_list_kernel(ResidentArgs a, const uint32_t* pids,
                                                                  const uint64_t* chunk_prefix, int n_pids) {
  constexpr uint32_t KE = sizeof(Code) == 8 ? 16 : 32;
  __shared__ WarpRecs<R> sh[kThreads / 32];
  const uint64_t s0 = a.tab_off[a.pid_begin], n_slots = a.tab_off[a.pid_end] - s0;
  uint32_t* ctr_base = reinterpret_cast<uint32_t*>(a.table + n_slots * KE);
  const uint64_t* off = a.tab_off;
  auto table_of = [=](uint32_t pid, uint64_t& t0, uint64_t& cap) {
    t0 = __ldg(off + pid) - s0;
    cap = __ldg(off + pid + 1) - __ldg(off + pid);
  };
  const int warp = threadIdx.x >> 5;
  const uint64_t n_chunks = chunk_prefix[n_pids];
  for (uint64_t c = (uint64_t)blockIdx.x * (kThreads / 32) + warp; c < n_chunks;
       c += (uint64_t)gridDim.x * (kThreads / 32)) {
    int lo = 0, hi = n_pids;  // listed partition holding chunk c
    while (hi - lo > 1) {
      const int mid = (lo + hi) >> 1;
      if (chunk_prefix[mid] <= c) lo = mid;
      else hi = mid;
    }
    const uint32_t pid = pids[lo];
    const uint64_t r0 = a.rec_off[pid] + 32 * (c - chunk_prefix[lo]);
    const int64_t n = (int64_t)min((uint64_t)32, a.rec_off[pid + 1] - r0);
    if (!hash_warp<Code, R>(a.records + r0 * R, n, a.k, a.table, ctr_base, table_of, sh[warp]))
      atomicOr(a.status, kStatusTableFull);
  }
}

template <int KW>
__global__ void __launch_bounds__(kThreads, 4) extract_kernel(ResidentArgs a, OutArgs oa) {
  constexpr uint32_t KE = KW == 1 ? 16 : 32;
  __shared__ XShared sh;
  const uint64_t s0 = a.tab_off[a.pid_begin], n_slots = a.tab_off[a.pid_end] - s0;
  uint32_t* ctr_base = reinterpret_cast<uint32_t*>(a.table + n_slots * KE);
  for (uint64_t t0 = (uint64_t)blockIdx.x * kExtractSlots; t0 < n_slots; t0 += (uint64_t)gridDim.x * kExtractSlots) {
    const uint64_t n = min((uint64_t)kExtractSlots, n_slots - t0);
    const int lo = a.pid_begin, hi = a.pid_end;
    const uint64_t* off = a.tab_off;
    extract_tile<KW>(a.table + t0 * KE, ctr_base + t0 * 8, n,
                     [=](uint64_t s) { return (uint32_t)find_part(off, lo, hi, s0 + t0 + s); }, oa, sh);
  }
}

// --------------------------------------------------------------- on-chip Step 2
//
// One CTA builds one fine partition at a time entirely in shared memory
// (dbg_build_subgraphs_smem).  The partition's records are loaded in batches
// into shared memory, a block scan of their K-mer counts flattens the batch,
// and each thread takes an equal contiguous run of K-mers, rolling the
// forward/reverse codes from one K-mer to the next inside a record
// (<kmer, edge> pair generation).  Each occurrence is inserted or
// updated in the shared-memory table (one insertion, multiple updates,
// P:L504-511): a 64/128-bit shared-memory CAS claims an empty slot, shared-
// memory atomics count the edges.  The CTA then compacts the occupied slots
// straight into the output and zeroes them again (clean-on-extract, so no
// zero pass between partitions).
//
// Slot = key (8 B; 16 B for K > 31) + 16-bit counter fields out[0..3],
// in[0..3], t_out packed two per 32-bit word: a field never exceeds the
// partition's K-mer count, and the on-chip path takes only partitions whose
// capacity (>= N^i_kmer) is below 65536, so the 32-bit shared-memory
// atomicAdd of (1 << 16*half) never carries across fields.

constexpr uint64_t kSmemMaxSlots = 65535;

// Shared-memory table, structure of arrays (dense keys keep random probes
// spread over the banks): keys[cap] (8 B, or 16 B for K > 31), then
// fields[cap][6] u32: out0|out1, out2|out3, in0|in1, in2|in3, t_out, fine pid.
template <int KW>
struct SmemSlot {
  static constexpr uint32_t kKeyBytes = KW == 1 ? 8 : 16;
  static constexpr uint32_t kFieldWords = 5;
  // the nine 16-bit fields packed at 18 bytes per slot (field f of slot s is half 9s + f of
  // the field array); the fine partition of a slot is found from the plan at extraction
  static constexpr uint32_t kBytes = kKeyBytes + 18;
};

// Decoded work item (32 B): records [r0, r0 + nrec) of partitions [first, last);
// P0 = the group's first slot in the plan's prefix P; meta = span (16 bits) |
// sub-table j << 16 | sub-table count ns << 24 (ns = 1: a group; 0: no more work).
struct __align__(16) ItemDesc {
  uint64_t r0, P0;
  uint32_t nrec, first, last, meta;
};
__host__ __device__ constexpr uint32_t item_meta(uint32_t span, uint32_t j, uint32_t ns) {
  return span | j << 16 | ns << 24;
}

constexpr int kGroupParts = 256;  // partitions per group at most (plan rule)

// Records per batch: 1024 four-word or 512 eight-word records (16 KB) from 512
// threads up; fewer for smaller CTAs.
template <int R, int T>
__host__ __device__ constexpr int smem_rec_batch() { return (T >= 512 ? 1024 : 2 * T) * 4 / R; }

template <int R, int T>
struct SmemStage {
  static constexpr int RB = smem_rec_batch<R, T>();
  uint32_t w[2][R][RB];                       // records of two batches, transposed: word q of record j at w[b][q][j]
  unsigned long long Pq[2][kGroupParts + 2];  // P[first .. last] of the current and the next item
  uint32_t pre[RB + 1];                       // K-mer offsets of the records with on-chip K-mers
  uint2 desc[RB];                             // their descriptors: x = batch position | n << 10 |
                                              // hl << 16 | hr << 17, y = table offset | capacity << 16
  uint16_t rwin[(RB * (16 * (R - 1) - 1) + 31) / 32 + 1];  // record of the first K-mer of each warp window
  ItemDesc it[4];                             // items i .. i+3 (ring)
  typename cub::BlockScan<uint32_t, T>::TempStorage scan;
  typename cub::BlockReduce<unsigned long long, T>::TempStorage red;
  unsigned long long base;
};

// cp.async (sm_80+ asynchronous global -> shared copies; completion per thread).
__device__ __forceinline__ void cp_async4(void* dst, const void* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"((uint32_t)__cvta_generic_to_shared(dst)),
               "l"(src));
}
__device__ __forceinline__ void cp_async8(void* dst, const void* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"((uint32_t)__cvta_generic_to_shared(dst)),
               "l"(src));
}
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"((uint32_t)__cvta_generic_to_shared(dst)),
               "l"(src));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;\n" ::: "memory"); }

template <int R, int T>
__host__ __device__ constexpr uint32_t smem_fixed_bytes() {
  return (uint32_t)((sizeof(SmemStage<R, T>) + 127) & ~size_t(127));
}

// 32-bit shared-window addresses (no generic-pointer arithmetic in the probe loop).
__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t lds64(uint32_t a) {
  uint64_t v;
  asm volatile("ld.volatile.shared.u64 %0, [%1];" : "=l"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ ulonglong2 lds_u4x(uint32_t a) {
  ulonglong2 v;
  asm volatile("ld.volatile.shared.v2.u64 {%0, %1}, [%2];" : "=l"(v.x), "=l"(v.y) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t lds32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ uint32_t lds_u16(uint32_t a) {
  uint16_t v;
  asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts64(uint32_t a, uint64_t v) {
  asm volatile("st.shared.u64 [%0], %1;" ::"r"(a), "l"(v) : "memory");
}
__device__ __forceinline__ void sts16(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u16 [%0], %1;" ::"r"(a), "h"((uint16_t)v) : "memory");
}
__device__ __forceinline__ uint2 lds_u2(uint32_t a) {
  uint2 v;
  asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
  return v;
}
__device__ __forceinline__ uint64_t cas_shared64(uint32_t a, uint64_t want) {
  uint64_t old;
  asm volatile("atom.shared.cas.b64 %0, [%1], %2, %3;" : "=l"(old) : "r"(a), "l"(0ull), "l"(want) : "memory");
  return old;
}
// Predicated CAS: cur = atom.cas(a, 0, want) when p, unchanged otherwise.
__device__ __forceinline__ void cas_shared64_if(bool p, uint32_t a, uint64_t want, uint64_t& cur) {
  asm volatile(
      "{ .reg .pred q; setp.ne.u32 q, %1, 0; @q atom.shared.cas.b64 %0, [%2], %3, %4; }"
      : "+l"(cur)
      : "r"((uint32_t)p), "r"(a), "l"(0ull), "l"(want)
      : "memory");
}
__device__ __forceinline__ void red_shared_or(uint32_t a, uint32_t v) {
  asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void red_shared_add(uint32_t a, uint32_t v) {
  asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void sts32(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}

__device__ __forceinline__ void smem_count(uint32_t* fields, int f) {
  atomicAdd(fields + (f >> 1), 1u << (16 * (f & 1)));
}

// 32-bit table hash of a code (the probe sequence is free, reading P).
__device__ __forceinline__ uint32_t smem_hash(uint64_t code) {
  return (uint32_t)(((code ^ (code >> 29)) * 0x9e3779b97f4a7c15ull) >> 32);
}
__device__ __forceinline__ uint32_t smem_hash(unsigned long long code) { return smem_hash((uint64_t)code); }
__device__ __forceinline__ uint32_t smem_hash(u128 code) {
  return smem_hash((uint64_t)((uint64_t)code ^ ((uint64_t)(code >> 64) * 0xc2b2ae3d27d4eb4full)));
}

struct SmemArgs {
  const uint32_t* records;
  const uint64_t* rec_off;
  const uint64_t* n_kmers;
  const unsigned long long* staged;  // pass-1 records; > staging_cap: overflow, nothing to build
  uint64_t staging_cap;
  int pid0, n_fine, k;  // fine partitions [pid0, pid0 + n_fine)
  double ratio;         // lambda / (4 alpha)
  uint64_t slots;       // table slots that fit one CTA
  uint32_t max_split;   // CTAs (sub-tables) an oversize partition may be split over; < 2: none
  FastMod np_mod;       // reported pid = fine pid mod NP
  uint64_t* P;          // [n_fine + 1] prefix of grouped on-chip capacities (0 for the others), local index
  uint32_t* gfirst;     // [n_fine + 2] first (absolute) partition of each group
  uint32_t* sp;         // [n_fine] split partitions (absolute ids), ascending
  uint32_t* ss;         // [n_fine + 1] exclusive prefix of their sub-table counts
  uint8_t* flag;        // [n_fine] group-start flags
  unsigned long long *t_gc, *t_sp, *t_fl;  // per-tile sums (scan.cuh), tiles + 1 each
  unsigned long long* ctr;  // [0] groups, [1] split partitions, [2] split items, [3] work counter
  ItemDesc* gdesc;          // [n_fine] decoded groups
};

// A partition's table capacity (Sec. IV-A), its grouped on-chip
// capacity (0 unless onchip_tables == 1) and its sub-table count when split
// (0 unless onchip_tables >= 2; dbg_device.cuh).
struct OnChip {
  uint64_t cap, gc;
  uint32_t ns;
};
__device__ __forceinline__ OnChip on_chip(const SmemArgs& a, uint64_t nk) {
  OnChip o;
  o.cap = table_capacity(a.ratio, nk);
  const uint32_t t = onchip_tables(nk, o.cap, a.slots, a.max_split);
  o.gc = t == 1 ? o.cap : 0;
  o.ns = t >= 2 ? t : 0;
  return o;
}

// The plan (5 launches, scan.cuh tiles): A per-tile sums of the grouped
// capacities and of the split counts; B scans of those; C writes P, the split
// list and the group-start flags; D scans the flag counts; E writes gfirst.
// Groups: with H = slots/2 and w(p) = floor(P[p]/H), partition p starts a
// group iff p == 0, w(p) != w(p-1), p or p-1 has capacity > H, or p is a
// multiple of kGroupParts (a group's partition offsets fit shared memory).  A group of
// small partitions lies in one H-window and spans < H + H = slots; a larger
// one is alone; a split or global partition is alone with span 0 (skipped).
constexpr unsigned long long kSplitOne = 1ull << 32;  // packed (split partitions << 32) | sub-tables

__global__ void __launch_bounds__(kTileThreads) smem_plan_reduce_kernel(SmemArgs a) {
  typedef cub::BlockReduce<unsigned long long, kTileThreads> Red;
  __shared__ typename Red::TempStorage tmp;
  const int base = blockIdx.x * kTileSize;
  unsigned long long gc = 0, sp = 0;
#pragma unroll
  for (int q = 0; q < kTileItems; ++q) {
    const int p = base + q * kTileThreads + threadIdx.x;
    if (p < a.n_fine) {
      const OnChip o = on_chip(a, a.n_kmers[a.pid0 + p]);
      gc += o.gc;
      sp += o.ns ? kSplitOne | o.ns : 0ull;
    }
  }
  gc = Red(tmp).Sum(gc);
  __syncthreads();
  sp = Red(tmp).Sum(sp);
  if (threadIdx.x == 0) {
    a.t_gc[blockIdx.x] = gc;
    a.t_sp[blockIdx.x] = sp;
  }
}

__global__ void __launch_bounds__(kTileThreads) smem_plan_apply_kernel(SmemArgs a) {
  typedef cub::BlockScan<unsigned long long, kTileThreads> Scan;
  typedef cub::BlockReduce<unsigned int, kTileThreads> Red;
  __shared__ union {
    typename Scan::TempStorage scan;
    typename Red::TempStorage red;
  } tmp;
  const uint64_t H = a.slots / 2;
  const int base = blockIdx.x * kTileSize + threadIdx.x * kTileItems;
  unsigned long long cap[kTileItems], P[kTileItems], sp[kTileItems];
  uint32_t is_split = 0;
#pragma unroll
  for (int q = 0; q < kTileItems; ++q) {
    const int p = base + q;
    const OnChip o = on_chip(a, p < a.n_fine ? a.n_kmers[a.pid0 + p] : 0ull);
    cap[q] = o.cap;
    P[q] = o.gc;
    sp[q] = o.ns ? kSplitOne | o.ns : 0ull;
    is_split |= (o.ns ? 1u : 0u) << q;
  }
  unsigned long long tot_gc, tot_sp;
  Scan(tmp.scan).ExclusiveSum(P, P, tot_gc);
  __syncthreads();
  Scan(tmp.scan).ExclusiveSum(sp, sp, tot_sp);
  __syncthreads();
  const unsigned long long o_gc = a.t_gc[blockIdx.x], o_sp = a.t_sp[blockIdx.x];
  unsigned int nflag = 0;
#pragma unroll
  for (int q = 0; q < kTileItems; ++q) {
    const int p = base + q;
    if (p >= a.n_fine) break;
    const unsigned long long Pp = o_gc + P[q];
    a.P[p] = Pp;
    if (is_split >> q & 1u) {
      const unsigned long long x = o_sp + sp[q];
      a.sp[x >> 32] = (uint32_t)(a.pid0 + p);
      a.ss[x >> 32] = (uint32_t)x;
    }
    bool f = p == 0;
    if (!f) {
      unsigned long long pcap, pP;
      if (q > 0) {
        pcap = cap[q - 1];
        pP = o_gc + P[q - 1];
      } else {  // the neighbour belongs to another thread or tile: recompute it
        const OnChip o = on_chip(a, a.n_kmers[a.pid0 + p - 1]);
        pcap = o.cap;
        pP = Pp - o.gc;
      }
      f = Pp / H != pP / H || cap[q] > H || pcap > H || p % kGroupParts == 0;
    }
    a.flag[p] = f;
    nflag += f;
  }
  nflag = Red(tmp.red).Sum(nflag);
  if (threadIdx.x == 0) {
    a.t_fl[blockIdx.x] = nflag;
    if (blockIdx.x == gridDim.x - 1) {
      const unsigned long long s = o_sp + tot_sp;
      a.P[a.n_fine] = o_gc + tot_gc;
      a.ss[s >> 32] = (uint32_t)s;
      a.ctr[1] = s >> 32;
      a.ctr[2] = (uint32_t)s;
    }
  }
}

// C': greedy packing (replaces C's group-start flags and their tile counts):
// inside each run of kGroupParts consecutive partitions, partitions are packed
// in order into groups while their grouped capacities fit one CTA table
// (span <= slots), so a group fills the table instead of one H-window of it;
// a split or global partition (capacity, nothing grouped) stays alone with
// span 0, as does an empty run.  One CTA per scan tile: the tile's N^i_kmer go
// to shared memory, then one thread per run packs it sequentially.
constexpr int kRunsPerTile = kTileSize / kGroupParts;
static_assert(kTileSize % kGroupParts == 0, "a scan tile holds whole group runs");
__global__ void __launch_bounds__(kTileThreads) smem_plan_pack_kernel(SmemArgs a) {
  typedef cub::BlockReduce<unsigned int, kTileThreads> Red;
  __shared__ uint32_t gc[kTileSize];  // grouped capacity; ~0u: alone (split or global)
  __shared__ uint8_t fl[kTileSize];
  __shared__ typename Red::TempStorage tmp;
  const int base = blockIdx.x * kTileSize;
  for (int q = threadIdx.x; q < kTileSize; q += kTileThreads) {
    const int p = base + q;
    uint32_t v = 0;
    if (p < a.n_fine) {
      const OnChip o = on_chip(a, a.n_kmers[a.pid0 + p]);
      v = o.gc ? (uint32_t)o.gc : (o.cap ? ~0u : 0u);
    }
    gc[q] = v;
  }
  __syncthreads();
  if (threadIdx.x < kRunsPerTile) {
    const int q0 = threadIdx.x * kGroupParts;
    uint64_t acc = 0;
    bool prev_alone = true;
    for (int q = q0; q < q0 + kGroupParts; ++q) {
      const uint32_t v = gc[q];
      const bool alone = v == ~0u;
      const uint32_t c = alone ? 0u : v;
      const bool f = q == q0 || alone || prev_alone || acc + c > a.slots;
      acc = f ? c : acc + c;
      prev_alone = alone;
      fl[q] = f;
    }
  }
  __syncthreads();
  unsigned int nflag = 0;
  for (int q = threadIdx.x; q < kTileSize; q += kTileThreads) {
    const int p = base + q;
    if (p < a.n_fine) {
      a.flag[p] = fl[q];
      nflag += fl[q];
    }
  }
  nflag = Red(tmp).Sum(nflag);
  if (threadIdx.x == 0) a.t_fl[blockIdx.x] = nflag;
}

__global__ void __launch_bounds__(kTileThreads) smem_plan_groups_kernel(SmemArgs a) {
  typedef cub::BlockScan<unsigned int, kTileThreads> Scan;
  __shared__ typename Scan::TempStorage tmp;
  const int base = blockIdx.x * kTileSize + threadIdx.x * kTileItems;
  unsigned int f[kTileItems];
#pragma unroll
  for (int q = 0; q < kTileItems; ++q) f[q] = base + q < a.n_fine ? a.flag[base + q] : 0u;
  unsigned int tot;
  Scan(tmp).ExclusiveSum(f, f, tot);
  const unsigned long long o = a.t_fl[blockIdx.x];
#pragma unroll
  for (int q = 0; q < kTileItems; ++q) {
    const int p = base + q;
    if (p < a.n_fine && a.flag[p]) a.gfirst[o + f[q]] = (uint32_t)(a.pid0 + p);
  }
  if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) {
    a.gfirst[o + tot] = (uint32_t)(a.pid0 + a.n_fine);
    a.ctr[0] = o + tot;
    a.ctr[3] = 0;  // work counter of smem_subgraph_kernel
  }
}

// F: one descriptor per group (records, plan offsets); groups with nothing on
// chip get no records.
__global__ void __launch_bounds__(256) smem_plan_desc_kernel(SmemArgs a) {
  const uint64_t ng = a.ctr[0];
  for (uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; g < ng; g += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t first = a.gfirst[g], last = a.gfirst[g + 1];
    const uint64_t P0 = a.P[first - a.pid0], span = a.P[last - a.pid0] - P0;
    ItemDesc d;
    d.r0 = a.rec_off[first];
    d.P0 = P0;
    d.nrec = span ? (uint32_t)(a.rec_off[last] - d.r0) : 0u;
    d.first = first;
    d.last = last;
    d.meta = item_meta((uint32_t)span, 0, 1);
    a.gdesc[g] = d;
  }
}

// Warp-wide: claim result g -> descriptor of item g in *out (visible after the
// caller's next cp_async_wait_all + barrier).  Groups: one 32-B cp.async of
// the plan's descriptor; split sub-tables: a 32-ary search of the split list.
__device__ __forceinline__ void fetch_item(const SmemArgs& a, uint64_t g, uint64_t n_split, uint64_t n_items,
                                           ItemDesc* out, int lane) {
  if (g >= n_items) {
    if (lane == 0) out->meta = 0;
    return;
  }
  if (g >= n_split) {
    if (lane == 0) {
      const char* src = reinterpret_cast<const char*>(a.gdesc + (g - n_split));
      cp_async16(out, src);
      cp_async16(reinterpret_cast<char*>(out) + 16, src + 16);
    }
    return;
  }
  uint32_t lo = 0, n = (uint32_t)a.ctr[1];  // last i in [lo, lo + n) with ss[i] <= g; ss[lo] <= g
  while (n > 1) {
    const uint32_t step = (n + 31) / 32;
    const bool le = (uint32_t)lane * step < n && a.ss[lo + lane * step] <= g;
    const int L = 31 - __clz(__ballot_sync(kFull, le));
    lo += L * step;
    n = min(step, n - L * step);
  }
  if (lane == 0) {
    const uint32_t p = a.sp[lo], j = (uint32_t)g - a.ss[lo], ns = a.ss[lo + 1] - a.ss[lo];
    out->r0 = a.rec_off[p];
    out->P0 = 0;
    out->nrec = (uint32_t)(a.rec_off[p + 1] - out->r0);
    out->first = p;
    out->last = p + 1;
    out->meta = item_meta((uint32_t)a.slots, j, ns);
  }
}

// Sub-table of a K-mer in a split partition: a hash independent of the slot hash.
template <typename Code>
__device__ __forceinline__ uint32_t sub_table(Code code, uint32_t n) {
  uint64_t x;
  if constexpr (sizeof(Code) == 8) x = (uint64_t)code;
  else x = (uint64_t)code ^ ((uint64_t)(code >> 64) * 0x9e3779b97f4a7c15ull);
  return __umulhi((uint32_t)(fmix64(x) >> 32), n);
}

// A 56-byte vertex record with 16-byte stores where aligned: record i starts at 56 i, which is
// 16-aligned for even i (words 0-11 as three 16-B stores, 12-13 as one 8-B store) and 8 past a
// 16-B boundary for odd i (words 0-1 as 8 B, 2-13 as three 16-B stores): five predicated store
// instructions per warp instead of seven 8-byte ones, with the same bytes.
__device__ __forceinline__ void store_vertex16(dbg_vertex* dst, const dbg_vertex& v, bool odd) {
  uint32_t w[14];
  w[0] = (uint32_t)v.kmer_hi; w[1] = (uint32_t)(v.kmer_hi >> 32);
  w[2] = (uint32_t)v.kmer_lo; w[3] = (uint32_t)(v.kmer_lo >> 32);
  w[4] = v.count;
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    w[5 + q] = v.out[q];
    w[9 + q] = v.in[q];
  }
  w[13] = v.pid;
  char* base = reinterpret_cast<char*>(dst);
  const int sh = odd ? 2 : 0;  // first word of the 16-B run
#pragma unroll
  for (int c = 0; c < 3; ++c) {
    const int q = 4 * c;
    const uint4 x = odd ? make_uint4(w[q + 2], w[q + 3], w[q + 4], w[q + 5]) : make_uint4(w[q], w[q + 1], w[q + 2], w[q + 3]);
    *reinterpret_cast<uint4*>(base + 4 * (q + sh)) = x;
  }
  const int r = odd ? 0 : 12;  // the 8-byte remainder
  *reinterpret_cast<uint2*>(base + 4 * r) = odd ? make_uint2(w[0], w[1]) : make_uint2(w[12], w[13]);
}

// A group of consecutive fine partitions shares one CTA table: each partition
// p owns slots [P[p] - P[first], P[p+1] - P[first]).
template <typename Code, int R, int kSmemThreads, int kMinCtas, int KC = 0, int PC = 0>
__global__ void __launch_bounds__(kSmemThreads, kMinCtas) smem_subgraph_kernel(SmemArgs a, OutArgs oa) {
  constexpr int KW = sizeof(Code) == 8 ? 1 : 2;
  constexpr uint32_t KB = SmemSlot<KW>::kKeyBytes;
  constexpr int RB = SmemStage<R, kSmemThreads>::RB;
  constexpr int kRPT = RB >= kSmemThreads ? RB / kSmemThreads : 1;  // records per thread per batch
  typedef cub::BlockScan<uint32_t, kSmemThreads> Scan;
  extern __shared__ __align__(128) unsigned char smem[];
  SmemStage<R, kSmemThreads>& st = *reinterpret_cast<SmemStage<R, kSmemThreads>*>(smem);
  char* keys = reinterpret_cast<char*>(smem + smem_fixed_bytes<R, kSmemThreads>());
  uint32_t* fld = reinterpret_cast<uint32_t*>(keys + a.slots * KB);
  const uint32_t keys_s = smem_addr(keys), fld_s = smem_addr(fld);
  const int K = KC ? KC : a.k;  // KC: compile-time K (shifts by constants)
  {  // the table starts clean; extraction keeps it clean (slots is a multiple of 64)
    uint4* z = reinterpret_cast<uint4*>(keys);
    for (uint64_t q = threadIdx.x; q < a.slots * SmemSlot<KW>::kBytes / 16; q += kSmemThreads)
      z[q] = make_uint4(0, 0, 0, 0);
  }
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  unsigned long long st_n = 0, st_count = 0, st_edges = 0;
  bool ok = true;
  if (a.staged && *a.staged > a.staging_cap) return;  // staging overflow: the records are incomplete
  const uint64_t n_split = a.ctr[2], n_items = n_split + a.ctr[0];
  // Work items are claimed from a global counter, first the sub-tables of the
  // split partitions (the longest items), then the groups, and decoded three
  // items ahead (ring st.it).  The CTA consumes a stream of record batches;
  // the next batch -- of the same item, or the next item's first with its plan
  // offsets -- is copied in with cp.async while the current one is hashed.
  uint64_t g_next = 0;  // warp 0 lane 0: the claim for the next item to decode
  if (warp == 0) {
    uint64_t g[4] = {0, 0, 0, 0};
    if (lane == 0)
      for (int q = 0; q < 4; ++q) g[q] = atomicAdd(a.ctr + 3, 1ull);
    for (int q = 0; q < 3; ++q) fetch_item(a, __shfl_sync(kFull, g[q], 0), n_split, n_items, st.it + q, lane);
    g_next = g[3];
    cp_async_wait_all();
  }
  __syncthreads();
  auto prefetch = [&](const ItemDesc& I, uint32_t rb, int bb, int ip, bool with_p) {
    const uint32_t n = min((uint32_t)RB, I.nrec - rb);
    const uint32_t* src = a.records + (I.r0 + rb) * R;
    for (uint32_t j = threadIdx.x; j < n; j += kSmemThreads)
#pragma unroll
      for (int q = 0; q < R; ++q) cp_async4(&st.w[bb][q][j], src + (uint64_t)j * R + q);
    if (with_p)
      for (uint32_t t = threadIdx.x; t <= I.last - I.first; t += kSmemThreads)
        cp_async8(&st.Pq[ip][t], a.P + (I.first - a.pid0) + t);
  };
  if (st.it[0].meta >> 24) prefetch(st.it[0], 0, 0, 0, (st.it[0].meta >> 24) == 1);
  cp_async_commit();
  int ci = 0, ip = 0, bb = 0;
  uint32_t rb = 0;
  for (;;) {
    cp_async_wait_all();
    __syncthreads();  // this batch is in st.w[bb]; the other buffer and the previous item are done
    const ItemDesc I = st.it[ci];
    const uint32_t sub_n = I.meta >> 24;
    if (sub_n == 0) break;
    const uint32_t sub_j = (I.meta >> 16) & 255u, span = I.meta & 0xffffu;
    const bool split = sub_n > 1;
    const int nb = (int)min((uint32_t)RB, I.nrec - rb);
    const bool last_batch = rb + RB >= I.nrec;
    if (rb == 0 && warp == 0) {  // item start: claim the next one and decode item i+3
      const uint64_t g = __shfl_sync(kFull, g_next, 0);
      if (lane == 0) g_next = atomicAdd(a.ctr + 3, 1ull);
      fetch_item(a, g, n_split, n_items, st.it + ((ci + 3) & 3), lane);
    }
    if (!last_batch) {
      prefetch(I, rb + RB, bb ^ 1, ip, false);
    } else {
      const ItemDesc& N = st.it[(ci + 1) & 3];
      if (N.meta >> 24) prefetch(N, 0, bb ^ 1, ip ^ 1, (N.meta >> 24) == 1);
    }
    cp_async_commit();
    const unsigned long long* Pq = st.Pq[ip];
    // Flatten the batch: one packed scan gives every record with on-chip K-mers its
    // K-mer offset (low 16 bits) and its index among those records (high 16 bits).
    uint32_t cnt[kRPT];
#pragma unroll
    for (int v = 0; v < kRPT; ++v) {
      const int j = kRPT * threadIdx.x + v;
      cnt[v] = 0;
      if (j < nb) {
        const uint32_t w0 = st.w[bb][0][j];
        uint32_t c;
        if (split) {
          c = hdr_n(w0);
        } else {
          const uint32_t x = hdr_pid(w0) - I.first;
          c = Pq[x + 1] != Pq[x] ? hdr_n(w0) : 0u;  // off-chip partition: skipped here
        }
        cnt[v] = c ? c | 1u << 16 : 0u;
      }
    }
    uint32_t excl[kRPT], packed_total;
    Scan(st.scan).ExclusiveSum(cnt, excl, packed_total);
    const uint32_t total = packed_total & 0xffffu, nc = packed_total >> 16;
    // Record c (compacted) holds K-mers [cpre[c], cpre[c+1]); rwin[m] = the record holding
    // K-mer 32m, the first of warp window m.
#pragma unroll
    for (int v = 0; v < kRPT; ++v) {
      if (cnt[v]) {
        const uint32_t c = excl[v] >> 16, e = excl[v] & 0xffffu, n = cnt[v] & 0xffffu;
        const int jj = kRPT * threadIdx.x + v;
        const uint32_t w0 = st.w[bb][0][jj];
        uint32_t t0 = 0, cp = (uint32_t)a.slots;
        if (!split) {
          const uint32_t x = hdr_pid(w0) - I.first;
          t0 = (uint32_t)(Pq[x] - I.P0);
          cp = (uint32_t)(Pq[x + 1] - Pq[x]);
        }
        st.pre[c] = e;
        st.desc[c] = make_uint2((uint32_t)jj | (w0 & 255u) << 10, t0 | cp << 16);
        for (uint32_t m = (e + 31) >> 5; 32 * m < e + n; ++m) st.rwin[m] = (uint16_t)c;
      }
    }
    if (threadIdx.x == 0) st.pre[nc] = total;
    __syncthreads();
    {
      // Warp windows: window m = K-mers [32m, 32m + 32), lane l takes K-mer 32m + l;
      // window m goes to warp m mod (warps), so the warps' loads differ by at most one
      // window and no thread waits on a long record.  All lanes run every step, so the
      // probe vote is warp-wide and the counter updates run reconverged.
      constexpr int S = RB;  // staging stride
      constexpr uint32_t kWarps = kSmemThreads / 32;
      typedef KeyOf<Code> KO;
      for (uint32_t m = warp; 32 * m < total; m += kWarps) {
        const uint32_t kb = 32 * m, kid = kb + lane;
        const bool act = kid < total;
        const uint32_t rb = st.rwin[m];
        // records starting inside the window: one bit each at their first K-mer
        const uint32_t nxt = rb + 1 + lane;
        const uint32_t x0 = nxt < nc ? st.pre[nxt] : total;
        const uint32_t starts = __reduce_or_sync(kFull, x0 < kb + 32 ? 1u << (x0 - kb) : 0u);
        const uint32_t c = rb + __popc(starts & ((2u << lane) - 1u));
        const uint32_t cc = act ? c : rb;
        const uint2 d = st.desc[cc];
        const int t = (int)(kid - st.pre[cc]);
        const int j = d.x & 1023u, n = (d.x >> 10) & kHdrNMask, hl = (d.x >> 16) & 1u, hr = (d.x >> 17) & 1u;
        const uint32_t t0 = d.y & 0xffffu, cap = d.y >> 16;
        const uint32_t* w = &st.w[bb][0][j];
        const int b = hl + t;
        Code fwd, rc;
        int pred, succ;
        if constexpr (R == 4) {
          // the three data words, loaded unconditionally and selected (no branches): a1..a3
          // hold bases b .. b + 47 - 16q
          const uint32_t d1 = w[S], d2 = w[2 * S], d3 = w[3 * S];
          const int q = b >> 4;
          const uint32_t a1 = q == 0 ? d1 : (q == 1 ? d2 : d3), a2 = q == 0 ? d2 : (q == 1 ? d3 : 0u),
                         a3 = q == 0 ? d3 : 0u;
          const int pb = b - 1, pq = pb >> 4;  // the predecessor base
          const uint32_t pw = pq <= 0 ? d1 : (pq == 1 ? d2 : d3);
          pred = b > 0 ? (int)((pw >> (30 - 2 * (pb & 15))) & 3u) : -1;
          if constexpr (sizeof(Code) == 8) {
            // 64 bits of the record from base b: two 32-bit funnel shifts
            const uint32_t sh = 2 * (b & 15);
            const uint64_t win = ((uint64_t)__funnelshift_l(a2, a1, sh) << 32) | __funnelshift_l(a3, a2, sh);
            fwd = win >> (64 - 2 * K);
            succ = (t < n - 1 || hr) ? (int)((win >> (62 - 2 * K)) & 3u) : -1;
            rc = revcomp64(fwd, K);
          } else {
            const u128 X = ((u128)(((uint64_t)a1 << 32) | a2) << 64) | ((u128)a3 << 32);
            const u128 Y = X << (2 * (b & 15));
            fwd = (Code)(Y >> (128 - 2 * K));
            succ = (t < n - 1 || hr) ? (int)((uint32_t)(uint64_t)(Y >> (126 - 2 * K)) & 3u) : -1;
            rc = revcomp128(fwd, K);
          }
        } else if constexpr (R == 8 && sizeof(Code) == 16 && KC > 48) {
          // compile-time K in 49..63 (bumblebee's 63): the five record words holding bases
          // b .. b + 79 are loaded once each and funnel-shifted; pred and succ come from them
          // (pred needs the previous word only when b starts a word)
          const int q = 1 + (b >> 4), sh = 2 * (b & 15);
          uint32_t x[5];
#pragma unroll
          for (int v = 0; v < 5; ++v) x[v] = q + v < R ? w[(q + v) * S] : 0u;
          const uint64_t A = ((uint64_t)x[0] << 32) | x[1], B = ((uint64_t)x[2] << 32) | x[3];
          const uint64_t hi = (A << sh) | ((uint64_t)x[2] >> (32 - sh));
          const uint64_t lo = (B << sh) | ((uint64_t)x[4] >> (32 - sh));
          fwd = (Code)((((u128)hi << 64) | (u128)lo) >> (128 - 2 * KC));
          rc = revcomp128(fwd, KC);
          const uint32_t pw = (b & 15) ? x[0] : w[(q - 1) * S];
          pred = b > 0 ? (int)((pw >> (30 - 2 * ((b - 1) & 15))) & 3u) : -1;
          const int rel = (b & 15) + KC;  // the successor, inside the five words
          const uint32_t sw = (rel >> 4) == 3 ? x[3] : x[4];
          succ = (t < n - 1 || hr) ? (int)((sw >> (30 - 2 * (rel & 15))) & 3u) : -1;
        } else {
          kmer_at(w, b, K, R, fwd, rc, S);
          pred = b > 0 ? (int)rec_base(w, b - 1, S) : -1;
          succ = (t < n - 1 || hr) ? (int)rec_base(w, b + K, S) : -1;
        }
        // canonical orientation and edge indices (readings C, J), selected branch-free so
        // that one probe serves both orientations
        const bool is_fwd = fwd < rc;
        const Code code = is_fwd ? fwd : rc;
        const int o = is_fwd ? (succ >= 0 ? succ : 4) : (pred >= 0 ? 3 - pred : 4);
        const int i = is_fwd ? pred : (succ >= 0 ? 3 - succ : -1);
        const bool want = act && (sub_n == 1 || sub_table(code, sub_n) == sub_j);
        // one insertion, multiple updates: probe rounds until every lane has
        // found or claimed its slot, then the counter updates, warp-converged
        const typename KO::T key = KO::make(code);
        uint32_t idx = __umulhi(smem_hash(code), cap);
        const uint32_t kaddr = keys_s + t0 * KB;
        if constexpr (KW == 1) {
          // every lane runs every probe round (predicated, no divergent branch): a lane with
          // nothing pending re-reads its current slot and keeps its state
          const uint32_t idx0 = idx;
          bool pend = want;
          for (;;) {
            const uint32_t ka = kaddr + idx * KB;
            uint64_t cur = lds64(ka);
            cas_shared64_if(pend && cur == 0, ka, key, cur);
            const bool hit = cur == 0 || cur == key;
            const bool adv = pend && !hit;
            const uint32_t nx = idx + 1 == cap ? 0u : idx + 1;
            idx = adv ? nx : idx;
            pend = adv && nx != idx0;
            if (adv && nx == idx0) ok = false;  // wrapped: table full (reading O)
            if (!__any_sync(kFull, pend)) break;
          }
          if (!ok && want) {
            const uint64_t cur = lds64(kaddr + idx * KB);
            if (cur != key) idx = ~0u;  // this occurrence found no slot
          }
        } else {
          // 16-byte keys: a plain 16-byte load first; the CAS (read-or-claim) only where the
          // entry may be empty.  A claimed entry never changes and a torn read of one being
          // published shows a zero word, so a load with both words nonzero is a whole key; a
          // zero word (empty, torn, or a key whose low word is 0) goes to the CAS, which
          // returns the entry atomically.
          const uint32_t idx0 = idx;
          bool pend = want;
          for (;;) {
            const uint32_t ka = kaddr + idx * KB;
            typename KO::T cur = lds_u4x(ka);
            if (pend && (cur.x == 0 || cur.y == 0)) cur = KO::cas(keys + (size_t)(t0 + idx) * KB, key);
            const bool emp = KO::empty(cur), hit = emp || KO::same(cur, key);
            const bool adv = pend && !hit;
            const uint32_t nx = idx + 1 == cap ? 0u : idx + 1;
            idx = adv ? nx : idx;
            pend = adv && nx != idx0;
            if (adv && nx == idx0) ok = false;  // wrapped: table full (reading O)
            if (!__any_sync(kFull, pend)) break;
          }
          if (!ok && want && !KO::same(lds_u4x(kaddr + idx * KB), key)) idx = ~0u;  // found no slot
        }
        if (want && idx != ~0u) {  // the multiple updates: 16-bit fields, two per word
          const int fo = o < 4 ? o : 8;
          const uint32_t h0 = (t0 + idx) * 9u, ho = h0 + (uint32_t)fo, hi = h0 + 4u + (uint32_t)i;
          red_shared_add(fld_s + (ho >> 1) * 4, 1u << (16 * (ho & 1)));
          if (i >= 0) red_shared_add(fld_s + (hi >> 1) * 4, 1u << (16 * (hi & 1)));
        }
      }
    }
    if (last_batch) {
      __syncthreads();
      // extraction: each warp owns a contiguous run of slots and works alone: it queues
      // the kept occupied slots of a chunk (16-bit indices, in the finished record buffer
      // of this batch), reserves their output with one global atomic and emits them with
      // every lane busy -- no block-wide scan or barrier.
      constexpr int kWarps = kSmemThreads / 32;
      constexpr uint32_t kQ = (uint32_t)(sizeof(st.w[0]) / 2 / kWarps) / 32 * 32;  // queue entries per warp
      const uint32_t wspan = (span + kWarps * 32 - 1) / (kWarps * 32) * 32;  // slots per warp
      const uint32_t ws0 = min(span, warp * wspan), ws1 = min(span, ws0 + wspan);
      uint16_t* queue = reinterpret_cast<uint16_t*>(&st.w[bb][0][0]) + warp * kQ;
      for (uint32_t sub = ws0; sub < ws1; sub += kQ) {
        const uint32_t se = min(ws1, sub + kQ);
        uint32_t qn = 0;
        if (oa.min_count <= 1) {
          // occupied slots: the sign bit of the key's high 32-bit word (OCC); 32-bit shared
          // addresses formed once; two 32-slot chunks per iteration
          const uint32_t q_s = smem_addr(queue), lt = (1u << lane) - 1u;
          uint32_t c = sub;
          for (; c + 64 <= se; c += 64) {
            const uint32_t s0 = c + lane, s1 = s0 + 32;
            const bool k0 = (int)lds32(keys_s + s0 * KB + 4) < 0, k1 = (int)lds32(keys_s + s1 * KB + 4) < 0;
            const uint32_t b0 = __ballot_sync(kFull, k0), b1 = __ballot_sync(kFull, k1);
            if (k0) sts16(q_s + 2 * (qn + __popc(b0 & lt)), s0);
            qn += __popc(b0);
            if (k1) sts16(q_s + 2 * (qn + __popc(b1 & lt)), s1);
            qn += __popc(b1);
          }
          for (; c < se; c += 32) {
            const uint32_t s0 = c + lane;
            const bool k0 = s0 < se && (int)lds32(keys_s + s0 * KB + 4) < 0;
            const uint32_t b0 = __ballot_sync(kFull, k0);
            if (k0) sts16(q_s + 2 * (qn + __popc(b0 & lt)), s0);
            qn += __popc(b0);
          }
        } else
        for (uint32_t c = sub; c < se; c += 32) {
          const uint32_t s = c + lane;
          bool keep = s < se && (lds64(keys_s + s * KB) & kOccupied);
          if (keep && oa.min_count > 1) {  // row f4: a low-count vertex is cleaned, never emitted
            uint16_t* f16 = reinterpret_cast<uint16_t*>(fld) + s * 9;
            if ((uint32_t)f16[0] + f16[1] + f16[2] + f16[3] + f16[8] < oa.min_count) {
              keep = false;
              unsigned long long* kp = reinterpret_cast<unsigned long long*>(keys + s * KB);
              kp[0] = 0;
              if (KW == 2) kp[1] = 0;
#pragma unroll
              for (int q = 0; q < 9; ++q) f16[q] = 0;
            }
          }
          const uint32_t bal = __ballot_sync(kFull, keep);
          if (keep) queue[qn + __popc(bal & ((1u << lane) - 1u))] = (uint16_t)s;
          qn += __popc(bal);
        }
        unsigned long long pos = 0;
        if (lane == 0 && qn) pos = atomicAdd(oa.n_out, (unsigned long long)qn);
        pos = __shfl_sync(kFull, pos, 0);
        __syncwarp();
        for (uint32_t e = lane; e < qn; e += 32) {
          const uint32_t s = queue[e];
          unsigned long long* kp = reinterpret_cast<unsigned long long*>(keys + s * KB);
          const uint64_t kw0 = kp[0];
          dbg_vertex v;
          if (KW == 1) {
            v.kmer_hi = 0;
            v.kmer_lo = kw0 & kCodeMask;
          } else {
            v.kmer_hi = kw0 & kCodeMask;
            v.kmer_lo = kp[1];
          }
          uint16_t* f16 = reinterpret_cast<uint16_t*>(fld) + s * 9;
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            v.out[q] = f16[q];
            v.in[q] = f16[4 + q];
          }
          v.count = v.out[0] + v.out[1] + v.out[2] + v.out[3] + f16[8];  // count = sum(out) + t_out
          // the fine partition owning slot s (last x with Pq[x] - P0 <= s), mod NP -- or the
          // paper's partition from the vertex's P-minimizer (reading V)
          uint32_t fpid = I.first;
          if (sub_n == 1) {
            uint32_t lo = 0, n = I.last - I.first;
            while (n > 1) {
              const uint32_t h = n >> 1;
              if (Pq[lo + h] - I.P0 <= s) lo += h, n -= h;
              else n = h;
            }
            fpid += lo;
          }
          if constexpr (PC > 0)  // compile-time (K, P) of the launch, fine_p != P (reading V)
            v.pid = kmer_partition_c<KC, PC>(v.kmer_lo, oa);
          else
            v.pid = oa.kmer_pid ? kmer_partition(v.kmer_hi, v.kmer_lo, oa) : fast_mod(a.np_mod, fpid);
          kp[0] = 0;  // clean-on-extract
          if (KW == 2) kp[1] = 0;
#pragma unroll
          for (int q = 0; q < 9; ++q) f16[q] = 0;
          const uint64_t my = pos + e;
          if (my < oa.out_cap) {
            store_vertex16(oa.out + my, v, (my & 1) != 0);
          }
          else atomicOr(oa.status, kStatusNoSpace);
          st_n += 1;
          st_count += v.count;
          st_edges += (uint64_t)v.out[0] + v.out[1] + v.out[2] + v.out[3] + v.in[0] + v.in[1] + v.in[2] + v.in[3];
        }
        __syncwarp();
      }
      ci = (ci + 1) & 3;
      ip ^= 1;
      rb = 0;
    } else {
      rb += RB;
    }
    bb ^= 1;
  }
  if (!ok) atomicOr(oa.status, kStatusTableFull);
  __syncthreads();
  typedef cub::BlockReduce<unsigned long long, kSmemThreads> Red;
  const unsigned long long n = Red(st.red).Sum(st_n);
  __syncthreads();
  const unsigned long long cc = Red(st.red).Sum(st_count);
  __syncthreads();
  const unsigned long long e = Red(st.red).Sum(st_edges);
  if (threadIdx.x == 0 && n) {
    atomicAdd(oa.stats + 0, n);
    atomicAdd(oa.stats + 1, cc);
    atomicAdd(oa.stats + 2, e);
  }
}

// --------------------------------------------------------------- checksum

// Order-independent checksum of vertex records: per record
// h = fmix64 chained over its 11 fields; the sum of h (mod 2^64) is added to
// *sum.  A validation statistic, computed apart from the path.
__global__ void __launch_bounds__(256) checksum_kernel(const dbg_vertex* __restrict__ v, uint64_t n,
                                                      unsigned long long* sum) {
  typedef cub::BlockReduce<unsigned long long, 256> Red;
  __shared__ typename Red::TempStorage tmp;
  unsigned long long acc = 0;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const dbg_vertex x = v[i];
    const uint64_t f[11] = {x.kmer_hi, x.kmer_lo, x.count, x.out[0], x.out[1], x.out[2], x.out[3],
                            x.in[0], x.in[1], x.in[2], x.in[3]};
    uint64_t h = 0;
#pragma unroll
    for (int t = 0; t < 11; ++t) h = fmix64(h ^ f[t]);
    acc += h;
  }
  const unsigned long long s = Red(tmp).Sum(acc);
  if (threadIdx.x == 0 && s) atomicAdd(sum, s);
}

// --------------------------------------------------------------- sort

__global__ void sort_prepare_kernel(const dbg_vertex* __restrict__ in, uint64_t n,
                                    unsigned long long* __restrict__ key, unsigned long long* __restrict__ idx) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    key[i] = in[i].kmer_lo;
    idx[i] = i;
  }
}

__global__ void sort_gather_hi_kernel(const dbg_vertex* __restrict__ in, uint64_t n,
                                      const unsigned long long* __restrict__ idx,
                                      unsigned long long* __restrict__ key) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    key[i] = in[idx[i]].kmer_hi;
}

__global__ void sort_gather_kernel(const dbg_vertex* __restrict__ in, uint64_t n,
                                   const unsigned long long* __restrict__ idx, dbg_vertex* __restrict__ out) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    out[i] = in[idx[i]];
}

}  // namespace dbg

using namespace dbg;

extern "C" uint32_t dbg_key_bytes(const dbg_params* prm) { return prm ? key_bytes(prm->k) : 0u; }

extern "C" uint32_t dbg_slot_bytes(const dbg_params* prm) { return prm ? key_bytes(prm->k) + kCtrBytes : 0u; }

extern "C" dbg_status dbg_hash_build(const dbg_params* prm, const dbg_partition_set* part, int32_t pid_begin,
                                     int32_t pid_end, void* d_table, const uint64_t* d_table_offset,
                                     uint32_t* d_status, cudaStream_t stream) {
  if (!dbg_params_ok(prm) || !part || !part->d_records || !part->d_record_offset || !d_table ||
      !d_table_offset || !d_status)
    return DBG_EINVAL;
  if (pid_begin < 0 || pid_end > fine_partitions(prm) || pid_begin > pid_end) return DBG_EINVAL;
  if (pid_begin == pid_end) return DBG_OK;
  if (prm->k > 63) return dbg_wide_hash_build(prm, part, pid_begin, pid_end, d_table, d_table_offset, d_status, stream);
  ResidentArgs a;
  a.records = part->d_records;
  a.rec_off = part->d_record_offset;
  a.tab_off = d_table_offset;
  a.table = static_cast<char*>(d_table);
  a.pid_begin = pid_begin;
  a.pid_end = pid_end;
  a.k = prm->k;
  a.status = d_status;
  const int grid = dbg_sm_count() * 8;
  if (prm->k <= 31) hash_build_kernel<uint64_t, 4><<<grid, kThreads, 0, stream>>>(a);
  else if (prm->k <= 39) hash_build_kernel<u128, 4><<<grid, kThreads, 0, stream>>>(a);
  else hash_build_kernel<u128, 8><<<grid, kThreads, 0, stream>>>(a);
  return cudaPeekAtLastError() == cudaSuccess ? DBG_OK : DBG_ECUDA;
}

extern "C" dbg_status dbg_hash_build_list(const dbg_params* prm, const dbg_partition_set* part, int32_t pid_begin,
                                          int32_t pid_end, const uint32_t* d_pids, const uint64_t* d_chunk_prefix,
                                          int32_t n_pids, void* d_table, const uint64_t* d_table_offset,
                                          uint32_t* d_status, cudaStream_t stream) {
  if (!dbg_params_ok(prm) || !part || !part->d_records || !part->d_record_offset || !d_table ||
      !d_table_offset || !d_status || n_pids < 0 || (n_pids && (!d_pids || !d_chunk_prefix)))
    return DBG_EINVAL;
  if (pid_begin < 0 || pid_end > fine_partitions(prm) || pid_begin > pid_end) return DBG_EINVAL;
  if (prm->k > 63) return DBG_EINVAL;  // K > 63: dbg_hash_build (resident tables only)
  if (n_pids == 0) return DBG_OK;
  ResidentArgs a;
  a.records = part->d_records;
  a.rec_off = part->d_record_offset;
  a.tab_off = d_table_offset;
  a.table = static_cast<char*>(d_table);
  a.pid_begin = pid_begin;
  a.pid_end = pid_end;
  a.k = prm->k;
  a.status = d_status;
  const int grid = dbg_sm_count() * 8;
  if (prm->k <= 31) hash_build_list_kernel<uint64_t, 4><<<grid, kThreads, 0, stream>>>(a, d_pids, d_chunk_prefix, n_pids);
  else if (prm->k <= 39) hash_build_list_kernel<u128, 4><<<grid, kThreads, 0, stream>>>(a, d_pids, d_chunk_prefix, n_pids);
  else hash_build_list_kernel<u128, 8><<<grid, kThreads, 0, stream>>>(a, d_pids, d_chunk_prefix, n_pids);
  return cudaPeekAtLastError() == cudaSuccess ? DBG_OK : DBG_ECUDA;
}

extern "C" dbg_status dbg_extract_graph(const dbg_params* prm, void* d_table, const uint64_t* d_table_offset,
                                        int32_t pid_begin, int32_t pid_end, dbg_vertex* d_out, uint64_t out_cap,
                                        uint64_t* d_n_out, dbg_stats* d_stats, uint32_t* d_status,
                                        cudaStream_t stream) {
  if (!dbg_params_ok(prm) || !d_table || !d_table_offset || !d_n_out || !d_stats || !d_status ||
      (out_cap && !d_out))
    return DBG_EINVAL;
  if (pid_begin < 0 || pid_end > fine_partitions(prm) || pid_begin > pid_end) return DBG_EINVAL;
  if (pid_begin == pid_end) return DBG_OK;
  if (prm->k > 63)  // d_out holds dbg_vertex_wide records (dbg.h)
    return dbg_wide_extract(prm, d_table, d_table_offset, pid_begin, pid_end, d_out, out_cap, d_n_out, d_stats,
                            d_status, stream);
  ResidentArgs a;
  a.records = nullptr;
  a.rec_off = nullptr;
  a.tab_off = d_table_offset;
  a.table = static_cast<char*>(d_table);
  a.pid_begin = pid_begin;
  a.pid_end = pid_end;
  a.k = prm->k;
  a.status = d_status;
  const OutArgs oa = make_out_args(prm, d_out, out_cap, d_n_out, d_stats, d_status);
  const int grid = dbg_sm_count() * 4;
  if (prm->k <= 31) extract_kernel<1><<<grid, kThreads, 0, stream>>>(a, oa);
  else extract_kernel<2><<<grid, kThreads, 0, stream>>>(a, oa);
  return cudaPeekAtLastError() == cudaSuccess ? DBG_OK : DBG_ECUDA;
}

template <int R, int T>
static uint64_t smem_slots_for(int k, int ctas) {
  const uint64_t avail = (227u * 1024u) / ctas - smem_fixed_bytes<R, T>() - 1024u;
  const uint32_t sb = k <= 31 ? SmemSlot<1>::kBytes : SmemSlot<2>::kBytes;
  const uint64_t n = (avail / sb) & ~(uint64_t)63;
  return n < kSmemMaxSlots ? n : kSmemMaxSlots;
}

// One persistent CTA of 1024 threads per SM (several smaller CTAs per SM measured slower,
// profiles/r01d_ab.txt).
static uint64_t smem_slots(int k) {
  return record_words(k) == 4 ? smem_slots_for<4, 1024>(k, 1) : smem_slots_for<8, 1024>(k, 1);
}

extern "C" uint64_t dbg_smem_table_slots(const dbg_params* prm) {
  if (!prm || prm->k > 63) return 0;
  return smem_slots(prm->k);
}

template <typename Code, int R, int T, int C, int KC = 0, int PC = 0>
static cudaError_t launch_smem_t(const SmemArgs& a, const OutArgs& oa, cudaStream_t stream) {
  constexpr int KW = sizeof(Code) == 8 ? 1 : 2;
  const size_t bytes = smem_fixed_bytes<R, T>() + a.slots * SmemSlot<KW>::kBytes;
  cudaError_t e = cudaFuncSetAttribute(smem_subgraph_kernel<Code, R, T, C, KC, PC>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
  if (e != cudaSuccess) return e;
  smem_subgraph_kernel<Code, R, T, C, KC, PC><<<dbg_sm_count() * C, T, bytes, stream>>>(a, oa);
  return cudaGetLastError();
}

template <typename Code, int R>
static cudaError_t launch_smem(const SmemArgs& a, const OutArgs& oa, cudaStream_t stream) {
  // the configurations' K (31, 63) as a compile-time constant (shifts and masks by constants)
  if constexpr (sizeof(Code) == 8 && R == 4)
    if (a.k == 31) {
      if (oa.kmer_pid && oa.p == 11)  // chr14's launch: P = 11 vertex partitions under fine_p > P
        return launch_smem_t<Code, R, 1024, 1, 31, 11>(a, oa, stream);
      return launch_smem_t<Code, R, 1024, 1, 31>(a, oa, stream);
    }
  if constexpr (sizeof(Code) == 16 && R == 8)
    if (a.k == 63) return launch_smem_t<Code, R, 1024, 1, 63>(a, oa, stream);
  return launch_smem_t<Code, R, 1024, 1>(a, oa, stream);
}

extern "C" int32_t dbg_smem_onchip(const dbg_params* prm, uint64_t n_kmers) {
  if (!dbg_params_ok(prm) || !(prm->lambda > 0.f) || !(prm->alpha > 0.f)) return -1;
  if (prm->k > 63) return 0;  // row f3: resident (global) tables only
  const double ratio = (double)prm->lambda / (4.0 * (double)prm->alpha);
  return (int32_t)onchip_tables(n_kmers, table_capacity(ratio, n_kmers), dbg_smem_table_slots(prm),
                                smem_max_split(prm));
}

static uint64_t al16(uint64_t x) { return (x + 15) & ~(uint64_t)15; }

// Workspace: P | 3 tile-sum arrays | counters | gfirst | sp | ss | flags.
static uint64_t smem_workspace(uint64_t n, SmemArgs* a, char* ws) {
  const uint64_t tiles = (uint64_t)scan_tiles((int)n) + 1;
  uint64_t o = 0;
  auto take = [&](uint64_t bytes) { const uint64_t at = o; o += al16(bytes); return ws + at; };
  char* P = take(8 * (n + 1));
  char* t_gc = take(8 * tiles);
  char* t_sp = take(8 * tiles);
  char* t_fl = take(8 * tiles);
  char* ctr = take(64);
  char* gfirst = take(4 * (n + 2));
  char* sp = take(4 * n + 4);
  char* ss = take(4 * (n + 1));
  char* flag = take(n + 1);
  char* gdesc = take(sizeof(ItemDesc) * (n + 1));
  if (a) {
    a->gdesc = reinterpret_cast<ItemDesc*>(gdesc);
    a->P = reinterpret_cast<uint64_t*>(P);
    a->t_gc = reinterpret_cast<unsigned long long*>(t_gc);
    a->t_sp = reinterpret_cast<unsigned long long*>(t_sp);
    a->t_fl = reinterpret_cast<unsigned long long*>(t_fl);
    a->ctr = reinterpret_cast<unsigned long long*>(ctr);
    a->gfirst = reinterpret_cast<uint32_t*>(gfirst);
    a->sp = reinterpret_cast<uint32_t*>(sp);
    a->ss = reinterpret_cast<uint32_t*>(ss);
    a->flag = reinterpret_cast<uint8_t*>(flag);
  }
  return o;
}

extern "C" uint64_t dbg_smem_workspace_bytes(const dbg_params* prm) {
  if (!prm) return 0;
  return smem_workspace((uint64_t)fine_partitions(prm), nullptr, nullptr);
}

extern "C" dbg_status dbg_build_subgraphs_smem(const dbg_params* prm, const dbg_partition_set* part,
                                               int32_t pid_begin, int32_t pid_end, void* d_work,
                                               uint64_t work_bytes, dbg_vertex* d_out, uint64_t out_cap,
                                               uint64_t* d_n_out, dbg_stats* d_stats, uint32_t* d_status,
                                               cudaStream_t stream) {
  if (!dbg_params_ok(prm) || !part || !part->d_records || !part->d_record_offset || !part->d_n_kmers || !d_work ||
      !d_n_out || !d_stats || !d_status || (out_cap && !d_out))
    return DBG_EINVAL;
  if (prm->k > 63) return DBG_EINVAL;  // row f3: resident tables only
  if (!(prm->lambda > 0.f) || !(prm->alpha > 0.f)) return DBG_EINVAL;
  if (pid_begin < 0 || pid_end > fine_partitions(prm) || pid_begin > pid_end) return DBG_EINVAL;
  if (pid_begin == pid_end) return DBG_OK;
  if (work_bytes < dbg_smem_workspace_bytes(prm)) return DBG_EINVAL;
  SmemArgs a;
  a.records = part->d_records;
  a.rec_off = part->d_record_offset;
  a.n_kmers = part->d_n_kmers;
  a.staged = reinterpret_cast<const unsigned long long*>(part->d_staged);
  a.staging_cap = part->staging_cap;
  a.pid0 = pid_begin;
  a.n_fine = pid_end - pid_begin;
  a.np_mod = make_fastmod((uint64_t)prm->num_partitions);
  a.k = prm->k;
  a.ratio = (double)prm->lambda / (4.0 * (double)prm->alpha);
  a.slots = dbg_smem_table_slots(prm);
  a.max_split = smem_max_split(prm);
  smem_workspace((uint64_t)a.n_fine, &a, static_cast<char*>(d_work));
  const int tiles = scan_tiles(a.n_fine);
  smem_plan_reduce_kernel<<<tiles, kTileThreads, 0, stream>>>(a);
  tile_scan_kernel<<<1, kTileScanThreads, 0, stream>>>(a.t_gc, tiles);
  tile_scan_kernel<<<1, kTileScanThreads, 0, stream>>>(a.t_sp, tiles);
  smem_plan_apply_kernel<<<tiles, kTileThreads, 0, stream>>>(a);
  smem_plan_pack_kernel<<<tiles, kTileThreads, 0, stream>>>(a);
  tile_scan_kernel<<<1, kTileScanThreads, 0, stream>>>(a.t_fl, tiles);
  smem_plan_groups_kernel<<<tiles, kTileThreads, 0, stream>>>(a);
  smem_plan_desc_kernel<<<(a.n_fine + 255) / 256 < dbg_sm_count() * 8 ? (a.n_fine + 255) / 256 : dbg_sm_count() * 8,
                          256, 0, stream>>>(a);
  const OutArgs oa = make_out_args(prm, d_out, out_cap, d_n_out, d_stats, d_status);
  cudaError_t e;
  if (prm->k <= 31) e = launch_smem<uint64_t, 4>(a, oa, stream);
  else if (prm->k <= 39) e = launch_smem<u128, 4>(a, oa, stream);
  else e = launch_smem<u128, 8>(a, oa, stream);
  return e == cudaSuccess ? DBG_OK : DBG_ECUDA;
}

extern "C" dbg_status dbg_checksum_vertices(const dbg_params* prm, const dbg_vertex* d_vertices, uint64_t n,
                                            dbg_stats* d_stats, cudaStream_t stream) {
  if (!dbg_params_ok(prm) || prm->k > 63 || !d_stats || (n && !d_vertices)) return DBG_EINVAL;
  if (n == 0) return DBG_OK;
  const uint64_t want = (n + 255) / 256, cap = (uint64_t)dbg_sm_count() * 8;
  checksum_kernel<<<(int)(want < cap ? want : cap), 256, 0, stream>>>(
      d_vertices, n, reinterpret_cast<unsigned long long*>(d_stats) + 3);
  return cudaPeekAtLastError() == cudaSuccess ? DBG_OK : DBG_ECUDA;
}

static size_t cub_sort_bytes(uint64_t n) {
  size_t bytes = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, bytes, (unsigned long long*)nullptr, (unsigned long long*)nullptr,
                                  (unsigned long long*)nullptr, (unsigned long long*)nullptr, (int64_t)n, 0, 64);
  return bytes;
}

static uint64_t align256(uint64_t x) { return (x + 255) & ~(uint64_t)255; }

extern "C" uint64_t dbg_sort_workspace_bytes(const dbg_params* prm, uint64_t n) {
  (void)prm;
  return 4 * align256(8 * (n ? n : 1)) + align256(cub_sort_bytes(n ? n : 1));
}

extern "C" dbg_status dbg_sort_vertices(const dbg_params* prm, const dbg_vertex* d_in, dbg_vertex* d_out, uint64_t n,
                                        void* d_workspace, uint64_t workspace_bytes, cudaStream_t stream) {
  if (!dbg_params_ok(prm) || prm->k > 63 || (n && (!d_in || !d_out || !d_workspace)) || d_in == d_out)
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
  const int grid = dbg_sm_count() * 4;
  sort_prepare_kernel<<<grid, 256, 0, stream>>>(d_in, n, k0, i0);
  const int k = prm->k;
  const int lo_bits = k <= 31 ? 2 * k : 64;
  if (cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, k0, k1, i0, i1, (int64_t)n, 0, lo_bits, stream) != cudaSuccess)
    return DBG_ECUDA;
  unsigned long long* idx = i1;
  if (k > 31) {  // LSD: then a stable sort by the high word
    sort_gather_hi_kernel<<<grid, 256, 0, stream>>>(d_in, n, i1, k0);
    if (cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, k0, k1, i1, i0, (int64_t)n, 0, 2 * k - 64, stream) !=
        cudaSuccess)
      return DBG_ECUDA;
    idx = i0;
  }
  sort_gather_kernel<<<grid, 256, 0, stream>>>(d_in, n, idx, d_out);
  return cudaPeekAtLastError() == cudaSuccess ? DBG_OK : DBG_ECUDA;
}
