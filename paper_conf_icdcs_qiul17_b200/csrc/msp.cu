// msp.cu -- Step 1 of ParaHash on sm_100a: MSP graph partitioning
// (Sec. III-B; Defs. 1-2), kernel (a) of the north star.
//
// Pass 1 (minimizers, superkmers, partition ids, sizes, staging), two kernels chosen by measured
// speed (profiles/r02_ab.txt):
//  * msp_warp_kernel (msp_warp.cuh): one WARP per read, lanes over P-mer positions -- the
//    warp-parallel sliding minimizer, reads staged in shared memory by TMA bulk copies.  Every
//    (K, P) except the ones below (bumblebee's K = 63, P = 19: 47.5 vs 49.2 ms for a thread per
//    read).
//  * msp_block_kernel: one THREAD per read (32 consecutive reads per warp), van Herk blocks of
//    W = K-P+1 canonical P-mer codes in registers, for K = 31 with P = 11..15 (chr14: 10.8 vs
//    15.6 ms for the warp kernel, whose per-read shuffles, ballots and descriptor ranks cost 5
//    warp instructions per K-mer against 3.2 here).
// Both append superkmer descriptors to shared memory and flush them per warp: pid = fmix64(m)
// mod NP (reading I) via a precomputed 64-bit reciprocal, per-partition sizes N^i_kmer
// (P:L972-975), one staging reservation per warp flush, fixed-width records (dbg.h) with the two
// adjacency bases (Sec. III-B).
//
// The paper computed only "superkmer ids and offsets" on the GPU and left
// the irregular copy to the CPU; here both run in these kernels.
//
// Pass 2, exclusive_scan (scan.cuh): record offsets per partition.
// Pass 3, scatter_kernel: counting-sort scatter of the staged records into
// their partitions' contiguous ranges (CTA histogram -> one global
// reservation per partition per tile).
#include <cub/block/block_scan.cuh>

#include <algorithm>
#include <type_traits>
#include <cstdlib>

#include "dbg_device.cuh"
#include "scan.cuh"

namespace dbg {

constexpr int kMspThreads = 128;
// msp_block_kernel variants (A/B builds, tools/build_variants.py)
// descriptors per thread between flushes of the register-blocked kernel (>= W + 3; a register cap
// for 6-7 CTAs/SM with 28-32 descriptors was no faster on chr14, profiles/r02_ab.txt)
constexpr int kMaxDescBlock = 40;
constexpr int kSmemHistMaxNp = 8192;

struct MspArgs {
  const uint64_t* words;
  uint64_t n_words;
  const uint64_t* offsets;
  uint64_t n_reads;
  int k, p, np, w;
  uint32_t rec_words, max_kmers;
  FastMod mod;
  unsigned long long* n_records;  // [np]
  unsigned long long* n_kmers;    // [np]
  uint32_t* staging;              // records in read order
  uint64_t staging_cap;           // records
  unsigned long long* staged;     // cursor (records reserved)
  uint32_t pid_lo, pid_hi;        // only superkmers of fine partitions [pid_lo, pid_hi) are counted and staged
  bool ranged;                    // pid_lo > 0 or pid_hi < np
};

template <typename CT>
struct MspSmem {
  // desc_e[d * kMspThreads + tid]: last K-mer of descriptor d (its first is the previous
  // descriptor's last + 1, or the carried start); desc_m: its minimizer
  uint32_t* desc_e;
  CT* desc_m;
};

// Writes one record (dbg.h layout) for K-mers [ps, pe] of the read at stream
// offset o, length L.
__device__ __forceinline__ void write_record(const MspArgs& a, uint32_t* dst, uint64_t o, int L, int ps, int pe,
                                             uint32_t pid) {
  const uint32_t hl = ps > 0 ? 1u : 0u;  // reading H
  const uint32_t hr = pe + a.k < L ? 1u : 0u;
  const int bs = ps - (int)hl;
  const int nb = (int)hl + (pe - ps + 1) + a.k - 1 + (int)hr;
  uint4* d4 = reinterpret_cast<uint4*>(dst);
  // 16-byte chunks of the record: word 0 = header, then 16 bases per word, two words per
  // 64-bit window of the stream (rec_words = 4, 8 or 16)
  for (int c = 0; c < (int)a.rec_words / 4; ++c) {
    uint32_t w[4];
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int q = 4 * c + 2 * h;  // record word q and q+1 hold data words q-1 and q ...
      // ... i.e. bases 16(q-1) .. 16(q+1)-1; word 0 is the header
      uint64_t v = 0;
      const int first = 16 * (q - 1);
      if (q == 0) {
        const int left = nb;
        if (left > 0) {
          v = window64(a.words, a.n_words, o + bs);
          if (left < 32) v &= ~(~0ull >> (2 * left));
        }
        w[0] = rec_header((uint32_t)(pe - ps + 1), hl, hr, pid);
        w[1] = (uint32_t)(v >> 32);  // bases 0..15
        continue;
      }
      const int left = nb - first;
      if (left > 0) {
        v = window64(a.words, a.n_words, o + bs + first);
        if (left < 32) v &= ~(~0ull >> (2 * left));  // zero the bases past the record
      }
      w[2 * h] = (uint32_t)(v >> 32);
      w[2 * h + 1] = (uint32_t)v;
    }
    d4[c] = make_uint4(w[0], w[1], w[2], w[3]);
  }
}

// 32-bit shared-window accesses for the per-base loop (keeps generic-pointer
// arithmetic and the shared-window base out of it).
__device__ __forceinline__ uint32_t sh_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void sh_st(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void sh_st(uint32_t a, uint64_t v) {
  asm volatile("st.shared.u64 [%0], %1;" ::"r"(a), "l"(v) : "memory");
}

// Records of a superkmer of n K-mers (pieces of at most nmax K-mers); the
// common case n <= nmax needs no division.
__device__ __forceinline__ uint32_t record_pieces(int n, int nmax) {
  return n <= nmax ? 1u : (uint32_t)((n + nmax - 1) / nmax);
}

// Writes one record for K-mers [ps, pe] of the read at stream offset o, length
// L, when it has 4 words (K <= 39): header + bases bs .. bs + 47, taken from
// the three stream words that hold them (one bounds check each).
__device__ __forceinline__ void write_record4(const MspArgs& a, uint32_t* dst, uint64_t o, int L, int ps, int pe,
                                              uint32_t pid) {
  const uint32_t hl = ps > 0 ? 1u : 0u;  // reading H
  const uint32_t hr = pe + a.k < L ? 1u : 0u;
  const int nb = (int)hl + (pe - ps + 1) + a.k - 1 + (int)hr;  // <= 48
  const uint64_t pos = o + (uint64_t)(ps - (int)hl);
  const uint64_t wi = pos >> 5;
  const uint32_t sh = (uint32_t)(pos & 31) * 2;
  const uint64_t x0 = wi < a.n_words ? __ldg(a.words + wi) : 0, x1 = wi + 1 < a.n_words ? __ldg(a.words + wi + 1) : 0;
  const uint64_t x2 = sh > 32 && wi + 2 < a.n_words ? __ldg(a.words + wi + 2) : 0;
  // bases 0..31 and 32..47 of the record (before masking)
  const uint64_t v0 = sh ? (x0 << sh) | (x1 >> (64 - sh)) : x0;
  const uint64_t v1 = sh ? (x1 << sh) | (x2 >> (64 - sh)) : x1;
  const uint64_t m0 = nb >= 32 ? ~0ull : ~(~0ull >> (2 * nb));
  const uint32_t m1 = nb >= 48 ? ~0u : (nb <= 32 ? 0u : ~(~0u >> (2 * (nb - 32))));
  const uint64_t b0 = v0 & m0;
  const uint32_t b1 = (uint32_t)(v1 >> 32) & m1;
  const uint4 rec = make_uint4(rec_header((uint32_t)(pe - ps + 1), hl, hr, pid), (uint32_t)(b0 >> 32),
                               (uint32_t)b0, b1);
  reinterpret_cast<uint4*>(dst)[0] = rec;
}

// Warp-collective flush of the per-thread descriptor lists: partition ids
// (computed once per descriptor and kept in place of the minimizer), size
// histograms, one staging reservation per warp, record writes.
// kK > 0: compile-time K (record geometry and pieces without runtime division).
template <typename CT, int kK = 0>
__device__ __forceinline__ void flush_descriptors(const MspArgs& a, const MspSmem<CT>& sm, int& ndesc,
                                                  int& s_next, uint64_t o, int L) {
  const int tid = threadIdx.x, lane = tid & 31;
  const int nmax = kK > 0 ? (int)record_max_kmers(kK) : (int)a.max_kmers;
  const bool r4 = kK > 0 ? record_words(kK) == 4 : a.rec_words == 4;
  constexpr CT kSkip = ~(CT)0;  // a superkmer of another pass's partition (row f2)
  uint32_t my_records = 0;
  {
    int s = s_next;
    for (int d = 0; d < ndesc; ++d) {
      const int e = (int)sm.desc_e[d * kMspThreads + tid];
      CT& dm = sm.desc_m[d * kMspThreads + tid];
      const uint32_t pid0 = a.np == 1 ? 0u : fast_mod(a.mod, fmix64((uint64_t)dm));
      const bool in = !a.ranged || (pid0 - a.pid_lo < a.pid_hi - a.pid_lo);
      dm = in ? (CT)pid0 : kSkip;
      if (in) {
        // the per-partition sizes here, so that the record loop below has no atomics between
        // its loads and stores (the loads of consecutive records overlap)
        const uint32_t pid = (uint32_t)dm, pieces = record_pieces(e - s + 1, nmax);
        my_records += pieces;
        atomicAdd(a.n_records + pid, (unsigned long long)pieces);
        atomicAdd(a.n_kmers + pid, (unsigned long long)(e - s + 1));
      }
      s = e + 1;
    }
  }
  uint32_t incl = my_records;
#pragma unroll
  for (int dlt = 1; dlt < 32; dlt <<= 1) {
    const uint32_t v = __shfl_up_sync(kFull, incl, dlt);
    if (lane >= dlt) incl += v;
  }
  const uint32_t total = __shfl_sync(kFull, incl, 31);
  unsigned long long base = 0;
  if (total) {
    if (lane == 0) base = atomicAdd(a.staged, (unsigned long long)total);
    base = __shfl_sync(kFull, base, 0);
  }
  uint64_t slot = base + incl - my_records;
  int s = s_next;
  for (int d = 0; d < ndesc; ++d) {
    const int e = (int)sm.desc_e[d * kMspThreads + tid];
    const CT dm = sm.desc_m[d * kMspThreads + tid];
    if (dm == kSkip) {
      s = e + 1;
      continue;
    }
    const uint32_t pid = (uint32_t)dm;
    for (int ps = s; ps <= e; ps += nmax, ++slot) {
      if (slot < a.staging_cap) {
        if (r4)
          write_record4(a, a.staging + slot * 4, o, L, ps, min(e, ps + nmax - 1), pid);
        else
          write_record(a, a.staging + slot * a.rec_words, o, L, ps, min(e, ps + nmax - 1), pid);
      }
    }
    s = e + 1;
  }
  s_next = s;
  ndesc = 0;
}

// Pass 3 (one level): scatter staged records into partition order, record of partition pid at
// rec_off[pid] + rank.  With nb <= kSmemHistMaxNp partitions a CTA tile ranks its records in
// shared memory and reserves once per partition, else one global atomic per record.
// L2 cache policies of the scatter: the staged records stream through once (evict first); the
// partitions' open sectors, their cursors and offsets stay (evict last), so a 32-byte sector
// that receives a 16-byte record is still in L2 when its other half arrives and is written back
// whole -- without it every record store costs a DRAM read-modify-write of its sector.
__device__ __forceinline__ uint64_t l2_policy_last() {
  uint64_t p;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t l2_policy_first() {
  uint64_t p;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint4 ld_stream16(const uint4* p, uint64_t pol) {
  uint4 v;
  asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v4.u32 {%0, %1, %2, %3}, [%4], %5;"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ void st_keep16(uint4* p, uint4 v, uint64_t pol) {
  asm volatile("st.global.L2::cache_hint.v4.u32 [%0], {%1, %2, %3, %4}, %5;"
               :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "l"(pol) : "memory");
}
__device__ __forceinline__ uint64_t ld_keep8(const uint64_t* p, uint64_t pol) {
  uint64_t v;
  asm volatile("ld.global.nc.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ unsigned long long atom_add_keep(unsigned long long* p, unsigned long long v,
                                                            uint64_t pol) {
  unsigned long long r;
  asm volatile("atom.global.add.L2::cache_hint.u64 %0, [%1], %2, %3;" : "=l"(r) : "l"(p), "l"(v), "l"(pol)
               : "memory");
  return r;
}

constexpr int kScatterThreads = 256;
constexpr int kScatterPer = 4;  // records per thread per tile
template <int R>
__global__ void __launch_bounds__(kScatterThreads, 4) scatter_kernel(const uint32_t* __restrict__ staging,
                                                                  const unsigned long long* staged,
                                                                  uint64_t staging_cap,
                                                                  const uint64_t* __restrict__ rec_off,
                                                                  unsigned long long* fill,
                                                                  uint32_t* __restrict__ records, int nb,
                                                                  uint32_t* const* peer_records,
                                                                  const int32_t* peer_bounds, int n_peers) {
  extern __shared__ unsigned long long sh_base[];  // [nb] global bases (per tile), then [nb] counts
  uint32_t* sh_cnt = reinterpret_cast<uint32_t*>(sh_base + nb);
  const uint64_t n = *staged;
  if (n > staging_cap) return;  // pass 1 overflowed the staging: the caller repeats it (dbg.h)
  const bool smem = nb <= kSmemHistMaxNp;
  const uint64_t pol_first = l2_policy_first(), pol_last = l2_policy_last();
  constexpr int kPer = R >= 16 ? 2 : kScatterPer;
  constexpr int kTile = kScatterThreads * kPer;
  for (uint64_t t0 = (uint64_t)blockIdx.x * kTile; t0 < n; t0 += (uint64_t)gridDim.x * kTile) {
    if (smem) {
      for (int i = threadIdx.x; i < nb; i += kScatterThreads) sh_cnt[i] = 0;
      __syncthreads();
    }
    uint4 rec[kPer][R / 4];
    uint32_t rank[kPer];
    // all loads of the tile first, then all rank atomics, then all stores: kPer records of
    // each thread in flight at every stage (the kernel is latency-bound)
#pragma unroll
    for (int v = 0; v < kPer; ++v) {
      const uint64_t idx = t0 + v * kScatterThreads + threadIdx.x;
      if (idx < n) {
        const uint4* src = reinterpret_cast<const uint4*>(staging + idx * R);
#pragma unroll
        for (int c = 0; c < R / 4; ++c) rec[v][c] = ld_stream16(src + c, pol_first);
      }
    }
#pragma unroll
    for (int v = 0; v < kPer; ++v) {
      const uint64_t idx = t0 + v * kScatterThreads + threadIdx.x;
      rank[v] = 0;
      if (idx < n) {
        const uint32_t bin = hdr_pid(rec[v][0].x);
        if (smem) rank[v] = atomicAdd(sh_cnt + bin, 1u);
        else rank[v] = (uint32_t)atom_add_keep(fill + bin, 1ull, pol_last);
      }
    }
    uint64_t base[kPer];
#pragma unroll
    for (int v = 0; v < kPer; ++v) {
      const uint64_t idx = t0 + v * kScatterThreads + threadIdx.x;
      const uint64_t* op = rec_off + hdr_pid(rec[v][0].x);
      base[v] = idx < n ? ld_keep8(op, pol_last) : 0;
    }
    if (smem) {
      __syncthreads();
      for (int i = threadIdx.x; i < nb; i += kScatterThreads)
        if (sh_cnt[i]) sh_base[i] = atomicAdd(fill + i, (unsigned long long)sh_cnt[i]);
      __syncthreads();
    }
#pragma unroll
    for (int v = 0; v < kPer; ++v) {
      const uint64_t idx = t0 + v * kScatterThreads + threadIdx.x;
      if (idx < n) {
        const uint32_t bin = hdr_pid(rec[v][0].x);
        const uint64_t pos = base[v] + (smem ? sh_base[bin] + rank[v] : rank[v]);
        uint32_t* out = records;
        if (n_peers) {  // multi-GPU emission: the owner's buffer, through its IPC-mapped pointer
          const int32_t pid = (int32_t)hdr_pid(rec[v][0].x);
          int o = 0;
          while (o + 1 < n_peers && pid >= __ldg(peer_bounds + o + 1)) ++o;
          out = peer_records[o];
        }
        uint4* dst = reinterpret_cast<uint4*>(out + pos * R);
#pragma unroll
        for (int c = 0; c < R / 4; ++c) st_keep16(dst + c, rec[v][c], pol_last);
      }
    }
    if (smem) __syncthreads();
  }
}

// Two-level scatter (pass 3 with d_scratch): two counting-sort passes over tiles of records.
// Level A ranks a tile of staged records by BUCKET (2^s consecutive fine partitions, <= 2048
// buckets) in shared memory, reserves once per (tile, non-empty bucket) from a global bucket
// cursor and writes the tile into the buckets' contiguous ranges of d_scratch (bucket b starts at
// the local prefix of this rank's counts).  Level B takes tiles inside one bucket, ranks them by
// partition in shared memory, reserves once per (tile, partition) from d_fill and writes each
// record to d_record_offset[pid] + rank -- in d_records or the owner's buffer.  A record costs a
// shared-memory atomic per level and ~0.1-0.4 global atomics, instead of one returning global
// atomic in a dependent chain (the one-level scatter above, latency-bound at ~36 G records/s).
constexpr int kTsThreads = 1024;
constexpr int kTsMaxBins = 4096;  // bins of one tile pass (buckets in level A, partitions in level B)
template <int R>
__host__ __device__ constexpr int ts_per() { return R == 4 ? 8 : (R == 8 ? 4 : 1); }
template <int R>
__host__ __device__ constexpr int ts_tile() { return kTsThreads * ts_per<R>(); }  // <= 128 KB of records
// log2 of the bucket width: the smallest s with <= 2048 buckets, at most 12 (4096 partitions a
// bucket; <= 4096 buckets for the 2^24 - 1 fine partitions of dbg.h)
__host__ __device__ inline int ts_shift(int np) {  // (r02z6: 1024 / 4096 buckets: mixed / slower)
  int s = 0;
  while (s < 12 && ((np + (1 << s) - 1) >> s) > 2048) ++s;
  return s;
}
// d_work layout (uint64): fill[nb] | boff[nb + 1] | tiles[nb + 1]
struct TsArgs {
  const uint32_t* src;
  uint32_t* dst;
  const unsigned long long* staged;
  uint64_t staging_cap;
  unsigned long long* fill;  // level A: bucket cursors (work); level B: partition cursors (d_fill)
  const uint64_t* boff;      // [nb + 1] local bucket offsets
  const uint64_t* tiles;     // [nb + 1] level B tiles before bucket b
  const uint64_t* rec_off;   // level B: d_record_offset (or the exchange plan's destinations)
  int nb, s, np;
  uint32_t* const* peer_records;
  const int32_t* peer_bounds;
  int n_peers;
};

// Per bucket: this rank's records in it (sum of d_n_records over its partitions).
__global__ void __launch_bounds__(256) ts_bucket_count_kernel(const uint64_t* __restrict__ n_records, int np, int s,
                                                             uint64_t* __restrict__ boff) {
  typedef cub::BlockReduce<unsigned long long, 256> Red;
  __shared__ typename Red::TempStorage tmp;
  const int b = blockIdx.x, f0 = b << s, f1 = min(np, (b + 1) << s);
  unsigned long long c = 0;
  for (int f = f0 + threadIdx.x; f < f1; f += 256) c += n_records[f];
  c = Red(tmp).Sum(c);
  if (threadIdx.x == 0) boff[b] = c;
}

// boff: counts -> exclusive prefix (boff[nb] = total); tiles: exclusive prefix of ceil(count / tile);
// fill = 0.  One CTA, nb <= 4096.
__global__ void __launch_bounds__(1024) ts_bucket_scan_kernel(uint64_t* work, int nb, int tile) {
  typedef cub::BlockScan<unsigned long long, 1024> Scan;
  __shared__ typename Scan::TempStorage tmp;
  unsigned long long* fill = reinterpret_cast<unsigned long long*>(work);
  uint64_t* boff = work + nb;
  uint64_t* tiles = boff + nb + 1;
  unsigned long long c[4], t[4];
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const int i = 4 * threadIdx.x + q;
    c[q] = i < nb ? boff[i] : 0ull;
    t[q] = (c[q] + tile - 1) / tile;
    if (i < nb) fill[i] = 0;
  }
  unsigned long long ct, tt;
  Scan(tmp).ExclusiveSum(c, c, ct);
  __syncthreads();
  Scan(tmp).ExclusiveSum(t, t, tt);
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const int i = 4 * threadIdx.x + q;
    if (i < nb) {
      boff[i] = c[q];
      tiles[i] = t[q];
    }
  }
  if (threadIdx.x == 0) {
    boff[nb] = ct;
    tiles[nb] = tt;
  }
}

// One tile [r0, r1) of a.src (a counting sort of the tile, onesweep-style): records ranked by bin
// in shared memory, the tile's bin counts scanned (local offsets) and reserved once per non-empty
// bin (base_of(bin, count)), the records placed in bin order in shared memory, then written out
// by consecutive threads to consecutive slots of each bin's global range -- coalesced stores of
// whole 32-byte sectors instead of one scattered 16-byte store per record.
template <int R, class BinFn, class BaseFn, class DstFn>
__device__ __forceinline__ void ts_tile_pass(const TsArgs& a, uint64_t r0, uint64_t r1, int nbins, uint32_t* srec,
                                             unsigned long long* gbase, uint32_t* hist, uint32_t* lbase,
                                             BinFn bin_of, BaseFn base_of, DstFn dst_of, uint64_t pol_first) {
  constexpr int kPer = ts_per<R>(), kItems = kTsMaxBins / kTsThreads;
  typedef cub::BlockScan<uint32_t, kTsThreads> Scan;
  __shared__ typename Scan::TempStorage scan_tmp;
  for (int i = threadIdx.x; i < nbins; i += kTsThreads) hist[i] = 0;
  __syncthreads();
  uint4 rec[kPer][R / 4];
  uint32_t bin[kPer], rank[kPer];
#pragma unroll
  for (int v = 0; v < kPer; ++v) {
    const uint64_t idx = r0 + (uint64_t)v * kTsThreads + threadIdx.x;
    if (idx < r1) {
      const uint4* s4 = reinterpret_cast<const uint4*>(a.src + idx * R);
#pragma unroll
      for (int c = 0; c < R / 4; ++c) rec[v][c] = ld_stream16(s4 + c, pol_first);
    }
  }
#pragma unroll
  for (int v = 0; v < kPer; ++v) {
    const uint64_t idx = r0 + (uint64_t)v * kTsThreads + threadIdx.x;
    if (idx < r1) {
      bin[v] = bin_of(hdr_pid(rec[v][0].x));
      rank[v] = atomicAdd(hist + bin[v], 1u);
    }
  }
  __syncthreads();
  {
    uint32_t c[kItems], ex[kItems];
#pragma unroll
    for (int q = 0; q < kItems; ++q) {
      const int i = kItems * threadIdx.x + q;
      c[q] = i < nbins ? hist[i] : 0u;
    }
    Scan(scan_tmp).ExclusiveSum(c, ex);
#pragma unroll
    for (int q = 0; q < kItems; ++q) {
      const int i = kItems * threadIdx.x + q;
      if (i < nbins) {
        lbase[i] = ex[q];
        if (c[q]) gbase[i] = base_of(i, c[q]);
      }
    }
  }
  __syncthreads();
#pragma unroll
  for (int v = 0; v < kPer; ++v) {
    const uint64_t idx = r0 + (uint64_t)v * kTsThreads + threadIdx.x;
    if (idx < r1) {
      uint4* d4 = reinterpret_cast<uint4*>(srec + (size_t)(lbase[bin[v]] + rank[v]) * R);
#pragma unroll
      for (int c = 0; c < R / 4; ++c) d4[c] = rec[v][c];
    }
  }
  __syncthreads();
  const uint32_t nt = (uint32_t)(r1 - r0);
  for (uint32_t p = threadIdx.x; p < nt; p += kTsThreads) {
    const uint4* sp = reinterpret_cast<const uint4*>(srec + (size_t)p * R);
    const uint4 x0 = sp[0];
    const uint32_t pid = hdr_pid(x0.x), b = bin_of(pid);
    uint4* d4 = reinterpret_cast<uint4*>(dst_of(pid) + (gbase[b] + (p - lbase[b])) * R);
    d4[0] = x0;
#pragma unroll
    for (int c = 1; c < R / 4; ++c) d4[c] = sp[c];
  }
  __syncthreads();
}

// Dynamic shared memory of a tile pass: records, then the bases and the counts (overwritten in
// place by their local offsets) of nbins.
template <int R>
__host__ __device__ constexpr size_t ts_rec_bytes() { return (size_t)ts_tile<R>() * R * 4; }
inline size_t ts_bin_bytes(int nbins) { return (size_t)nbins * (8 + 4); }

template <int R>
__global__ void __launch_bounds__(kTsThreads) ts_level_a_kernel(TsArgs a) {
  extern __shared__ __align__(16) unsigned char ts_smem[];
  uint32_t* srec = reinterpret_cast<uint32_t*>(ts_smem);
  unsigned long long* gbase = reinterpret_cast<unsigned long long*>(ts_smem + ts_rec_bytes<R>());
  uint32_t* hist = reinterpret_cast<uint32_t*>(gbase + a.nb);
  uint32_t* lbase = hist;  // each thread reads its counts before writing their offsets
  const uint64_t n = *a.staged;
  if (n > a.staging_cap) return;  // pass 1 overflowed the staging: the caller repeats it (dbg.h)
  constexpr int kTile = ts_tile<R>();
  const int s = a.s;
  auto bin_of = [s](uint32_t pid) { return pid >> s; };
  auto base_of = [&](int b, uint32_t c) { return a.boff[b] + atomicAdd(a.fill + b, (unsigned long long)c); };
  auto dst_of = [&](uint32_t) { return a.dst; };
  const uint64_t pol_first = l2_policy_first();
  for (uint64_t t0 = (uint64_t)blockIdx.x * kTile; t0 < n; t0 += (uint64_t)gridDim.x * kTile)
    ts_tile_pass<R>(a, t0, min(n, t0 + kTile), a.nb, srec, gbase, hist, lbase, bin_of, base_of, dst_of, pol_first);
}

template <int R>
__global__ void __launch_bounds__(kTsThreads) ts_level_b_kernel(TsArgs a) {
  extern __shared__ __align__(16) unsigned char ts_smem[];
  const int w = 1 << a.s;
  uint32_t* srec = reinterpret_cast<uint32_t*>(ts_smem);
  unsigned long long* gbase = reinterpret_cast<unsigned long long*>(ts_smem + ts_rec_bytes<R>());
  unsigned long long* tiles = gbase + w;  // [nb + 1] tile prefix
  uint32_t* hist = reinterpret_cast<uint32_t*>(tiles + a.nb + 1);
  uint32_t* lbase = hist;  // each thread reads its counts before writing their offsets
  if (*a.staged > a.staging_cap) return;
  for (int i = threadIdx.x; i <= a.nb; i += kTsThreads) tiles[i] = a.tiles[i];
  const uint64_t pol_first = l2_policy_first();
  __syncthreads();
  constexpr int kTile = ts_tile<R>();
  const uint64_t n_tiles = tiles[a.nb];
  for (uint64_t g = blockIdx.x; g < n_tiles; g += gridDim.x) {
    int b = 0, cnt = a.nb;  // the bucket of tile g: last b with tiles[b] <= g (shared-memory search)
    while (cnt > 1) {
      const int h = cnt >> 1;
      if (tiles[b + h] <= g) b += h, cnt -= h;
      else cnt = h;
    }
    const uint32_t f0 = (uint32_t)b << a.s;
    const uint64_t r0 = a.boff[b] + (g - tiles[b]) * kTile, r1 = min(a.boff[b + 1], r0 + kTile);
    const int nbins = min(w, a.np - (int)f0);
    auto bin_of = [f0](uint32_t pid) { return pid - f0; };
    auto base_of = [&](int i, uint32_t c) {
      return a.rec_off[f0 + i] + atomicAdd(a.fill + f0 + i, (unsigned long long)c);
    };
    auto dst_of = [&](uint32_t pid) -> uint32_t* {
      if (!a.n_peers) return a.dst;  // multi-GPU emission: the owner's buffer, through its IPC pointer
      int o = 0;
      while (o + 1 < a.n_peers && (int32_t)pid >= __ldg(a.peer_bounds + o + 1)) ++o;
      return a.peer_records[o];
    };
    ts_tile_pass<R>(a, r0, r1, nbins, srec, gbase, hist, lbase, bin_of, base_of, dst_of, pol_first);
  }
}

// Register-blocked variant for compile-time W = K - P + 1 and P <= 16 (the
// configurations' K = 31 with P = 11..15): the van Herk blocks of W P-mer
// values live in registers (fully unrolled), so the per-base work is the
// rolling P-mer, one prefix minimum and, per block, the suffix minima --
// no shared-memory row.  K-mer i's minimizer (Def. 1) is
// min(suffix_min_prev[t], prefix_min_cur[t-1]) for i = q0 - W + t, where the
// current block holds P-mers q0 .. q0+W-1.  Same descriptors and flush as
// the warp kernel; reads of any length (lanes past their read end run masked).
// P-mer codes of the register-blocked kernel: 32-bit up to P = 16, else 64-bit (K = 63, P = 19);
// descriptor lists hold at least W + 3 entries (a block of W bases closes at most W superkmers,
// plus the read's last one and the carry).
template <int W, int P>
struct MspBlockCfg {
  typedef std::conditional_t<(P <= 16), uint32_t, uint64_t> CT;
  static constexpr int kDesc = W + 3 > kMaxDescBlock ? W + 3 : kMaxDescBlock;
  static constexpr size_t smem() { return (sizeof(CT) + sizeof(uint32_t)) * kDesc * kMspThreads; }
};

template <int W, int P>
__global__ void __launch_bounds__(kMspThreads, 1) msp_block_kernel(MspArgs a) {
  typedef typename MspBlockCfg<W, P>::CT CT;
  constexpr int kDesc = MspBlockCfg<W, P>::kDesc;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int tid = threadIdx.x, lane = tid & 31;
  MspSmem<CT> sm;
  unsigned char* sp = smem_raw;
  sm.desc_m = reinterpret_cast<CT*>(sp);
  sp += sizeof(CT) * kDesc * kMspThreads;
  sm.desc_e = reinterpret_cast<uint32_t*>(sp);
  constexpr CT kMaskP = (CT)((2 * P == 8 * (int)sizeof(CT)) ? ~(CT)0 : (((CT)1 << (2 * P)) - 1));
  constexpr CT kInf = ~(CT)0;
  constexpr int kTopP = 2 * P - 2;
  constexpr int K = W + P - 1;
  const uint32_t de_a = sh_addr(sm.desc_e + tid), dm_a = sh_addr(sm.desc_m + tid);
  constexpr uint32_t kDescStep = kMspThreads * 4, kDescStepM = kMspThreads * sizeof(CT);
  const uint64_t stride = (uint64_t)gridDim.x * kMspThreads;
  for (uint64_t r0 = (uint64_t)blockIdx.x * kMspThreads + (tid & ~31); r0 < a.n_reads; r0 += stride) {
    const uint64_t r = r0 + lane;
    uint64_t o = 0;
    int L = 0;
    if (r < a.n_reads) {
      o = a.offsets[r];
      L = (int)(a.offsets[r + 1] - o);
    }
    const int nk = L - K + 1;
    if (nk <= 0) L = 0;  // reading N: no K-mers
    const int nP = L > 0 ? L - P + 1 : 0;  // P-mers of the read
    int nPmax = nP;
#pragma unroll
    for (int dlt = 16; dlt; dlt >>= 1) nPmax = max(nPmax, __shfl_xor_sync(kFull, nPmax, dlt));
    int ndesc = 0, s_next = 0;
    CT f = 0, rc = 0, m_cur = 0;
    // the bases: a 64-bit window of the stream at base j, reloaded before a run of
    // bases that could exhaust it (one reload per block, no per-base check)
    int j = 0, nbuf = 0;
    uint64_t wbuf = 0;
    auto refill = [&](int need) {
      if (nbuf < need) {
        wbuf = j < L ? window64(a.words, a.n_words, o + j) : 0;
        nbuf = 32;
      }
    };
    auto next_base = [&]() -> uint32_t {
      const uint32_t b = (uint32_t)(wbuf >> 62);
      wbuf <<= 2;
      --nbuf;
      ++j;
      return b;
    };
    refill(P - 1);
#pragma unroll
    for (int t = 0; t < P - 1; ++t) {  // the first P-1 bases: no P-mer yet
      const uint32_t b = next_base();
      f = ((f << 2) | b) & kMaskP;
      rc = (rc >> 2) | ((CT)(3u - b) << kTopP);
    }
    CT suf[W];  // suffix minima of the previous block
#pragma unroll
    for (int t = 0; t < W; ++t) suf[t] = kInf;
    // blocks of W P-mers; one extra block of padding emits the last K-mers.  K-mer
    // i = q0 - W + t is complete once P-mer q0 + t - 1 is read: its minimizer is
    // min(suf[t], prefix minimum of the current block's first t values) -- the
    // prefix is a running scalar, the block's values are kept for its suffix minima.
    for (int q0 = 0; q0 < nPmax + W; q0 += W) {
      CT c[W], pre[W];
      refill(W < 32 ? W : 32);  // a 64-bit window holds 32 bases: W > 32 reloads once more
#pragma unroll
      for (int t = 0; t < W; ++t) {
        CT v = kInf;
        if (t > 0 && t % 32 == 0) refill(W - t < 32 ? W - t : 32);
        if (q0 + t < nP) {
          const uint32_t b = next_base();
          f = ((f << 2) | b) & kMaskP;
          rc = (rc >> 2) | ((CT)(3u - b) << kTopP);
          v = f < rc ? f : rc;  // canonical P-mer (reading D)
        }
        c[t] = v;
        pre[t] = t == 0 ? v : (v < pre[t - 1] ? v : pre[t - 1]);
      }
      if (q0 >= W) {  // K-mers i = q0 - W + t of the previous block's windows
#pragma unroll
        for (int t = 0; t < W; ++t) {
          const int i = q0 - W + t;
          if (i < nk) {
            const CT m = t == 0 ? suf[0] : (suf[t] < pre[t - 1] ? suf[t] : pre[t - 1]);
            if (i > 0 && m != m_cur) {  // a superkmer ends at K-mer i-1 (Def. 2)
              sh_st(de_a + (uint32_t)ndesc * kDescStep, (uint32_t)(i - 1));
              sh_st(dm_a + (uint32_t)ndesc * kDescStepM, m_cur);
              ++ndesc;
            }
            m_cur = m;
            if (i == nk - 1) {  // the read's last superkmer
              sh_st(de_a + (uint32_t)ndesc * kDescStep, (uint32_t)i);
              sh_st(dm_a + (uint32_t)ndesc * kDescStepM, m_cur);
              ++ndesc;
            }
          }
        }
      }
      suf[W - 1] = c[W - 1];
#pragma unroll
      for (int t = W - 2; t >= 0; --t) suf[t] = c[t] < suf[t + 1] ? c[t] : suf[t + 1];
      // one flush site (the code is inlined once): lists nearly full, or the reads' end
      const bool last = q0 + W >= nPmax + W;
      if (__any_sync(kFull, ndesc > kDesc - W - 2 || (last && ndesc > 0)))
        flush_descriptors<CT, K>(a, sm, ndesc, s_next, o, L);
    }
  }
}

}  // namespace dbg

int dbg_sm_count();
#include "msp_warp.cuh"

using namespace dbg;

int dbg_sm_count() {
  int dev = 0, n = 148;
  if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
  return n;
}

bool dbg_params_ok(const dbg_params* prm) {
  // K <= 127 (row f3); K > 63 keeps the device partitioning on P (no fine_p, reading V)
  if (prm && prm->k > 63 && prm->fine_p != 0 && prm->fine_p != prm->p) return false;
  return prm && prm->k >= 1 && prm->k <= 127 && (prm->k & 1) && prm->p >= 1 && prm->p <= prm->k &&
         prm->p <= 31 && prm->fine_p >= 0 && prm->fine_p <= prm->k && prm->fine_p <= 31 &&
         prm->num_partitions >= 1 && prm->refine >= 0 &&
         (uint64_t)prm->num_partitions * (uint64_t)(prm->refine > 1 ? prm->refine : 1) <= kMaxPid;
}

// Grid of the grid-stride MSP kernels: at most one wave of resident CTAs (a partial second
// wave would start its reads only when first-wave CTAs finish theirs).
static int msp_grid(const void* fn, int want, size_t smem) {
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kMspThreads, smem) != cudaSuccess ||
      per_sm < 1)
    per_sm = 8;
  const int cap = dbg_sm_count() * per_sm;
  return want < cap ? want : cap;
}

template <int W, int P>
static cudaError_t launch_msp_block(const MspArgs& a, int grid, cudaStream_t stream) {
  const size_t smem = MspBlockCfg<W, P>::smem();
  cudaError_t e = cudaFuncSetAttribute(msp_block_kernel<W, P>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  grid = msp_grid((const void*)msp_block_kernel<W, P>, grid, smem);
  msp_block_kernel<W, P><<<grid, kMspThreads, smem, stream>>>(a);
  return cudaGetLastError();
}

// The register-blocked kernel for the configurations' K = 31 (P = 11..15), else the generic one
// (for K = 63, P = 19 the 64-bit blocks of W = 45 need 255 registers and spill: measured 1.5x
// slower than the generic kernel, profiles/r02e).
static bool msp_block_launch(const MspArgs& a, int grid, cudaStream_t stream, cudaError_t* e) {
  if (a.k != 31) return false;
  switch (a.p) {
    case 11: *e = launch_msp_block<21, 11>(a, grid, stream); return true;
    case 12: *e = launch_msp_block<20, 12>(a, grid, stream); return true;
    case 13: *e = launch_msp_block<19, 13>(a, grid, stream); return true;
    case 14: *e = launch_msp_block<18, 14>(a, grid, stream); return true;
    case 15: *e = launch_msp_block<17, 15>(a, grid, stream); return true;
  }
  return false;
}

static dbg_status msp_partition(const dbg_params* prm, const uint64_t* d_bases, uint64_t n_words,
                                const uint64_t* d_offsets, uint64_t n_reads, const dbg_partition_set* part,
                                int32_t pid_lo, int32_t pid_hi, int append, cudaStream_t stream);

extern "C" dbg_status dbg_msp_partition(const dbg_params* prm, const uint64_t* d_bases,
                                        uint64_t n_words, const uint64_t* d_offsets,
                                        uint64_t n_reads, const dbg_partition_set* part,
                                        cudaStream_t stream) {
  if (!dbg_params_ok(prm)) return DBG_EINVAL;
  return msp_partition(prm, d_bases, n_words, d_offsets, n_reads, part, 0, fine_partitions(prm), 0, stream);
}

extern "C" dbg_status dbg_msp_partition_range(const dbg_params* prm, const uint64_t* d_bases, uint64_t n_words,
                                              const uint64_t* d_offsets, uint64_t n_reads,
                                              const dbg_partition_set* part, int32_t pid_lo, int32_t pid_hi,
                                              int append, cudaStream_t stream) {
  if (!dbg_params_ok(prm) || !part || part->d_records) return DBG_EINVAL;
  return msp_partition(prm, d_bases, n_words, d_offsets, n_reads, part, pid_lo, pid_hi, append, stream);
}

static dbg_status msp_partition(const dbg_params* prm, const uint64_t* d_bases, uint64_t n_words,
                                const uint64_t* d_offsets, uint64_t n_reads, const dbg_partition_set* part,
                                int32_t pid_lo, int32_t pid_hi, int append, cudaStream_t stream) {
  if (!dbg_params_ok(prm) || !part || !d_offsets || !part->d_record_offset || !part->d_n_records ||
      !part->d_n_kmers || !part->d_staged)
    return DBG_EINVAL;
  if (n_reads && (!d_bases || !n_words)) return DBG_EINVAL;
  const int np = fine_partitions(prm);
  const uint32_t R = record_words(prm->k);
  if (pid_lo < 0 || pid_hi > np || pid_lo >= pid_hi) return DBG_EINVAL;
  if (part->d_records == nullptr) {
    // passes 1 + 2: minimizers, superkmers, staging, sizes, offsets
    if (part->staging_cap && !part->d_staging) return DBG_EINVAL;
    MspArgs a;
    a.words = d_bases;
    a.n_words = n_words;
    a.offsets = d_offsets;
    a.n_reads = n_reads;
    a.k = prm->k;
    a.p = partition_p(prm);  // the fine partitioning's minimizer (dbg.h fine_p)
    a.np = np;
    a.w = prm->k - a.p + 1;
    a.rec_words = R;
    a.max_kmers = record_max_kmers(prm->k);
    a.mod = make_fastmod((uint64_t)np);
    a.n_records = reinterpret_cast<unsigned long long*>(part->d_n_records);
    a.n_kmers = reinterpret_cast<unsigned long long*>(part->d_n_kmers);
    a.staging = part->d_staging;
    a.staging_cap = part->staging_cap;
    a.staged = reinterpret_cast<unsigned long long*>(part->d_staged);
    a.pid_lo = (uint32_t)pid_lo;
    a.pid_hi = (uint32_t)pid_hi;
    a.ranged = pid_lo > 0 || pid_hi < np;
    if (!append && (cudaMemsetAsync(part->d_n_records, 0, sizeof(uint64_t) * np, stream) != cudaSuccess ||
                    cudaMemsetAsync(part->d_n_kmers, 0, sizeof(uint64_t) * np, stream) != cudaSuccess ||
                    cudaMemsetAsync(part->d_staged, 0, sizeof(uint64_t), stream) != cudaSuccess))
      return DBG_ECUDA;
    if (n_reads) {
      const uint64_t want = (n_reads + kMspThreads - 1) / kMspThreads;
      const uint64_t cap = (uint64_t)dbg_sm_count() * 32;  // the launchers cap it at one resident wave
      const int grid = (int)(want < cap ? want : cap);
      cudaError_t e = cudaSuccess;
      if (!msp_block_launch(a, grid, stream, &e)) e = launch_msp_warp_any(a, stream);
      if (e != cudaSuccess) return DBG_ECUDA;
    }
    // d_fill is idle until pass 2 (which zeroes it): scratch for the tile sums
    if (exclusive_scan(IdentityOp{part->d_n_records}, np, part->d_record_offset,
                       reinterpret_cast<unsigned long long*>(part->d_fill), stream) != cudaSuccess)
      return DBG_ECUDA;
  } else {
    // pass 3: scatter (a no-op after a staging overflow, *d_staged > staging_cap)
    if (!part->d_fill || !part->d_staging) return DBG_EINVAL;
    if (part->d_scratch && (part->d_scratch == part->d_staging || part->d_scratch == part->d_records))
      return DBG_EINVAL;
    if (part->n_peers < 0 ||
        (part->n_peers > 0 && (!part->d_peer_records || !part->d_peer_bounds)))
      return DBG_EINVAL;
    // Above kSmemHistMaxNp fine partitions a one-level scatter writes every record to a random
    // place of a multi-GB output with one returning global atomic each (chr14: ~36 G records/s,
    // latency-bound); with d_scratch and d_work the records go in two counting-sort levels
    // (ts_level_a/b_kernel).
    const bool two = part->d_scratch && part->d_work && np > kSmemHistMaxNp;
    if (part->d_scratch && !part->d_work && np > kSmemHistMaxNp) return DBG_EINVAL;
    if (cudaMemsetAsync(part->d_fill, 0, sizeof(uint64_t) * np, stream) != cudaSuccess) return DBG_ECUDA;
    const unsigned long long* staged = reinterpret_cast<const unsigned long long*>(part->d_staged);
    unsigned long long* fill = reinterpret_cast<unsigned long long*>(part->d_fill);
    if (!two) {
      const size_t smem = np <= kSmemHistMaxNp ? (sizeof(unsigned long long) + sizeof(uint32_t)) * np : 0;
      // one full wave: the kernel is grid-stride, a partial second wave would idle SMs
      auto scatter_grid = [&](const void* fn) {
        int per_sm = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kScatterThreads, smem) != cudaSuccess ||
            per_sm < 1)
          per_sm = 4;
        return dbg_sm_count() * per_sm;
      };
#define DBG_SCATTER(RW)                                                                                         \
  cudaFuncSetAttribute(scatter_kernel<RW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);            \
  scatter_kernel<RW><<<scatter_grid((const void*)scatter_kernel<RW>), kScatterThreads, smem, stream>>>(        \
      part->d_staging, staged, part->staging_cap, part->d_record_offset, fill, part->d_records, np,             \
      part->d_peer_records, part->d_peer_bounds, part->n_peers);
      if (R == 4) {
        DBG_SCATTER(4)
      } else if (R == 8) {
        DBG_SCATTER(8)
      } else {
        DBG_SCATTER(16)
      }
#undef DBG_SCATTER
    } else {
      const int s = ts_shift(np), nb = (np + (1 << s) - 1) >> s;
      TsArgs ta;
      ta.staged = staged;
      ta.staging_cap = part->staging_cap;
      ta.boff = part->d_work + nb;
      ta.tiles = part->d_work + 2 * nb + 1;
      ta.rec_off = part->d_record_offset;
      ta.nb = nb;
      ta.s = s;
      ta.np = np;
      ta.peer_records = part->d_peer_records;
      ta.peer_bounds = part->d_peer_bounds;
      ta.n_peers = part->n_peers;
      const int tile = R == 4 ? ts_tile<4>() : (R == 8 ? ts_tile<8>() : ts_tile<16>());
      ts_bucket_count_kernel<<<nb, 256, 0, stream>>>(part->d_n_records, np, s, part->d_work + nb);
      ts_bucket_scan_kernel<<<1, 1024, 0, stream>>>(part->d_work, nb, tile);
      const size_t rec_bytes = R == 4 ? ts_rec_bytes<4>() : (R == 8 ? ts_rec_bytes<8>() : ts_rec_bytes<16>());
      const size_t smem_a = rec_bytes + ts_bin_bytes(nb);
      const size_t smem_b = rec_bytes + ts_bin_bytes(1 << s) + sizeof(unsigned long long) * (nb + 1);
      auto ts_grid = [&](const void* fn, size_t smem) {
        int per_sm = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kTsThreads, smem) != cudaSuccess || per_sm < 1)
          per_sm = 1;
        return dbg_sm_count() * per_sm;
      };
#define DBG_TS(RW)                                                                                              \
  {                                                                                                             \
    TsArgs x = ta;                                                                                              \
    x.src = part->d_staging;                                                                                    \
    x.dst = part->d_scratch;                                                                                    \
    x.fill = reinterpret_cast<unsigned long long*>(part->d_work);                                               \
    cudaFuncSetAttribute(ts_level_a_kernel<RW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_a);     \
    ts_level_a_kernel<RW><<<ts_grid((const void*)ts_level_a_kernel<RW>, smem_a), kTsThreads, smem_a, stream>>>(x); \
    x.src = part->d_scratch;                                                                                    \
    x.dst = part->d_records;                                                                                    \
    x.fill = fill;                                                                                              \
    cudaFuncSetAttribute(ts_level_b_kernel<RW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_b);     \
    ts_level_b_kernel<RW><<<ts_grid((const void*)ts_level_b_kernel<RW>, smem_b), kTsThreads, smem_b, stream>>>(x); \
  }
      if (R == 4) {
        DBG_TS(4)
      } else if (R == 8) {
        DBG_TS(8)
      } else {
        DBG_TS(16)
      }
#undef DBG_TS
    }
  }
  return cudaPeekAtLastError() == cudaSuccess ? DBG_OK : DBG_ECUDA;
}

static dbg_status table_plan(const dbg_params* prm, const uint64_t* d_n_kmers, uint64_t slots,
                             uint64_t* d_table_offset, uint64_t* d_scratch, cudaStream_t stream) {
  if (!dbg_params_ok(prm) || !d_n_kmers || !d_table_offset) return DBG_EINVAL;
  if (!(prm->lambda > 0.f) || !(prm->alpha > 0.f)) return DBG_EINVAL;
  const double ratio = (double)prm->lambda / (4.0 * (double)prm->alpha);
  const cudaError_t e = exclusive_scan(CapacityOp{d_n_kmers, ratio, slots, smem_max_split(prm)},
                                       fine_partitions(prm), d_table_offset,
                                       reinterpret_cast<unsigned long long*>(d_scratch), stream);
  return e == cudaSuccess ? DBG_OK : DBG_ECUDA;
}

extern "C" dbg_status dbg_table_plan(const dbg_params* prm, const uint64_t* d_n_kmers, uint64_t* d_table_offset,
                                     uint64_t* d_scratch, cudaStream_t stream) {
  return table_plan(prm, d_n_kmers, 0, d_table_offset, d_scratch, stream);
}

extern "C" dbg_status dbg_table_plan_split(const dbg_params* prm, const uint64_t* d_n_kmers, uint64_t* d_table_offset,
                                           uint64_t* d_scratch, cudaStream_t stream) {
  if (!prm || prm->k > 63) return DBG_EINVAL;
  return table_plan(prm, d_n_kmers, dbg_smem_table_slots(prm), d_table_offset, d_scratch, stream);
}

// ---- multi-GPU exchange plan (dbg.h dbg_exchange_plan) ----------------
// Entry i: records of fine partition i summed over the world ranks' rows of the gathered counts.
struct GatheredSumOp {
  const uint64_t* counts;
  int np, world;
  __device__ __forceinline__ unsigned long long operator()(int i) const {
    unsigned long long s = 0;
    for (int r = 0; r < world; ++r) s += counts[(size_t)r * np + i];
    return s;
  }
};

// prefix = exclusive scan of the summed counts over ALL partitions; partition f of owner o
// starts at prefix[f] - prefix[bounds[o]] in o's buffer, and this rank's share of it after the
// records of the lower ranks.
__global__ void exchange_plan_kernel(const uint64_t* __restrict__ counts, const uint64_t* kmers_sum, int np,
                                     int world, int rank, const int32_t* __restrict__ bounds,
                                     const uint64_t* __restrict__ prefix, uint64_t* __restrict__ dest,
                                     uint64_t* __restrict__ own_n, uint64_t* own_k, uint64_t* __restrict__ own_off) {
  const int lo = bounds[rank], hi = bounds[rank + 1];
  for (int f = blockIdx.x * blockDim.x + threadIdx.x; f <= np; f += gridDim.x * blockDim.x) {
    if (f < np) {
      int o = 0;
      while (o + 1 < world && f >= bounds[o + 1]) ++o;
      uint64_t d = prefix[f] - prefix[bounds[o]];
      for (int r = 0; r < rank; ++r) d += counts[(size_t)r * np + f];
      dest[f] = d;
      const bool mine = f >= lo && f < hi;
      own_n[f] = mine ? prefix[f + 1] - prefix[f] : 0;
      const uint64_t k = kmers_sum[f];
      own_k[f] = mine ? k : 0;
    }
    const int c = f < lo ? lo : (f > hi ? hi : f);
    own_off[f] = prefix[c] - prefix[lo];
  }
}

extern "C" dbg_status dbg_exchange_plan(const dbg_params* prm, const uint64_t* d_counts, const uint64_t* d_kmers_sum,
                                        int32_t world, int32_t rank, const int32_t* d_bounds,
                                        uint64_t* d_dest_offset, uint64_t* d_owned_n_records,
                                        uint64_t* d_owned_n_kmers, uint64_t* d_owned_record_offset,
                                        uint64_t* d_prefix, uint64_t* d_scratch, cudaStream_t stream) {
  if (!dbg_params_ok(prm) || !d_counts || !d_kmers_sum || !d_bounds || !d_dest_offset || !d_owned_n_records ||
      !d_owned_n_kmers || !d_owned_record_offset || !d_prefix || world < 1 || rank < 0 || rank >= world)
    return DBG_EINVAL;
  if (d_prefix == d_owned_record_offset || d_prefix == d_dest_offset || d_prefix == d_owned_n_records ||
      (d_scratch && (d_scratch == d_prefix || d_scratch == d_owned_record_offset)))
    return DBG_EINVAL;
  const int np = fine_partitions(prm);
  if (exclusive_scan(GatheredSumOp{d_counts, np, world}, np, d_prefix,
                     reinterpret_cast<unsigned long long*>(d_scratch), stream) != cudaSuccess)
    return DBG_ECUDA;
  const int grid = (int)std::min<int64_t>(((int64_t)np + 256) / 256, (int64_t)dbg_sm_count() * 8);
  exchange_plan_kernel<<<grid, 256, 0, stream>>>(d_counts, d_kmers_sum, np, world, rank, d_bounds, d_prefix,
                                                 d_dest_offset, d_owned_n_records, d_owned_n_kmers,
                                                 d_owned_record_offset);
  return cudaPeekAtLastError() == cudaSuccess ? DBG_OK : DBG_ECUDA;
}
