// msp.cu -- Step 1 of ParaHash on sm_100a: MSP graph partitioning
// (Sec. III-B; Defs. 1-2), kernel (a) of the north star.
//
// One warp scans one read at a time in chunks of 32 K-mers (lane t <-> K-mer
// i0+t).  For the chunk, the canonical value of every P-mer it needs
// (c_j = min(code(s_j), code(rc(s_j))), readings A/D/E) is computed by the
// lanes from the 2-bit stream (two u64 loads + funnel shift + bit-reverse)
// into a per-warp shared-memory row; each lane then takes the minimum over
// its window of w = K-P+1 values (Def. 1).  Superkmer boundaries (Def. 2,
// reading G: maximal runs of equal minimizer) come from a warp ballot; the
// lane that sees a boundary emits the superkmer that closes there.  The
// partition id is fmix64(m) mod NP (reading I).
//
// The paper left superkmer generation ("memory movement of irregular
// lengths") to the CPU; here the same kernel emits fixed-width
// records (dbg.h) straight into the per-partition HBM buffers: a count pass
// sizes them (per-partition histograms in shared memory, P:L972-975's
// prefix sum of superkmer lengths gives N^i_kmer), a scan turns sizes into
// offsets, and an emit pass writes the records.
#include <cub/block/block_scan.cuh>

#include "dbg_device.cuh"

namespace dbg {

constexpr int kMspWarps = 8;
constexpr int kMspThreads = kMspWarps * kWarp;
constexpr int kCbuf = 96;  // >= 32 + w - 1 for w <= 63, padded
constexpr int kSmemHistMaxNp = 4096;

struct MspArgs {
  const uint64_t* words;
  uint64_t n_words;
  const uint64_t* offsets;
  uint64_t n_reads;
  int k, p, np;
  uint32_t rec_words, max_kmers;
  unsigned long long* n_records;  // [np] (count mode)
  unsigned long long* n_kmers;    // [np] (count mode)
  const uint64_t* rec_off;        // [np+1] (emit mode)
  unsigned long long* fill;       // [np]   (emit mode)
  uint32_t* records;              // (emit mode)
};

// Canonical P-mer value at stream position pos (Def. 1 with readings A/D).
__device__ __forceinline__ uint64_t canon_pmer(const MspArgs& a, uint64_t pos) {
  uint64_t f = window64(a.words, a.n_words, pos) >> (64 - 2 * a.p);
  uint64_t r = revcomp64(f, a.p);
  return f < r ? f : r;
}

// Writes the pieces of superkmer [s, e] (K-mer start positions within the
// read at stream offset o of length L) into partition pid (emit mode), or
// counts them (count mode).
template <bool kEmit>
__device__ __forceinline__ void emit_superkmer(const MspArgs& a, uint64_t o, int64_t L, int64_t s,
                                               int64_t e, uint32_t pid, unsigned long long* sh_rec,
                                               unsigned long long* sh_kmer) {
  const int64_t n = e - s + 1;
  const int64_t nmax = a.max_kmers;
  const uint64_t pieces = (uint64_t)((n + nmax - 1) / nmax);
  if (!kEmit) {
    if (sh_rec) {
      atomicAdd(sh_rec + pid, (unsigned long long)pieces);
      atomicAdd(sh_kmer + pid, (unsigned long long)n);
    } else {
      atomicAdd(a.n_records + pid, (unsigned long long)pieces);
      atomicAdd(a.n_kmers + pid, (unsigned long long)n);
    }
    return;
  }
  uint64_t slot = a.rec_off[pid] + atomicAdd(a.fill + pid, (unsigned long long)pieces);
  for (int64_t ps = s; ps <= e; ps += nmax, ++slot) {
    const int64_t pe = min(e, ps + nmax - 1);
    const uint32_t hl = ps > 0 ? 1u : 0u;                 // reading H
    const uint32_t hr = pe + a.k < L ? 1u : 0u;
    const int64_t bs = ps - hl;
    const int64_t nb = (int64_t)hl + (pe - ps + 1) + a.k - 1 + hr;
    uint32_t w[8];
    w[0] = (uint32_t)(pe - ps + 1) | (hl << 8) | (hr << 9) | (pid << 10);
#pragma unroll
    for (int q = 0; q < 7; ++q) {
      if (q + 1 < (int)a.rec_words) {
        int64_t left = nb - 16 * q;  // bases still to place
        uint32_t v = 0;
        if (left > 0) {
          v = (uint32_t)(window64(a.words, a.n_words, o + bs + 16 * q) >> 32);
          if (left < 16) v &= ~(0xffffffffu >> (2 * left));  // zero the bases past the record
        }
        w[q + 1] = v;
      }
    }
    uint4* dst = reinterpret_cast<uint4*>(a.records + slot * a.rec_words);
    dst[0] = make_uint4(w[0], w[1], w[2], w[3]);
    if (a.rec_words == 8) dst[1] = make_uint4(w[4], w[5], w[6], w[7]);
  }
}

template <bool kEmit>
__global__ void __launch_bounds__(kMspThreads) msp_kernel(MspArgs a) {
  extern __shared__ unsigned long long smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  uint64_t* cbuf = reinterpret_cast<uint64_t*>(smem) + warp * kCbuf;
  unsigned long long* sh_rec = nullptr;
  unsigned long long* sh_kmer = nullptr;
  const bool smem_hist = !kEmit && a.np <= kSmemHistMaxNp;
  if (smem_hist) {
    sh_rec = smem + kMspWarps * kCbuf;
    sh_kmer = sh_rec + a.np;
    for (int i = threadIdx.x; i < 2 * a.np; i += blockDim.x) sh_rec[i] = 0;
    __syncthreads();
  }
  const int K = a.k;
  const int w = a.k - a.p + 1;  // P-mers per K-mer window (Def. 1: j in [i, i+K-P])
  const uint64_t n_warps = (uint64_t)gridDim.x * kMspWarps;
  for (uint64_t r = (uint64_t)blockIdx.x * kMspWarps + warp; r < a.n_reads; r += n_warps) {
    const uint64_t o = a.offsets[r];
    const int64_t L = (int64_t)(a.offsets[r + 1] - o);
    if (L < K) continue;  // reading N
    const int64_t nk = L - K + 1;
    const int64_t npm = L - a.p + 1;  // P-mers in the read
    int64_t s_open = 0;               // start of the superkmer still open
    uint64_t m_carry = 0;             // minimizer of K-mer i0-1
    for (int64_t i0 = 0; i0 < nk; i0 += 32) {
      const int jn = (int)(npm - i0 < (int64_t)(32 + w - 1) ? npm - i0 : (int64_t)(32 + w - 1));
      for (int t = lane; t < jn; t += 32) cbuf[t] = canon_pmer(a, o + i0 + t);
      __syncwarp();
      const int64_t i = i0 + lane;
      const bool valid = i < nk;
      uint64_t m = ~0ull;
      if (valid)
        for (int d = 0; d < w; ++d) m = min(m, cbuf[lane + d]);
      __syncwarp();
      uint64_t mp = __shfl_up_sync(kFull, m, 1);
      if (lane == 0) mp = m_carry;
      const bool is_start = valid && (i == 0 || m != mp);
      const uint32_t starts = __ballot_sync(kFull, is_start);
      // (1) the superkmer that closes at K-mer i-1, emitted by the lane starting the next one
      if (is_start && i > 0) {
        const uint32_t below = starts & ((1u << lane) - 1u);
        const int64_t s = below ? i0 + 31 - __clz(below) : s_open;
        emit_superkmer<kEmit>(a, o, L, s, i - 1, (uint32_t)(fmix64(mp) % (uint64_t)a.np), sh_rec,
                              sh_kmer);
      }
      // (2) the read's last superkmer, emitted by the lane holding the last K-mer
      if (valid && i == nk - 1) {
        const uint32_t upto = starts & (lane == 31 ? kFull : ((2u << lane) - 1u));
        const int64_t s = upto ? i0 + 31 - __clz(upto) : s_open;
        emit_superkmer<kEmit>(a, o, L, s, i, (uint32_t)(fmix64(m) % (uint64_t)a.np), sh_rec,
                              sh_kmer);
      }
      if (starts) s_open = i0 + 31 - __clz(starts);
      m_carry = __shfl_sync(kFull, m, 31);
    }
  }
  if (smem_hist) {
    __syncthreads();
    for (int i = threadIdx.x; i < a.np; i += blockDim.x) {
      if (sh_rec[i]) atomicAdd(a.n_records + i, sh_rec[i]);
      if (sh_kmer[i]) atomicAdd(a.n_kmers + i, sh_kmer[i]);
    }
  }
}

// Exclusive prefix sum out[0..n] of f(in[0..n-1]) in one CTA (n = NP is small);
// f = identity (record offsets) or the table capacity of Sec. IV-A.
constexpr int kScanThreads = 256;
template <bool kCapacity>
__global__ void __launch_bounds__(kScanThreads) scan_kernel(const uint64_t* __restrict__ in,
                                                            uint64_t* __restrict__ out, int n,
                                                            double ratio) {
  using Scan = cub::BlockScan<unsigned long long, kScanThreads>;
  __shared__ typename Scan::TempStorage tmp;
  __shared__ unsigned long long carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (int base = 0; base < n; base += kScanThreads) {
    const int i = base + threadIdx.x;
    unsigned long long v = 0;
    if (i < n) {
      v = in[i];
      if (kCapacity && v) {
        // capacity_i = ceil(lambda / (4 alpha) * N^i_kmer), at least 1
        double c = ceil(ratio * (double)v);
        v = c < 1.0 ? 1ull : (unsigned long long)c;
      }
    }
    unsigned long long excl, total;
    Scan(tmp).ExclusiveSum(v, excl, total);
    if (i < n) out[i] = carry + excl;
    __syncthreads();
    if (threadIdx.x == 0) carry += total;
    __syncthreads();
  }
  if (threadIdx.x == 0) out[n] = carry;
}

}  // namespace dbg

using namespace dbg;

static int sm_count() {
  int dev = 0, n = 148;
  if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
  return n;
}

static bool params_ok(const dbg_params* prm) {
  return prm && prm->k >= 1 && prm->k <= 63 && (prm->k & 1) && prm->p >= 1 && prm->p <= prm->k &&
         prm->p <= 31 && prm->num_partitions >= 1 && (uint32_t)prm->num_partitions <= kMaxPid;
}

extern "C" dbg_status dbg_msp_partition(const dbg_params* prm, const uint64_t* d_bases,
                                        uint64_t n_words, const uint64_t* d_offsets,
                                        uint64_t n_reads, const dbg_partition_set* part,
                                        cudaStream_t stream) {
  if (!params_ok(prm) || !part || !d_offsets || !part->d_record_offset) return DBG_EINVAL;
  if (n_reads && (!d_bases || !n_words)) return DBG_EINVAL;
  const bool emit = part->d_records != nullptr;
  if (!emit && (!part->d_n_records || !part->d_n_kmers)) return DBG_EINVAL;
  if (emit && !part->d_fill) return DBG_EINVAL;
  const int np = prm->num_partitions;
  MspArgs a;
  a.words = d_bases;
  a.n_words = n_words;
  a.offsets = d_offsets;
  a.n_reads = n_reads;
  a.k = prm->k;
  a.p = prm->p;
  a.np = np;
  a.rec_words = record_words(prm->k);
  a.max_kmers = record_max_kmers(prm->k);
  a.n_records = reinterpret_cast<unsigned long long*>(part->d_n_records);
  a.n_kmers = reinterpret_cast<unsigned long long*>(part->d_n_kmers);
  a.rec_off = part->d_record_offset;
  a.fill = reinterpret_cast<unsigned long long*>(part->d_fill);
  a.records = part->d_records;
  const uint64_t want = (n_reads + kMspWarps - 1) / kMspWarps;
  const uint64_t cap = (uint64_t)sm_count() * 8;
  const int grid = (int)(want < cap ? (want ? want : 1) : cap);
  size_t smem = sizeof(unsigned long long) * kMspWarps * kCbuf;
  if (!emit) {
    if (cudaMemsetAsync(part->d_n_records, 0, sizeof(uint64_t) * np, stream) != cudaSuccess ||
        cudaMemsetAsync(part->d_n_kmers, 0, sizeof(uint64_t) * np, stream) != cudaSuccess)
      return DBG_ECUDA;
    if (np <= kSmemHistMaxNp) smem += sizeof(unsigned long long) * 2 * np;
    static bool attr_set = false;
    if (!attr_set) {
      cudaFuncSetAttribute(msp_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           (int)(sizeof(unsigned long long) * (kMspWarps * kCbuf + 2 * kSmemHistMaxNp)));
      attr_set = true;
    }
    if (n_reads) msp_kernel<false><<<grid, kMspThreads, smem, stream>>>(a);
    scan_kernel<false><<<1, kScanThreads, 0, stream>>>(part->d_n_records, part->d_record_offset, np, 0.0);
  } else {
    if (cudaMemsetAsync(part->d_fill, 0, sizeof(uint64_t) * np, stream) != cudaSuccess) return DBG_ECUDA;
    if (n_reads) msp_kernel<true><<<grid, kMspThreads, smem, stream>>>(a);
  }
  return cudaPeekAtLastError() == cudaSuccess ? DBG_OK : DBG_ECUDA;
}

extern "C" dbg_status dbg_table_plan(const dbg_params* prm, const uint64_t* d_n_kmers,
                                     uint64_t* d_table_offset, cudaStream_t stream) {
  if (!params_ok(prm) || !d_n_kmers || !d_table_offset) return DBG_EINVAL;
  if (!(prm->lambda > 0.f) || !(prm->alpha > 0.f)) return DBG_EINVAL;
  const double ratio = (double)prm->lambda / (4.0 * (double)prm->alpha);
  scan_kernel<true><<<1, kScanThreads, 0, stream>>>(d_n_kmers, d_table_offset, prm->num_partitions, ratio);
  return cudaPeekAtLastError() == cudaSuccess ? DBG_OK : DBG_ECUDA;
}
