// msp_warp.cuh -- pass 1 of Step 1 (MSP graph partitioning, Sec. III-B; Definitions
// 1-2 P:L221-230) with one WARP per read: the north star's "warp-parallel sliding minimizer".
// Included by msp.cu (MspArgs, record_pieces, sh_addr).
//
// Work unit: a chunk of 32 consecutive reads per warp (lane t holds read t's offsets).  The chunk's
// 2-bit words are contiguous in the stream; one lane copies them into the warp's shared-memory
// buffer with a TMA bulk copy (cp.async.bulk, completion on an mbarrier), double-buffered: the
// copy of the warp's next chunk is in flight while the current one is hashed.  A chunk whose
// words exceed the buffer (long reads) is read from global memory instead.
//
// Per read the 32 lanes cover 32R consecutive P-mer positions ("a piece"; R per lane,
// contiguous): lane l owns positions x0 = i0 + lR .. x0 + R - 1.
//  * canonical P-mer codes (readings A, D, E): one 64-bit window of bases at x0 (two when
//    P + R - 1 > 32) and its reverse complement; code j = min(forward, reverse) by constant shifts.
//  * Definition 1, the window minimum over w = K - P + 1 positions, for K-mer i = x0 + j:
//    positions i .. i+w-1 span lane l (from j: the lane's suffix minimum), lanes l+1 .. l+d-1
//    (whole lanes: a sparse table of lane minima built with log2 shuffles) and lane l+d (up to
//    e: that lane's prefix minimum, one shuffle), d = (j+w-1) div R, e = (j+w-1) mod R -- the
//    same d, e for every lane, so every shuffle has a uniform offset.
//  * Definition 2 (reading G): K-mer i starts a superkmer iff its minimizer differs from K-mer
//    i-1's (i = 0: always); each start finds its end from its own flag bits or the next lane
//    with a start (ballot); ranks from per-position ballots give dense descriptor slots.
//  * reads longer than a piece (32R - w + 1 K-mers) take several pieces; the superkmer open at
//    a piece's end is carried into the next piece.
// Descriptors (start, end, minimizer, read) collect in shared memory; a warp flush per chunk
// (or when the list could overflow) computes partition ids (reading I), the per-partition
// sizes N^i_kmer and record counts, reserves the chunk's staging range with ONE atomic and
// writes the fixed-width records (dbg.h) with the two adjacency bases (Sec. III-B
// P:L443-451), taking the bases from the staged chunk.
#pragma once

namespace dbg {

constexpr int kWarpMspThreads = 256;
constexpr int kWarpMspWarps = kWarpMspThreads / 32;
constexpr int kChunkWords = 192;  // staged 64-bit words per chunk buffer (32 reads of <= ~180 bases)

template <typename CT, int DESC>
struct alignas(16) WarpMspSmem {  // one warp's shared memory
  uint64_t buf[2][kChunkWords + 2];  // +2: the second word of a window at the buffer's end
  uint64_t mbar[2];
  uint32_t ds[DESC], de[DESC];  // first and last K-mer of a superkmer (read coordinates)
  CT dm[DESC];                  // its minimizer; after the flush's first pass its partition id
  uint8_t dt[DESC];             // its read within the chunk
};

// Reverse complement of all 32 bases of a 64-bit window (reading A: complement = 3 - c).
__device__ __forceinline__ uint64_t revcomp32(uint64_t x) {
  const uint64_t y = __brevll(~x);
  return ((y >> 1) & 0x5555555555555555ull) | ((y & 0x5555555555555555ull) << 1);
}

template <typename T>
__device__ __forceinline__ T tmin(T x, T y) { return y < x ? y : x; }

// R: P-mer positions per lane; KC, PC > 0: compile-time K and P; DESC: descriptor list length;
// MINB: CTAs per SM the registers are capped for (K = 63: 4 CTAs x 8 warps with <= 64 registers and
// 192 descriptors, 46.8 vs 47.4 ms with 3 CTAs, profiles/r02_ab.txt; runtime K, P: 3, no spills).
template <typename CT, int R, int KC, int PC, int DESC, int MINB>
__global__ void __launch_bounds__(kWarpMspThreads, MINB) msp_warp_kernel(MspArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  typedef WarpMspSmem<CT, DESC> S;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  S& sm = reinterpret_cast<S*>(smem_raw)[wid];
  const int K = KC ? KC : a.k, P = PC ? PC : a.p, w = K - P + 1;
  constexpr CT kInf = ~(CT)0, kSkip = ~(CT)0;
  const CT maskP = (CT)((2 * P == 8 * (int)sizeof(CT)) ? ~(CT)0 : (((CT)1 << (2 * P)) - 1));
  const int cap = 32 * R - w + 1;  // K-mers per piece (the launcher checks w <= 32R)
  const bool two_win = P + R - 1 > 32;
  const int nmax = KC ? (int)record_max_kmers(KC) : (int)a.max_kmers;
  const uint32_t rw = KC ? record_words(KC) : a.rec_words;
  // lanes l + 1 .. l + D (D = d - 1 <= Dmax) from a sparse table of lane minima
  const int Dmax = (R - 1 + w - 1) / R - 1;
  const uint32_t lt_mask = (1u << lane) - 1u;

  const uint64_t n_chunks = (a.n_reads + 31) / 32;
  const uint64_t gw = (uint64_t)blockIdx.x * kWarpMspWarps + wid, nw = (uint64_t)gridDim.x * kWarpMspWarps;
  if (lane == 0) {
    mbar_init(&sm.mbar[0], 1);
    mbar_init(&sm.mbar[1], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();

  // Offsets of chunk c (lane t: read 32c + t; L = 0 past the last read), and the TMA copy of its
  // words into buffer b.  Every call arrives once on mbar[b], so its phase flips once per use.
  auto load_chunk = [&](uint64_t c, int b, uint64_t& o_l, int& L_l, uint64_t& wlo, bool& staged) {
    const uint64_t r = c * 32 + lane;
    o_l = __ldg(a.offsets + (r < a.n_reads ? r : a.n_reads));
    const uint64_t e_l = __ldg(a.offsets + (r < a.n_reads ? r + 1 : a.n_reads));
    L_l = (int)(e_l - o_l);
    const uint64_t first = __shfl_sync(kFull, o_l, 0), last = __shfl_sync(kFull, e_l, 31);
    uint64_t lo = first >> 5;
    const uint64_t hi_w = (last + 31) / 32 + 3, hi = hi_w < a.n_words ? hi_w : a.n_words;
    if ((reinterpret_cast<uintptr_t>(a.words + lo) & 15u) && lo > 0) --lo;  // 16-byte aligned source
    staged = !(reinterpret_cast<uintptr_t>(a.words + lo) & 15u) && (hi <= lo || hi - lo <= (uint64_t)kChunkWords);
    wlo = lo;
    if (lane == 0) {
      const uint64_t nwds = staged && hi > lo ? hi - lo : 0;
      const uint32_t nbulk = (uint32_t)(nwds & ~1ull);
      // the buffer's previous contents were read through the generic proxy (ordered by the
      // __syncwarp at the end of that chunk): order them before the async-proxy write
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      if (nwds & 1) sm.buf[b][nwds - 1] = __ldg(a.words + hi - 1);  // odd tail: a plain copy
      if (nbulk) {
        mbar_arrive_tx(&sm.mbar[b], nbulk * 8u);
        tma_bulk_g2s(&sm.buf[b][0], a.words + lo, nbulk * 8u, &sm.mbar[b]);
      } else {
        mbar_arrive(&sm.mbar[b]);
      }
    }
  };

  int ndesc = 0;
  uint64_t o_cur = 0, wlo_cur = 0;
  int L_cur = 0;
  bool st_cur = false;
  if (gw < n_chunks) load_chunk(gw, 0, o_cur, L_cur, wlo_cur, st_cur);
  int it = 0;
  for (uint64_t c = gw; c < n_chunks; c += nw, ++it) {
    const int b = it & 1;
    uint64_t o_nx = 0, wlo_nx = 0;
    int L_nx = 0;
    bool st_nx = false;
    if (c + nw < n_chunks) load_chunk(c + nw, b ^ 1, o_nx, L_nx, wlo_nx, st_nx);
    mbar_wait(&sm.mbar[b], (uint32_t)(it >> 1) & 1u);
    __syncwarp();  // the odd-tail word written by lane 0
    const uint64_t* buf = sm.buf[b];
    const bool staged = st_cur;
    const uint64_t wbase = wlo_cur << 5;
    // 64 bases from stream base position pos (bits past the stream's end are unspecified when
    // staged; callers use only bases inside the reads)
    auto win = [&](uint64_t pos) -> uint64_t {
      if (staged) {
        const uint64_t rel = pos - wbase;
        const uint32_t q = (uint32_t)(rel >> 5), sh = (uint32_t)(rel & 31) * 2;
        const uint64_t h = buf[q], l = buf[q + 1];
        return sh ? (h << sh) | (l >> (64 - sh)) : h;
      }
      return window64(a.words, a.n_words, pos);
    };

    // Warp flush of the descriptor list: partition ids and sizes, one staging reservation,
    // record writes.
    auto flush = [&]() {
      __syncwarp();
      uint32_t mine = 0;
      for (int k0 = 0; k0 < ndesc; k0 += 32) {
        const int k = k0 + lane;
        if (k < ndesc) {
          const uint32_t pid = a.np == 1 ? 0u : fast_mod(a.mod, fmix64((uint64_t)sm.dm[k]));
          const bool in = !a.ranged || pid - a.pid_lo < a.pid_hi - a.pid_lo;
          const uint32_t n = sm.de[k] - sm.ds[k] + 1u, pcs = record_pieces((int)n, nmax);
          if (in) {
            atomicAdd(a.n_records + pid, (unsigned long long)pcs);
            atomicAdd(a.n_kmers + pid, (unsigned long long)n);
            mine += pcs;
          }
          sm.dm[k] = in ? (CT)pid : kSkip;
        }
      }
      uint32_t total = mine;
#pragma unroll
      for (int dlt = 16; dlt; dlt >>= 1) total += __shfl_xor_sync(kFull, total, dlt);
      unsigned long long base = 0;
      if (lane == 0 && total) base = atomicAdd(a.staged, (unsigned long long)total);
      uint64_t run = __shfl_sync(kFull, base, 0);
      for (int k0 = 0; k0 < ndesc; k0 += 32) {
        const int k = k0 + lane;
        const bool act = k < ndesc && sm.dm[k] != kSkip;
        const uint32_t s = act ? sm.ds[k] : 0u, e = act ? sm.de[k] : 0u;
        const uint32_t pcs = act ? record_pieces((int)(e - s + 1u), nmax) : 0u;
        uint32_t incl = pcs;
#pragma unroll
        for (int dlt = 1; dlt < 32; dlt <<= 1) {
          const uint32_t v = __shfl_up_sync(kFull, incl, dlt);
          if (lane >= dlt) incl += v;
        }
        const int tk = k < ndesc ? (int)sm.dt[k] : 0;
        const uint64_t o = __shfl_sync(kFull, o_cur, tk);
        const int L = __shfl_sync(kFull, L_cur, tk);
        uint64_t slot = run + incl - pcs;
        run += __shfl_sync(kFull, incl, 31);
        if (act) {
          const uint32_t pid = (uint32_t)sm.dm[k];
          for (int ps = (int)s; ps <= (int)e; ps += nmax, ++slot) {
            if (slot >= a.staging_cap) continue;  // overflow: counted, the caller repeats the step
            const int pe = min((int)e, ps + nmax - 1);
            const uint32_t hl = ps > 0 ? 1u : 0u, hr = pe + K < L ? 1u : 0u;  // reading H
            const int nb = (int)hl + (pe - ps + 1) + K - 1 + (int)hr;
            const uint64_t pos = o + (uint64_t)(ps - (int)hl);
            uint4* d4 = reinterpret_cast<uint4*>(a.staging + slot * rw);
            const uint32_t hdr = rec_header((uint32_t)(pe - ps + 1), hl, hr, pid);
            // data word q (1 .. rw-1) holds bases 16(q-1) .. 16q-1: 32-base window u = (q-1)/2,
            // high half for odd q
            for (int c4 = 0; c4 < (int)rw / 4; ++c4) {
              uint32_t wv[4];
              // window v covers record words 1+2v (high) and 2+2v (low)
#pragma unroll
              for (int x = 0; x < 4; ++x) {
                const int q = 4 * c4 + x;
                if (q == 0) {
                  wv[x] = hdr;
                  continue;
                }
                const int v = (q - 1) >> 1, left = nb - 32 * v;
                uint32_t word = 0;
                if (left > 0) {
                  uint64_t wd = win(pos + 32u * (uint32_t)v);
                  if (left < 32) wd &= ~(~0ull >> (2 * left));  // zero the bases past the record
                  word = (q & 1) ? (uint32_t)(wd >> 32) : (uint32_t)wd;
                }
                wv[x] = word;
              }
              d4[c4] = make_uint4(wv[0], wv[1], wv[2], wv[3]);
            }
          }
        }
      }
      ndesc = 0;
      __syncwarp();
    };

    for (int t = 0; t < 32; ++t) {
      const uint64_t o = __shfl_sync(kFull, o_cur, t);
      const int L = __shfl_sync(kFull, L_cur, t);
      const int nk = L - K + 1, nP = L - P + 1;
      if (nk <= 0) continue;  // reading N: no K-mers
      uint32_t s_carry = 0;
      CT m_carry = 0;
      for (int i0 = 0; i0 < nk; i0 += cap) {
        const int i_end = min(nk - 1, i0 + cap - 1);
        const bool last_piece = i_end == nk - 1;
        if (ndesc + (i_end - i0 + 2) > DESC) flush();
        // canonical P-mer codes of this lane's positions
        const int x0 = i0 + lane * R;
        CT c[R];
#pragma unroll
        for (int j = 0; j < R; ++j) c[j] = kInf;
        if (x0 < nP) {
          const uint64_t hw = win(o + (uint64_t)x0);
          if (!two_win) {
            const uint64_t rh = revcomp32(hw);
#pragma unroll
            for (int j = 0; j < R; ++j) {
              const CT f = (CT)(hw >> (64 - 2 * (j + P))) & maskP;
              const CT r = (CT)(rh >> (2 * j)) & maskP;
              if (x0 + j < nP) c[j] = tmin(f, r);
            }
          } else {
            const uint64_t lw = win(o + (uint64_t)x0 + 32u);
            const uint64_t rh = revcomp32(hw), rl = revcomp32(lw);  // 128-bit rc = rl : rh
#pragma unroll
            for (int j = 0; j < R; ++j) {
              const uint64_t top = j ? (hw << (2 * j)) | (lw >> (64 - 2 * j)) : hw;
              const uint64_t bot = j ? (rh >> (2 * j)) | (rl << (64 - 2 * j)) : rh;
              const CT f = (CT)(top >> (64 - 2 * P)) & maskP;
              const CT r = (CT)bot & maskP;
              if (x0 + j < nP) c[j] = tmin(f, r);
            }
          }
        }
        CT pre[R], suf[R];
        pre[0] = c[0];
#pragma unroll
        for (int j = 1; j < R; ++j) pre[j] = tmin(pre[j - 1], c[j]);
        suf[R - 1] = c[R - 1];
#pragma unroll
        for (int j = R - 2; j >= 0; --j) suf[j] = tmin(c[j], suf[j + 1]);
        // T[k][l] = min of the lane minima of lanes l .. l + 2^k - 1 (clamped at lane 31)
        CT T[5];
        T[0] = pre[R - 1];
#pragma unroll
        for (int k = 1; k < 5; ++k) {
          T[k] = T[k - 1];
          if ((1 << k) <= Dmax) T[k] = tmin(T[k - 1], (CT)__shfl_down_sync(kFull, T[k - 1], 1 << (k - 1)));
        }
        // Definition 1: minimizer of K-mer i0 + lane R + j
        CT m[R];
#pragma unroll
        for (int j = 0; j < R; ++j) {
          const int q = j + w - 1, d = q / R, e = q - d * R;
          if (d == 0) {
            CT v = kInf;
#pragma unroll
            for (int u = 0; u < R; ++u)
              if (u >= j && u <= q) v = tmin(v, c[u]);
            m[j] = v;
          } else {
            CT pe = pre[0];
#pragma unroll
            for (int u = 1; u < R; ++u)
              if (u == e) pe = pre[u];
            CT v = tmin(suf[j], (CT)__shfl_down_sync(kFull, pe, d));
            const int D = d - 1;
            if (D > 0) {
              const int kq = 31 - __clz(D);
              CT tk = T[0];
#pragma unroll
              for (int k = 1; k < 5; ++k)
                if (k == kq) tk = T[k];
              v = tmin(v, (CT)__shfl_down_sync(kFull, tk, 1));
              v = tmin(v, (CT)__shfl_down_sync(kFull, tk, 1 + D - (1 << kq)));
            }
            m[j] = v;
          }
        }
        // Definition 2: superkmer starts
        bool cont = false;
        if (i0 > 0) {  // a piece after the first: continue or close the carried superkmer
          cont = __shfl_sync(kFull, m[0], 0) == m_carry;
          if (!cont) {
            if (lane == 0) {
              sm.ds[ndesc] = s_carry;
              sm.de[ndesc] = (uint32_t)(i0 - 1);
              sm.dm[ndesc] = m_carry;
              sm.dt[ndesc] = (uint8_t)t;
            }
            ++ndesc;
          }
        }
        const CT prevm = __shfl_up_sync(kFull, m[R - 1], 1);
        uint32_t fl = 0;
#pragma unroll
        for (int j = 0; j < R; ++j) {
          const int i = x0 + j;
          const bool f = i <= i_end && ((lane == 0 && j == 0) || m[j] != (j == 0 ? prevm : m[j - 1]));
          fl |= (uint32_t)f << j;
        }
        const uint32_t am = __ballot_sync(kFull, fl != 0);  // lane 0 always has K-mer i0
        const uint32_t higher = lane == 31 ? 0u : (am >> (lane + 1)) << (lane + 1);
        const int ffj = fl ? __ffs(fl) - 1 : 0;
        const int nl = higher ? __ffs(higher) - 1 : 0;
        const int nl_j = __shfl_sync(kFull, ffj, nl);
        const int next_lane_start = higher ? i0 + nl * R + nl_j : -1;
        int rank = 0, nst = 0;
#pragma unroll
        for (int j = 0; j < R; ++j) {
          const uint32_t bj = __ballot_sync(kFull, (fl >> j) & 1u);
          rank += __popc(bj & lt_mask);
          nst += __popc(bj);
        }
        uint32_t s_last = 0;
        CT m_last = 0;
#pragma unroll
        for (int j = 0; j < R; ++j) {
          if ((fl >> j) & 1u) {
            const int i = x0 + j;
            const uint32_t rest = fl >> (j + 1);
            const int e = rest ? i + __ffs(rest) - 1 : (next_lane_start >= 0 ? next_lane_start - 1 : (last_piece ? i_end : -1));
            const uint32_t s = (lane == 0 && j == 0 && cont) ? s_carry : (uint32_t)i;
            if (e >= 0) {
              const int idx = ndesc + rank + __popc(fl & ((1u << j) - 1u));
              sm.ds[idx] = s;
              sm.de[idx] = (uint32_t)e;
              sm.dm[idx] = m[j];
              sm.dt[idx] = (uint8_t)t;
            }
            s_last = s;
            m_last = m[j];
          }
        }
        if (!last_piece) {  // the superkmer open at the piece's end: the warp's last start
          const int hl = 31 - __clz(am);
          s_carry = __shfl_sync(kFull, s_last, hl);
          m_carry = __shfl_sync(kFull, m_last, hl);
        }
        ndesc += last_piece ? nst : nst - 1;
      }
    }
    if (ndesc) flush();
    __syncwarp();  // the buffer is free for the copy of the chunk after next
    o_cur = o_nx;
    L_cur = L_nx;
    wlo_cur = wlo_nx;
    st_cur = st_nx;
  }
}

template <typename CT, int R, int KC, int PC, int DESC, int MINB>
static cudaError_t launch_msp_warp(const MspArgs& a, cudaStream_t stream) {
  const size_t smem = sizeof(WarpMspSmem<CT, DESC>) * kWarpMspWarps;
  auto fn = msp_warp_kernel<CT, R, KC, PC, DESC, MINB>;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kWarpMspThreads, smem) != cudaSuccess || per_sm < 1)
    per_sm = 1;
  const uint64_t chunks = (a.n_reads + 31) / 32, want = (chunks + kWarpMspWarps - 1) / kWarpMspWarps;
  const uint64_t cap = (uint64_t)dbg_sm_count() * per_sm;  // one resident wave, grid-stride over chunks
  const int grid = (int)(want < cap ? want : cap);
  fn<<<grid, kWarpMspThreads, smem, stream>>>(a);
  return cudaGetLastError();
}

// Compile-time (K, P) = (63, 19) for bumblebee (64-bit codes, 4 positions per lane), else runtime
// K, P with 4 positions per lane (w <= 128 for every K <= 127).  K = 31 with P = 11..15 never gets
// here: msp_block_kernel is faster for it (msp.cu).
static cudaError_t launch_msp_warp_any(const MspArgs& a, cudaStream_t stream) {
  if (a.k == 63 && a.p == 19) return launch_msp_warp<uint64_t, 4, 63, 19, 192, 4>(a, stream);
  return a.p <= 16 ? launch_msp_warp<uint32_t, 4, 0, 0, 384, 3>(a, stream)
                   : launch_msp_warp<uint64_t, 4, 0, 0, 256, 3>(a, stream);
}

}  // namespace dbg
