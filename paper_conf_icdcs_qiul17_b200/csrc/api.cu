// api.cu -- host side of libdbg.so: sizes, the host 2-bit encoder (row a0) and
// status handling.  See include/dbg.h for the contract of every entry point.
#include <cmath>
#include <cstdio>
#include <cstring>

#include "dbg_device.cuh"

using namespace dbg;

static_assert(sizeof(dbg_graph_header) == 64, "graph file header is 64 bytes");
static const char kGraphMagic[8] = {'P', 'H', 'D', 'B', 'G', 0, 0, 1};

extern "C" int dbg_abi_version(void) { return DBG_ABI_VERSION; }

extern "C" uint32_t dbg_record_words(const dbg_params* prm) {
  return prm ? record_words(prm->k) : 0u;
}

extern "C" uint32_t dbg_record_max_kmers(const dbg_params* prm) {
  return prm ? record_max_kmers(prm->k) : 0u;
}

// Two-level scatter workspace (msp.cu ts_*): cursors, offsets and tile counts of <= 4096 buckets.
extern "C" uint64_t dbg_scatter_work_words(const dbg_params* prm) {
  if (!prm || prm->num_partitions < 1) return 0;
  const int64_t np = (int64_t)prm->num_partitions * (prm->refine > 1 ? prm->refine : 1);
  int s = 0;
  while (s < 12 && ((np + (1ll << s) - 1) >> s) > 2048) ++s;  // msp.cu ts_shift's rule
  const uint64_t nb = (uint64_t)((np + (1ll << s) - 1) >> s);
  return 3 * nb + 2;
}

// Sec. IV-A: "we use [N^i_kmer] with a load ratio alpha to set the
// hash table size as lambda/(4 alpha) N^i_kmer"; lambda = 2, alpha = 0.5 by
// default, which makes the capacity N^i_kmer (Table II).
// The same double-precision expression runs on the device in dbg_table_plan.
extern "C" uint64_t dbg_table_capacity(const dbg_params* prm, uint64_t n_kmers) {
  if (!prm || n_kmers == 0 || !(prm->lambda > 0.f) || !(prm->alpha > 0.f)) return 0;
  const double ratio = (double)prm->lambda / (4.0 * (double)prm->alpha);
  const double c = std::ceil(ratio * (double)n_kmers);
  return c < 1.0 ? 1ull : (uint64_t)c;
}

extern "C" uint32_t dbg_slot_bytes(const dbg_params* prm);

extern "C" uint64_t dbg_table_bytes(const dbg_params* prm, uint64_t n_kmers) {
  if (!prm || prm->k < 1 || prm->k > 127) return 0;
  return dbg_table_capacity(prm, n_kmers) * (uint64_t)dbg_slot_bytes(prm);
}

extern "C" uint64_t dbg_packed_words(uint64_t n_bases) { return (n_bases + 31) / 32 + 1; }

// Sec. II-A: characters are transformed into {A,C,G,T}, unknown
// bases to A; Sec. III-B: 2 bits per base.
extern "C" dbg_status dbg_encode_ascii(const char* seq, uint64_t n_bases, uint64_t* h_words) {
  if (!h_words || (n_bases && !seq)) return DBG_EINVAL;
  uint8_t lut[256];
  memset(lut, 0, sizeof(lut));  // reading B: anything else -> A
  lut['C'] = lut['c'] = 1;
  lut['G'] = lut['g'] = 2;
  lut['T'] = lut['t'] = 3;
  const uint64_t nw = dbg_packed_words(n_bases);
  const unsigned char* s = reinterpret_cast<const unsigned char*>(seq);
  const uint64_t full = n_bases / 32;
  for (uint64_t w = 0; w < full; ++w) {
    uint64_t v = 0;
    const unsigned char* p = s + 32 * w;
    for (int t = 0; t < 32; ++t) v = (v << 2) | lut[p[t]];
    h_words[w] = v;
  }
  for (uint64_t w = full; w < nw; ++w) {
    uint64_t v = 0;
    for (int t = 0; t < 32; ++t) {
      const uint64_t i = 32 * w + t;
      v = (v << 2) | (i < n_bases ? lut[s[i]] : 0u);
    }
    h_words[w] = v;
  }
  return DBG_OK;
}

// Row f4 graph writer: the paper writes the constructed subgraphs to an output
// graph file.  Format (little endian): a 64-byte
// header {char magic[8] = "PHDBG\0\0\1"; u32 k, p, num_partitions, min_count;
// u64 n_vertices; u64 reserved[4]} followed by n_vertices dbg_vertex records.
// append != 0 adds records to an existing file and updates its count.
extern "C" dbg_status dbg_write_graph(const char* path, const dbg_params* prm, const dbg_vertex* h_vertices,
                                      uint64_t n, int append) {
  if (!path || !prm || (n && !h_vertices)) return DBG_EINVAL;
  dbg_graph_header h;
  memset(&h, 0, sizeof(h));
  FILE* f = nullptr;
  if (append) f = fopen(path, "r+b");
  if (f) {
    if (fread(&h, sizeof(h), 1, f) != 1 || memcmp(h.magic, kGraphMagic, 8) != 0 || h.k != (uint32_t)prm->k) {
      fclose(f);
      return DBG_EINVAL;
    }
    if (fseek(f, 0, SEEK_END) != 0) {
      fclose(f);
      return DBG_EINVAL;
    }
  } else {
    f = fopen(path, "wb");
    if (!f) return DBG_EINVAL;
    memcpy(h.magic, kGraphMagic, 8);
    h.k = (uint32_t)prm->k;
    h.p = (uint32_t)prm->p;
    h.num_partitions = (uint32_t)prm->num_partitions;
    h.min_count = prm->min_count;
    if (fwrite(&h, sizeof(h), 1, f) != 1) {
      fclose(f);
      return DBG_EINVAL;
    }
  }
  bool ok = n == 0 || fwrite(h_vertices, sizeof(dbg_vertex), n, f) == n;
  h.n_vertices += n;
  ok = ok && fseek(f, 0, SEEK_SET) == 0 && fwrite(&h, sizeof(h), 1, f) == 1;
  ok = (fclose(f) == 0) && ok;
  return ok ? DBG_OK : DBG_EINVAL;
}

extern "C" dbg_status dbg_sync_status(const uint32_t* d_status, cudaStream_t stream) {
  if (!d_status) return DBG_EINVAL;
  uint32_t h = 0;
  if (cudaMemcpyAsync(&h, d_status, sizeof(h), cudaMemcpyDeviceToHost, stream) != cudaSuccess)
    return DBG_ECUDA;
  if (cudaStreamSynchronize(stream) != cudaSuccess) return DBG_ECUDA;
  if (h & kStatusTableFull) return DBG_ETABLEFULL;
  if (h & (kStatusNoSpace | 4u)) return DBG_ENOSPACE;
  return DBG_OK;
}

extern "C" const char* dbg_status_string(dbg_status s) {
  switch (s) {
    case DBG_OK: return "ok";
    case DBG_EINVAL: return "invalid argument";
    case DBG_ENOSPACE: return "output buffer too small";
    case DBG_ETABLEFULL: return "hash table full (probe sequence wrapped)";
    case DBG_ECUDA: return "CUDA error";
  }
  return "unknown status";
}

// Multi-GPU emission (dbg_partition_set.d_peer_records): kernels of the current device write into
// the record buffers of the other GPUs through their IPC-mapped pointers, which needs peer access
// from this device to theirs (NVLink / NVSwitch).  Idempotent.
extern "C" dbg_status dbg_enable_peer_access(int32_t peer_device) {
  int cur = 0;
  if (cudaGetDevice(&cur) != cudaSuccess) return DBG_ECUDA;
  if (peer_device == cur) return DBG_OK;
  int can = 0;
  if (cudaDeviceCanAccessPeer(&can, cur, peer_device) != cudaSuccess) return DBG_ECUDA;
  if (!can) return DBG_EINVAL;
  const cudaError_t e = cudaDeviceEnablePeerAccess(peer_device, 0);
  if (e == cudaErrorPeerAccessAlreadyEnabled) {
    (void)cudaGetLastError();  // clear the (non-sticky) error
    return DBG_OK;
  }
  return e == cudaSuccess ? DBG_OK : DBG_ECUDA;
}
