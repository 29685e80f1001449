/*
 * dbg.h -- C ABI of the B200 hot path of ParaHash (Qiu & Luo, ICDCS 2017):
 * MSP partitioning of reads into superkmer partitions, then one shared
 * open-addressing hash table of <canonical K-mer, in/out edge multiplicities>
 * per partition.  Citations "P:L<a>-<b>" are lines of the paper text
 * (PAPER.md); readings A..T are listed in DESIGN.md Sec. 2.
 *
 * Conventions (all calls):
 *  - The library never allocates or frees device memory: the caller (the
 *    Python binding uses PyTorch tensors) owns every buffer and passes device
 *    pointers ("d_" prefix) or host pointers ("h_" prefix).
 *  - Device calls are stream-ordered and asynchronous; they validate their
 *    arguments on the host and return before any launch on error.  Launch
 *    failures return DBG_ECUDA.  Device-side conditions (table overflow,
 *    output overflow) are recorded in a caller-owned uint32 status word and
 *    reported by dbg_sync_status, the only call that synchronizes.
 *  - Thread-safe across distinct buffers; one host thread per device.
 *  - K must be odd (reading C), 1 <= K <= 127; 1 <= P <= min(K, 31).  K > 63
 *    (row f3: four-word keys, the paper's empty/locked/occupied protocol) runs
 *    only through the resident tables: dbg_msp_partition[_range],
 *    dbg_table_plan, dbg_hash_build, dbg_extract_graph (dbg_vertex_wide
 *    output); fine_p must be 0 or P; the on-chip, sort and checksum
 *    calls return DBG_EINVAL;
 *    1 <= num_partitions * refine <= 16,777,215 (2^24 - 1, the record header's pid field).  Every per-partition array
 *    and pid range below is in FINE partitions (NP * refine of them); only
 *    dbg_vertex.pid reports the paper's partition (fine pid mod NP).  Reads shorter than K contribute
 *    nothing and are not an error (reading N).
 */
#ifndef PARAHASH_DBG_H
#define PARAHASH_DBG_H

#include <stdint.h>
#include <cuda_runtime_api.h>

#ifdef __cplusplus
extern "C" {
#endif

#define DBG_ABI_VERSION 12

#if defined(__GNUC__)
#define DBG_API __attribute__((visibility("default")))
#else
#define DBG_API
#endif

typedef enum {
  DBG_OK = 0,
  DBG_EINVAL = 1,      /* invalid argument (nothing launched) */
  DBG_ENOSPACE = 2,    /* output buffer too small (count still written) */
  DBG_ETABLEFULL = 3,  /* a probe sequence wrapped: table unusable, rebuild larger (reading O) */
  DBG_ECUDA = 4        /* CUDA launch / runtime error */
} dbg_status;

/* Parameters of Sec. IV-A and Sec. V-A. */
typedef struct {
  int32_t k;              /* K-mer length, odd, 1..127 (readings C, T; > 63: row f3) */
  int32_t p;              /* minimizer length P, 1..min(k,31) (Def. 1) */
  int32_t num_partitions; /* NP, number of superkmer partitions (Sec. III-B) */
  float lambda;           /* average errors per read (Property 1); default 2 */
  float alpha;            /* load ratio; default 0.5 => capacity = N^i_kmer */
  int32_t refine;         /* F >= 1: the device works on NP*F fine partitions, fine pid =
                             fmix64(m) mod (NP*F), so a fine partition's table fits one SM;
                             the paper's partition of a vertex is fine pid mod NP (0 = 1) */
  int32_t smem_split;     /* on-chip path only: most CTAs (sub-tables) one partition too large
                             for a CTA table may be split over, 1..64; 1 = no splitting,
                             0 = default (32).  Larger partitions take the global tables. */
  int32_t fine_p;         /* minimizer length of the device's fine partitioning, 1..min(k,31);
                             0 = p.  Step 1 then cuts superkmers at changes of this minimizer
                             and fine pid = fmix64(its minimizer) mod (NP*F), which spreads the
                             K-mers of large genomes (few distinct P-mers per base) evenly;
                             dbg_vertex.pid stays the paper's partition, computed from the
                             vertex's canonical P-minimizer (reading V). */
  uint32_t min_count;     /* row f4: vertices with count < min_count are dropped at extraction
                             ("erroneous vertices can only be filtered by the number of their
                             occurrences after the graph is constructed"; reading R).
                             Their slots are still cleaned; dbg_stats and *d_n_out count only
                             the vertices written; edge counters of kept vertices are unchanged.
                             0 or 1 = keep every vertex (the unfiltered graph of Def. 3). */
} dbg_params;

/* One vertex of Definition 3: the canonical K-mer (the
 * lexicographically smaller of a K-mer and its reverse complement,
 * P:L197-201) as a 2K-bit code, first base most significant, split into two
 * 64-bit halves (K <= 31: kmer_hi = 0); its multiplicity; and the
 * multiplicities of its out- and in-edges indexed by the neighbour's extreme
 * base A,C,G,T in the vertex's canonical orientation
 * (reading J); pid = its MSP partition.  56 bytes. */
typedef struct {
  uint64_t kmer_hi, kmer_lo;
  uint32_t count;
  uint32_t out[4];
  uint32_t in[4];
  uint32_t pid;
} dbg_vertex;

/* Row f3 (K > 63, up to 127; Sec. III-C3): the same vertex with a
 * 2K-bit code of up to 254 bits in four 64-bit words, kmer[0] most
 * significant (the code is sum_i code(v_i) 4^(K-1-i)).  72 bytes.  Written by
 * dbg_extract_graph when K > 63 (d_out then points to dbg_vertex_wide
 * records and out_cap counts them). */
typedef struct {
  uint64_t kmer[4];
  uint32_t count;
  uint32_t out[4];
  uint32_t in[4];
  uint32_t pid;
} dbg_vertex_wide;

/* Totals (filled by the extraction calls); checksum = sum over vertices of
 * h, h = fmix64 chained over (kmer_hi, kmer_lo, count, out[0..3], in[0..3])
 * (SURVEY.md 8(d)), filled by dbg_checksum_vertices. */
typedef struct {
  uint64_t distinct, sum_count, sum_edges, checksum;
} dbg_stats;

/* Superkmer partitions (Sec. III-A Fig. 3) resident in HBM.
 * All arrays are device memory owned by the caller.  Records of partition i
 * occupy record slots [d_record_offset[i], d_record_offset[i+1]) of
 * d_records; one record is dbg_record_words() uint32 words:
 *   word 0: n_kmers (bits 0-5, <= 63) | has_left (bit 6) | has_right (bit 7) | fine pid (bits 8-31)
 *   words 1..: the bases S[s-has_left .. e+K-1+has_right], 2-bit, 16 per word,
 *              first base in the most significant bits (Sec. III-B).
 * A superkmer longer than the record holds is stored as consecutive pieces,
 * each with its own adjacency bases (the graph is unchanged).  Records are
 * first written in read order to d_staging (capacity staging_cap records),
 * then scattered into partition order. */
typedef struct {
  uint64_t* d_n_records;     /* [NP]   records per partition (pass 1) */
  uint64_t* d_n_kmers;       /* [NP]   N^i_kmer, K-mers per partition (pass 1; sizes tables) */
  uint64_t* d_record_offset; /* [NP+1] exclusive prefix sum of d_n_records (pass 1) */
  uint64_t* d_fill;          /* [NP]   scatter cursors (pass 2; zeroed by the call) */
  uint64_t* d_staged;        /* [1]    records reserved in d_staging (pass 1) */
  uint32_t* d_staging;       /* staging_cap records, read order (pass 1 output, pass 2 input) */
  uint64_t staging_cap;      /* capacity of d_staging in records */
  uint32_t* d_records;       /* d_record_offset[NP] records in partition order; NULL => pass 1 */
  uint32_t* d_scratch;       /* optional, staging_cap records (not aliasing d_staging or d_records):
                                with more than 8192 fine partitions pass 2 then scatters in two
                                counting-sort levels -- into buckets of 2^s consecutive partitions
                                (d_scratch), then within each bucket (d_records / the peers) --
                                each level ranking a tile of records in shared memory and
                                reserving once per (tile, bin); needs d_work.  NULL: one level,
                                one global rank atomic per record */
  /* Multi-GPU emission: with n_peers > 0, pass 2 writes
     each record of fine partition f into the partition buffer of f's owner GPU o -- the o with
     d_peer_bounds[o] <= f < d_peer_bounds[o+1] -- at record slot d_record_offset[f] + rank, i.e.
     straight into peer memory over NVLink (IPC-mapped device pointers).  d_record_offset must
     then hold dbg_exchange_plan's d_dest_offset; d_records is not written.  Both scatters
     support peers (the two-level one buckets locally from d_n_records, then writes the peers).
     n_peers = 0: local pass 2. */
  uint32_t* const* d_peer_records; /* [n_peers] device array of the owners' record buffers */
  const int32_t* d_peer_bounds;    /* [n_peers+1] device array, owner o owns [b[o], b[o+1]) */
  int32_t n_peers;
  uint64_t* d_work;          /* with d_scratch: dbg_scatter_work_words(prm) uint64 of caller memory
                                (bucket offsets, cursors and tile counts of the two-level scatter) */
} dbg_partition_set;

/* uint64 words of dbg_partition_set.d_work for the two-level scatter. */
DBG_API uint64_t dbg_scatter_work_words(const dbg_params* prm);

/* ---- sizes ------------------------------------------------------------ */
DBG_API int dbg_abi_version(void);
/* uint32 words per superkmer record for these params (4 for K <= 39, 8 for
 * K <= 63, 16 for K <= 127). */
DBG_API uint32_t dbg_record_words(const dbg_params* prm);
/* K-mers a record holds at most. */
DBG_API uint32_t dbg_record_max_kmers(const dbg_params* prm);
/* Bytes per hash-table slot: a key entry (dbg_key_bytes: 16 for K <= 31, 32
 * for K <= 63, 48 for K <= 127) plus a 32-byte counter record. */
DBG_API uint32_t dbg_slot_bytes(const dbg_params* prm);
DBG_API uint32_t dbg_key_bytes(const dbg_params* prm);
/* Table capacity for a partition with n_kmers K-mers: ceil(lambda/(4 alpha) * n_kmers)
 * (Sec. IV-A), at least 1 when n_kmers > 0 (Property 1 sizing). */
DBG_API uint64_t dbg_table_capacity(const dbg_params* prm, uint64_t n_kmers);
/* Bytes of the global (resident) hash table of such a partition: dbg_table_capacity slots of
 * dbg_slot_bytes each (the d_table block dbg_hash_build takes for it; Table II, P:L1005-1013,
 * prints the paper's analogue at 32 B per entry).  0 for invalid params. */
DBG_API uint64_t dbg_table_bytes(const dbg_params* prm, uint64_t n_kmers);
/* uint64 words of the packed 2-bit stream for n_bases bases, including one pad word. */
DBG_API uint64_t dbg_packed_words(uint64_t n_bases);

/* ---- a0: host encoder (Sec. II-A; Sec. III-B) ---- */
/* seq: n_bases ASCII characters (all reads concatenated).  Writes
 * dbg_packed_words(n_bases) words to h_words: base i at word i/32, bits
 * 63-2(i%32) .. 62-2(i%32); A=0 C=1 G=2 T=3, anything else -> A (reading A, B). */
DBG_API dbg_status dbg_encode_ascii(const char* seq, uint64_t n_bases, uint64_t* h_words);

/* ---- a2-a4: Step 1, MSP (Sec. III-B; Defs. 1-2) ------------
 * d_bases: packed stream (dbg_packed_words(total) words), d_offsets: [n_reads+1]
 * base offsets of the reads in the stream.
 * part->d_records == NULL: pass 1 -- zeroes and fills d_n_records, d_n_kmers,
 *   d_record_offset and *d_staged, and writes the records (read order) into
 *   d_staging while they fit.  The caller reads d_record_offset[NP] (or the
 *   sizes); if it exceeds staging_cap, it grows d_staging and repeats pass 1.
 * part->d_records != NULL: pass 2 -- scatters the staged records into
 *   partition order (d_record_offset[NP] records), through d_scratch when it is
 *   set (two levels; the order of the records inside a partition is not
 *   specified either way).
 * A caller may enqueue pass 2 and Step 2 before reading the sizes back: after a
 * staging overflow (*d_staged > staging_cap) pass 2 and
 * dbg_build_subgraphs_smem do nothing, and the caller grows d_staging and
 * repeats the step.  d_records then needs room for staging_cap records. */
DBG_API dbg_status dbg_msp_partition(const dbg_params* prm, const uint64_t* d_bases, uint64_t n_words,
                             const uint64_t* d_offsets, uint64_t n_reads,
                             const dbg_partition_set* part, cudaStream_t stream);

/* ---- f2: pass 1 over read batches and partition ranges (Sec. III-E)
 * As dbg_msp_partition pass 1 (part->d_records must be NULL), but only the
 * superkmers of fine partitions [pid_lo, pid_hi) are counted (d_n_records,
 * d_n_kmers) and staged; the others are dropped.  append != 0 keeps the
 * counters and *d_staged of the previous calls (the reads of this call are
 * another batch of the same input: its records go after the staged ones);
 * append == 0 zeroes them first.  d_record_offset is recomputed by every call
 * (it is final after the last batch).  Staging overflow behaves as in
 * dbg_msp_partition.  Pass 2 is dbg_msp_partition with d_records set.
 * With staging_cap = 0 the call only counts (a sizing pass over all batches
 * that chooses the partition ranges of the passes). */
DBG_API dbg_status dbg_msp_partition_range(const dbg_params* prm, const uint64_t* d_bases, uint64_t n_words,
                                   const uint64_t* d_offsets, uint64_t n_reads,
                                   const dbg_partition_set* part, int32_t pid_lo, int32_t pid_hi,
                                   int append, cudaStream_t stream);

/* ---- e: multi-GPU exchange plan (Sec. III-A) -----
 * world ranks split the reads by range; rank r's pass 1 gives its records per fine partition,
 * and d_counts[world * NP] holds every rank's d_n_records (gathered: rank q's row is
 * d_counts[q*NP .. q*NP+NP)).  Fine partition f is owned by the rank o with
 * d_bounds[o] <= f < d_bounds[o+1] (d_bounds: world+1 int32, device).  In the owner's buffer the
 * records are in partition order, and inside a partition in source-rank order.  Writes:
 *   d_dest_offset[NP]          where THIS rank's records of f start in owner(f)'s buffer (records;
 *                              pass 2 with peers uses it as d_record_offset);
 *   d_owned_n_records[NP]      sum over ranks of d_counts for the partitions this rank owns, 0
 *                              for the others;
 *   d_owned_n_kmers[NP]        d_kmers_sum (the K-mers per partition summed over ranks) for the
 *                              owned partitions, 0 for the others (may alias d_kmers_sum);
 *   d_owned_record_offset[NP+1] exclusive prefix sum of d_owned_n_records: the partition set of
 *                              this rank's Step 2 (its last entry = records this rank receives).
 * d_prefix: NP+1 uint64 and d_scratch: NP uint64 of caller memory (no alias with the outputs). */
DBG_API dbg_status dbg_exchange_plan(const dbg_params* prm, const uint64_t* d_counts, const uint64_t* d_kmers_sum,
                                     int32_t world, int32_t rank, const int32_t* d_bounds,
                                     uint64_t* d_dest_offset, uint64_t* d_owned_n_records,
                                     uint64_t* d_owned_n_kmers, uint64_t* d_owned_record_offset,
                                     uint64_t* d_prefix, uint64_t* d_scratch, cudaStream_t stream);

/* Peer access from the current device to peer_device (cudaDeviceEnablePeerAccess; already enabled
 * is not an error), needed before pass 2 writes into d_peer_records that live on other GPUs.
 * DBG_EINVAL if the devices cannot access each other. */
DBG_API dbg_status dbg_enable_peer_access(int32_t peer_device);

/* ---- a5: sizing (Property 1; Sec. IV-A) ----------------------
 * d_table_offset[NP+1] = exclusive prefix sum of dbg_table_capacity(N^i_kmer)
 * (in slots).  d_scratch: NP uint64 of caller memory for the multi-CTA scan
 * (e.g. the idle d_fill of the partition set), or NULL (one CTA: slow for
 * large NP). */
DBG_API dbg_status dbg_table_plan(const dbg_params* prm, const uint64_t* d_n_kmers,
                          uint64_t* d_table_offset, uint64_t* d_scratch, cudaStream_t stream);

/* ---- a5-a7 on-chip: Step 2 in shared memory (the hot path) ---------------
 * Every fine partition in [pid_begin, pid_end) whose table (capacity from Property 1, Sec. IV-A
 * P:L783-788) fits one CTA's shared memory -- at most dbg_smem_table_slots()
 * slots -- is built and extracted on chip: consecutive such partitions are
 * grouped so that a group's tables fill one CTA's table space; the CTA hashes
 * the group's records (shared-memory 64/128-bit CAS claims a key, shared-
 * memory atomics count the edges in 16-bit fields) and compacts the occupied
 * slots straight into d_out.  A partition with capacity c above the slots is
 * split over ns = ceil(1.25 c / slots) <= prm->smem_split CTAs
 * (dbg_smem_onchip): each reads all of its records and keeps the K-mers whose key hash
 * selects its sub-table (one vertex, one sub-table), so each CTA table holds
 * an expected <= 80% of its slots.  Counters on chip are 16-bit, so only
 * partitions with N^i_kmer <= 65535 (a bound on any of their vertex counts)
 * go on chip.  The other partitions are skipped here and left to the global-table path
 * (dbg_table_plan_split + dbg_hash_build_list + dbg_extract_graph).
 * d_work: dbg_smem_workspace_bytes() bytes of caller memory (the plan).
 * Output appends to d_out[*d_n_out ...] and accumulates *d_stats. */
DBG_API uint64_t dbg_smem_table_slots(const dbg_params* prm);
/* Where a partition with n_kmers K-mers is built: 1 = grouped on chip, ns >= 2
 * = split over ns CTAs, 0 = global tables (N^i_kmer > 65535, or ns > smem_split);
 * -1 for invalid params. */
DBG_API int32_t dbg_smem_onchip(const dbg_params* prm, uint64_t n_kmers);
DBG_API uint64_t dbg_smem_workspace_bytes(const dbg_params* prm);
DBG_API dbg_status dbg_build_subgraphs_smem(const dbg_params* prm, const dbg_partition_set* part,
                                    int32_t pid_begin, int32_t pid_end, void* d_work,
                                    uint64_t work_bytes, dbg_vertex* d_out, uint64_t out_cap,
                                    uint64_t* d_n_out, dbg_stats* d_stats, uint32_t* d_status,
                                    cudaStream_t stream);
/* As dbg_table_plan, but partitions built on chip (dbg_smem_onchip > 0) get
 * capacity 0, so resident tables cover only the rest. */
DBG_API dbg_status dbg_table_plan_split(const dbg_params* prm, const uint64_t* d_n_kmers,
                                uint64_t* d_table_offset, uint64_t* d_scratch, cudaStream_t stream);

/* ---- a6: Step 2 with resident tables (Sec. III-C) ------------
 * Inserts every K-mer occurrence of partitions [pid_begin, pid_end) into that
 * partition's table.  d_table holds the tables of all these partitions,
 * n = d_table_offset[pid_end] - d_table_offset[pid_begin] slots: first the n
 * key entries (dbg_key_bytes each), then n 32-byte counter records; partition
 * i owns slots [d_table_offset[i] - d_table_offset[pid_begin], ...) of both
 * arrays.  The table must be all-zero (memset once when allocated:
 * dbg_extract_graph zeroes every slot it reads, so an extracted table is
 * clean again).  Overflow sets bit 0 of *d_status (dbg_sync_status). */
DBG_API dbg_status dbg_hash_build(const dbg_params* prm, const dbg_partition_set* part, int32_t pid_begin,
                          int32_t pid_end, void* d_table, const uint64_t* d_table_offset,
                          uint32_t* d_status, cudaStream_t stream);

/* As dbg_hash_build for the table block of partitions [pid_begin, pid_end)
 * (d_table_offset from dbg_table_plan_split), but only for the n_pids listed
 * partitions (all inside the range): d_pids[n_pids] fine partition ids,
 * d_chunk_prefix[n_pids+1] the exclusive prefix sum of ceil(records of
 * d_pids[j] / 32).  Used for the partitions too large for the on-chip path. */
DBG_API dbg_status dbg_hash_build_list(const dbg_params* prm, const dbg_partition_set* part, int32_t pid_begin,
                               int32_t pid_end, const uint32_t* d_pids, const uint64_t* d_chunk_prefix,
                               int32_t n_pids, void* d_table, const uint64_t* d_table_offset,
                               uint32_t* d_status, cudaStream_t stream);

/* ---- a7: output (Def. 3) -------------------------------------
 * Compacts the occupied slots of resident tables (layout of dbg_hash_build)
 * into d_out[*d_n_out ...] (appends; the caller zeroes *d_n_out and *d_stats
 * once), accumulates *d_stats, and zeroes every slot it read (the table is
 * clean for the next dbg_hash_build).  Records beyond out_cap are dropped and
 * set bit 1 of *d_status (DBG_ENOSPACE; *d_n_out still counts them).
 * Record order is unspecified (reading S): use dbg_sort_vertices. */
DBG_API dbg_status dbg_extract_graph(const dbg_params* prm, void* d_table,
                             const uint64_t* d_table_offset, int32_t pid_begin, int32_t pid_end,
                             dbg_vertex* d_out, uint64_t out_cap, uint64_t* d_n_out,
                             dbg_stats* d_stats, uint32_t* d_status, cudaStream_t stream);

/* Sorts n vertices ascending by (kmer_hi, kmer_lo) (reading Q) from d_in to
 * d_out (distinct buffers) using a caller workspace of
 * dbg_sort_workspace_bytes(n) bytes. */
DBG_API uint64_t dbg_sort_workspace_bytes(const dbg_params* prm, uint64_t n);
DBG_API dbg_status dbg_sort_vertices(const dbg_params* prm, const dbg_vertex* d_in, dbg_vertex* d_out,
                             uint64_t n, void* d_workspace, uint64_t workspace_bytes,
                             cudaStream_t stream);

/* Adds the order-independent checksum of n vertex records (SURVEY.md 8(d):
 * per record h = fmix64 chained over kmer_hi, kmer_lo, count, out[0..3],
 * in[0..3]; the sum of h mod 2^64) to d_stats->checksum.  The extraction
 * calls fill distinct / sum_count / sum_edges only; this validation
 * statistic is computed apart from the path. */
DBG_API dbg_status dbg_checksum_vertices(const dbg_params* prm, const dbg_vertex* d_vertices, uint64_t n,
                                 dbg_stats* d_stats, cudaStream_t stream);

/* ---- f4: graph writer ---------------------------
 * Writes n host records (any order; sorted records from dbg_sort_vertices
 * give a sorted file) to the file at path: a 64-byte dbg_graph_header, then
 * the records.  append != 0 and an existing file with the same magic and K:
 * the records are appended and header.n_vertices updated (one call per
 * batch of partitions); otherwise the file is created or truncated.
 * DBG_EINVAL on a bad argument, an I/O error or a header mismatch. */
typedef struct {
  char magic[8];           /* "PHDBG\0\0\1" (format version 1) */
  uint32_t k, p, num_partitions, min_count;
  uint64_t n_vertices;
  uint64_t reserved[4];
} dbg_graph_header;
DBG_API dbg_status dbg_write_graph(const char* path, const dbg_params* prm, const dbg_vertex* h_vertices,
                           uint64_t n, int append);

/* Synchronizes the stream, then decodes *d_status: bit 0 -> DBG_ETABLEFULL,
 * bit 1 or 2 -> DBG_ENOSPACE; also returns DBG_ECUDA on a sticky CUDA error. */
DBG_API dbg_status dbg_sync_status(const uint32_t* d_status, cudaStream_t stream);

DBG_API const char* dbg_status_string(dbg_status s);

#ifdef __cplusplus
}
#endif
#endif /* PARAHASH_DBG_H */
