// oracle/dbg_oracle.cpp -- CPU ORACLE. TEST INFRASTRUCTURE ONLY.
//
// Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
// --impl reference) may load this library.  The product path
// (paper_conf_icdcs_qiul17_b200/, include/dbg.h) never links, imports or calls
// it, and this file shares no code, header, table or constant generator with
// the CUDA path.
//
// What it computes: the De Bruijn graph of Definition 3 (PAPER.md L232-237,
// Sec. II-A) -- every canonical K-mer vertex with its multiplicity and the
// multiplicities of its 4 out-edges and 4 in-edges -- by the plain
// definition, one K-mer occurrence at a time, with one std::map per MSP
// partition.  MSP partitioning (Sec. III-B) never changes the graph;
// the oracle evaluates the partition id of every K-mer only so that tests can
// check per-partition placement.  Readings of ambiguous passages follow
// SURVEY.md Sec. 8(c) and DESIGN.md "Readings" (letters A..T below).
//
// Deliberately slow and obvious: strings are reverse-complemented character
// by character, every P-mer is encoded from characters (Definition 1: the
// canonical value of each P-mer, then the minimum over each K-mer's window),
// and counting goes through std::map.
//
// Parity pins for this file: tests/test_oracle_pins.py (Fig. 1 worked
// example, Python string brute force, (K+1)-mer closed form, invariants
// I1..I6, Fig. 4 encoding example; fmix64 by SMHasher's published
// MurmurHash3_x64_128 verification value; oracle_checksum by its per-field
// closed form over the pinned fmix64; the pid / key filters by the
// unfiltered graph restricted).
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <map>
#include <vector>
#include <string>
#include <thread>
#include <algorithm>

typedef unsigned __int128 u128;

extern "C" {

// One output vertex (Def. 3): canonical code split in two 64-bit halves,
// count = occurrences of v or rc(v) (reading L), out/in indexed A,C,G,T
// (reading J), pid = MSP partition (Sec. III-B, reading I).
typedef struct {
  uint64_t key_hi, key_lo;
  uint32_t count;
  uint32_t out[4];
  uint32_t in[4];
  uint32_t pid;
} oracle_vertex;

// One superkmer (Def. 2 + the two adjacency bases of Sec. III-B):
// K-mers start at read positions start .. start+n_kmers-1 of read `read`.
typedef struct {
  uint64_t read;
  uint64_t minimizer;   // canonical minimizer value (2P-bit code)
  uint32_t start;
  uint32_t n_kmers;
  uint32_t pid;
  uint32_t has_left;    // 1 iff S[start-1] exists (reading H)
  uint32_t has_right;   // 1 iff S[start+n_kmers-1+K] exists (reading H)
  uint32_t pad;
} oracle_superkmer;

}  // extern "C"

namespace {

// Sec. II-A: characters are mapped into {A,C,G,T}; unknown bases
// become "A".  Reading B: lower case is treated as upper case.
char normalise(char c) {
  switch (c) {
    case 'A': case 'a': return 'A';
    case 'C': case 'c': return 'C';
    case 'G': case 'g': return 'G';
    case 'T': case 't': return 'T';
    default: return 'A';
  }
}

// Reading A: A<C<G<T, 2-bit codes A=0 C=1 G=2 T=3 (Sec. III-B,
// Fig. 4).
uint32_t code_of(char c) {
  switch (c) {
    case 'A': return 0;
    case 'C': return 1;
    case 'G': return 2;
    default: return 3;  // 'T' (input is normalised)
  }
}

char complement(char c) {
  switch (c) {
    case 'A': return 'T';
    case 'C': return 'G';
    case 'G': return 'C';
    default: return 'A';
  }
}

// Reverse complement of a string (Sec. II-A).
std::string reverse_complement(const std::string& s) {
  std::string r(s.size(), 'A');
  for (size_t t = 0; t < s.size(); ++t) r[s.size() - 1 - t] = complement(s[t]);
  return r;
}

// enc(x): first base most significant, so numeric order of codes equals the
// lexicographic order of equal-length strings (reading A).
u128 encode(const std::string& s) {
  u128 v = 0;
  for (char c : s) v = (v << 2) | (u128)code_of(c);
  return v;
}

// Reading I: the "hash bit value ... modulo the number of partitions"
// (Sec. III-B) is MurmurHash3's 64-bit finaliser fmix64.
uint64_t fmix64(uint64_t k) {
  k ^= k >> 33;
  k *= 0xff51afd7ed558ccdULL;
  k ^= k >> 33;
  k *= 0xc4ceb9fe1a85ec53ULL;
  k ^= k >> 33;
  return k;
}

// Definition 1 (L221-225) with reading D (canonical: a P-mer and its reverse
// complement are the same candidate) and reading E (plain lexicographic
// order): minimum over j in [i, i+K-P] of min(enc(s_j), enc(rc(s_j))).
uint64_t canonical_minimizer(const std::string& read, size_t i, int K, int P) {
  u128 best = ~(u128)0;
  for (size_t j = i; j + P <= i + K; ++j) {
    std::string s = read.substr(j, P);
    u128 f = encode(s);
    u128 r = encode(reverse_complement(s));
    u128 c = f < r ? f : r;
    if (c < best) best = c;
  }
  return (uint64_t)best;  // P <= 31 so the code fits 62 bits
}

// Definition 1 written in its two steps: first every
// P-mer position j of the read gets its canonical value
// c_j = min(enc(S[j..j+P-1]), enc(rc(S[j..j+P-1]))) (reading D), each encoded
// from characters as above; then the minimizer of the K-mer at i is
// min_{j in [i, i+K-P]} c_j (window_minimum).  The same values as
// canonical_minimizer(S, i, K, P), without re-encoding each P-mer K-P+1 times.
std::vector<uint64_t> canonical_pmer_values(const std::string& read, int P) {
  std::vector<uint64_t> c;
  for (size_t j = 0; j + P <= read.size(); ++j) {
    u128 f = 0, r = 0;
    for (int t = 0; t < P; ++t) f = (f << 2) | (u128)code_of(read[j + t]);  // enc(s_j)
    for (int t = P - 1; t >= 0; --t)                                          // enc(rc(s_j))
      r = (r << 2) | (u128)code_of(complement(read[j + t]));
    c.push_back((uint64_t)(f < r ? f : r));
  }
  return c;
}

uint64_t window_minimum(const std::vector<uint64_t>& c, size_t i, int K, int P) {
  uint64_t best = ~(uint64_t)0;
  for (size_t j = i; j <= i + (size_t)(K - P); ++j)
    if (c[j] < best) best = c[j];
  return best;
}

uint32_t partition_of(uint64_t minimizer, int NP) {
  return (uint32_t)(fmix64(minimizer) % (uint64_t)NP);
}

struct Rec {
  uint32_t count = 0;
  uint32_t out[4] = {0, 0, 0, 0};
  uint32_t in[4] = {0, 0, 0, 0};
};

typedef std::map<u128, Rec> PartitionMap;

std::string read_string(const char* seq, const uint64_t* offs, uint64_t r) {
  std::string s(seq + offs[r], seq + offs[r + 1]);
  for (char& c : s) c = normalise(c);
  return s;
}

// The per-occurrence update of SURVEY.md Sec. 8(c) steps 1-7 (readings J, K):
// for K-mer x = S[i..i+K-1], y = rc(x): if x <= y the vertex is x in forward
// orientation, its successor base S[i+K] is an out-edge and its predecessor
// S[i-1] an in-edge; otherwise the vertex is y, and the successor c becomes
// the in-edge comp(c) and the predecessor c the out-edge comp(c).
void add_occurrence(const std::string& S, size_t i, int K, PartitionMap& map) {
  std::string x = S.substr(i, K);
  u128 fx = encode(x);
  u128 ry = encode(reverse_complement(x));
  bool fwd = fx <= ry;
  u128 v = fwd ? fx : ry;
  Rec& r = map[v];
  r.count += 1;
  bool has_pred = i > 0;
  bool has_succ = i + K < S.size();
  if (fwd) {
    if (has_succ) r.out[code_of(S[i + K])] += 1;
    if (has_pred) r.in[code_of(S[i - 1])] += 1;
  } else {
    if (has_succ) r.in[3 - code_of(S[i + K])] += 1;
    if (has_pred) r.out[3 - code_of(S[i - 1])] += 1;
  }
}

}  // namespace

extern "C" {

int oracle_abi_version(void) { return 1; }

uint64_t oracle_fmix64(uint64_t k) { return fmix64(k); }

// Canonical code of one K-mer given as characters (test helper).
void oracle_canonical(const char* kmer, int K, uint64_t* hi, uint64_t* lo) {
  std::string x(kmer, kmer + K);
  for (char& c : x) c = normalise(c);
  u128 fx = encode(x), ry = encode(reverse_complement(x));
  u128 v = fx <= ry ? fx : ry;
  *hi = (uint64_t)(v >> 64);
  *lo = (uint64_t)v;
}

// Canonical minimizer of the K-mer S[0..K-1] given as characters (test helper).
uint64_t oracle_kmer_minimizer(const char* kmer, int K, int P) {
  std::string x(kmer, kmer + K);
  for (char& c : x) c = normalise(c);
  return canonical_minimizer(x, 0, K, P);
}

// The graph.  Returns 0 on success, 1 on invalid arguments, 2 if a vertex
// was found in two partitions (violates Sec. III-B), 3 on OOM.
// pid_filter: NULL for all partitions, else one byte per partition (nonzero =
// keep); key_filter: NULL, or n_keys canonical codes as (hi, lo) pairs sorted
// ascending -- only those vertices are counted.  Both are for sampled parity
// at full size; they drop occurrences, never change the per-occurrence rule.
// *out is malloc'ed; release it with oracle_free.  Records are sorted
// ascending by the 2K-bit code (reading Q).
int oracle_graph_filtered(const char* seq, const uint64_t* offs, uint64_t n_reads, int K,
                          int P, int NP, int n_threads, const uint8_t* pid_filter,
                          const uint64_t* key_filter, uint64_t n_keys,
                          oracle_vertex** out, uint64_t* n_out) {
  *out = nullptr;
  *n_out = 0;
  if (K < 1 || K > 63 || P < 1 || P > K || P > 31 || NP < 1) return 1;
  if (n_threads < 1) n_threads = 1;
  if ((uint64_t)n_threads > n_reads && n_reads > 0) n_threads = (int)n_reads;
  if (n_reads == 0) n_threads = 1;

  // Phase 1: read ranges in parallel, one std::map per partition per thread.
  std::vector<std::vector<PartitionMap>> maps(n_threads, std::vector<PartitionMap>(NP));
  auto work = [&](int t) {
    uint64_t r0 = n_reads * t / n_threads, r1 = n_reads * (t + 1) / n_threads;
    for (uint64_t r = r0; r < r1; ++r) {
      std::string S = read_string(seq, offs, r);
      if (S.size() < (size_t)K) continue;  // reading N: no K-mers
      const std::vector<uint64_t> c = canonical_pmer_values(S, P);
      for (size_t i = 0; i + K <= S.size(); ++i) {
        const uint32_t pid = partition_of(window_minimum(c, i, K, P), NP);
        if (pid_filter && !pid_filter[pid]) continue;
        if (key_filter) {
          std::string x = S.substr(i, K);
          u128 fx = encode(x), ry = encode(reverse_complement(x));
          u128 v = fx <= ry ? fx : ry;
          uint64_t hi = (uint64_t)(v >> 64), lo = (uint64_t)v;
          uint64_t a = 0, b = n_keys;  // binary search in the sorted (hi, lo) list
          while (a < b) {
            uint64_t m = (a + b) / 2;
            uint64_t mh = key_filter[2 * m], ml = key_filter[2 * m + 1];
            if (mh < hi || (mh == hi && ml < lo)) a = m + 1;
            else b = m;
          }
          if (a == n_keys || key_filter[2 * a] != hi || key_filter[2 * a + 1] != lo) continue;
        }
        add_occurrence(S, i, K, maps[t][pid]);
      }
    }
  };
  {
    std::vector<std::thread> th;
    for (int t = 1; t < n_threads; ++t) th.emplace_back(work, t);
    work(0);
    for (auto& x : th) x.join();
  }
  // Phase 2: merge the per-thread maps of each partition (sum of counts).
  for (int t = 1; t < n_threads; ++t)
    for (int p = 0; p < NP; ++p) {
      for (auto& kv : maps[t][p]) {
        Rec& d = maps[0][p][kv.first];
        d.count += kv.second.count;
        for (int c = 0; c < 4; ++c) {
          d.out[c] += kv.second.out[c];
          d.in[c] += kv.second.in[c];
        }
      }
      PartitionMap().swap(maps[t][p]);
    }
  uint64_t n = 0;
  for (int p = 0; p < NP; ++p) n += maps[0][p].size();
  oracle_vertex* v = (oracle_vertex*)malloc(sizeof(oracle_vertex) * (n ? n : 1));
  if (!v) return 3;
  uint64_t w = 0;
  for (int p = 0; p < NP; ++p)
    for (auto& kv : maps[0][p]) {
      oracle_vertex& o = v[w++];
      o.key_hi = (uint64_t)(kv.first >> 64);
      o.key_lo = (uint64_t)kv.first;
      o.count = kv.second.count;
      for (int c = 0; c < 4; ++c) {
        o.out[c] = kv.second.out[c];
        o.in[c] = kv.second.in[c];
      }
      o.pid = (uint32_t)p;
    }
  std::sort(v, v + n, [](const oracle_vertex& a, const oracle_vertex& b) {
    return a.key_hi != b.key_hi ? a.key_hi < b.key_hi : a.key_lo < b.key_lo;
  });
  for (uint64_t i = 1; i < n; ++i)
    if (v[i].key_hi == v[i - 1].key_hi && v[i].key_lo == v[i - 1].key_lo) {
      free(v);
      return 2;
    }
  *out = v;
  *n_out = n;
  return 0;
}

int oracle_graph(const char* seq, const uint64_t* offs, uint64_t n_reads, int K, int P, int NP,
                 int n_threads, const uint8_t* pid_filter, oracle_vertex** out, uint64_t* n_out) {
  return oracle_graph_filtered(seq, offs, n_reads, K, P, NP, n_threads, pid_filter, nullptr, 0,
                               out, n_out);
}

// MSP diagnostics (Sec. III-B): per read, the K-mers' canonical minimizers
// m_i, superkmers = maximal runs of consecutive K-mers with equal m_i
// (Def. 2, reading G), each with its partition id and adjacency-base flags.
int oracle_msp(const char* seq, const uint64_t* offs, uint64_t n_reads, int K, int P,
               int NP, oracle_superkmer** out, uint64_t* n_out) {
  *out = nullptr;
  *n_out = 0;
  if (K < 1 || K > 63 || P < 1 || P > K || P > 31 || NP < 1) return 1;
  std::vector<oracle_superkmer> sk;
  for (uint64_t r = 0; r < n_reads; ++r) {
    std::string S = read_string(seq, offs, r);
    if (S.size() < (size_t)K) continue;
    size_t nk = S.size() - K + 1;
    std::vector<uint64_t> m(nk);
    for (size_t i = 0; i < nk; ++i) m[i] = canonical_minimizer(S, i, K, P);
    size_t s = 0;
    for (size_t i = 1; i <= nk; ++i) {
      if (i == nk || m[i] != m[s]) {
        oracle_superkmer o;
        o.read = r;
        o.minimizer = m[s];
        o.start = (uint32_t)s;
        o.n_kmers = (uint32_t)(i - s);
        o.pid = partition_of(m[s], NP);
        o.has_left = s > 0 ? 1 : 0;
        o.has_right = (i - 1 + K < S.size()) ? 1 : 0;
        o.pad = 0;
        sk.push_back(o);
        s = i;
      }
    }
  }
  oracle_superkmer* v = (oracle_superkmer*)malloc(sizeof(oracle_superkmer) * (sk.size() ? sk.size() : 1));
  if (!v) return 3;
  if (!sk.empty()) memcpy(v, sk.data(), sizeof(oracle_superkmer) * sk.size());
  *out = v;
  *n_out = sk.size();
  return 0;
}

// Order-independent checksum over records: per record
// h = 0, then h = fmix64(h ^ field) over key_hi, key_lo, count, out[0..3],
// in[0..3]; the checksum is the sum of h modulo 2^64.
uint64_t oracle_checksum(const oracle_vertex* v, uint64_t n) {
  uint64_t sum = 0;
  for (uint64_t i = 0; i < n; ++i) {
    uint64_t f[11] = {v[i].key_hi, v[i].key_lo, v[i].count,
                      v[i].out[0], v[i].out[1], v[i].out[2], v[i].out[3],
                      v[i].in[0], v[i].in[1], v[i].in[2], v[i].in[3]};
    uint64_t h = 0;
    for (int t = 0; t < 11; ++t) h = fmix64(h ^ f[t]);
    sum += h;
  }
  return sum;
}

// Row f3 (K up to 127, keys of up to four 64-bit words): the same definition,
// with the vertex held as its canonical string (std::map<std::string, Rec> per
// partition; string order = lexicographic order = numeric order of the codes,
// reading A).  The code of a vertex is sum_i code(v_i) 4^(K-1-i) as a 256-bit
// integer, written as four 64-bit words, most significant first.
typedef struct {
  uint64_t key[4];
  uint32_t count;
  uint32_t out[4];
  uint32_t in[4];
  uint32_t pid;
} oracle_vertex_wide;

int oracle_graph_wide(const char* seq, const uint64_t* offs, uint64_t n_reads, int K, int P, int NP,
                      oracle_vertex_wide** out, uint64_t* n_out) {
  *out = nullptr;
  *n_out = 0;
  if (K < 1 || K > 127 || P < 1 || P > K || P > 31 || NP < 1) return 1;
  std::vector<std::map<std::string, Rec>> maps(NP);
  for (uint64_t r = 0; r < n_reads; ++r) {
    std::string S = read_string(seq, offs, r);
    if (S.size() < (size_t)K) continue;  // reading N
    for (size_t i = 0; i + K <= S.size(); ++i) {
      const uint32_t pid = partition_of(canonical_minimizer(S, i, K, P), NP);
      const std::string x = S.substr(i, K), y = reverse_complement(x);
      const bool fwd = x <= y;
      Rec& rec = maps[pid][fwd ? x : y];
      rec.count += 1;
      const bool has_pred = i > 0, has_succ = i + K < S.size();
      if (fwd) {
        if (has_succ) rec.out[code_of(S[i + K])] += 1;
        if (has_pred) rec.in[code_of(S[i - 1])] += 1;
      } else {
        if (has_succ) rec.in[3 - code_of(S[i + K])] += 1;
        if (has_pred) rec.out[3 - code_of(S[i - 1])] += 1;
      }
    }
  }
  std::map<std::string, std::pair<Rec, uint32_t>> all;  // sorted by the canonical string
  for (int p = 0; p < NP; ++p)
    for (auto& kv : maps[p]) {
      if (all.count(kv.first)) return 2;  // a vertex in two partitions
      all[kv.first] = std::make_pair(kv.second, (uint32_t)p);
    }
  oracle_vertex_wide* v = (oracle_vertex_wide*)malloc(sizeof(oracle_vertex_wide) * (all.size() ? all.size() : 1));
  if (!v) return 3;
  uint64_t w = 0;
  for (auto& kv : all) {
    oracle_vertex_wide& o = v[w++];
    memset(o.key, 0, sizeof(o.key));
    const std::string& t = kv.first;
    for (int i = 0; i < K; ++i) {  // base i is bit pair 2(K-1-i) of the 256-bit code
      const int bit = 2 * (K - 1 - i);
      o.key[3 - bit / 64] |= (uint64_t)code_of(t[i]) << (bit % 64);
    }
    o.count = kv.second.first.count;
    for (int c = 0; c < 4; ++c) {
      o.out[c] = kv.second.first.out[c];
      o.in[c] = kv.second.first.in[c];
    }
    o.pid = kv.second.second;
  }
  *out = v;
  *n_out = all.size();
  return 0;
}

void oracle_free(void* p) { free(p); }

}  // extern "C"
