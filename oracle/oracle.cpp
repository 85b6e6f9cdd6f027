// oracle.cpp — TEST INFRASTRUCTURE ONLY.  A plain, slow, single-threaded, obviously correct
// CPU MapReduce that states what the libbmr hot path must compute.  Only tests/,
// __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg may load it.
// It shares no code, header, table or constant generator with the CUDA path
// (paper_conf_ipps_jim11_b200/csrc); it includes only the C++ standard library.
//
// Citations: "L<n>" = /root/reference/PAPER.md line n; "C-1"/"C-2"/"C-3 #k" = the readings in
// SURVEY.md §8(c), restated in DESIGN.md §3.
//
//   Generic semantics (C-1; "Map, Shuffle, Reduce ... <key,value> pairs"):
//     1. for each batch in call order, each record i: map_w(bytes[off[i], off[i+1]), global
//        offset batch_base + off[i]) appends (key bytes, value bytes) pairs;
//     2. Map-only (SM): the output is that list;
//     3. otherwise std::stable_sort by key (unsigned lexicographic bytes; a proper prefix sorts
//        first), walk equal-key runs, reduce_w(key, values);
//     4. canonicalise (keys ascending; II values ascending; SM/KM keys numeric ascending).
//   Workloads (C-2; "Word Count ... String Match ... Inverted Index ... KMeans"):
//     WC  word = maximal [0-9A-Za-z] run inside a record; emit (word, u32 1); reduce = u64 sum.
//     SM  every j with j+16 <= len and rec[j..j+16) == P: emit u64 global offset (overlaps count).
//     SML (SM per line, the paper's own output, L125 "search a line for the keyword; emit the
//         line if found"): a record with at least one such j emits the u64 global offset of its
//         first byte, once (Map-only).
//     KM  d_j = fmaf chain of (x_t - c_jt)^2 in fp32 RN, argmin with ties -> lowest j; emit
//         (u32 j, 32-B point); reduce: cnt (u64), sum in fp64, c'_j = (float)(sum/cnt),
//         empty cluster keeps c_j; output all k clusters.
//     II  every p with rec[p..p+9) == `<a href="`: q = first '"' at >= p+9 inside the record;
//         if q exists and q > p+9 emit (rec[p+9..q), u64 global offset of p+9); identity reduce
//         (values of a URL ascending).
// Built with -O2 -ffp-contract=off (no FMA contraction except the explicit std::fmaf).
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <string>
#include <utility>
#include <vector>

namespace {

enum { WC = 1, SM = 2, KM = 3, II = 4, SML = 5 };

struct Job {
  int workload = 0;
  uint8_t pattern[16] = {0};
  uint32_t k = 0;
  std::vector<float> centroids;                          // k x 8, row-major
  std::vector<std::pair<std::string, std::string>> pairs;  // intermediate (key, value)
  // canonical output
  std::vector<uint8_t> keys, vals;
  std::vector<uint64_t> key_off, val_off;
};

std::string u64_bytes(uint64_t v) { std::string s(8, '\0'); std::memcpy(&s[0], &v, 8); return s; }
std::string u32_bytes(uint32_t v) { std::string s(4, '\0'); std::memcpy(&s[0], &v, 4); return s; }
uint64_t bytes_u64(const std::string& s) { uint64_t v = 0; std::memcpy(&v, s.data(), 8); return v; }

bool is_word_byte(uint8_t c) {  // C-3 #1: [0-9A-Za-z], case-sensitive
  return (c >= '0' && c <= '9') || (c >= 'A' && c <= 'Z') || (c >= 'a' && c <= 'z');
}

// ---- user Map functions (C-2) ----
void map_wc(Job& J, const uint8_t* b, uint64_t len) {
  uint64_t i = 0;
  while (i < len) {
    if (is_word_byte(b[i])) {
      uint64_t j = i;
      while (j < len && is_word_byte(b[j])) ++j;
      J.pairs.emplace_back(std::string(reinterpret_cast<const char*>(b + i), j - i), u32_bytes(1));
      i = j;
    } else {
      ++i;
    }
  }
}

void map_sm(Job& J, const uint8_t* b, uint64_t len, uint64_t gpos) {
  if (len < 16) return;
  for (uint64_t j = 0; j + 16 <= len; ++j)
    if (std::memcmp(b + j, J.pattern, 16) == 0) J.pairs.emplace_back(u64_bytes(gpos + j), std::string());
}

void map_sml(Job& J, const uint8_t* b, uint64_t len, uint64_t gpos) {
  for (uint64_t j = 0; j + 16 <= len; ++j)
    if (std::memcmp(b + j, J.pattern, 16) == 0) {
      J.pairs.emplace_back(u64_bytes(gpos), std::string());
      return;
    }
}

void map_km(Job& J, const uint8_t* b, uint64_t len) {
  if (len != 32) return;  // fixed 32-B records (C-3 #23)
  float x[8];
  std::memcpy(x, b, 32);
  uint32_t best = 0;
  float best_d = 0.0f;
  for (uint32_t j = 0; j < J.k; ++j) {
    float d = 0.0f;
    for (int t = 0; t < 8; ++t) {
      float e = x[t] - J.centroids[j * 8 + t];
      d = std::fmaf(e, e, d);
    }
    if (j == 0 || d < best_d) { best = j; best_d = d; }  // strict <: ties -> lowest j
  }
  J.pairs.emplace_back(u32_bytes(best), std::string(reinterpret_cast<const char*>(b), 32));
}

void map_ii(Job& J, const uint8_t* b, uint64_t len, uint64_t gpos) {
  static const char kMarker[] = "<a href=\"";
  for (uint64_t p = 0; p + 9 <= len; ++p) {
    if (std::memcmp(b + p, kMarker, 9) != 0) continue;
    uint64_t q = p + 9;
    while (q < len && b[q] != '"') ++q;
    if (q < len && q > p + 9)
      J.pairs.emplace_back(std::string(reinterpret_cast<const char*>(b + p + 9), q - (p + 9)), u64_bytes(gpos + p + 9));
  }
}

bool key_less(const std::pair<std::string, std::string>& a, const std::pair<std::string, std::string>& b) {
  return std::lexicographical_compare(
      reinterpret_cast<const uint8_t*>(a.first.data()), reinterpret_cast<const uint8_t*>(a.first.data()) + a.first.size(),
      reinterpret_cast<const uint8_t*>(b.first.data()), reinterpret_cast<const uint8_t*>(b.first.data()) + b.first.size());
}

void push(Job& J, const std::string& k, const std::string& v) {
  J.keys.insert(J.keys.end(), k.begin(), k.end());
  J.key_off.push_back(J.keys.size());
  J.vals.insert(J.vals.end(), v.begin(), v.end());
  J.val_off.push_back(J.vals.size());
}

void reduce(Job& J) {
  J.keys.clear(); J.vals.clear();
  J.key_off.assign(1, 0); J.val_off.assign(1, 0);
  if (J.workload == SM || J.workload == SML) {  // Map-only; canonical = offsets ascending
    std::vector<uint64_t> o;
    o.reserve(J.pairs.size());
    for (auto& p : J.pairs) o.push_back(bytes_u64(p.first));
    std::sort(o.begin(), o.end());
    for (uint64_t v : o) push(J, u64_bytes(v), std::string());
    return;
  }
  std::stable_sort(J.pairs.begin(), J.pairs.end(), key_less);  // group by key (C-1 step 3)
  if (J.workload == KM) {
    std::vector<uint64_t> cnt(J.k, 0);
    std::vector<double> sum(static_cast<size_t>(J.k) * 8, 0.0);
    for (auto& p : J.pairs) {
      uint32_t j = 0;
      std::memcpy(&j, p.first.data(), 4);
      float x[8];
      std::memcpy(x, p.second.data(), 32);
      cnt[j] += 1;
      for (int t = 0; t < 8; ++t) sum[j * 8 + t] += static_cast<double>(x[t]);
    }
    for (uint32_t j = 0; j < J.k; ++j) {
      float c[8];
      for (int t = 0; t < 8; ++t)
        c[t] = cnt[j] ? static_cast<float>(sum[j * 8 + t] / static_cast<double>(cnt[j])) : J.centroids[j * 8 + t];
      std::string v(reinterpret_cast<const char*>(c), 32);
      v += u64_bytes(cnt[j]);
      push(J, u32_bytes(j), v);
    }
    return;
  }
  size_t i = 0;
  while (i < J.pairs.size()) {
    size_t e = i;
    while (e < J.pairs.size() && J.pairs[e].first == J.pairs[i].first) ++e;  // equal-key run
    if (J.workload == WC) {
      uint64_t s = 0;
      for (size_t r = i; r < e; ++r) { uint32_t v; std::memcpy(&v, J.pairs[r].second.data(), 4); s += v; }
      push(J, J.pairs[i].first, u64_bytes(s));
    } else {  // II: identity reduce, values ascending
      std::vector<uint64_t> o;
      for (size_t r = i; r < e; ++r) o.push_back(bytes_u64(J.pairs[r].second));
      std::sort(o.begin(), o.end());
      std::string v;
      for (uint64_t x : o) v += u64_bytes(x);
      push(J, J.pairs[i].first, v);
    }
    i = e;
  }
}

}  // namespace

extern "C" {

typedef struct {
  uint64_t n_keys;
  const uint8_t* keys; const uint64_t* key_offsets;
  const uint8_t* vals; const uint64_t* val_offsets;
} oracle_result;

void* oracle_create(int workload, const uint8_t* pattern16, uint32_t k, const float* centroids) {
  if (workload < WC || workload > SML) return nullptr;
  Job* J = new Job();
  J->workload = workload;
  if (pattern16) std::memcpy(J->pattern, pattern16, 16);
  if (workload == KM) {
    if (!centroids || k == 0) { delete J; return nullptr; }
    J->k = k;
    J->centroids.assign(centroids, centroids + static_cast<size_t>(k) * 8);
  }
  return J;
}

// records: host bytes; offsets: n+1 u64 (or NULL with stride > 0); batch_base: global byte
// offset of records[0].
int oracle_map(void* job, const uint8_t* records, const uint64_t* offsets, uint64_t n,
               uint32_t stride, uint64_t batch_base) {
  Job* J = static_cast<Job*>(job);
  if (!J || (n && !records) || (!offsets && stride == 0)) return 1;
  for (uint64_t i = 0; i < n; ++i) {
    uint64_t a = offsets ? offsets[i] : i * stride;
    uint64_t e = offsets ? offsets[i + 1] : (i + 1) * stride;
    const uint8_t* b = records + a;
    switch (J->workload) {
      case WC: map_wc(*J, b, e - a); break;
      case SM: map_sm(*J, b, e - a, batch_base + a); break;
      case SML: map_sml(*J, b, e - a, batch_base + a); break;
      case KM: map_km(*J, b, e - a); break;
      case II: map_ii(*J, b, e - a, batch_base + a); break;
    }
  }
  return 0;
}

uint64_t oracle_pairs(void* job) { return static_cast<Job*>(job)->pairs.size(); }

int oracle_reduce(void* job, oracle_result* out) {
  Job* J = static_cast<Job*>(job);
  if (!J || !out) return 1;
  reduce(*J);
  out->n_keys = J->key_off.size() - 1;
  out->keys = J->keys.data();
  out->key_offsets = J->key_off.data();
  out->vals = J->vals.data();
  out->val_offsets = J->val_off.data();
  return 0;
}

void oracle_destroy(void* job) { delete static_cast<Job*>(job); }

}  // extern "C"
