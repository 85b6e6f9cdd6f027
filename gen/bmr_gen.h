/* bmr_gen.h — seeded, counter-based synthetic INPUT generators (test/bench infrastructure).
 *
 * This header holds NO MapReduce arithmetic: no tokenising, matching, hashing, sorting,
 * grouping, distance or reduction.  It only produces input bytes (and, on the host, the
 * ground truth of what it planted).  It is the one module shared by the CUDA path's inputs
 * and by the oracle's inputs (task rule ③): both sides consume the same bytes.
 *
 * Compiled twice: as plain C on the host (gen/gen_host.c -> libbmrgen.so) and as CUDA
 * device code (gen/gen_device.cu -> libbmrgen_cuda.so).  Every operation is integer
 * arithmetic, so host and device produce bit-identical bytes (tests/test_gen_device.py).
 * Tables that need transcendental functions (Zipf and log-normal quantiles) are built once
 * on the host (gen_host.c) and passed to both sides as plain arrays.
 *
 * Workload shapes follow PAPER.md Table II (L195-270) as restated in SURVEY.md §8(d) D-1:
 *   WC text: lines 27+U[0,6)+U[0,7) B (mean 32.5, std 2.63 vs 32.44±2.59), Zipf(1) words (L125, L127)
 *   SM text: lines 39+U[0,6)+U[0,7) B (44.5 ± 2.63 vs 44.52±2.68) + a 16-B pattern planted w.p. p
 *   II html: log-normal line lengths (63.9±123.2), links `<a href="URL">` w.p. 1/7.94
 *   KM:      8 x fp32 points (32-B value), 32 Gaussian blobs.
 */
#ifndef BMR_GEN_H
#define BMR_GEN_H
#include <stdint.h>
#include <stddef.h>

#if defined(__CUDACC__)
#define BMRG_FN __host__ __device__ __forceinline__ static
#else
#define BMRG_FN static inline
#endif

#define BMRG_PHI 0x9E3779B97F4A7C15ULL
#define BMRG_MAX_WORD 13u
#define BMRG_IH_MEAN 24570 /* mean of a sum of 12 uniform 12-bit ints (12 * 4095 / 2) */

enum { BMRG_TEXT = 1, BMRG_HTML = 2 };

/* ---- counter-based generator (splitmix64) ---- */
typedef struct { uint64_t s; } bmrg_rng;

BMRG_FN uint64_t bmrg_mix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
BMRG_FN bmrg_rng bmrg_stream(uint64_t seed, uint64_t unit) {
  bmrg_rng r; r.s = bmrg_mix(seed ^ (unit * BMRG_PHI)); return r;
}
BMRG_FN uint64_t bmrg_next(bmrg_rng* r) { r->s += BMRG_PHI; return bmrg_mix(r->s); }
/* uniform integer in [0, m) (multiply-shift; m < 2^32) */
BMRG_FN uint32_t bmrg_below(bmrg_rng* r, uint32_t m) {
  return (uint32_t)(((bmrg_next(r) >> 32) * (uint64_t)m) >> 32);
}
/* Irwin-Hall: sum of 12 uniform 12-bit integers; mean 24570, std ~4096 (an approximate
 * normal with sigma = 4096 units).  Integer-only so host and device agree exactly. */
BMRG_FN int32_t bmrg_ih12(bmrg_rng* r) {
  int32_t s = 0;
  for (int k = 0; k < 3; ++k) {
    uint64_t x = bmrg_next(r);
    for (int j = 0; j < 4; ++j) { s += (int32_t)(x & 0xFFF); x >>= 12; }
  }
  return s;
}
/* sample from a quantile table q[0..n] (n+1 entries, non-decreasing): piecewise uniform */
BMRG_FN uint32_t bmrg_quantile(bmrg_rng* r, const uint32_t* q, uint32_t n) {
  uint64_t x = bmrg_next(r);
  uint32_t j = (uint32_t)(((x >> 32) * (uint64_t)n) >> 32);
  uint32_t lo = q[j], hi = q[j + 1];
  if (hi <= lo) return lo;
  return lo + (uint32_t)((((x & 0xFFFFFFFFULL)) * (uint64_t)(hi - lo + 1)) >> 32);
}

/* ---- word spellings: rank r -> unique lowercase string, shorter for frequent ranks ---- */
BMRG_FN uint32_t bmrg_bitlen(uint64_t v) { uint32_t b = 0; while (v) { ++b; v >>= 1; } return b; }
BMRG_FN uint32_t bmrg_word_len(uint32_t r) {
  uint32_t nd = 1; uint64_t p = 26;
  while (p <= r) { ++nd; p *= 26; }
  uint32_t L = 3 + (bmrg_bitlen((uint64_t)r + 1) - 1) * 3 / 20;
  uint64_t h = bmrg_mix((uint64_t)r ^ 0x5157AB1Eull);
  if ((h & 7) == 0) L += (uint32_t)((h >> 20) % 7);
  if (L < nd) L = nd;
  if (L > BMRG_MAX_WORD) L = BMRG_MAX_WORD;
  return L;
}
/* writes bmrg_word_len(r) letters; bijective for a fixed length (r < 26^L) */
BMRG_FN uint32_t bmrg_word(uint32_t r, uint8_t* out) {
  uint32_t L = bmrg_word_len(r);
  uint32_t v = r, acc = 0;
  for (uint32_t i = 0; i < L; ++i) {
    uint32_t d = v % 26; v /= 26;
    uint32_t c = (d + acc * 7 + i * 11 + L * 5) % 26;
    acc += d;
    out[L - 1 - i] = (uint8_t)('a' + c);
  }
  return L;
}

/* ---- parameters shared by host and device page generators ---- */
typedef struct {
  uint64_t seed;
  uint32_t kind;              /* BMRG_TEXT or BMRG_HTML */
  uint32_t page_bytes;
  /* TEXT (WC, SM) */
  uint32_t line_base, line_u1, line_u2; /* target line length incl. '\n' = base + U[0,u1) + U[0,u2) */
  uint32_t vocab;                  /* V */
  uint32_t punct_ppm;              /* punctuation after a word, per million */
  uint32_t plant_ppm;              /* SM: pattern planted in a line, per million lines */
  uint8_t  pattern[16];
  const uint32_t* zipf_q; uint32_t zipf_qn;   /* word-rank quantiles (Zipf), zipf_qn+1 entries */
  /* HTML (II) */
  const uint32_t* len_q;  uint32_t len_qn;    /* line-length quantiles (log-normal) */
  const uint32_t* url_q;  uint32_t url_qn;    /* URL-id quantiles (Zipf 0.8 over 2^24) */
  uint32_t link_ppm, name_ppm, upper_ppm, unclosed_ppm;
} bmrg_text_params;

/* ground-truth sinks (host only; NULL on device) */
typedef struct {
  uint32_t* word_hist;        /* TEXT: count per rank (size vocab) */
  uint64_t* plants; uint64_t plants_cap; uint64_t nplants;   /* SM: global offsets */
  uint64_t* links;  uint64_t links_cap;  uint64_t nlinks;    /* II: (url_id << 40 | global offset) */
} bmrg_truth;

/* decimal digits */
BMRG_FN uint32_t bmrg_dec(uint32_t v, uint8_t* o) {
  uint8_t t[10]; uint32_t n = 0;
  do { t[n++] = (uint8_t)('0' + v % 10); v /= 10; } while (v);
  for (uint32_t i = 0; i < n; ++i) o[i] = t[n - 1 - i];
  return n;
}
/* URL spelling for id (unique by construction: host part id%4096, 3 base-26 letters of id>>12).
 * Total length ~ N(31.67, 17.34) (Table II II output key) clamped to [prefix, 512]. */
BMRG_FN uint32_t bmrg_url(uint32_t id, uint8_t* o /* >= 512 B */) {
  const char* a = "http://h"; uint32_t n = 0;
  for (; a[n]; ++n) o[n] = (uint8_t)a[n];
  n += bmrg_dec(id & 4095u, o + n);
  const char* b = ".example/";
  for (uint32_t i = 0; b[i]; ++i) o[n++] = (uint8_t)b[i];
  uint32_t hi = id >> 12;
  for (int i = 0; i < 3; ++i) { o[n++] = (uint8_t)('a' + hi % 26); hi /= 26; }
  bmrg_rng r = bmrg_stream(0x0E1E0E1Eull, id);
  int32_t z = bmrg_ih12(&r) - BMRG_IH_MEAN;               /* ~N(0, 4096) */
  int32_t total = 32 + (z * 1734) / (4096 * 100);         /* 31.67 + 17.34 z */
  if (total > 512) total = 512;
  const char* alpha = "abcdefghijklmnopqrstuvwxyz0123456789/.-_";
  while ((int32_t)n < total) o[n++] = (uint8_t)alpha[bmrg_below(&r, 40)];
  return n;
}

/* One TEXT page (WC / SM).  Records are lines ending in '\n'; the page holds whole lines;
 * the last line absorbs the remainder (padded with spaces).  Returns the line count. */
BMRG_FN uint32_t bmrg_text_page(const bmrg_text_params* P, uint64_t page, uint8_t* out,
                                uint64_t page_base, bmrg_truth* T) {
  bmrg_rng r = bmrg_stream(P->seed, page);
  const uint32_t PB = P->page_bytes;
  const char* punct = ",.;:!?";
  uint32_t pos = 0, nlines = 0;
  uint8_t w[BMRG_MAX_WORD];
  while (pos < PB) {
    uint32_t rem = PB - pos;
    uint32_t target = P->line_base + bmrg_below(&r, P->line_u1) + bmrg_below(&r, P->line_u2);
    if (target >= rem || rem - target < P->line_base) target = rem;
    uint32_t cap = target - 1, len = 0;
    for (;;) {
      uint32_t rank = bmrg_quantile(&r, P->zipf_q, P->zipf_qn);
      if (rank >= P->vocab) rank = P->vocab - 1;
      uint32_t wl = bmrg_word(rank, w);
      uint32_t pu = bmrg_below(&r, 1000000u) < P->punct_ppm;
      uint32_t need = (len ? 1u : 0u) + wl + pu;
      if (len + need > cap) break;
      if (len) out[pos + len++] = ' ';
      for (uint32_t i = 0; i < wl; ++i) out[pos + len++] = w[i];
      if (pu) out[pos + len++] = (uint8_t)punct[bmrg_below(&r, 6)];
      if (T && T->word_hist) T->word_hist[rank] += 1;
    }
    while (len < cap) out[pos + len++] = ' ';
    out[pos + cap] = '\n';
    if (P->plant_ppm && cap >= 16 && bmrg_below(&r, 1000000u) < P->plant_ppm) {
      uint32_t j = bmrg_below(&r, cap - 15);
      for (uint32_t i = 0; i < 16; ++i) out[pos + j + i] = P->pattern[i];
      if (T && T->plants) {
        if (T->nplants < T->plants_cap) T->plants[T->nplants] = page_base + pos + j;
        T->nplants++;
      }
    }
    pos += target; ++nlines;
  }
  return nlines;
}

/* One HTML page (II).  Lines of log-normal length; links `<a href="URL">` planted w.p.
 * link_ppm; distractors that must produce nothing: `<a name="...">`, `<A HREF="...">`,
 * and an unclosed `<a href="...` at the end of a line.  Filler never contains '"' or '<'. */
BMRG_FN uint32_t bmrg_html_page(const bmrg_text_params* P, uint64_t page, uint8_t* out,
                                uint64_t page_base, bmrg_truth* T) {
  bmrg_rng r = bmrg_stream(P->seed, page);
  const uint32_t PB = P->page_bytes;
  const char* fill = "abcdefghijklmnopqrstuvwxyz abcdefghijklmnop   ,.=/>;:-_0123456789 ";
  uint32_t pos = 0, nlines = 0;
  uint8_t url[512];
  while (pos < PB) {
    uint32_t rem = PB - pos;
    uint32_t target = bmrg_quantile(&r, P->len_q, P->len_qn);
    if (target < 1) target = 1;
    uint32_t u = bmrg_below(&r, 1000000u);
    uint32_t kind = 0;                                   /* 0 none, 1 link, 2 name, 3 upper, 4 unclosed */
    if (u < P->link_ppm) kind = 1;
    else if (u < P->link_ppm + P->name_ppm) kind = 2;
    else if (u < P->link_ppm + P->name_ppm + P->upper_ppm) kind = 3;
    else if (u < P->link_ppm + P->name_ppm + P->upper_ppm + P->unclosed_ppm) kind = 4;
    uint32_t id = 0, ul = 0;
    if (kind) { id = bmrg_quantile(&r, P->url_q, P->url_qn); ul = bmrg_url(id, url); }
    /* tag text */
    const char* pre = kind == 3 ? "<A HREF=\"" : (kind == 2 ? "<a name=\"" : "<a href=\"");
    uint32_t tl = kind ? 9u + ul + (kind == 4 ? 0u : 2u) : 0u;      /* + '">' */
    if (kind && target < tl + 1) target = tl + 1;
    if (target >= rem || rem - target < 1) target = rem;
    uint32_t cap = target - 1;
    if (kind && tl > cap) kind = 0;                                  /* does not fit: skip */
    for (uint32_t i = 0; i < cap; i += 8) {
      uint64_t x = bmrg_next(&r);
      for (uint32_t k = 0; k < 8 && i + k < cap; ++k) { out[pos + i + k] = (uint8_t)fill[(x & 0xFF) % 64]; x >>= 8; }
    }
    if (kind) {
      uint32_t j = (kind == 4) ? cap - tl : bmrg_below(&r, cap - tl + 1);
      uint8_t* o = out + pos + j;
      for (uint32_t i = 0; i < 9; ++i) o[i] = (uint8_t)pre[i];
      for (uint32_t i = 0; i < ul; ++i) o[9 + i] = url[i];
      if (kind != 4) { o[9 + ul] = '"'; o[10 + ul] = '>'; }
      if (kind == 1 && T && T->links) {
        if (T->nlinks < T->links_cap) T->links[T->nlinks] = ((uint64_t)id << 40) | (page_base + pos + j + 9);
        T->nlinks++;
      }
    }
    out[pos + cap] = '\n';
    pos += target; ++nlines;
  }
  return nlines;
}

/* ---- KMeans points (fixed 32-B records: 8 little-endian fp32) ----
 * Blob of point i = i mod k; coordinate = centre + Irwin-Hall noise (sigma = 4), in units of
 * 2^-10, clamped to (-128, 128): every value is exact in fp32. */
BMRG_FN void bmrg_km_point(uint64_t seed, uint64_t i, const int32_t* centres /* k*8 */,
                           uint32_t k, float* x /* 8 */) {
  bmrg_rng r = bmrg_stream(seed, i);
  uint32_t b = (uint32_t)(i % k);
  for (int t = 0; t < 8; ++t) {
    int32_t units = centres[b * 8 + t] * 1024 + (bmrg_ih12(&r) - BMRG_IH_MEAN);
    if (units > 131071) units = 131071;
    if (units < -131071) units = -131071;
    x[t] = (float)units * (1.0f / 1024.0f);
  }
}

#endif /* BMR_GEN_H */
