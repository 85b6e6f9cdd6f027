/* gen_host.c — host (CPU) build of the seeded input generators in bmr_gen.h, plus the
 * quantile tables they sample from.  Test/bench infrastructure only; no MapReduce arithmetic.
 * Built into gen/libbmrgen.so (plain C, pthreads); wrapped by gen/pygen.py. */
#include "bmr_gen.h"
#include <math.h>
#include <pthread.h>
#include <stdlib.h>
#include <string.h>

/* Zipf(s) over ranks [0, V): continuous inverse CDF with a +0.5 continuity correction,
 * tabulated at qn+1 quantiles (q[j] = rank at probability j/qn). */
int bmrg_build_zipf_q(double s, uint32_t V, uint32_t qn, uint32_t* q) {
  if (!q || V == 0 || qn == 0) return 1;
  for (uint32_t j = 0; j <= qn; ++j) {
    double u = (double)j / (double)qn, k;
    if (fabs(s - 1.0) < 1e-12) {
      double a = log(0.5), b = log((double)V + 0.5);
      k = exp(a + u * (b - a)) - 0.5;
    } else {
      double e = 1.0 - s, a = pow(0.5, e), b = pow((double)V + 0.5, e);
      k = pow(a + u * (b - a), 1.0 / e) - 0.5;
    }
    if (k < 0) k = 0;
    if (k > (double)(V - 1)) k = (double)(V - 1);
    q[j] = (uint32_t)k;
  }
  return 0;
}

/* log-normal(mu, sigma) line lengths, clamped to [lo, hi], at qn+1 quantiles.  The normal
 * quantile uses bisection on erfc (libm) — only the host ever builds this table. */
static double norm_cdf(double z) { return 0.5 * erfc(-z / sqrt(2.0)); }
static double norm_ppf(double p) {
  double lo = -12, hi = 12;
  for (int i = 0; i < 200; ++i) { double m = 0.5 * (lo + hi); if (norm_cdf(m) < p) lo = m; else hi = m; }
  return 0.5 * (lo + hi);
}
int bmrg_build_lognormal_q(double mu, double sigma, uint32_t lo, uint32_t hi, uint32_t qn, uint32_t* q) {
  if (!q || qn == 0) return 1;
  for (uint32_t j = 0; j <= qn; ++j) {
    double p = ((double)j + 0.5) / ((double)qn + 1.0);
    double v = exp(mu + sigma * norm_ppf(p));
    double r = floor(v + 0.5);
    if (r < lo) r = lo;
    if (r > hi) r = hi;
    q[j] = (uint32_t)r;
  }
  return 0;
}

/* KMeans blob centres: k x 8 integers ~U[-64,64], each redrawn until its distance to every
 * earlier centre is >= min_dist (16 sigma at sigma=4). */
int bmrg_km_centres(uint64_t seed, uint32_t k, uint32_t min_dist, int32_t* c) {
  if (!c || k == 0) return 1;
  bmrg_rng r = bmrg_stream(seed, 0xCE27E5ull);
  for (uint32_t b = 0; b < k; ++b) {
    for (int tries = 0;; ++tries) {
      for (int t = 0; t < 8; ++t) c[b * 8 + t] = (int32_t)bmrg_below(&r, 129) - 64;
      int ok = 1;
      for (uint32_t a = 0; a < b && ok; ++a) {
        int64_t d2 = 0;
        for (int t = 0; t < 8; ++t) { int64_t d = c[a * 8 + t] - c[b * 8 + t]; d2 += d * d; }
        if (d2 < (int64_t)min_dist * min_dist) ok = 0;
      }
      if (ok) break;
      if (tries > 100000) return 2;
    }
  }
  return 0;
}

/* ---------------- multi-threaded page generation ---------------- */
typedef struct {
  const bmrg_text_params* P;
  uint64_t page0, npages, tid, nthreads;
  uint8_t* out;
  uint32_t* page_lines;
  bmrg_truth truth;
} text_job;

static void* text_worker(void* arg) {
  text_job* J = (text_job*)arg;
  for (uint64_t p = J->tid; p < J->npages; p += J->nthreads) {
    uint8_t* o = J->out + p * (uint64_t)J->P->page_bytes;
    uint64_t gbase = (J->page0 + p) * (uint64_t)J->P->page_bytes;
    bmrg_truth* T = (J->truth.word_hist || J->truth.plants || J->truth.links) ? &J->truth : NULL;
    uint32_t nl = (J->P->kind == BMRG_HTML) ? bmrg_html_page(J->P, J->page0 + p, o, gbase, T)
                                             : bmrg_text_page(J->P, J->page0 + p, o, gbase, T);
    if (J->page_lines) J->page_lines[p] = nl;
  }
  return NULL;
}

/* Generate pages [page0, page0+npages) into out (npages*page_bytes bytes).  Global byte
 * offsets in the truth are (page0+p)*page_bytes + in-page offset.  Truth sinks are optional:
 * word_hist (vocab u32), plants (cap u64), links (cap u64); counts returned in *nplants /
 * *nlinks (may exceed cap: then the lists are truncated).  Lists come back grouped by thread;
 * callers sort them. */
int bmrg_host_pages(const bmrg_text_params* P, uint64_t page0, uint64_t npages, uint8_t* out,
                    uint32_t* page_lines, int nthreads, uint32_t* word_hist,
                    uint64_t* plants, uint64_t plants_cap, uint64_t* nplants,
                    uint64_t* links, uint64_t links_cap, uint64_t* nlinks) {
  if (!P || !out) return 1;
  if (nthreads < 1) nthreads = 1;
  if ((uint64_t)nthreads > npages) nthreads = (int)(npages ? npages : 1);
  text_job* J = (text_job*)calloc((size_t)nthreads, sizeof(text_job));
  pthread_t* th = (pthread_t*)calloc((size_t)nthreads, sizeof(pthread_t));
  uint64_t pcap = plants ? plants_cap / (uint64_t)nthreads : 0;
  uint64_t lcap = links ? links_cap / (uint64_t)nthreads : 0;
  for (int t = 0; t < nthreads; ++t) {
    J[t].P = P; J[t].page0 = page0; J[t].npages = npages; J[t].tid = (uint64_t)t;
    J[t].nthreads = (uint64_t)nthreads; J[t].out = out; J[t].page_lines = page_lines;
    if (word_hist) J[t].truth.word_hist = (uint32_t*)calloc(P->vocab, sizeof(uint32_t));
    if (plants) { J[t].truth.plants = plants + (uint64_t)t * pcap; J[t].truth.plants_cap = pcap; }
    if (links) { J[t].truth.links = links + (uint64_t)t * lcap; J[t].truth.links_cap = lcap; }
    pthread_create(&th[t], NULL, text_worker, &J[t]);
  }
  uint64_t np = 0, nl = 0;
  for (int t = 0; t < nthreads; ++t) {
    pthread_join(th[t], NULL);
    if (word_hist) {
      for (uint32_t i = 0; i < P->vocab; ++i) word_hist[i] += J[t].truth.word_hist[i];
      free(J[t].truth.word_hist);
    }
    /* compact per-thread lists to the front */
    if (plants) {
      uint64_t m = J[t].truth.nplants < pcap ? J[t].truth.nplants : pcap;
      memmove(plants + np, J[t].truth.plants, m * sizeof(uint64_t));
      np += m;
    }
    if (links) {
      uint64_t m = J[t].truth.nlinks < lcap ? J[t].truth.nlinks : lcap;
      memmove(links + nl, J[t].truth.links, m * sizeof(uint64_t));
      nl += m;
    }
  }
  if (nplants) { uint64_t tot = 0; for (int t = 0; t < nthreads; ++t) tot += J[t].truth.nplants; *nplants = tot; }
  if (nlinks) { uint64_t tot = 0; for (int t = 0; t < nthreads; ++t) tot += J[t].truth.nlinks; *nlinks = tot; }
  free(J); free(th);
  return 0;
}

/* Record offsets of newline-terminated lines: offsets[0]=0, offsets[i+1] = end of line i.
 * page_lines gives the line count of each page (from bmrg_host_pages). */
typedef struct { const uint8_t* data; uint64_t npages, tid, nthreads; uint32_t pb; const uint64_t* base; uint64_t* off; } off_job;
static void* off_worker(void* arg) {
  off_job* J = (off_job*)arg;
  for (uint64_t p = J->tid; p < J->npages; p += J->nthreads) {
    const uint8_t* d = J->data + p * (uint64_t)J->pb;
    uint64_t k = J->base[p];
    for (uint32_t i = 0; i < J->pb; ++i)
      if (d[i] == '\n') J->off[++k] = p * (uint64_t)J->pb + i + 1;
  }
  return NULL;
}
int bmrg_host_offsets(const uint8_t* data, uint64_t npages, uint32_t page_bytes,
                      const uint32_t* page_lines, uint64_t* offsets, int nthreads) {
  if (!data || !offsets || !page_lines) return 1;
  uint64_t* base = (uint64_t*)malloc((npages + 1) * sizeof(uint64_t));
  base[0] = 0;
  for (uint64_t p = 0; p < npages; ++p) base[p + 1] = base[p] + page_lines[p];
  offsets[0] = 0;
  if (nthreads < 1) nthreads = 1;
  off_job* J = (off_job*)calloc((size_t)nthreads, sizeof(off_job));
  pthread_t* th = (pthread_t*)calloc((size_t)nthreads, sizeof(pthread_t));
  for (int t = 0; t < nthreads; ++t) {
    J[t] = (off_job){data, npages, (uint64_t)t, (uint64_t)nthreads, page_bytes, base, offsets};
    pthread_create(&th[t], NULL, off_worker, &J[t]);
  }
  for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
  free(J); free(th); free(base);
  return 0;
}

/* KMeans points [i0, i0+n) -> out (n*8 floats). */
typedef struct { uint64_t seed, i0, n, tid, nthreads; const int32_t* c; uint32_t k; float* out; } km_job;
static void* km_worker(void* arg) {
  km_job* J = (km_job*)arg;
  uint64_t lo = J->n * J->tid / J->nthreads, hi = J->n * (J->tid + 1) / J->nthreads;
  for (uint64_t i = lo; i < hi; ++i) bmrg_km_point(J->seed, J->i0 + i, J->c, J->k, J->out + i * 8);
  return NULL;
}
int bmrg_host_km(uint64_t seed, uint64_t i0, uint64_t n, const int32_t* centres, uint32_t k,
                 float* out, int nthreads) {
  if (!centres || !out || k == 0) return 1;
  if (nthreads < 1) nthreads = 1;
  km_job* J = (km_job*)calloc((size_t)nthreads, sizeof(km_job));
  pthread_t* th = (pthread_t*)calloc((size_t)nthreads, sizeof(pthread_t));
  for (int t = 0; t < nthreads; ++t) {
    J[t] = (km_job){seed, i0, n, (uint64_t)t, (uint64_t)nthreads, centres, k, out};
    pthread_create(&th[t], NULL, km_worker, &J[t]);
  }
  for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
  free(J); free(th);
  return 0;
}

/* word spelling of a rank (for ground-truth checks) */
uint32_t bmrg_host_word(uint32_t rank, uint8_t* out) { return bmrg_word(rank, out); }
uint32_t bmrg_host_url(uint32_t id, uint8_t* out) { return bmrg_url(id, out); }
