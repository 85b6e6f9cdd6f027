// kernels.h — host-visible launchers of the libbmr device kernels (internal to libbmr.so;
// the public C ABI is include/bmr.h).  No torch types anywhere.
#pragma once
#include <atomic>
#include <cstdint>
#include <cuda_runtime.h>

namespace bmr {

// process-wide count of libbmr kernel launches (reported through mr_stats::kernel_launches)
extern std::atomic<unsigned long long> g_kernel_launches;
inline void count_launch(unsigned n = 1) { g_kernel_launches.fetch_add(n, std::memory_order_relaxed); }

enum Workload : int { kWC = 1, kSM = 2, kKM = 3, kII = 4 };
// WordCount streams (map.cu): exact (words of <= kExactMax bytes, keys < 2^kExactBits), mid
// (<= kMidMax bytes, keys < 2^kMidBits), both keys only; longer words hashed with references.
constexpr uint32_t kExactMax = 5, kExactBits = 30;
constexpr uint32_t kMidMax = 8, kMidBits = 48;

// Device-resident job state (one per job).
struct DevState {
  unsigned long long pair_cursor;  // D7: demand in pairs (counts past capacity -> replay)
  unsigned long long flushes;      // number of output-half flushes (one global atomic each)
  unsigned int err;                // kErr* bits
  unsigned int collisions;         // hashed-key mismatches inside equal-hash runs
  unsigned long long seg_total;    // S
  unsigned long long key_bytes;    // total output key bytes
  unsigned long long large_items;  // reduce work list length (large segments x tiles)
  unsigned long long large_done;   // work-list cursor for the persistent large-segment kernel
  unsigned int tile_counter[32];   // dynamic tile ids of the look-back kernels (one per launch slot)
  unsigned long long pads;         // sentinel filler pairs written by the flushes (sort last, excluded)
  unsigned long long pair_cursor_b;  // WC hashed stream: demand in pairs
  unsigned long long pair_cursor_c;  // WC mid stream: demand in pairs
  unsigned long long pair_cursor_p;  // WC combiner partials: demand in entries
  unsigned long long n_extra;        // WC: partial-only keys found by the merge (mr_group)
  unsigned long long words_comb;     // WC: words absorbed by the combiners (sum of partial counts)
  unsigned long long pads_b, pads_c; // WC hashed / mid stream: sentinel entries in unused chunk tails
  unsigned long long mid_fail;       // WC mid table: inserts that found no slot (-> grow + replay)
  unsigned long long long_fail;      // WC long-word table: inserts that found no slot (-> grow + replay)
  unsigned long long seal_waits;     // Map: seals that waited for a buffer still flushing (ring full)
  unsigned long long spills;         // Map: warp results written straight to HBM while the ring was full
  unsigned long long km_scanned;     // KMeans Map: points that scanned every centroid (bound test failed / off)
  unsigned long long tile_next;      // text Map: dynamic tile counter of the current batch (k_tile_bounds zeroes it)
};
constexpr unsigned int kErrKeyTooLong = 1u, kErrCollision = 2u, kErrTileCap = 4u, kErrNullRecords = 8u,
                       kErrMidTable = 16u, kErrLongTable = 32u;
// WC mid-word table: open addressing over 48-bit exact keys, empty slot = all ones
constexpr uint64_t kMidEmpty = ~0ULL;
constexpr uint32_t kMidProbes = 32;
// counts of a slot are striped over kMidStripes words (the warp's stripe), so the Zipf-hot mid
// words do not serialise every RED on one address; the extraction sums the stripes
#ifndef BMR_MID_STRIPES
#define BMR_MID_STRIPES 16
#endif
constexpr uint32_t kMidStripes = BMR_MID_STRIPES;
// stripe-major: stripe q of slot h at q * 2^bits + h, so the stripes of a Zipf-hot word sit in
// kMidStripes different L2 lines (slot-major they shared one line, and its REDs serialised there)
__host__ __device__ inline uint64_t stripe_at(uint64_t slot, uint32_t stripe, uint32_t bits) {
  return (static_cast<uint64_t>(stripe) << bits) | slot;
}
__host__ __device__ inline uint64_t mid_slot(uint64_t key, uint32_t bits) {
  return (key * 0x9E3779B97F4A7C15ULL) >> (64 - bits);
}
// long-table key of a word of <= 8 bytes: the zero-padded bytes in lo, this marker in hi (byte 15
// = 0x80, never a word byte; nonzero, so a slot whose hi reads 0 is still a torn view)
constexpr uint64_t kShortHi = 0x8000000000000000ULL;
__host__ __device__ inline uint64_t long_slot(uint64_t lo, uint64_t hi, uint32_t bits) {
  return ((lo * 0x9E3779B97F4A7C15ULL) ^ (hi * 0xC2B2AE3D27D4EB4FULL) ^ (lo >> 29)) * 0x94D049BB133111EBULL >> (64 - bits);
}

// Intermediate pairs, SoA in HBM (SURVEY §8(a) layout): sort key, key reference, value.
// WordCount Map output is three streams: exact keys (hx, u32: the key is the record, value 1),
// mid keys (hc, u64 exact 48-bit) and hashed keys (hb + krefb); see map.cu.
struct PairBufs {
  uint64_t* h = nullptr;     // 64-bit sort key (inline key / hash / SM offset / KM id)
  uint32_t* hx = nullptr;    // WC exact stream: 30-bit exact keys (u32; 0xFFFFFFFF = filler)
  uint64_t* hp = nullptr;    // WC combiner partials (exact key | count << 32); nullptr = no combiner
  uint64_t cap_p = 0;
  double* km_sums = nullptr;             // KM combiner: cluster sums / counts accumulated by the
  unsigned long long* km_cnts = nullptr; //   Map itself (nullptr = emit (id, point) pairs)
  uint64_t* kref = nullptr;  // (device address of key bytes << 16) | key length
  uint8_t* v = nullptr;      // value bytes (vbytes per pair)
  uint64_t cap = 0;          // capacity in pairs
  uint64_t* hb = nullptr;    // WC hashed stream: keys, key references, capacity
  uint64_t* krefb = nullptr;
  uint64_t cap_b = 0;
  uint64_t* hc = nullptr;    // WC mid stream: keys, capacity
  uint64_t cap_c = 0;
  uint32_t* xtab = nullptr;  // WC two-level combiner: L2 count table (2^30 u32, by exact key)
  uint64_t* mkeys = nullptr; // WC mid words (6..8 symbols): open-addressing table of 48-bit exact keys
  uint32_t* mcnt = nullptr;  //   and their counts, 2^mbits slots
  uint32_t mbits = 0;
  uint64_t* lkeys = nullptr; // WC long words (9..16 symbols): open-addressing table of their 16 key bytes
  uint32_t* lcnt = nullptr;  //   (zero-padded; 2 x u64 per slot, all-zero = empty) and counts, 2^lbits slots
  uint32_t lbits = 0;
};

// f-3 fused exchange: a destination rank's receive window (device pointers valid in this
// process: a peer GPU's buffers opened through CUDA IPC, or same-GPU buffers for virtual ranks).
// cursor[0] = entries appended, cursor[1] = heap bytes appended (demand, may pass the capacity).
struct XWindow {
  uint8_t* entries;                 // XEntry[ecap]
  uint8_t* heap;                    // key bytes, hcap bytes (8-B aligned records)
  unsigned long long* cursor;       // 2 x u64
  uint64_t ecap, hcap;
};

struct MapArgs {
  int workload = 0;
  uint32_t flags = 0;
  const uint8_t* records = nullptr;
  const uint64_t* offsets = nullptr;  // n+1 (text) or nullptr (fixed stride)
  uint64_t n = 0;                     // records
  uint64_t nbytes = 0;                // records bytes (offsets[n] or n*stride)
  uint32_t stride = 0;
  uint64_t gbase = 0;                 // global byte offset of records[0]
  uint8_t pattern[16] = {0};          // SM
  const float* centroids = nullptr;   // KM, device, k x 8
  uint32_t k = 0;
  PairBufs out;
  DevState* st = nullptr;
  uint64_t* tile_bounds = nullptr;    // scratch: 2 u64 per tile
  uint64_t hash_seed = 0;
  uint32_t key_bits = 64;             // sort-key width of hashed / inline keys (48 or 64)
  int grid = 0;                       // persistent CTAs (0 = one per SM)
  const XWindow* xwin = nullptr;      // f-3: InvertedIndex records go straight to these R windows
  uint32_t xranks = 0;
  // text batches: dimensions derived on the device (map.cu k_tile_bounds)
  uint64_t* desc = nullptr;            // this batch's descriptor: nbytes, ntiles, gbase, tile-cap overflow
  const uint64_t* prev_desc = nullptr; // the previous batch's (nullptr: the first batch, base = input_base)
  uint64_t input_base = 0;
  uint64_t tb_cap = 0;                 // tiles tile_bounds can hold
};

int vbytes_of(int workload);                 // value bytes per pair (WC Map output: none, value 1)
bool has_kref(int workload);
uint64_t map_tiles(const MapArgs& a);        // number of tiles of a batch (fixed stride, or nbytes known)
constexpr uint64_t kMapTileBytes = 16384;    // owned bytes per text tile (map.cu kT)
uint32_t map_prefetch(int w);
uint32_t map_wait_hint();
uint32_t map_dyn_windows(int workload);
uint32_t map_wc_balanced();
bool map_wc_table_ok(uint32_t flags);           // the WC Map can feed the L2 count table (SIO fast path)
bool map_fast_path();                           // the WC / II SIO fast paths are on (BMR_MAP_FAST)
bool map_wc_tab();                              // WordCount table mode uses wc_window_tab (BMR_WC_TAB)
cudaError_t launch_map(const MapArgs& a, int num_sms, cudaStream_t s);

// ---- group-by-key (hash radix sort + segment boundaries) ----
struct SortBufs {
  uint64_t* keys_a = nullptr; uint64_t* keys_b = nullptr;
  uint32_t* idx_a = nullptr;  uint32_t* idx_b = nullptr;
  uint64_t* status = nullptr; uint64_t status_cap = 0;  // look-back words (tiles x 256)
  uint32_t* hist = nullptr;    // 8 x 256 digit histograms
  uint32_t* bases = nullptr;   // 8 x 256 exclusive digit bases
  uint64_t cap = 0;
};
constexpr int kSortThreads = 256;
constexpr int kBinStride = 512;   // histogram / base tables: 8 digits x kBinStride bins (digits of 8 or 9 bits)
int sort_tile();          // keys per onesweep tile (payload passes)
int sort_tile_keys();     // the same for the keys-only passes
int sort_tile_keys32();   // the same for the keys-only passes over u32 keys
// ranking of a onesweep pass: match.any groups, or shared-memory OR match masks (a first pass
// whose 32-key groups carry many distinct digits)
constexpr int kRankMatch = 0, kRankOrMask = 1;
// histograms of digits [0, nd) of `bits` bits each (8 or 9); hist holds 8 x kBinStride u32
cudaError_t launch_hist(const uint64_t* keys, uint64_t m, uint32_t* hist, int nd, int bits, int num_sms,
                        cudaStream_t s);
cudaError_t launch_hist32(const uint32_t* keys, uint64_t m, uint32_t* hist, int nd, int bits, int num_sms,
                          cudaStream_t s);
// one LSD pass on digit `digit` of `bits` bits (8, or 9 for keys-only passes); idx_in ==
// nullptr means the identity permutation; idx_out == nullptr: keys only (no payload).
// bases: 8 x kBinStride table of global digit bases; status: tiles x 2^bits look-back words
cudaError_t launch_onesweep(const uint64_t* keys_in, const uint32_t* idx_in, uint64_t* keys_out,
                            uint32_t* idx_out, uint64_t m, int digit, int bits, const uint32_t* bases,
                            uint64_t* status, uint32_t epoch, unsigned int* tile_counter, cudaStream_t s,
                            int rank_kind = kRankMatch);   // kRankOrMask: keys-only passes only
// keys-only LSD pass over u32 keys (the WordCount exact stream)
cudaError_t launch_onesweep32(const uint32_t* keys_in, uint32_t* keys_out, uint64_t m, int digit, int bits,
                              const uint32_t* bases, uint64_t* status, uint32_t epoch, unsigned int* tile_counter,
                              cudaStream_t s, int rank_kind = kRankMatch);
// ranking kind of a keys-only pass from its digit histogram (hist[0..255], m keys): kRankOrMask
// for a first pass whose digits of 32 keys are mostly distinct, else kRankMatch
int choose_rank_kind32(const uint32_t* hist, uint64_t m, bool first_pass);

// ---- segments ----
// heads per sort tile + byte verification of hashed keys; counts[t] = heads in tile t
// kmask: bits of the sorted word that form the key (packed WC values live above bit 48)
cudaError_t launch_seg_count(const uint64_t* skeys, const uint32_t* perm, const uint64_t* kref, uint64_t m,
                             uint32_t* counts, DevState* st, uint32_t key_bits, uint64_t kmask, cudaStream_t s);
// exclusive scan of u64 (in-place allowed); writes total to *total if non-null
cudaError_t launch_scan_u64(const uint64_t* in, uint64_t* out, uint64_t n, unsigned long long* total,
                            uint64_t* status, uint32_t epoch, unsigned int* tile_counter, cudaStream_t s);
cudaError_t launch_scan_u32to64(const uint32_t* in, uint64_t* out, uint64_t n, unsigned long long* total,
                                uint64_t* status, uint32_t epoch, unsigned int* tile_counter, cudaStream_t s);
cudaError_t launch_seg_write(const uint64_t* skeys, uint64_t m, const uint64_t* tile_base, uint64_t* seg_start,
                             uint64_t kmask, cudaStream_t s);
// the same two steps over sorted u32 keys (keys-only, nothing to verify)
cudaError_t launch_seg_count32(const uint32_t* skeys, uint64_t m, uint32_t* counts, cudaStream_t s);
cudaError_t launch_seg_write32(const uint32_t* skeys, uint64_t m, const uint64_t* tile_base, uint64_t* seg_start,
                               cudaStream_t s);

// ---- reduce + output assembly ----
struct OutBufs {
  uint8_t* keys = nullptr; uint64_t* key_off = nullptr;
  uint8_t* vals = nullptr; uint64_t* val_off = nullptr;
};
cudaError_t launch_key_lengths(const uint64_t* seg_start, uint64_t nseg, const uint32_t* perm,
                               const uint64_t* kref, uint64_t* lens, cudaStream_t s);
cudaError_t launch_key_copy(const uint64_t* seg_start, uint64_t nseg, const uint32_t* perm, const uint64_t* kref,
                            const uint64_t* key_off, uint8_t* keys, cudaStream_t s);
// vmode 0: u32 values through perm, 1: u64 values through perm, 2: packed in skeys >> 48
cudaError_t launch_reduce_wc(const uint64_t* seg_start, uint64_t nseg, const uint64_t* skeys, const uint32_t* perm,
                             const uint8_t* v, int vmode, uint64_t* counts, uint64_t* worklist, DevState* st,
                             int num_sms, cudaStream_t s);
cudaError_t launch_reduce_km(const uint64_t* seg_start, uint64_t nseg, const uint64_t* skeys, const uint32_t* perm,
                             const uint8_t* v, double* sums, unsigned long long* cnts, uint32_t k,
                             uint64_t* worklist, DevState* st, int num_sms, cudaStream_t s);
// list == nullptr: all k clusters; else the nlist cluster ids in `list` (multi-GPU owners)
cudaError_t launch_km_finalize(const double* sums, const unsigned long long* cnts, const float* centroids,
                               uint32_t k, const uint32_t* list, uint32_t nlist, uint8_t* vals, uint64_t* val_off,
                               uint8_t* keys, uint64_t* key_off, cudaStream_t s);
// WC exact stream: counts = segment lengths; key lengths / bytes decoded from the sorted keys
cudaError_t launch_seg_lengths(const uint64_t* seg_start, uint64_t nseg, uint64_t* out, cudaStream_t s);
cudaError_t launch_key_lengths_exact(const uint64_t* seg_start, uint64_t nseg, const uint64_t* skeys, uint64_t* lens,
                                     cudaStream_t s);
cudaError_t launch_key_decode(const uint64_t* seg_start, uint64_t nseg, const uint64_t* skeys, const uint64_t* key_off,
                              uint8_t* keys, cudaStream_t s);
cudaError_t launch_key_lengths_exact32(const uint64_t* seg_start, uint64_t nseg, const uint32_t* skeys, uint64_t* lens,
                                       cudaStream_t s);
cudaError_t launch_key_decode32(const uint64_t* seg_start, uint64_t nseg, const uint32_t* skeys,
                                const uint64_t* key_off, uint8_t* keys, cudaStream_t s);
cudaError_t launch_gather_u64(const uint32_t* perm, const uint8_t* v, uint64_t m, uint64_t* out, cudaStream_t s);
cudaError_t launch_seg_keys(const uint64_t* seg, uint64_t nseg, const uint64_t* sk, uint64_t* out, cudaStream_t s);
// WC combiner partials (f-1): merge into the exact stream's segments (midx / psum) or the extra
// list of partial-only keys (xkeys / xcounts, *nextra of them)
cudaError_t launch_comb_merge(const uint64_t* segp, uint64_t nsegp, const uint64_t* skp, const uint64_t* sega,
                              uint64_t nsega, const uint32_t* skx, uint32_t* midx, uint64_t* psum, uint32_t* xkeys,
                              uint64_t* xcounts, unsigned long long* nextra, cudaStream_t s);
cudaError_t launch_comb_add(const uint32_t* midx, const uint64_t* psum, uint64_t nsegp, uint64_t* counts,
                            cudaStream_t s);
cudaError_t launch_key_lengths_list32(const uint32_t* keys, uint64_t n, uint64_t* lens, cudaStream_t s);
// WC two-level combiner: the nonzero counts of the L2 table -> combiner partial entries
// (key | count << 32) at out[*cursor ...] while *cursor < cap (those entries are zeroed; the rest
// stay for a second call after growing out); *cursor counts every nonzero entry found
cudaError_t launch_xtab_extract(uint32_t* tab, uint64_t nent, uint64_t* out, uint64_t cap,
                                unsigned long long* cursor, int num_sms, cudaStream_t s);
// the same into separate lists (keys u32, counts u64) — the final exact keys — and *wsum += the
// counts (words absorbed)
cudaError_t launch_xtab_extract_list(uint32_t* tab, uint64_t nent, uint32_t* okeys, uint64_t* ocounts, uint64_t cap,
                                     unsigned long long* cursor, unsigned long long* wsum, int num_sms, cudaStream_t s);
// WC long-word table -> the final long keys: 16 zero-padded key bytes per key (okeys, 2 x u64),
// their references (okref = (address of the bytes << 16) | length) and counts; slots reset
cudaError_t launch_ltab_extract(uint64_t* lkeys, uint32_t* lcnt, uint64_t nslots, uint32_t bits, uint64_t* okeys, uint64_t* okref,
                                uint64_t* ocounts, uint64_t cap, unsigned long long* cursor, unsigned long long* wsum,
                                int num_sms, cudaStream_t s);
// WC mid table -> (48-bit key, count) lists; extracted slots are reset (key empty, count 0)
cudaError_t launch_mtab_extract(uint64_t* mkeys, uint32_t* mcnt, uint64_t nslots, uint32_t bits, uint64_t* okeys, uint64_t* ocounts,
                                uint64_t cap, unsigned long long* cursor, unsigned long long* wsum, int num_sms,
                                cudaStream_t s);
cudaError_t launch_key_decode_list32(const uint32_t* keys, uint64_t n, const uint64_t* key_off, uint8_t* out,
                                     cudaStream_t s);
cudaError_t launch_offsets_scaled(const uint64_t* seg_start, uint64_t nseg, uint64_t scale, uint64_t* out,
                                  cudaStream_t s);
cudaError_t launch_iota_scaled(uint64_t n, uint64_t scale, uint64_t* out, cudaStream_t s);
// recompute every key in the 64-bit format with a fresh hash seed (collision slow path)
cudaError_t launch_rehash(uint64_t* h, const uint64_t* kref, uint64_t m, uint64_t seed, cudaStream_t s);

// ---- record directory of '\n'-terminated text (lines.cu) ----
uint64_t line_tiles(uint64_t lo, uint64_t hi);
cudaError_t launch_line_count(const uint8_t* base, uint64_t lo, uint64_t hi, uint32_t* counts, cudaStream_t s);
cudaError_t launch_line_write(const uint8_t* base, uint64_t lo, uint64_t hi, const uint64_t* tile_base, uint64_t* off,
                              cudaStream_t s);

// ---- multi-GPU exchange (exchange.cu) ----
constexpr int kMaxRanks = 64;
enum XMode : int { kXPairs = 0, kXSegs = 1, kXKM = 2, kXSplit = 3 };
struct XEntry { uint64_t koff_len; uint64_t v; };          // WC / II (16 B)
struct XEntryKM { uint64_t id, cnt; double sums[8]; };      // KM partial (80 B)
struct XSource {
  int mode = kXPairs;
  uint32_t nranks = 1;
  uint64_t n = 0;                              // records of the source
  const uint64_t* kref = nullptr;              // kXPairs; kXSplit: hashed-stream krefs
  const uint32_t* hx = nullptr;                // kXSplit: exact-stream keys (nx of them, first),
  uint64_t nx = 0;                             //   then the mid-stream keys (nc), then the hashed
  const uint64_t* hc = nullptr;                //   stream (kref)
  uint64_t nc = 0;
  const uint64_t* hp = nullptr;                // kXSplit: combiner partials (key | count << 32),
  uint64_t np = 0;                             //   after the exact stream
  const uint8_t* v = nullptr;
  int vbytes = 8;
  const uint8_t* keys = nullptr;               // kXSegs
  const uint64_t* key_off = nullptr;
  const uint64_t* counts = nullptr;
  const double* sums = nullptr;                // kXKM
  const unsigned long long* cnts = nullptr;
  const unsigned long long* heap_base = nullptr;  // device: heap slice start of every destination
};
uint32_t km_owner(uint32_t j, uint32_t nranks);
cudaError_t launch_x_count(const XSource& S, unsigned long long* counts, int num_sms, cudaStream_t s);
cudaError_t launch_x_scatter(const XSource& S, unsigned long long* cursors, uint8_t* entries, uint8_t* heap,
                             cudaStream_t s);
cudaError_t launch_x_ingest(const void* entries, const uint8_t* heap, uint64_t n, const uint64_t* src_e,
                            const uint64_t* src_h, uint32_t R, uint64_t* h, uint64_t* kref, uint64_t* v,
                            uint64_t seed, uint32_t weak, uint32_t key_bits, cudaStream_t s);
cudaError_t launch_x_ingest_km(const void* entries, uint64_t n, double* sums, unsigned long long* cnts, uint32_t k,
                               cudaStream_t s);

}  // namespace bmr
