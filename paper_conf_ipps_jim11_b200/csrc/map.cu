// map.cu — the Map phase: persistent, warp-specialised CTAs.
//
// PAPER.md §III (L66-113) stages input into shared memory, runs the user Map per record,
// collects results in a shared-memory output area and flushes it to global memory with one
// global atomic per flush.  Its GT200 mechanics (16 KB SMEM, all threads alternating between
// stage-in / compute / stage-out, software wait-signal flags, yield by dummy global reads) are
// prior art; the B200 re-derivation here (one persistent CTA per SM):
//   * two producer warps (A1/A2): an elected lane issues TMA bulk copies (cp.async.bulk) of the
//     tile bytes and of the tile's record-offset slice into an SMEM ring (WordCount 4 stages,
//     InvertedIndex 6, KMeans 8, StringMatch 12 of bytes only) guarded by mbarrier full/empty
//     pairs; WordCount / InvertedIndex take tiles from a global counter; kLag tiles later the
//     producer turns the staged offsets into a record-start bitmap and releases the stage
//     (ready mbarrier) — replaces the barrier-separated staging loop (L68, L85);
//   * map warps (A3; 24 for StringMatch / InvertedIndex, 25 for WordCount, 16 for KMeans): byte-parallel, record-agnostic
//     scanning — each lane owns a 16-byte chunk of a 512-B window, record boundaries come from
//     the bitmap; no map-warp barrier at all, so the per-record imbalance the paper blames for
//     SO overhead (L273) disappears;
//   * emit allocator (A11/A12, D3/D4): a warp result is reserved with ONE shared 32-bit
//     atomicAdd on a packed [generation:6 | cb:12 | ca:14] cursor of the current output buffer;
//   * overflow (A13, L113): the unique warp whose reservation crosses the buffer's capacity
//     seals it and switches every warp to the next buffer of a 4-buffer ring at once (replaces
//     the wait/signal flag protocol, L96-100); it waits only if all buffers are still flushing;
//   * flush warp (A4): waits (acquire loads) for the sealed buffer's in-flight writers, takes ONE
//     global atomicAdd for the whole buffer, and writes its SoA arrays with TMA bulk stores
//     (cp.async.bulk.global.shared::cta).  Flushes are rounded to 4 pairs (16-B alignment) with
//     sentinel filler pairs.  The global cursor counts demand even past capacity (D7), so the
//     host can grow the buffers and replay the batch.
#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include <climits>

#include "common.cuh"

namespace bmr {
namespace {

// Map warps per CTA: KMeans 16 (one 32-point slice each of a 512-point tile); the text workloads
// 24 (their Map is issue-bound on dependent integer chains: more warps per scheduler hide them)
constexpr int kNMap = 16;
#ifndef BMR_SM_NMAP
#define BMR_SM_NMAP 24   // StringMatch map warps
#endif
#ifndef BMR_WC_COMB_BITS
#define BMR_WC_COMB_BITS 13     // WordCount SMEM combiner: 2^bits direct-mapped slots (u32 key + u32 count);
                                // 13 (64 KB): round 1, exact stream 672 M -> 599 M keys; round 2 (L2 count
                                // table behind it): 12 bits cost the C5 Map 0.5 ms in extra REDs
#endif
#ifndef BMR_WC_LQ
#define BMR_WC_LQ 32            // WordCount long-word queue entries per map warp (>= 32; 64 measured no better)
#endif
#ifndef BMR_WC_OUT_BYTES
#define BMR_WC_OUT_BYTES 3072   // WordCount output buffer bytes (x kNOut).  With the L2 count table and the
                                // warp-chunked long-word output only rare > 16-byte words pass through them
                                // (C5 Map, round 2: 4 KB 21.2 ms, 3 KB 18.0 ms, 2.6 KB 17.9 ms)
#endif
#ifndef BMR_WC_OFFCAP
#define BMR_WC_OFFCAP 640       // WordCount: record offsets staged per tile (C1/C5 lines >= 27 B: <= 617 per
                                // staged window; denser tiles read offsets from global memory)
#endif
#ifndef BMR_KM_UNROLL
#define BMR_KM_UNROLL 8   // KMeans: centroid pairs per unrolled distance-loop iteration (C3: 2 -> 8, Map 1.97 -> 1.91 ms)
#endif
constexpr int kKmUnroll = BMR_KM_UNROLL;
#ifndef BMR_WC_COMB_PROBES
#define BMR_WC_COMB_PROBES 1   // WordCount combiner probes per word (2: C5 absorbs 4.6% more words but the Map costs 0.9 ms more than the sort saves)
#endif
#ifndef BMR_SM_DYN
#define BMR_SM_DYN 1   // StringMatch super-windows: 0 static round-robin, 1 shared counter (C2 Map 1.03 -> 0.81 ms)
#endif
#ifndef BMR_SM_WAIT_NS
#define BMR_SM_WAIT_NS 1000   // StringMatch map warps: suspend-time hint of the stage wait (0: spin)
#endif
#ifndef BMR_SM_SUB
#define BMR_SM_SUB 4     // StringMatch 512-B windows per map-warp super-window
#endif
constexpr int kNMapText = 24;
#ifndef BMR_WC_NMAP
#define BMR_WC_NMAP 25   // WordCount map warps (24 -> 25: C5 Map 11.79 -> 11.68 ms; 28 warps x 72 registers fill the register file)
#endif
#ifndef BMR_II_STAGES
#define BMR_II_STAGES 6    // InvertedIndex stages in flight per SM (round 2: 4 -> 6 with 8 KB output
                           // buffers, C4 Map 7.81 -> 7.66 ms)
#endif
#ifndef BMR_II_OUT_BYTES
#define BMR_II_OUT_BYTES 8192   // InvertedIndex output buffer bytes (x kNOut; 24-B pairs, ~1 per 500 B)
#endif
#ifndef BMR_KM_STAGES
#define BMR_KM_STAGES 8      // KMeans stages in flight per SM (round 3: with the bound test the KM Map is
                             // read-bound, 4 x 16 KiB in flight per SM capped it at ~1/3 of HBM)
#endif
#ifndef BMR_KM_OUT_BYTES
#define BMR_KM_OUT_BYTES 4096   // KMeans output buffer bytes (x kNOut; only the sorted path, NO_MAP_COMBINE, emits)
#endif
#ifndef BMR_II_NMAP
#define BMR_II_NMAP 24   // InvertedIndex map warps
#endif
template <int W>
constexpr int nmap() { return W == 3 ? kNMap : W == 2 ? BMR_SM_NMAP : W == 4 ? BMR_II_NMAP : BMR_WC_NMAP; }
// Producer warps kProdWarp0 .. + kNProd - 1: producer p owns the iterations it == p (mod kNProd)
// (and so the stages s == p (mod kNProd)); one warp alone is latency-bound at ~465 instructions
// per tile (TMA issue + bitmap), slower than HBM delivers a tile (ncu, C2 round 1).
#ifndef BMR_II_NPROD
#define BMR_II_NPROD 2
#endif
template <int W>
constexpr int nprod() { return W == 4 ? BMR_II_NPROD : 2; }
// Flush warps (flush_loop takes generations f == fw mod nflush).  One: a second WordCount flush
// warp removed the map warps' spinning on sealed buffers but cost the Map more than it saved
// (C5 Map 20.4 -> 21.3 ms, round 2: a 28th warp lowers the register budget of every warp).
// Warps: map 0 .. nmap-1, producers nmap .. nmap+kNProd-1, then the flush warps.
#ifndef BMR_LTAB
#define BMR_LTAB 1
#endif
#ifndef BMR_STREAM_HINT
#define BMR_STREAM_HINT 1   // WC Map input TMA loads L2 evict-first (C5 Map 21.4 -> 20.5 ms, DRAM 15.8 -> 14.4 GB)
#endif
#ifndef BMR_MID_MATCH
#define BMR_MID_MATCH 1
#endif
#ifndef BMR_MID_LDCA
#define BMR_MID_LDCA 0
#endif
#ifndef BMR_WC_TAB
#define BMR_WC_TAB 1   // WordCount table mode: per-lane start loop (wc_window_tab); 0: the queued rounds of wc_window
#endif
#ifndef BMR_WC_LSCAN
#define BMR_WC_LSCAN 1   // WordCount table mode: long words of <= 16 bytes queued at their warp rank (no rounds)
#endif
#ifndef BMR_WC_XLOOP
#define BMR_WC_XLOOP 1   // WordCount table mode: lean exact-word loop (bfind starts, 32-bit shared addresses, unconditional shared RED)
#endif
#ifndef BMR_WC_XPAIR
#define BMR_WC_XPAIR 1   // WordCount table mode: two exact words per loop iteration
#endif
#ifndef BMR_WC_LBALLOT
#define BMR_WC_LBALLOT 1   // WordCount table mode: long-word queue offsets from ballots (no shuffle scan)
#endif
#ifndef BMR_WC_X2WAY
#define BMR_WC_X2WAY 0   // WordCount table mode: second combiner slot (home ^ 1) for exact words
#endif
#ifndef BMR_WC_PAIRWIN
#define BMR_WC_PAIRWIN 1   // WordCount table mode: two 512-B windows per window fetch
#endif
#ifndef BMR_II_PAIRWIN
#define BMR_II_PAIRWIN 1   // InvertedIndex: two 512-B windows per window fetch
#endif
#ifndef BMR_WC_UNITAB
#define BMR_WC_UNITAB 1   // WordCount table mode: words of 6..16 symbols in one 16-byte-key table
#endif
#ifndef BMR_II_LAG
#define BMR_II_LAG 2   // InvertedIndex: tiles between a stage's TMA issue and its bitmap (4 = stages - 2: C4 Map 7.72 ms; 2: 6.55 ms)
#endif
#ifndef BMR_WC_CLS16
#define BMR_WC_CLS16 1   // WordCount table mode: each lane classifies its own 16 bytes only (next chunk by shuffle)
#endif
#ifndef BMR_WC_ADRAIN
#define BMR_WC_ADRAIN 1   // WordCount table mode: long-word table probes prefetched by cp.async one drain ahead
#endif
#ifndef BMR_DYN_TILES
#define BMR_DYN_TILES 1   // WordCount / InvertedIndex: tiles from a global counter (producer_loop_dyn)
#endif
#ifndef BMR_WC_NFLUSH
#define BMR_WC_NFLUSH 1u
#endif
template <int W>
constexpr uint32_t nflush() { return W == kWC ? BMR_WC_NFLUSH : 1u; }
template <int W>
constexpr int threads_of() { return (nmap<W>() + nprod<W>() + static_cast<int>(nflush<W>())) * 32; }
constexpr int kT = static_cast<int>(kMapTileBytes);   // owned bytes per tile (text) / bytes per tile (KM)
constexpr int kLead = 16;        // bytes staged before the tile (previous-byte context)
constexpr int kHalo = 256;       // bytes staged after the tile (words / matches / URLs crossing it)
constexpr int kWin = 512;        // bytes per warp window = 32 lanes x 16 B
constexpr int kNWin = kT / kWin;
constexpr int kStageBytes = 16768;             // >= kLead + kT + kHalo + 32, multiple of 128
static_assert(kStageBytes <= (1 << 15), "WC long-word queue entries hold a 15-bit stage offset");
constexpr int kBitWords = kStageBytes / 32 + 4;
constexpr int kBitBytes = 2176;                // >= kBitWords * 4, multiple of 128
constexpr int kNOut = 4;         // output buffers in the flush ring (generation g uses buffer g % kNOut)
// Per-workload SMEM budget: StringMatch is read-bound with almost no output -> more input stages
// (more bytes in flight per SM) and small output buffers; the emitting workloads keep 4 stages
// and 4 x 20 KB output buffers.
#ifndef BMR_SM_STAGES
#define BMR_SM_STAGES 12   // StringMatch stages in flight per SM (12 x 16.4 KiB)
#endif
template <int W>
struct Cfg {
  // StringMatch (read-bound, almost no output, lazy record directory below: no offsets or bitmap
  // regions): 8 stages of bytes in flight
  static constexpr int kStages = (W == kSM) ? BMR_SM_STAGES : (W == kII) ? BMR_II_STAGES : (W == kKM) ? BMR_KM_STAGES : 4;
  // record offsets staged per tile (more: read from global); KM has fixed-stride records
  static constexpr int kOffCap = (W == kSM || W == kKM) ? 0 : (W == kWC) ? BMR_WC_OFFCAP : 1024;
  // StringMatch reads the record directory lazily: record boundaries matter only where the
  // pattern's first byte matches (planted, rare), so no offsets are staged and no bitmap is built;
  // a candidate checks for a record start inside its 16 bytes by a binary search over the tile's
  // offsets slice in global memory.  The producers only issue the byte TMA.
  static constexpr bool kLazyDir = (W == kSM);
  static constexpr int kOffBytes = (W == kSM || W == kKM) ? 0 : ((kOffCap + 2) * 8 + 127) / 128 * 128;
  static constexpr int kBits = (W == kSM || W == kKM) ? 0 : kBitBytes;   // record-start bitmap bytes per stage
  static constexpr int kOutHalf = (W == kSM) ? 4096 : (W == kWC) ? BMR_WC_OUT_BYTES : (W == kII) ? BMR_II_OUT_BYTES : BMR_KM_OUT_BYTES;   // bytes per output buffer
  // the producer builds the bitmap of tile it - kLag right after issuing tile it: kLag stages of
  // TMA traffic stay in flight per SM while one stage is being consumed
  static constexpr int kLag = (W == kII) ? BMR_II_LAG : kStages - 2;
  static_assert(kStages % nprod<W>() == 0 && kLag % nprod<W>() == 0, "a producer owns every kNProd-th stage");
  // WC: per-warp queue of the window's long (hashed) words, hashed by all 32 lanes together
  // after the emission rounds (a lane-per-word hash inside the rounds diverges: with 10% long
  // words, most rounds would carry at least one).  A window holds at most 512 / 6 + 1 starts
  // of words longer than kWcExact bytes.
  static constexpr int kHashQ = (W == kWC) ? 96 : (W == kII) ? 192 : 0;   // II: URL queue, 64 x (u64 pos + u32 len)
  // WC: per-warp queue of the window's exact keys that missed the combiner (u32), copied into
  // the output buffer after the one reservation; <= 257 word starts per window
  static constexpr int kXQ = (W == kWC) ? 264 : 0;
  // WC: in-SMEM combiner (MapCG-style): kCombSlots u64 entries
  // (u32 exact keys + u32 counts), direct-mapped, a slot keeps the first key that claims it
  static constexpr int kCombSlots = (W == kWC) ? (1 << BMR_WC_COMB_BITS) : 0;
  // WC: per-warp queue of long words (> kWcExact bytes, <= 16) carried ACROSS windows with their
  // bytes, so the stage can be released: keyed 32 at a time (one reservation per 32 words)
  static constexpr int kLQ = (W == kWC) ? BMR_WC_LQ : 0;
};
struct LWord { uint64_t lo, hi, meta; };   // key bytes 0..7, 8..15; (batch position << 16) | length
constexpr uint32_t kLQMaxLen = 16;
constexpr int kCombBits = BMR_WC_COMB_BITS;
static_assert(Cfg<kWC>::kCombSlots == (1 << kCombBits), "combiner slots");
constexpr uint32_t kCombEmpty32 = 0xFFFFFFFFu;   // exact keys are < 2^30
// WC words of <= kWcExact bytes get an exact 30-bit key (common.cuh exact_key30) and travel in
// the exact stream (4-B u32 entries: the key is the whole record).  Longer words are queued; in the
// queue pass words of <= kMidMax bytes get an exact 48-bit key (mid stream, key only), longer
// ones a hash (hashed stream, with their key reference).  Queued entries are 16 B (key, kref;
// kref 0 marks a mid-stream key) and the flush warp routes them.
constexpr uint32_t kWcExact = kExactMax;
static_assert(kWin / (kWcExact + 1) + 1 <= Cfg<kWC>::kHashQ, "hash queue too small");
static_assert(kWin / 2 + 1 <= Cfg<kWC>::kXQ, "exact-key queue too small");
constexpr int kKmPts = kT / 32;                // 512 points per KM tile
// KM combiner (k <= kKmCombMax): per-warp fp32 accumulators [kNMap][64][8] + counts [kNMap][64]
// in the (otherwise unused for KM) offsets + bitmap stage regions
constexpr int kKmCombMax = 64;
// KM bound test (MR_FLAG_KM_FULL_SCAN off): for k <= kKmBoundMax the CTA keeps a row-layout copy of
// the centroids and s2[g] = (squared distance from centroid g to its nearest other centroid,
// rounded down) after the paired copy.  A point whose fp32 distance d_g to its lane's previous
// winner g satisfies 4 d_g (1 + 1e-5) < s2[g] is assigned g: exactly, ||x - c_g|| < s/2 gives
// ||x - c_j|| >= s - ||x - c_g|| > ||x - c_g|| for every j != g (triangle inequality), and the
// 1e-5 margin exceeds the relative error of the two fp32 distance chains (<= ~10 ulp each), so
// the fp32 d_j the full scan would compute are all strictly greater than d_g.
constexpr int kKmBoundMax = 128;
constexpr float kKmBoundFactor = 4.00004f;
constexpr int kKmWaccBytes = kNMap * kKmCombMax * 8 * 4;

static_assert(kLead + kT + kHalo + 32 <= kStageBytes, "stage too small");
static_assert(kBitWords * 4 <= kBitBytes, "bitmap too small");
static_assert(kKmPts == kNMap * 32, "one KM point per map lane");

struct StageHdr {
  long long t;                   // tile id (-1: end of work)
  long long sbase;               // input position of stage byte 0
  long long chunk0;              // first (possibly negative) position of the tile's chunk grid
  long long lo, hi;              // owned positions [lo, hi) clipped to [0, N); KM: points
  long long stg_hi;              // staged bytes cover positions < stg_hi
  unsigned long long ra, rb;     // record starts staged: offsets[ra..rb)
  unsigned int off_shift;        // byte offset of offsets[ra] inside the offsets region
  unsigned int off_staged;       // offsets slice is in SMEM
};

struct OutCtl {
  unsigned int cur;              // [generation:6 | cb:12 | ca:14]; buffer = generation % kNOut
  unsigned int final_seq;        // full generation number of the final flush
  unsigned int committed[kNOut];     // entries fully written into each buffer (current generation)
  unsigned int fcount[kNOut];        // sealed entry count of each buffer
  unsigned long long fbase[kNOut];   // global base reserved for the sealed buffer (one atomic per flush)
  unsigned int nsealed, is_final;  // sealed generations so far (full count); final flush flag
  unsigned int win_next;         // text: next window (tile * kNWin + window) to hand to a map warp
  unsigned int congested;        // the sealing warp waits for a flushing buffer: overflowing warps spill
  uint64_t req[kNOut];           // mbarrier: buffer sealed -> flush warp
  uint64_t done[kNOut];          // mbarrier: buffer flushed -> free
  unsigned int pout[2];          // dynamic tiles: first iteration producer p found no tile (~0: not yet)
  unsigned int plast[2];         // dynamic tiles: last iteration producer p filled with a tile (+1; 0: none)
};

template <int W>
struct Layout {
  static constexpr int kStages = Cfg<W>::kStages;
  static constexpr int ctl = 0;                                   // OutCtl
  static constexpr int hdr = 256;                                 // kStages x 128
  static constexpr int full = hdr + kStages * 128;                // kStages x 8
  static constexpr int empty = full + kStages * 8;
  static constexpr int ready = empty + kStages * 8;               // kStages x 8 (text: bitmap built)
  static constexpr int bytes = (ready + kStages * 8 <= 2048) ? 2048 : (ready + kStages * 8 + 127) / 128 * 128;   // kStages x kStageBytes
  static constexpr int offs = bytes + kStages * kStageBytes;      // kStages x kOffBytes
  static constexpr int bits = offs + kStages * Cfg<W>::kOffBytes; // kStages x kBitBytes
  static constexpr int out = bits + kStages * Cfg<W>::kBits;      // kNOut x Cfg<W>::kOutHalf
  static constexpr int hq = out + kNOut * Cfg<W>::kOutHalf;       // nmap x kHashQ x 4 (WC)
  static constexpr int xq = hq + nmap<W>() * Cfg<W>::kHashQ * 4;  // nmap x kXQ x 4 (WC)
  static constexpr int comb = xq + nmap<W>() * Cfg<W>::kXQ * 4;   // kCombSlots x 8 (WC)
  static constexpr int lq = comb + Cfg<W>::kCombSlots * 8;        // nmap x kLQ x 24 (WC)
  static constexpr int kmacc = lq + nmap<W>() * Cfg<W>::kLQ * 24;  // KM combiner: per-warp fp32 sums + counts
  static constexpr int cent = kmacc + ((W == kKM) ? kKmWaccBytes + kNMap * kKmCombMax * 4 : 0);   // KM centroids
  static_assert(sizeof(OutCtl) <= hdr, "OutCtl overlaps the stage headers");
};
static_assert(64 % kNOut == 0, "6-bit generation counter must wrap on a buffer boundary");
static_assert(Layout<kWC>::cent <= 232448 && Layout<kSM>::cent <= 232448 && Layout<kII>::cent <= 232448 &&
                  Layout<kKM>::cent + 1024 * 32 <= 232448,
              "SMEM layout exceeds 227 KB per CTA");


// Output-buffer formats.  SM / KM / II: SoA runs [keys | krefs | values] of kCap entries.
// WC: exact-key entries (u32 key) fill the buffer from the bottom, queued long-word entries (u64
// key, u64 kref) from the top; capacity is counted in 4-byte units (exact 1, queued 4).  WC
// values are all 1 and are not stored: a key's count is its segment length.
template <int W>
struct PairFmt {
  static constexpr bool kKref = (W == kII);
  static constexpr int kV = (W == kKM) ? 32 : (W == kII) ? 8 : 0;
  static constexpr int kPairBytes = 8 + (kKref ? 8 : 0) + kV;
  static constexpr uint32_t kCap = (W == kWC) ? (Cfg<W>::kOutHalf / 4 - 4) : (Cfg<W>::kOutHalf / kPairBytes) & ~3u;
  // largest single warp reservation (units): WC <= 257 word starts in 512 B (a start follows a
  // delimiter; +1 crossing word) of which <= kHashQ queued (4 units each), SM 16 matches / 16 B,
  // II 2, KM 1 per lane
  static constexpr uint32_t kMaxReserve = (W == kWC) ? 257 + 4 * Cfg<kWC>::kHashQ : (W == kSM) ? 512 : 32 * ((W == kII) ? 2 : 1);
  static_assert(kCap >= kMaxReserve, "output half smaller than one warp result");
};

// Dimensions of the mapped batch: (byte length, tiles, global byte base).  Text batches are
// enqueued without a host round trip (mr_map never reads offsets[n] back): k_tile_bounds derives
// them from offsets[n] on the device into the batch's descriptor, and every CTA of k_map copies
// them into shared memory at start-up.  Fixed-stride batches (KM) carry host values.
__shared__ unsigned long long s_bd[4];
__device__ __forceinline__ long long bd_nbytes() { return static_cast<long long>(s_bd[0]); }
__device__ __forceinline__ uint64_t bd_ntiles() { return s_bd[1]; }
__device__ __forceinline__ uint64_t bd_gbase() { return s_bd[2]; }

struct Params {
  const uint8_t* rec;
  const uint64_t* off;
  uint64_t n, nbytes;
  long long a0;            // rec & 15 (text chunk alignment)
  uint64_t ntiles;
  uint64_t gbase;
  uint32_t pat[4];
  const float* cent;
  uint32_t k;
  uint64_t* oh;
  uint64_t* okref;
  uint8_t* ov;
  uint64_t cap_pairs;
  uint64_t* ohb;           // WC hashed stream: keys, krefs, capacity
  uint64_t* okrefb;
  uint64_t cap_b;
  uint64_t* ohc;           // WC mid stream: keys, capacity
  uint64_t cap_c;
  uint32_t* ohx;           // WC exact stream: u32 keys (capacity cap_pairs)
  uint64_t* ohp;           // WC combiner partials: (exact key | count << 32), capacity cap_p
  uint64_t cap_p;
  uint32_t comb;           // WC / KM: in-SMEM combiner on
  double* km_sums;         // KM combiner: job accumulators (k x 8 fp64, k u64), zeroed by the host
  unsigned long long* km_cnts;
  uint32_t out_cap;        // per-half capacity actually used (FORCE_TINY_OUT shrinks it)
  uint32_t flags;
  DevState* st;
  const uint64_t* tb;      // tile bounds
  const uint8_t* off_end;  // end of the offsets array rounded DOWN to 16 B (aligned TMA limit)
  uint64_t hash_seed;
  uint32_t key_bits;       // sort-key width (48 or 64)
  uint32_t pf;             // L2 prefetch distance in producer tiles (0: off)
  uint32_t wait_hint;      // idle mbarrier waits: 0 plain try_wait, 1 suspend-time hint, 2 helpers sleep-poll
  uint32_t dyn;            // text: windows handed out dynamically (1) or in static warp order (0)
  // memory-mode ablations (§IV-C): so = no input staging
  // (map warps read record bytes from global memory; the record directory is still staged),
  // si = no output staging (each warp result is appended to global memory with one global
  // atomic per warp, L135 / L171-173); both = the paper's G mode
  uint32_t so, si;
  uint32_t sm_lines;       // StringMatch: emit the matching record's start (MR_FLAG_SM_LINES)
  uint32_t wc_bal;         // WordCount: balanced two-phase emission (BMR_WC_BAL, default on)
  uint32_t wc_fast;        // WordCount: wc_map_loop / wc_window (BMR_WC_FAST, default on)
  const XWindow* xwin;     // f-3: InvertedIndex records appended straight to these windows
  uint32_t xranks;         // number of windows (0: local output)
  const uint64_t* desc;    // text: the batch descriptor (nbytes, ntiles, gbase, tile-bounds overflow)
  uint32_t* xtab;          // WC: second combiner level, the L2-resident direct-address count table
                           // (2^30 u32 counts indexed by the exact key); nullptr: exact stream
  uint64_t* mkeys;         // WC: mid words (6..8 symbols) counted in an open-addressing table of
  uint32_t* mcnt;          //   their 48-bit exact keys (2^mbits slots); nullptr: mid stream
  uint32_t mbits;
  uint64_t* lkeys;         // WC: words of 9..16 symbols counted in an open-addressing table of their
  uint32_t* lcnt;          //   16 zero-padded key bytes (2^lbits slots); nullptr: hashed stream
  uint32_t lbits;
  uint32_t km_bound;       // KM: the exact bound test before the full centroid scan (kKmBoundMax)
  unsigned long long* tile_next;   // text (WC / II): dynamic tile counter of the batch (zeroed by k_tile_bounds)
};

// Idle wait of a role warp on an mbarrier phase (map warps on a staged tile, producers on a free
// stage, the flush warp on a sealed buffer).
__device__ __forceinline__ void map_wait(const Params& P, uint64_t* bar, uint32_t parity, uint32_t ns) {
  if (P.wait_hint == 1) mbar_wait_idle(bar, parity, ns);
  else mbar_wait(bar, parity);
}
// Waits of the helper warps (producers on a free stage, the flush warp on a sealed buffer): with
// wait_hint == 2 they poll with __nanosleep between attempts, leaving issue slots to the map
// warps (the Map of the text workloads is issue-bound).
__device__ __forceinline__ void helper_wait(const Params& P, uint64_t* bar, uint32_t parity, uint32_t sleep_ns) {
  if (P.wait_hint == 2) {
    while (!mbar_try_wait(bar, parity)) __nanosleep(sleep_ns);
  } else {
    map_wait(P, bar, parity, 20000);
  }
}

constexpr uint32_t kFull = 0xffffffffu;
constexpr uint32_t kReadyWaitNs = 2000;   // map warps: suspend hint while waiting for a staged tile

// ---------------------------------------------------------------- packed fp32 (sm_100a FADD2/FFMA2)
__device__ __forceinline__ uint64_t f2pack(float a, float b) {
  uint64_t r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b));
  return r;
}
__device__ __forceinline__ void f2unpack(uint64_t v, float& a, float& b) {
  asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(v));
}
__device__ __forceinline__ uint64_t f2sub(uint64_t a, uint64_t b) {
  uint64_t r;
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
  return r;
}
__device__ __forceinline__ uint64_t f2fma(uint64_t a, uint64_t b, uint64_t c) {
  uint64_t r;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c));
  return r;
}

// ---------------------------------------------------------------- byte-class helpers
__device__ __forceinline__ uint32_t movemask4(uint32_t m) {  // 0xFF/0x00 bytes -> 4 bits
  return ((((m >> 7) & 0x01010101u) * 0x01020408u) >> 24) & 0xFu;
}
__device__ __forceinline__ uint32_t word_mask4(uint32_t x) {  // [0-9A-Za-z] (C-3 #1)
  // carry-free byte compares on the low 7 bits (bias so that bit 7 flags c >= bound), bytes
  // >= 0x80 excluded: 4 x (digit or letter) -> 4 bits
  const uint32_t x7 = x & 0x7F7F7F7Fu;
  const uint32_t l = x7 | 0x20202020u;                         // letters -> 0x61..0x7A
  const uint32_t dig = (x7 + 0x50505050u) & ~(x7 + 0x46464646u);   // 0x30 <= c < 0x3A
  const uint32_t alp = (l + 0x1F1F1F1Fu) & ~(l + 0x05050505u);     // 0x61 <= l < 0x7B
  const uint32_t m = (dig | alp) & ~x & 0x80808080u;
  return ((m >> 7) * 0x01020408u) >> 24;
}
__device__ __forceinline__ uint32_t eq_mask4(uint32_t x, uint32_t b4) {   // bytes == b4's -> 4 bits
  // exact per-byte zero test of x ^ b4 (no borrow crosses a byte: (t & 0x7F) + 0x7F <= 0xFE)
  const uint32_t t = x ^ b4;
  const uint32_t z = ~(((t & 0x7F7F7F7Fu) + 0x7F7F7F7Fu) | t | 0x7F7F7F7Fu);
  return ((z >> 7) * 0x01020408u) >> 24;
}
__device__ __forceinline__ bool is_word_byte(uint32_t c) {
  return (c - '0' < 10u) || ((c | 0x20u) - 'a' < 26u);
}
// bits j (0..31) with lo <= p0 + j < hi
__device__ __forceinline__ uint32_t range_mask32(long long p0, long long lo, long long hi) {
  long long a = lo - p0, b = hi - p0;
  uint32_t mb = b >= 32 ? kFull : (b <= 0 ? 0u : ((1u << b) - 1u));
  uint32_t ma = a <= 0 ? kFull : (a >= 32 ? 0u : ~((1u << a) - 1u));
  return ma & mb;
}
__device__ __forceinline__ uint32_t bits32(const uint32_t* bm, long long i0) {  // i0 % 16 == 0
  uint32_t wi = static_cast<uint32_t>(i0 >> 5), sh = static_cast<uint32_t>(i0 & 31);
  return sh ? ((bm[wi] >> 16) | (bm[wi + 1] << 16)) : bm[wi];
}
// select 3 consecutive words x[wi..wi+2] of an 8-word window (wi in 0..3, no local memory)
__device__ __forceinline__ uint64_t window8(const uint32_t (&x)[8], uint32_t j) {
  // branch-free selection (selects, not a divergent switch): words j/4 .. j/4 + 2
  const uint32_t sh = (j & 3) * 8;
  const bool b2 = (j & 8) != 0, b1 = (j & 4) != 0;
  const uint32_t w0 = b2 ? x[2] : x[0], w1 = b2 ? x[3] : x[1], w2 = b2 ? x[4] : x[2], w3 = b2 ? x[5] : x[3];
  const uint32_t a = b1 ? w1 : w0, b = b1 ? w2 : w1, c = b1 ? w3 : w2;
  return (static_cast<uint64_t>(__funnelshift_r(b, c, sh)) << 32) | __funnelshift_r(a, b, sh);
}
// 16 bytes starting at j (0..15) of the 8-word window, as 4 words
__device__ __forceinline__ void window16(const uint32_t (&x)[8], uint32_t j, uint32_t (&o)[4]) {
  uint32_t wi = j >> 2, sh = (j & 3) * 8, y0, y1, y2, y3, y4;
  switch (wi) {
    case 0: y0 = x[0]; y1 = x[1]; y2 = x[2]; y3 = x[3]; y4 = x[4]; break;
    case 1: y0 = x[1]; y1 = x[2]; y2 = x[3]; y3 = x[4]; y4 = x[5]; break;
    case 2: y0 = x[2]; y1 = x[3]; y2 = x[4]; y3 = x[5]; y4 = x[6]; break;
    default: y0 = x[3]; y1 = x[4]; y2 = x[5]; y3 = x[6]; y4 = x[7]; break;
  }
  o[0] = __funnelshift_r(y0, y1, sh); o[1] = __funnelshift_r(y1, y2, sh);
  o[2] = __funnelshift_r(y2, y3, sh); o[3] = __funnelshift_r(y3, y4, sh);
}

// smallest record start > p (global binary search over offsets[0..n]; rare slow path)
__device__ uint64_t next_start_after(const uint64_t* off, uint64_t n, uint64_t p) {
  uint64_t lo = 0, hi = n + 1;  // first index with off[i] > p
  while (lo < hi) {
    uint64_t mid = (lo + hi) >> 1;
    if (off[mid] > p) hi = mid; else lo = mid + 1;
  }
  return lo <= n ? off[lo] : ~0ULL;
}

struct TileView {
  const uint8_t* sb;       // stage bytes
  const uint32_t* bm;      // record-start bitmap
  long long sbase, stg_hi;
  unsigned long long ra, rb;   // the tile's record starts offsets[ra..rb) (lazy directory)
  __device__ bool is_start(long long q) const {
    long long i = q - sbase;
    return (bm[i >> 5] >> (i & 31)) & 1u;
  }
};

// Word length for a word at position p whose end lies beyond the 32-byte window [p0, p0+32).
__device__ uint32_t slow_word_len(const Params& P, const TileView& tv, long long p, long long from) {
  long long q = from;
  const long long N = bd_nbytes();
  const long long lim = min(tv.stg_hi, N);
  // inside the stage: 4 bytes per step (SWAR word classes + bitmap record starts)
  while (q < lim && ((q - tv.sbase) & 3)) {
    if (tv.is_start(q) || !is_word_byte(tv.sb[q - tv.sbase])) return static_cast<uint32_t>(q - p);
    ++q;
  }
  while (q + 4 <= lim) {
    const long long i = q - tv.sbase;
    const uint32_t w = *reinterpret_cast<const uint32_t*>(tv.sb + i);
    const uint32_t m = ((~word_mask4(w)) & 0xFu) | ((tv.bm[i >> 5] >> (i & 31)) & 0xFu);
    if (m) return static_cast<uint32_t>(q + (__ffs(m) - 1) - p);
    q += 4;
  }
  while (q < lim) {
    if (tv.is_start(q) || !is_word_byte(tv.sb[q - tv.sbase])) return static_cast<uint32_t>(q - p);
    ++q;
  }
  if (q >= N) return static_cast<uint32_t>(q - p);
  // beyond the staged halo (words longer than ~256 bytes): global memory, record end by search
  const uint64_t rec_end = next_start_after(P.off, P.n, static_cast<uint64_t>(p));
  for (; q < N && static_cast<uint64_t>(q) < rec_end; ++q)
    if (!is_word_byte(P.rec[q])) break;
  return static_cast<uint32_t>(q - p);
}

// Position of the closing '"' of a URL starting at q0, or -1 if the record (or input) ends
// first.  Scans the stage 16 bytes at a time, then global memory (slow path).
__device__ long long find_quote(const Params& P, const TileView& tv, long long q0, long long p_marker) {
  const long long N = bd_nbytes();
  const long long lim = min(tv.stg_hi, N);
  long long q = q0;
  while (q < lim && ((q - tv.sbase) & 3)) {               // align to a 4-byte SMEM word
    if (tv.is_start(q)) return -1;
    if (tv.sb[q - tv.sbase] == '"') return q;
    ++q;
  }
  while (q + 4 <= lim) {                                   // 4 bytes per step (SWAR)
    const long long i = q - tv.sbase;
    const uint32_t w = *reinterpret_cast<const uint32_t*>(tv.sb + i);
    const uint32_t st = (tv.bm[i >> 5] >> (i & 31)) & 0xFu;
    const uint32_t m = eq_mask4(w, 0x22222222u) | st;
    if (m) {
      const uint32_t j = __ffs(m) - 1;
      return ((st >> j) & 1u) ? -1 : q + j;               // record ends first -> unclosed
    }
    q += 4;
  }
  while (q < lim) {
    if (tv.is_start(q)) return -1;
    if (tv.sb[q - tv.sbase] == '"') return q;
    ++q;
  }
  if (q >= N) return -1;
  uint64_t rec_end = next_start_after(P.off, P.n, static_cast<uint64_t>(p_marker));
  for (; q < N && static_cast<uint64_t>(q) < rec_end; ++q)
    if (P.rec[q] == '"') return q;
  return -1;
}

// Same function as hash_bytes (common.cuh) for a key lying inside the SMEM stage: aligned
// 4-byte SMEM loads + funnel shifts instead of byte loads.
__device__ __forceinline__ uint32_t smem_word_at(const uint8_t* sb, uint32_t i) {  // 4 bytes at any i
  const uint32_t a = i & ~3u, sh = (i & 3u) * 8;
  const uint32_t w0 = *reinterpret_cast<const uint32_t*>(sb + a);
  if (!sh) return w0;
  const uint32_t w1 = *reinterpret_cast<const uint32_t*>(sb + a + 4);
  return __funnelshift_r(w0, w1, sh);
}
__device__ __forceinline__ uint64_t hash_smem(const uint8_t* sb, uint32_t i, uint32_t len, uint64_t seed) {
  KeyHash hs(seed, len);
  uint32_t k = 0;
  for (; k + 4 <= len; k += 4) hs.add(smem_word_at(sb, i + k));
  if (k < len) hs.add(smem_word_at(sb, i + k) & ((1u << (8 * (len - k))) - 1u));
  return hs.finish();
}

// The <= 8 key bytes [q, q + len) little-endian (bytes beyond len unspecified).
__device__ __forceinline__ uint64_t bytes8_at(const Params& P, const TileView& tv, long long q, uint32_t len) {
  if (q + 8 <= tv.stg_hi && q - tv.sbase + 8 + 12 <= kStageBytes) {
    const uint32_t i = static_cast<uint32_t>(q - tv.sbase);
    return static_cast<uint64_t>(smem_word_at(tv.sb, i)) | (static_cast<uint64_t>(smem_word_at(tv.sb, i + 4)) << 32);
  }
  uint64_t b = 0;
  for (uint32_t k = 0; k < len; ++k) b |= static_cast<uint64_t>(P.rec[q + k]) << (8 * k);
  return b;
}

// Sort key of the key bytes [q, q + len): inline when short, else the hash (common.cuh).
__device__ __forceinline__ uint64_t key_at(const Params& P, const TileView& tv, long long q, uint32_t len) {
  const bool in_stage = (q + static_cast<long long>(len) <= tv.stg_hi) && (q - tv.sbase + len + 12 <= kStageBytes);
  if (len <= inline_max(P.key_bits)) {
    uint64_t b = 0;
    if (in_stage) {
      const uint32_t i = static_cast<uint32_t>(q - tv.sbase);
      b = static_cast<uint64_t>(smem_word_at(tv.sb, i)) | (static_cast<uint64_t>(smem_word_at(tv.sb, i + 4)) << 32);
    } else {
      for (uint32_t k = 0; k < len; ++k) b |= static_cast<uint64_t>(P.rec[q + k]) << (8 * k);
    }
    return inline_key(b, len, P.key_bits);
  }
  const uint64_t h = in_stage ? hash_smem(tv.sb, static_cast<uint32_t>(q - tv.sbase), len, P.hash_seed)
                              : hash_bytes(P.rec + q, len, P.hash_seed);
  return hashed_key(h, (P.flags & 8u) != 0, P.key_bits);
}

// ---------------------------------------------------------------- emit allocator
// Flush bases are kept multiples of 4 pairs so that every SoA run of a flushed half is 16-byte
// aligned in global memory and leaves SMEM as one TMA bulk store (cp.async.bulk global<-shared);
// the <= 3 filler entries carry the workload's sentinel key, which sorts after every real key
// and is excluded from the groups (DevState::pads).  StringMatch (Map-only, sparse) flushes with
// plain stores and needs no filler.
// Shared cursor: 32-bit [generation:6 | cb:12 | ca:14].  ca counts entries (WC: exact-key
// entries), cb the WC hashed entries; one atomicAdd reserves both.  Field bounds: a buffer holds
// <= 2558 units and at most kNMap reservations of <= kMaxReserve overshoot it before the seal.
struct Slot { uint32_t half, base; };   // base: packed (cb << 14 | ca) at the reservation
constexpr uint32_t kGenShift = 26, kCbShift = 14;
constexpr uint32_t kCaMask = (1u << kCbShift) - 1u, kCbMask = (1u << (kGenShift - kCbShift)) - 1u;
constexpr uint32_t kCntBits = (1u << kGenShift) - 1u;
__device__ __forceinline__ uint32_t cur_gen(uint32_t c) { return c >> kGenShift; }
__device__ __forceinline__ uint32_t cur_ca(uint32_t c) { return c & kCaMask; }
__device__ __forceinline__ uint32_t cur_cb(uint32_t c) { return (c >> kCbShift) & kCbMask; }
template <int W>
__device__ __forceinline__ uint32_t units(uint32_t c) {   // buffer space of packed counts
  if constexpr (W == kWC) return cur_ca(c) + 4u * cur_cb(c);
  else return cur_ca(c);
}
// WC: a reservation carries <= kWin / 2 + 1 exact entries (ca) and <= kHashQ queued ones (cb)
static_assert(PairFmt<kWC>::kCap + nmap<kWC>() * (kWin / 2 + 1) <= kCaMask, "ca field overflow");
static_assert(PairFmt<kWC>::kCap / 4 + nmap<kWC>() * Cfg<kWC>::kHashQ <= kCbMask, "cb field overflow");
static_assert(PairFmt<kSM>::kCap + kNMapText * PairFmt<kSM>::kMaxReserve <= kCaMask, "ca field overflow");
static_assert(PairFmt<kII>::kCap + kNMapText * PairFmt<kII>::kMaxReserve <= kCaMask, "ca field overflow");

template <int W>
__device__ __forceinline__ uint64_t sentinel_key(const Params& P) {
  if constexpr (W == kKM) return P.k <= 255 ? 255ULL : 65535ULL;
  return sentinel_of(P.key_bits);
}

// Seal buffer h of the current generation: switch every warp to the next buffer at once (the
// in-flight writers of h finish on their own), then hand h to the flush warp.  Only when all
// kNOut buffers are busy does the sealing warp wait (for the oldest flush).
template <int W>
__device__ void seal(const Params& P, OutCtl* oc, uint32_t gen8, uint32_t h, uint32_t cnt, bool last) {
  const uint32_t full_gen = oc->nsealed;                       // full generation number
  if (!last) {
    if (full_gen + 1 >= kNOut) {                               // next buffer last used by gen q
      const uint32_t q = full_gen + 1 - kNOut;
      if (!mbar_try_wait(&oc->done[q % kNOut], (q / kNOut) & 1u)) {   // every buffer still flushing
        atomicAdd(&P.st->seal_waits, 1ULL);
        st_release_cta_shared_u32(&oc->congested, 1u);         // overflowing warps spill meanwhile
        mbar_wait(&oc->done[q % kNOut], (q / kNOut) & 1u);
        st_release_cta_shared_u32(&oc->congested, 0u);
      }
    }
    oc->committed[(h + 1) % kNOut] = 0;
    oc->nsealed = full_gen + 1;
    __threadfence_block();
    atomicExch(&oc->cur, ((gen8 + 1) & 0x3Fu) << kGenShift);   // other warps continue in the next buffer
  } else {
    oc->final_seq = full_gen;
    oc->is_final = 1;
  }
  oc->fcount[h] = cnt;
  __threadfence_block();
  mbar_arrive(&oc->req[h]);
}
// cnt: packed counts (cb << 14 | ca); cap: buffer capacity in units.  spill_ok: the caller can
// write its result straight to HBM (§8(a) a5 overflow spill): an overflowing warp that is not the
// sealer then returns kSpill instead of waiting while the ring is congested (the sealer waits for
// a flushing buffer).
constexpr uint32_t kSpill = 0xFFFFFFFFu;
template <int W>
__device__ __forceinline__ Slot reserve(const Params& P, OutCtl* oc, uint8_t* outh, uint32_t cnt, uint32_t cap,
                                        bool spill_ok = false) {
  const uint32_t lane = threadIdx.x & 31;
  for (;;) {
    uint32_t old = 0;
    if (lane == 0) old = atomicAdd(&oc->cur, cnt);
    old = __shfl_sync(kFull, old, 0);
    const uint32_t gen = cur_gen(old), base = old & kCntBits;
    const uint32_t h = gen % kNOut;
    const uint32_t u0 = units<W>(base);
    if (u0 + units<W>(cnt) <= cap) return {h, base};
    uint32_t spill = 0;
    const bool force = spill_ok && (P.flags & 0x800u);   // MR_FLAG_FORCE_SPILL (tests)
    if (lane == 0) {
      if (u0 <= cap) {
        // This warp crossed the capacity first (units grow monotonically within a generation):
        // it seals half h (L113 "overflow handling").
        seal<W>(P, oc, gen, h, base, false);
        if (force) {
          spill = 1;
          atomicAdd(&P.st->spills, 1ULL);
        }
      } else {
        while (cur_gen(ld_acquire_cta_shared_u32(&oc->cur)) == gen) {
          if (spill_ok && (force || ld_acquire_cta_shared_u32(&oc->congested))) {
            spill = 1;
            atomicAdd(&P.st->spills, 1ULL);
            break;
          }
          __nanosleep(128);
        }
      }
    }
    if (__shfl_sync(kFull, spill, 0)) return {kSpill, 0};
    __syncwarp();
  }
}
__device__ __forceinline__ void commit(OutCtl* oc, Slot s, uint32_t cnt) {
  fence_proxy_async_shared();   // generic SMEM writes -> visible to the TMA store of the flush
  __syncwarp();
  if ((threadIdx.x & 31) == 0) {
    __threadfence_block();
    atomicAdd(&oc->committed[s.half], cnt);
  }
}

// ---------------------------------------------------------------- flush warp
__device__ __forceinline__ void tma_store_1d(void* gdst, const void* ssrc, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gdst), "r"(smem_u32(ssrc)),
               "r"(bytes)
               : "memory");
}

// Flush warps (A4, L113): flush warp fw of nflush<W>() takes the sealed generations
// f == fw (mod nflush).  Per buffer: wait for its committed writers (acquire), pad the exact run
// to 16 B, count the queued WC entries per stream (SMEM only), then ONE round of global atomics
// (one lane per stream: all three reservations in flight together), the TMA bulk store of the
// buffer's SoA runs, the routed stores of the queued entries while the TMA reads SMEM, and only
// then the wait for the TMA's reads before the buffer is handed back.
template <int W>
__device__ void flush_loop(const Params& P, uint8_t* smem, OutCtl* oc, uint32_t fw) {
  using F = PairFmt<W>;
  constexpr uint32_t NF = nflush<W>();
  const uint32_t lane = threadIdx.x & 31;
  unsigned long long nflushes = 0, npads = 0;
  for (uint32_t f = fw;; f += NF) {
    const uint32_t h = f % kNOut;
    // wait for generation f to be sealed; with several flush warps the one waiting past the
    // final generation sees the final flag instead (no arrival ever comes for it)
    bool past = false;
    // (suspended try_wait: a polling flush warp would take issue slots from the map warps; an idle
    // flush warp's sleep-polls measured no cheaper, C5 round 2)
    while (!mbar_try_wait_hint(&oc->req[h], (f / kNOut) & 1u, 2000)) {
      if (NF > 1 && ld_acquire_cta_shared_u32(&oc->is_final) && ld_acquire_cta_shared_u32(&oc->final_seq) < f) {
        past = true;
        break;
      }
    }
    if (past) break;
    // (the sealing warp wrote these before its release-arrive on req[h]; the wait above acquires)
    const bool fin = ld_acquire_cta_shared_u32(&oc->is_final) && ld_acquire_cta_shared_u32(&oc->final_seq) == f;
    const uint32_t cnt0 = ld_acquire_cta_shared_u32(&oc->fcount[h]);
    uint8_t* half = smem + Layout<W>::out + h * Cfg<W>::kOutHalf;
    // the sealed buffer's writers finish on their own: wait until all cnt0 entries are committed
    if (lane == 0) {
      while (ld_acquire_cta_shared_u32(&oc->committed[h]) != cnt0) __nanosleep(32);
    }
    __syncwarp();
    const uint32_t ca0 = cur_ca(cnt0);
    const uint32_t cb = (W == kWC) ? cur_cb(cnt0) : 0u;
    uint32_t cnt = ca0;
    if constexpr (W == kWC) {
      cnt = (ca0 + 3u) & ~3u;                                   // 16-B aligned exact run (TMA store)
      if (lane < cnt - ca0) reinterpret_cast<uint32_t*>(half)[ca0 + lane] = 0xFFFFFFFFu;   // filler: sorts last
    } else if constexpr (W != kSM) {
      cnt = (ca0 + 3u) & ~3u;                                   // 4-pair aligned flush (TMA store)
      if (lane < cnt - ca0) {                                   // sentinel filler entries
        reinterpret_cast<uint64_t*>(half)[ca0 + lane] = sentinel_key<W>(P);
        if constexpr (F::kKref) reinterpret_cast<uint64_t*>(half)[F::kCap + ca0 + lane] = 0;
      }
    }
    // WC queued entries (key, kref) at the top of the buffer: kref 0 -> mid stream (key only),
    // else hashed stream (key + kref)
    const ulonglong2* top = reinterpret_cast<const ulonglong2*>(half + Cfg<W>::kOutHalf);
    uint32_t nc = 0;
    if constexpr (W == kWC) {
      for (uint32_t i0 = 0; i0 < cb; i0 += 32) {
        const bool v = i0 + lane < cb && top[-1 - static_cast<int>(i0 + lane)].y == 0;
        nc += __popc(__ballot_sync(kFull, v));
      }
    }
    // one global atomic per stream run (L113), issued by lanes 0 / 1 / 2 together
    unsigned long long g = 0;
    {
      unsigned long long* cur = lane == 0 ? &P.st->pair_cursor : lane == 1 ? &P.st->pair_cursor_b : &P.st->pair_cursor_c;
      const uint32_t want = lane == 0 ? cnt : lane == 1 ? cb - nc : nc;
      if (lane < 3 && want) g = atomicAdd(cur, static_cast<unsigned long long>(want));
    }
    const unsigned long long gb = __shfl_sync(kFull, g, 0);
    nflushes += (cnt || cb) ? 1 : 0;
    npads += cnt - ca0;
    bool tma = false;
    if (cnt && gb + cnt <= P.cap_pairs) {
      const uint64_t* sh = reinterpret_cast<const uint64_t*>(half);
      const uint8_t* sv = half + F::kCap * (F::kKref ? 16 : 8);
      if constexpr (W == kSM) {
        for (uint32_t i = lane; i < cnt; i += 32) P.oh[gb + i] = sh[i];
      } else {
        tma = true;
        fence_proxy_async_shared();   // every lane's filler writes -> visible to the TMA store
        __syncwarp();
        if (lane == 0) {
          // A4 staging-out as TMA bulk stores (16-B aligned: gb and cnt even / multiples of 4)
          if constexpr (W == kWC) tma_store_1d(P.ohx + gb, sh, cnt * 4);
          else tma_store_1d(P.oh + gb, sh, cnt * 8);
          if constexpr (F::kKref) tma_store_1d(P.okref + gb, sh + F::kCap, cnt * 8);
          if constexpr (F::kV > 0) tma_store_1d(P.ov + gb * F::kV, sv, cnt * F::kV);
          asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        }
      }
    }
    if constexpr (W == kWC) {
      // routed plain stores (coalesced per 32 entries), overlapping the TMA store's SMEM reads
      const unsigned long long gbb = __shfl_sync(kFull, g, 1), gc = __shfl_sync(kFull, g, 2);
      const bool okb = gbb + (cb - nc) <= P.cap_b, okc = gc + nc <= P.cap_c;
      uint32_t rb = 0, rc = 0;
      for (uint32_t i0 = 0; i0 < cb; i0 += 32) {
        const bool in = i0 + lane < cb;
        ulonglong2 e = make_ulonglong2(0ULL, 0ULL);
        if (in) e = top[-1 - static_cast<int>(i0 + lane)];
        const uint32_t mc = __ballot_sync(kFull, in && e.y == 0), mb = __ballot_sync(kFull, in && e.y != 0);
        if (in && e.y == 0 && okc) P.ohc[gc + rc + __popc(mc & lanemask_lt())] = e.x;
        if (in && e.y != 0 && okb) {
          const uint64_t o = gbb + rb + __popc(mb & lanemask_lt());
          P.ohb[o] = e.x;
          P.okrefb[o] = e.y;
        }
        rc += __popc(mc);
        rb += __popc(mb);
      }
    }
    if (tma && lane == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");   // SMEM reusable
    __syncwarp();
    if (lane == 0) mbar_arrive(&oc->done[h]);
    if (fin) break;
  }
  if (lane == 0) {
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");   // global writes complete
    atomicAdd(&P.st->flushes, nflushes);
    if (npads) atomicAdd(&P.st->pads, npads);
  }
}

// ---------------------------------------------------------------- producer warp
// cp.async.bulk.prefetch.L2 of the 16-B aligned interior of [lo, hi) (never touches bytes outside)
__device__ __forceinline__ void l2_prefetch_range(const uint8_t* lo, const uint8_t* hi) {
  const uintptr_t a = (reinterpret_cast<uintptr_t>(lo) + 15u) & ~static_cast<uintptr_t>(15u);
  const uintptr_t b = reinterpret_cast<uintptr_t>(hi) & ~static_cast<uintptr_t>(15u);
  if (b > a)
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a), "r"(static_cast<uint32_t>(b - a)) : "memory");
}
__device__ void stage_copy_edges(uint8_t* d, const uint8_t* g, uint64_t len, uint32_t lane, uint32_t& body_off,
                                 uint32_t& body_len) {
  const uint32_t head = static_cast<uint32_t>(
      min(static_cast<uint64_t>((16u - (reinterpret_cast<uintptr_t>(g) & 15u)) & 15u), len));
  const uint32_t body = static_cast<uint32_t>((len - head) & ~15ULL);
  const uint32_t tail = static_cast<uint32_t>(len - head - body);
  for (uint32_t i = lane; i < head; i += 32) d[i] = g[i];
  for (uint32_t i = lane; i < tail; i += 32) d[head + body + i] = g[head + body + i];
  body_off = head;
  body_len = body;
}

// Text tiles: once the TMA of stage s has landed, the producer warp turns the staged offsets
// slice into the record-start bitmap and releases the stage to the map warps (ready[s]).
// Done one tile behind the TMA issue, so the copy latency is hidden.
template <int W>
__device__ void finish_stage(const Params& P, uint8_t* smem, uint32_t it) {
  constexpr int kStages = Cfg<W>::kStages;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t s = it % kStages, ph = (it / kStages) & 1u;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + Layout<W>::full);
  uint64_t* ready = reinterpret_cast<uint64_t*>(smem + Layout<W>::ready);
  const StageHdr* hd = reinterpret_cast<const StageHdr*>(smem + Layout<W>::hdr + s * 128);
  if (hd->t < 0) return;   // a skip stage (dynamic tiles): released when it was posted
  mbar_wait(&full[s], ph);
  uint32_t* bm = reinterpret_cast<uint32_t*>(smem + Layout<W>::bits + s * Cfg<W>::kBits);
  const uint64_t* soff =
      reinterpret_cast<const uint64_t*>(smem + Layout<W>::offs + s * Cfg<W>::kOffBytes + hd->off_shift);
  const uint64_t ra = hd->ra, cnt = hd->rb - hd->ra;
  const long long sbase = hd->sbase;
  const bool staged = hd->off_staged != 0;
  for (uint64_t r = lane; r < cnt; r += 32) {
    const uint64_t pos = staged ? soff[r] : P.off[ra + r];
    const long long i = static_cast<long long>(pos) - sbase;
    atomicOr(&bm[i >> 5], 1u << (i & 31));
  }
  __syncwarp();
  if (lane == 0) mbar_arrive(&ready[s]);
}

// Text tile t into stage s: bytes (+ lead / halo) and the offsets slice offsets[ra..rb) by TMA,
// the stage header, the bitmap cleared (built by finish_stage once the bytes have landed).
template <int W>
__device__ __forceinline__ void issue_text_stage(const Params& P, uint8_t* smem, uint32_t s, uint64_t t, uint64_t ra,
                                                 uint64_t rb) {
  const uint32_t lane = threadIdx.x & 31;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + Layout<W>::full);
  const long long N = bd_nbytes();
  StageHdr* hd = reinterpret_cast<StageHdr*>(smem + Layout<W>::hdr + s * 128);
  uint8_t* sb = smem + Layout<W>::bytes + s * kStageBytes;
  uint32_t b_off = 0, b_len = 0, o_off = 0, o_len = 0;
  uint8_t* so = smem + Layout<W>::offs + s * Cfg<W>::kOffBytes;
  const long long chunk0 = static_cast<long long>(t) * kT - P.a0;
  const long long sbase = chunk0 - kLead;
  const long long w_lo = max(0LL, sbase);
  const long long w_hi = chunk0 + kT + kHalo;
  const long long stg_hi = min(w_hi, N);
  // stage bytes [w_lo, stg_hi) at sb + (w_lo - sbase); (rec + sbase) is 16-B aligned
  uint8_t* d = sb + (w_lo - sbase);
  const uint8_t* g = P.rec + w_lo;
  if (!P.so) stage_copy_edges(d, g, static_cast<uint64_t>(max(0LL, stg_hi - w_lo)), lane, b_off, b_len);
  // clear the record-start bitmap (map warps set bits after the full barrier)
  if constexpr (!Cfg<W>::kLazyDir) {
    uint32_t* bm = reinterpret_cast<uint32_t*>(smem + Layout<W>::bits + s * Cfg<W>::kBits);
    for (uint32_t i = lane; i < Cfg<W>::kBits / 16; i += 32) reinterpret_cast<uint4*>(bm)[i] = make_uint4(0, 0, 0, 0);
  }
  // offsets slice offsets[ra..rb) (record starts in the staged window)
  const uint64_t cnt = rb - ra;
  const bool staged = !Cfg<W>::kLazyDir && cnt <= static_cast<uint64_t>(Cfg<W>::kOffCap);
  uint32_t shift = 0;
  const uint8_t* og = reinterpret_cast<const uint8_t*>(P.off + ra);
  if (staged && cnt) {
    shift = static_cast<uint32_t>(reinterpret_cast<uintptr_t>(og) & 15u);
    // Copy the 16-B aligned superset of the slice with TMA alone (no synchronous edge
    // loads on the producer's critical path) whenever it stays inside offsets[0..n].
    const uint8_t* a_lo = og - shift;
    const uint8_t* a_hi = reinterpret_cast<const uint8_t*>(
        (reinterpret_cast<uintptr_t>(og + cnt * 8) + 15u) & ~static_cast<uintptr_t>(15u));
    if (a_lo >= reinterpret_cast<const uint8_t*>(P.off) && a_hi <= P.off_end) {
      o_off = 0;
      o_len = static_cast<uint32_t>(a_hi - a_lo);
      og = a_lo;
      // so + shift still addresses offsets[ra]; the TMA below starts at so (= a_lo)
    } else {
      stage_copy_edges(so + shift, og, cnt * 8, lane, o_off, o_len);
      og = og - shift;
      o_off += shift;
    }
  }
  if (lane == 0) {
    hd->t = static_cast<long long>(t);
    hd->sbase = sbase;
    hd->chunk0 = chunk0;
    hd->lo = max(0LL, chunk0);
    hd->hi = min(N, chunk0 + kT);
    hd->stg_hi = stg_hi;
    hd->ra = ra;
    hd->rb = rb;
    hd->off_shift = shift;
    hd->off_staged = staged ? 1u : 0u;
  }
  __syncwarp();
  if (lane == 0) {
    mbar_arrive_expect_tx(&full[s], b_len + o_len);
    if (BMR_STREAM_HINT && P.xtab) {   // WC with the L2 count table: the input streams past it
      const uint64_t pol = l2_policy_evict_first();
      if (b_len) tma_load_1d_stream(d + b_off, g + b_off, b_len, &full[s], pol);
      if (o_len) tma_load_1d_stream(so + o_off, og + o_off, o_len, &full[s], pol);
    } else {
      if (b_len) tma_load_1d(d + b_off, g + b_off, b_len, &full[s]);
      if (o_len) tma_load_1d(so + o_off, og + o_off, o_len, &full[s]);
    }
  }
}

// Dynamic tile scheduling (WordCount / InvertedIndex): the producers take tiles from the batch's
// global counter, kTileChunk at a time, instead of the static blockIdx.x + it * G order — the
// per-SM time of the text Maps varies by a quarter (ncu C5: sm__cycles_active min 30.4 M / max
// 41.4 M cycles of 40.9 M), so static shares leave the fast SMs idle for the last sixth.
// Producer p still owns the CTA iterations it == p (mod 2).  A producer whose fetch finds no tile
// publishes that first empty iteration x0 (pout[p]); the batch ends at E = max(x0_0, x0_1) (every
// tile lies at an earlier iteration): the owner of E posts the end marker there, and each of the
// producer's empty iterations below E is posted as a skip stage (no bytes; hi = LLONG_MIN, so its
// windows are empty).  An empty iteration x below the other producer's x0 is only known to be a
// skip once the other has filled an iteration > x (plast) or run out itself; it can always get
// there (its next iteration needs x - 1 consumed at most), so the wait never deadlocks.
#ifndef BMR_TILE_CHUNK
#define BMR_TILE_CHUNK 4
#endif
template <int W>
__device__ void producer_loop_dyn(const Params& P, uint8_t* smem, uint32_t pw) {
  constexpr int kStages = Cfg<W>::kStages;
  constexpr uint32_t kNP = nprod<W>(), kLag = Cfg<W>::kLag, kChunk = BMR_TILE_CHUNK;
  static_assert(kNP == 2 && kChunk <= 32, "dynamic tiles: two producers");
  const uint32_t lane = threadIdx.x & 31;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + Layout<W>::full);
  uint64_t* empty = reinterpret_cast<uint64_t*>(smem + Layout<W>::empty);
  uint64_t* ready = reinterpret_cast<uint64_t*>(smem + Layout<W>::ready);
  OutCtl* oc = reinterpret_cast<OutCtl*>(smem + Layout<W>::ctl);
  const uint64_t ntiles = bd_ntiles();
  // small batches take single tiles (chunks would leave most SMs without a tile: C1, 64 tiles)
  const uint32_t chunk = ntiles >= 16ULL * kChunk * gridDim.x ? kChunk : 1u;
  uint32_t it = pw;
  for (;;) {   // chunks of tiles
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(P.tile_next, static_cast<unsigned long long>(chunk));
    base = __shfl_sync(kFull, base, 0);
    if (base >= ntiles) break;
    const uint32_t cnt = static_cast<uint32_t>(min(static_cast<unsigned long long>(chunk), ntiles - base));
    uint64_t my_ra = 0, my_rb = 0;
    if (lane < cnt) {
      my_ra = P.tb[2 * (base + lane)];
      my_rb = P.tb[2 * (base + lane) + 1];
    }
    for (uint32_t j = 0; j < cnt; ++j, it += kNP) {
      const uint64_t ra = __shfl_sync(kFull, my_ra, j), rb = __shfl_sync(kFull, my_rb, j);
      const uint32_t s = it % kStages, ph = (it / kStages) & 1u;
      if (it >= kLag) finish_stage<W>(P, smem, it - kLag);
      helper_wait(P, &empty[s], ph ^ 1u, 128);
      if (lane == 0) *reinterpret_cast<volatile unsigned int*>(&oc->plast[pw]) = it + 1u;
      issue_text_stage<W>(P, smem, s, base + j, ra, rb);
    }
  }
  const uint32_t x0 = it;   // this producer's first empty iteration
  if (lane == 0) {
    *reinterpret_cast<volatile unsigned int*>(&oc->pout[pw]) = x0;
    __threadfence_block();
  }
  __syncwarp();
  const uint32_t other = pw ^ 1u;
  for (;; it += kNP) {
    // E = max(x0, x0_other) once the other has run out; below it, iterations past the other's
    // filled ones are skips
    bool post_end = false, post_skip = false;
    for (uint32_t spin = 0;; ++spin) {
      const uint32_t xo = *reinterpret_cast<volatile unsigned int*>(&oc->pout[other]);
      if (xo != ~0u) {
        const uint32_t E = max(x0, xo);
        post_end = it == E || it == E + 1u;   // (two end iterations: window-pair fetches, wc_map_loop)
        post_skip = it < E;
        break;
      }
      if (*reinterpret_cast<volatile unsigned int*>(&oc->plast[other]) > it + 1u) { post_skip = true; break; }
      __nanosleep(spin < 4 ? 32 : 256);
    }
    if (!post_end && !post_skip) break;   // E is the other producer's iteration
    const uint32_t s = it % kStages, ph = (it / kStages) & 1u;
    if (it >= kLag) finish_stage<W>(P, smem, it - kLag);
    helper_wait(P, &empty[s], ph ^ 1u, 128);
    if (lane == 0) {
      StageHdr* hd = reinterpret_cast<StageHdr*>(smem + Layout<W>::hdr + s * 128);
      hd->t = post_end ? -1 : -2;
      hd->sbase = 0;
      hd->chunk0 = 0;
      hd->lo = 0;
      hd->hi = LLONG_MIN;
      hd->stg_hi = 0;
      hd->ra = hd->rb = 0;
      hd->off_shift = 0;
      hd->off_staged = 0;
      mbar_arrive(&full[s]);    // keeps the stage's full phase in step (no bytes)
      mbar_arrive(&ready[s]);
    }
    __syncwarp();
    if (post_end && it + kNP > max(x0, *reinterpret_cast<volatile unsigned int*>(&oc->pout[other])) + 1u) {
      it += kNP;
      break;
    }
  }
  // this producer's tiles whose bitmap is still pending (skip stages return at once)
  for (uint32_t j = it >= kLag + kNP ? it - kLag : pw; j < it; j += kNP)
    if (j + kLag >= it) finish_stage<W>(P, smem, j);
}

template <int W>
__device__ void producer_loop(const Params& P, uint8_t* smem, uint32_t pw) {
  if constexpr (W == kWC || W == kII) {
    if (P.tile_next) {
      producer_loop_dyn<W>(P, smem, pw);
      return;
    }
  }
  constexpr int kStages = Cfg<W>::kStages;
  const uint32_t lane = threadIdx.x & 31;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + Layout<W>::full);
  uint64_t* empty = reinterpret_cast<uint64_t*>(smem + Layout<W>::empty);
  const long long N = bd_nbytes();
  const uint64_t G = gridDim.x;
  // iterations of this CTA: tiles blockIdx.x + it * G; this producer takes it == pw (mod nprod<W>())
  const uint32_t T = blockIdx.x < bd_ntiles() ? static_cast<uint32_t>((bd_ntiles() - blockIdx.x + G - 1) / G) : 0u;
  for (uint32_t i0 = pw; i0 < T; i0 += 32u * nprod<W>()) {
    // lanes prefetch the bounds of this producer's next 32 tiles (one latency per 32 tiles)
    const uint32_t my_it = i0 + lane * nprod<W>();
    uint64_t my_ra = 0, my_rb = 0;
    if constexpr (W != kKM) {
      if (my_it < T) {
        const uint64_t my_t = blockIdx.x + static_cast<uint64_t>(my_it) * G;
        my_ra = P.tb[2 * my_t];
        my_rb = P.tb[2 * my_t + 1];
      }
    }
    for (uint32_t j = 0; j < 32; ++j) {
      const uint32_t it = i0 + j * nprod<W>();
      if (it >= T) break;
      const uint64_t t = blockIdx.x + static_cast<uint64_t>(it) * G;
      const uint64_t ra = __shfl_sync(kFull, my_ra, j), rb = __shfl_sync(kFull, my_rb, j);
      const uint32_t s = it % kStages, ph = (it / kStages) & 1u;
      // release the bitmap of tile it - kLag (its bytes have landed) BEFORE blocking on a free
      // stage: that wait lasts until the oldest tile's last window is done, and the map warps
      // need the next tile meanwhile
      if constexpr (W != kKM && !Cfg<W>::kLazyDir) {
        if (it >= static_cast<uint32_t>(Cfg<W>::kLag)) finish_stage<W>(P, smem, it - Cfg<W>::kLag);   // same owner
      }
      helper_wait(P, &empty[s], ph ^ 1u, 128);
      StageHdr* hd = reinterpret_cast<StageHdr*>(smem + Layout<W>::hdr + s * 128);
      uint8_t* sb = smem + Layout<W>::bytes + s * kStageBytes;
      uint32_t b_off = 0, b_len = 0, o_off = 0, o_len = 0;
      uint8_t* so = smem + Layout<W>::offs + s * Cfg<W>::kOffBytes;
      if constexpr (W == kKM) {
        const uint64_t p_lo = t * kKmPts, p_hi = min(P.n, p_lo + kKmPts);
        const uint8_t* g = P.rec + p_lo * 32;
        uint8_t* d = sb + (reinterpret_cast<uintptr_t>(g) & 15u);   // same 16-B phase as the source
        if (!P.so) stage_copy_edges(d, g, (p_hi - p_lo) * 32, lane, b_off, b_len);
        if (lane == 0) {
          hd->t = static_cast<long long>(t);
          hd->lo = static_cast<long long>(p_lo);
          hd->hi = static_cast<long long>(p_hi);
        }
        __syncwarp();
        if (lane == 0) {
          mbar_arrive_expect_tx(&full[s], b_len);
          if (b_len) tma_load_1d(d + b_off, g + b_off, b_len, &full[s]);
        }
      } else {
        issue_text_stage<W>(P, smem, s, t, ra, rb);
        // L2 prefetch of this producer's tile P.pf tiles ahead (bytes + offsets slice): the TMA of
        // that tile then hits L2, so the kLag stages in flight cover L2 latency, not HBM latency
        if (P.pf) {
          const uint32_t jf = j + P.pf;
          const uint64_t raf = __shfl_sync(kFull, my_ra, jf & 31), rbf = __shfl_sync(kFull, my_rb, jf & 31);
          const uint32_t itf = i0 + jf * nprod<W>();
          if (lane == 0 && itf < T) {
            const long long c0 = static_cast<long long>(blockIdx.x + static_cast<uint64_t>(itf) * G) * kT - P.a0;
            l2_prefetch_range(P.rec + max(0LL, c0 - kLead), P.rec + min(c0 + kT + kHalo, N));
            if (!Cfg<W>::kLazyDir && jf < 32 && rbf > raf)   // (SM stages no offsets)
              l2_prefetch_range(reinterpret_cast<const uint8_t*>(P.off + raf), reinterpret_cast<const uint8_t*>(P.off + rbf));
          }
        }

      }
    }
  }
  if constexpr (W != kKM && !Cfg<W>::kLazyDir) {   // this producer's tiles whose bitmap is still pending
    const uint32_t j0 = T > static_cast<uint32_t>(Cfg<W>::kLag) ? T - Cfg<W>::kLag : 0u;
    for (uint32_t j = j0; j < T; ++j)
      if (j % nprod<W>() == pw) finish_stage<W>(P, smem, j);
  }
  // end-of-work marker at iteration T, written by its owner
  if (T % nprod<W>() != pw) return;
  const uint32_t s = T % kStages, ph = (T / kStages) & 1u;
  mbar_wait(&empty[s], ph ^ 1u);
  if (lane == 0) {
    reinterpret_cast<StageHdr*>(smem + Layout<W>::hdr + s * 128)->t = -1;
    if constexpr (W == kKM || Cfg<W>::kLazyDir) mbar_arrive(&full[s]);
    else mbar_arrive(reinterpret_cast<uint64_t*>(smem + Layout<W>::ready) + s);
  }
}

// ---------------------------------------------------------------- map warps
// Combiner probe (f-1): adds one occurrence of exact key `key` to its slot if the slot holds the
// key or is free (claimed by a 32-bit CAS); false = the slot belongs to another key (emit
// normally).  Keys and counts are separate u32 arrays: 32-bit shared atomics are native (a
// 64-bit shared atomicAdd is a CAS spin loop, which serialises on the Zipf head's slots).
// BMR_WC_COMB_PROBES probes (home slot, home ^ 1, ...): with 2, a key whose home slot belongs to
// another key gets a second chance (measured on C5, round 1: not worth its Map instructions).  Slots are never freed within a batch,
// so a key lives in at most one of its two slots; partials are summed per key anyway.
__device__ __forceinline__ bool comb_add(uint32_t* ckey, uint32_t key) {
  const uint32_t home = (key * 0x9E3779B1u) >> (32 - kCombBits);
#pragma unroll
  for (uint32_t probe = 0; probe < BMR_WC_COMB_PROBES; ++probe) {
    const uint32_t slot = home ^ probe;
    uint32_t v = *reinterpret_cast<volatile uint32_t*>(ckey + slot);
    if (v == kCombEmpty32) v = atomicCAS(ckey + slot, kCombEmpty32, key);
    if (v == key || v == kCombEmpty32) {
      atomicAdd(ckey + Cfg<kWC>::kCombSlots + slot, 1u);   // count array follows the key array
      return true;
    }
  }
  return false;
}
// WordCount emission of one warp window.  Each start is classified BEFORE the reservation: a
// word is exact iff it ends within kWcExact bytes (nb bit q: a word cannot continue at q, so the
// word at j ends at the first nb bit above j).  Only a lane's highest start can lack a visible
// end; it is measured by the slow path up front.  One shared atomic reserves ta exact entries
// and tb hashed entries; the rounds write exact keys directly and queue the hashed words, which
// all 32 lanes then hash together.
__device__ __forceinline__ void emit_wc(const Params& P, OutCtl* oc, uint8_t* outh, const TileView& tv,
                                        const uint32_t (&x)[8], long long p0, uint32_t emit_mask, uint32_t nb) {
  const uint32_t lane = threadIdx.x & 31;
  uint32_t len_slow = 0, slow_bit = 0;
  if (emit_mask) {
    const uint32_t jh = 31 - __clz(emit_mask);
    if ((nb >> (jh + 1)) == 0) {
      slow_bit = 1u << jh;
      len_slow = slow_word_len(P, tv, p0 + jh, p0 + 32);
    }
  }
  uint32_t near = 0;                                   // bit j: an nb bit in (j, j + kWcExact]
#pragma unroll
  for (uint32_t d = 1; d <= kWcExact; ++d) near |= nb >> d;
  uint32_t longm = emit_mask & ~near & ~slow_bit;
  if (slow_bit && len_slow > kWcExact) longm |= slow_bit;
  (void)longm;
  if (__all_sync(kFull, emit_mask == 0)) return;
  uint32_t* hq = reinterpret_cast<uint32_t*>(outh + (Layout<kWC>::hq - Layout<kWC>::out)) +
                 (threadIdx.x >> 5) * Cfg<kWC>::kHashQ;
  uint32_t* xq = reinterpret_cast<uint32_t*>(outh + (Layout<kWC>::xq - Layout<kWC>::out)) +
                 (threadIdx.x >> 5) * Cfg<kWC>::kXQ;
  uint32_t* ctab = reinterpret_cast<uint32_t*>(outh + (Layout<kWC>::comb - Layout<kWC>::out));
  uint32_t nx = 0, nq = 0;
  if (P.wc_bal && !P.so) {
    // Balanced emission.  Phase 1: each lane writes a descriptor (stage offset | length << 15)
    // of every word it starts at the word's warp rank (cheap divergent loop); phase 2: the warp
    // processes the descriptors 32 at a time (rounds = words / 32 instead of the busiest lane's
    // word count), reading the word bytes from the stage.  Phase 2 compacts the exact keys that
    // miss the combiner into the same queue (its writes stay below the round being read).
    const uint32_t cnt = __popc(emit_mask);
    const uint32_t incl = warp_inclusive_add(cnt);
    const uint32_t W = __shfl_sync(kFull, incl, 31);
    if (W == 0) return;
    uint32_t k = incl - cnt;
    const uint32_t i0 = static_cast<uint32_t>(p0 - tv.sbase);
    for (uint32_t m = emit_mask; m; m &= m - 1) {
      const uint32_t j = __ffs(m) - 1;
      const uint32_t rest = nb >> (j + 1);
      uint32_t len = rest ? static_cast<uint32_t>(__ffs(rest)) : len_slow;
      if (len > 0xFFFFu) { atomicOr(&P.st->err, kErrKeyTooLong); len = 0xFFFFu; }
      xq[k++] = (i0 + j) | (len << 15);
    }
    __syncwarp();
    for (uint32_t b = 0; b < W; b += 32) {
      const bool act = b + lane < W;
      const uint32_t d = act ? xq[b + lane] : 0u;
      __syncwarp();                            // this round's reads before the compacting writes
      const uint32_t len = d >> 15, pos = d & 0x7FFFu;
      bool ex = act && len <= kWcExact;
      uint32_t key = 0;
      if (ex) {   // the <= 5 word bytes from the stage: two aligned words cover [pos, pos + 5)
        const uint32_t a = pos & ~3u, sh = (pos & 3u) * 8;
        const uint32_t w0 = *reinterpret_cast<const uint32_t*>(tv.sb + a);
        const uint32_t w1 = *reinterpret_cast<const uint32_t*>(tv.sb + a + 4);
        const uint64_t bts = static_cast<uint64_t>(__funnelshift_r(w0, w1, sh)) | (static_cast<uint64_t>(w1 >> sh) << 32);
        key = exact_key30(bts, len);
        if (P.comb && comb_add(ctab, key)) ex = false;   // absorbed by the combiner
      }
      const bool lg = act && len > kWcExact;
      const uint32_t ma = __ballot_sync(kFull, ex), mb = __ballot_sync(kFull, lg);
      if (ex) xq[nx + __popc(ma & lanemask_lt())] = key;
      else if (lg) hq[nq + __popc(mb & lanemask_lt())] = d;
      nx += __popc(ma);
      nq += __popc(mb);
      __syncwarp();
    }
  } else {
  uint32_t m_left = emit_mask;
  while (__any_sync(kFull, m_left != 0)) {
    const bool act = m_left != 0;
    uint32_t j = 0, len = 0;
    if (act) {
      j = __ffs(m_left) - 1;
      m_left &= m_left - 1;
      const uint32_t rest = nb >> (j + 1);
      len = rest ? static_cast<uint32_t>(__ffs(rest)) : len_slow;
    }
    bool ex = act && len <= kWcExact;
    uint32_t key = 0;
    if (ex) {
      key = exact_key30(window8(x, j), len);   // an exact word lies inside the 32 loaded bytes
      if (P.comb && comb_add(ctab, key)) ex = false;   // absorbed by the combiner
    }
    const uint32_t ma = __ballot_sync(kFull, ex), mb = __ballot_sync(kFull, act && len > kWcExact);
    if (ex) {
      xq[nx + __popc(ma & lanemask_lt())] = key;
    } else if (act && len > kWcExact) {
      if (len > 0xFFFFu) { atomicOr(&P.st->err, kErrKeyTooLong); len = 0xFFFFu; }
      // u32 queue entry: stage offset (< 2^15) | length << 15 (<= 0xFFFF)
      hq[nq + __popc(mb & lanemask_lt())] = static_cast<uint32_t>(p0 + j - tv.sbase) | (len << 15);
    }
    nx += __popc(ma);
    nq += __popc(mb);
  }
  }
  if (nx + nq == 0) return;
  if (P.si) {   // SI / G ablation: append straight to the three global streams, one atomic each
    __syncwarp();
    unsigned long long gx = 0;
    if (lane == 0 && nx) gx = atomicAdd(&P.st->pair_cursor, static_cast<unsigned long long>(nx));
    gx = __shfl_sync(kFull, gx, 0);
    for (uint32_t i = lane; i < nx; i += 32)
      if (gx + i < P.cap_pairs) P.ohx[gx + i] = xq[i];
    for (uint32_t q0 = 0; q0 < nq; q0 += 32) {
      const uint32_t q = q0 + lane;
      const bool in = q < nq;
      ulonglong2 ent = make_ulonglong2(0ULL, 0ULL);
      if (in) {
        const uint32_t e = hq[q];
        const long long p = tv.sbase + static_cast<long long>(e & 0x7FFFu);
        const uint32_t len = e >> 15;
        ent = len <= kMidMax ? make_ulonglong2(exact_key(bytes8_at(P, tv, p, len), len), 0ULL)
                             : make_ulonglong2(key_at(P, tv, p, len), (reinterpret_cast<uint64_t>(P.rec + p) << 16) | len);
      }
      const uint32_t mc = __ballot_sync(kFull, in && ent.y == 0), mbm = __ballot_sync(kFull, in && ent.y != 0);
      unsigned long long gc = 0, gbb = 0;
      if (lane == 0) {
        if (mc) gc = atomicAdd(&P.st->pair_cursor_c, static_cast<unsigned long long>(__popc(mc)));
        if (mbm) gbb = atomicAdd(&P.st->pair_cursor_b, static_cast<unsigned long long>(__popc(mbm)));
      }
      gc = __shfl_sync(kFull, gc, 0);
      gbb = __shfl_sync(kFull, gbb, 0);
      if (in && ent.y == 0) {
        const uint64_t o = gc + __popc(mc & lanemask_lt());
        if (o < P.cap_c) P.ohc[o] = ent.x;
      } else if (in) {
        const uint64_t o = gbb + __popc(mbm & lanemask_lt());
        if (o < P.cap_b) { P.ohb[o] = ent.x; P.okrefb[o] = ent.y; }
      }
    }
    return;
  }
  const uint32_t packed = nx | (nq << kCbShift);
  const Slot slot = reserve<kWC>(P, oc, outh, packed, P.out_cap);
  uint8_t* half = outh + slot.half * Cfg<kWC>::kOutHalf;
  uint32_t* sh = reinterpret_cast<uint32_t*>(half);
  ulonglong2* top = reinterpret_cast<ulonglong2*>(half + Cfg<kWC>::kOutHalf);   // hashed entry i: top[-1 - i]
  const uint32_t kb0 = cur_cb(slot.base), ka = cur_ca(slot.base);
  __syncwarp();
  for (uint32_t i = lane; i < nx; i += 32) sh[ka + i] = xq[i];
  __syncwarp();
  for (uint32_t q = lane; q < nq; q += 32) {           // lane-parallel keys of the long words
    const uint32_t e = hq[q];
    const long long p = tv.sbase + static_cast<long long>(e & 0x7FFFu);
    const uint32_t len = e >> 15;
    ulonglong2 ent;
    if (len <= kMidMax) {                                // mid stream: exact 48-bit key, no kref
      ent = make_ulonglong2(exact_key(bytes8_at(P, tv, p, len), len), 0ULL);
    } else {
      ent = make_ulonglong2(key_at(P, tv, p, len), (reinterpret_cast<uint64_t>(P.rec + p) << 16) | len);
    }
    top[-1 - static_cast<int>(kb0 + q)] = ent;
  }
  commit(oc, slot, packed);
}

// ---------------------------------------------------------------- WordCount fast path (SIO)
// The same computation as emit_text_chunk<kWC> + emit_wc (balanced mode) for one 512-B window,
// written for instruction count: no lane-0 / lane-31 divergent sections (every lane loads the
// byte before its chunk and classifies the next 16 bytes itself), one loop over the word starts
// that files exact and long words into separate queues (so the combiner rounds see exact words
// only), branch-free exact keys, predicated lane-0 shared atomics.
__device__ __forceinline__ uint32_t lane0_atom_add_shared(uint32_t* a, uint32_t v) {
  uint32_t old = 0;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.eq.u32 p, %2, 0;\n\t"
      "@p atom.shared.add.u32 %0, [%1], %3;\n\t}"
      : "+r"(old)
      : "r"(smem_u32(a)), "r"(threadIdx.x & 31u), "r"(v)
      : "memory");
  return __shfl_sync(kFull, old, 0);
}
__device__ __forceinline__ void lane0_mbar_arrive(uint64_t* bar) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.eq.u32 p, %1, 0;\n\t"
      "@p mbarrier.arrive.shared::cta.b64 _, [%0];\n\t}" ::"r"(smem_u32(bar)),
      "r"(threadIdx.x & 31u)
      : "memory");
}
// exact_key30 (common.cuh) without branches: lo = word bytes 0..3, b4 = byte 4, len 1..5
__device__ __forceinline__ uint32_t exact_key30_bf(uint32_t lo, uint32_t b4, uint32_t len) {
  const uint32_t c = exact_codes4(lo) & __funnelshift_lc(0xFFFFFFFFu, 0u, 8u * len);   // bytes < len
  uint32_t y = (c & 0x003F003Fu) | ((c >> 2) & 0x0FC00FC0u);   // byte pairs -> 12 bits
  y = (y & 0x00000FFFu) | ((y >> 4) & 0x00FFF000u);            // -> 24 bits
  const uint32_t c4 = exact_codes4(b4) & 0x3Fu;
  return y | (len == 5u ? (c4 << 24) : 0u);
}

// The same key from the word's first 4 bytes and the 4 bytes from byte 4 on (hiw, only its low
// byte used): the fifth code is computed on the whole word and masked, not narrowed by the
// compiler into byte-wise selects (8 instructions fewer per word)
__device__ __forceinline__ uint32_t opaque_u32(uint32_t x) {
  asm("" : "+r"(x));
  return x;
}
__device__ __forceinline__ uint32_t exact_key30_w(uint32_t lo, uint32_t hiw, uint32_t len) {
  const uint32_t c = exact_codes4(lo) & __funnelshift_lc(0xFFFFFFFFu, 0u, 8u * len);   // bytes < len
  uint32_t y = (c & 0x003F003Fu) | ((c >> 2) & 0x0FC00FC0u);   // byte pairs -> 12 bits
  y = (y & 0x00000FFFu) | ((y >> 4) & 0x00FFF000u);            // -> 24 bits
  const uint32_t c4 = opaque_u32(exact_codes4(opaque_u32(hiw)));
  return y | ((c4 << 24) & (len == 5u ? 0x3F000000u : 0u));
}

// 128-bit compare-and-swap on global memory (sm_90+ ATOMG.CAS.128): returns the old low half,
// the old high half in *ohi
__device__ __forceinline__ unsigned long long cas128(unsigned long long* p, unsigned long long clo,
                                                     unsigned long long chi, unsigned long long nlo,
                                                     unsigned long long nhi, unsigned long long& ohi) {
  unsigned long long olo;
  asm volatile(
      "{\n\t.reg .b128 c, n, r;\n\t"
      "mov.b128 c, {%2, %3};\n\t"
      "mov.b128 n, {%4, %5};\n\t"
      "atom.global.cas.b128 r, [%6], c, n;\n\t"
      "mov.b128 {%0, %1}, r;\n\t}"
      : "=l"(olo), "=l"(ohi)
      : "l"(clo), "l"(chi), "l"(nlo), "l"(nhi), "l"(p)
      : "memory");
  return olo;
}

// Output of the keyed long words: warp-private chunks of kLChunk entries of the mid stream (key
// only) and of the hashed stream (key + kref), each taken with ONE global atomic on the stream's
// cursor (the demand counter, D7) — the same amortisation as a buffer flush (L113) without the
// flush warp's routing pass.  A warp's unused chunk tail is filled with sentinel entries at the
// end (they sort last and are excluded: DevState::pads_b / pads_c).
constexpr uint32_t kLChunk = 256;
struct LOut { unsigned long long mid_base, hb_base; uint32_t mid_left, hb_left; };

// n lanes (mask m, rank r) append to a chunked stream; returns each lane's slot
__device__ __forceinline__ unsigned long long chunk_slot(unsigned long long* cursor, unsigned long long& base,
                                                        uint32_t& left, uint32_t m) {
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t n = __popc(m), r = __popc(m & lanemask_lt());
  unsigned long long nb = 0;
  if (n > left) {   // the rest goes into a fresh chunk
    if (lane == 0) nb = atomicAdd(cursor, static_cast<unsigned long long>(kLChunk));
    nb = __shfl_sync(kFull, nb, 0);
  }
  const unsigned long long slot = r < left ? base + r : nb + (r - left);
  if (n > left) {
    base = nb + (n - left);
    left = kLChunk - (n - left);
  } else {
    base += n;
    left -= n;
  }
  return slot;
}

// Key up to 32 queued long words (one per lane): mid words (6..8 bytes) get their exact 48-bit key
// (mid stream, no kref), longer ones the hash of their bytes (the same words KeyHash / hash_smem
// feed) with the batch-relative reference; stored into the warp's output chunks.
__device__ __forceinline__ void wc_drain(const Params& P, LOut& lo, LWord* lq, uint32_t& qn) {
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t n = min(qn, 32u);
  if (n == 0) return;
  __syncwarp();
  const bool in = lane < n;
  LWord w{0, 0, 0};
  if (in) w = lq[lane];
  const uint32_t len = static_cast<uint32_t>(w.meta & 0xFFFFu);
  const bool mid = in && len <= kMidMax;
  uint64_t key = 0, kref = 0;
  if (mid) {
    key = exact_key(w.lo, len);
  } else if (in) {
    KeyHash hs(P.hash_seed, len);
    const uint32_t wd[4] = {static_cast<uint32_t>(w.lo), static_cast<uint32_t>(w.lo >> 32), static_cast<uint32_t>(w.hi),
                            static_cast<uint32_t>(w.hi >> 32)};
#pragma unroll
    for (uint32_t k = 0; k < 4; ++k) {
      if (4 * k >= len) break;
      const uint32_t rem = len - 4 * k;
      hs.add(rem >= 4 ? wd[k] : (wd[k] & ((1u << (8 * rem)) - 1u)));
    }
    key = hashed_key(hs.finish(), (P.flags & 8u) != 0, P.key_bits);
    kref = (reinterpret_cast<uint64_t>(P.rec + (w.meta >> 16)) << 16) | len;
  }
  if (P.mkeys) {   // mid table: equal keys of the drain aggregated (match.any), then the group's
                  // leader finds the key (or claims an empty slot) and adds the group size to its
                  // warp's stripe of the slot's count (one RED)
    const uint32_t grp = BMR_MID_MATCH ? __match_any_sync(kFull, mid ? key : kMidEmpty) : (1u << lane);
    const bool lead = mid && lane == static_cast<uint32_t>(__ffs(grp) - 1);
    const uint64_t mask = (1ULL << P.mbits) - 1ULL;
    uint64_t h = mid_slot(key, P.mbits);
    bool done = !lead;
    for (uint32_t pr = 0; lead && pr < kMidProbes; ++pr, h = (h + 1) & mask) {
      // (an L1-cached read: a claimed slot never changes during the Map, and a stale empty only
      // sends the lane to the CAS, which returns the slot's real key)
      unsigned long long k = BMR_MID_LDCA ? __ldca(reinterpret_cast<const unsigned long long*>(P.mkeys + h))
                                          : *reinterpret_cast<volatile unsigned long long*>(P.mkeys + h);
      if (k == kMidEmpty) k = atomicCAS(reinterpret_cast<unsigned long long*>(P.mkeys + h), kMidEmpty, key);
      if (k == key || k == kMidEmpty) {
        red_add_u32(P.mcnt + stripe_at(h, (blockIdx.x * 7u + (threadIdx.x >> 5)) & (kMidStripes - 1), P.mbits),
                    static_cast<uint32_t>(__popc(grp)));
        done = true;
        break;
      }
    }
    if (!done) {   // table too full: counted, the batch is replayed with a larger table (D7)
      atomicOr(&P.st->err, kErrMidTable);
      atomicAdd(&P.st->mid_fail, 1ULL);
    }
  }
  if (P.lkeys) {   // long-word table (9..16 symbols): the same, keyed by the zero-padded key bytes
                  // (exact: words have no zero byte), slots claimed with a 128-bit CAS
    const bool lng = in && !mid;
    const uint64_t klo = lng ? w.lo : ~0ULL;
    const uint64_t khi = lng ? (len >= 16 ? w.hi : (w.hi & ((1ULL << (8 * (len - 8))) - 1ULL))) : ~0ULL;
    const uint32_t grp = __match_any_sync(kFull, klo) & __match_any_sync(kFull, khi);
    const bool lead = lng && lane == static_cast<uint32_t>(__ffs(grp) - 1);
    const uint64_t mask = (1ULL << P.lbits) - 1ULL;
    uint64_t h = long_slot(klo, khi, P.lbits);
    bool done = !lead;
    for (uint32_t pr = 0; lead && pr < kMidProbes; ++pr, h = (h + 1) & mask) {
      unsigned long long* slot = reinterpret_cast<unsigned long long*>(P.lkeys + 2 * h);
      unsigned long long olo, ohi;   // one 16-B access: the slot as the 128-bit CAS wrote it
      asm volatile("ld.volatile.global.v2.u64 {%0, %1}, [%2];" : "=l"(olo), "=l"(ohi) : "l"(slot) : "memory");
      // (two separate 8-B reads were measured to see claims half-done; should a 16-B read ever
      // do so — a key of 9+ bytes has hi != 0 — an atomic read settles it: CAS of zero by zero)
      if (olo != 0 && ohi == 0) olo = cas128(slot, 0ULL, 0ULL, 0ULL, 0ULL, ohi);
      if (olo == 0) {   // empty: claim it (128-bit CAS from all-zero)
        olo = cas128(slot, 0ULL, 0ULL, klo, khi, ohi);
        if (olo == 0) { olo = klo; ohi = khi; }   // claimed by this lane
      }
      if (olo == klo && ohi == khi) {
        red_add_u32(P.lcnt + stripe_at(h, (blockIdx.x * 7u + (threadIdx.x >> 5)) & (kMidStripes - 1), P.lbits),
                    static_cast<uint32_t>(__popc(grp)));
        done = true;
        break;
      }
    }
    if (!done) {
      atomicOr(&P.st->err, kErrLongTable);
      atomicAdd(&P.st->long_fail, 1ULL);
    }
  }
  const uint32_t mm = P.mkeys ? 0u : __ballot_sync(kFull, mid), mh = P.lkeys ? 0u : __ballot_sync(kFull, in && !mid);
  if (mm) {
    const unsigned long long o = chunk_slot(&P.st->pair_cursor_c, lo.mid_base, lo.mid_left, mm);
    if (mid && o < P.cap_c) P.ohc[o] = key;
  }
  if (mh) {
    const unsigned long long o = chunk_slot(&P.st->pair_cursor_b, lo.hb_base, lo.hb_left, mh);
    if (in && !mid && o < P.cap_b) {
      P.ohb[o] = key;
      P.okrefb[o] = kref;
    }
  }
  // the remaining entries (<= kLQ - 32) move to the queue's front
  const uint32_t rest = qn - n;
  LWord r{0, 0, 0};
  if (lane < rest) r = lq[n + lane];
  __syncwarp();
  if (lane < rest) lq[lane] = r;
  __syncwarp();
  qn = rest;
}
// Table mode (mid AND long tables present): the same counts as wc_drain with one probe pass.
// Mid words (6..8) and long words (9..16) share the match groups — a lane's (klo, khi) is
// (48-bit exact key, 0) for a mid word and its zero-padded key bytes for a long word; the two
// never collide (a long word's first 8 bytes are all non-zero: klo >= 2^56 > any 48-bit key) —
// and each group leader issues its table load (8-B mid slot or 16-B long slot) in the same
// round, so the two L2 round trips overlap.  No hash is computed (the tables are exact).
template <bool kUni>
__device__ __forceinline__ void wc_drain_tab(const Params& P, LWord* lq, uint32_t& qn) {
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t n = min(qn, 32u);
  if (n == 0) return;
  __syncwarp();
  LWord w{0, 0, 0};
  if (lane < n) w = lq[lane];
  const uint32_t len = static_cast<uint32_t>(w.meta & 0xFFFFu);
  const bool in = lane < n && len != 0;   // (len 0: a word left to the round loop)
  // with the exact-key table (kMode 1) the words of 6..8 symbols share the long table: key = the
  // zero-padded bytes, hi = kShortHi (no 48-bit key, no mid / long divergence in the drains)
  constexpr bool uni = kUni;
  const bool mid = in && !uni && len <= kMidMax, lng = in && !mid;
  const uint64_t klo = mid ? exact_key(w.lo, len) : lng ? (len >= 8 ? w.lo : (w.lo & ((1ULL << (8 * len)) - 1ULL))) : ~0ULL;
  const uint64_t khi = mid ? 0ULL
                       : lng ? (len >= 16 ? w.hi : len > 8 ? (w.hi & ((1ULL << (8 * (len - 8))) - 1ULL)) : kShortHi)
                             : ~0ULL;
  const uint32_t grp = __match_any_sync(kFull, klo) & __match_any_sync(kFull, khi);
  bool todo = in && lane == static_cast<uint32_t>(__ffs(grp) - 1);
  const uint32_t stripe = (blockIdx.x * 7u + (threadIdx.x >> 5)) & (kMidStripes - 1);
  const uint64_t mmask = (1ULL << P.mbits) - 1ULL, lmask = (1ULL << P.lbits) - 1ULL;
  uint64_t h = mid ? mid_slot(klo, P.mbits) : long_slot(klo, khi, P.lbits);
  for (uint32_t pr = 0; todo && pr < kMidProbes; ++pr) {
    if (mid) {
      unsigned long long k = *reinterpret_cast<volatile unsigned long long*>(P.mkeys + h);
      if (k == kMidEmpty) k = atomicCAS(reinterpret_cast<unsigned long long*>(P.mkeys + h), kMidEmpty, klo);
      if (k == klo || k == kMidEmpty) {
        red_add_u32(P.mcnt + stripe_at(h, stripe, P.mbits), static_cast<uint32_t>(__popc(grp)));
        todo = false;
      }
      h = (h + 1) & mmask;
    } else {
      unsigned long long* slot = reinterpret_cast<unsigned long long*>(P.lkeys + 2 * h);
      unsigned long long olo, ohi;   // one 16-B access: the slot as the 128-bit CAS wrote it
      asm volatile("ld.volatile.global.v2.u64 {%0, %1}, [%2];" : "=l"(olo), "=l"(ohi) : "l"(slot) : "memory");
      if (olo != 0 && ohi == 0) olo = cas128(slot, 0ULL, 0ULL, 0ULL, 0ULL, ohi);   // (see wc_drain)
      if (olo == 0) {
        olo = cas128(slot, 0ULL, 0ULL, klo, khi, ohi);
        if (olo == 0) { olo = klo; ohi = khi; }
      }
      if (olo == klo && ohi == khi) {
        red_add_u32(P.lcnt + stripe_at(h, stripe, P.lbits), static_cast<uint32_t>(__popc(grp)));
        todo = false;
      }
      h = (h + 1) & lmask;
    }
  }
  if (todo) {   // table too full: counted, the batch is replayed with a larger table (D7)
    atomicOr(&P.st->err, mid ? kErrMidTable : kErrLongTable);
    atomicAdd(mid ? &P.st->mid_fail : &P.st->long_fail, 1ULL);
  }
  const uint32_t rest = qn - n;
  LWord r{0, 0, 0};
  if (lane < rest) r = lq[n + lane];
  __syncwarp();
  if (lane < rest) lq[lane] = r;
  __syncwarp();
  qn = rest;
}

// Table mode with asynchronous probes (BMR_WC_ADRAIN): a drain resolves the warp's PREVIOUS batch
// of 32 long words and only issues this one.  Issue: the same keys, match groups and first slot
// as wc_drain_tab; each group leader stores its key in the warp's pending area and starts a
// cp.async of its first probe slot (8-B mid slot / 16-B long slot) next to it.  Resolve (one drain
// later, several windows of work after the issue, so the L2 round trip is long over): the
// prefetched slot is used as the first probe.  A stale slot value is safe — a slot only ever goes
// from empty to one key: a key seen is the slot's key for good, an empty slot is claimed by CAS
// (which returns the real value), and a torn 16-B view (low half only) is re-read atomically.
struct PEnt { unsigned long long klo, khi, vlo, vhi; };
struct PendQ {
  PEnt* e;          // 32 entries per warp (the exact-key queue region, unused in table mode)
  uint32_t* meta;   // per lane: bit 31 pending, bit 30 mid, bits 0..5 group size
  uint32_t* slot;   // per lane: first probe slot
};
template <bool kUni>
__device__ __forceinline__ void wc_probe_resolve(const Params& P, const PendQ& pq) {
  const uint32_t lane = threadIdx.x & 31;
  cp_async_wait_all();
  const uint32_t meta = pq.meta[lane];
  if (meta >> 31) {
    const PEnt e = pq.e[lane];
    const bool mid = !kUni && ((meta >> 30) & 1u);
    const uint32_t cnt = meta & 63u;
    const uint32_t stripe = (blockIdx.x * 7u + (threadIdx.x >> 5)) & (kMidStripes - 1);
    uint64_t h = pq.slot[lane];
    bool todo = true;
    unsigned long long vlo = e.vlo, vhi = e.vhi;   // first probe: the prefetched slot
    if (mid) {
      const uint64_t mmask = (1ULL << P.mbits) - 1ULL;
      for (uint32_t pr = 0; pr < kMidProbes; ++pr) {
        unsigned long long k = pr ? *reinterpret_cast<volatile unsigned long long*>(P.mkeys + h) : vlo;
        if (k == kMidEmpty) k = atomicCAS(reinterpret_cast<unsigned long long*>(P.mkeys + h), kMidEmpty, e.klo);
        if (k == e.klo || k == kMidEmpty) {
          red_add_u32(P.mcnt + stripe_at(h, stripe, P.mbits), cnt);
          todo = false;
          break;
        }
        h = (h + 1) & mmask;
      }
    } else {
      const uint64_t lmask = (1ULL << P.lbits) - 1ULL;
      for (uint32_t pr = 0; pr < kMidProbes; ++pr) {
        unsigned long long* sl = reinterpret_cast<unsigned long long*>(P.lkeys + 2 * h);
        unsigned long long olo = vlo, ohi = vhi;
        if (pr) asm volatile("ld.volatile.global.v2.u64 {%0, %1}, [%2];" : "=l"(olo), "=l"(ohi) : "l"(sl) : "memory");
        if (olo != 0 && ohi == 0) olo = cas128(sl, 0ULL, 0ULL, 0ULL, 0ULL, ohi);   // torn view: atomic re-read
        if (olo == 0) {
          olo = cas128(sl, 0ULL, 0ULL, e.klo, e.khi, ohi);
          if (olo == 0) { olo = e.klo; ohi = e.khi; }
        }
        if (olo == e.klo && ohi == e.khi) {
          red_add_u32(P.lcnt + stripe_at(h, stripe, P.lbits), cnt);
          todo = false;
          break;
        }
        h = (h + 1) & lmask;
      }
    }
    if (todo) {   // table too full: counted, the batch is replayed with a larger table (D7)
      atomicOr(&P.st->err, mid ? kErrMidTable : kErrLongTable);
      atomicAdd(mid ? &P.st->mid_fail : &P.st->long_fail, 1ULL);
    }
    pq.meta[lane] = 0;
  }
  __syncwarp();
}
template <bool kUni>
__device__ __forceinline__ void wc_probe_issue(const Params& P, LWord* lq, uint32_t& qn, const PendQ& pq) {
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t n = min(qn, 32u);
  if (n == 0) return;
  __syncwarp();
  LWord w{0, 0, 0};
  if (lane < n) w = lq[lane];
  const uint32_t len = static_cast<uint32_t>(w.meta & 0xFFFFu);
  const bool in = lane < n && len != 0;   // (len 0: a word left to the round loop)
  // with the exact-key table (kMode 1) the words of 6..8 symbols share the long table: key = the
  // zero-padded bytes, hi = kShortHi (no 48-bit key, no mid / long divergence in the drains)
  const bool uni = BMR_WC_UNITAB && P.xtab != nullptr;
  const bool mid = in && !uni && len <= kMidMax, lng = in && !mid;
  const uint64_t klo = mid ? exact_key(w.lo, len) : lng ? (len >= 8 ? w.lo : (w.lo & ((1ULL << (8 * len)) - 1ULL))) : ~0ULL;
  const uint64_t khi = mid ? 0ULL
                       : lng ? (len >= 16 ? w.hi : len > 8 ? (w.hi & ((1ULL << (8 * (len - 8))) - 1ULL)) : kShortHi)
                             : ~0ULL;
  const uint32_t grp = __match_any_sync(kFull, klo) & __match_any_sync(kFull, khi);
  const bool lead = in && lane == static_cast<uint32_t>(__ffs(grp) - 1);
  if (lead) {
    const uint64_t h = mid ? mid_slot(klo, P.mbits) : long_slot(klo, khi, P.lbits);
    PEnt* e = pq.e + lane;
    e->klo = klo;
    e->khi = khi;
    if (mid) cp_async_8(&e->vlo, P.mkeys + h);
    else cp_async_16(&e->vlo, P.lkeys + 2 * h);
    pq.slot[lane] = static_cast<uint32_t>(h);
    pq.meta[lane] = (1u << 31) | (mid ? (1u << 30) : 0u) | static_cast<uint32_t>(__popc(grp));
  }
  cp_async_commit();
  const uint32_t rest = qn - n;
  if (rest) {   // (warp-uniform; a queue of <= 32 entries drains whole)
    LWord r{0, 0, 0};
    if (lane < rest) r = lq[n + lane];
    __syncwarp();
    if (lane < rest) lq[lane] = r;
  }
  __syncwarp();
  qn = rest;
}
// drain of the table mode: synchronous (wc_drain_tab) or resolve-previous + issue
// kUni: the exact-key table mode (kMode 1) with the unified 6..16-symbol table, decided at compile time
template <bool kUni>
__device__ __forceinline__ void wc_drain_tq(const Params& P, LWord* lq, uint32_t& qn, const PendQ& pq) {
#if BMR_WC_ADRAIN
  wc_probe_resolve<kUni>(P, pq);
  wc_probe_issue<kUni>(P, lq, qn, pq);
#else
  wc_drain_tab<kUni>(P, lq, qn);
#endif
}

// end of a warp's work: sentinel entries in its chunks' unused tails
__device__ __forceinline__ void wc_chunk_pads(const Params& P, const LOut& lo) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t sent = sentinel_of(P.key_bits);
  for (uint32_t i = lane; i < lo.mid_left; i += 32)
    if (lo.mid_base + i < P.cap_c) P.ohc[lo.mid_base + i] = (1ULL << kMidBits) - 1ULL;
  for (uint32_t i = lane; i < lo.hb_left; i += 32)
    if (lo.hb_base + i < P.cap_b) {
      P.ohb[lo.hb_base + i] = sent;
      P.okrefb[lo.hb_base + i] = 0;
    }
  if (lane == 0) {
    if (lo.mid_left) atomicAdd(&P.st->pads_c, static_cast<unsigned long long>(lo.mid_left));
    if (lo.hb_left) atomicAdd(&P.st->pads_b, static_cast<unsigned long long>(lo.hb_left));
  }
}

// One 512-B window [p0w, p0w + 512) of a WordCount tile (lane = 16-byte chunk).  tv: the stage.
__device__ __forceinline__ void wc_window(const Params& P, OutCtl* oc, uint8_t* outh, const TileView& tv,
                                          long long p0w, uint32_t* xq, uint32_t* hq, uint32_t* ctab, LWord* lq,
                                          uint32_t& qn, LOut& lo) {
  const uint32_t lane = threadIdx.x & 31;
  const long long N = bd_nbytes();
  const long long p0 = p0w + 16 * lane;
  const uint32_t i0 = static_cast<uint32_t>(p0 - tv.sbase);   // 16-B aligned stage offset
  const uint4 c0 = *reinterpret_cast<const uint4*>(tv.sb + i0);
  const uint4 c1 = *reinterpret_cast<const uint4*>(tv.sb + i0 + 16);   // next chunk (lane 31: the halo)
  const uint32_t pb = tv.sb[i0 - 1];                                    // byte before the chunk (lead bytes)
  uint32_t wm = word_mask4(c0.x) | (word_mask4(c0.y) << 4) | (word_mask4(c0.z) << 8) | (word_mask4(c0.w) << 12) |
                (word_mask4(c1.x) << 16) | (word_mask4(c1.y) << 20) | (word_mask4(c1.z) << 24) |
                (word_mask4(c1.w) << 28);
  const bool edge = p0w < 0 || p0w + kWin + 16 > N;   // warp-uniform: only the input's first / last window
  if (edge) wm &= range_mask32(p0, 0, N);
  const uint32_t R = bits32(tv.bm, i0);                // record starts at p0 .. p0 + 31
  const uint32_t prevw = (p0 > 0 && is_word_byte(pb)) ? 1u : 0u;
  const uint32_t nb = ~wm | R;                          // a word cannot continue here
  const uint32_t S = wm & 0xFFFFu & ~(((wm << 1) | prevw) & ~R);   // word starts (C-2 WC)
  const uint32_t near = (nb >> 1) | (nb >> 2) | (nb >> 3) | (nb >> 4) | (nb >> 5);   // ends within 5 bytes
  // only the lane's highest start can lack a visible end (no stop in the 31 - j bytes after it)
  uint32_t len_slow = 0;
  if (S) {
    const uint32_t jh = 31 - __clz(S);
    if ((nb >> (jh + 1)) == 0) len_slow = slow_word_len(P, tv, p0 + jh, p0 + 32);
  }
  const uint32_t cx = __popc(S & near), cl = __popc(S & ~near);
  const uint32_t v = cx | (cl << 16);
  const uint32_t incl = warp_inclusive_add(v);
  const uint32_t tot = __shfl_sync(kFull, incl, 31);
  if (tot == 0) return;
  const uint32_t Wx = tot & 0xFFFFu, nl = tot >> 16;
  // phase 1: descriptors at the words' warp ranks — exact words (stage offset | len << 16) into
  // xq, long words (stage offset | len << 15) into hq
  {
    uint32_t kx = (incl - v) & 0xFFFFu, kl = (incl - v) >> 16;
    for (uint32_t m = S; m; m &= m - 1) {
      const uint32_t j = __ffs(m) - 1;
      const uint32_t rest = nb >> (j + 1);
      const uint32_t len = rest ? static_cast<uint32_t>(__ffs(rest)) : len_slow;
      const bool ex = (near >> j) & 1u;
      const uint32_t pos = i0 + j;
      const uint32_t ll = min(len, 0xFFFFu);
      uint32_t* dst = ex ? xq + kx : hq + kl;
      *dst = ex ? (pos | (len << 16)) : (pos | (ll << 15));
      kx += ex ? 1u : 0u;
      kl += ex ? 0u : 1u;
      if (len > 0xFFFFu) atomicOr(&P.st->err, kErrKeyTooLong);
    }
  }
  __syncwarp();
  // phase 2: exact words 32 at a time: key from the stage, combiner probe, misses compacted into xq
  uint32_t nx = 0;
  for (uint32_t b = 0; b < Wx; b += 32) {
    const bool act = b + lane < Wx;
    const uint32_t d = act ? xq[b + lane] : 0u;
    __syncwarp();                            // this round's reads before the compacting writes
    const uint32_t pos = d & 0xFFFFu, len = d >> 16;
    const uint32_t a = pos & ~3u, sh = (pos & 3u) * 8;
    const uint32_t w0 = *reinterpret_cast<const uint32_t*>(tv.sb + a);
    const uint32_t w1 = *reinterpret_cast<const uint32_t*>(tv.sb + a + 4);
    const uint32_t key = exact_key30_bf(__funnelshift_r(w0, w1, sh), (w1 >> sh) & 0xFFu, max(len, 1u));
    bool miss = act;
    if (act && P.comb) miss = !comb_add(ctab, key);
    if (P.xtab) {   // second level: one fire-and-forget L2 atomic per miss (RED.ADD), no pair
      if (miss) red_add_u32(P.xtab + key, 1u);
      continue;
    }
    const uint32_t ma = __ballot_sync(kFull, miss);
    if (miss) xq[nx + __popc(ma & lanemask_lt())] = key;
    nx += __popc(ma);
  }
  // exact keys that missed (exact-stream mode: no L2 table): one reservation, copied out
  if (nx) {
    const Slot slot = reserve<kWC>(P, oc, outh, nx, P.out_cap, true);
    __syncwarp();
    if (slot.half == kSpill) {   // ring congested: straight to HBM, padded to 4 keys like a flush
      const uint32_t r = (nx + 3u) & ~3u;
      unsigned long long gb = 0;
      if (lane == 0) {
        gb = atomicAdd(&P.st->pair_cursor, static_cast<unsigned long long>(r));
        if (r > nx) atomicAdd(&P.st->pads, static_cast<unsigned long long>(r - nx));
      }
      gb = __shfl_sync(kFull, gb, 0);
      for (uint32_t i = lane; i < r; i += 32)
        if (gb + i < P.cap_pairs) P.ohx[gb + i] = i < nx ? xq[i] : 0xFFFFFFFFu;
    } else {
      uint32_t* sh = reinterpret_cast<uint32_t*>(outh + slot.half * Cfg<kWC>::kOutHalf);
      const uint32_t ka = cur_ca(slot.base);
      for (uint32_t i = lane; i < nx; i += 32) sh[ka + i] = xq[i];
      commit(oc, slot, nx);
    }
  }
  // long words: their bytes into the warp's cross-window queue (keyed 32 at a time by wc_drain);
  // words longer than kLQMaxLen bytes (rare) are keyed here, one lane each
  for (uint32_t q0 = 0; q0 < nl; q0 += 32) {
    const uint32_t chunk = min(32u, nl - q0);
    if (qn + chunk > static_cast<uint32_t>(Cfg<kWC>::kLQ)) wc_drain(P, lo, lq, qn);
    const bool in = lane < chunk;
    const uint32_t e = in ? hq[q0 + lane] : 0u;
    const uint32_t pos = e & 0x7FFFu, len = e >> 15;
    const bool small = in && len <= kLQMaxLen;
    const uint32_t ms = __ballot_sync(kFull, small), mb = __ballot_sync(kFull, in && !small);
    if (small) {   // (a word of <= 16 bytes starting in the tile lies inside the staged window)
      LWord* d = lq + qn + __popc(ms & lanemask_lt());
      d->lo = static_cast<uint64_t>(smem_word_at(tv.sb, pos)) | (static_cast<uint64_t>(smem_word_at(tv.sb, pos + 4)) << 32);
      d->hi = static_cast<uint64_t>(smem_word_at(tv.sb, pos + 8)) | (static_cast<uint64_t>(smem_word_at(tv.sb, pos + 12)) << 32);
      d->meta = (static_cast<uint64_t>(tv.sbase + pos) << 16) | len;
    }
    qn += __popc(ms);
    if (mb) {
      const Slot slot = reserve<kWC>(P, oc, outh, __popc(mb) << kCbShift, P.out_cap);
      ulonglong2* top = reinterpret_cast<ulonglong2*>(outh + slot.half * Cfg<kWC>::kOutHalf + Cfg<kWC>::kOutHalf);
      if (in && !small) {
        const long long p = tv.sbase + static_cast<long long>(pos);
        top[-1 - static_cast<int>(cur_cb(slot.base) + __popc(mb & lanemask_lt()))] =
            make_ulonglong2(key_at(P, tv, p, len), (reinterpret_cast<uint64_t>(P.rec + p) << 16) | len);
      }
      commit(oc, slot, __popc(mb) << kCbShift);
    }
  }
  __syncwarp();
}

// One lane adds `cnt` occurrences of `key` (a 48-bit exact key: a word of <= 8 symbols; a word of
// <= 5 symbols has the same key as in the exact stream) to the mid table — the small-table mode's
// path for exact words that miss the SMEM combiner (no match-group aggregation: rare per lane).
__device__ __forceinline__ void mid_insert(const Params& P, uint64_t key, uint32_t cnt) {
  const uint64_t mask = (1ULL << P.mbits) - 1ULL;
  uint64_t h = mid_slot(key, P.mbits);
  const uint32_t stripe = (blockIdx.x * 7u + (threadIdx.x >> 5)) & (kMidStripes - 1);
  for (uint32_t pr = 0; pr < kMidProbes; ++pr, h = (h + 1) & mask) {
    unsigned long long k = *reinterpret_cast<volatile unsigned long long*>(P.mkeys + h);
    if (k == kMidEmpty) k = atomicCAS(reinterpret_cast<unsigned long long*>(P.mkeys + h), kMidEmpty, key);
    if (k == key || k == kMidEmpty) {
      red_add_u32(P.mcnt + stripe_at(h, stripe, P.mbits), cnt);
      return;
    }
  }
  atomicOr(&P.st->err, kErrMidTable);   // table too full: counted, the batch is replayed with a larger table
  atomicAdd(&P.st->mid_fail, 1ULL);
}

// Combiner update of one exact word without branches (predicated PTX): the slot's key is read;
// an empty slot is claimed by CAS; a slot holding the key (or just claimed) counts the word in
// SMEM, any other slot sends it to the L2 count table (RED).  Same semantics as comb_add + RED.
__device__ __forceinline__ void comb_or_table(uint32_t* slot_key, uint32_t* slot_cnt, uint32_t* tab, uint32_t key) {
  asm volatile(
      "{\n\t.reg .pred pe, ph;\n\t.reg .b32 v;\n\t"
      "ld.volatile.shared.u32 v, [%0];\n\t"
      "setp.eq.u32 pe, v, -1;\n\t"
      "@pe atom.shared.cas.b32 v, [%0], -1, %3;\n\t"
      "setp.eq.u32 ph, v, %3;\n\t"
      "@!ph setp.eq.u32 ph, v, -1;\n\t"
      "@ph red.shared.add.u32 [%1], 1;\n\t"
      "@!ph red.relaxed.gpu.global.add.u32 [%2], 1;\n\t}" ::"r"(smem_u32(slot_key)),
      "r"(smem_u32(slot_cnt)), "l"(tab), "r"(key)
      : "memory");
}

// One 512-B window in table mode (the default for large batches: exact words counted in the
// SMEM combiner + the L2 count table, longer words in the L2 mid / long tables, so the window
// emits nothing): no descriptor queues, no warp scan.  Each lane walks the exact-word starts of
// its own 16 bytes (a loop of max-over-lanes iterations; ~2.7 starts per lane at C5) and counts
// each word where it finds it; the starts of longer words are then moved into the warp's
// long-word queue one per lane per round.  The same words, keys and tables as wc_window.
template <bool kX>
__device__ __forceinline__ void wc_window_tab(const Params& P, OutCtl* oc, uint8_t* outh, const TileView& tv,
                                              long long p0w, uint32_t* ctab, LWord* lq, uint32_t& qn,
                                              uint32_t* dummy, const PendQ& pq) {
  const uint32_t lane = threadIdx.x & 31;
  const long long N = bd_nbytes();
  const long long p0 = p0w + 16 * lane;
  const uint32_t i0 = static_cast<uint32_t>(p0 - tv.sbase);   // 16-B aligned stage offset
  const uint4 c0 = *reinterpret_cast<const uint4*>(tv.sb + i0);
  const uint32_t pb = tv.sb[i0 - 1];                                    // byte before the chunk (lead bytes)
#if BMR_WC_CLS16
  // classes of the lane's own 16 bytes; those of the next 16 come from the next lane, and lane
  // 31's (the 16 bytes after the window) from lanes 0..3, one 4-byte word each (OR-reduced)
  const uint32_t own = word_mask4(c0.x) | (word_mask4(c0.y) << 4) | (word_mask4(c0.z) << 8) | (word_mask4(c0.w) << 12);
  const uint32_t hw = *reinterpret_cast<const uint32_t*>(tv.sb + (i0 - 16u * lane) + kWin + 4u * (lane & 3u));
  const uint32_t halo = __reduce_or_sync(kFull, lane < 4u ? word_mask4(hw) << (4u * lane) : 0u);
  const uint32_t nxt = __shfl_down_sync(kFull, own, 1);
  uint32_t wm = own | ((lane == 31u ? halo : nxt) << 16);
#else
  const uint4 c1 = *reinterpret_cast<const uint4*>(tv.sb + i0 + 16);   // next chunk (lane 31: the halo)
  uint32_t wm = word_mask4(c0.x) | (word_mask4(c0.y) << 4) | (word_mask4(c0.z) << 8) | (word_mask4(c0.w) << 12) |
                (word_mask4(c1.x) << 16) | (word_mask4(c1.y) << 20) | (word_mask4(c1.z) << 24) |
                (word_mask4(c1.w) << 28);
#endif
  const bool edge = p0w < 0 || p0w + kWin + 16 > N;   // warp-uniform: only the input's first / last window
  if (edge) wm &= range_mask32(p0, 0, N);
  const uint32_t R = bits32(tv.bm, i0);                // record starts at p0 .. p0 + 31
  const uint32_t prevw = (p0 > 0 && is_word_byte(pb)) ? 1u : 0u;
  const uint32_t nb = ~wm | R;                          // a word cannot continue here
  const uint32_t S = wm & 0xFFFFu & ~(((wm << 1) | prevw) & ~R);   // word starts (C-2 WC)
  const uint32_t near = (nb >> 1) | (nb >> 2) | (nb >> 3) | (nb >> 4) | (nb >> 5);   // ends within 5 bytes
  uint32_t* ccnt = ctab + Cfg<kWC>::kCombSlots;
  // exact words (<= 5 bytes): key from the stage, combiner slot or L2 count table
#if BMR_WC_XLOOP
  if constexpr (kX) {
    // The same words, keys and tables as the loop below, written for fewer instructions per
    // word: starts taken from the top (bfind), the length from the bit-reversed stop mask,
    // 32-bit shared addresses throughout, and the combiner hit counted by an unconditional
    // shared RED (a miss adds into this lane's dummy word) -- ptxas wraps every predicated
    // atomic in a divergent loop in its own branch region.
    const uint32_t sb32 = smem_u32(tv.sb) + i0;
    const uint32_t kb32 = smem_u32(ctab);
    const uint32_t dmy = smem_u32(dummy) + 4u * lane;
    // stops above byte j, bit-reversed and shifted so that the first one is the highest set bit:
    // len = 32 - bfind(rnb1 << j)
    const uint32_t rnb1 = __brev(nb) << 1;
    // key of the exact word starting at chunk byte j (a stop within 5 bytes after it)
    auto xkey = [&](uint32_t j) {
      const uint32_t len = 32u - bfind_u32(rnb1 << j);   // first stop above j
      const uint32_t a = sb32 + (j & ~3u);
      const uint32_t w0 = lds_u32(a), w1 = lds_u32(a + 4u);
      return exact_key30_w(__funnelshift_r(w0, w1, j << 3), __funnelshift_r(w1, w1, j << 3), len);
    };
#if BMR_WC_XPAIR
    // two words per iteration (the highest and the lowest start left): the same instructions per
    // word, two independent dependency chains (the loop is latency-bound), half the iterations
    for (uint32_t E = S & near; E;) {
      const uint32_t j1 = bfind_u32(E);                          // highest start left
      const uint32_t j2 = static_cast<uint32_t>(__ffs(E)) - 1u;   // lowest (== j1: one left)
      const bool two = j2 != j1;
      E &= (E - 1u) & ~(1u << j1);
      const uint32_t k1 = xkey(j1), k2 = xkey(j2);
      uint32_t ka1 = kb32 + 4u * ((k1 * 0x9E3779B1u) >> (32 - kCombBits));
      uint32_t ka2 = kb32 + 4u * ((k2 * 0x9E3779B1u) >> (32 - kCombBits));
      uint32_t v1 = lds_volatile_u32(ka1), v2 = lds_volatile_u32(ka2);
      if (v1 == kCombEmpty32 || v2 == kCombEmpty32) {   // (claims: only until the table has filled)
        if (v1 == kCombEmpty32) v1 = atom_cas_shared_u32(ka1, kCombEmpty32, k1);
        if (two && v2 == kCombEmpty32) v2 = atom_cas_shared_u32(ka2, kCombEmpty32, k2);   // (CAS: the real slot)
      }
      bool h1 = v1 == k1 || v1 == kCombEmpty32;
      bool h2 = two && (v2 == k2 || v2 == kCombEmpty32);
#if BMR_WC_X2WAY
      // a key whose home slot belongs to another key gets a second slot (home ^ 1): fewer words
      // left to the L2 table, whose REDs on Zipf-hot keys serialise
      if (!h1) {
        const uint32_t kb = ka1 ^ 4u;
        uint32_t v = lds_volatile_u32(kb);
        if (v == kCombEmpty32) v = atom_cas_shared_u32(kb, kCombEmpty32, k1);
        h1 = v == k1 || v == kCombEmpty32;
        ka1 = h1 ? kb : ka1;
      }
      if (two && !h2) {
        const uint32_t kb = ka2 ^ 4u;
        uint32_t v = lds_volatile_u32(kb);
        if (v == kCombEmpty32) v = atom_cas_shared_u32(kb, kCombEmpty32, k2);
        h2 = v == k2 || v == kCombEmpty32;
        ka2 = h2 ? kb : ka2;
      }
#endif
      // the slot's count gets 1 on a hit, 0 on a miss (a no-op on another key's count): no
      // predicated atomic, no dummy address
      red_shared_add_u32(ka1 + 4u * Cfg<kWC>::kCombSlots, h1 ? 1u : 0u);
      red_shared_add_u32(ka2 + 4u * Cfg<kWC>::kCombSlots, h2 ? 1u : 0u);
      if (!h1) red_add_u32(P.xtab + k1, 1u);
      if (two && !h2) red_add_u32(P.xtab + k2, 1u);
    }
#else
    for (uint32_t E = S & near; E;) {
      const uint32_t j = bfind_u32(E);
      E &= ~(1u << j);
      const uint32_t key = xkey(j);
      const uint32_t ka = kb32 + 4u * ((key * 0x9E3779B1u) >> (32 - kCombBits));
      uint32_t v = lds_volatile_u32(ka);
      if (v == kCombEmpty32) v = atom_cas_shared_u32(ka, kCombEmpty32, key);
      const bool hit = v == key || v == kCombEmpty32;
      red_shared_add_u32(hit ? ka + 4u * Cfg<kWC>::kCombSlots : dmy, 1u);
      if (!hit) red_add_u32(P.xtab + key, 1u);
    }
#endif
  } else
#endif
  for (uint32_t E = S & near; E; E &= E - 1) {
    const uint32_t j = __ffs(E) - 1;
    const uint32_t len = __ffs(nb >> (j + 1));         // 1..5: a stop within 5 bytes
    const uint32_t pos = i0 + j;
    const uint32_t a = pos & ~3u, sh = (pos & 3u) * 8;
    const uint32_t w0 = *reinterpret_cast<const uint32_t*>(tv.sb + a);
    const uint32_t w1 = *reinterpret_cast<const uint32_t*>(tv.sb + a + 4);
    const uint32_t key = exact_key30_bf(__funnelshift_r(w0, w1, sh), (w1 >> sh) & 0xFFu, len);
    const uint32_t home = (key * 0x9E3779B1u) >> (32 - kCombBits);
    if constexpr (kX) {
      comb_or_table(ctab + home, ccnt + home, P.xtab + key, key);
    } else {   // small-table mode: a combiner miss goes to the mid table
      uint32_t v = *reinterpret_cast<volatile uint32_t*>(ctab + home);
      if (v == kCombEmpty32) v = atomicCAS(ctab + home, kCombEmpty32, key);
      if (v == key || v == kCombEmpty32) atomicAdd(ccnt + home, 1u);
      else mid_insert(P, key, 1u);
    }
  }
  // longer words: only the lane's highest start can lack a visible end (no stop in the 31 - j
  // bytes after it)
  uint32_t L = S & ~near;
  if (!__any_sync(kFull, L)) return;
#if BMR_WC_LSCAN
  {
    // every long start goes to the queue at its warp rank, each lane writing its own (no rounds):
    // a lane holds at most 3 of them (a long word and its delimiter take >= 7 of its 16 bytes),
    // so the warp prefix comes from three ballots.  An entry's meta is the word length (6..16);
    // a word with no stop within 16 bytes gets meta 0 (skipped by the drain) and is left to the
    // round loop below, as are all of a window with more long words than a queue holds.
    const uint32_t cs = __popc(L);
    const uint32_t b1 = __ballot_sync(kFull, cs >= 1u), b2 = __ballot_sync(kFull, cs >= 2u),
                   b3 = __ballot_sync(kFull, cs >= 3u);
    const uint32_t lt = lanemask_lt();
    const uint32_t incl = __popc(b1 & lt) + __popc(b2 & lt) + __popc(b3 & lt) + cs;
    const uint32_t tot = __popc(b1) + __popc(b2) + __popc(b3);
    if (tot <= static_cast<uint32_t>(Cfg<kWC>::kLQ)) {
      uint32_t big = 0;
      while (qn + tot > static_cast<uint32_t>(Cfg<kWC>::kLQ)) wc_drain_tq<kX && BMR_WC_UNITAB>(P, lq, qn, pq);
      LWord* d = lq + qn + incl - cs;
      for (uint32_t m = L; m; m &= m - 1, ++d) {
        const uint32_t j = __ffs(m) - 1;
        const uint32_t len = __ffs(nb >> (j + 1));   // 6..31, 0: no stop in view
        const bool ok = len != 0 && len <= kLQMaxLen;
        big |= ok ? 0u : (1u << j);
        const uint32_t pos = i0 + j;
        const uint32_t* src = reinterpret_cast<const uint32_t*>(tv.sb + (pos & ~3u));
        const uint32_t sh = pos << 3;   // 5 aligned words, funnel-shifted (shift amount mod 32)
        const uint32_t y0 = src[0], y1 = src[1], y2 = src[2], y3 = src[3], y4 = src[4];
        d->lo = static_cast<uint64_t>(__funnelshift_r(y0, y1, sh)) | (static_cast<uint64_t>(__funnelshift_r(y1, y2, sh)) << 32);
        d->hi = static_cast<uint64_t>(__funnelshift_r(y2, y3, sh)) | (static_cast<uint64_t>(__funnelshift_r(y3, y4, sh)) << 32);
        d->meta = ok ? len : 0u;
      }
      qn += tot;
      __syncwarp();
      L = big;
      if (!__any_sync(kFull, L)) return;
    }
  }
#endif
  uint32_t len_slow = 0;
  if (L) {
    const uint32_t jh = 31 - __clz(S);
    if ((nb >> (jh + 1)) == 0) len_slow = slow_word_len(P, tv, p0 + jh, p0 + 32);
  }
  for (;;) {   // one long word per lane per round, appended to the warp's queue
    const uint32_t m = __ballot_sync(kFull, L != 0);
    if (!m) break;
    if (qn + __popc(m) > static_cast<uint32_t>(Cfg<kWC>::kLQ)) wc_drain_tq<kX && BMR_WC_UNITAB>(P, lq, qn, pq);
    uint32_t j = 0, len = 0;
    if (L) {
      j = __ffs(L) - 1;
      L &= L - 1;
      const uint32_t rest = nb >> (j + 1);
      len = rest ? static_cast<uint32_t>(__ffs(rest)) : len_slow;
      if (len > 0xFFFFu) atomicOr(&P.st->err, kErrKeyTooLong);
    }
    const bool in = (m >> lane) & 1u;
    const bool small = in && len <= kLQMaxLen;
    const uint32_t ms = __ballot_sync(kFull, small), mb = m & ~ms;
    const uint32_t pos = i0 + j;
    if (small) {   // (a word of <= 16 bytes starting in the tile lies inside the staged window)
      LWord* d = lq + qn + __popc(ms & lanemask_lt());
      const uint32_t* src = reinterpret_cast<const uint32_t*>(tv.sb + (pos & ~3u));
      const uint32_t sh = (pos & 3u) * 8;   // 5 aligned words, funnel-shifted
      const uint32_t y0 = src[0], y1 = src[1], y2 = src[2], y3 = src[3], y4 = src[4];
      d->lo = static_cast<uint64_t>(__funnelshift_r(y0, y1, sh)) | (static_cast<uint64_t>(__funnelshift_r(y1, y2, sh)) << 32);
      d->hi = static_cast<uint64_t>(__funnelshift_r(y2, y3, sh)) | (static_cast<uint64_t>(__funnelshift_r(y3, y4, sh)) << 32);
      d->meta = (static_cast<uint64_t>(tv.sbase + pos) << 16) | len;
    }
    qn += __popc(ms);
    if (mb) {   // words of > 16 bytes (rare): hashed-stream entries through the output ring
      const Slot slot = reserve<kWC>(P, oc, outh, __popc(mb) << kCbShift, P.out_cap);
      ulonglong2* top = reinterpret_cast<ulonglong2*>(outh + slot.half * Cfg<kWC>::kOutHalf + Cfg<kWC>::kOutHalf);
      if (in && !small) {
        const long long p = tv.sbase + static_cast<long long>(pos);
        top[-1 - static_cast<int>(cur_cb(slot.base) + __popc(mb & lanemask_lt()))] =
            make_ulonglong2(key_at(P, tv, p, len), (reinterpret_cast<uint64_t>(P.rec + p) << 16) | len);
      }
      commit(oc, slot, __popc(mb) << kCbShift);
    }
  }
  __syncwarp();
}

// WordCount map warps in SIO mode: windows from the shared counter (tile order), the stage
// header read once per tile change, the window loop of wc_window (wc_window_tab in table mode).
// kMode: 0 wc_window (streams, or tables behind the old rounds), 1 wc_window_tab with the exact-key
// table, 2 wc_window_tab in small-table mode (no exact-key table)
template <int kMode>
__device__ void wc_map_loop(const Params& P, uint8_t* smem, OutCtl* oc) {
  constexpr bool kTab = kMode != 0;
  constexpr int W = kWC;
  constexpr int kStages = Cfg<W>::kStages;
  const uint32_t warp = threadIdx.x >> 5;
  uint64_t* empty = reinterpret_cast<uint64_t*>(smem + Layout<W>::empty);
  uint64_t* ready = reinterpret_cast<uint64_t*>(smem + Layout<W>::ready);
  uint8_t* outh = smem + Layout<W>::out;
  uint32_t* hq = reinterpret_cast<uint32_t*>(smem + Layout<kWC>::hq) + warp * Cfg<kWC>::kHashQ;
  uint32_t* xq = reinterpret_cast<uint32_t*>(smem + Layout<kWC>::xq) + warp * Cfg<kWC>::kXQ;
  uint32_t* ctab = reinterpret_cast<uint32_t*>(smem + Layout<kWC>::comb);
  LWord* lq = reinterpret_cast<LWord*>(smem + Layout<kWC>::lq) + warp * Cfg<kWC>::kLQ;
  uint32_t qn = 0;   // long words queued by this warp
  LOut lo{0, 0, 0, 0};   // this warp's output chunks (none yet)
  // table mode: the exact-key / hash queues are unused -> dummy words, pending probes
  const PendQ pq{reinterpret_cast<PEnt*>(xq), hq + 32, hq + 64};
  if constexpr (kTab) {
    pq.meta[threadIdx.x & 31] = 0;
    __syncwarp();
  }
  uint32_t have_it = ~0u;
  long long t = 0, sbase = 0, hi = 0, stg_hi = 0;
  // table mode with dynamic tiles: two windows per fetch (one window-counter atomic, stage check
  // and empty arrival per pair; the producers post the end marker at two iterations, so every
  // map warp meets it: 16 pairs per tile < 24 map warps)
  constexpr uint32_t kPW = (kTab && BMR_WC_PAIRWIN && BMR_DYN_TILES) ? 2u : 1u;
  static_assert(kNWin % kPW == 0, "window pairs must not straddle tiles");
  for (;;) {
    const uint32_t g = lane0_atom_add_shared(&oc->win_next, kPW);
    const uint32_t it = g / kNWin, w = g % kNWin;
    const uint32_t s = it % kStages;
    if (it != have_it) {   // wait for the tile's record-start bitmap, then its header
      map_wait(P, ready + s, (it / kStages) & 1u, kReadyWaitNs);
      const StageHdr* hd = reinterpret_cast<const StageHdr*>(smem + Layout<W>::hdr + s * 128);
      t = hd->t;
      sbase = hd->sbase;
      hi = hd->hi;
      stg_hi = hd->stg_hi;
      have_it = it;
    }
    if (t == -1) break;   // (-2: a skip stage, no windows)
    const TileView tv{smem + Layout<W>::bytes + s * kStageBytes,
                      reinterpret_cast<const uint32_t*>(smem + Layout<W>::bits + s * Cfg<W>::kBits), sbase, stg_hi, 0,
                      0};
#pragma unroll 1
    for (uint32_t q = 0; q < kPW; ++q) {
      const long long wp = sbase + kLead + static_cast<long long>(w + q) * kWin;
      if (wp < hi) {   // warp-uniform
        if constexpr (kTab) wc_window_tab<kMode == 1>(P, oc, outh, tv, wp, ctab, lq, qn, hq, pq);
        else wc_window(P, oc, outh, tv, wp, xq, hq, ctab, lq, qn, lo);
        if (qn >= 32) {
          if constexpr (kTab) wc_drain_tq<kMode == 1 && BMR_WC_UNITAB>(P, lq, qn, pq);
          else wc_drain(P, lo, lq, qn);
        }
      }
    }
    __syncwarp();
    if (kPW == 1) lane0_mbar_arrive(&empty[s]);
    else if ((threadIdx.x & 31) == 0) mbar_arrive_cnt(&empty[s], kPW);
  }
  while (qn) {   // this warp's last long words
    if constexpr (kTab) wc_drain_tq<kMode == 1 && BMR_WC_UNITAB>(P, lq, qn, pq);
    else wc_drain(P, lo, lq, qn);
  }
#if BMR_WC_ADRAIN
  if constexpr (kTab) wc_probe_resolve<kMode == 1 && BMR_WC_UNITAB>(P, pq);   // the last batch issued
#endif
  wc_chunk_pads(P, lo);
}

// InvertedIndex URL queue (per map warp, in the hq region): the markers of a window are queued as
// (URL position, length) and the queue is drained 32..64 entries at a time, one entry per lane:
// key (inline or the hash of the URL bytes, read from global memory so the stage can go), one
// reservation, SoA stores.  A window holds about one URL, so hashing it in the window's emission
// round left 31 lanes idle for the whole hash (ncu C4 round 1: ~15% of the Map's instructions).
__device__ __forceinline__ uint64_t* ii_qpos(uint8_t* outh) {
  return reinterpret_cast<uint64_t*>(outh + (Layout<kII>::hq - Layout<kII>::out)) +
         (threadIdx.x >> 5) * (Cfg<kII>::kHashQ / 2);
}
// f-3: fused Map flush + shuffle.  The drained URLs go straight to the receive
// window of their destination rank (dest_of_bytes of the URL bytes, as in the partition pass):
// per destination one pair of atomics per warp (entries, heap bytes) on the window's cursor —
// over NVLink when the window lives on a peer GPU — then the 16-B entry and the key bytes are
// stored into it.  No local pairs, no partition pass, no all-to-all: the transfer overlaps the
// Map.  Demand past a window's capacity is still counted (mr_ingest_xwindow reports it).
__device__ void ii_drain_xwin(const Params& P, uint32_t qn, const uint64_t* qpos, const uint32_t* qlen) {
  const uint32_t lane = threadIdx.x & 31;
  for (uint32_t e0 = 0; e0 < qn; e0 += 32) {
    const uint32_t e = e0 + lane;
    const bool in = e < qn;
    const long long q0 = in ? static_cast<long long>(qpos[e]) : 0;
    const uint32_t len = in ? qlen[e] : 0u;
    const uint8_t* kp = P.rec + q0;
    const uint32_t d = in ? dest_of_bytes_g(kp, len, P.xranks) : ~0u;
    const uint32_t hb = (len + 7u) & ~7u;
    unsigned long long ie = 0, ih = 0;
    for (uint32_t r = 0; r < P.xranks; ++r) {
      const uint32_t m = __ballot_sync(kFull, d == r);
      if (!m) continue;
      const uint32_t hv = d == r ? hb : 0u;
      const uint32_t incl = warp_inclusive_add(hv);
      const uint32_t tot = __shfl_sync(kFull, incl, 31);
      const uint32_t leader = __ffs(m) - 1;
      unsigned long long be = 0, bh = 0;
      if (lane == leader) {
        be = atomicAdd(P.xwin[r].cursor, static_cast<unsigned long long>(__popc(m)));
        bh = atomicAdd(P.xwin[r].cursor + 1, static_cast<unsigned long long>(tot));
      }
      be = __shfl_sync(kFull, be, leader);
      bh = __shfl_sync(kFull, bh, leader);
      if (d == r) {
        ie = be + __popc(m & lanemask_lt());
        ih = bh + incl - hv;
      }
    }
    if (in) {
      const XWindow w = P.xwin[d];
      if (ie < w.ecap && ih + hb <= w.hcap) {
        XEntry* o = reinterpret_cast<XEntry*>(w.entries) + ie;
        o->koff_len = (static_cast<uint64_t>(ih) << 16) | len;
        o->v = bd_gbase() + static_cast<uint64_t>(q0);
        for (uint32_t k = 0; k < len; k += 8)   // heap records are 8-B aligned
          *reinterpret_cast<uint64_t*>(w.heap + ih + k) = load8(kp + k, min(8u, len - k));
      }
    }
  }
}

__device__ void ii_drain(const Params& P, OutCtl* oc, uint8_t* outh, uint32_t& qn) {
  using F = PairFmt<kII>;
  if (qn == 0) return;
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t* qpos = ii_qpos(outh);
  const uint32_t* qlen = reinterpret_cast<const uint32_t*>(qpos + 64);
  __syncwarp();
  if (P.xranks) {
    ii_drain_xwin(P, qn, qpos, qlen);
    __syncwarp();
    qn = 0;
    return;
  }
  const Slot slot = reserve<kII>(P, oc, outh, qn, P.out_cap, true);
  const TileView gv{nullptr, nullptr, 0, LLONG_MIN, 0, 0};   // key bytes from global memory
  if (slot.half == kSpill) {   // ring congested: straight to HBM, padded to 4 pairs like a flush
    const uint32_t r = (qn + 3u) & ~3u;
    unsigned long long gb = 0;
    if (lane == 0) {
      gb = atomicAdd(&P.st->pair_cursor, static_cast<unsigned long long>(r));
      if (r > qn) atomicAdd(&P.st->pads, static_cast<unsigned long long>(r - qn));
    }
    gb = __shfl_sync(kFull, gb, 0);
    for (uint32_t e = lane; e < r; e += 32) {
      if (gb + e >= P.cap_pairs) continue;
      if (e < qn) {
        const long long q0 = static_cast<long long>(qpos[e]);
        const uint32_t len = qlen[e];
        P.oh[gb + e] = key_at(P, gv, q0, len);
        P.okref[gb + e] = (reinterpret_cast<uint64_t>(P.rec + q0) << 16) | len;
        reinterpret_cast<uint64_t*>(P.ov)[gb + e] = bd_gbase() + static_cast<uint64_t>(q0);
      } else {
        P.oh[gb + e] = sentinel_key<kII>(P);
        P.okref[gb + e] = 0;
        reinterpret_cast<uint64_t*>(P.ov)[gb + e] = 0;
      }
    }
    __syncwarp();
    qn = 0;
    return;
  }
  uint8_t* half = outh + slot.half * Cfg<kII>::kOutHalf;
  uint64_t* sh = reinterpret_cast<uint64_t*>(half);
  uint64_t* sk = sh + F::kCap;
  uint64_t* sv = reinterpret_cast<uint64_t*>(half + F::kCap * 16);
  for (uint32_t e = lane; e < qn; e += 32) {
    const long long q0 = static_cast<long long>(qpos[e]);
    const uint32_t len = qlen[e];
    const uint32_t idx = slot.base + e;
    sh[idx] = key_at(P, gv, q0, len);
    sk[idx] = (reinterpret_cast<uint64_t>(P.rec + q0) << 16) | len;
    sv[idx] = bd_gbase() + static_cast<uint64_t>(q0);
  }
  commit(oc, slot, qn);
  qn = 0;
}

// ---------------------------------------------------------------- InvertedIndex fast path (SIO)
// The computation of emit_text_chunk<kII> for one 512-B window, with the work done lazily: the
// has-'<' test first (most 16-B chunks have none), the '<' positions and marker checks only in
// lanes that have one, the '"' / record-start stop masks only when the warp found a marker, the
// range masks only in the input's first / last window; predicated lane-0 atomics.
__device__ __forceinline__ void ii_window(const Params& P, OutCtl* oc, uint8_t* outh, const TileView& tv,
                                          long long p0w, uint32_t& qn) {
  const uint32_t lane = threadIdx.x & 31;
  const long long N = bd_nbytes();
  const long long p0 = p0w + 16 * lane;
  const uint32_t i0 = static_cast<uint32_t>(p0 - tv.sbase);
  const uint4 c0 = *reinterpret_cast<const uint4*>(tv.sb + i0);
  uint32_t a = 0;
  {
    const uint32_t t0 = c0.x ^ 0x3C3C3C3Cu, t1 = c0.y ^ 0x3C3C3C3Cu, t2 = c0.z ^ 0x3C3C3C3Cu, t3 = c0.w ^ 0x3C3C3C3Cu;
    a = (((t0 - 0x01010101u) & ~t0) | ((t1 - 0x01010101u) & ~t1) | ((t2 - 0x01010101u) & ~t2) |
         ((t3 - 0x01010101u) & ~t3)) & 0x80808080u;
  }
  if (!__any_sync(kFull, a != 0)) return;   // no '<' in the window: no marker (exact has-byte test)
  const bool edge = p0w < 0 || p0w + kWin + 16 > N;   // warp-uniform
  const uint32_t vm = edge ? range_mask32(p0, 0, N) : kFull;
  const uint32_t R = bits32(tv.bm, i0);
  const uint4 c1 = *reinterpret_cast<const uint4*>(tv.sb + i0 + 16);
  const uint32_t x[8] = {c0.x, c0.y, c0.z, c0.w, c1.x, c1.y, c1.z, c1.w};
  uint32_t mk = 0;
  if (a) {   // markers of this lane's chunk (rare lanes)
    uint32_t cand = (eq_mask4(x[0], 0x3C3C3C3Cu) | (eq_mask4(x[1], 0x3C3C3C3Cu) << 4) |
                     (eq_mask4(x[2], 0x3C3C3C3Cu) << 8) | (eq_mask4(x[3], 0x3C3C3C3Cu) << 12)) & vm & 0xFFFFu;
    while (cand) {
      const uint32_t j = __ffs(cand) - 1;
      cand &= cand - 1;
      if (p0 + j + 9 > N) continue;
      if ((R >> (j + 1)) & 0xFFu) continue;               // marker inside one record
      uint32_t w[4];
      window16(x, j, w);
      // "<a href=\"" little-endian: 3C 61 20 68 | 72 65 66 3D | 22
      if (w[0] != 0x6820613Cu || w[1] != 0x3D666572u || (w[2] & 0xFFu) != 0x22u) continue;
      mk |= 1u << j;
    }
  }
  if (!__any_sync(kFull, mk != 0)) return;
  // the URL of a marker ends at the first '"' unless a record starts first (C-3 #9): every lane
  // publishes its 16-bit stop mask and a marker finds the first stop after its URL start with two
  // shuffles; only URLs leaving the window scan onwards
  const uint32_t qm = eq_mask4(x[0], 0x22222222u) | (eq_mask4(x[1], 0x22222222u) << 4) |
                      (eq_mask4(x[2], 0x22222222u) << 8) | (eq_mask4(x[3], 0x22222222u) << 12);
  const uint32_t st16 = ((qm & vm) | R) & 0xFFFFu;
  const uint32_t lanes_st = __ballot_sync(kFull, st16 != 0);
  const uint32_t r16 = R & 0xFFFFu;
  uint32_t emit_mask = 0, aux[2] = {0, 0};
  int nm = 0;
  for (int mi = 0; mi < 2; ++mi) {          // a 9-byte marker: at most two start in 16 bytes
    if (!__any_sync(kFull, mk != 0)) break;
    const bool has = mk != 0;
    const uint32_t j = has ? static_cast<uint32_t>(__ffs(mk) - 1) : 0u;
    if (has) mk &= mk - 1;
    const uint32_t au = lane * 16 + j + 9;   // window offset of the URL start
    const uint32_t T = min(au >> 4, 31u);
    const uint32_t sT = __shfl_sync(kFull, st16, T), rT = __shfl_sync(kFull, r16, T);
    const uint32_t cT = au < static_cast<uint32_t>(kWin) ? (sT >> (au & 15u)) << (au & 15u) : 0u;
    const uint32_t later = T < 31 ? (lanes_st & ~((2u << T) - 1u)) : 0u;
    const uint32_t F = later ? static_cast<uint32_t>(__ffs(later) - 1) : 31u;
    const uint32_t sF = __shfl_sync(kFull, st16, F), rF = __shfl_sync(kFull, r16, F);
    if (!has) continue;
    const long long q0 = p0 + j + 9;
    long long q;
    if (cT) {
      const uint32_t b = __ffs(cT) - 1;
      q = ((rT >> b) & 1u) ? -1 : p0w + T * 16 + b;     // record ends first -> unclosed
    } else if (later && au < static_cast<uint32_t>(kWin)) {
      const uint32_t b = __ffs(sF) - 1;
      q = ((rF >> b) & 1u) ? -1 : p0w + F * 16 + b;
    } else {                                           // no stop in the window: scan onwards
      q = find_quote(P, tv, max(q0, p0w + kWin), p0 + j);
    }
    if (q > q0 && nm < 2) {
      aux[nm++] = static_cast<uint32_t>(q - q0);
      emit_mask |= 1u << j;
    }
  }
  // queue the URLs (drained lane-parallel by ii_drain)
  const uint32_t cnt = __popc(emit_mask);   // <= 2 markers start in 16 bytes
  // the warp prefix from two ballots (cnt <= 2) instead of a 5-step shuffle scan
  const uint32_t b1 = __ballot_sync(kFull, cnt >= 1u), b2 = __ballot_sync(kFull, cnt >= 2u);
  const uint32_t tot = __popc(b1) + __popc(b2);
  if (tot == 0) return;
  const uint32_t lt = lanemask_lt();
  const uint32_t incl = __popc(b1 & lt) + __popc(b2 & lt) + cnt;
  if (qn + tot > 64) ii_drain(P, oc, outh, qn);
  uint64_t* qpos = ii_qpos(outh);
  uint32_t* qlen = reinterpret_cast<uint32_t*>(qpos + 64);
  uint32_t k = qn + incl - cnt;
  int nth = 0;
  for (uint32_t m = emit_mask; m; m &= m - 1) {
    const uint32_t j = __ffs(m) - 1;
    uint32_t len = nth == 0 ? aux[0] : aux[1];
    ++nth;
    if (len > 0xFFFFu) { atomicOr(&P.st->err, kErrKeyTooLong); len = 0xFFFFu; }
    qpos[k] = static_cast<uint64_t>(p0 + j + 9);
    qlen[k] = len;
    ++k;
  }
  qn += tot;
  if (qn >= 32) ii_drain(P, oc, outh, qn);
}

__device__ __forceinline__ void ii_map_loop(const Params& P, uint8_t* smem, OutCtl* oc, uint32_t& qn) {
  constexpr int W = kII;
  constexpr int kStages = Cfg<W>::kStages;
  uint64_t* empty = reinterpret_cast<uint64_t*>(smem + Layout<W>::empty);
  uint64_t* ready = reinterpret_cast<uint64_t*>(smem + Layout<W>::ready);
  uint8_t* outh = smem + Layout<W>::out;
  uint32_t have_it = ~0u;
  long long t = 0, sbase = 0, hi = 0, stg_hi = 0;
  // two windows per fetch with dynamic tiles (the end marker sits at two iterations), as wc_map_loop
  constexpr uint32_t kPW = (BMR_II_PAIRWIN && BMR_DYN_TILES) ? 2u : 1u;
  static_assert(kNWin % kPW == 0, "window pairs must not straddle tiles");
  for (;;) {
    const uint32_t g = lane0_atom_add_shared(&oc->win_next, kPW);
    const uint32_t it = g / kNWin, w = g % kNWin;
    const uint32_t s = it % kStages;
    if (it != have_it) {
      map_wait(P, ready + s, (it / kStages) & 1u, kReadyWaitNs);
      const StageHdr* hd = reinterpret_cast<const StageHdr*>(smem + Layout<W>::hdr + s * 128);
      t = hd->t;
      sbase = hd->sbase;
      hi = hd->hi;
      stg_hi = hd->stg_hi;
      have_it = it;
    }
    if (t == -1) break;   // (-2: a skip stage, no windows)
    const TileView tv{smem + Layout<W>::bytes + s * kStageBytes,
                      reinterpret_cast<const uint32_t*>(smem + Layout<W>::bits + s * Cfg<W>::kBits), sbase, stg_hi, 0,
                      0};
#pragma unroll 1
    for (uint32_t q = 0; q < kPW; ++q) {
      const long long wp = sbase + kLead + static_cast<long long>(w + q) * kWin;
      if (wp < hi) ii_window(P, oc, outh, tv, wp, qn);   // warp-uniform
    }
    __syncwarp();
    if (kPW == 1) lane0_mbar_arrive(&empty[s]);
    else if ((threadIdx.x & 31) == 0) mbar_arrive_cnt(&empty[s], kPW);
  }
}

template <int W>
__device__ void emit_text_chunk(const Params& P, OutCtl* oc, uint8_t* outh, const TileView& tv,
                                long long p0, long long i0, bool live, uint32_t& qn) {
  using F = PairFmt<W>;
  const long long N = bd_nbytes();
  uint32_t x[8];
  uint32_t vm = 0, R = 0;
  if (live) {
    if (P.so) {   // SO / G ablation: the 32 bytes straight from global memory (rec + p0 is 16-B aligned)
      if (p0 >= 0 && p0 + 32 <= N) {
        const uint4 c0 = __ldg(reinterpret_cast<const uint4*>(P.rec + p0));
        const uint4 c1 = __ldg(reinterpret_cast<const uint4*>(P.rec + p0 + 16));
        x[0] = c0.x; x[1] = c0.y; x[2] = c0.z; x[3] = c0.w;
        x[4] = c1.x; x[5] = c1.y; x[6] = c1.z; x[7] = c1.w;
      } else {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          uint32_t w = 0;
          for (int b = 0; b < 4; ++b) {
            const long long q = p0 + 4 * i + b;
            if (q >= 0 && q < N) w |= static_cast<uint32_t>(P.rec[q]) << (8 * b);
          }
          x[i] = w;
        }
      }
    } else {
      const uint4 c0 = *reinterpret_cast<const uint4*>(tv.sb + i0);
      const uint4 c1 = *reinterpret_cast<const uint4*>(tv.sb + i0 + 16);
      x[0] = c0.x; x[1] = c0.y; x[2] = c0.z; x[3] = c0.w;
      x[4] = c1.x; x[5] = c1.y; x[6] = c1.z; x[7] = c1.w;
    }
    vm = range_mask32(p0, 0, N);
    if constexpr (!Cfg<W>::kLazyDir) R = bits32(tv.bm, i0);
  } else {
#pragma unroll
    for (int i = 0; i < 8; ++i) x[i] = 0;
  }
  uint32_t emit_mask = 0;       // bit j: an emission anchored at p0 + j
  uint32_t aux[2] = {0, 0};     // II: closing-quote distance for up to two markers
  uint32_t wm = 0, nb = 0;
  const uint32_t lane = threadIdx.x & 31;
  if constexpr (W == kWC) {
    // word bytes of this chunk; the next chunk's mask comes from lane + 1 (same window), so each
    // lane classifies only its own 16 bytes.  Lane 31 classifies the 16 bytes after the window
    // itself (already loaded: x[4..7]); only words running past the 32 loaded bytes take the slow
    // path.
    uint32_t w16 = 0;
    if (live) {
#pragma unroll
      for (int i = 0; i < 4; ++i) w16 |= word_mask4(x[i]) << (4 * i);
    }
    uint32_t nxt = __shfl_down_sync(kFull, w16, 1);
    const uint32_t prv = __shfl_up_sync(kFull, w16, 1);
    if (live) {
      if (lane == 31) {
        nxt = 0;
#pragma unroll
        for (int i = 0; i < 4; ++i) nxt |= word_mask4(x[4 + i]) << (4 * i);
      }
      const uint32_t known = 0xFFFFFFFFu;
      wm = (w16 | (nxt << 16)) & vm;
      uint32_t prevw;
      if (lane == 0) prevw = (p0 - 1 >= 0 && p0 - 1 < N && is_word_byte(P.so ? P.rec[p0 - 1] : tv.sb[i0 - 1])) ? 1u : 0u;
      else prevw = (prv >> 15) & 1u;
      nb = (~wm | R) & known;                                  // a word cannot continue here
      emit_mask = wm & 0xFFFFu & ~(((wm << 1) | prevw) & ~R);  // word starts (C-2 WC)
    }
  } else if constexpr (W == kSM) {
    if (live) {
      const uint32_t b0 = (P.pat[0] & 0xFFu) * 0x01010101u;
      // any byte equal to the pattern's first byte?  (exact has-zero-byte test on x ^ b0: the
      // first byte is rare in text, so the per-byte mask is computed only when one exists)
      uint32_t any = 0;
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const uint32_t t = x[i] ^ b0;
        any |= (t - 0x01010101u) & ~t & 0x80808080u;
      }
      uint32_t cand = 0;
      if (any) {
#pragma unroll
        for (int i = 0; i < 4; ++i) cand |= eq_mask4(x[i], b0) << (4 * i);
        cand &= vm & 0xFFFFu;
      }
      while (cand) {
        const uint32_t j = __ffs(cand) - 1;
        cand &= cand - 1;
        if (p0 + j + 16 > N) continue;
        uint32_t w[4];
        window16(x, j, w);
        if (w[0] != P.pat[0] || w[1] != P.pat[1] || w[2] != P.pat[2] || w[3] != P.pat[3]) continue;
        // the match must lie inside one record: no record start in (p, p + 15] (lazy directory)
        unsigned long long lo = tv.ra, hi = tv.rb;
        const unsigned long long p = static_cast<unsigned long long>(p0 + j);
        while (lo < hi) {                                   // first record start > p in the slice
          const unsigned long long mid = (lo + hi) >> 1;
          if (P.off[mid] > p) hi = mid; else lo = mid + 1;
        }
        if (lo < tv.rb && P.off[lo] <= p + 15) continue;   // (offsets[rb] lies beyond the halo)
        emit_mask |= 1u << j;
      }
    }
  } else if constexpr (W == kII) {
    // markers of this lane's chunk, then the closing quote of each marker by a warp-cooperative
    // search: every lane publishes its 16-bit "stop" mask (a '"' or a record start) and a marker
    // finds the first stop at or after its URL start with two shuffles (the URL ends at the first
    // '"' unless the record ends first, C-3 #9); only URLs leaving the 512-B window scan onwards.
    // '<' is rare in the text outside markers: a window without one in any lane emits nothing
    // (exact has-byte test, 3 ALU ops per 4 bytes, before the per-byte masks)
    {
      uint32_t a = 0;
      if (live) {
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const uint32_t t = x[i] ^ 0x3C3C3C3Cu;
          a |= (t - 0x01010101u) & ~t;
        }
      }
      if (!__any_sync(kFull, (a & 0x80808080u) != 0)) return;
    }
    uint32_t mk = 0, st16 = 0;
    if (live) {
      uint32_t cand = 0, qm = 0;
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        cand |= eq_mask4(x[i], 0x3C3C3C3Cu) << (4 * i);  // '<'
        qm |= eq_mask4(x[i], 0x22222222u) << (4 * i);    // '"'
      }
      cand &= vm & 0xFFFFu;
      st16 = ((qm & vm) | R) & 0xFFFFu;
      while (cand) {
        const uint32_t j = __ffs(cand) - 1;
        cand &= cand - 1;
        if (p0 + j + 9 > N) continue;
        if ((R >> (j + 1)) & 0xFFu) continue;               // marker inside one record
        uint32_t w[4];
        window16(x, j, w);
        // "<a href=\"" little-endian: 3C 61 20 68 | 72 65 66 3D | 22
        if (w[0] != 0x6820613Cu || w[1] != 0x3D666572u || (w[2] & 0xFFu) != 0x22u) continue;
        mk |= 1u << j;
      }
    }
    const uint32_t lanes_st = __ballot_sync(kFull, st16 != 0);
    const uint32_t r16 = R & 0xFFFFu;
    const long long wp = p0 - static_cast<long long>(lane) * 16;   // window start
    int nm = 0;
    for (int mi = 0; mi < 2; ++mi) {          // a 9-byte marker: at most two start in 16 bytes
      if (!__any_sync(kFull, mk != 0)) break;
      const bool has = mk != 0;
      const uint32_t j = has ? static_cast<uint32_t>(__ffs(mk) - 1) : 0u;
      if (has) mk &= mk - 1;
      const uint32_t a = lane * 16 + j + 9;   // window offset of the URL start
      const uint32_t T = min(a >> 4, 31u);
      const uint32_t sT = __shfl_sync(kFull, st16, T), rT = __shfl_sync(kFull, r16, T);
      const uint32_t cT = a < static_cast<uint32_t>(kWin) ? (sT >> (a & 15u)) << (a & 15u) : 0u;
      const uint32_t later = T < 31 ? (lanes_st & ~((2u << T) - 1u)) : 0u;
      const uint32_t F = later ? static_cast<uint32_t>(__ffs(later) - 1) : 31u;
      const uint32_t sF = __shfl_sync(kFull, st16, F), rF = __shfl_sync(kFull, r16, F);
      if (!has) continue;
      const long long q0 = p0 + j + 9;
      long long q;
      if (cT) {
        const uint32_t b = __ffs(cT) - 1;
        q = ((rT >> b) & 1u) ? -1 : wp + T * 16 + b;     // record ends first -> unclosed
      } else if (later && a < static_cast<uint32_t>(kWin)) {
        const uint32_t b = __ffs(sF) - 1;
        q = ((rF >> b) & 1u) ? -1 : wp + F * 16 + b;
      } else {                                           // no stop in the window: scan onwards
        q = find_quote(P, tv, max(q0, wp + kWin), p0 + j);
      }
      if (q > q0 && nm < 2) {
        aux[nm++] = static_cast<uint32_t>(q - q0);
        emit_mask |= 1u << j;
      }
    }
  }
  if constexpr (W == kWC) {
    emit_wc(P, oc, outh, tv, x, p0, emit_mask, nb);
    return;
  }
  if constexpr (W == kII) {
    if (!P.si || P.xranks) {   // queue the URLs (drained lane-parallel, see ii_drain)
      const uint32_t cnt = __popc(emit_mask);   // <= 2 markers start in 16 bytes
      const uint32_t incl = warp_inclusive_add(cnt);
      const uint32_t tot = __shfl_sync(kFull, incl, 31);
      if (tot == 0) return;
      if (qn + tot > 64) ii_drain(P, oc, outh, qn);
      uint64_t* qpos = ii_qpos(outh);
      uint32_t* qlen = reinterpret_cast<uint32_t*>(qpos + 64);
      uint32_t k = qn + incl - cnt;
      int nth = 0;
      for (uint32_t m = emit_mask; m; m &= m - 1) {
        const uint32_t j = __ffs(m) - 1;
        uint32_t len = nth == 0 ? aux[0] : aux[1];
        ++nth;
        if (len > 0xFFFFu) { atomicOr(&P.st->err, kErrKeyTooLong); len = 0xFFFFu; }
        qpos[k] = static_cast<uint64_t>(p0 + j + 9);
        qlen[k] = len;
        ++k;
      }
      qn += tot;
      if (qn >= 32) ii_drain(P, oc, outh, qn);
      return;
    }
  }
  // ---- reserve one warp result, then lane-major emission rounds
  const uint32_t total = __reduce_add_sync(kFull, __popc(emit_mask));
  if (total == 0) return;
  Slot slot{0, 0};
  uint64_t* sh;
  uint64_t* sk;
  uint8_t* sv;
  uint64_t k, cap = ~0ULL;
  if (P.si) {   // SI / G ablation: one global atomic per warp result, lanes write HBM directly
    unsigned long long gb = 0;
    if (lane == 0) gb = atomicAdd(&P.st->pair_cursor, static_cast<unsigned long long>(total));
    k = __shfl_sync(kFull, gb, 0);
    sh = P.oh;
    sk = P.okref;
    sv = P.ov;
    cap = P.cap_pairs;
  } else {
    slot = reserve<W>(P, oc, outh, total, P.out_cap);
    uint8_t* half = outh + slot.half * Cfg<W>::kOutHalf;
    sh = reinterpret_cast<uint64_t*>(half);
    sk = sh + F::kCap;
    sv = half + F::kCap * (F::kKref ? 16 : 8);
    k = slot.base;
  }
  uint32_t m_left = emit_mask;
  int nth = 0;
  while (__any_sync(kFull, m_left != 0)) {
    const bool act = m_left != 0;
    const uint32_t m = __ballot_sync(kFull, act);
    if (act) {
      const uint32_t j = __ffs(m_left) - 1;
      m_left &= m_left - 1;
      const uint64_t idx = k + __popc(m & lanemask_lt());
      const long long p = p0 + j;
      if constexpr (W == kSM) {
        uint64_t key = static_cast<uint64_t>(p);
        if (P.sm_lines) {   // the paper's per-line output (L125): the match's record start instead
          unsigned long long lo = tv.ra, hi = tv.rb;
          while (lo < hi) {
            const unsigned long long mid = (lo + hi) >> 1;
            if (P.off[mid] > key) hi = mid; else lo = mid + 1;
          }
          key = P.off[lo - 1];   // lo >= 1: offsets[0] = 0 <= p
        }
        if (idx < cap) sh[idx] = bd_gbase() + key;
      } else if constexpr (W == kII) {
        uint32_t len = nth == 0 ? aux[0] : aux[1];
        ++nth;
        const long long q0 = p + 9;
        if (len > 0xFFFFu) { atomicOr(&P.st->err, kErrKeyTooLong); len = 0xFFFFu; }
        const uint64_t key = key_at(P, tv, q0, len);
        if (idx < cap) {
          sh[idx] = key;
          sk[idx] = (reinterpret_cast<uint64_t>(P.rec + q0) << 16) | len;
          reinterpret_cast<uint64_t*>(sv)[idx] = bd_gbase() + static_cast<uint64_t>(q0);
        }
      }
    }
    k += __popc(m);
  }
  if (!P.si) commit(oc, slot, total);
}

// StringMatch map warps (all memory modes): super-windows of kSmSub 512-B windows, handed out
// from a shared counter (BMR_SM_DYN) or in a static round-robin.  The
// pattern's first byte is rare in text, so each lane first runs the exact has-byte test over its
// kSmSub 16-B chunks (one LDS.128 + 3 ALU ops per 4 bytes); only a 512-B window in which some
// lane saw the byte runs the full per-byte path (emit_text_chunk: candidate mask, 16-byte
// compare, record check, emission).  The per-window bookkeeping (window index, stage header,
// range masks, the warp reduction of the emission count) is paid once per 2 KiB instead of per
// 512 B (ncu, C2 round 1: it was ~80% of the Map's instructions).
constexpr int kSmSub = BMR_SM_SUB, kNSup = kNWin / kSmSub;
template <bool kSO>
__device__ __noinline__ void sm_fast_loop(const Params& P, uint8_t* smem, OutCtl* oc) {
  constexpr int W = kSM;
  constexpr int kStages = Cfg<W>::kStages;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + Layout<W>::full);
  uint64_t* empty = reinterpret_cast<uint64_t*>(smem + Layout<W>::empty);
  uint8_t* outh = smem + Layout<W>::out;
  const uint32_t b0 = (P.pat[0] & 0xFFu) * 0x01010101u;
  const long long N = bd_nbytes();
  // this CTA's iterations (as producer_loop): a warp's super-windows are nmap apart and may skip
  // whole tiles (kNSup < nmap), so it must stop at T itself rather than wait for the end marker
  const uint64_t G = gridDim.x;
  const uint32_t T = blockIdx.x < bd_ntiles() ? static_cast<uint32_t>((bd_ntiles() - blockIdx.x + G - 1) / G) : 0u;
  uint32_t have_it = ~0u;
  StageHdr hd{};
  for (uint32_t kseq = 0;; ++kseq) {
    uint32_t g;
    if (BMR_SM_DYN) {   // super-windows from a shared counter: a warp busy with a match's record
      uint32_t gg = 0;  // check does not hold up the super-windows it would own in static order
      if (lane == 0) gg = atomicAdd(&oc->win_next, 1u);
      g = __shfl_sync(kFull, gg, 0);
    } else {
      g = warp + kseq * static_cast<uint32_t>(nmap<W>());
    }
    const uint32_t it = g / kNSup, sw = g % kNSup;
    if (it >= T) break;
    const uint32_t s = it % kStages, ph = (it / kStages) & 1u;
    if (it != have_it) {
      // suspended wait (try_wait with a time hint): spinning map warps took 30% of the issued
      // instructions (ncu C2), competing with the producers for issue slots
      if (BMR_SM_WAIT_NS) mbar_wait_idle(&full[s], ph, BMR_SM_WAIT_NS);
      else mbar_wait(&full[s], ph);
      hd = *reinterpret_cast<const StageHdr*>(smem + Layout<W>::hdr + s * 128);
      have_it = it;
    }
    if (hd.t < 0) break;
    const uint8_t* sb = smem + Layout<W>::bytes + s * kStageBytes;
    const long long wp0 = hd.chunk0 + static_cast<long long>(sw) * (kSmSub * kWin);
    // has-byte test (exact: (t - 0x01..) & ~t & 0x80.. is non-zero iff t has a zero byte); bytes
    // outside [0, N) only cause a spurious slow-path visit, which masks them exactly
    uint32_t anym = 0;
    const uint8_t* c0 = sb + (wp0 - hd.sbase) + lane * 16;
    // SO / G ablation (MR_FLAG_NO_SMEM_IN): the same loads from global memory (the stage is empty)
    auto ld16 = [&](long long q, const uint8_t* sp) -> uint4 {
      if constexpr (!kSO) return *reinterpret_cast<const uint4*>(sp);
      if (q >= 0 && q + 16 <= N) return __ldg(reinterpret_cast<const uint4*>(P.rec + q));   // rec + q: 16-B aligned
      uint32_t w[4] = {0, 0, 0, 0};
      for (int b = 0; b < 16; ++b)
        if (q + b >= 0 && q + b < N) w[b >> 2] |= static_cast<uint32_t>(P.rec[q + b]) << (8 * (b & 3));
      return make_uint4(w[0], w[1], w[2], w[3]);
    };
#pragma unroll
    for (int k = 0; k < kSmSub; ++k) {
      const uint4 c = ld16(wp0 + k * kWin + lane * 16, c0 + k * kWin);
      const uint32_t t0 = c.x ^ b0, t1 = c.y ^ b0, t2 = c.z ^ b0, t3 = c.w ^ b0;
      const uint32_t a = ((t0 - 0x01010101u) & ~t0) | ((t1 - 0x01010101u) & ~t1) | ((t2 - 0x01010101u) & ~t2) |
                         ((t3 - 0x01010101u) & ~t3);
      anym |= ((a & 0x80808080u) ? 1u : 0u) << k;
    }
    uint32_t need = 0;
#pragma unroll
    for (int k = 0; k < kSmSub; ++k) need |= (__any_sync(kFull, (anym >> k) & 1u) ? 1u : 0u) << k;
    // Rare path, part 1 (stage reads only): 16-byte compares at the first-byte candidates of the
    // windows that have any; a lane keeps the global positions of its (<= 2 per 16 B) matches.
    uint64_t mp[2];
    uint32_t nm = 0;
    while (need) {                                     // warp-uniform
      const int k = __ffs(need) - 1;
      need &= need - 1;
      const long long p0 = wp0 + static_cast<long long>(k) * kWin + lane * 16;
      if (!((anym >> k) & 1u)) continue;
      const uint8_t* c = c0 + k * kWin;
      const uint4 u0 = ld16(p0, c), u1 = ld16(p0 + 16, c + 16);
      const uint32_t x[8] = {u0.x, u0.y, u0.z, u0.w, u1.x, u1.y, u1.z, u1.w};
      uint32_t cand = 0;
#pragma unroll
      for (int i = 0; i < 4; ++i) cand |= eq_mask4(x[i], b0) << (4 * i);
      cand &= range_mask32(p0, 0, min(N, hd.hi) ) & 0xFFFFu;   // own bytes of this tile, inside the input
      while (cand) {
        const uint32_t j = __ffs(cand) - 1;
        cand &= cand - 1;
        if (p0 + j + 16 > N) continue;
        uint32_t w[4];
        window16(x, j, w);
        if (w[0] != P.pat[0] || w[1] != P.pat[1] || w[2] != P.pat[2] || w[3] != P.pat[3]) continue;
        if (nm < 2) mp[nm] = static_cast<uint64_t>(p0 + j);
        ++nm;   // (16-byte pattern whose first byte recurs: > 2 matches per 16 B -> fallback below)
      }
    }
    const bool over = __any_sync(kFull, nm > 2);
    const StageHdr h = hd;
    // the stage is no longer read: release it before the global-memory record checks, so a
    // match never holds up the stage ring (ncu C2: the per-lane binary search over global
    // offsets stalled the in-order stage release)
    if (!over) {
      __syncwarp();
      if (lane == 0) mbar_arrive_cnt(&empty[s], kSmSub);
    } else {
      // rare self-overlapping pattern (e.g. a run of one byte): the general per-window path
      for (int k = 0; k < kSmSub; ++k) {
        const long long wp = wp0 + static_cast<long long>(k) * kWin;
        if (wp >= h.hi || !__any_sync(kFull, (anym >> k) & 1u)) continue;
        TileView tv{sb, nullptr, h.sbase, h.stg_hi, h.ra, h.rb};
        const long long p0 = wp + lane * 16;
        uint32_t qn_unused = 0;
        emit_text_chunk<W>(P, oc, outh, tv, p0, p0 - h.sbase, (p0 + 16 > 0) && (p0 < N), qn_unused);
      }
      __syncwarp();
      if (lane == 0) mbar_arrive_cnt(&empty[s], kSmSub);
      continue;
    }
    // Rare path, part 2: each match, one at a time with the whole warp: the first record start
    // after p by a two-round warp-cooperative search of offsets[ra, rb) (32 samples, then <= 32
    // entries), then emission of p (or its record start, MR_FLAG_SM_LINES) when no record start
    // lies in (p, p + 15] (C-3 #3: a match lies inside one record).
    for (;;) {
      const uint32_t bal = __ballot_sync(kFull, nm > 0);
      if (!bal) break;
      const uint32_t src = __ffs(bal) - 1;
      const unsigned long long p = __shfl_sync(kFull, static_cast<unsigned long long>(mp[0]), src);
      if (lane == src) { mp[0] = mp[1]; --nm; }
      unsigned long long lo = h.ra, hi = h.rb;       // first i in [lo, hi) with off[i] > p (hi if none)
      while (hi - lo > 32) {
        const unsigned long long step = (hi - lo + 31) / 32;
        const unsigned long long i = lo + lane * step;
        const uint32_t gt = __ballot_sync(kFull, i >= hi || P.off[i] > p);
        if (gt == 0) { lo = lo + 31 * step + 1; continue; }
        const uint32_t f = __ffs(gt) - 1;
        if (f == 0) { hi = lo; break; }
        hi = min(hi, lo + f * step);
        lo = lo + (f - 1) * step + 1;
      }
      if (hi > lo) {
        const unsigned long long i = lo + lane;
        const uint32_t gt = __ballot_sync(kFull, i >= hi || P.off[i] > p);
        hi = gt ? lo + (__ffs(gt) - 1) : hi;
      }
      const unsigned long long u = hi;               // (offsets[rb] lies beyond the halo)
      const bool ok = !(u < h.rb && P.off[u] <= p + 15);
      if (!ok) continue;
      const uint64_t key = bd_gbase() + (P.sm_lines ? P.off[u - 1] : p);   // u >= 1: offsets[0] = 0 <= p
      if (P.si) {
        if (lane == 0) {
          const unsigned long long g = atomicAdd(&P.st->pair_cursor, 1ULL);
          if (g < P.cap_pairs) P.oh[g] = key;
        }
      } else {
        const Slot slot = reserve<W>(P, oc, outh, 1u, P.out_cap, true);
        if (slot.half == kSpill) {   // ring congested: straight to HBM (SM flushes need no alignment)
          if (lane == 0) {
            const unsigned long long g = atomicAdd(&P.st->pair_cursor, 1ULL);
            if (g < P.cap_pairs) P.oh[g] = key;
          }
          continue;
        }
        if (lane == 0) reinterpret_cast<uint64_t*>(outh + slot.half * Cfg<W>::kOutHalf)[slot.base] = key;
        commit(oc, slot, 1u);
      }
    }
  }
}

// KMeans f-1 combiner step of one warp (one point per valid lane, cluster `best`): a point of the
// lane's own cluster (cluster == lane; the lane holds the fp64 accumulators kacc of clusters lane
// and lane + 32) is added to the lane's fp32 partial of it, folded into kacc every 32 points
// (<= 32 values per fp32 partial, as in the sorted Reduce: DESIGN.md reading 5); the other points
// are summed into per-warp fp32 SMEM partials of this tile, which are folded into their owner
// lanes' kacc right away.  Lanes with the same cluster form a match group and add in rank order,
// one member per round (plain read-modify-write: no two lanes of a round share a cluster) —
// shared-memory fp32 atomics are CAS loops on sm_100a (ATOMS.CAST.SPIN, ncu round 2: 19% of the
// KM Map's instructions, 38% of its stall samples).
__device__ __forceinline__ void km_flush_partial(double (&acc)[8], unsigned long long& cnt, float (&pa)[8],
                                                 uint32_t& pn) {
  cnt += pn;
#pragma unroll
  for (int t = 0; t < 8; ++t) {
    acc[t] += static_cast<double>(pa[t]);
    pa[t] = 0.0f;
  }
  pn = 0;
}
__device__ __forceinline__ void km_combine(uint8_t* smem, uint32_t warp, uint32_t lane, bool valid, uint32_t best,
                                           const float (&x)[8], uint32_t k, double (&kacc)[kKmCombMax / 32][8],
                                           unsigned long long (&kcnt)[kKmCombMax / 32], float (&pacc)[8],
                                           uint32_t& pn) {
  const bool own = valid && best == lane;
  if (own) {
#pragma unroll
    for (int t = 0; t < 8; ++t) pacc[t] += x[t];
    if (++pn == 32u) km_flush_partial(kacc[0], kcnt[0], pacc, pn);
  }
  const bool other = valid && !own;
  if (!__any_sync(kFull, other)) return;
  float* wacc = reinterpret_cast<float*>(smem + Layout<kKM>::kmacc) + warp * (kKmCombMax * 8);
  uint32_t* wcnt = reinterpret_cast<uint32_t*>(smem + Layout<kKM>::kmacc + kKmWaccBytes) + warp * kKmCombMax;
  const uint32_t grp = __match_any_sync(kFull, other ? best : 0xFFFFFFFFu);
  const uint32_t rank = __popc(grp & lanemask_lt());
  const uint32_t rounds = __reduce_max_sync(kFull, other ? static_cast<uint32_t>(__popc(grp)) : 0u);
  for (uint32_t r = 0; r < rounds; ++r) {
    if (other && rank == r) {
#pragma unroll
      for (int t = 0; t < 8; ++t) wacc[t * kKmCombMax + best] += x[t];   // [dim][cluster]: no bank conflicts
      wcnt[best] += 1u;
    }
    __syncwarp();
  }
#pragma unroll
  for (int q = 0; q < kKmCombMax / 32; ++q) {
    const uint32_t c = lane + 32 * q;
    if (c < k) {
      const uint32_t nc = wcnt[c];
      if (nc) {
        wcnt[c] = 0;
        kcnt[q] += nc;
#pragma unroll
        for (int t = 0; t < 8; ++t) {
          kacc[q][t] += static_cast<double>(wacc[t * kKmCombMax + c]);
          wacc[t * kKmCombMax + c] = 0.0f;
        }
      }
    }
  }
  __syncwarp();
}

// KMeans full scan of one point (reading 4): fp32 RN chain d = fma(x_t - c_t, x_t - c_t, d) over
// t = 0..7, ties -> lowest j.  Two centroids per instruction with packed FADD2/FFMA2 (each lane of
// the pair performs exactly the scalar RN operations, so the result is bit-identical); cent is
// the pair layout (centroids 2p, 2p+1 interleaved per coordinate), an odd last centroid unpaired.
__device__ __forceinline__ uint32_t km_scan(const float (&x)[8], const float* cent, uint32_t k) {
  uint32_t best = 0;
  float bd = 0.0f;
  uint64_t X[8];
#pragma unroll
  for (int t = 0; t < 8; ++t) X[t] = f2pack(x[t], x[t]);
  const uint32_t kp = k & ~1u;
  bool first = true;
#pragma unroll kKmUnroll
  for (uint32_t j = 0; j < kp; j += 2) {
    const ulonglong2* cp = reinterpret_cast<const ulonglong2*>(cent + j * 8);   // pair layout
    const ulonglong2 q0 = cp[0], q1 = cp[1], q2 = cp[2], q3 = cp[3];
    const uint64_t C[8] = {q0.x, q0.y, q1.x, q1.y, q2.x, q2.y, q3.x, q3.y};
    uint64_t D = 0;
#pragma unroll
    for (int t = 0; t < 8; ++t) {
      const uint64_t E = f2sub(X[t], C[t]);
      D = f2fma(E, E, D);
    }
    float d0, d1;
    f2unpack(D, d0, d1);
    if (first || d0 < bd) { bd = d0; best = j; }
    first = false;
    if (d1 < bd) { bd = d1; best = j + 1; }
  }
  if (k & 1u) {
    const uint32_t j = k - 1;
    const float* c = cent + j * 8;   // last centroid stored unpaired
    float d = 0.0f, e;
#pragma unroll
    for (int t = 0; t < 8; ++t) { e = __fsub_rn(x[t], c[t]); d = __fmaf_rn(e, e, d); }
    if (first || d < bd) { bd = d; best = j; }
  }
  return best;
}

// KMeans Map, bound-test instantiation with the combiner in SIO mode (the default C3 path): one
// point per map lane per tile; the lane's previous winner g first — if 4 d_g (1 + 1e-5) < s2[g]
// the point is g's (reading 12), else the full scan.  No ablation branches in the loop.
__device__ void km_bound_loop(const Params& P, uint8_t* smem, double (&kacc)[kKmCombMax / 32][8],
                              unsigned long long (&kcnt)[kKmCombMax / 32], float (&pacc)[8], uint32_t& pn,
                              uint32_t guess) {
  constexpr int W = kKM;
  constexpr int kStages = Cfg<W>::kStages;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31, tid = threadIdx.x;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + Layout<W>::full);
  uint64_t* empty = reinterpret_cast<uint64_t*>(smem + Layout<W>::empty);
  const float* cent = reinterpret_cast<const float*>(smem + Layout<W>::cent);
  const uint32_t k = P.k;
  const float* crow = cent + k * 8;
  const float* s2 = cent + k * 16;
  const uint32_t phase16 = static_cast<uint32_t>(reinterpret_cast<uintptr_t>(P.rec) & 15u);
  unsigned long long scanned = 0;
  for (uint32_t it = 0;; ++it) {
    const uint32_t s = it % kStages;
    mbar_wait(&full[s], (it / kStages) & 1u);
    const StageHdr* hd = reinterpret_cast<const StageHdr*>(smem + Layout<W>::hdr + s * 128);
    const long long t = hd->t;
    if (t < 0) break;
    const long long lo = hd->lo, hi = hd->hi;
    const bool valid = lo + static_cast<long long>(tid) < hi;
    // stage byte offset of the first point: the source's 16-B phase (points are 32 B)
    const float4* pt = reinterpret_cast<const float4*>(smem + Layout<W>::bytes + s * kStageBytes +
                                                       ((phase16 + static_cast<uint32_t>(lo) * 32u) & 15u) + tid * 32u);
    float x[8];
    uint32_t best = guess;
    bool scan = false;
    if (valid) {
      const float4 a = pt[0], b = pt[1];
      x[0] = a.x; x[1] = a.y; x[2] = a.z; x[3] = a.w; x[4] = b.x; x[5] = b.y; x[6] = b.z; x[7] = b.w;
      const float4* cg = reinterpret_cast<const float4*>(crow + guess * 8);
      const float4 g0 = cg[0], g1 = cg[1];
      const float c[8] = {g0.x, g0.y, g0.z, g0.w, g1.x, g1.y, g1.z, g1.w};
      float d = 0.0f;
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        const float e = __fsub_rn(x[q], c[q]);
        d = __fmaf_rn(e, e, d);
      }
      scan = !(d * kKmBoundFactor < s2[guess]);
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[s]);   // x is in registers: the stage can go
    if (scan) best = km_scan(x, cent, k);
    scanned += __popc(__ballot_sync(kFull, scan));
    if (valid) guess = best;
    km_combine(smem, warp, lane, valid, best, x, k, kacc, kcnt, pacc, pn);
  }
  if (lane == 0 && scanned) atomicAdd(&P.st->km_scanned, scanned);
}

// V: 1 = the WordCount table-mode instantiation (wc_window_tab) / the KMeans bound-test
// instantiation, kernels of their own so that the two paths do not share one register allocation
template <int W, int V>
__device__ void map_loop(const Params& P, uint8_t* smem, OutCtl* oc) {
  constexpr int kStages = Cfg<W>::kStages;
  using F = PairFmt<W>;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t tid = threadIdx.x;  // 0 .. kNMap*32-1
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + Layout<W>::full);
  uint64_t* empty = reinterpret_cast<uint64_t*>(smem + Layout<W>::empty);
  uint8_t* outh = smem + Layout<W>::out;
  const float* cent = reinterpret_cast<const float*>(smem + Layout<W>::cent);
  // Text: windows are handed out dynamically (one shared atomic per 512-B window, in tile order),
  // so a warp that drew cheap windows takes the next one instead of idling until the slowest
  // warp of the tile is done; a stage is released after all kNWin of its windows (empty[s]
  // counts windows).  KM: one point per map lane, kNMap arrivals per stage.
  // KM combiner: lane-owned fp64 sums / counts of clusters lane, lane + 32 (k <= kKmCombMax)
  double kacc[kKmCombMax / 32][8];
  unsigned long long kcnt[kKmCombMax / 32];
#pragma unroll
  for (int q = 0; q < kKmCombMax / 32; ++q) {
    kcnt[q] = 0;
#pragma unroll
    for (int t = 0; t < 8; ++t) kacc[q][t] = 0.0;
  }
  // (P.dyn == 0: static order, map warp w takes windows w, w + nmap, w + 2 nmap, ... of the CTA's
  // window sequence)
  uint32_t kseq = 0, have_it = ~0u;
  uint32_t km_guess = W == kKM && P.k ? lane % P.k : 0u;   // KM: this lane's previous winner (bound test)
  float pacc[8];   // KM: fp32 partial of the lane's own cluster (km_combine)
  uint32_t pn = 0;
#pragma unroll
  for (int t = 0; t < 8; ++t) pacc[t] = 0.0f;
  uint32_t qn = 0;   // II: queued URLs of this warp (ii_drain)
  StageHdr hd{};
  bool fast = W == kSM && !P.dyn;
  if constexpr (W == kSM) {
    if (fast) {   // (SO / G ablation: a separate instantiation, no per-load mode test on the SIO path)
      if (P.so) sm_fast_loop<true>(P, smem, oc);
      else sm_fast_loop<false>(P, smem, oc);
    }
  }
  if constexpr (W == kWC) {
    fast = !P.so && !P.si && P.wc_bal && P.dyn && P.wc_fast;
    if (fast) {
      if constexpr (V == 1) wc_map_loop<1>(P, smem, oc);
      else if constexpr (V == 2) wc_map_loop<2>(P, smem, oc);
      else wc_map_loop<0>(P, smem, oc);
    }
  }
  if constexpr (W == kII) {
    fast = !P.so && !P.si && P.dyn && P.wc_fast;
    if (fast) ii_map_loop(P, smem, oc, qn);
  }
  if constexpr (W == kKM && V == 1) {
    fast = P.comb && !P.so && !P.si;
    if (fast) km_bound_loop(P, smem, kacc, kcnt, pacc, pn, km_guess);
  }
  for (uint32_t it = 0; !fast; ++it) {
    uint32_t w = 0;
    if constexpr (W != kKM) {
      uint32_t g = 0;
      if (P.dyn) {
        if (lane == 0) g = atomicAdd(&oc->win_next, 1u);
        g = __shfl_sync(kFull, g, 0);
      } else {
        g = warp + kseq * static_cast<uint32_t>(nmap<W>());
        ++kseq;
      }
      it = g / kNWin;
      w = g % kNWin;
    }
    const uint32_t s = it % kStages, ph = (it / kStages) & 1u;
    if (it != have_it) {   // a warp's consecutive windows are mostly in one tile: wait + header once
      if constexpr (W == kKM || Cfg<W>::kLazyDir) mbar_wait(&full[s], ph);
      else map_wait(P, reinterpret_cast<uint64_t*>(smem + Layout<W>::ready) + s, ph, kReadyWaitNs);
      hd = *reinterpret_cast<const StageHdr*>(smem + Layout<W>::hdr + s * 128);
      have_it = it;
    }
    if (hd.t == -1) break;   // (-2: a skip stage, no windows)
    const uint8_t* sb = smem + Layout<W>::bytes + s * kStageBytes;
    if constexpr (W == kKM) {
      const uint64_t i = static_cast<uint64_t>(hd.lo) + tid;
      const bool valid = i < static_cast<uint64_t>(hd.hi);
      // stage byte offset of the first point: same 16-B phase as the source
      const uint8_t* pt = sb + ((reinterpret_cast<uintptr_t>(P.rec) + static_cast<uint64_t>(hd.lo) * 32) & 15u) +
                          static_cast<uint64_t>(tid) * 32;
      float x[8];
      uint32_t best = 0;
      bool scan = valid;
      if (V == 1 && valid) {   // the lane's previous winner first: bound test (kKmBoundMax)
        const float4* cg = reinterpret_cast<const float4*>(cent + P.k * 8 + km_guess * 8);
        const float4 a = P.so ? __ldg(reinterpret_cast<const float4*>(P.rec + i * 32)) : reinterpret_cast<const float4*>(pt)[0];
        const float4 b = P.so ? __ldg(reinterpret_cast<const float4*>(P.rec + i * 32) + 1) : reinterpret_cast<const float4*>(pt)[1];
        const float4 g0 = cg[0], g1 = cg[1];
        float d = 0.0f, e;
        e = __fsub_rn(a.x, g0.x); d = __fmaf_rn(e, e, d);
        e = __fsub_rn(a.y, g0.y); d = __fmaf_rn(e, e, d);
        e = __fsub_rn(a.z, g0.z); d = __fmaf_rn(e, e, d);
        e = __fsub_rn(a.w, g0.w); d = __fmaf_rn(e, e, d);
        e = __fsub_rn(b.x, g1.x); d = __fmaf_rn(e, e, d);
        e = __fsub_rn(b.y, g1.y); d = __fmaf_rn(e, e, d);
        e = __fsub_rn(b.z, g1.z); d = __fmaf_rn(e, e, d);
        e = __fsub_rn(b.w, g1.w); d = __fmaf_rn(e, e, d);
        if (d * kKmBoundFactor < cent[P.k * 16 + km_guess]) {
          best = km_guess;
          scan = false;
          x[0] = a.x; x[1] = a.y; x[2] = a.z; x[3] = a.w; x[4] = b.x; x[5] = b.y; x[6] = b.z; x[7] = b.w;
        }
      }
      if (scan) {
        const float4* src = P.so ? reinterpret_cast<const float4*>(P.rec + i * 32) : reinterpret_cast<const float4*>(pt);
        const float4 a = P.so ? __ldg(src) : src[0];
        const float4 b = P.so ? __ldg(src + 1) : src[1];
        x[0] = a.x; x[1] = a.y; x[2] = a.z; x[3] = a.w; x[4] = b.x; x[5] = b.y; x[6] = b.z; x[7] = b.w;
        best = km_scan(x, cent, P.k);   // C-2 KM (reading 4)
      }
      if (valid) km_guess = best;   // the next point of this lane starts from this winner
      const uint32_t m = __ballot_sync(kFull, valid);
      {
        const uint32_t ms = __ballot_sync(kFull, scan);
        if (lane == 0 && ms) atomicAdd(&P.st->km_scanned, static_cast<unsigned long long>(__popc(ms)));
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[s]);   // stage no longer read by this warp
      if (P.comb) {
        km_combine(smem, warp, lane, valid, best, x, P.k, kacc, kcnt, pacc, pn);
      } else if (m && P.si) {   // SI / G ablation: global append per warp result
        unsigned long long gb = 0;
        if (lane == 0) gb = atomicAdd(&P.st->pair_cursor, static_cast<unsigned long long>(__popc(m)));
        gb = __shfl_sync(kFull, gb, 0);
        const uint64_t o = gb + __popc(m & lanemask_lt());
        if (valid && o < P.cap_pairs) {
          P.oh[o] = best;
          float4* gv = reinterpret_cast<float4*>(P.ov + o * 32);
          gv[0] = make_float4(x[0], x[1], x[2], x[3]);
          gv[1] = make_float4(x[4], x[5], x[6], x[7]);
        }
      } else if (m) {
        const uint32_t total = __popc(m);
        const Slot slot = reserve<W>(P, oc, outh, total, P.out_cap, true);
        if (slot.half == kSpill) {   // ring congested: straight to HBM, padded to 4 pairs like a flush
          const uint32_t r = (total + 3u) & ~3u;
          unsigned long long gb = 0;
          if (lane == 0) {
            gb = atomicAdd(&P.st->pair_cursor, static_cast<unsigned long long>(r));
            if (r > total) atomicAdd(&P.st->pads, static_cast<unsigned long long>(r - total));
          }
          gb = __shfl_sync(kFull, gb, 0);
          const uint32_t rk = __popc(m & lanemask_lt());
          if (valid && gb + rk < P.cap_pairs) {
            P.oh[gb + rk] = best;
            float4* gv = reinterpret_cast<float4*>(P.ov + (gb + rk) * 32);
            gv[0] = make_float4(x[0], x[1], x[2], x[3]);
            gv[1] = make_float4(x[4], x[5], x[6], x[7]);
          }
          if (lane < r - total && gb + total + lane < P.cap_pairs) P.oh[gb + total + lane] = sentinel_key<W>(P);
        } else {
          if (valid) {
            const uint32_t idx = slot.base + __popc(m & lanemask_lt());
            uint8_t* half = outh + slot.half * Cfg<W>::kOutHalf;
            reinterpret_cast<uint64_t*>(half)[idx] = best;
            float4* sv = reinterpret_cast<float4*>(half + F::kCap * 8 + static_cast<size_t>(idx) * 32);
            sv[0] = make_float4(x[0], x[1], x[2], x[3]);
            sv[1] = make_float4(x[4], x[5], x[6], x[7]);
          }
          commit(oc, slot, total);
        }
      }
    } else {
      const uint32_t* bm = reinterpret_cast<const uint32_t*>(smem + Layout<W>::bits + s * Cfg<W>::kBits);
      // (SO: an empty stage makes every helper read global memory)
      TileView tv{sb, bm, hd.sbase, P.so ? hd.sbase : hd.stg_hi, hd.ra, hd.rb};
      const long long wp = hd.chunk0 + static_cast<long long>(w) * kWin;
      if (wp < hd.hi) {                               // warp-uniform
        const long long p0 = wp + lane * 16;
        const bool live = (p0 + 16 > 0) && (p0 < bd_nbytes());
        emit_text_chunk<W>(P, oc, outh, tv, p0, p0 - hd.sbase, live, qn);
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[s]);
    }
  }
  if constexpr (W == kKM) {
    if (P.comb) {   // this lane's clusters -> global fp64 sums / u64 counts (job accumulators)
      if (pn) km_flush_partial(kacc[0], kcnt[0], pacc, pn);
#pragma unroll
      for (int q = 0; q < kKmCombMax / 32; ++q) {
        const uint32_t c = lane + 32 * q;
        if (c < P.k && kcnt[q]) {
          atomicAdd(P.km_cnts + c, kcnt[q]);
#pragma unroll
          for (int t = 0; t < 8; ++t) atomicAdd(P.km_sums + c * 8 + t, kacc[q][t]);
        }
      }
    }
  }
  if constexpr (W == kII) ii_drain(P, oc, outh, qn);   // this warp's last queued URLs
  // final flush of the partially filled half (all map warps done, nothing pending)
  named_bar_sync(2, nmap<W>() * 32);
  if constexpr (W == kWC) {
    if (P.comb && P.xtab) {   // two-level combiner: the CTA's slots are added into the L2 table
      const uint32_t* ctab = reinterpret_cast<const uint32_t*>(smem + Layout<W>::comb);
      for (uint32_t i = warp * 32 + lane; i < static_cast<uint32_t>(Cfg<W>::kCombSlots); i += nmap<W>() * 32) {
        const uint32_t k = ctab[i], c = ctab[Cfg<W>::kCombSlots + i];
        if (k != kCombEmpty32) red_add_u32(P.xtab + k, c);
      }
    } else if (P.comb && P.mkeys) {   // small-table mode: the CTA's slots go to the mid table
      const uint32_t* ctab = reinterpret_cast<const uint32_t*>(smem + Layout<W>::comb);
      for (uint32_t i = warp * 32 + lane; i < static_cast<uint32_t>(Cfg<W>::kCombSlots); i += nmap<W>() * 32) {
        const uint32_t k = ctab[i], c = ctab[Cfg<W>::kCombSlots + i];
        if (k != kCombEmpty32 && c) mid_insert(P, k, c);
      }
    } else if (P.comb) {   // combiner partials -> global (one atomic per warp step; demand counted past capacity)
      const uint32_t* ctab = reinterpret_cast<const uint32_t*>(smem + Layout<W>::comb);
      for (uint32_t i0 = warp * 32; i0 < static_cast<uint32_t>(Cfg<W>::kCombSlots); i0 += nmap<W>() * 32) {
        const uint32_t k = ctab[i0 + lane], c = ctab[Cfg<W>::kCombSlots + i0 + lane];
        const uint64_t v = static_cast<uint64_t>(k) | (static_cast<uint64_t>(c) << 32);
        const uint32_t mv = __ballot_sync(kFull, k != kCombEmpty32);
        if (!mv) continue;
        unsigned long long gb = 0;
        if (lane == 0) gb = atomicAdd(&P.st->pair_cursor_p, static_cast<unsigned long long>(__popc(mv)));
        gb = __shfl_sync(kFull, gb, 0);
        const uint64_t o = gb + __popc(mv & lanemask_lt());
        if (k != kCombEmpty32 && o < P.cap_p) P.ohp[o] = v;
      }
    }
  }
  if (threadIdx.x == 0) {
    const uint32_t cur = ld_acquire_cta_shared_u32(&oc->cur);
    seal<W>(P, oc, cur_gen(cur), cur_gen(cur) % kNOut, cur & kCntBits, true);
  }
}

template <int W, int V = 0>
__global__ void __launch_bounds__(threads_of<W>(), 1) k_map(Params P) {
  constexpr int kStages = Cfg<W>::kStages;
  extern __shared__ __align__(128) uint8_t smem[];
  OutCtl* oc = reinterpret_cast<OutCtl*>(smem + Layout<W>::ctl);
  if (threadIdx.x == 0) {
    oc->cur = 0;
    oc->final_seq = 0;
    for (int b = 0; b < kNOut; ++b) { oc->fbase[b] = 0; oc->committed[b] = 0; oc->fcount[b] = 0; }
    oc->nsealed = 0;
    oc->is_final = 0;
    oc->win_next = 0;
    oc->congested = 0;
    oc->pout[0] = oc->pout[1] = ~0u;
    oc->plast[0] = oc->plast[1] = 0;
    for (int b = 0; b < kNOut; ++b) { mbar_init(&oc->req[b], 1); mbar_init(&oc->done[b], 1); }
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + Layout<W>::full);
    uint64_t* empty = reinterpret_cast<uint64_t*>(smem + Layout<W>::empty);
    uint64_t* ready = reinterpret_cast<uint64_t*>(smem + Layout<W>::ready);
    for (int s = 0; s < kStages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], W == kKM ? kNMap : kNWin);   // text: one arrival per window
      mbar_init(&ready[s], 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    if (P.desc) {   // text: the dimensions k_tile_bounds derived on the device
      for (int i = 0; i < 4; ++i) s_bd[i] = P.desc[i];
    } else {        // fixed stride: host values
      s_bd[0] = P.nbytes;
      s_bd[1] = P.ntiles;
      s_bd[2] = P.gbase;
      s_bd[3] = 0;
    }
  }
  if constexpr (W == kWC) {
    uint32_t* ctab = reinterpret_cast<uint32_t*>(smem + Layout<W>::comb);   // keys, then counts
    for (uint32_t i = threadIdx.x; i < static_cast<uint32_t>(Cfg<W>::kCombSlots); i += blockDim.x) {
      ctab[i] = kCombEmpty32;
      ctab[Cfg<W>::kCombSlots + i] = 0;
    }
  }
  if constexpr (W == kKM) {
    if (P.comb) {
      uint32_t* z = reinterpret_cast<uint32_t*>(smem + Layout<W>::kmacc);
      for (uint32_t i = threadIdx.x; i < static_cast<uint32_t>(kKmWaccBytes / 4 + kNMap * kKmCombMax); i += blockDim.x)
        z[i] = 0;
    }
    float* cent = reinterpret_cast<float*>(smem + Layout<W>::cent);
    // pair layout: centroids (2p, 2p+1) interleaved per coordinate -> f32x2 operands
    for (uint32_t i = threadIdx.x; i < P.k * 8; i += blockDim.x) {
      const uint32_t j = i / 8, t = i % 8;
      const uint32_t kp = P.k & ~1u;
      cent[j < kp ? ((j & ~1u) * 8 + t * 2 + (j & 1u)) : i] = P.cent[i];
      if (P.km_bound) cent[P.k * 8 + i] = P.cent[i];   // row-layout copy (the bound test's centroid g)
    }
    if (P.km_bound) {   // s2[g]: squared distance to the nearest other centroid, fp64, rounded down
      float* s2 = cent + P.k * 16;
      for (uint32_t g = threadIdx.x; g < P.k; g += blockDim.x) {
        double m = 1.0 / 0.0;
        for (uint32_t j = 0; j < P.k; ++j) {
          if (j == g) continue;
          double d = 0.0;
          for (int t = 0; t < 8; ++t) {
            const double e = static_cast<double>(P.cent[g * 8 + t]) - static_cast<double>(P.cent[j * 8 + t]);
            d += e * e;
          }
          m = d < m ? d : m;
        }
        const float f = __double2float_rd(m * (1.0 - 1e-12));
        s2[g] = f < 1e-30f ? 0.0f : f;   // coincident / nearly coincident centroids: never take the shortcut
      }
    }
  }
  __syncthreads();
  if (s_bd[3]) return;   // more tiles than tile-bounds capacity: nothing mapped, the host grows + replays
  const uint32_t warp = threadIdx.x >> 5;
  if (warp >= static_cast<uint32_t>(nmap<W>()) && warp < static_cast<uint32_t>(nmap<W>() + nprod<W>()))
    producer_loop<W>(P, smem, warp - nmap<W>());
  else if (warp >= static_cast<uint32_t>(nmap<W>() + nprod<W>())) flush_loop<W>(P, smem, oc, warp - nmap<W>() - nprod<W>());
  else map_loop<W, V>(P, smem, oc);
}

// Batch dimensions + tile bounds of a text batch, on the device (mr_map enqueues without reading
// offsets[n] back): nbytes = offsets[n], ntiles, the batch's global byte base (the previous
// batch's base + length, or input_base) into desc[0..2]; desc[3] = 1 (and kErrTileCap) if the
// tile-bounds buffer is too small.  Then, grid-stride, the record starts inside the staged window
// [w_lo, w_hi) of every tile.
__global__ void k_tile_bounds(const uint64_t* off, uint64_t n, long long a0, uint64_t tb_cap, const uint64_t* prev,
                              uint64_t input_base, const uint8_t* rec, uint64_t* desc, uint64_t* tb,
                              unsigned int* err, unsigned long long* tile_next) {
  const uint64_t nbytes = off[n];
  const uint64_t ntiles = nbytes ? (nbytes + static_cast<uint64_t>(a0) + kT - 1) / kT : 0;
  const bool null_rec = nbytes && !rec;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    desc[0] = nbytes;
    desc[1] = ntiles;
    desc[2] = prev ? prev[2] + prev[0] : input_base;
    desc[3] = (ntiles > tb_cap || null_rec) ? 1ULL : 0ULL;   // the Map skips the batch
    *tile_next = 0;                                           // the Map's dynamic tile counter
    if (ntiles > tb_cap) atomicOr(err, kErrTileCap);
    if (null_rec) atomicOr(err, kErrNullRecords);
  }
  if (ntiles > tb_cap || null_rec) return;
  for (uint64_t t = blockIdx.x * static_cast<uint64_t>(blockDim.x) + threadIdx.x; t < ntiles;
       t += static_cast<uint64_t>(gridDim.x) * blockDim.x) {
    const long long chunk0 = static_cast<long long>(t) * kT - a0;
    const long long w_lo = max(0LL, chunk0 - kLead), w_hi = chunk0 + kT + kHalo;
    uint64_t res[2];
    const long long qs[2] = {w_lo, w_hi};
    for (int k = 0; k < 2; ++k) {  // lower_bound over offsets[0..n]
      uint64_t lo = 0, hi = n + 1;
      const uint64_t q = static_cast<uint64_t>(qs[k]);
      while (lo < hi) {
        const uint64_t mid = (lo + hi) >> 1;
        if (off[mid] < q) lo = mid + 1; else hi = mid;
      }
      res[k] = lo;
    }
    tb[2 * t] = res[0];
    tb[2 * t + 1] = res[1];
  }
}

template <int W>
cudaError_t launch_w(const MapArgs& a, int num_sms, cudaStream_t s) {
  using F = PairFmt<W>;
  Params P{};
  P.rec = a.records;
  P.off = a.offsets;
  P.n = a.n;
  P.nbytes = a.nbytes;   // (fixed stride; text batches: on the device, P.desc)
  P.a0 = static_cast<long long>(reinterpret_cast<uintptr_t>(a.records) & 15u);
  P.ntiles = W == kKM ? map_tiles(a) : 0;
  P.gbase = a.gbase;
  P.desc = W == kKM ? nullptr : a.desc;
  for (int i = 0; i < 4; ++i)
    P.pat[i] = a.pattern[4 * i] | (a.pattern[4 * i + 1] << 8) | (a.pattern[4 * i + 2] << 16) |
               (static_cast<uint32_t>(a.pattern[4 * i + 3]) << 24);
  P.cent = a.centroids;
  P.k = a.k;
  P.oh = a.out.h;
  P.okref = a.out.kref;
  P.ov = a.out.v;
  P.cap_pairs = a.out.cap;
  P.out_cap = (a.flags & 4u) ? F::kMaxReserve : F::kCap;   // MR_FLAG_FORCE_TINY_OUT
  P.flags = a.flags;
  P.st = a.st;
  P.tb = a.tile_bounds;
  P.off_end = a.offsets ? reinterpret_cast<const uint8_t*>(
                              reinterpret_cast<uintptr_t>(a.offsets + a.n + 1) & ~static_cast<uintptr_t>(15u))
                        : nullptr;
  P.hash_seed = a.hash_seed;
  P.key_bits = a.key_bits;
  P.xwin = a.xwin;
  P.xranks = (W == kII) ? a.xranks : 0u;
  P.ohb = a.out.hb;
  P.okrefb = a.out.krefb;
  P.cap_b = a.out.cap_b;
  P.ohc = a.out.hc;
  P.cap_c = a.out.cap_c;
  P.ohx = a.out.hx;
  P.ohp = a.out.hp;
  P.cap_p = a.out.cap_p;
  P.comb = (W == kWC && a.out.hp != nullptr) || (W == kKM && a.out.km_sums != nullptr && a.k <= kKmCombMax) ? 1u : 0u;
  P.km_sums = a.out.km_sums;
  P.km_cnts = a.out.km_cnts;
  P.pf = map_prefetch(W);
  P.wait_hint = map_wait_hint();
  P.dyn = map_dyn_windows(W);
  P.so = (a.flags & 1u) ? 1u : 0u;   // MR_FLAG_NO_SMEM_IN
  P.si = (a.flags & 2u) ? 1u : 0u;   // MR_FLAG_NO_SMEM_OUT
  P.sm_lines = (W == kSM && (a.flags & 0x200u)) ? 1u : 0u;   // MR_FLAG_SM_LINES
  P.wc_bal = map_wc_balanced();
  P.wc_fast = map_fast_path() ? 1u : 0u;
  P.xtab = (W == kWC && P.comb && map_wc_table_ok(a.flags)) ? a.out.xtab : nullptr;
  // the mid / long tables: with the exact-key table, or alone in small-table mode (which needs the
  // table-mode window; the host enables it only then, map_wc_tab)
  const bool tabs = W == kWC && P.comb && map_wc_table_ok(a.flags) && a.out.mkeys && (P.xtab || map_wc_tab());
  P.mkeys = tabs ? a.out.mkeys : nullptr;
  P.mcnt = tabs ? a.out.mcnt : nullptr;
  P.mbits = a.out.mbits;
  P.lkeys = (BMR_LTAB && tabs) ? a.out.lkeys : nullptr;
  P.lcnt = (BMR_LTAB && tabs) ? a.out.lcnt : nullptr;
  P.lbits = a.out.lbits;
  P.tile_next = (BMR_DYN_TILES && (W == kWC || W == kII)) ? &a.st->tile_next : nullptr;
  P.km_bound = (W == kKM && !(a.flags & 0x1000u) && a.k <= static_cast<uint32_t>(kKmBoundMax)) ? 1u : 0u;   // MR_FLAG_KM_FULL_SCAN
  if (W == kKM && P.ntiles == 0) return cudaSuccess;
  if constexpr (W != kKM) {
    const unsigned blocks = static_cast<unsigned>(std::min<uint64_t>((a.tb_cap + 255) / 256 + 1, 8ULL * num_sms));
    k_tile_bounds<<<blocks, 256, 0, s>>>(a.offsets, a.n, P.a0, a.tb_cap, a.prev_desc, a.input_base, a.records,
                                         a.desc, a.tile_bounds, &a.st->err, &a.st->tile_next);
    count_launch();
  }
  const size_t smem = Layout<W>::cent + (W == kKM ? static_cast<size_t>(a.k) * (P.km_bound ? 68 : 32) : 0);
  // WordCount table mode (the fast SIO path with the L2 tables): its own instantiation
  const bool tab = W == kWC && map_wc_tab() && P.mkeys && P.lkeys && P.comb && !P.so && !P.si && P.wc_bal && P.dyn && P.wc_fast;
  auto kern = k_map<W, 0>;
  if constexpr (W == kWC) {
    if (tab) kern = P.xtab ? k_map<W, 1> : k_map<W, 2>;
  }
  if constexpr (W == kKM) {   // the bound-test instantiation (the full scan keeps its own registers)
    if (P.km_bound) kern = k_map<W, 1>;
  }
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(smem));
  if (e != cudaSuccess) return e;
  int grid = a.grid > 0 ? a.grid : num_sms;   // persistent CTAs; CTAs without a tile exit at once
  if (W == kKM && static_cast<uint64_t>(grid) > P.ntiles) grid = static_cast<int>(P.ntiles);
  kern<<<grid, threads_of<W>(), smem, s>>>(P);
  count_launch();
  return cudaGetLastError();
}

}  // namespace

// L2 prefetch distance of the Map producers (BMR_MAP_PF, tiles; default 0 = off: measured slower
// on C2/C4 in round 1 with 2 producers)
// L2 prefetch distance of the producers in tiles (BMR_MAP_PF; default off: with the StringMatch
// record checks moved after the stage release it no longer helps, C2 round 1 sweep 0/1/2/4)
uint32_t map_prefetch(int w) {
  static int v = [] {
    const char* e = getenv("BMR_MAP_PF");
    return e ? atoi(e) : -1;
  }();
  (void)w;
  return v >= 0 ? static_cast<uint32_t>(v) : 0u;
}

// idle-wait flavour of the Map role warps (BMR_MAP_WAIT: 0 = plain try_wait, 1 = suspend-time
// hint, 2 = plain for the map warps and __nanosleep polling for the producers / flush warp)
// WordCount table-mode window path (BMR_WC_TAB env, default BMR_WC_TAB = 1: wc_window_tab; 0: the
// queued rounds of wc_window)
bool map_wc_tab() {
  static bool v = [] {
    const char* e = getenv("BMR_WC_TAB");
    return e ? atoi(e) != 0 : BMR_WC_TAB != 0;
  }();
  return v;
}

uint32_t map_wait_hint() {
  static uint32_t v = [] {
    const char* e = getenv("BMR_MAP_WAIT");   // (1: C5 13.90 -> 13.81 ms once the Map was issue-bound)
    return e ? static_cast<uint32_t>(atoi(e)) : 1u;
  }();
  return v;
}

// text window scheduling (BMR_MAP_DYN: 0 static, 1 dynamic; default: dynamic except StringMatch,
// whose windows are uniformly cheap -- measured on C2/C4/C5 in round 1)
uint32_t map_dyn_windows(int w) {
  static int v = [] {
    const char* e = getenv("BMR_MAP_DYN");
    return e ? atoi(e) : -1;
  }();
  return v >= 0 ? static_cast<uint32_t>(v) : (w == kSM ? 0u : 1u);
}

// WordCount emission: balanced two-phase rounds (BMR_WC_BAL=1, default) or lane-serial rounds (0)
uint32_t map_wc_balanced() {
  static uint32_t v = [] {
    const char* e = getenv("BMR_WC_BAL");
    return e ? static_cast<uint32_t>(atoi(e)) : 1u;
  }();
  return v;
}

// The WordCount L2 count table is fed by the SIO fast path only (wc_window); the memory-mode
// ablations and the lane-serial emission keep the exact stream
bool map_wc_table_ok(uint32_t flags) {
  return !(flags & 3u) && map_wc_balanced() && map_dyn_windows(kWC) && map_fast_path();
}

// WordCount / InvertedIndex SIO fast paths (wc_window / ii_window); BMR_MAP_FAST=0 selects the
// generic per-window path for A/B measurements (same results)
bool map_fast_path() {
  static const bool v = [] {
    const char* e = getenv("BMR_MAP_FAST");
    return e ? atoi(e) != 0 : true;
  }();
  return v;
}

int vbytes_of(int w) { return w == kKM ? 32 : w == kII ? 8 : 0; }
bool has_kref(int w) { return w == kII; }

uint64_t map_tiles(const MapArgs& a) {
  if (a.workload == kKM) return (a.n + kKmPts - 1) / kKmPts;
  const uint64_t a0 = reinterpret_cast<uintptr_t>(a.records) & 15u;
  return a.nbytes ? (a.nbytes + a0 + kT - 1) / kT : 0;
}

cudaError_t launch_map(const MapArgs& a, int num_sms, cudaStream_t s) {
  switch (a.workload) {
    case kWC: return launch_w<kWC>(a, num_sms, s);
    case kSM: return launch_w<kSM>(a, num_sms, s);
    case kKM: return launch_w<kKM>(a, num_sms, s);
    case kII: return launch_w<kII>(a, num_sms, s);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace bmr
