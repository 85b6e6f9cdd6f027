/* bmr.h — C ABI of libbmr, a B200-native (sm_100a) implementation of the data-parallel hot
 * path of Ji & Ma, "Using Shared Memory to Accelerate MapReduce on GPUs" (IPDPS 2011):
 * Map (stage-in -> user map -> emit -> flush) -> group-by-key (hash + LSD radix sort + segment
 * boundaries) -> Reduce.
 *
 * Citations: "L<n>" = line n of the paper text (reference PAPER.md); "§8(x)" = SURVEY.md.
 *
 * Data model (L51-52 "Input, intermediate, and output are all in the format of <key, value>
 * pairs"; L85 key/value index arrays; L36 "no assumption on input/output data sizes, size
 * variations, or record counts"): an input batch is `records` (bytes) + `offsets` (n+1 u64;
 * record i is records[offsets[i], offsets[i+1])) or fixed-stride records.  The record index is
 * the implicit input value (Table II, 4-byte input value).
 *
 * Threading: a job is used by one host thread at a time; distinct jobs are independent.
 * Errors: every call returns an mr_status; nothing aborts, exits or throws across the ABI.
 * Asynchronous device faults surface as MR_ERR_CUDA at the next synchronising call
 * (mr_group, mr_fetch); mr_last_error() gives the detail.
 */
#ifndef BMR_H
#define BMR_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MR_ABI_VERSION 1

typedef struct mr_job mr_job; /* opaque; owned by the library */

typedef enum {
  MR_OK = 0,
  MR_ERR_INVALID = 1,     /* bad argument (NULL, abi_version, k, dim, alignment, ...) */
  MR_ERR_STATE = 2,       /* call out of order (see state machine below) */
  MR_ERR_OOM = 3,         /* device cannot hold the demanded intermediate / output */
  MR_ERR_OVERFLOW = 4,    /* an emitted key exceeds 65535 bytes; the batch is rejected */
  MR_ERR_CUDA = 5,        /* CUDA runtime / kernel error (detail in mr_last_error) */
  MR_ERR_NCCL = 6,        /* collective failure (multi-GPU) */
  MR_ERR_UNSUPPORTED = 7  /* e.g. >= 2^32 intermediate pairs in one group */
} mr_status;

/* Workloads (L125): compiled-in device functors. */
typedef enum { MR_WORDCOUNT = 1, MR_STRINGMATCH = 2, MR_KMEANS = 3, MR_INVINDEX = 4 } mr_workload;

/* Flags */
#define MR_FLAG_NO_SMEM_IN      0x01u /* SO ablation (L134): map warps read record bytes from global memory */
#define MR_FLAG_NO_SMEM_OUT     0x02u /* SI ablation (L135): one global atomic per warp result, direct HBM writes */
                                      /* both = G (L173); neither = SIO, the default (L133, C-3 #18) */
#define MR_FLAG_FORCE_TINY_OUT  0x04u /* output half = one warp result: every warp result overflows (L113) */
#define MR_FLAG_WEAK_HASH_DEBUG 0x08u /* 4-bit key hash: forces collisions, exercises verification */
#define MR_FLAG_VALIDATE        0x10u /* host-side argument validation of offsets (reads them back) */
#define MR_FLAG_NO_COMBINE      0x20u /* multi-GPU: exchange raw pairs (no combiner) */
#define MR_FLAG_PROFILE         0x40u /* record CUDA events per phase on the job stream (mr_stats *_ms) */
#define MR_FLAG_OWN_STREAM      0x80u /* ignore cfg.stream: the job creates a private non-blocking stream */
#define MR_FLAG_NO_MAP_COMBINE  0x100u /* WC: no in-SMEM combiner in the Map (every word is emitted as a pair) */
#define MR_FLAG_SM_LINES        0x200u /* SM: the paper's per-line output (L125): the global offset of every
                                          record containing the pattern, once (grouped by key) */
#define MR_FLAG_FORCE_SPILL     0x800u /* test hook: every warp result that overflows the output buffer is
                                          written straight to HBM (the a5 spill path), not only while the
                                          buffer ring is congested */
#define MR_FLAG_KM_FULL_SCAN    0x1000u /* KM: every point scans all k centroids (the paper's literal Map); by
                                          default a point whose distance to its lane's previous winner g is
                                          below a quarter of the squared distance from g to its nearest other
                                          centroid (with an fp32 rounding margin) is assigned g directly: the
                                          triangle inequality makes every other centroid strictly farther, so
                                          the assignment is the one the full scan computes */
#define MR_FLAG_BATCH_COMBINE   0x400u /* WC: each mapped batch is grouped + reduced (combined) when the next
                                          one is mapped — mr_map then synchronises — and its (key, count)
                                          partials kept; mr_group merges the partials (exact sums).  For
                                          jobs larger than one group (>= 2^32 pairs) or HBM: batched
                                          processing "at another level" (L74).  Ignored by SM / KM / II. */

typedef struct { uint8_t pattern[16]; } mr_sm_params;                      /* StringMatch */
typedef struct { uint32_t k, dim; const float* centroids; } mr_km_params;  /* KMeans: host ptr, k x dim fp32, dim == 8, 1 <= k <= 1024 */

typedef struct {
  uint32_t abi_version;      /* must equal MR_ABI_VERSION */
  mr_workload workload;
  int device;                /* CUDA ordinal; made current on every call */
  void* stream;              /* cudaStream_t to enqueue on; NULL = job-owned stream */
  uint32_t record_stride;    /* 0: variable-size records (offsets required); KM: 32 */
  const void* params;        /* mr_sm_params* / mr_km_params* / NULL; copied at create */
  uint64_t input_base;       /* global byte offset of this rank's first record (SM/II offsets are global) */
  int rank, nranks;          /* nranks == 1: single GPU */
  void* nccl_comm;           /* nranks > 1: an NCCL communicator over the nranks processes (one per GPU)
                                from mr_comm_init — mr_group then performs the exchange itself; NULL:
                                the caller moves the bytes (mr_partition_count / _write / mr_ingest) */
  uint64_t max_pairs_hint;   /* initial intermediate capacity in pairs (0: heuristic) */
  uint64_t heap_bytes_hint;  /* reserved */
  uint32_t flags;            /* MR_FLAG_* */
} mr_config;

/* Job-owned host memory, valid until the next mr_* call on the job or mr_job_destroy.
 *   WC: key = word bytes,        val = u64 count                       (L125 "number of occurrences")
 *   SM: key = u64 global offset, val = empty    (Map-only; one entry per match, overlaps counted)
 *   KM: key = u32 cluster id,    val = 8 x fp32 new centroid || u64 count (all k clusters)
 *   II: key = URL bytes,         val = u64[] global offsets of the URL (L125 "link's position")
 * Key order is unspecified (hash order); callers canonicalise. */
typedef struct {
  uint64_t n_keys;
  const uint8_t* keys; const uint64_t* key_offsets; /* n_keys + 1 */
  const uint8_t* vals; const uint64_t* val_offsets; /* n_keys + 1 */
} mr_result;

typedef struct {
  uint64_t pairs;          /* intermediate pairs emitted by Map (M) */
  uint64_t flushes;        /* SMEM output-half flushes (one global atomic each, L113) */
  uint64_t replays;        /* batches replayed after capacity growth */
  uint64_t n_keys;         /* distinct keys (S) */
  uint64_t collisions;     /* hashed-key mismatches found by verification (then re-sorted) */
  uint64_t sort_passes;    /* LSD passes executed (constant digits skipped) */
  uint64_t map_tiles;      /* input tiles staged by the producer warps */
  uint64_t input_bytes;    /* record bytes mapped */
  uint64_t capacity_pairs; /* current intermediate capacity */
  uint64_t kernel_launches;/* libbmr kernels launched since create / reset */
  /* MR_FLAG_PROFILE: device time per phase (CUDA events on the job stream), ms */
  double map_ms, hist_ms, sort_ms, seg_ms, reduce_ms;
  /* WordCount Map output streams: pairs of the hashed stream (included in
   * `pairs`), LSD passes of the keys-only exact-stream sort (included in `sort_passes`) and
   * their device time (included in `sort_ms`) */
  uint64_t pairs_hashed;
  uint64_t sort_passes_keys;
  double sort_keys_ms;
  /* WordCount mid stream (6..8-byte words, exact 48-bit keys, sorted keys-only): pairs and LSD
   * passes (included in `pairs` / `sort_passes`; its device time is in `sort_ms`) */
  uint64_t pairs_mid;
  uint64_t sort_passes_mid;
  /* WordCount in-SMEM combiner: partial (key, count) entries flushed by the
   * Map CTAs (not included in `pairs`), and the words they absorbed (not emitted as pairs) */
  uint64_t pairs_partial;
  uint64_t words_combined;
  /* the exchange inside mr_group (nranks > 1 with nccl_comm): bytes sent / received by this rank
   * (entries + key bytes; WC / KM after the local combiner) and its device time (MR_FLAG_PROFILE) */
  uint64_t xchg_send_bytes;
  uint64_t xchg_recv_bytes;
  double xchg_ms;
  /* Map output ring (L113, §8(a) a5): seals that found every buffer still flushing, and the warp
   * results written straight to HBM (the overflow spill) while the sealer waited */
  uint64_t map_seal_waits;
  uint64_t map_spills;
  /* KMeans Map: points that scanned all k centroids (the rest were assigned by the bound test,
   * MR_FLAG_KM_FULL_SCAN off) */
  uint64_t km_points_scanned;
} mr_stats;

/* State machine: CREATED -> mr_map x k (batches append) -> mr_group -> mr_reduce -> mr_fetch
 * (-> mr_job_reset -> CREATED, keeping device buffers).  Out of order -> MR_ERR_STATE.
 * SM (Map-only): mr_group and mr_reduce are valid no-ops. */

/* Create a job.  Copies cfg and params.  Allocates nothing large until the first mr_map. */
mr_status mr_job_create(const mr_config* cfg, mr_job** out);

/* Map one batch of DEVICE-resident records (§8(a) a1-a5).
 *   records: device bytes.  Keys are emitted BY REFERENCE into records (L110 "addressable
 *            place"), so every mapped batch must stay alive and unmodified until mr_reduce has
 *            completed.  KM (record_stride 32) requires 16-byte aligned records.
 *   offsets: device, n+1 u64, offsets[0] == 0, non-decreasing, offsets[n] = batch length;
 *            NULL iff record_stride > 0 (then record i = records[i*stride, (i+1)*stride)).
 *   n:       number of records (0 allowed).
 * Asynchronous (§8(b): enqueue and return): a text batch's length offsets[n], its tile count
 * and global byte base are derived on the device (never read back here), so no call but the
 * synchronising ones (mr_group, mr_fetch) waits for the device.  Global byte offsets emitted by
 * SM/II are input_base + (sum of earlier batch lengths) + in-batch offset.  Errors found on the
 * device (records NULL for a non-empty batch, a key > 65535 bytes) surface at mr_group.
 * Exception: MR_FLAG_BATCH_COMBINE folds the previous batches first (synchronising). */
mr_status mr_map(mr_job* job, const uint8_t* records, const uint64_t* offsets, uint64_t n);

/* Same as mr_map for HOST buffers: the library copies records/offsets into job-owned device
 * memory on the job stream (the end-to-end path of bench.py). */
mr_status mr_map_host(mr_job* job, const uint8_t* records, const uint64_t* offsets, uint64_t n);

/* Map HOST text whose records are its '\n'-terminated lines (the record model of the text
 * configs, Table II "a line"): record i ends with the i-th '\n' (inclusive); bytes after
 * the last '\n' form one more record.  Equivalent to mr_map_host(text, offsets, n) with those
 * offsets, without an offsets array crossing the host link: the library copies the text in
 * batches (~256 MiB, ending after a '\n') on its own copy stream and, per batch, derives the
 * offsets on the device and runs the Map while the next batch is in flight.  `text` (caller-
 * owned) must stay valid until the call returns; pin it (cudaHostRegister / cudaMallocHost) for
 * the copies to overlap.  Each batch becomes one mapped batch (SM/II offsets stay global).
 * MR_ERR_INVALID for fixed-stride workloads (KM) or text == NULL with nbytes > 0. */
mr_status mr_map_host_lines(mr_job* job, const uint8_t* text, uint64_t nbytes);

/* Group by key (§8(a) a6-a8): capacity check (grow + replay on overflow), digit histogram,
 * onesweep LSD passes over non-constant digits, segment boundaries with byte verification of
 * hashed keys (re-sort with a fresh hash on collision).  Synchronises the stream.
 * nranks > 1 with cfg.nccl_comm: first the exchange —
 * partition by destination rank mix64(hash of the key bytes) mod nranks (WC / KM after a local
 * group + reduce, the combiner; II and MR_FLAG_NO_COMBINE WC raw pairs), ncclAlltoAll of the
 * count matrix, one NCCL group of send / recv for the entries and key bytes, ingest — then the
 * local group of the keys this rank owns.  Collective: every rank of the communicator calls
 * mr_group.  MR_ERR_NCCL on a communication failure (detail in mr_last_error). */
mr_status mr_group(mr_job* job);

/* Reduce (§8(a) a9) and device-side output assembly.  Asynchronous. */
mr_status mr_reduce(mr_job* job);

/* Copy the output to job-owned pinned host memory; synchronises.  *out valid until the next
 * call on the job. */
mr_status mr_fetch(mr_job* job, mr_result* out);

/* Back to CREATED, keeping every device buffer (repeated runs without reallocation). */
mr_status mr_job_reset(mr_job* job);

/* Fill min(bytes, sizeof(mr_stats)) bytes of an mr_stats. */
mr_status mr_get_stats(const mr_job* job, void* stats, size_t bytes);

mr_status mr_job_destroy(mr_job* job); /* NULL-safe */
const char* mr_status_string(mr_status s);
const char* mr_last_error(const mr_job* job);

/* ---- Multi-GPU exchange: one all-to-all between Map and group-by ----
 * Input is sharded by byte range (no communication in Map; input_base keeps SM/II offsets
 * global).  Records are routed to rank mix64(hash of the key bytes) mod nranks.  WC and KM first
 * run the local group + reduce as a combiner (the original MapReduce combiner; the paper uses
 * none) unless MR_FLAG_NO_COMBINE (WC only); II exchanges raw pairs.  StringMatch
 * is Map-only and has no exchange (MR_ERR_UNSUPPORTED).  With cfg.nccl_comm, mr_group runs these
 * steps itself over NCCL; without it the caller moves the bytes (e.g. torch.distributed
 * all_to_all_single, gloo in CPU-staged tests) through:
 *   1. mr_partition_count(job, counts, &entry_bytes): counts[2r] = entries for rank r,
 *      counts[2r+1] = heap bytes for rank r (host array of 2*nranks u64); synchronises.
 *   2. caller allocates device buffers of sum(entries)*entry_bytes and sum(heap) bytes;
 *      mr_partition_write(job, entries, heap) fills them, slices in rank order (asynchronous).
 *   3. all-to-all; then mr_ingest(job, recv_entries, recv_heap, recv_counts) with the received
 *      buffers concatenated in source-rank order and recv_counts[2r], [2r+1] from source r.
 *      The received heap holds the key bytes, referenced until mr_reduce completes (caller-owned).
 *   4. mr_group / mr_reduce / mr_fetch as usual; each rank outputs the keys it owns.
 * State: MAPPED -> partition_count -> partition_write -> ingest -> MAPPED (ingested). */
mr_status mr_partition_count(mr_job* job, uint64_t* counts, uint64_t* entry_bytes);
mr_status mr_partition_write(mr_job* job, void* entries, void* heap);
mr_status mr_ingest(mr_job* job, const void* entries, const void* heap, const uint64_t* recv_counts);

/* ---- NCCL communicator for the exchange inside mr_group ----
 * libnccl.so.2 is loaded at run time (BMR_NCCL_LIB, else the copy already in the process — e.g.
 * torch's — else the loader's): no link-time dependency, single-GPU jobs never load it.
 *   mr_comm_unique_id(id): rank 0 fills MR_NCCL_ID_BYTES bytes (host buffer), which the caller
 *     broadcasts to every rank (e.g. torch.distributed.broadcast_object_list);
 *   mr_comm_init(id, nranks, rank, device, &comm): collective over the nranks processes; comm is
 *     an ncclComm_t owned by the caller, passed to jobs as mr_config.nccl_comm;
 *   mr_comm_destroy(comm) after the last job using it (NULL-safe).
 * MR_ERR_NCCL if NCCL cannot be loaded or fails; mr_comm_backend() names the loaded NCCL. */
#define MR_NCCL_ID_BYTES 128
mr_status mr_comm_unique_id(void* id);
mr_status mr_comm_init(const void* id, int nranks, int rank, int device, void** comm);
mr_status mr_comm_destroy(void* comm);
const char* mr_comm_backend(void);

/* ---- Fused Map flush + shuffle over peer memory, InvertedIndex ----
 * Instead of partition + all-to-all, the Map's flush appends every record straight to the
 * receive window of its destination rank (same destination function as mr_partition_*): per
 * warp and destination one atomic pair on the window cursor, then the 16-byte entry
 * (heap offset << 16 | key length, u64 value) and the key bytes (8-byte aligned records).
 * A window = entries (16-B aligned, entry_cap x 16 B) + heap (8-B aligned, heap_cap bytes) +
 * cursor (2 x u64: entries, heap bytes appended; counts demand past the capacity), all device
 * memory the CALLER owns and zeroes, addressable from this process: a peer GPU's buffers opened
 * through CUDA IPC (NVLink stores and atomics), or same-GPU buffers (virtual ranks, tests).
 *   mr_set_xwindows(job, R, entries[R], heaps[R], cursors[R], entry_cap, heap_cap) — host arrays
 *     of device pointers, window r = rank r; CREATED state (before mr_map); R = 0 disables.
 *     MR_ERR_INVALID: not InvertedIndex, NULL / misaligned pointer, R > 64.
 *   mr_map ... (the records leave through the windows; nothing stays local)
 *   all ranks' Maps complete (caller's barrier), then on every rank
 *   mr_ingest_xwindow(job, own_entries, own_heap, own_cursor, entry_cap, heap_cap): reads the
 *     cursor, MR_ERR_OOM if the window overflowed (nothing ingested; re-run with larger windows),
 *     else ingests like mr_ingest -> MAPPED; then mr_group / mr_reduce / mr_fetch. */
mr_status mr_set_xwindows(mr_job* job, uint32_t nranks, void* const* entries, void* const* heaps,
                          uint64_t* const* cursors, uint64_t entry_cap, uint64_t heap_cap);
mr_status mr_ingest_xwindow(mr_job* job, const void* entries, const void* heap, const uint64_t* cursor,
                            uint64_t entry_cap, uint64_t heap_cap);

/* Device memory and CUDA IPC helpers for windows shared between processes (one per GPU):
 * mr_dev_alloc: cudaMalloc of >= bytes on `device` (a whole allocation, so its IPC handle maps
 * it at offset 0; MR_ERR_OOM).  mr_dev_free / mr_dev_zero / mr_dev_copy (synchronous,
 * cudaMemcpyDefault).  mr_ipc_handle: the MR_IPC_HANDLE_BYTES-byte handle of an mr_dev_alloc
 * pointer (host buffer out).  mr_ipc_open: maps another process's handle on `device` (peer
 * access enabled lazily: NVLink on B200 boxes); mr_ipc_close unmaps.  Failures -> MR_ERR_CUDA. */
#define MR_IPC_HANDLE_BYTES 64
mr_status mr_dev_alloc(int device, uint64_t bytes, void** dptr);
mr_status mr_dev_free(void* dptr);
mr_status mr_dev_zero(void* dptr, uint64_t bytes);
mr_status mr_dev_copy(void* dst, const void* src, uint64_t bytes);
mr_status mr_ipc_handle(const void* dptr, void* handle);
mr_status mr_ipc_open(int device, const void* handle, void** dptr);
mr_status mr_ipc_close(void* dptr);

/* Group-by primitive exposed for testing (§8(a) a7): stable LSD radix sort of n u64 device
 * keys; writes the sorted keys and the u32 permutation (perm[i] = source index of the i-th
 * key).  Synchronises `stream`. n < 2^32. */
mr_status mr_sort_u64(const uint64_t* keys, uint64_t* keys_out, uint32_t* perm_out, uint64_t n, void* stream);

#ifdef __cplusplus
}
#endif
#endif /* BMR_H */
