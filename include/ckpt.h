/* include/ckpt.h — C ABI of the B200-native GPU Merkle-tree checkpoint de-duplication
 * library (libckpt.so), after Tan et al., "Scalable Incremental Checkpointing using
 * GPU-Accelerated De-Duplication", ICPP'23. "P:n" cites /root/reference/PAPER.md line n;
 * "Rk" cites reading k in DESIGN.md §3.
 *
 * Problem statement: a process owns one GPU and repeatedly hands a
 * device buffer to the library; it stops while the buffer is de-duplicated on the GPU
 * ("stops during checkpointing to perform the de-duplication") and receives one
 * consolidated difference — compact metadata followed by the first-occurrence chunks
 * (P:81). Any checkpoint of the lineage can later be restored.
 *
 * General rules for every function:
 *  - Return value: a CKPT_* status; 0 (CKPT_OK) on success. Nothing is silently degraded
 *    and there is no CPU fallback: without a usable sm_100a GPU, calls fail.
 *  - A handle is bound to the CUDA device current at ckpt_create (every call makes that
 *    device current in the calling thread) and is not thread-safe: any host thread may use
 *    it, one at a time; different handles (one per GPU / process) are independent.
 *  - After any CUDA failure the handle is poisoned: every later call except ckpt_destroy
 *    returns CKPT_ESTATE.
 *  - "stream" arguments are cudaStream_t values passed as void* (NULL = legacy default
 *    stream) so this header needs no CUDA include.
 */
#ifndef CKPT_H_
#define CKPT_H_

#include <stdint.h>

#if defined(__GNUC__)
#define CKPT_API __attribute__((visibility("default")))
#else
#define CKPT_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct ckpt_ctx* ckpt_handle;

/* Pipelined calls in flight at most (ckpt_checkpoint_submit). */
#define CKPT_PIPELINE_DEPTH 2

enum {
  CKPT_OK = 0,
  CKPT_EINVAL = 1, /* bad argument / precondition violated; nothing changed           */
  CKPT_ENOMEM = 2, /* device allocation (record growth, diff arena) failed; nothing committed */
  CKPT_ECUDA = 3,  /* CUDA runtime/driver error; the handle is now poisoned            */
  CKPT_ERANGE = 4, /* checkpoint id out of range                                       */
  CKPT_ESTATE = 5, /* handle poisoned by an earlier CUDA error                          */
  CKPT_ECOLLIDE = 6 /* a 128-bit digest collision was detected (R14: out of scope). A WARNING,
                       not a failure: the checkpoint IS committed (diff filled, id advanced),
                       only the colliding phase-2 record insert was skipped. The one status
                       after which the lineage has changed. */
};

/* Statistics and location of one consolidated difference. */
typedef struct {
  uint32_t id;              /* 0-based position in this handle's lineage (R19)               */
  uint32_t chunk_bytes;     /* C                                                             */
  const uint8_t* dev_ptr;   /* serialized diff in device memory, OWNED BY THE HANDLE, valid
                               until ckpt_destroy (format: DESIGN.md §4, reading R13)        */
  uint64_t bytes;           /* meta_bytes + data_bytes                                       */
  uint64_t meta_bytes;      /* 64-B header + 4 B per FIRST region + 12 B per SHIFT region,
                               zero-padded to 16 B                                            */
  uint64_t data_bytes;      /* bytes of first-occurrence regions                      */
  uint64_t buf_bytes;       /* B                                                             */
  uint64_t n_leaves;        /* n = ceil(B / C)                                               */
  uint64_t n_first_regions; /* Tree metadata entries for first occurrences            */
  uint64_t n_shift_regions; /* Tree metadata entries for shifted duplicates                  */
  uint64_t n_first;         /* leaves labelled FIRST_OCUR (Alg.1 l.9)                        */
  uint64_t n_fixed;         /* leaves labelled FIXED_DUPL (Alg.1 l.4): unchanged             */
  uint64_t n_spatial;       /* SHIFT_DUPL leaves whose source is this checkpoint            */
  uint64_t n_temporal;      /* SHIFT_DUPL leaves whose source is an earlier checkpoint      */
  uint64_t list_entries;    /* List-method entries = n_first + n_spatial + n_temporal*/
  uint64_t record_size;     /* entries in the historical record after this checkpoint */
  uint64_t record_capacity; /* slots of the device record table                              */
  uint64_t phase2_inserts;  /* FIRST internal nodes inserted (Alg.1 l.29)                    */
  uint64_t phase3_inserts;  /* CKPT_VARIANT_SHIFT_INSERT: shifted regions inserted (R24)*/
} ckpt_diff;

/* De-duplication methods compared in the paper; the diff header's u16 `flags`
 * field (bytes 6-7) holds the method.
 *   CKPT_MODE_TREE   Algorithm 1 with Merkle-tree metadata compaction (ours, the default).
 *   CKPT_MODE_LIST   "identical to our method except for the metadata compaction, which is
 *                    omitted. Instead, a full list of all first-time occurrences and shifted
 *                    duplicates is stored along the new chunks": the Tree format with one
 *                    entry per non-FIXED leaf; the record holds leaves only.
 *   CKPT_MODE_BASIC  "breaks the checkpoint into chunks, hashes the chunks, then builds a
 *                    bitmap to indicate what chunks are new and what chunks remain
 *                    unchanged. It saves the bitmap and the new chunks": header
 *                    (n_first_regions = changed chunks, n_shift_regions = 0), ceil(n/32) u32
 *                    bitmap words (bit i of word i/32 = chunk i changed since checkpoint
 *                    k-1; all set at k = 0), zero pad to 16 B, the changed chunks in chunk
 *                    order at their true length. No record. */
enum { CKPT_MODE_TREE = 0, CKPT_MODE_LIST = 1, CKPT_MODE_BASIC = 2 };

/* Variants of the Tree method (readings R22, R23). Set with
 * ckpt_set_variant before the handle's first checkpoint.
 *   CKPT_VARIANT_FULL_FIRST   "a single first checkpoint that was taken fully", "we
 *                             capture a full initial checkpoint": checkpoint 0 runs
 *                             Algorithm 1 as usual (same record, same statistics of its
 *                             leaves), but its difference is stored in full.
 *   CKPT_VARIANT_FULL_SWITCH  "the worst-case scenario encountered only when the checkpointed
 *                             data fully changes during the checkpoint interval. This can be
 *                             easily detected, and incremental checkpointing can be
 *                             deactivated accordingly": a checkpoint k >= 1 with
 *                             1000 * (non-FIXED leaves) >= switch_permille * n is stored in
 *                             full and makes no record operation (Alg.1 l.6-46 skipped; the
 *                             leaf digests are still updated, l.21). Its statistics count the
 *                             changed chunks as n_first (n_spatial = n_temporal = 0) and
 *                             phase2_inserts = 0; record_size is unchanged.
 *   CKPT_VARIANT_SHIFT_INSERT "If this is the case, the new region is added to the historical
 *                             record of unique hashes", reading R24: after phase 2,
 *                             every internal node whose leaves are all shifted duplicates and
 *                             whose hash is new enters the record (minimum node id among
 *                             equal hashes, as R6); in phase 3 a parent of two shifted
 *                             children that finds ITS OWN entry is the first occurrence of
 *                             that content: its children are saved and it is not a region.
 *                             Repeated content then collapses into few regions (an all-zero
 *                             buffer of n = 2^h chunks: 2h regions instead of n). Such a node
 *                             can be the source of a later region although its bytes are no
 *                             first-occurrence data: restore resolves those sources chunk by
 *                             chunk through the source checkpoint's own regions (R25). Its
 *                             Tree differences carry header flags CKPT_FLAGS_SHIFT_INSERT.
 * A difference stored in full has header flags CKPT_FLAGS_FULL and the Tree layout with
 * n_first_regions = 1 (the root, node 0), n_shift_regions = 0 and the whole buffer as data
 * (meta_bytes = 80, data_bytes = B); ckpt_restore and ckpt_import accept it. */
enum { CKPT_VARIANT_FULL_FIRST = 1, CKPT_VARIANT_FULL_SWITCH = 2, CKPT_VARIANT_SHIFT_INSERT = 4 };
enum { CKPT_FLAGS_FULL = 3, CKPT_FLAGS_SHIFT_INSERT = 4 };

/* Create a handle.  P:77: fixed-size chunks of "tens or hundreds of bytes".
 *   chunk_bytes  C, a multiple of 16 with 32 <= C <= 65536 (C > 2 x 16-B digest).
 *   out          receives the handle (owned by the caller; free with ckpt_destroy).
 * Binds the handle to the current CUDA device.  Errors: CKPT_EINVAL (bad C / NULL out),
 * CKPT_ECUDA (no usable sm_100 device). */
CKPT_API int ckpt_create(uint32_t chunk_bytes, ckpt_handle* out);

/* ckpt_create with an explicit method (CKPT_MODE_*). ckpt_create is
 * ckpt_create_mode(chunk_bytes, CKPT_MODE_TREE, out). All other calls behave as described
 * for every mode; the statistics of a Basic diff count changed chunks as n_first and
 * n_first_regions (no spatial / temporal de-duplication).
 * Errors: as ckpt_create, and CKPT_EINVAL for an unknown mode. */
CKPT_API int ckpt_create_mode(uint32_t chunk_bytes, int mode, ckpt_handle* out);

/* Select the Tree-method variants above.
 *   flags            bitwise OR of CKPT_VARIANT_* (0 = Algorithm 1 only, the default).
 *   switch_permille  threshold of CKPT_VARIANT_FULL_SWITCH, 0..1000 (1000 = every leaf
 *                    changed, the paper's "fully changes"); ignored without that flag.
 * Errors: CKPT_EINVAL (handle not in CKPT_MODE_TREE, a checkpoint already taken, unknown
 * flag bits, switch_permille > 1000; nothing changed), CKPT_ESTATE. */
CKPT_API int ckpt_set_variant(ckpt_handle h, uint32_t flags, uint32_t switch_permille);

/* De-duplicate one checkpoint (Alg.1; serialization P:81).
 *   dev_ptr  device buffer of `bytes` bytes, 16-byte aligned, BORROWED: the call's kernels on
 *            `stream` read it; modify it only with work ordered after them (later work on
 *            `stream`, or after synchronising `stream`).
 *   bytes    B >= 1 with ceil(B / C) <= 2^31; every checkpoint of a handle must have the
 *            same B (R17: the fixed-duplicate test is positional).
 *   stream   cudaStream_t (as void*) all GPU work is enqueued on, in order.
 *   diff     receives the statistics and the device pointer of the new diff.
 * The call returns after exactly one host wait (ckpt_host_syncs): a spin on the flag the last
 * kernel publishes to mapped host memory as soon as the checkpoint's statistics are final —
 * after phases 2 and 3, when the gather kernel has summed the region counts (the process
 * "stops during checkpointing"). The rest of that kernel (writing the entries and data
 * of the diff) completes in stream order on `stream`: every later call of this library that
 * reads the lineage (the next ckpt_checkpoint on any stream, ckpt_diff_to_host[_async],
 * ckpt_restore[_stream], ckpt_import, the introspection calls) first waits on it (a stream
 * wait on an event, not a host wait); other readers of diff->dev_ptr order themselves after
 * `stream`. A call that grows the record table does so in stream order on `stream`. Capacity for the
 * record table and the diff is reserved before the first kernel, so an error leaves the
 * lineage unchanged (CKPT_ECOLLIDE is a committed checkpoint, see above).
 * Errors: CKPT_EINVAL, CKPT_ENOMEM, CKPT_ECUDA, CKPT_ESTATE, CKPT_ECOLLIDE. */
CKPT_API int ckpt_checkpoint(ckpt_handle h, const void* dev_ptr, uint64_t bytes, void* stream, ckpt_diff* diff);

/* Pipelined de-duplication of a lineage: the same checkpoint as ckpt_checkpoint, enqueued
 * without waiting for its statistics, so that checkpoint k + 1's leaf pass (K1, HBM-bound)
 * runs while checkpoint k's record and tree phases (latency-bound, "waves") do. The
 * method's arithmetic and every result are those of ckpt_checkpoint (the diffs are
 * bit-identical); only the overlap of consecutive calls differs.
 *   dev_ptr, bytes  as ckpt_checkpoint. BORROWED until ckpt_checkpoint_wait(id) returns AND
 *                   the caller's later work is ordered after the stream passed to it.
 *   stream          cudaStream_t (as void*) the leaf pass is ordered after; the leaf pass runs
 *                   on it, or (SM partitions) on an internal stream of a green
 *                   context ordered after it by an event; the record and tree phases and the
 *                   gather run on an internal non-blocking stream, ordered after the leaf pass.
 *                   SM partitions: created at the handle's first submit when the buffer is at
 *                   most 2 GiB (host time once); each call picks one from the candidate count of
 *                   the last collected call, or none. Environment CKPT_GREEN=0 disables them;
 *                   they are also off under a profiling tool (CUDA_INJECTION64_PATH set).
 *   id              receives the checkpoint id (= the number of checkpoints before it).
 * At most CKPT_PIPELINE_DEPTH (2) calls are in flight: a submit with that many outstanding
 * first collects the oldest (a host wait). Every other call of this library (ckpt_checkpoint, diff access, restore,
 * import, introspection) first collects all outstanding calls, oldest first.
 * Errors: as ckpt_checkpoint (an error of the collected older call is returned here). */
CKPT_API int ckpt_checkpoint_submit(ckpt_handle h, const void* dev_ptr, uint64_t bytes, void* stream, uint32_t* id);

/* Collect checkpoint `id` (and every older outstanding one): returns its statistics once they
 * are final (one host wait per collected call, ckpt_host_syncs), like ckpt_checkpoint.
 *   stream  cudaStream_t (as void*) made to wait (an event, not a host wait) for the rest of
 *           call id's work (the gather of its entries and data, which reads the buffer);
 *           enqueue reuse of the buffer or reads of diff->dev_ptr after it. May be the
 *           stream of a later submit: that call's leaf pass is already enqueued before it.
 *   diff    receives the statistics and the device pointer of diff `id`.
 * Errors: CKPT_ERANGE (id not submitted), CKPT_EINVAL, CKPT_ECUDA, CKPT_ESTATE,
 * CKPT_ECOLLIDE (committed, R14). */
CKPT_API int ckpt_checkpoint_wait(ckpt_handle h, uint32_t id, void* stream, ckpt_diff* diff);

/* Rebuild checkpoint `id` into the caller's device buffer ("start from the
 * first-time occurrences, then fill the fixed duplicates and finally assemble the shifted
 * duplicates from the corresponding checkpoint ID"). Equivalent to replaying diffs 0..id
 * (R16), computed directly: each chunk is written once, from the newest diff <= id whose
 * regions cover it: per diff, newest first, the chunks it covers
 * are claimed (source address per chunk), then one kernel copies every chunk once.
 * Per-diff restore plans are built by the first restore that needs them and cached: about
 * 2-3x the diff's metadata plus 12 bytes per chunk the diff covers, in device memory; the
 * handle also keeps 8 bytes per chunk of the buffer for the claims.
 *   dev_ptr  device buffer of B bytes, 16-byte aligned, owned by the caller; overwritten.
 * Synchronous. Runs on an internal stream of the handle that is a BLOCKING stream: work
 * enqueued earlier on the legacy default stream (and on other blocking streams) completes
 * before the restore touches dev_ptr; work on non-blocking streams is NOT ordered — use
 * ckpt_restore_stream for those.
 * Errors: CKPT_ERANGE (id >= number of checkpoints), CKPT_EINVAL, CKPT_ECUDA, CKPT_ESTATE. */
CKPT_API int ckpt_restore(ckpt_handle h, uint32_t id, void* dev_ptr);

/* ckpt_restore with every kernel enqueued on `stream` (cudaStream_t as void*), in order
 * after the caller's earlier work there; returns after synchronising `stream`. The plan
 * building of a diff's first restore runs on `stream` too.  Errors as ckpt_restore. */
CKPT_API int ckpt_restore_stream(ckpt_handle h, uint32_t id, void* dev_ptr, void* stream);

/* Statistics / device pointer of an earlier diff.  Errors: CKPT_ERANGE, CKPT_EINVAL. */
CKPT_API int ckpt_diff_info(ckpt_handle h, uint32_t id, ckpt_diff* diff);

/* Copy diff `id` to host memory with ONE device-to-host transfer ("initiating a
 * single device-to-host data transfer is enough").
 *   host_ptr  caller-owned host memory (pinned for full PCIe bandwidth) of >= capacity B.
 * Synchronous. Errors: CKPT_ERANGE, CKPT_EINVAL (capacity < diff bytes), CKPT_ECUDA. */
CKPT_API int ckpt_diff_to_host(ckpt_handle h, uint32_t id, void* host_ptr, uint64_t capacity);

/* ckpt_diff_to_host without waiting (the single D2H of P:81, overlapped
 * with the next de-duplication): enqueues the one device-to-host copy of diff `id` on
 * `stream` (cudaStream_t as void*) and returns. Diffs are immutable and never move, so the
 * copy may run while later ckpt_checkpoint calls de-duplicate on another stream; the host
 * data is valid once `stream` has completed the copy (the caller synchronises it). A diff
 * already collected (ckpt_checkpoint_wait) is copied without collecting the pipelined calls
 * still in flight; the copy is ordered after that call's gather.
 *   host_ptr  caller-owned PINNED host memory of >= capacity bytes (pageable memory would make
 *             the copy synchronous), borrowed until the copy completes.
 * Errors: CKPT_ERANGE, CKPT_EINVAL (capacity < diff bytes), CKPT_ECUDA, CKPT_ESTATE. */
CKPT_API int ckpt_diff_to_host_async(ckpt_handle h, uint32_t id, void* host_ptr, uint64_t capacity, void* stream);

/* End-to-end convenience path over HOST memory (P:196's throughput definition: create
 * the incremental checkpoint and copy it to host memory): copies `bytes` from host_ptr
 * into a handle-owned device staging buffer, runs ckpt_checkpoint on `stream`, then
 * copies the diff into host_diff (capacity host_diff_cap) — one H2D, one D2H.
 * host_diff may be NULL to skip the D2H.  Errors as ckpt_checkpoint and ckpt_diff_to_host. */
CKPT_API int ckpt_checkpoint_host(ckpt_handle h, const void* host_ptr, uint64_t bytes, void* stream,
                         void* host_diff, uint64_t host_diff_cap, ckpt_diff* diff);

/* Rebuild a lineage after a restart (the GPU cannot keep the
 * record across runs, the diffs live in host memory / storage): appends diff `id` =
 * ckpt_num_checkpoints() from host memory to this handle as if the checkpoint had just been
 * taken. The checkpoint is restored from the lineage plus the imported diff and
 * de-duplicated again, which rebuilds the record and the leaf digests (R5) exactly;
 * the regenerated diff must equal the imported one byte for byte.
 *   host_diff  a diff produced by a handle of the same chunk size and method (header
 *              `flags`), for checkpoint number ckpt_num_checkpoints(h); borrowed.
 *   bytes      its size; stream as for ckpt_checkpoint (the re-de-duplication runs there).
 * Synchronous. Errors: CKPT_EINVAL (bad header, wrong id / size / chunk size / method: the
 * handle is unchanged; or the regenerated diff differs: the handle is poisoned), CKPT_ENOMEM,
 * CKPT_ECUDA, CKPT_ESTATE. */
CKPT_API int ckpt_import(ckpt_handle h, const void* host_diff, uint64_t bytes, void* stream);

/* Number of checkpoints taken so far. */
CKPT_API int ckpt_num_checkpoints(ckpt_handle h, uint32_t* count);

/* Introspection for parity tests (not on the hot path):
 * ckpt_leaf_digests copies the persistent leaf digests Tree(leaf) of the latest checkpoint
 * (Alg.1 l.21; 16 B per chunk, h1 LE || h2 LE, R1) into device memory dev_out (16 n bytes).
 * ckpt_record_dump copies the historical record to host arrays: keys (16 B each),
 * node ids and checkpoint ids, at most `cap` entries; *count receives the record size. */
CKPT_API int ckpt_leaf_digests(ckpt_handle h, void* dev_out);
CKPT_API int ckpt_record_dump(ckpt_handle h, uint8_t* host_keys, uint32_t* host_nodes, uint32_t* host_ckpts,
                     uint64_t cap, uint64_t* count);

/* Per-phase device times (ms) of the latest ckpt_checkpoint, measured with CUDA events on
 * the caller's stream when profiling is enabled: ckpt_set_profiling(h, level), level 0 = off,
 * 1 = events around K1 and the whole call only (an event between two kernels stops the
 * second from launching early, so level 1 is the one to time under), 2 = every phase.
 * times[0] leaf hash pass (K1), [1] record insert (K1b), [2] phase 2 (all stages),
 * [3] phase 3 (all stages), [4] compaction (offsets + gather), [5] whole call (first
 * kernel to last kernel; [1]..[4] are 0 at level 1); host wall times of the same call
 * (always recorded): [6] entry to first enqueue, [7] enqueue of the kernel sequence, [8]
 * wait in the one stream synchronisation, [9] bookkeeping after it, and within [6]: [10]
 * record-table growth (stream-ordered allocation, fill and rehash enqueued), [11] diff-arena
 * growth (physical memory mapped).  n <= 12 values are written.  ckpt_set_profiling errors: CKPT_EINVAL (level outside 0..2). */
CKPT_API int ckpt_set_profiling(ckpt_handle h, int enable);
CKPT_API int ckpt_phase_times(ckpt_handle h, float* times, int n);
/* Same for checkpoint `id` (device times kept for the latest 256 profiled checkpoints; the
 * event queries happen here, never inside ckpt_checkpoint). Errors: CKPT_ERANGE. */
CKPT_API int ckpt_phase_times_of(ckpt_handle h, uint32_t id, float* times, int n);

/* Number of kernels this handle has enqueued so far (ckpt_checkpoint, ckpt_restore and the
 * calls built on them), counted at the launch sites; bench.py reports the difference over
 * its timed region. */
CKPT_API int ckpt_kernel_launches(ckpt_handle h, uint64_t* count);

/* Number of times this handle has blocked the host on the device so far (stream
 * synchronisations and the completion spin of ckpt_checkpoint), counted at the wait sites.
 * ckpt_checkpoint adds exactly one, including a call that grows the record table (the
 * growth enqueues the fill and rehash on the caller's stream; the replaced table is kept
 * until ckpt_destroy, at most the size of the current one since growth doubles it).
 * Errors: CKPT_EINVAL. */
CKPT_API int ckpt_host_syncs(ckpt_handle h, uint64_t* count);

/* Release all device memory of the handle (record, leaf digests, every diff). */
CKPT_API int ckpt_destroy(ckpt_handle h);

/* Static description of a status code. */
CKPT_API const char* ckpt_strerror(int status);

#ifdef __cplusplus
}
#endif
#endif /* CKPT_H_ */
