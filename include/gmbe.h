/* gmbe.h -- C ABI of the B200 (sm_100a) maximal-biclique-enumeration library (libgmbe.so).
 *
 * The operation (PAPER.md = Pan et al., SC'23, cited P:<line>):
 *   Given a bipartite graph G(U, V, E), enumerate all maximal bicliques:
 *   pairs (L, R), L ⊆ U, R ⊆ V, both non-empty, every u∈L adjacent to every v∈R, and no biclique
 *   (L', R') with L ∪ R ⊂ L' ∪ R'.  The library returns their number and an
 *   order-independent 64-bit checksum, and optionally writes the pairs.
 *   The search is the set-enumeration tree of Alg 1/2 with an explicit
 *   excluded set Q for the maximality check, Alg 3 root tasks, pro-active pruning by
 *   local neighbourhood size (Thm 4.1) and load-aware task splitting (Alg 4,
 *   P:930-1010), run by a persistent CUDA kernel.
 *
 * Conventions (all calls):
 *   - Return 0 (GMBE_OK) on success, a negative GMBE_E* code otherwise; gmbe_last_error() gives a
 *     thread-local message for the last failing call on this thread.
 *   - All ids are the CALLER's original 0-based ids and roles, in every output and in the
 *     checksum, even when the library internally swaps U and V (it takes V := the side with fewer
 *     vertices; on a tie the caller's orientation is kept).
 *   - Duplicate (u, v) pairs collapse to one edge.  Isolated vertices are in no
 *     biclique.  An empty graph enumerates to count 0, checksum 0.
 *   - The library never takes ownership of caller memory; it copies what it needs.
 */
#ifndef GMBE_H_
#define GMBE_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum {
  GMBE_OK = 0,
  GMBE_EINVAL = -1,       /* bad argument: NULL pointer, id >= n_u / n_v, bad option value */
  GMBE_ENOMEM = -2,       /* device allocation failed (nothing leaks, the graph stays valid) */
  GMBE_ECUDA = -3,        /* a CUDA runtime call or kernel failed */
  GMBE_EUNSUPPORTED = -4, /* input beyond implemented limits (n_edges >= 2^31, |U| or |V| >= 2^31) */
  GMBE_EINTERNAL = -5     /* a device-side capacity was exceeded (workspace too small) */
};

enum { GMBE_ORDER_DEGREE = 0 /* ascending degree, ties by id */,
       GMBE_ORDER_IDENTITY = 1 /* vertex id order; reproduces Fig 2 / Fig 5 */ };

typedef struct gmbe_graph gmbe_graph; /* opaque, owned by the library */

/* Options of gmbe_load_bipartite.  NULL = defaults.  Zero-initialised fields mean defaults. */
typedef struct {
  uint32_t struct_size;     /* sizeof(gmbe_load_opts) */
  int32_t device;           /* CUDA device ordinal, or -1 = the current device (opts == NULL) */
  void* cuda_stream;        /* cudaStream_t used for the build; NULL = library-owned stream */
  uint32_t edges_on_device; /* 1: edges_uv is a device pointer (e.g. torch int32 data_ptr()) */
  uint32_t order;           /* GMBE_ORDER_* */
} gmbe_load_opts;

/* Build the device-resident graph (steps a1-a2 of DESIGN.md): edge ingest, dedupe, orientation,
 * degree ordering, both-side CSR, degree / 2-hop bounds and the hash tables of the checksum.
 *   n_u, n_v   : sizes of the caller's vertex sets U and V (ids must be < n_u / < n_v)
 *   edges_uv   : n_edges (u, v) pairs, interleaved uint32 [u0, v0, u1, v1, ...]; host memory, or
 *                device memory if opts->edges_on_device.  Read during the call only.
 *   out        : receives the new graph handle (free with gmbe_free_graph).
 * Errors: EINVAL (NULL out, NULL edges with n_edges>0, id out of range), EUNSUPPORTED
 * (n_edges >= 2^31 or n_u, n_v >= 2^31), ENOMEM, ECUDA. */
int gmbe_load_bipartite(uint32_t n_u, uint32_t n_v, const uint32_t* edges_uv, uint64_t n_edges,
                        const gmbe_load_opts* opts, gmbe_graph** out);

typedef struct {
  uint64_t n_u, n_v;         /* caller's sizes */
  uint64_t n_edges_unique;   /* |E| after dedupe */
  uint32_t delta_u, delta_v; /* Δ(U), Δ(V) in the library's orientation (V = smaller side) */
  uint32_t wedge_bound_v;    /* max_v Σ_{u∈N(v)} |N(u)|  (> Δ2(V)) */
  uint32_t swapped;          /* 1 if the library's U is the caller's V */
  uint32_t order;            /* GMBE_ORDER_* used at load */
  uint32_t device;
} gmbe_graph_info;

int gmbe_graph_info_get(const gmbe_graph* g, gmbe_graph_info* out);
void gmbe_free_graph(gmbe_graph* g); /* NULL-safe */

/* Paper's node_buf bound (Sec 4.1): (3·Δ(V) + 2·Δ2(V)) · sizeof(int) bytes per
 * subtree procedure -- e.g. BookCrossing 13,601 / 53,915 -> 594,532 B ("595 KB").
 * Pure function, no device needed. */
uint64_t gmbe_node_buf_bound_bytes(uint64_t delta_v, uint64_t delta2_v);
/* Paper's per-subtree size without node reuse (Sec 3.1): Δ(V)·(Δ(V)+Δ2(V))·4 B. */
uint64_t gmbe_naive_alloc_bytes(uint64_t delta_v, uint64_t delta2_v);

/* Options of gmbe_enumerate.  NULL = defaults; zero-initialised fields mean the default noted. */
typedef struct {
  uint32_t struct_size;   /* sizeof(gmbe_opts); 0 = treat the struct as all-defaults */
  uint32_t no_prune;      /* 1 disables Thm 4.1 pruning (GMBE-W/O_PRUNE ablation) */
  uint32_t no_split;      /* 1 disables load-aware splitting (Alg 4 L17-26) */
  uint32_t bound_height;  /* split if min(|L|,|C|) > bound_height ...   (default 10; paper 20) */
  uint32_t bound_size;    /* ... and min(|L|,|C|)·|C| > bound_size       (default 500; paper 1500,
                             P:1175; retuned on B200 with scripts/sweep.py) */
  uint32_t warps_per_sm;  /* resident warps per SM of the persistent kernel (0 = auto) */
  uint32_t part_index;    /* root shard: enumerate the roots whose degree rank r satisfies */
  uint32_t part_count;    /*   r % part_count == part_index (0 = 1 part); shards partition the
                               output, so counts / checksums add (mod 2^64) across parts */
  uint32_t reserved0;     /* debug bits for tests / experiments (0 in production use) */
  uint32_t scheduler;     /* GMBE_SCHED_*: how root tasks map to the GPU (Sec 4.3):
                             TASK (0, default) = GMBE's load-aware task-centric scheme (Alg 4);
                             WARP (1) = GMBE-WARP, one warp per Alg 3 task, no splitting, one node
                             per warp step; BLOCK (2) = GMBE-BLOCK, one thread block per Alg 3 task,
                             no splitting, every node generated by the whole block.  The variants of
                             Sec 6.3 (Fig 8/9); the result and the canonical-tree counters are the
                             same in all three. */
  /* Optional bounded output (device-accessible memory: device or mapped pinned host).
   * Record = [|L|, |R|, L ids (caller U ids), R ids (caller V ids)], order within a record and of
   * records unspecified; out_offsets[i] = word offset of record i in out_ids.  A full buffer is
   * not an error: result.truncated = 1 while count / checksum stay complete; a record that did
   * not fit has out_offsets[i] = UINT64_MAX when i < out_offsets_cap. */
  uint64_t* out_offsets;
  uint64_t out_offsets_cap;
  uint32_t* out_ids;
  uint64_t out_ids_cap;
  /* Optional per-root counts (HOST memory, length = library-internal |V|): bicliques emitted under
   * each root vertex, indexed by the root's caller id on the library's V side. */
  uint64_t* per_root_count;
  /* Optional profiling (HOST memory, same indexing): SM clock cycles the warps spent on each root's
   * tree (root build + in-place search + its queued subtasks). */
  uint64_t* per_root_cycles;
  /* Optional profiling (HOST uint64_t[16]): SM cycles summed over warps per phase (names in the
   * Python binding's PHASES). */
  uint64_t* phase_cycles;
  /* Optional profiling timeline (DEVICE memory, timeline_cap uint64 words): word 0 = number of
   * records, then per root / task: [smid<<56 | kind<<48 | root rank, start ns, end ns,
   * nodes<<32 | min(|L_top|,65535)<<16 | min(|C_top|,65535)] (%globaltimer; kind 0 root, 1 split
   * subtask, 2 split descriptor) -- the active-SM timeline of PAPER.md Fig 4 / Fig 9. */
  uint64_t* timeline;
  uint64_t timeline_cap;
  /* Workspace (0 = auto): words of the per-warp dynamic region (root record, node stack; a caller-given
   * size is the first attempt's, see gmbe_result.retries); words
   * of the task pool (split subtasks and shared Γ columns; when it is exhausted work simply stays
   * with the warp that generated it); capacity of the task queue (entries). */
  uint64_t arena_words;
  uint64_t pool_words;
  uint64_t queue_cap;
  void* cuda_stream;      /* NULL = the graph's stream */
  /* B200 scheduling knobs (0 = default; both leave the result and the canonical-tree counters
   * unchanged): */
  uint32_t split_wide;    /* also split a task over a wide universe (|L| > 64 bits) when
                             |C|·⌈|L|/32⌉ >= split_wide (default 32): such nodes cost ~|L|/32 words
                             each, so even small subtrees are worth spreading over warps */
  uint32_t thr_min;       /* thread-level tier: jobs (<= 32 candidates over <= 64 universe bits)
                             with Σ_c (|N(c) ∩ L| - 1) >= thr_min run one subtree per lane
                             (default 16; UINT32_MAX disables the tier) */
  /* Dynamic cross-GPU root distribution (Sec 5: GPUs take
   * root tasks from one shared pool instead of a fixed split).  NULL = off.  Otherwise a
   * device-accessible uint64 counter shared by several concurrent gmbe_enumerate calls on replicas
   * of the SAME graph (same edges, same order; possibly on other GPUs or in other processes, see
   * gmbe_shared_cursor_*): every call draws positions of the graph's full root issue list from it
   * with system-scope atomics, so the union of the calls enumerates every root exactly once and
   * their counts / checksums add (mod 2^64) to the single-call result.  Requires part_count <= 1.
   * The counter must be 0 when the first call starts and must not be reused (or reset) before every
   * call sharing it has returned. */
  uint64_t* root_cursor;
  /* How part_index / part_count split the roots:
   *   GMBE_PART_INTERLEAVE (0): degree rank r % part_count == part_index;
   *   GMBE_PART_COST (1): cost-model LPT -- the roots in the issue order (root cost = its Alg 3
   *     wedge count Σ_{u∈N(v_s)} |N(u)|, heaviest first) dealt out in snake order (block b of
   *     part_count consecutive roots goes to parts 0..P-1 if b is even, P-1..0 if odd), the
   *     parallel form of greedy LPT on a sorted cost list.  Either way the parts partition the
   *     roots, so counts / checksums add (mod 2^64). */
  uint32_t part_mode;
  uint32_t root_chunk;    /* root positions a warp claims per atomic once past the first 1/8 (the
                             heavy head) of the issue list: 0 = default 1 (one root per atomic),
                             at most 32.  Fewer atomics on the (local or N1 shared) root cursor --
                             e.g. 16 for light-root graphs under N1; the result and the
                             canonical-tree counters do not depend on it. */
} gmbe_opts;

enum { GMBE_PART_INTERLEAVE = 0, GMBE_PART_COST = 1 };
enum { GMBE_SCHED_TASK = 0, GMBE_SCHED_WARP = 1, GMBE_SCHED_BLOCK = 2 };

typedef struct {
  uint64_t count;         /* maximal bicliques enumerated (this shard) */
  uint64_t checksum;      /* Σ h(L,R) mod 2^64 (this shard) */
  uint64_t n_written;     /* records written to the output buffer */
  uint64_t truncated;     /* 1 if the output buffer was too small */
  uint64_t roots_run;     /* roots not skipped by the Alg 3 L7 check */
  uint64_t nodes;         /* generated, unpruned child nodes (canonical tree; roots excluded) */
  uint64_t nonmax;        /* nodes failing the maximality check */
  uint64_t algo_bytes_cand; /* wedge + candidate-scan algorithmic bytes of the canonical tree
                               (the Q term is not computed on the GPU) */
  uint64_t splits;        /* nodes expanded in split mode */
  uint64_t tasks;         /* subtasks enqueued */
  uint64_t donations;     /* subtasks donated to idle warps (dynamic load balancing) */
  double kernel_ms;       /* device time of the enumeration kernel (CUDA events; the last run) */
  uint64_t retries;       /* re-runs after a per-warp workspace overflow (degrade path: larger per-warp
                             regions -- a caller-given arena_words is replaced by the automatic size, an
                             automatic size goes to fewer resident warps, 24 -> 16 -> 8 per SM; not for
                             streaming calls) */
} gmbe_result;

/* Enumerate all maximal bicliques of g (or of one root shard).  Synchronous: returns after the
 * result is on the host.  Concurrent calls on one graph must use distinct streams.
 * Errors: EINVAL (NULL g/out, part_index >= part_count), ENOMEM, ECUDA, EINTERNAL (a per-warp workspace
 * still overflowed after the degrade path's re-runs). */
int gmbe_enumerate(const gmbe_graph* g, const gmbe_opts* opts, gmbe_result* out);

/* Streaming output (the problem statement asks to *enumerate* all maximal
 * bicliques, Output() of Alg 1/2): every record [|L|, |R|, L ids (caller U ids),
 * R ids (caller V ids)] is delivered exactly once to `sink`, in batches of whole records
 * (n_words words holding n_records records, order unspecified), on the calling thread while the
 * kernel runs.  The kernel writes into a ring of ring_words 32-bit words (rounded up to a power of
 * two, at least 4x the largest possible record; 0 = 16 Mi words) in mapped pinned host memory and
 * waits when it is full (back-pressure), so any output size streams through a bounded buffer.
 * `words` is valid only during the call.  count / checksum / counters are as in gmbe_enumerate;
 * result.n_written = records delivered (== count).  opts must not carry out_offsets / out_ids.
 * Errors: as gmbe_enumerate; EINVAL (NULL sink, bounded buffers given, the sink returned non-zero
 * -- the remaining records are drained but not delivered).  A slow sink only slows the kernel down
 * (producers wait for room; there is no timeout), so the sink must eventually return. */
typedef int (*gmbe_sink_fn)(const uint32_t* words, uint64_t n_words, uint64_t n_records, void* user);
int gmbe_enumerate_stream(const gmbe_graph* g, const gmbe_opts* opts, gmbe_sink_fn sink, void* user,
                          uint64_t ring_words, gmbe_result* out);

/* Shared root cursors for gmbe_opts.root_cursor.  A cursor block holds
 * GMBE_CURSOR_SLOTS independent uint64 counters in device memory of one GPU (the owner); other
 * processes map it through CUDA IPC (peer access over NVLink / NVSwitch is enabled on open, or the
 * same device in another process).  Rotating slots lets consecutive calls run with a single
 * synchronisation between them: call k uses slot k % SLOTS and the owner zeroes slot (k+1) % SLOTS
 * before call k starts.
 *   Slot i is the counter at dptr + 16·i (one 128-byte line each).
 *   create : cudaMalloc on `device` (zeroed, synchronous); *dptr = device pointer of slot 0;
 *            ipc_handle (GMBE_IPC_HANDLE_BYTES bytes, may be NULL) receives the export handle.
 *   open   : map another process's block on `device` (the current GPU of this process);
 *            *dptr = this process's pointer to slot 0.  EINVAL for NULL args, ECUDA if CUDA IPC or
 *            peer access is unavailable (the caller falls back to static parts).
 *   reset  : zero slot `slot` of the block at dptr on `cuda_stream` (NULL = legacy) and wait for it
 *            (synchronous, so the zero is visible to every stream and process when it returns);
 *            call with the device that owns (or maps) dptr current.  EINVAL: NULL dptr, bad slot.
 *   close  : unmap (opened) or free (created, owner = 1) the block.  NULL-safe. */
enum { GMBE_CURSOR_SLOTS = 16, GMBE_IPC_HANDLE_BYTES = 64 };
int gmbe_shared_cursor_create(int32_t device, uint64_t** dptr, void* ipc_handle);
int gmbe_shared_cursor_open(const void* ipc_handle, int32_t device, uint64_t** dptr);
int gmbe_shared_cursor_reset(uint64_t* dptr, uint32_t slot, void* cuda_stream);
void gmbe_shared_cursor_close(uint64_t* dptr, int32_t owner);

/* gmbe_enumerate keeps its device workspace (node-stack arenas, task slabs, queues) in a
 * per-device pool for reuse by later calls.  This frees the idle workspaces of g's device.
 * NULL-safe. */
void gmbe_release_workspace(const gmbe_graph* g);

/* Number of this library's own kernels launched so far in this process (all devices); CUB
 * primitives used by the graph build are not counted. */
uint64_t gmbe_kernel_launch_count(void);

const char* gmbe_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* GMBE_H_ */
