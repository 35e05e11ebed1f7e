// gmbe_enum.cu -- the persistent sm_100a enumeration kernel (DESIGN.md steps a3-a8).
//
// One warp = one "procedure".  Each warp loops (Alg 4):
//   1. dequeue a split subtask from the global task queue, else
//   2. take the next root v_s from an atomic cursor (heavy roots first) and build its root node
//      (Alg 3 / Alg 4 L6-13): wedge scan of N2(v_s) into a per-warp hash table with the
//      local neighbourhood sizes k(v) = |N(v) ∩ L_r|; R_r = {v : k(v) = |L_r|}; the root is skipped
//      unless v_s is the earliest vertex of R_r (Alg 3 L7); later-ordered partial neighbours are the
//      candidates C_r; emission of (L_r, R_r);
//   3. either split the task's top node into subtasks (Alg 4 L17-26, heavy-node estimate
//      min(|L|,|C|)·|C| > bound_size and min(|L|,|C|) > bound_height) or walk its
//      subtree depth-first (Alg 2) on a per-warp reusable node stack (Sec 4.1);
//   4. exit when all roots are issued and no task is queued or running.
//
// Node representation: all sets of one task are bitmaps over the task's
// universe (the root's L_r).  A node record holds its L mask and one entry per live candidate
//     entry = [row[0..W) = N(c) ∩ L_node as bits, id (rank), k = |N(c) ∩ L_node|]
// so child generation (Alg 2 L8-13) is AND + POPC over rows and Thm 4.1 compares k' with k.
// Candidates pruned by Thm 4.1 are compacted out of the parent in the same pass.  Like the paper
// no excluded set is stored: maximality (Alg 2 L14, "R' == Γ(L')") is decided by
// counting Γ(L') = ∩_{u∈L'} N(u) over N(u*) for the lowest-degree u* ∈ L' (|Γ(L')| = |R'| iff
// maximal, since R' ⊆ Γ(L')); for |L'| = 1 this is just deg(u*) == |R'|.
#include <algorithm>
#include <atomic>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include <cub/cub.cuh>

#include "gmbe_internal.cuh"

namespace {

constexpr uint32_t kHdr = 8;  // node record header words
constexpr uint32_t kNone = 0xffffffffu;
constexpr uint32_t kSmemSort = 256;  // per-warp shared-memory sort capacity (keys)
constexpr unsigned long long kCTag = 1ull << 63;  // table value tag of a candidate (entry index)

// Control block: every hot atomic on its own 128-byte line, so polling warps do not serialise the
// atomics of working warps.
struct alignas(128) Line {
  unsigned long long v;
  unsigned long long pad[15];
};
struct Ctrl {
  Line root_cursor, q_head, q_tail, q_avail, pending, pool_next;
  Line hungry;  // warps idle-waiting for work (all roots issued, queue empty): triggers donation
  unsigned long long count, checksum, roots_run, nodes, nonmax, abytes, splits, tasks, donations;
  unsigned long long out_rec, out_ids;
  unsigned long long phase[16];
  unsigned int truncated, error;
  unsigned long long stream_tail;  // streaming output: largest consumer position seen by a producer
};

static_assert(sizeof(Ctrl) == 1152, "bench.py reports sizeof(Ctrl) as the per-step D2H / H2D control bytes");

enum : unsigned int { kErrArena = 1, kErrStream = 2 };

struct Params {
  DevGraph g;
  uint32_t n_roots;  // roots of this shard
  const uint32_t* issue;  // the shard's roots (ranks) in issue order: most wedges first
  uint32_t part_index, part_count;
  uint32_t prune, split, bound_height, bound_size;
  uint32_t hu_side;   // checksum side of the library's U vertices (0 = caller U)
  uint32_t* arena;    // per warp: keys[tmax] | vals[tmax] (u64) | occ[omax] | dynamic
  uint64_t arena_words;
  uint64_t col_budget;  // max words of a root's Γ-column store
  uint32_t tmax, omax, bmax;   // table slots, occupied-list words, rank-bitmap words
  uint32_t* rbuf;     // per-warp R-list stack (only with output)
  uint32_t rbuf_words;
  uint32_t* pool;     // task pool: subtasks and shared Γ columns, bump-allocated per call
  uint64_t pool_words;
  uint32_t* tq;       // task ring: pool offsets (16-byte units) + 1; 0 = empty slot
  uint32_t qmask, qcap;
  Ctrl* ctrl;
  unsigned long long* out_offsets;
  uint64_t out_offsets_cap;
  uint32_t* out_ids;
  uint64_t out_ids_cap;
  uint32_t* sring;                              // streaming output ring (mapped host memory) or null
  unsigned long long smask;                     // ring words - 1 (power of two)
  const unsigned long long* stail;              // host-written consumer position (mapped)
  unsigned long long* per_root;
  unsigned long long* per_root_cycles;
  uint32_t profile;
  uint32_t debug;  // opts.reserved0 bits (tests / experiments): 4 = no donation, 8 = donate whenever possible,
                   // 16 = no thread-level tier (run_thr), 32 = path statistics into ctrl.phase,
                   // 64 = no suffix-mode roots, 128 = every root in suffix mode, 256 = no dense-mode roots,
                   // 512 = dense mode whenever the table can hold it, 1024 = build the roots only
                   // (timing experiments: no subtree is walked, the result is incomplete),
                   // 2048 = no register-resident tiny-root build (run_root_tiny), 4096 = no sort-mode
                   // roots, 8192 = sort mode for every small-universe full-scan root above the smem table
  uint32_t donate;  // dynamic donation to idle warps (donate_reg)
  uint32_t thr_min_est;  // run_thr tier threshold on Σ_c (k_c - 1) (opts.thr_min)
  uint32_t split_wide;   // wide-universe split threshold on |C|·⌈|L|/32⌉ (opts.split_wide)
  uint32_t chunk, chunk_from;  // root claims: `chunk` issue positions per atomic past position chunk_from
  uint32_t sort_min;           // sort-mode roots from this many wedges (kNone: off for this call)
  unsigned long long* timeline;  // profiling: [cursor, then (smid<<56|kind<<48|root), t0, t1, info]*
  uint64_t timeline_cap;
  unsigned long long* shared_cursor;  // N1: root cursor shared across GPUs / processes (opts.root_cursor)
};

// Per-warp result counters, one per lane (lane k holds counter k, in Ctrl's field order): a warp-uniform
// update is one predicated add, and the nine counters cost one register pair instead of nine.
enum : uint32_t { kAcCount, kAcChecksum, kAcRootsRun, kAcNodes, kAcNonmax, kAcAbytes, kAcSplits, kAcTasks,
                  kAcDonations, kAcN };
struct Acc {
  unsigned long long v;
  // add the warp-uniform value x to counter k (called by every lane of the warp)
  __device__ __forceinline__ void add(uint32_t k, unsigned long long x) {
    uint32_t l;
    asm("mov.u32 %0, %%laneid;" : "=r"(l));
    if (l == k) v += x;
  }
  // counter k (a warp-wide shuffle: every lane must call it)
  __device__ __forceinline__ unsigned long long get(uint32_t k) const {
    const uint32_t lo = __shfl_sync(0xffffffffu, (uint32_t)v, k), hi = __shfl_sync(0xffffffffu, (uint32_t)(v >> 32), k);
    return ((unsigned long long)hi << 32) | lo;
  }
#ifdef GMBE_PROFILE
  unsigned long long ph[16];  // profiling build only: SM cycles per phase (opts.phase_cycles)
  long long t0;
#endif
};
// Phase profiling (libgmbe_prof.so, built with -DGMBE_PROFILE; compiled out of libgmbe.so):
// 0 root wedge pass, 1 classify, 2 sort, 3 root finish, 4 candidate scan, 5 maximality, 6 emit,
// 7 task queue, 8.. root sub-phases (names in the Python binding's PHASES)
#ifdef GMBE_PROFILE
#define PH_START(A) \
  if (P.profile) (A).t0 = clock64()
#define PH_STOP(A, k)                                   \
  if (P.profile) {                                      \
    const long long _t = clock64();                     \
    (A).ph[k] += (unsigned long long)(_t - (A).t0);     \
    (A).t0 = _t;                                        \
  }
#else
#define PH_START(A) \
  do {              \
  } while (0)
#define PH_STOP(A, k) \
  do {                \
  } while (0)
#endif

// per-task constants (warp-uniform)
struct TaskCtx {
  const uint32_t* map;  // universe bit j -> library U id
  uint32_t W, W4, E;    // words per row, padded L-mask words, entry stride
  uint32_t root;        // rank of the root vertex
  uint32_t* rlist;      // R-list stack (output only)
  // Γ index of the root (maximality count without binary searches), one of:
  //   gx  (universe <= 64 bits): [nx, l, -, -] | xrow u64[nx] (row of each X2 vertex x over the
  //        universe) | xid u32[r4(nx)] (rank of x) | coff u32[l+1] | cx u32[] (X2 indices adjacent
  //        to universe vertex j)
  //   cols (larger universes): cols[j*ncw ..] = bitmap of the X2 vertices adjacent to vertex j
  // X2 = the root's 2-hop vertices adjacent to >= 2 universe vertices (the only ones that can cover
  // an L' with |L'| >= 2).
  // or neither (count Γ by binary search over the adjacency lists).
  const uint32_t* gx;
  const uint32_t* cols;
  uint32_t ncw;
  uint32_t auxref;      // pool offset (16-byte units) + 1 of gx / cols when shared with subtasks, else 0
  // lane-resident copies for universes <= 64 bits (universe vertices lane and lane + 32), filled by
  // small_task_init: Γ-list offsets / lengths and the checksum hashes of the universe vertices
  uint32_t go0, go1, gl0, gl1;
  uint32_t dg0, dg1;          // degrees of the universe vertices (run_thr's |L'| = 1 test)
  unsigned long long hu0, hu1;
  uint32_t nx;                // gx: |X2|; <= 64: the X2 rows are lane-resident in xr0 / xr1
  unsigned long long xr0, xr1;
  const uint32_t* gxl;  // gx: base of the per-vertex 2-hop lists
};

// per-warp memory
// Code size: k_enum's hot paths are inlined; per-root / per-task entry points can be kept out of
// line (GMBE_NI_* = 1) so the instruction footprint stays within the SM's instruction caches.
#ifndef GMBE_NI_ROOT
#define GMBE_NI_ROOT 0
#endif
#ifndef GMBE_NI_DISPATCH
#define GMBE_NI_DISPATCH 0
#endif
#ifndef GMBE_NI_REG
#define GMBE_NI_REG 0
#endif
#ifndef GMBE_NI_DONATE_THR
#define GMBE_NI_DONATE_THR 0  // 1: the thread tier's rare paths (cross-warp donation, records) out of line
#endif
#ifndef GMBE_NI_GAMMA
#define GMBE_NI_GAMMA 0
#endif
#define GMBE_NI_IF(x) GMBE_NI_IF_(x)
#define GMBE_NI_IF_(x) GMBE_NI_IF_##x
#define GMBE_NI_IF_0
#define GMBE_NI_IF_1 __noinline__

struct WarpMem {
  uint32_t* keys;               // clean hash table keys (EMPTY)
  unsigned long long* vals;     // clean hash table values (0)
  uint32_t* occ;                // occupied slots of the current root
  uint32_t* bits;               // clean bitmap over the ranks (dense-mode roots' occupied ranks)
  uint32_t* skeys;              // the shared-memory table (kSmemTable slots)
  unsigned long long* svals;
  uint32_t* socc;
  uint32_t* dyn;                // dynamic region: root record, node stack, scratch
  uint32_t* dyn_end;
  uint32_t* rbuf;
  unsigned long long* sm_sort;  // this warp's shared-memory sort slice
};

__device__ __forceinline__ uint32_t lane_id() {
  uint32_t l;
  asm("mov.u32 %0, %%laneid;" : "=r"(l));  // non-volatile: the compiler may CSE it
  return l;
}
__device__ __forceinline__ uint32_t lanemask_lt() { return (1u << lane_id()) - 1u; }
__device__ __forceinline__ uint32_t r4(uint32_t x) { return (x + 3u) & ~3u; }
__device__ __forceinline__ uint32_t* align4(uint32_t* p) {
  return (uint32_t*)(((uintptr_t)p + 15) & ~(uintptr_t)15);
}
__device__ __forceinline__ uint32_t warp_sum(uint32_t x) { return __reduce_add_sync(GMBE_FULL, x); }
__device__ __forceinline__ unsigned long long warp_sum64(unsigned long long x) {
  for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(GMBE_FULL, x, o);
  return x;
}
// 64-bit warp sum with three 32-bit REDUX ops (21/21/22-bit limbs cannot overflow over 32 lanes)
__device__ __forceinline__ unsigned long long warp_sum64r(unsigned long long x) {
  const uint32_t a = __reduce_add_sync(GMBE_FULL, (uint32_t)(x & 0x1fffffull));
  const uint32_t b = __reduce_add_sync(GMBE_FULL, (uint32_t)((x >> 21) & 0x1fffffull));
  const uint32_t c = __reduce_add_sync(GMBE_FULL, (uint32_t)(x >> 42));
  return (unsigned long long)a + ((unsigned long long)b << 21) + ((unsigned long long)c << 42);
}
// sum over aligned groups of lpe lanes (lpe a power of two <= 32; runtime, one code copy)
__device__ __forceinline__ uint32_t group_sum(uint32_t x, uint32_t lpe) {
  for (uint32_t o = lpe >> 1; o; o >>= 1) x += __shfl_xor_sync(GMBE_FULL, x, o);
  return x;
}
__device__ __forceinline__ uint32_t next_pow2(uint32_t x) { return x <= 1 ? 1u : 1u << (32 - __clz(x - 1)); }

__device__ __forceinline__ bool fits(const Params& P, const uint32_t* p, const uint32_t* end) {
  if (p <= end) return true;
  if (lane_id() == 0) atomicOr(&P.ctrl->error, kErrArena);
  return false;
}

// ---------------------------------------------------------------- per-warp hash table (a3)
// Two instances per warp: a small one in shared memory (roots with <= kSmemTable/2 wedges, i.e.
// almost every root of the light-tailed shapes) and the large one in the warp's HBM arena.  Both are
// accessed through generic pointers: table reads are volatile (the slots are written by atomics, so
// a global table must not be read through a stale L1 line), atomics resolve the address space.
#ifndef GMBE_SMEM_TABLE
#define GMBE_SMEM_TABLE 128
#endif
constexpr uint32_t kSmemTable = GMBE_SMEM_TABLE;
__device__ __forceinline__ uint32_t ldv(const uint32_t* p) { return *(const volatile uint32_t*)p; }
__device__ __forceinline__ unsigned long long ldv(const unsigned long long* p) {
  return *(const volatile unsigned long long*)p;
}
__device__ __forceinline__ uint32_t ht_hash(uint32_t v, uint32_t shift) { return (v * 2654435761u) >> shift; }

// warp-cooperative insert of v (lanes with act); new slots are appended to occ so the table can
// be cleaned in O(occupied).  Returns the slot.
__device__ __forceinline__ uint32_t ht_insert_warp(uint32_t* keys, uint32_t shift, uint32_t mask, uint32_t v,
                                                   bool act, uint32_t* occ, uint32_t& nocc) {
  uint32_t h = act ? ht_hash(v, shift) : 0, slot = kNone;
  bool pend = act;
  while (__any_sync(GMBE_FULL, pend)) {
    bool ins = false;
    if (pend) {
      // one round trip per probe: a CAS on a slot that already holds v just returns v
      const uint32_t old = atomicCAS(keys + h, GMBE_EMPTY, v);
      if (old == GMBE_EMPTY || old == v) {
        slot = h;
        pend = false;
        ins = old == GMBE_EMPTY;
      } else {
        h = (h + 1) & mask;
      }
    }
    const uint32_t b = __ballot_sync(GMBE_FULL, ins);
    if (ins) occ[nocc + __popc(b & lanemask_lt())] = h;
    nocc += __popc(b);
  }
  return slot;
}
__device__ __forceinline__ uint32_t ht_find(const uint32_t* keys, uint32_t shift, uint32_t mask, uint32_t v) {
  uint32_t h = ht_hash(v, shift);
  while (true) {
    const uint32_t k = ldv(keys + h);
    if (k == v) return h;
    if (k == GMBE_EMPTY) return kNone;
    h = (h + 1) & mask;
  }
}

// first position in the rank-sorted list a[0, n) holding a rank > r
__device__ __forceinline__ uint32_t upper_rank(const uint32_t* a, uint32_t n, uint32_t r) {
  uint32_t lo = 0, hi = n;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (__ldg(a + mid) <= r) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

// Visit every wedge (i, v): u_i = L[i], v ∈ N(u_i), load-balanced across the warp.
// f(i, v, active) is called by all 32 lanes each step.  after != kNone: only the wedges to ranks
// > after (a suffix of each rank-sorted list).
#ifndef GMBE_WEDGE_UNROLL
#define GMBE_WEDGE_UNROLL 1
#endif
template <class F>
__device__ __forceinline__ void for_each_wedge(const DevGraph& g, const uint32_t* L, uint32_t l, F f,
                                               uint32_t after = 0xffffffffu) {
  const uint32_t lane = lane_id();
  for (uint32_t b = 0; b < l; b += 32) {
    uint32_t i = b + lane, beg = 0, deg = 0;
    if (i < l) {
      const uint32_t u = L[i];
      beg = g.off_u[u];
      deg = g.off_u[u + 1] - beg;
      if (after != 0xffffffffu) {
        const uint32_t s = upper_rank(g.adj_u + beg, deg, after);
        beg += s;
        deg -= s;
      }
    }
    uint32_t inc = deg;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t t = __shfl_up_sync(GMBE_FULL, inc, o);
      if (lane >= (uint32_t)o) inc += t;
    }
    const uint32_t total = __shfl_sync(GMBE_FULL, inc, 31);
    const uint32_t excl = inc - deg;
    // GMBE_WEDGE_UNROLL chunks of 32 wedges per step (knob; 1 = default, 2/4/8 measured slower at
    // N=1 and no better for 1/8 shards, profiles/r01_wedge_unroll_ab.txt): all their loads are in flight
    // before the first callback (a lone heavy root is one warp's latency chain otherwise); the
    // callbacks then run in the original chunk order, so the result is unchanged
    for (uint32_t base = 0; base < total; base += 32 * GMBE_WEDGE_UNROLL) {
      uint32_t vq[GMBE_WEDGE_UNROLL], iq[GMBE_WEDGE_UNROLL];
#pragma unroll
      for (int q = 0; q < GMBE_WEDGE_UNROLL; q++) {
        const uint32_t p = base + 32 * q + lane;
        uint32_t lo = 0;
#pragma unroll
        for (int st = 16; st; st >>= 1) {
          const uint32_t cand = lo + st;
          const uint32_t e = __shfl_sync(GMBE_FULL, excl, cand & 31);
          if (cand < 32 && e <= p) lo = cand;
        }
        const uint32_t ob = __shfl_sync(GMBE_FULL, beg, lo);
        const uint32_t oe = __shfl_sync(GMBE_FULL, excl, lo);
        vq[q] = p < total ? g.adj_u[ob + p - oe] : 0;
        iq[q] = b + lo;
      }
#pragma unroll
      for (int q = 0; q < GMBE_WEDGE_UNROLL; q++)
        if (base + 32 * q < total) f(iq[q], vq[q], base + 32 * q + lane < total);
    }
  }
}

// ---------------------------------------------------------------- warp sorts
// bitonic sort of a[0..next_pow2(n)) (padded with ~0) by one warp
__device__ void warp_bitonic64(unsigned long long* a, uint32_t n) {
  const uint32_t lane = lane_id();
  const uint32_t N = next_pow2(n);
  for (uint32_t i = n + lane; i < N; i += 32) a[i] = ~0ull;
  __syncwarp();
  for (uint32_t k = 2; k <= N; k <<= 1) {
    for (uint32_t j = k >> 1; j > 0; j >>= 1) {
      for (uint32_t t = lane; t < N / 2; t += 32) {
        const uint32_t i = ((t & ~(j - 1)) << 1) | (t & (j - 1));
        const uint32_t p = i + j;
        const unsigned long long x = a[i], y = a[p];
        if ((x > y) == ((i & k) == 0)) {
          a[i] = y;
          a[p] = x;
        }
      }
      __syncwarp();
    }
  }
}
// register bitonic network: lane holds x; returns the lane-th smallest of the 32 values
__device__ __forceinline__ unsigned long long warp_sort32(unsigned long long x) {
  const uint32_t lane = lane_id();
#pragma unroll
  for (uint32_t k = 2; k <= 32; k <<= 1) {
#pragma unroll
    for (uint32_t j = k >> 1; j > 0; j >>= 1) {
      const unsigned long long y = __shfl_xor_sync(GMBE_FULL, x, j);
      const bool up = (lane & k) == 0, lower = (lane & j) == 0;
      x = (lower == up) ? (x < y ? x : y) : (x < y ? y : x);
    }
  }
  return x;
}
// one stable LSD radix pass by one warp: dst = src sorted by bits [shift, shift + dbits) (dbits <= 8),
// histogram in shared memory (hist: 256 words)
__device__ void warp_radix_pass(const unsigned long long* src, unsigned long long* dst, uint32_t n, uint32_t shift,
                                uint32_t dbits, uint32_t* hist) {
  const uint32_t lane = lane_id(), nb = 1u << dbits;
  for (uint32_t i = lane; i < nb; i += 32) hist[i] = 0;
  __syncwarp();
  for (uint32_t b = 0; b < n; b += 32) {
    const uint32_t j = b + lane;
    const uint32_t d = j < n ? (uint32_t)(src[j] >> shift) & (nb - 1) : nb;
    const uint32_t peers = __match_any_sync(GMBE_FULL, d);
    if (j < n && lane == __ffs(peers) - 1) hist[d] += __popc(peers);
    __syncwarp();
  }
  // exclusive scan of hist (lane t owns the nb/32 consecutive entries of chunk t)
  const uint32_t per = (nb + 31) / 32;
  uint32_t loc = 0;
  for (uint32_t k = 0; k < per; k++)
    if (lane * per + k < nb) loc += hist[lane * per + k];
  uint32_t inc = loc;
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t t = __shfl_up_sync(GMBE_FULL, inc, o);
    if (lane >= (uint32_t)o) inc += t;
  }
  uint32_t run = inc - loc;
  __syncwarp();
  for (uint32_t k = 0; k < per; k++)
    if (lane * per + k < nb) {
      const uint32_t c = hist[lane * per + k];
      hist[lane * per + k] = run;
      run += c;
    }
  __syncwarp();
  for (uint32_t b = 0; b < n; b += 32) {
    const uint32_t j = b + lane;
    const unsigned long long x = j < n ? src[j] : 0ull;
    const uint32_t d = j < n ? (uint32_t)(x >> shift) & (nb - 1) : nb;
    const uint32_t peers = __match_any_sync(GMBE_FULL, d);
    if (j < n) dst[hist[d] + __popc(peers & lanemask_lt())] = x;
    __syncwarp();
    if (j < n && lane == __ffs(peers) - 1) hist[d] += __popc(peers);
    __syncwarp();
  }
}
// the same pass over 32-bit keys, digits of up to 9 bits (hist: 1 << dbits words)
__device__ void warp_radix_pass32(const uint32_t* src, uint32_t* dst, uint32_t n, uint32_t shift, uint32_t dbits,
                                  uint32_t* hist) {
  const uint32_t lane = lane_id(), nb = 1u << dbits;
  for (uint32_t i = lane; i < nb; i += 32) hist[i] = 0;
  __syncwarp();
  for (uint32_t b = 0; b < n; b += 64) {  // two chunks of loads in flight
    const uint32_t j0 = b + lane, j1 = b + 32 + lane;
    const uint32_t x0 = j0 < n ? src[j0] : 0u, x1 = j1 < n ? src[j1] : 0u;
#pragma unroll
    for (int h = 0; h < 2; h++) {
      const uint32_t j = h ? j1 : j0;
      const uint32_t d = j < n ? ((h ? x1 : x0) >> shift) & (nb - 1) : nb;
      const uint32_t peers = __match_any_sync(GMBE_FULL, d);
      if (j < n && lane == __ffs(peers) - 1) hist[d] += __popc(peers);
      __syncwarp();
    }
  }
  const uint32_t per = (nb + 31) / 32;
  uint32_t loc = 0;
  for (uint32_t k = 0; k < per; k++)
    if (lane * per + k < nb) loc += hist[lane * per + k];
  uint32_t inc = loc;
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t t = __shfl_up_sync(GMBE_FULL, inc, o);
    if (lane >= (uint32_t)o) inc += t;
  }
  uint32_t run = inc - loc;
  __syncwarp();
  for (uint32_t k = 0; k < per; k++)
    if (lane * per + k < nb) {
      const uint32_t c = hist[lane * per + k];
      hist[lane * per + k] = run;
      run += c;
    }
  __syncwarp();
  for (uint32_t b = 0; b < n; b += 64) {
    const uint32_t j0 = b + lane, j1 = b + 32 + lane;
    const uint32_t x0 = j0 < n ? src[j0] : 0u, x1 = j1 < n ? src[j1] : 0u;
#pragma unroll
    for (int h = 0; h < 2; h++) {
      const uint32_t j = h ? j1 : j0, x = h ? x1 : x0;
      const uint32_t d = j < n ? (x >> shift) & (nb - 1) : nb;
      const uint32_t peers = __match_any_sync(GMBE_FULL, d);
      if (j < n) dst[hist[d] + __popc(peers & lanemask_lt())] = x;
      __syncwarp();
      if (j < n && lane == __ffs(peers) - 1) hist[d] += __popc(peers);
      __syncwarp();
    }
  }
}
// sort n keys in a[0..n) (room for next_pow2(n)); keys above kSmemSort with a scratch tmp[0..n)
// and key_bits (significant high bits, keys compared on [64 - key_bits, 64) and then low bits
// irrelevant -- the callers' keys are unique in their high part) use an LSD radix sort
__device__ void warp_sort_keys(unsigned long long* a, uint32_t n, unsigned long long* smem,
                               unsigned long long* tmp = nullptr, uint32_t hi_bits = 0) {
  const uint32_t lane = lane_id();
  if (n <= 1) return;
  if (n <= 32) {
    const unsigned long long x = warp_sort32(lane < n ? a[lane] : ~0ull);
    __syncwarp();
    if (lane < n) a[lane] = x;
    __syncwarp();
    return;
  }
  if (smem && next_pow2(n) <= kSmemSort) {
    for (uint32_t j = lane; j < n; j += 32) smem[j] = a[j];
    __syncwarp();
    warp_bitonic64(smem, n);
    for (uint32_t j = lane; j < n; j += 32) a[j] = smem[j];
    __syncwarp();
    return;
  }
  if (smem && tmp && hi_bits) {  // keys = (unique value < 2^hi_bits) << 32 | payload
    const uint32_t passes = hi_bits <= 16 ? 2u : 4u, dbits = (hi_bits + passes - 1) / passes;
    for (uint32_t p = 0; p < passes; p++)
      warp_radix_pass(p & 1 ? tmp : a, p & 1 ? a : tmp, n, 32 + p * dbits, dbits, (uint32_t*)smem);
    return;
  }
  warp_bitonic64(a, n);
}

// ---------------------------------------------------------------- task pool and queue (a7)
__device__ __forceinline__ unsigned long long ld_volatile(const unsigned long long* p) {
  return *(volatile const unsigned long long*)p;
}
// Bump-allocate `words` (multiple of 4) from the task pool; returns the offset in 16-byte units,
// or kNone when the pool is exhausted (the caller then keeps the work in place).
__device__ uint32_t pool_alloc(const Params& P, uint64_t words) {
  unsigned long long off = 0;
  if (lane_id() == 0) off = atomicAdd(&P.ctrl->pool_next.v, (unsigned long long)words);
  off = __shfl_sync(GMBE_FULL, off, 0);
  return off + words <= P.pool_words ? (uint32_t)(off >> 2) : kNone;
}
__device__ __forceinline__ uint32_t* pool_ptr(const Params& P, uint32_t off16) { return P.pool + 4ull * off16; }
// is there room in the task ring (with a margin for concurrent producers)?
__device__ bool queue_room(const Params& P) {
  uint32_t ok = 0;
  if (lane_id() == 0) {
    const unsigned long long t = ld_volatile(&P.ctrl->q_tail.v), h = ld_volatile(&P.ctrl->q_head.v);
    ok = t - h + 8192 < P.qcap;
  }
  return __shfl_sync(GMBE_FULL, ok, 0) != 0;
}
// publish a task (one lane): pending += 1, then the slot, then the availability count
__device__ void queue_push(const Params& P, uint32_t off16) {
  atomicAdd(&P.ctrl->pending.v, 1ull);
  const unsigned long long t = atomicAdd(&P.ctrl->q_tail.v, 1ull);
  uint32_t* slot = P.tq + (t & P.qmask);
  while (atomicCAS(slot, 0u, off16 + 1) != 0u) __nanosleep(64);
  atomicAdd(&P.ctrl->q_avail.v, 1ull);
}
// take a task (one lane): reserve through the availability count (fetch-add, no CAS storms), then
// claim the next ticket and wait for its slot.  Returns kNone if nothing is available.
__device__ uint32_t queue_pop(const Params& P) {
  if ((long long)ld_volatile(&P.ctrl->q_avail.v) <= 0) return kNone;
  if ((long long)atomicAdd(&P.ctrl->q_avail.v, ~0ull) <= 0) {
    atomicAdd(&P.ctrl->q_avail.v, 1ull);
    return kNone;
  }
  const unsigned long long h = atomicAdd(&P.ctrl->q_head.v, 1ull);
  uint32_t* slot = P.tq + (h & P.qmask);
  uint32_t x;
  while ((x = atomicExch(slot, 0u)) == 0u) __nanosleep(32);
  return x - 1;
}
// task record: [0]=W [1]=map length [2]=root rank [3]=R length [4]=node offset [5]=auxref
//              [6]=column words [7]=aux kind (0 none, 1 cols, 2 gx) | map | R list | node record
__device__ __forceinline__ uint32_t task_node_off(uint32_t lmap, uint32_t rlen) { return kHdr + r4(lmap) + r4(rlen); }
// Copy the node record `rec` (words) into a new self-contained subtask and publish it (Alg 4 L25).
// Returns false (nothing published) if the pool or the queue is full.
__device__ bool task_publish(const Params& P, const TaskCtx& T, uint32_t lmap, uint32_t rlen, const uint32_t* rec,
                             uint32_t words, Acc& A) {
  const uint32_t lane = lane_id();
  if (!queue_room(P)) return false;
  const uint32_t node_off = task_node_off(lmap, T.rlist ? rlen : 0);
  const uint32_t off16 = pool_alloc(P, r4(node_off + words));
  if (off16 == kNone) return false;
  uint32_t* s = pool_ptr(P, off16);
  for (uint32_t j = lane; j < lmap; j += 32) s[kHdr + j] = T.map[j];
  if (T.rlist)
    for (uint32_t j = lane; j < rlen; j += 32) s[kHdr + r4(lmap) + j] = T.rlist[j];
  for (uint32_t j = lane; j < words; j += 32) s[node_off + j] = rec[j];
  __syncwarp();
  if (lane == 0) {
    s[0] = T.W;
    s[1] = lmap;
    s[2] = T.root;
    s[3] = T.rlist ? rlen : 0;
    s[4] = node_off;
    s[5] = T.auxref;
    s[6] = T.ncw;
    s[7] = T.auxref ? (T.gx ? 2u : 1u) : 0u;
    s[node_off + 3] = 0;      // next candidate
    s[node_off + 4] = kNone;  // no parent: top of its task
  }
  A.add(kAcTasks, 1);
  __threadfence();  // release the task before it becomes visible in the queue
  __syncwarp();
  if (lane == 0) queue_push(P, off16);
  return true;
}

// ---------------------------------------------------------------- emission (a8)
__device__ __forceinline__ unsigned long long hash_u(const Params& P, uint32_t u) { return gmbe_hid(u, P.hu_side); }
// combine the sums of the library's L (U side) and R (V side) in the caller's roles
__device__ __forceinline__ unsigned long long pair_hash(const Params& P, unsigned long long sl, unsigned long long sr) {
  return P.hu_side ? gmbe_pair_hash(sr, sl) : gmbe_pair_hash(sl, sr);
}

// ---- output records.  Bounded buffer: record i at out_ids[out_offsets[i]].  Streaming (N2): a ring
// of words in mapped host memory; a record is [h = 1 + words, words...] at ring positions pos..,
// published by writing h last (after a system-scope fence); the host consumes in position order,
// zeroes the words and advances its tail, which producers wait on when the ring is full.
struct RecOut {
  uint32_t* p;
  unsigned long long base, mask;
  __device__ __forceinline__ uint32_t& at(unsigned long long k) const { return p[(base + k) & mask]; }
};
__device__ __forceinline__ unsigned long long globaltimer_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// reserve room for a record of `need` words (one thread); false: nothing to write
__device__ bool rec_open(const Params& P, unsigned long long need, RecOut& O, unsigned long long& tok) {
  if (P.sring) {
    const unsigned long long pos = atomicAdd(&P.ctrl->out_ids, need + 1);
    atomicAdd(&P.ctrl->out_rec, 1ull);
    const unsigned long long end = pos + need + 1, cap = P.smask + 1;
    // ring full: back-pressure.  No timeout -- a slow consumer only slows the call; the wait ends
    // when the consumer frees room, or at once when the host raises its abort word
    while (end - ld_volatile(&P.ctrl->stream_tail) > cap) {
      const unsigned long long t = *(volatile const unsigned long long*)P.stail;  // host memory
      atomicMax(&P.ctrl->stream_tail, t);
      if (end - t <= cap) break;
      if (*(volatile const unsigned long long*)(P.stail + 1)) {  // the consumer gave up
        atomicOr(&P.ctrl->error, kErrStream);
        return false;
      }
      __nanosleep(2000);
    }
    O = RecOut{P.sring, pos + 1, P.smask};
    tok = pos;
    return true;
  }
  const unsigned long long rec = atomicAdd(&P.ctrl->out_rec, 1ull);
  const unsigned long long off = atomicAdd(&P.ctrl->out_ids, need);
  if (rec >= P.out_offsets_cap || off + need > P.out_ids_cap) {
    atomicOr(&P.ctrl->truncated, 1u);
    if (rec < P.out_offsets_cap) P.out_offsets[rec] = ~0ull;
    return false;
  }
  O = RecOut{P.out_ids, off, ~0ull};
  tok = rec;
  return true;
}
// publish (one thread, after every writer's words are done -- and fenced, when streaming)
__device__ void rec_close(const Params& P, const RecOut& O, unsigned long long need, unsigned long long tok) {
  if (P.sring) {
    __threadfence_system();
    *(volatile uint32_t*)(P.sring + (tok & P.smask)) = (uint32_t)(need + 1);
  } else {
    P.out_offsets[tok] = O.base;
  }
}

// Write one output record: L given by bitmap words lmask (W words over map) or, if lmask == null,
// by the explicit list lids[0..nl); R by ranks rl[0..nr).
__device__ void write_record(const Params& P, const uint32_t* lmask, uint32_t W, const uint32_t* map,
                             const uint32_t* lids, uint32_t nl, const uint32_t* rl, uint32_t nr) {
  const uint32_t lane = lane_id();
  const unsigned long long need = 2ull + nl + nr;
  RecOut O{nullptr, 0, 0};
  unsigned long long tok = 0;
  uint32_t ok = 0;
  if (lane == 0) ok = rec_open(P, need, O, tok);
  if (!__shfl_sync(GMBE_FULL, ok, 0)) return;
  O.p = (uint32_t*)__shfl_sync(GMBE_FULL, (unsigned long long)O.p, 0);
  O.base = __shfl_sync(GMBE_FULL, O.base, 0);
  O.mask = __shfl_sync(GMBE_FULL, O.mask, 0);
  const bool sw = P.hu_side != 0;  // caller U ids first: the library's L unless swapped
  const unsigned long long lpos = sw ? 2 + nr : 2, rpos = sw ? 2 : 2 + nl;
  if (lane == 0) {
    O.at(0) = sw ? nr : nl;
    O.at(1) = sw ? nl : nr;
  }
  for (uint32_t j = lane; j < nr; j += 32) O.at(rpos + j) = P.g.rank2id[rl[j]];
  if (lmask) {
    uint32_t c = 0;
    for (uint32_t w = 0; w < W; w++) {
      const uint32_t word = lmask[w];
      const bool b = (word >> lane) & 1u;
      const uint32_t bal = __ballot_sync(GMBE_FULL, b);
      if (b) O.at(lpos + c + __popc(bal & lanemask_lt())) = map[w * 32 + lane];
      c += __popc(bal);
    }
  } else {
    for (uint32_t j = lane; j < nl; j += 32) O.at(lpos + j) = lids[j];
  }
  if (P.sring) __threadfence_system();
  __syncwarp();
  if (lane == 0) rec_close(P, O, need, tok);
}

// ---------------------------------------------------------------- maximality (a5)
__device__ __forceinline__ bool bsearch_rank(const uint32_t* a, uint32_t n, uint32_t x) {
  uint32_t lo = 0, hi = n;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (__ldg(a + mid) < x) lo = mid + 1;
    else hi = mid;
  }
  return lo < n && __ldg(a + lo) == x;
}

// Alg 2 L14: is R' == Γ(L')?  Γ(L') = ∩_{u∈L'} N(u) ⊇ R', so maximal iff |Γ(L')| == |R'|.
// Count over N(u*) for the lowest-degree u* ∈ L' (|Γ(L')| <= deg(u*)), 32 vertices x ∈ N(u*) per
// step: a cheap necessary filter first (deg(x) >= |L'|), then member-major binary searches of x in
// the lists of the lowest-degree members while many lanes survive (most x fail at the first ones),
// then survivor-major verification -- one survivor at a time, its tests against 32 members per step
// -- once the survivors are few (the members of Γ(L'), i.e. the vertices of R', pass every test:
// ⌈|L'|/32⌉ steps each instead of |L'| - 1 serial searches).  L' = the lc set bits of lmask (W words)
// over map.  scratch: room for lc 64-bit keys (used when lc > 32).
__device__ GMBE_NI_IF(GMBE_NI_GAMMA) bool gamma_is_r(const Params& P, const uint32_t* lmask, uint32_t W, const uint32_t* map, uint32_t lc,
                           uint32_t rlen, unsigned long long* scratch, unsigned long long* smem) {
  const uint32_t lane = lane_id();
  const DevGraph& g = P.g;
  // members as (deg << 32 | begin of N(u)) keys.  lc <= 32: lane j holds the member of j-th lowest
  // degree.  Wider: all members go to scratch; lane j holds the j-th lowest of the lane-local minima
  // (the filter members; lane 0 = u*)
  unsigned long long key = ~0ull;
  if (lc <= 32) {
    uint32_t c = 0;  // members gathered so far; the t-th set bit of a word goes to lane c + t
    for (uint32_t w = 0; w < W && c < lc; w++) {
      const uint32_t word = lmask[w];
      if (!word) continue;
      const uint32_t nb = __popc(word);
      const bool mine = lane >= c && lane < c + nb;
      const uint32_t src = mine ? __fns(word, 0, lane - c + 1) : 0;
      const uint32_t mine_u = ((word >> lane) & 1u) ? map[w * 32 + lane] : 0u;
      const uint32_t u = __shfl_sync(GMBE_FULL, mine_u, src);
      if (mine) {
        const uint32_t b = g.off_u[u];
        key = ((unsigned long long)(g.off_u[u + 1] - b) << 32) | b;
      }
      c += nb;
    }
  } else {
    uint32_t c = 0;
    for (uint32_t wb = 0; wb < W; wb += 32) {
      const uint32_t w = wb + lane;
      const uint32_t word = w < W ? lmask[w] : 0u;
      const uint32_t nb = __popc(word);
      uint32_t inc = nb;
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t t = __shfl_up_sync(GMBE_FULL, inc, o);
        if (lane >= (uint32_t)o) inc += t;
      }
      uint32_t pos = c + inc - nb;
      for (uint32_t x = word; x; x &= x - 1) {
        const uint32_t u = map[w * 32 + __ffs(x) - 1];
        const uint32_t b = g.off_u[u];
        const unsigned long long kk = ((unsigned long long)(g.off_u[u + 1] - b) << 32) | b;
        scratch[pos++] = kk;
        key = min(key, kk);
      }
      c += __shfl_sync(GMBE_FULL, inc, 31);
    }
    __syncwarp();
  }
  key = warp_sort32(key);
  const unsigned long long k0 = __shfl_sync(GMBE_FULL, key, 0);
  const uint32_t d0 = (uint32_t)(k0 >> 32);
  if (lc == 1 || d0 <= rlen) return d0 == rlen;  // |Γ(L')| <= deg(u*); |L'| = 1: Γ = N(u*)
  const uint32_t nf = lc <= 32 ? lc : __popc(__ballot_sync(GMBE_FULL, key != ~0ull));  // filter members
  const uint32_t fb = (uint32_t)key, fd = (uint32_t)(key >> 32);
  const uint32_t nstep = (lc + 31) >> 5;  // verification steps per survivor
  const uint32_t* n0 = g.adj_u + (uint32_t)k0;
  uint32_t count = 0;
  for (uint32_t b = 0; b < d0; b += 32) {
    const uint32_t idx = b + lane;
    bool ok = idx < d0;
    const uint32_t v = ok ? __ldg(n0 + idx) : 0;
    if (ok && lc >= 8) ok = g.off_v[v + 1] - g.off_v[v] >= lc;  // a dominator of L' has degree >= |L'|
    // member-major filter while the survivors would cost more to verify one by one
    uint32_t j = 1;
    while (j < nf) {
      const uint32_t s = __popc(__ballot_sync(GMBE_FULL, ok));
      if (s * nstep <= nf - j) break;
      const uint32_t jb = __shfl_sync(GMBE_FULL, fb, j), jd = __shfl_sync(GMBE_FULL, fd, j);
      if (ok) ok = bsearch_rank(g.adj_u + jb, jd, v);
      j++;
    }
    uint32_t sv = __ballot_sync(GMBE_FULL, ok);
    if (j >= nf && lc <= 32) {  // every member tested
      count += __popc(sv);
      if (count > rlen) return false;
      continue;
    }
    while (sv) {  // survivor-major: 32 members per step, first miss ends the survivor
      const uint32_t x = __shfl_sync(GMBE_FULL, v, __ffs(sv) - 1);
      sv &= sv - 1;
      bool all = true;
      for (uint32_t j0 = 0; j0 < lc && all; j0 += 32) {
        const uint32_t jj = j0 + lane;
        bool in = true;
        if (jj < lc) {
          uint32_t mb = fb, md = fd;  // lc <= 32: lane jj holds member jj
          if (lc > 32) {
            const unsigned long long kj = scratch[jj];
            mb = (uint32_t)kj;
            md = (uint32_t)(kj >> 32);
          }
          in = bsearch_rank(g.adj_u + mb, md, x);
        }
        all = __all_sync(GMBE_FULL, in);
      }
      count += all;
      if (count > rlen) return false;
    }
  }
  return count == rlen;
}

// Alg 2 L14 with the root's Γ columns: every v ∈ Γ(L') other than v_s lies in the root's 2-hop set
// X, so |Γ(L')| = 1 + popc(AND_{j ∈ L'} col_j); maximal iff that equals |R'|.
__device__ GMBE_NI_IF(GMBE_NI_GAMMA) bool gamma_cols_is_r(const TaskCtx& T, const uint32_t* lmask, uint32_t W, uint32_t rlen) {
  const uint32_t lane = lane_id();
  const uint32_t need = rlen - 1;  // dominators in X that are already in R'
  uint32_t count = 0;
  for (uint32_t xb = 0; xb < T.ncw; xb += 32) {
    const uint32_t xw = xb + lane;
    uint32_t acc = xw < T.ncw ? GMBE_FULL : 0u;
    for (uint32_t w = 0; w < W; w++) {
      uint32_t word = lmask[w];
      while (word) {
        const uint32_t j = w * 32 + __ffs(word) - 1;
        word &= word - 1;
        if (acc) acc &= __ldg(T.cols + (size_t)j * T.ncw + xw);
        if (!__any_sync(GMBE_FULL, acc)) break;
      }
      if (!__any_sync(GMBE_FULL, acc)) break;
    }
    count += warp_sum(__popc(acc));
    if (count > need) return false;
  }
  return count == need;
}

// ---------------------------------------------------------------- child generation (a4, a5)
// Generate the child of node `par` via its candidate i into `ch` (Alg 2 L6-16).  The parent's later
// candidates are compacted in place (Thm 4.1 prunes removed), so par[0] shrinks.
// Returns 0: non-maximal; 1: maximal leaf (C' empty); 2: maximal with C' != ∅ (ch holds the child
// node record, header filled except the parent link).
// LPE (lanes per candidate entry, 4..32) is a runtime value: one code copy serves every width
__device__ int gen_child(const Params& P, const TaskCtx& T, uint32_t* par, uint32_t i, uint32_t* ch, Acc& A,
                         unsigned long long* smem, const uint32_t LPE) {
  const uint32_t G = 32 / LPE;
  const uint32_t lane = lane_id(), sub = lane & (LPE - 1), grp = lane / LPE;
  const bool leader = sub == 0;
  const uint32_t W = T.W, E = T.E;
  const uint32_t nC = par[0];
  uint32_t* pent = par + kHdr + T.W4;
  uint32_t* cent = ch + kHdr + T.W4;
  const uint32_t* vrow = pent + (size_t)i * E;
  const uint32_t vid = vrow[W];
  PH_START(A);
  // L' = L_p ∩ N(v')   (Alg 2 L8)
  uint32_t lpart = 0, xw = 0;
  for (uint32_t w = lane; w < W; w += 32) {
    const uint32_t x = par[kHdr + w] & vrow[w];
    ch[kHdr + w] = x;
    if (w == lane) xw = x;
    lpart += __popc(x);
  }
  const uint32_t lc = warp_sum(lpart);
  uint32_t lp0 = __shfl_sync(GMBE_FULL, xw, sub);
  if (sub >= W) lp0 = 0;
  __syncwarp();
  const uint32_t* lpm = ch + kHdr;  // L' words (W > LPE only)
  PH_STOP(A, 14);
  // later candidates: k' (Alg 2 L9-13), Thm 4.1 pruning with in-place compaction of
  // the survivors, absorption into R' (k' = |L'|), C' (0 < k' < |L'|)
  uint32_t nCc = 0, nsurv = 0, r_abs = 0;
  unsigned long long sr_abs = 0, later_k = 0;
  const uint32_t rl_base = par[5] + 1;  // R-list position of the first absorbed vertex
  for (uint32_t base = i + 1; base < nC; base += G) {
    const uint32_t j = base + grp;
    const bool in = j < nC;
    const uint32_t* ej = pent + (size_t)j * E;
    uint32_t raw0 = 0, cnt = 0, x0 = 0, id = 0, kp = 0;
    if (in) {
      if (sub < W) raw0 = ej[sub];
      x0 = raw0 & lp0;
      cnt = __popc(x0);
      for (uint32_t w = sub + LPE; w < W; w += LPE) cnt += __popc(ej[w] & lpm[w]);
      id = ej[W];
      kp = ej[W + 1];
    }
    cnt = group_sum(cnt, LPE);
    const bool pruned = in && P.prune && cnt == kp;
    const bool surv = in && !pruned;
    const bool absorb = in && cnt == lc;
    const bool cand = in && cnt > 0 && cnt < lc;
    if (in && leader) later_k += kp;
    if (absorb && leader) sr_abs += P.g.hv[id];
    const uint32_t ba = __ballot_sync(GMBE_FULL, absorb && leader);
    if (T.rlist && absorb && leader) T.rlist[rl_base + r_abs + __popc(ba & lanemask_lt())] = id;
    r_abs += __popc(ba);
    // C' entry
    const uint32_t bc = __ballot_sync(GMBE_FULL, cand && leader);
    const uint32_t cpos = __shfl_sync(GMBE_FULL, nCc + __popc(bc & lanemask_lt()), grp * LPE);
    nCc += __popc(bc);
    if (cand) {
      uint32_t* ce = cent + (size_t)cpos * E;
      if (sub < W) ce[sub] = x0;
      for (uint32_t w = sub + LPE; w < W; w += LPE) ce[w] = ej[w] & lpm[w];
      if (leader) {
        ce[W] = id;
        ce[W + 1] = cnt;
      }
    }
    // survivor compaction (write position <= read position; all reads of this step are done)
    const uint32_t bs = __ballot_sync(GMBE_FULL, surv && leader);
    const uint32_t spos = __shfl_sync(GMBE_FULL, i + 1 + nsurv + __popc(bs & lanemask_lt()), grp * LPE);
    nsurv += __popc(bs);
    __syncwarp();
    if (surv && spos != j) {
      uint32_t* se = pent + (size_t)spos * E;
      if (sub < W) se[sub] = raw0;
      for (uint32_t w = sub + LPE; w < W; w += LPE) se[w] = ej[w];
      if (leader) {
        se[W] = id;
        se[W + 1] = kp;
      }
    }
    __syncwarp();
  }
  if (lane == 0) par[0] = i + 1 + nsurv;
  A.add(kAcNodes, 1);
  A.add(kAcAbytes, 4ull * (lc + warp_sum64(later_k)));
  const uint32_t rlen = par[5] + 1 + r_abs;
  __syncwarp();
  unsigned long long* gscr = (unsigned long long*)align4(cent + (size_t)nCc * E);
  PH_STOP(A, 4);
  bool maximal;
  if (lc == 1) {  // Γ({u}) = N(u)
    uint32_t w = 0;
    while (!lpm[w]) w++;
    const uint32_t u = T.map[w * 32 + __ffs(lpm[w]) - 1];
    maximal = P.g.off_u[u + 1] - P.g.off_u[u] == rlen;
  } else if (T.cols) {  // (W > 2 here: the gx index only exists for universes <= 64 bits)
    maximal = gamma_cols_is_r(T, lpm, W, rlen);
  } else {
    maximal = gamma_is_r(P, lpm, W, T.map, lc, rlen, gscr, smem);
  }
#ifndef GMBE_PROFILE
  if ((P.debug & 32) && lane == 0) atomicAdd(&P.ctrl->phase[lc == 1 ? 4 : (T.cols ? 5 : 6)], 1ull);
#endif
  PH_STOP(A, 5);
  if (!maximal) {
    A.add(kAcNonmax, 1);
    return 0;
  }
  // Output(L', R') (Alg 2 L15)
  const unsigned long long par_sr = ((unsigned long long)par[7] << 32) | par[6];
  const unsigned long long sr = par_sr + P.g.hv[vid] + warp_sum64(sr_abs);
  unsigned long long sl = 0;  // lane t sums the members in words t, t + 32, ...
  for (uint32_t w = lane; w < W; w += 32)
    for (uint32_t word = lpm[w]; word; word &= word - 1) sl += hash_u(P, T.map[w * 32 + __ffs(word) - 1]);
  sl = warp_sum64(sl);
  A.add(kAcCount, 1);
  A.add(kAcChecksum, pair_hash(P, sl, sr));
  if (P.per_root && lane == 0) atomicAdd(P.per_root + T.root, 1ull);
  if (T.rlist) {
    if (lane == 0) T.rlist[par[5]] = vid;
    __syncwarp();
    if (P.out_ids || P.sring) write_record(P, lpm, W, T.map, nullptr, lc, T.rlist, rlen);
  }
  PH_STOP(A, 6);
  if (nCc == 0) return 1;
  if (lane == 0) {
    ch[0] = nCc;
    ch[1] = 0;
    ch[2] = lc;
    ch[3] = 0;
    ch[5] = rlen;
    ch[6] = (uint32_t)sr;
    ch[7] = (uint32_t)(sr >> 32);
  }
  __syncwarp();
  return 2;
}

// ---------------------------------------------------------------- small universes (<= 64 bits)
// Per-task lane-resident data for W <= 2 (see TaskCtx).
__device__ void small_task_init(const Params& P, TaskCtx& T, uint32_t lmap) {
  const uint32_t lane = lane_id();
  T.go0 = T.go1 = T.gl0 = T.gl1 = 0;
  T.hu0 = lane < lmap ? gmbe_hid(T.map[lane], P.hu_side) : 0ull;
  T.hu1 = lane + 32 < lmap ? gmbe_hid(T.map[lane + 32], P.hu_side) : 0ull;
  T.dg0 = T.dg1 = 0;
  if (lane < lmap) {
    const uint32_t u = T.map[lane];
    T.dg0 = P.g.off_u[u + 1] - P.g.off_u[u];
  }
  if (lane + 32 < lmap) {
    const uint32_t u = T.map[lane + 32];
    T.dg1 = P.g.off_u[u + 1] - P.g.off_u[u];
  }
  T.gxl = nullptr;
  T.nx = kNone;
  T.xr0 = T.xr1 = 0;
  if (T.gx) {
    T.nx = T.gx[0];
    const unsigned long long* xrow = (const unsigned long long*)(T.gx + 4);
    if (T.nx <= 64) {
      if (lane < T.nx) T.xr0 = xrow[lane];
      if (lane + 32 < T.nx) T.xr1 = xrow[lane + 32];
    }
    const uint32_t* coff = T.gx + 4 + 2 * T.gx[0] + r4(T.gx[0]);
    const uint32_t l = T.nx > 64 ? T.gx[1] : 0u;  // |X2| <= 64: no lists (rows are lane-resident)
    T.gxl = coff + r4(T.gx[1] + 1);
    if (lane < l) {
      T.go0 = coff[lane];
      T.gl0 = coff[lane + 1] - T.go0;
    }
    if (lane + 32 < l) {
      T.go1 = coff[lane + 32];
      T.gl1 = coff[lane + 33] - T.go1;
    }
  }
}

// Alg 2 L14 with the root's Γ index gx (universe <= 64 bits, L' = lm): Γ(L') ⊆ {v_s} ∪ X2 for
// |L'| >= 2.  |X2| <= 64: count the lane-resident rows covering L'.  Otherwise walk the X2 list of the
// member u* with the shortest list: |Γ(L')| <= 1 + |list(u*)|, so equality with |R'| proves
// maximality at once; else count the listed rows covering L'.
__device__ __forceinline__ bool gamma_gx_small(const TaskCtx& T, unsigned long long lm, uint32_t rlen) {
  const uint32_t lane = lane_id();
  if (T.nx <= 64) {  // lane-resident X2 rows: |Γ(L')| = 1 + #rows covering L'
    uint32_t count = 1 + __popc(__ballot_sync(GMBE_FULL, (T.xr0 & lm) == lm));
    if (T.nx > 32) count += __popc(__ballot_sync(GMBE_FULL, (T.xr1 & lm) == lm));
    return count == rlen;
  }
  uint32_t key = 0xffffffffu;
  if ((lm >> lane) & 1ull) key = (T.gl0 << 7) | lane;
  if ((lm >> (lane + 32)) & 1ull) key = min(key, (T.gl1 << 7) | (lane + 32));
  key = __reduce_min_sync(GMBE_FULL, key);
  const uint32_t js = key & 127u, len = key >> 7;
  if (len + 1 == rlen) return true;  // |Γ(L')| <= deg(u*) = len + 1
  const uint32_t off = __shfl_sync(GMBE_FULL, js < 32 ? T.go0 : T.go1, js & 31);
  const unsigned long long* xrow = (const unsigned long long*)(T.gx + 4);
  const uint32_t* lst = T.gxl + off;
  uint32_t count = 1;  // v_s
  for (uint32_t b = 0; b < len; b += 32) {
    bool full = false;
    if (b + lane < len) full = (xrow[lst[b + lane]] & lm) == lm;
    count += __popc(__ballot_sync(GMBE_FULL, full));
    if (count > rlen) return false;
  }
  return count == rlen;
}

// gen_child for W <= 2: one lane per candidate entry, loaded as one 16-byte vector
// ({row, id, k, -} for W = 1, {row_lo, row_hi, id, k} for W = 2); L' and rows as 64-bit masks.
__device__ int gen_child_small(const Params& P, const TaskCtx& T, uint32_t* par, uint32_t i, uint32_t* ch, Acc& A,
                               unsigned long long* smem) {
  const uint32_t lane = lane_id();
  const bool w2 = T.W == 2;
  const uint32_t nC = par[0];
  uint4* pent = (uint4*)(par + kHdr + 4);
  uint4* cent = (uint4*)(ch + kHdr + 4);
  PH_START(A);
  const uint4 vr = pent[i];
  const unsigned long long vrow = w2 ? (((unsigned long long)vr.y << 32) | vr.x) : vr.x;
  const uint32_t vid = w2 ? vr.z : vr.y;
  const unsigned long long lpar = ((unsigned long long)par[kHdr + 1] << 32) | par[kHdr];
  const unsigned long long lm = lpar & vrow;  // L' = L_p ∩ N(v')   (Alg 2 L8)
  const uint32_t lc = __popcll(lm);
  if (lane == 0) {
    ch[kHdr] = (uint32_t)lm;
    ch[kHdr + 1] = (uint32_t)(lm >> 32);
  }
  PH_STOP(A, 14);
  // later candidates: k' (Alg 2 L9-13), Thm 4.1 pruning with in-place compaction, R', C'
  uint32_t nCc = 0, nsurv = 0, r_abs = 0;
  unsigned long long sr_abs = 0, later_k = 0;
  const uint32_t rl_base = par[5] + 1;
  for (uint32_t base = i + 1; base < nC; base += 32) {
    const uint32_t j = base + lane;
    const bool in = j < nC;
    uint4 x = make_uint4(0, 0, 0, 0);
    if (in) x = pent[j];
    const unsigned long long row = w2 ? (((unsigned long long)x.y << 32) | x.x) : x.x;
    const uint32_t id = w2 ? x.z : x.y, kp = w2 ? x.w : x.z;
    const unsigned long long xr = row & lm;
    const uint32_t cnt = __popcll(xr);
    const bool pruned = in && P.prune && cnt == kp;
    const bool surv = in && !pruned;
    const bool absorb = in && cnt == lc;
    const bool cand = in && cnt > 0 && cnt < lc;
    if (in) later_k += kp;
    if (absorb) sr_abs += P.g.hv[id];
    const uint32_t ba = __ballot_sync(GMBE_FULL, absorb);
    if (T.rlist && absorb) T.rlist[rl_base + r_abs + __popc(ba & lanemask_lt())] = id;
    r_abs += __popc(ba);
    const uint32_t bc = __ballot_sync(GMBE_FULL, cand);
    if (cand)
      cent[nCc + __popc(bc & lanemask_lt())] =
          w2 ? make_uint4((uint32_t)xr, (uint32_t)(xr >> 32), id, cnt) : make_uint4((uint32_t)xr, id, cnt, 0);
    nCc += __popc(bc);
    const uint32_t bs = __ballot_sync(GMBE_FULL, surv);
    const uint32_t spos = i + 1 + nsurv + __popc(bs & lanemask_lt());
    nsurv += __popc(bs);
    __syncwarp();
    if (surv && spos != j) pent[spos] = x;
    __syncwarp();
  }
  if (lane == 0) par[0] = i + 1 + nsurv;
  A.add(kAcNodes, 1);
  A.add(kAcAbytes, 4ull * (lc + warp_sum64r(later_k)));
  const uint32_t rlen = par[5] + 1 + r_abs;
  PH_STOP(A, 4);
  bool maximal;
  if (lc == 1) {  // Γ({u}) = N(u); the universe vertices' degrees are lane-resident (small_task_init)
    const uint32_t j = __ffsll(lm) - 1;
    maximal = __shfl_sync(GMBE_FULL, j < 32 ? T.dg0 : T.dg1, j & 31) == rlen;
  } else if (T.gx) {
    maximal = gamma_gx_small(T, lm, rlen);
  } else {
    __syncwarp();
    maximal = gamma_is_r(P, ch + kHdr, T.W, T.map, lc, rlen,
                         (unsigned long long*)align4((uint32_t*)(cent + nCc)), smem);
  }
  PH_STOP(A, 5);
  if (!maximal) {
    A.add(kAcNonmax, 1);
    return 0;
  }
  // Output(L', R') (Alg 2 L15)
  const unsigned long long par_sr = ((unsigned long long)par[7] << 32) | par[6];
  const unsigned long long sl =
      warp_sum64r(((lm >> lane) & 1ull ? T.hu0 : 0ull) + ((lm >> (lane + 32)) & 1ull ? T.hu1 : 0ull));
  const unsigned long long sr = par_sr + P.g.hv[vid] + warp_sum64r(sr_abs);
  A.add(kAcCount, 1);
  A.add(kAcChecksum, pair_hash(P, sl, sr));
  if (P.per_root && lane == 0) atomicAdd(P.per_root + T.root, 1ull);
  if (T.rlist) {
    if (lane == 0) T.rlist[par[5]] = vid;
    __syncwarp();
    if (P.out_ids || P.sring) write_record(P, ch + kHdr, T.W, T.map, nullptr, lc, T.rlist, rlen);
  }
  PH_STOP(A, 6);
  if (nCc == 0) return 1;
  if (lane == 0) {
    ch[0] = nCc;
    ch[1] = 0;
    ch[2] = lc;
    ch[3] = 0;
    ch[5] = rlen;
    ch[6] = (uint32_t)sr;
    ch[7] = (uint32_t)(sr >> 32);
  }
  __syncwarp();
  return 2;
}

__device__ __forceinline__ uint32_t rec_words(const TaskCtx& T, const uint32_t* rec) {
  return kHdr + T.W4 + rec[0] * T.E;
}
__device__ __forceinline__ bool heavy(const Params& P, uint32_t l, uint32_t nC) {
  if (!P.split) return false;
  const unsigned long long h = min(l, nC);  // tree height estimate
  if (h > P.bound_height && h * nC > P.bound_size) return true;
  // wide universes: every node costs ~|L|/32 words of AND/POPC plus a Γ test over |L'| members, so
  // the node count alone under-estimates the work (B200 addition, reading B4)
  return l > 64 && nC >= 2 && (unsigned long long)nC * ((l + 31) / 32) >= P.split_wide;
}
// Late-phase split (B200 addition): once GMBE_LATE_PCT % of the roots have been issued, the GPU is
// about to drain, and a mid-size task started now would run alone in the tail -- so tasks above the
// lower (GMBE_LATE_BH, GMBE_LATE_BS) thresholds split too.  Schedule only: the tree is unchanged.
// Knob, off by default: measured +0.5-3% at N=1 and 3-5x slower on 1/8 root shards (a shard's
// cursor passes the mark almost at once), profiles/r01_late_split_ab.txt.
#ifndef GMBE_LATE_PCT
#define GMBE_LATE_PCT 0
#endif
#ifndef GMBE_LATE_BH
#define GMBE_LATE_BH 6
#endif
#ifndef GMBE_LATE_BS
#define GMBE_LATE_BS 120
#endif
__device__ __forceinline__ bool late_heavy(const Params& P, uint32_t l, uint32_t nC) {
  if (GMBE_LATE_PCT == 0 || !P.split) return false;
  const unsigned long long h = min(l, nC);
  if (h <= GMBE_LATE_BH || h * nC <= GMBE_LATE_BS) return false;
  const unsigned long long c = ld_volatile(P.shared_cursor ? P.shared_cursor : &P.ctrl->root_cursor.v);
  return 100ull * c >= (unsigned long long)GMBE_LATE_PCT * P.n_roots;
}
__device__ __forceinline__ bool heavy_wide(const Params& P, uint32_t l, uint32_t nC) {
  return P.split && l > 64 && nC >= 2 && (unsigned long long)nC * ((l + 31) / 32) >= P.split_wide;
}

// Walk the subtree of `top` (Alg 2) on the node stack [stack_lo, stack_hi) -- or, when the task is
// heavy (Alg 4 L17), hand top's children to the task queue as self-contained subtasks.
// ---------------------------------------------------------------- register-resident subtrees
// A node with <= 32 candidates over a <= 64-bit universe: every descendant's candidates are a subset
// of its candidates, so lane j keeps candidate j's row / id / hV for the whole subtree and a node is
// just (L mask, candidate lane mask).  Alg 2 on that representation: child via lane i -> L' = L & row_i;
// later = candidate lanes > i; k' = popc(row & L'), k = popc(row & L); Thm 4.1 clears the lanes with
// k' == k from the node; R' absorbs k' == |L'|; C' = 0 < k' < |L'|.  Levels (<= 32) live in the warp's
// shared-memory slice.  `split_top`: the node is a heavy task top -- publish its children (Alg 4 L25).
struct RegLevel {
  unsigned long long L, SR;
  uint32_t C, next, rlen, pad;
};
__device__ __forceinline__ unsigned long long shfl64(unsigned long long x, uint32_t src) {
  const uint32_t lo = __shfl_sync(GMBE_FULL, (uint32_t)x, src);
  const uint32_t hi = __shfl_sync(GMBE_FULL, (uint32_t)(x >> 32), src);
  return ((unsigned long long)hi << 32) | lo;
}
// Dynamic donation (beyond the paper's static estimate): while warps are idle-waiting
// (ctrl.hungry > 0), a warp deep in a subtree hands the remaining children of its shallowest
// unfinished level to the queue as a subtask.  The subtask's node is (L_k, R_k, remaining
// candidates of level k); its children, their later sets and their Thm 4.1 marks are exactly the
// ones the donor would have generated, so the tree and every counter are unchanged.
__device__ __forceinline__ bool hungry(const Params& P) {
  uint32_t h = 0;
  if (lane_id() == 0) h = P.donate && ((P.debug & 8) || ld_volatile(&P.ctrl->hungry.v) != 0);
  return __shfl_sync(GMBE_FULL, h, 0) != 0;
}
#ifndef GMBE_DONATE
#define GMBE_DONATE 2  // 0: compiled out; 1: checked every 32 nodes; 2: checked every 8th push
#endif
#ifndef GMBE_DONATE_INLINE
#define GMBE_DONATE_INLINE 1
#endif
#if GMBE_DONATE_INLINE
#define GMBE_DONATE_ATTR __forceinline__
#else
#define GMBE_DONATE_ATTR __noinline__
#endif
__device__ GMBE_DONATE_ATTR bool donate_reg(const Params& P, const TaskCtx& T, uint32_t lmap, Acc& A, RegLevel* st, uint32_t d,
                           unsigned long long row, uint32_t id, uint32_t* scratch, const uint32_t* scratch_end) {
  const uint32_t lane = lane_id();
  const bool w2 = T.W == 2;
  uint32_t av = 0;
  if (lane < d) {
    const uint32_t nx = st[lane].next;
    av = nx >= 32 ? 0u : (st[lane].C & ~((1u << nx) - 1u));
  }
  const uint32_t b = __ballot_sync(GMBE_FULL, av != 0);
  if (!b) return false;
  const uint32_t k = __ffs(b) - 1;
  av = __shfl_sync(GMBE_FULL, av, k);
  const unsigned long long Lk = st[k].L, SRk = st[k].SR;
  const uint32_t rk = st[k].rlen, n = __popc(av);
  const uint32_t words = kHdr + 4 + 4 * n;
  if (scratch + words > scratch_end) return false;
  uint4* ce = (uint4*)(scratch + kHdr + 4);
  if ((av >> lane) & 1u) {
    const unsigned long long xr = row & Lk;
    const uint32_t kc = __popcll(xr);
    ce[__popc(av & lanemask_lt())] = w2 ? make_uint4((uint32_t)xr, (uint32_t)(xr >> 32), id, kc)
                                        : make_uint4((uint32_t)xr, id, kc, 0);
  }
  if (lane == 0) {
    scratch[0] = n;
    scratch[1] = 0;
    scratch[2] = __popcll(Lk);
    scratch[3] = 0;
    scratch[4] = kNone;
    scratch[5] = rk;
    scratch[6] = (uint32_t)SRk;
    scratch[7] = (uint32_t)(SRk >> 32);
    scratch[kHdr] = (uint32_t)Lk;
    scratch[kHdr + 1] = (uint32_t)(Lk >> 32);
    scratch[kHdr + 2] = 0;
    scratch[kHdr + 3] = 0;
  }
  __syncwarp();
  if (!task_publish(P, T, lmap, T.rlist ? rk : 0, scratch, words, A)) return false;
  if (lane == 0) st[k].next = 32;  // the donated children are no longer this warp's
  __syncwarp();
  A.add(kAcDonations, 1);
  return true;
}

__device__ GMBE_NI_IF(GMBE_NI_REG) void run_reg(const Params& P, const TaskCtx& T, const uint32_t* rec, uint32_t lmap, Acc& A,
                        RegLevel* st, uint32_t* scratch, const uint32_t* scratch_end, bool split_top,
                        unsigned long long* smem) {
  const uint32_t lane = lane_id();
  const bool w2 = T.W == 2;
  const uint32_t nC = rec[0];
  unsigned long long row = 0, hvj = 0;
  uint32_t id = 0;
  if (lane < nC) {
    const uint4 x = ((const uint4*)(rec + kHdr + 4))[lane];
    row = w2 ? (((unsigned long long)x.y << 32) | x.x) : x.x;
    id = w2 ? x.z : x.y;
    hvj = P.g.hv[id];
  }
  unsigned long long L = ((unsigned long long)rec[kHdr + 1] << 32) | rec[kHdr];
  unsigned long long SR = ((unsigned long long)rec[7] << 32) | rec[6];
  uint32_t C = nC >= 32 ? GMBE_FULL : ((1u << nC) - 1u), next = 0, rlen = rec[5];
  int d = 0;
#if GMBE_DONATE
  uint32_t tick = 0;
#endif
  while (true) {
#if GMBE_DONATE == 1
    if (d > 0 && (++tick & 31) == 0 && hungry(P)) donate_reg(P, T, lmap, A, st, d, row, id, scratch, scratch_end);
#endif
    const uint32_t avail = next >= 32 ? 0u : (C & ~((1u << next) - 1u));
    if (!avail) {  // pop (Alg 2 L4)
      if (d == 0) break;
      d--;
      L = st[d].L;
      SR = st[d].SR;
      C = st[d].C;
      next = st[d].next;
      rlen = st[d].rlen;
      __syncwarp();  // every lane has read level d before lane 0 overwrites it at the next push
      continue;
    }
    const uint32_t i = __ffs(avail) - 1;
    next = i + 1;
    const unsigned long long lp = L & shfl64(row, i);  // L' = L_p ∩ N(v')
    const uint32_t lc = __popcll(lp);
    const uint32_t later = i >= 31 ? 0u : (C & ~((2u << i) - 1u));
    const bool inl = (later >> lane) & 1u;
    const uint32_t kp = __popcll(row & L), kc = __popcll(row & lp);
    const uint32_t pr = __ballot_sync(GMBE_FULL, inl && P.prune && kc == kp);
    const uint32_t ab = __ballot_sync(GMBE_FULL, inl && kc == lc);
    const uint32_t cd = __ballot_sync(GMBE_FULL, inl && kc > 0 && kc < lc);
    C &= ~pr;  // Thm 4.1
    A.add(kAcNodes, 1);
    A.add(kAcAbytes, 4ull * (lc + __reduce_add_sync(GMBE_FULL, inl ? kp : 0u)));
    const uint32_t rl = rlen + 1 + __popc(ab);
    bool maximal;
    if (lc == 1) {  // (degrees lane-resident, small_task_init)
      const uint32_t j = __ffsll(lp) - 1;
      maximal = __shfl_sync(GMBE_FULL, j < 32 ? T.dg0 : T.dg1, j & 31) == rl;
    } else if (T.gx) {
      maximal = gamma_gx_small(T, lp, rl);
    } else {
      if (lane == 0) {
        scratch[0] = (uint32_t)lp;
        scratch[1] = (uint32_t)(lp >> 32);
      }
      __syncwarp();
      maximal = gamma_is_r(P, scratch, T.W, T.map, lc, rl, (unsigned long long*)(scratch + 4), nullptr);
    }
    if (!maximal) {
      A.add(kAcNonmax, 1);
      continue;
    }
    // Output(L', R') (Alg 2 L15)
    const uint32_t idi = __shfl_sync(GMBE_FULL, id, i);
    const unsigned long long srn = SR + shfl64(hvj, i) + warp_sum64r(((ab >> lane) & 1u) ? hvj : 0ull);
    const unsigned long long sl =
        warp_sum64r(((lp >> lane) & 1ull ? T.hu0 : 0ull) + ((lp >> (lane + 32)) & 1ull ? T.hu1 : 0ull));
    A.add(kAcCount, 1);
    A.add(kAcChecksum, pair_hash(P, sl, srn));
    if (P.per_root && lane == 0) atomicAdd(P.per_root + T.root, 1ull);
    if (T.rlist) {
      if (lane == 0) T.rlist[rlen] = idi;
      if ((ab >> lane) & 1u) T.rlist[rlen + 1 + __popc(ab & lanemask_lt())] = id;
      if (lane == 0) {
        scratch[0] = (uint32_t)lp;
        scratch[1] = (uint32_t)(lp >> 32);
      }
      __syncwarp();
      if (P.out_ids || P.sring) write_record(P, scratch, T.W, T.map, nullptr, lc, T.rlist, rl);
    }
    if (!cd) continue;
    if (split_top && d == 0) {
      // publish the child as a subtask: node record [hdr | L' | entries (row & L', id, k')]
      const uint32_t words = kHdr + 4 + 4 * __popc(cd);
      if (scratch + words <= scratch_end) {
        uint4* ce = (uint4*)(scratch + kHdr + 4);
        if ((cd >> lane) & 1u) {
          const unsigned long long xr = row & lp;
          ce[__popc(cd & lanemask_lt())] = w2 ? make_uint4((uint32_t)xr, (uint32_t)(xr >> 32), id, kc)
                                              : make_uint4((uint32_t)xr, id, kc, 0);
        }
        if (lane == 0) {
          scratch[0] = __popc(cd);
          scratch[1] = 0;
          scratch[2] = lc;
          scratch[3] = 0;
          scratch[4] = kNone;
          scratch[5] = rl;
          scratch[6] = (uint32_t)srn;
          scratch[7] = (uint32_t)(srn >> 32);
          scratch[kHdr] = (uint32_t)lp;
          scratch[kHdr + 1] = (uint32_t)(lp >> 32);
          scratch[kHdr + 2] = 0;
          scratch[kHdr + 3] = 0;
        }
        __syncwarp();
        if (task_publish(P, T, lmap, T.rlist ? rl : 0, scratch, words, A)) continue;
      }
    }
    // push (Alg 2 L16)
#if GMBE_DONATE == 2
    if (d > 0 && (++tick & 7) == 0 && hungry(P)) donate_reg(P, T, lmap, A, st, d, row, id, scratch, scratch_end);
#endif
    if (lane == 0) {
      st[d].L = L;
      st[d].SR = SR;
      st[d].C = C;
      st[d].next = next;
      st[d].rlen = rlen;
    }
    __syncwarp();
    d++;
    L = lp;
    SR = srn;
    C = cd;
    next = 0;
    rlen = rl;
  }
}

// ---------------------------------------------------------------- thread-level subtrees
// The same nodes as run_reg (<= 32 candidates over a <= 64-bit universe), walked one subtree per
// THREAD instead of one node per warp: a node is generated by one lane with scalar AND/POPC over
// the job's candidate rows in shared memory, so the 32 lanes of a warp generate up to 32 nodes at a
// time (Alg 2 unchanged; the paper's warp-per-procedure granularity, is kept for the
// heavier node layouts).  Work is spread inside the warp by donation: an idle lane receives the
// remaining children of a busy lane's shallowest stacked level (the node (L_k, R_k, remaining
// candidates of level k) -- its children, later sets and Thm 4.1 marks are exactly the ones the
// donor would have generated, so the tree and every counter stay those of the canonical tree).
// Maximality (Alg 2 L14), |L'| >= 2: L' is non-maximal iff some x ∈ Γ(L') lies outside R'.  Under
// the job (L0, R_job = Γ(L0), candidates C0) such an x is either a job candidate outside R' (tested
// with per-vertex candidate columns) or one of the job's Q patterns N(x) ∩ L0 (x ∈ X2 \ (R_job ∪ C0),
// deduplicated, reduced to the maximal ones above 64; tested with per-vertex pattern columns):
// both are one AND per member of L'.  |L'| = 1: deg(u) == |R'|.
struct ThrSmem {
  unsigned long long row[32];  // candidate rows over the universe (the job's top node)
  unsigned long long hv[32];   // hV of each candidate
  uint32_t ccol[64];           // bit c: job candidate c is adjacent to universe vertex j
  uint32_t deg[64];            // degree of each universe vertex
  uint32_t id[32];             // rank of each candidate
};
// One stacked DFS level of a lane (16 B): the node's L, candidate mask C and R-mask Rm.  Its SR and
// `next` are not stored: the child above it has Rm' = Rm ∪ {i} ∪ absorbed with every absorbed
// candidate ranked after the branch candidate i, so next = i + 1 = ffs(Rm' \ Rm) and
// SR = SR' - Σ_{c ∈ Rm' \ Rm} hV(c) (derived on pop, and for donation from the current node).
struct ThrLevel {
  unsigned long long L;
  uint32_t C, Rm;
};

// one output record from one lane: L' = bits of lp over map, R' = the job's R list + candidates rm
__device__ GMBE_NI_IF(GMBE_NI_DONATE_THR) void write_record_thr(const Params& P, const TaskCtx& T, const ThrSmem* ts, unsigned long long lp,
                                 uint32_t nl, uint32_t rlen0, uint32_t rm, uint32_t nr) {
  const unsigned long long need = 2ull + nl + nr;
  RecOut O;
  unsigned long long tok;
  if (!rec_open(P, need, O, tok)) return;
  const bool sw = P.hu_side != 0;
  const unsigned long long lpos = sw ? 2 + nr : 2, rpos = sw ? 2 : 2 + nl;
  O.at(0) = sw ? nr : nl;
  O.at(1) = sw ? nl : nr;
  uint32_t t = 0;
  for (; t < rlen0; t++) O.at(rpos + t) = P.g.rank2id[T.rlist[t]];
  for (uint32_t m = rm; m; m &= m - 1) O.at(rpos + t++) = P.g.rank2id[ts->id[__ffs(m) - 1]];
  t = 0;
  for (unsigned long long m = lp; m; m &= m - 1) O.at(lpos + t++) = T.map[__ffsll(m) - 1];
  rec_close(P, O, need, tok);
}

// Publish lane `src`'s stacked level k (its remaining children) as a subtask for idle warps
// (cross-warp donation, see donate_reg).  Warp-cooperative; returns whether it was published.
__device__ GMBE_NI_IF(GMBE_NI_DONATE_THR) bool donate_thr(const Params& P, const TaskCtx& T, uint32_t lmap, Acc& A, const ThrSmem* ts,
                           uint32_t nC, uint32_t rlen0, uint32_t src, unsigned long long Lk, unsigned long long SRk,
                           uint32_t Ck, uint32_t Rmk, uint32_t nextk, uint32_t* scratch, const uint32_t* scratch_end) {
  const uint32_t lane = lane_id();
  const bool w2 = T.W == 2;
  Lk = shfl64(Lk, src);
  SRk = shfl64(SRk, src);
  Ck = __shfl_sync(GMBE_FULL, Ck, src);
  Rmk = __shfl_sync(GMBE_FULL, Rmk, src);
  nextk = __shfl_sync(GMBE_FULL, nextk, src);
  const uint32_t av = Ck & (GMBE_FULL << nextk);
  const uint32_t n = __popc(av);
  const uint32_t words = kHdr + 4 + 4 * n;
  if (scratch + words > scratch_end) return false;
  uint4* ce = (uint4*)(scratch + kHdr + 4);
  if (lane < nC && ((av >> lane) & 1u)) {
    const unsigned long long xr = ts->row[lane] & Lk;
    const uint32_t id = ts->id[lane], kc = __popcll(xr);
    ce[__popc(av & lanemask_lt())] = w2 ? make_uint4((uint32_t)xr, (uint32_t)(xr >> 32), id, kc)
                                        : make_uint4((uint32_t)xr, id, kc, 0);
  }
  const uint32_t rk = rlen0 + __popc(Rmk);
  if (T.rlist && lane < nC && ((Rmk >> lane) & 1u)) T.rlist[rlen0 + __popc(Rmk & lanemask_lt())] = ts->id[lane];
  if (lane == 0) {
    scratch[0] = n;
    scratch[1] = 0;
    scratch[2] = __popcll(Lk);
    scratch[3] = 0;
    scratch[4] = kNone;
    scratch[5] = rk;
    scratch[6] = (uint32_t)SRk;
    scratch[7] = (uint32_t)(SRk >> 32);
    scratch[kHdr] = (uint32_t)Lk;
    scratch[kHdr + 1] = (uint32_t)(Lk >> 32);
    scratch[kHdr + 2] = 0;
    scratch[kHdr + 3] = 0;
  }
  __syncwarp();
  if (!task_publish(P, T, lmap, T.rlist ? rk : 0, scratch, words, A)) return false;
  A.add(kAcDonations, 1);
  return true;
}

#ifndef GMBE_NI_THR
#define GMBE_NI_THR 0  // 1: run_thr out of line -- gh_work -1.5% but dblp +26%, bx +10% (round 2)
#endif
#ifndef GMBE_SPLIT_WIDE
#define GMBE_SPLIT_WIDE 32
#endif
#ifndef GMBE_DENSE_CS
#define GMBE_DENSE_CS 0
#endif
#ifndef GMBE_THR_DONATE_MASK
#define GMBE_THR_DONATE_MASK 3  // run_thr checks ctrl.hungry every (mask + 1) steps
#endif
#ifndef GMBE_TINY_REDUX
#define GMBE_TINY_REDUX 0  // tiny roots: rows by per-group OR-reduction (1) or one ballot per member (0)
#endif
#ifndef GMBE_ROOT_CHUNK
#define GMBE_ROOT_CHUNK 1  // light roots claimed per atomic (opts.root_chunk); >1 measured slower on the heavy-tailed shapes
#endif
#ifndef GMBE_WARP_DONATE
#define GMBE_WARP_DONATE 1  // run_task: warp-level donation of a node's remaining children to idle warps
#endif
#ifndef GMBE_THR_DONATE_BURST
#define GMBE_THR_DONATE_BURST 1  // run_thr: levels donated per check while other warps are hungry (4, 16 measured no better)
#endif
#ifndef GMBE_THR_MIN_EST
#define GMBE_THR_MIN_EST 16  // jobs with fewer adjacency bits (Σ(k-1)) stay on run_reg (setup > work)
#endif
// smem layout of the column store (the warp's s_sort slice, kSmemSort u64): [0, 128) pattern hash
// table during setup, then [128, 256) = one ThrCol per universe vertex j
struct ThrCol {
  unsigned long long q;   // bit t: Q-pattern t contains j
  unsigned long long hu;  // hU of universe vertex j (the emission sum rides on the same loop)
};
constexpr uint32_t kThrHash = 128;
static_assert(kSmemSort * 8 >= kThrHash * 8 + 64 * sizeof(ThrCol), "column store exceeds the s_sort slice");
__device__ __forceinline__ bool sorted_has(const uint32_t* a, uint32_t n, uint32_t x) {
  uint32_t lo = 0, hi = n;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (a[mid] < x) lo = mid + 1;
    else hi = mid;
  }
  return lo < n && a[lo] == x;
}
// Does a job fit the thread-level tier?  A Γ index (gx) and enough work: adjacency bits beyond one per
// candidate (a candidate with k = 1 only yields a leaf) -- checked inline by the caller, so the
// out-of-line run_thr is only entered for jobs it takes.
__device__ __forceinline__ bool thr_eligible(const Params& P, const TaskCtx& T, const uint32_t* rec) {
  if (!T.gx) return false;
  const uint32_t lane = lane_id(), nC = rec[0];
  uint32_t k = 0;
  if (lane < nC) k = rec[kHdr + 4 + 4 * lane + (T.W == 2 ? 3 : 2)] - 1u;
  return warp_sum(k) >= P.thr_min_est;
}
// Returns false (nothing done) when the job does not fit this tier (more than 64 Q patterns after
// reduction); the caller then runs it with run_reg.
__device__ GMBE_NI_IF(GMBE_NI_THR) bool run_thr(const Params& P, const TaskCtx& T, const uint32_t* rec, uint32_t lmap,
                                                Acc& A, ThrSmem* ts, unsigned long long* smem, uint32_t* scratch,
                                                const uint32_t* scratch_end) {
  const uint32_t lane = lane_id();
  const uint32_t nC = rec[0];
  const bool w2 = T.W == 2;
  uint4 x = make_uint4(0, 0, 0, 0);
  if (lane < nC) x = ((const uint4*)(rec + kHdr + 4))[lane];
  const unsigned long long L0 = ((unsigned long long)rec[kHdr + 1] << 32) | rec[kHdr];
  PH_START(A);
  // the job's candidates (rank order) and universe
  unsigned long long crow = 0;
  if (lane < nC) {
    crow = w2 ? (((unsigned long long)x.y << 32) | x.x) : x.x;
    const uint32_t id = w2 ? x.z : x.y;
    ts->row[lane] = crow;
    ts->id[lane] = id;
    ts->hv[lane] = P.g.hv[id];
  }
  ts->deg[lane] = T.dg0;
  ts->deg[lane + 32] = T.dg1;
  unsigned long long* ht = smem;
  for (uint32_t t = lane; t < kThrHash; t += 32) ht[t] = 0ull;
  __syncwarp();
  // Q patterns of the job: N(x) ∩ L0 for x ∈ X2 with |N(x) ∩ L0| >= 2 that is neither in R_job
  // (N(x) ⊇ L0: the job node is maximal, so Γ(L0) = R_job) nor a job candidate; deduplicated.
  // Under the job every such x lies outside R', and L' is non-maximal if one of them covers it.
  const uint32_t nx = T.gx[0];
  const unsigned long long* xrow = (const unsigned long long*)(T.gx + 4);
  const uint32_t* xid = T.gx + 4 + 2 * nx;
  bool over = false;
  auto consider = [&](uint32_t x, bool in, uint32_t first) {
    const unsigned long long p = in ? xrow[x] & L0 : 0ull;
    bool q = __popcll(p) >= 2 && p != L0 && (first >= 64 || (uint32_t)(__ffsll(p) - 1) == first);
    if (q) q = !sorted_has(ts->id, nC, xid[x]);
    if (q) {  // insert p (linear probing; 0 = empty)
      uint32_t h = (uint32_t)((p * 0x9E3779B97F4A7C15ull) >> 57), n = 0;
      while (true) {
        const unsigned long long old = atomicCAS(ht + h, 0ull, p);
        if (old == 0ull || old == p) break;
        h = (h + 1) & (kThrHash - 1);
        if (++n == kThrHash) {
          over = true;
          break;
        }
      }
    }
  };
  // X2 vertices touching >= 2 members of L0: scan all of X2, or -- when the per-vertex X2 lists of
  // the members of L0 are shorter in total -- walk those lists (x taken from the list of its first
  // member in L0 only)
  const uint32_t listed = nx > 64 ? warp_sum(((L0 >> lane) & 1ull ? T.gl0 : 0u) + ((L0 >> (lane + 32)) & 1ull ? T.gl1 : 0u))
                                  : kNone;
  if (listed < nx) {
    for (unsigned long long m = L0; m; m &= m - 1) {
      const uint32_t j = __ffsll(m) - 1;
      const uint32_t off = __shfl_sync(GMBE_FULL, j < 32 ? T.go0 : T.go1, j & 31);
      const uint32_t len = __shfl_sync(GMBE_FULL, j < 32 ? T.gl0 : T.gl1, j & 31);
      for (uint32_t b = 0; b < len; b += 32) {
        const bool in = b + lane < len;
        consider(in ? T.gxl[off + b + lane] : 0u, in, j);
      }
    }
  } else {
    for (uint32_t b = 0; b < nx; b += 32) consider(b + lane, b + lane < nx, 64);
  }
  __syncwarp();
  if (__any_sync(GMBE_FULL, over)) return false;
  // distinct patterns: compact the table to ht[0, npat); above 64, keep only the maximal ones (a
  // pattern inside another covers no L' the other does not)
  unsigned long long pk[4];
  uint32_t npat = 0;
#pragma unroll
  for (int k = 0; k < 4; k++) {
    pk[k] = ht[k * 32 + lane];
    npat += __popc(__ballot_sync(GMBE_FULL, pk[k] != 0ull));
  }
  if (npat > 64) {
    for (uint32_t t = 0; t < kThrHash; t++) {
      const unsigned long long o = ht[t];  // broadcast read
      if (!o) continue;
#pragma unroll
      for (int k = 0; k < 4; k++)
        if ((pk[k] & o) == pk[k] && pk[k] != o) pk[k] = 0ull;
    }
  }
  __syncwarp();
  npat = 0;
#pragma unroll
  for (int k = 0; k < 4; k++) {
    const uint32_t bal = __ballot_sync(GMBE_FULL, pk[k] != 0ull);
    if (pk[k]) ht[npat + __popc(bal & lanemask_lt())] = pk[k];
    npat += __popc(bal);
  }
  if (npat > 64) return false;
  __syncwarp();
  const unsigned long long q0 = lane < npat ? ht[lane] : 0ull, q1 = lane + 32 < npat ? ht[lane + 32] : 0ull;
  __syncwarp();
  ThrCol* cols = (ThrCol*)(smem + kThrHash);
  for (unsigned long long m = L0; m; m &= m - 1) {
    const uint32_t j = __ffsll(m) - 1;
    const unsigned long long qj = __ballot_sync(GMBE_FULL, (q0 >> j) & 1ull) |
                                  ((unsigned long long)__ballot_sync(GMBE_FULL, (q1 >> j) & 1ull) << 32);
    const uint32_t cj = __ballot_sync(GMBE_FULL, (crow >> j) & 1ull);
    if (lane == (j & 31)) {
      cols[j].q = qj;
      cols[j].hu = j < 32 ? T.hu0 : T.hu1;
      ts->ccol[j] = cj;
    }
  }
  __syncwarp();
  PH_STOP(A, 13);
  const uint32_t rlen0 = rec[5];
  ThrLevel stk[32];
  bool has = lane == 0;
  unsigned long long L = L0, SR = ((unsigned long long)rec[7] << 32) | rec[6];
  const uint32_t cand_all = nC >= 32 ? GMBE_FULL : ((1u << nC) - 1u);
  uint32_t C = cand_all, next = 0, Rm = 0, d = 0, dmask = 0;
  uint32_t bd = 0;  // tree depth (below the job's top) of this lane's level 0
  uint32_t n_nodes = 0, n_nonmax = 0, n_count = 0;
#ifdef GMBE_STATS
  unsigned long long st_l = 0, st_lp = 0, st_later = 0, st_push = 0;  // path statistics (debug 32)
#endif
  unsigned long long abytes = 0, cks = 0;
#if GMBE_DONATE
  uint32_t tick = 0, hflag = 0;  // hflag: lane 0's in-flight read of ctrl.hungry (consumed 4 steps later)
#endif
  while (true) {
    if (has) {  // pop (Alg 2 L4) until a node with an untraversed candidate
      while (true) {
        if (next < 32 && (C & (GMBE_FULL << next))) break;
        if (d == 0) {
          has = false;
          break;
        }
        d--;
        const uint32_t rmp = stk[d].Rm, diff = Rm & ~rmp;  // {i} ∪ absorbed of the finished child
        next = __ffs(diff);
        for (uint32_t m = diff; m; m &= m - 1) SR -= ts->hv[__ffs(m) - 1];
        L = stk[d].L;
        C = stk[d].C;
        Rm = rmp;
        dmask &= ~(1u << d);
      }
    }
    const uint32_t idle = __ballot_sync(GMBE_FULL, !has);
    if (idle == GMBE_FULL) break;
#if GMBE_DONATE
    bool want = false;
    if (P.donate && (++tick & GMBE_THR_DONATE_MASK) == 0) {
      want = __shfl_sync(GMBE_FULL, hflag, 0) != 0 || (P.debug & 8);
      if (lane == 0) hflag = ld_volatile(&P.ctrl->hungry.v) != 0;  // latency hidden until the next check
    }
    // cross-warp donation to idle warps: up to GMBE_THR_DONATE_BURST levels per check
    for (uint32_t burst = 0; want && burst < GMBE_THR_DONATE_BURST; burst++) {
      // the donor: the lane whose shallowest stacked level with untraversed children is the
      // shallowest in the job's tree (the largest piece of remaining work)
      const uint32_t key =
          __reduce_min_sync(GMBE_FULL, dmask ? ((bd + (uint32_t)(__ffs(dmask) - 1)) << 5) | lane : kNone);
      want = key != kNone;
      if (want) {
        const uint32_t src = key & 31u;
        const uint32_t k = lane == src ? (uint32_t)(__ffs(dmask) - 1) : 0u;
        unsigned long long kL = 0, kSR = 0;
        uint32_t kC = 0, kRm = 0, knext = 0;
        if (lane == src) {
          kL = stk[k].L;
          kC = stk[k].C;
          kRm = stk[k].Rm;
          knext = __ffs((k + 1 < d ? stk[k + 1].Rm : Rm) & ~kRm);
          kSR = SR;
          for (uint32_t m = Rm & ~kRm; m; m &= m - 1) kSR -= ts->hv[__ffs(m) - 1];
        }
        const bool ok = donate_thr(P, T, lmap, A, ts, nC, rlen0, src, kL, kSR, kC, kRm, knext, scratch, scratch_end);
        if (ok && lane == src) {
          stk[k].C &= knext >= 32 ? GMBE_FULL : (1u << knext) - 1u;  // its remaining children left
          dmask &= ~(1u << k);
        }
        want = ok;
      }
    }
#endif
    if (idle) {  // in-warp donation: the r-th idle lane takes the shallowest level of the r-th donor
      const uint32_t donors = __ballot_sync(GMBE_FULL, dmask != 0);
      if (donors) {
        const uint32_t nd = min(__popc(idle), __popc(donors));
        unsigned long long* slot = smem;  // the setup hash region: 32 slots of 4 words
        const uint32_t rd = __popc(donors & lanemask_lt());
        if (dmask && rd < nd) {
          const uint32_t k = __ffs(dmask) - 1;
          unsigned long long* o = slot + 4 * rd;
          const uint32_t rmk = stk[k].Rm, ck = stk[k].C;
          const uint32_t nk = __ffs((k + 1 < d ? stk[k + 1].Rm : Rm) & ~rmk);
          unsigned long long srk = SR;
          for (uint32_t m = Rm & ~rmk; m; m &= m - 1) srk -= ts->hv[__ffs(m) - 1];
          o[0] = stk[k].L;
          o[1] = srk;
          o[2] = ((unsigned long long)rmk << 32) | ck;
          o[3] = ((unsigned long long)(bd + k) << 32) | nk;
          // the remaining children of level k are no longer this lane's
          stk[k].C = ck & (nk >= 32 ? GMBE_FULL : (1u << nk) - 1u);
          dmask &= ~(1u << k);
        }
        __syncwarp();
        const uint32_t ir = __popc(idle & lanemask_lt());
        if (!has && ir < nd) {
          const unsigned long long* o = slot + 4 * ir;
          has = true;
          L = o[0];
          SR = o[1];
          C = (uint32_t)o[2];
          Rm = (uint32_t)(o[2] >> 32);
          next = (uint32_t)o[3];
          bd = (uint32_t)(o[3] >> 32);
          d = 0;
          dmask = 0;
        }
        __syncwarp();  // the slots are read before any donor of a later step rewrites them
      }
    }
    if (!has) continue;
    // generate the child via the next candidate i (Alg 2 L6-13)
    const uint32_t i = __ffs(C & (GMBE_FULL << next)) - 1;
    next = i + 1;
    const unsigned long long lp = L & ts->row[i];  // L' = L ∩ N(v')
    const uint32_t lc = __popcll(lp);
    const uint32_t later = i >= 31 ? 0u : (C & (GMBE_FULL << (i + 1)));
    uint32_t pr = 0, ab = 0, cd = 0, ksum = 0;
    unsigned long long srab = 0;
    for (uint32_t m = later; m; m &= m - 1) {
      const uint32_t c = __ffs(m) - 1;
      const unsigned long long rc = ts->row[c];
      const uint32_t kp = __popcll(rc & L), kc = __popcll(rc & lp);
      const uint32_t bit = 1u << c;
      ksum += kp;
      if (kc == kp) pr |= bit;  // Thm 4.1
      if (kc == lc) {           // absorbed into R'
        ab |= bit;
        srab += ts->hv[c];
      } else if (kc) {
        cd |= bit;
      }
    }
    if (P.prune) C &= ~pr;
    n_nodes++;
    abytes += lc + ksum;
#ifdef GMBE_STATS
    if (P.debug & 32) {
      st_l += __popcll(L);
      st_lp += lc;
      st_later += __popc(later);
    }
#endif
    const uint32_t rl = rlen0 + __popc(Rm) + 1 + __popc(ab);
    // maximality (Alg 2 L14): |Γ(L')| == |R'|; the emission's SL = Σ_{u∈L'} hU(u) on the same pass
    bool maximal;
    unsigned long long sl = 0;
    if (lc == 1) {
      const uint32_t j = __ffsll(lp) - 1;
      maximal = ts->deg[j] == rl;
      sl = cols[j].hu;
    } else {  // |L'| >= 2: no Q pattern and no job candidate outside R' may cover L'
      const uint32_t outside = cand_all & ~(Rm | (1u << i) | ab);
      unsigned long long qa = ~0ull, m = lp;
      uint32_t ca = GMBE_FULL;
      for (; m; m &= m - 1) {
        const uint32_t j = __ffsll(m) - 1;
        const ThrCol tc = cols[j];
        qa &= tc.q;
        sl += tc.hu;
        ca &= ts->ccol[j];
        if (!qa && !(ca & outside)) {
          m &= m - 1;
          break;
        }
      }
      maximal = !qa && !(ca & outside);
      if (maximal)
        for (; m; m &= m - 1) sl += cols[__ffsll(m) - 1].hu;
    }
    if (!maximal) {
      n_nonmax++;
      continue;
    }
    // Output(L', R') (Alg 2 L15)
    const unsigned long long srn = SR + ts->hv[i] + srab;
    const uint32_t rmn = Rm | (1u << i) | ab;
    n_count++;
    cks += pair_hash(P, sl, srn);
    if (P.per_root) atomicAdd(P.per_root + T.root, 1ull);
    if (T.rlist && (P.out_ids || P.sring)) write_record_thr(P, T, ts, lp, lc, rlen0, rmn, rl);
    if (!cd) continue;
#ifdef GMBE_STATS
    if (P.debug & 32) st_push++;
#endif
    // push (Alg 2 L16)
    stk[d].L = L;
    stk[d].C = C;
    stk[d].Rm = Rm;
    if (next < 32 && (C & (GMBE_FULL << next))) dmask |= 1u << d;
    d++;
    L = lp;
    SR = srn;
    C = cd;
    Rm = rmn;
    next = 0;
  }
#ifdef GMBE_STATS
  if (P.debug & 32) {
    st_l = warp_sum64(st_l);
    st_lp = warp_sum64(st_lp);
    st_later = warp_sum64(st_later);
    st_push = warp_sum64(st_push);
    if (lane == 0) {
      atomicAdd(&P.ctrl->phase[8], st_l);
      atomicAdd(&P.ctrl->phase[9], st_lp);
      atomicAdd(&P.ctrl->phase[10], st_later);
      atomicAdd(&P.ctrl->phase[11], st_push);
    }
  }
#endif
  A.add(kAcNodes, warp_sum(n_nodes));
  A.add(kAcNonmax, warp_sum(n_nonmax));
  A.add(kAcCount, warp_sum(n_count));
  A.add(kAcAbytes, 4ull * warp_sum64r(abytes));
  A.add(kAcChecksum, warp_sum64r(cks));
  PH_STOP(A, 4);
  return true;
}

// SMALL: universes <= 64 bits (16-byte entries, register / thread tiers); else wide universes with
// lpe lanes per candidate entry
template <bool SMALL>
__device__ void run_task(const Params& P, const TaskCtx& T, uint32_t* top, uint32_t* stack_lo, uint32_t* stack_hi,
                         uint32_t lmap, Acc& A, unsigned long long* smem, ThrSmem* ts, uint32_t lpe) {
  const uint32_t lane = lane_id();
  uint32_t* cur = top;
  uint32_t* sp = stack_lo;  // first free word
  const bool split_mode = heavy(P, top[2], top[0]) || late_heavy(P, top[2], top[0]);
  if (split_mode) A.add(kAcSplits, 1);
  // register-resident DFS (one inline site): the whole task if its top has <= 32 candidates,
  // else every pushed child with <= 32 candidates
  const uint32_t* reg = nullptr;
  uint32_t* reg_scratch = stack_lo;
  if constexpr (SMALL) {
    if (top[0] <= 32) reg = top;
  }
  while (true) {
    if constexpr (SMALL) {
      if (reg) {
        const bool st = split_mode && reg == top;  // heavy top: publish its children (run_reg)
#ifndef GMBE_PROFILE
        const unsigned long long n0 = (P.debug & 32) ? A.get(kAcNodes) : 0ull;
#endif
        const bool thr = !st && !(P.debug & 16) && thr_eligible(P, T, reg) &&
                         run_thr(P, T, reg, lmap, A, ts, smem, reg_scratch, stack_hi);
        if (!thr) run_reg(P, T, reg, lmap, A, (RegLevel*)smem, reg_scratch, stack_hi, st, smem);
#ifndef GMBE_PROFILE
        if (P.debug & 32) {  // path statistics (experiments): jobs / nodes per tier
          const unsigned long long dn = A.get(kAcNodes) - n0;  // (a warp-wide shuffle)
          if (lane == 0) {
            atomicAdd(&P.ctrl->phase[thr ? 0 : 2], 1ull);
            atomicAdd(&P.ctrl->phase[thr ? 1 : 3], dn);
          }
        }
#endif
        if (reg == top) return;
        reg = nullptr;
        continue;
      }
    }
    __syncwarp();
    const uint32_t i = cur[3];
    if (i >= cur[0]) {  // all candidates of this node traversed: pop (Alg 2 L4)
      if (cur == top) break;
      sp = cur;
      const uint32_t po = cur[4];
      cur = po == kNone ? top : stack_lo + po;
      continue;
    }
    __syncwarp();
    if (lane == 0) cur[3] = i + 1;
    // child record bound: later candidates + the Γ-check scratch
    const uint64_t need = kHdr + T.W4 + (uint64_t)(cur[0] - i - 1) * T.E + 4ull * 32 * T.W + 16;
    if (!fits(P, sp + need, stack_hi)) return;
    uint32_t* ch = sp;  // children are generated on this warp's stack; only a published one is copied
    int r;
    if constexpr (SMALL) r = gen_child_small(P, T, cur, i, ch, A, smem);
    else r = gen_child(P, T, cur, i, ch, A, smem, lpe);
    // dynamic donation at the warp level (as donate_reg / donate_thr do in the tiers below): while
    // other warps are idle, the remaining children of cur -- its candidates after i, already
    // compacted by this child's Thm 4.1 pass -- go to the queue as one subtask (node (L, R, SR of cur,
    // those candidates)); its children, later sets and prune marks are the ones this warp would have
    // generated, so the tree and every counter are unchanged
    // Only a task's top donates, once (it keeps no remaining children afterwards), and never a top
    // that is itself a donated piece (node word 1 = 1): without that, a piece is re-donated by every
    // warp that takes it, copying O(n^2) entries (measured 2-3x slower W/O_PRUNE runs).  A node's
    // remaining children cannot be split between two warps: Thm 4.1's marks flow from every child to
    // its later siblings, in order.
    const uint32_t nrem = cur[0] - (i + 1);
#ifndef GMBE_WARP_DONATE_MIN
#define GMBE_WARP_DONATE_MIN 64  // warp-level donation of a top's remaining children: min(|L|, n) * n at least this
#endif
    if (GMBE_WARP_DONATE && P.donate && cur == top && !split_mode && cur[1] == 0 && nrem >= 4 &&
        min(cur[2], nrem) * nrem >= GMBE_WARP_DONATE_MIN && hungry(P)) {
      uint32_t* scr = align4(ch + (r == 2 ? rec_words(T, ch) : 0));
      const uint32_t n = nrem;
      const uint32_t words = kHdr + T.W4 + n * T.E;
      if (scr + words <= stack_hi) {
        const uint32_t* src = cur + kHdr + T.W4 + (size_t)(i + 1) * T.E;
        for (uint32_t j = lane; j < T.W4; j += 32) scr[kHdr + j] = cur[kHdr + j];
        for (uint32_t j = lane; j < n * T.E; j += 32) scr[kHdr + T.W4 + j] = src[j];
        if (lane == 0) {
          scr[0] = n;
          scr[1] = 1;  // a donated piece: its warp does not donate its top again
          scr[2] = cur[2];
          scr[3] = 0;
          scr[4] = kNone;
          scr[5] = cur[5];
          scr[6] = cur[6];
          scr[7] = cur[7];
        }
        __syncwarp();
        if (task_publish(P, T, lmap, T.rlist ? cur[5] : 0, scr, words, A)) {
          A.add(kAcDonations, 1);
          if (lane == 0) cur[0] = i + 1;  // cur's remaining children now belong to the subtask
          __syncwarp();
        }
      }
    }
    // Alg 4 L25: hand the child to the task queue as a self-contained subtask -- every child of a
    // heavy top, and (wide universes) any child that is itself heavy (reading B4)
    if (r == 2 && ((split_mode && cur == top) || (!SMALL && heavy_wide(P, lmap, ch[0])))) {
      PH_START(A);
      const bool done = task_publish(P, T, lmap, T.rlist ? ch[5] : 0, ch, rec_words(T, ch), A);
      PH_STOP(A, 7);
      if (done) continue;
    }
    if constexpr (SMALL) {
      if (r == 2 && ch[0] <= 32) {  // the child's subtree fits the register-resident DFS
        reg = ch;
        reg_scratch = align4(ch + rec_words(T, ch));
        continue;
      }
    }
    if (r == 2) {  // push (Alg 2 L16)
      if (lane == 0) {
        ch[4] = (cur == top) ? kNone : (uint32_t)(cur - stack_lo);
        ch[3] = 0;
      }
      __syncwarp();
      cur = ch;
      sp = align4(ch + rec_words(T, ch));
    }
  }
}

__device__ GMBE_NI_IF(GMBE_NI_DISPATCH) void dispatch_task(const Params& P, TaskCtx& T, uint32_t* top, uint32_t* lo, uint32_t* hi,
                              uint32_t lmap, Acc& A, unsigned long long* smem, ThrSmem* ts) {
  if (T.W <= 2) {
    small_task_init(P, T, lmap);
    run_task<true>(P, T, top, lo, hi, lmap, A, smem, ts, 0);
  } else {  // lanes per entry: the row words rounded up to a power of two, 4..32
    run_task<false>(P, T, top, lo, hi, lmap, A, smem, ts, T.W <= 4 ? 4u : T.W <= 8 ? 8u : T.W <= 16 ? 16u : 32u);
  }
}

// ---------------------------------------------------------------- root task (a3)
// Alg 3 L7 for a root scanned in suffix mode (below): is some vertex ranked before v_s adjacent to
// all of L_r?  Such a vertex x lies in N(u*) for the lowest-degree u* ∈ L_r, below rank r in its
// rank-sorted list, and has deg(x) >= |L_r|; each survivor of that filter is tested warp-wide by
// binary searches of the members of L_r in the sorted list N(x) (first miss ends the test).
__device__ bool earlier_dominator(const DevGraph& g, const uint32_t* Lr, uint32_t l, uint32_t r) {
  const uint32_t lane = lane_id();
  unsigned long long key = ~0ull;
  for (uint32_t j = lane; j < l; j += 32) {
    const uint32_t u = Lr[j];
    key = min(key, ((unsigned long long)(g.off_u[u + 1] - g.off_u[u]) << 32) | j);
  }
  for (int o = 16; o; o >>= 1) key = min(key, (unsigned long long)__shfl_xor_sync(GMBE_FULL, key, o));
  const uint32_t us = Lr[(uint32_t)key];
  const uint32_t* a = g.adj_u + g.off_u[us];
  const uint32_t n = r ? upper_rank(a, (uint32_t)(key >> 32), r - 1) : 0u;  // ranks < r
  for (uint32_t b = 0; b < n; b += 32) {
    const uint32_t x = b + lane < n ? __ldg(a + b + lane) : kNone;
    uint32_t xb = 0, xd = 0;
    if (x != kNone) {
      xb = g.off_v[x];
      xd = g.off_v[x + 1] - xb;
    }
    uint32_t cand = __ballot_sync(GMBE_FULL, x != kNone && xd >= l);
    while (cand) {
      const uint32_t src = __ffs(cand) - 1;
      cand &= cand - 1;
      const uint32_t cb = __shfl_sync(GMBE_FULL, xb, src), cd = __shfl_sync(GMBE_FULL, xd, src);
      bool all = true;
      for (uint32_t base = 0; base < l && all; base += 32) {
        const uint32_t j = base + lane;
        all = __all_sync(GMBE_FULL, j >= l || bsearch_rank(g.adj_v + cb, cd, Lr[j]));
      }
      if (all) return true;
    }
  }
  return false;
}
#ifndef GMBE_DENSE_RATIO
#define GMBE_DENSE_RATIO 32  // dense root tables when the scanned rank range <= this x the wedges
#endif
#ifndef GMBE_SUFFIX_MAX_KEEP_L
#define GMBE_SUFFIX_MAX_KEEP_L 1024  // universes up to this size keep a full (dense) scan and their Γ index (256: bx_work 25.45 ms, 1024: 22.95)
#endif
#ifndef GMBE_SORT_MIN
#define GMBE_SORT_MIN 1024  // small-universe roots with at least this many wedges build their rows by sorting
#endif
#ifndef GMBE_SORT_MAX
#define GMBE_SORT_MAX 4096  // heavier roots keep the dense table: one pass has a shorter chain than six sweeps (65536: gh_work 14.4 vs 14.2 ms)
#endif
#ifndef GMBE_SUFFIX_MIN
#define GMBE_SUFFIX_MIN 8192  // roots with at least this many wedges may scan only later ranks
#endif

// Tiny roots (|L_r| <= 32 and <= 32 wedges: most roots of light-tailed graphs such as the DBLP
// shape) are built entirely in registers: lane p holds wedge p = (u_i, v) after one scan of the
// degrees; __match_any_sync groups the wedges by v, so a group leader knows k(v) = |N(v) ∩ L_r| (its
// group size) and the row N(v) ∩ L_r (an OR-reduction over the group) without a hash table, an
// occupied list, a sort or a table clean-up.  Classification (Alg 3 L3-7), emission, the Γ index
// (X2 rows) and the candidate record (rank order by counting smaller candidates) are then the same
// as run_root's, written straight to the warp's dynamic region.  lane j < l: (beg, deg) of N(u_j).
__device__ bool run_root_tiny(const Params& P, uint32_t r, uint32_t l, const uint32_t* Lr, uint32_t beg,
                              uint32_t deg, uint32_t wedges, WarpMem& M, Acc& A, TaskCtx& Tc, uint32_t** top,
                              uint32_t** lo) {
  const uint32_t lane = lane_id();
  const DevGraph& g = P.g;
  // wedge p -> (i, v): owner i by a binary search over the exclusive degree prefix
  uint32_t inc = deg;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t t = __shfl_up_sync(GMBE_FULL, inc, o);
    if (lane >= (uint32_t)o) inc += t;
  }
  const uint32_t excl = inc - deg;
  uint32_t own = 0;
#pragma unroll
  for (int st = 16; st; st >>= 1) {
    const uint32_t cand = own + st;
    const uint32_t e = __shfl_sync(GMBE_FULL, excl, cand & 31);
    if (cand < l && e <= lane) own = cand;
  }
  const uint32_t ob = __shfl_sync(GMBE_FULL, beg, own), oe = __shfl_sync(GMBE_FULL, excl, own);
  const bool act0 = lane < wedges;
  const uint32_t v = act0 ? __ldg(g.adj_u + ob + lane - oe) : kNone;
  const bool act = act0 && v != r;
  const uint32_t peers = __match_any_sync(GMBE_FULL, act ? v : kNone - 1 - lane);
  const uint32_t k = __popc(peers);
  // the row N(v) ∩ L_r over the universe: bit i iff a wedge of u_i is in v's group (one ballot per
  // member -- a per-group OR-reduction would serialise over the groups)
#if GMBE_TINY_REDUX
  const uint32_t row = __reduce_or_sync(peers, 1u << own);
#else
  uint32_t row = 0;
  for (uint32_t i = 0; i < l; i++)
    if (peers & __ballot_sync(GMBE_FULL, act0 && own == i)) row |= 1u << i;
#endif
  const bool leader = act && lane == (uint32_t)(__ffs(peers) - 1);
  // Alg 3 L3-7: k == |L| -> R (skip the root unless v_s is R's earliest vertex); later -> C
  const bool isR = leader && k == l;
  if (__any_sync(GMBE_FULL, isR && v < r)) return false;
  const bool isC = leader && k < l && v > r;
  const bool isX = leader && k >= 2;  // X2: can cover an L' with |L'| >= 2
  const unsigned long long hv_r = g.hv[r];
  const unsigned long long hvx = isR ? g.hv[v] : 0ull;
  const unsigned long long sl = warp_sum64r(lane < l ? hash_u(P, Lr[lane]) : 0ull);
  const unsigned long long sr = warp_sum64r(hvx) + hv_r;
  const uint32_t bR = __ballot_sync(GMBE_FULL, isR), bC = __ballot_sync(GMBE_FULL, isC),
                 bX = __ballot_sync(GMBE_FULL, isX);
  const uint32_t nR = __popc(bR), nC = __popc(bC), nx = __popc(bX);
  uint32_t* gx = align4(M.dyn);
  uint32_t* rec = align4(gx + 4 + 2 * nx + r4(nx));
  if (!fits(P, rec + kHdr + 4 + 4 * nC + 64, M.dyn_end)) return false;
  A.add(kAcRootsRun, 1);
  A.add(kAcCount, 1);  // emit (L_r, R_r) (A5)
  A.add(kAcChecksum, pair_hash(P, sl, sr));
  if (P.per_root && lane == 0) atomicAdd(P.per_root + r, 1ull);
  if (M.rbuf) {
    if (lane == 0) M.rbuf[0] = r;
    if (isR) M.rbuf[1 + __popc(bR & lanemask_lt())] = v;
    __syncwarp();
    if (P.out_ids || P.sring) write_record(P, nullptr, 0, nullptr, Lr, l, M.rbuf, nR + 1);
  }
  if (nC == 0) return false;
  // Γ index (universe <= 32 bits, |X2| <= 32: the rows are lane-resident in every task of the root)
  if (lane == 0) {
    gx[0] = nx;
    gx[1] = l;
  }
  if (isX) {
    const uint32_t xp = __popc(bX & lanemask_lt());
    ((unsigned long long*)(gx + 4))[xp] = row;
    gx[4 + 2 * nx + xp] = v;
  }
  // the root's node record: candidates in rank order (a candidate's position = smaller candidates)
  uint32_t pos = 0;
  for (uint32_t m = bC; m; m &= m - 1) pos += __shfl_sync(GMBE_FULL, v, __ffs(m) - 1) < v;
  if (isC) ((uint4*)(rec + kHdr + 4))[pos] = make_uint4(row, v, k, 0);
  if (lane < 4) rec[kHdr + lane] = lane == 0 ? (l >= 32 ? GMBE_FULL : (1u << l) - 1u) : 0u;
  if (lane == 0) {
    rec[0] = nC;
    rec[1] = 0;
    rec[2] = l;
    rec[3] = 0;
    rec[4] = kNone;
    rec[5] = nR + 1;
    rec[6] = (uint32_t)sr;
    rec[7] = (uint32_t)(sr >> 32);
  }
  __syncwarp();
  Tc.map = Lr;
  Tc.W = 1;
  Tc.W4 = 4;
  Tc.E = 4;
  Tc.root = r;
  Tc.rlist = M.rbuf;
  Tc.cols = nullptr;
  Tc.gx = gx;
  Tc.ncw = 0;
  Tc.auxref = 0;
  if (heavy(P, l, nC)) {  // the root will be split: share its Γ index with the subtasks
    const uint32_t words = 4 + 2 * nx + r4(nx);
    const uint32_t co = pool_alloc(P, r4(words));
    if (co != kNone) {
      uint32_t* cp = pool_ptr(P, co);
      for (uint32_t j = lane; j < words; j += 32) cp[j] = gx[j];
      __syncwarp();
      Tc.gx = cp;
      Tc.auxref = co + 1;
    }
  }
  *top = rec;
  *lo = align4(rec + kHdr + 4 + 4 * nC);
  return true;
}

// Root v_s (rank r): L_r = N(v_s); wedge scan of N2(v_s) with k(v) = |N(v) ∩ L_r|.  Emits the root
// biclique and, if it has candidates, prepares its node record as a task (Tc, *top, stack from *lo)
// for the caller's single dispatch site; returns whether it did.
__device__ GMBE_NI_IF(GMBE_NI_ROOT) bool run_root(const Params& P, uint32_t r, uint32_t lb, uint32_t l, WarpMem& M,
                                                  Acc& A, TaskCtx& Tc, uint32_t** top, uint32_t** lo) {
  const uint32_t lane = lane_id();
  const DevGraph& g = P.g;  // N(v_s) = adj_v[lb, lb + l) (prefetched by the caller)
  if (l == 0) return false;  // isolated vertex: in no biclique (A17)
  const uint32_t* Lr = g.adj_v + lb;
  const unsigned long long hv_r = g.hv[r];  // issued early, consumed at the root's emission
  uint32_t wp = 0, beg0 = 0;  // (lane j < 32: beg0 / wp = N(u_j) of the first 32 members)
  for (uint32_t j = lane; j < l; j += 32) {
    const uint32_t u = Lr[j];
    const uint32_t b = g.off_u[u], d = g.off_u[u + 1] - b;
    if (j < 32) beg0 = b;
    wp += d;
  }
  const uint32_t wedges = warp_sum(wp);
  A.add(kAcAbytes, 4ull * (l + wedges));
  if (l <= 32 && wedges <= 32 && !(P.debug & (128 | 2048)))  // tiny root: register-resident build
    return run_root_tiny(P, r, l, Lr, beg0, wp, wedges, M, A, Tc, top, lo);
  // Suffix mode (B200 addition, reading B5): a root with many wedges but few of them to
  // later-ranked vertices (high degree rank: few candidates, huge excluded set) counts k only over
  // the rank suffix of each list; the skip test (Alg 3 L7) then looks for an earlier dominator
  // directly, and the children test maximality without a Γ index (gamma_is_r).
  uint32_t after = kNone, scanned = wedges;
  if (P.debug & 128) {  // tests: every root in suffix mode
    after = r;
  } else if (wedges >= GMBE_SUFFIX_MIN && !(P.debug & 64)) {
    // a universe that a dense full scan can afford keeps its Γ index (thread tier / Γ columns): up to
    // 256 vertices always, up to GMBE_SUFFIX_MAX_KEEP_L when enough wedges reach later ranks that
    // the subtree is likely to be worked (B5; bx-shaped roots of 300-1,000 vertices with ~1,000 later
    // wedges vs GH-shaped hubs with ~100)
    const bool keepable = l <= GMBE_SUFFIX_MAX_KEEP_L && g.n_v <= P.tmax && (uint64_t)g.n_v <= 16ull * wedges &&
                          !(P.debug & 256);
    if (!keepable || l > 256) {
      uint32_t sp = 0;
      for (uint32_t j = lane; j < l; j += 32) {
        const uint32_t u = Lr[j], ub = g.off_u[u], du = g.off_u[u + 1] - ub;
        sp += du - upper_rank(g.adj_u + ub, du, r);
      }
      sp = warp_sum(sp);
#ifndef GMBE_SUFFIX_RATIO
#define GMBE_SUFFIX_RATIO 4  // suffix mode when fewer than 1/ratio of the wedges reach later ranks
#endif
#ifndef GMBE_SUFFIX_KEEP_SP
#define GMBE_SUFFIX_KEEP_SP 512
#endif
      if ((unsigned long long)GMBE_SUFFIX_RATIO * sp < wedges && !(keepable && sp >= GMBE_SUFFIX_KEEP_SP)) {
        after = r;
        scanned = sp;
      }
    }
  }
  if (after != kNone && (P.debug & 128)) {
    uint32_t sp = 0;
    for (uint32_t j = lane; j < l; j += 32) {
      const uint32_t u = Lr[j], ub = g.off_u[u], du = g.off_u[u + 1] - ub;
      sp += du - upper_rank(g.adj_u + ub, du, r);
    }
    scanned = warp_sum(sp);
  }
  const uint32_t T = next_pow2(max(64u, 2u * scanned));
  if (T > P.tmax || scanned > P.omax) {
    if (lane == 0) atomicOr(&P.ctrl->error, kErrArena);
    return false;
  }
  const uint32_t shift = 32 - (31 - __clz(T)), mask = T - 1;
  const bool stab = kSmemTable && T <= kSmemTable;  // shared-memory table
  uint32_t* keys = stab ? M.skeys : M.keys;
  unsigned long long* vals = stab ? M.svals : M.vals;
  uint32_t* occl = stab ? M.socc : M.occ;
  const bool small = l <= 64;  // rows (<= 64 bits) straight from the table
  // Sort mode (B200 addition): a small-universe root with a mid-size wedge scan (the bulk of the
  // root-construction time on the work-shaped graphs) builds its rows by sorting the wedge keys
  // (rank << 6 | member index) in a per-root buffer -- LSD radix passes over the rank bits, then one
  // sweep OR-ing each run of equal rank into its row -- instead of a per-warp table indexed by rank
  // or by hash.  The buffer (~5 words per wedge) stays in L2, where the dense table's scattered
  // 8-byte slots (n_v per warp) miss to DRAM.  The occupied ranks come out in rank order, with the
  // same rows as the tables' (so the same classification, Γ index and candidate order).
  // Scratch at the end of the warp's dynamic region: keys | keys' | ranks | rows (u64).
  uint32_t* dyn_end = M.dyn_end;  // the root record and Γ index must end below the sort scratch
  const uint64_t sort_words = 5ull * r4(scanned) + 32;
  const bool sorted = small && after == kNone && (!stab || (P.debug & 8192)) && !(P.debug & 4096) &&
                      g.n_v < (1u << 26) &&  // keys rank << 6 | member must fit 32 bits
                      (scanned >= P.sort_min || (P.debug & 8192)) && scanned <= GMBE_SORT_MAX &&
                      M.dyn + 4 * sort_words <= M.dyn_end;
  uint32_t* s_ck = nullptr;
  if (sorted) {
    dyn_end = (uint32_t*)((uintptr_t)(M.dyn_end - sort_words) & ~(uintptr_t)15);
    s_ck = dyn_end + 2 * r4(scanned);
    keys = s_ck;
    vals = (unsigned long long*)(s_ck + r4(scanned));
  }
  // Dense mode (heavy roots): the warp's table values indexed by rank directly (n_v <= table
  // slots).  Pass 1 is then fire-and-forget atomics (no probing), and the occupied list comes from
  // a scan of the rank range -- in rank order, so the candidates need no sort.
  const uint32_t lo_v = after != kNone ? r + 1 : 0u;
  // The occupied ranks are marked in a per-warp bitmap as well (fire-and-forget atomics), so the
  // scan for them reads (n_v - lo_v)/32 words instead of the whole value range.
  const bool dense = !stab && !sorted && g.n_v <= P.tmax && !(P.debug & 256) &&
                     ((uint64_t)(g.n_v - lo_v) <= (uint64_t)GMBE_DENSE_RATIO * scanned || (P.debug & 512));
  const bool ident = sorted;  // occupied slot j is entry j of the compact (rank, row) arrays
  PH_START(A);
  // pass 1 (Alg 3 L2-3)
  uint32_t nocc = 0;
  if (sorted) {
    uint32_t* kb = dyn_end;
    uint32_t* kt = dyn_end + r4(scanned);
    uint32_t wpos = 0;
    for_each_wedge(g, Lr, l, [&](uint32_t i, uint32_t v, bool act) {
      if (act) kb[wpos + lane] = (v << 6) | i;
      wpos += __popc(__ballot_sync(GMBE_FULL, act));
    });
    __syncwarp();
    const uint32_t n = wpos;
    const uint32_t vb = 32 - __clz(max(g.n_v, 2u) - 1);
    const uint32_t passes = vb <= 9 ? 1u : vb <= 18 ? 2u : 3u, db = (vb + passes - 1) / passes;
    for (uint32_t p = 0; p < passes; p++)
      warp_radix_pass32(p & 1 ? kt : kb, p & 1 ? kb : kt, n, 6 + p * db, db, (uint32_t*)M.sm_sort);
    const uint32_t* srt = passes & 1 ? kt : kb;
    __syncwarp();
    // runs of equal rank -> (rank, row); a run may continue into the next chunk (carry)
    uint32_t cv = kNone;
    unsigned long long crow = 0;
    for (uint32_t b = 0; b < n; b += 32) {
      const uint32_t j = b + lane;
      const bool in = j < n;
      const uint32_t key = in ? srt[j] : 0u;
      const uint32_t v = in ? key >> 6 : kNone;
      unsigned long long x = in ? 1ull << (key & 63u) : 0ull;
      const uint32_t v0 = __shfl_sync(GMBE_FULL, v, 0);
      if (cv != kNone && v0 != cv && cv != r) {  // the carried run ended with the previous chunk
        if (lane == 0) {
          s_ck[nocc] = cv;
          vals[nocc] = crow;
        }
        nocc++;
      }
      if (lane == 0 && v == cv) x |= crow;
      const uint32_t vp = __shfl_up_sync(GMBE_FULL, v, 1);
      const uint32_t heads = __ballot_sync(GMBE_FULL, lane == 0 || v != vp);
      const uint32_t ss = 31 - __clz(heads & (lane == 31 ? GMBE_FULL : ((2u << lane) - 1u)));
#pragma unroll
      for (uint32_t o = 1; o < 32; o <<= 1) {
        const unsigned long long y = ((unsigned long long)__shfl_up_sync(GMBE_FULL, (uint32_t)(x >> 32), o) << 32) |
                                     __shfl_up_sync(GMBE_FULL, (uint32_t)x, o);
        if (lane >= o && lane - o >= ss) x |= y;
      }
      const uint32_t vn = __shfl_down_sync(GMBE_FULL, v, 1);
      const bool last = b + 32 >= n;
      const bool end = in && (lane < 31 ? vn != v : last);
      const bool emit = end && v != r;
      const uint32_t be = __ballot_sync(GMBE_FULL, emit);
      if (emit) {
        const uint32_t q = nocc + __popc(be & lanemask_lt());
        s_ck[q] = v;
        vals[q] = x;
      }
      nocc += __popc(be);
      cv = last ? kNone : __shfl_sync(GMBE_FULL, v, 31);
      crow = ((unsigned long long)__shfl_sync(GMBE_FULL, (uint32_t)(x >> 32), 31) << 32) |
             __shfl_sync(GMBE_FULL, (uint32_t)x, 31);
    }
    __syncwarp();
  } else if (dense) {
    uint32_t* bits = M.bits;
    for_each_wedge(g, Lr, l, [&](uint32_t i, uint32_t v, bool act) {
      if (act && v != r) {
        if (small) atomicOr(vals + v, 1ull << i);
        else atomicAdd(vals + v, 1ull);
        atomicOr(bits + (v >> 5), 1u << (v & 31));
      }
    }, after);
    __syncwarp();
    __threadfence();
    // occupied ranks from the bitmap, in rank order; the words are cleared behind the scan
    const uint32_t wend = (g.n_v + 31) >> 5;
    for (uint32_t wb = lo_v >> 5; wb < wend; wb += 64) {
      const uint32_t w0 = wb + lane, w1 = wb + 32 + lane;
      const uint32_t x0 = w0 < wend ? __ldcg(bits + w0) : 0u;  // L2: pass 1 wrote with atomics
      const uint32_t x1 = w1 < wend ? __ldcg(bits + w1) : 0u;
      if (x0) bits[w0] = 0u;
      if (x1) bits[w1] = 0u;
#pragma unroll
      for (int h = 0; h < 2; h++) {
        uint32_t x = h ? x1 : x0;
        const uint32_t c = __popc(x);
        uint32_t incl = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t t = __shfl_up_sync(GMBE_FULL, incl, o);
          if (lane >= (uint32_t)o) incl += t;
        }
        uint32_t q = nocc + incl - c;
        const uint32_t base = (h ? w1 : w0) << 5;
        for (; x; x &= x - 1) occl[q++] = base + __ffs(x) - 1;
        nocc += __shfl_sync(GMBE_FULL, incl, 31);
      }
    }
    __syncwarp();
  } else {
    for_each_wedge(g, Lr, l, [&](uint32_t i, uint32_t v, bool act) {
      const bool a = act && v != r;
      const uint32_t h = ht_insert_warp(keys, shift, mask, v, a, occl, nocc);
      if (a) {
        if (small) atomicOr(vals + h, 1ull << i);
        else atomicAdd(vals + h, 1ull);
      }
    }, after);
    __syncwarp();
  }
  PH_STOP(A, 0);
  // classify: k == |L| -> R (root skipped unless v_s is the earliest vertex of R, Alg 3 L7);
  // later-ordered partial neighbours -> C (Alg 3 L5-6); earlier-ordered ones are never candidates
  unsigned long long* sortbuf = (unsigned long long*)align4(M.dyn);
  const uint32_t W = (l + 31) / 32, W4 = r4(W), E = r4(W + 2);
  uint32_t nC = 0, nR = 0, nx2 = 0, sum2 = 0;
  bool skip = false;
  unsigned long long sr = 0;
  const bool sort_fits = fits(P, (uint32_t*)(sortbuf + next_pow2(max(nocc, 1u))) + 64, dyn_end);
#ifndef GMBE_CLS_UNROLL
#define GMBE_CLS_UNROLL 2  // occupied-list chunks whose loads are in flight together (memory-level parallelism)
#endif
  for (uint32_t b0 = 0; b0 < nocc && sort_fits; b0 += 32 * GMBE_CLS_UNROLL) {
  uint32_t sq[GMBE_CLS_UNROLL], vq[GMBE_CLS_UNROLL];
  unsigned long long xq[GMBE_CLS_UNROLL];
#pragma unroll
  for (int q = 0; q < GMBE_CLS_UNROLL; q++)
    sq[q] = b0 + 32 * q + lane < nocc ? (ident ? b0 + 32 * q + lane : occl[b0 + 32 * q + lane]) : 0u;
#pragma unroll
  for (int q = 0; q < GMBE_CLS_UNROLL; q++) {
    const bool o = b0 + 32 * q + lane < nocc;
    vq[q] = o ? (dense ? sq[q] : ldv(keys + sq[q])) : 0u;
    xq[q] = o ? ldv(vals + sq[q]) : 0ull;
  }
#pragma unroll
  for (int q = 0; q < GMBE_CLS_UNROLL; q++) {
    const uint32_t b = b0 + 32 * q;
    if (b >= nocc) break;
    const uint32_t j = b + lane;
    const bool occ = j < nocc;
    const uint32_t s = sq[q];
    const uint32_t v = vq[q];
    uint32_t c = 0;
    if (occ) {
      const unsigned long long x = xq[q];
      c = small ? __popcll(x) : (uint32_t)x;
    }
    const bool isR = occ && c == l;
    skip |= isR && v < r;
    // X2: only 2-hop vertices sharing >= 2 universe vertices can cover an L' with |L'| >= 2
    nx2 += __popc(__ballot_sync(GMBE_FULL, occ && c >= 2));
    sum2 += occ && c >= 2 ? c : 0u;
    const bool isC = occ && !isR && v > r;
    if (isR) sr += g.hv[v];
    const uint32_t bR = __ballot_sync(GMBE_FULL, isR);
    if (M.rbuf && isR) M.rbuf[1 + nR + __popc(bR & lanemask_lt())] = v;
    nR += __popc(bR);
    const uint32_t bC = __ballot_sync(GMBE_FULL, isC);
    if (isC) sortbuf[nC + __popc(bC & lanemask_lt())] = ((unsigned long long)v << 32) | s;
    nC += __popc(bC);
  }
  }
  skip = __any_sync(GMBE_FULL, skip);
  if (after != kNone && !skip && sort_fits) skip = earlier_dominator(g, Lr, l, r);
  sum2 = warp_sum(sum2);
  PH_STOP(A, 1);
  // Γ index over X2 = {x in the 2-hop set X : |N(x) ∩ L_r| >= 2} (the maximality test of an L' with
  // |L'| >= 2 only counts vertices covering >= 2 universe vertices; |L'| = 1 uses the degree): gx for
  // universes <= 64 bits, columns otherwise (see TaskCtx).  x2 = position of x among X2 in occ order.
  const uint32_t ncw = (nx2 + 31) / 32;
  uint32_t* aux = align4((uint32_t*)(sortbuf + next_pow2(max(nC, 1u))));
  const uint64_t aux_words = small ? 4ull + 2ull * nx2 + r4(nx2) + r4(l + 1) + sum2 : (uint64_t)l * ncw;
  const bool want_aux = !skip && nC > 0 && after == kNone && aux_words <= P.col_budget;
  const bool want_cols = want_aux && !small;
  uint32_t* cols = aux;
  uint32_t* gx = aux;
  uint32_t* rec = align4(aux + (want_aux ? aux_words : 0));
  const uint64_t rec_need = kHdr + W4 + (uint64_t)nC * E;
  if (sort_fits && !skip && fits(P, rec + rec_need + 64, dyn_end)) {
    A.add(kAcRootsRun, 1);
    sr = warp_sum64r(sr) + hv_r;
    unsigned long long sl = 0;
    for (uint32_t j = lane; j < l; j += 32) sl += hash_u(P, Lr[j]);
    sl = warp_sum64r(sl);
    A.add(kAcCount, 1);  // emit (L_r, R_r) (A5)
    A.add(kAcChecksum, pair_hash(P, sl, sr));
    if (P.per_root && lane == 0) atomicAdd(P.per_root + r, 1ull);
    if (M.rbuf) {
      if (lane == 0) M.rbuf[0] = r;
      __syncwarp();
      if (P.out_ids || P.sring) write_record(P, nullptr, 0, nullptr, Lr, l, M.rbuf, nR + 1);
    }
    PH_STOP(A, 8);
    if (want_aux && small) {
      // gx: rows of the X2 vertices, and per universe vertex u_j the list of its X2 neighbours
      unsigned long long* xrow = (unsigned long long*)(gx + 4);
      uint32_t* xid = gx + 4 + 2 * nx2;
      uint32_t* coff = xid + r4(nx2);
      uint32_t* cx = coff + r4(l + 1);
      if (lane == 0) {
        gx[0] = nx2;
        gx[1] = l;
      }
      uint32_t n2 = 0;
      for (uint32_t b0 = 0; b0 < nocc; b0 += 32 * GMBE_CLS_UNROLL) {
        uint32_t sq[GMBE_CLS_UNROLL];
        unsigned long long rq[GMBE_CLS_UNROLL];
#pragma unroll
        for (int q = 0; q < GMBE_CLS_UNROLL; q++)
          sq[q] = b0 + 32 * q + lane < nocc ? (ident ? b0 + 32 * q + lane : occl[b0 + 32 * q + lane]) : 0u;
#pragma unroll
        for (int q = 0; q < GMBE_CLS_UNROLL; q++) rq[q] = b0 + 32 * q + lane < nocc ? ldv(vals + sq[q]) : 0ull;
#pragma unroll
        for (int q = 0; q < GMBE_CLS_UNROLL; q++) {
          if (b0 + 32 * q >= nocc) break;
          const uint32_t slot = sq[q];
          const unsigned long long row = rq[q];
          const bool is2 = __popcll(row) >= 2;
          const uint32_t bal = __ballot_sync(GMBE_FULL, is2);
          if (is2) {
            const uint32_t pos = n2 + __popc(bal & lanemask_lt());
            xrow[pos] = row;
            xid[pos] = dense ? slot : ldv(keys + slot);
          }
          n2 += __popc(bal);
        }
      }
      __syncwarp();
      // list lengths: lane j counts universe vertex j (cnt0) and j + 32 (cnt1).  With |X2| <= 64 the
      // rows are lane-resident in every task of this root (small_task_init) and no list is needed.
      uint32_t cnt0 = 0, cnt1 = 0;
      for (uint32_t b = 0; b < nx2 && nx2 > 64; b += 32) {
        const unsigned long long row = b + lane < nx2 ? xrow[b + lane] : 0ull;
        unsigned long long any = ((unsigned long long)__reduce_or_sync(GMBE_FULL, (uint32_t)(row >> 32)) << 32) |
                                 __reduce_or_sync(GMBE_FULL, (uint32_t)row);
        while (any) {
          const uint32_t j = __ffsll(any) - 1;
          any &= any - 1;
          const uint32_t c = __popc(__ballot_sync(GMBE_FULL, (row >> j) & 1ull));
          if (lane == (j & 31)) {
            if (j < 32) cnt0 += c;
            else cnt1 += c;
          }
        }
      }
      uint32_t carry = 0, cur0 = 0, cur1 = 0;
      for (uint32_t h = 0; h < 2 && nx2 > 64; h++) {  // (|X2| <= 64: rows lane-resident, no lists)
        const uint32_t j = h * 32 + lane;
        const uint32_t c = h ? cnt1 : cnt0;
        uint32_t inc = c;
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t t = __shfl_up_sync(GMBE_FULL, inc, o);
          if (lane >= (uint32_t)o) inc += t;
        }
        const uint32_t ex = carry + inc - c;
        if (j <= l) coff[j] = ex;
        if (h == 0) cur0 = ex;
        else cur1 = ex;
        carry += __shfl_sync(GMBE_FULL, inc, 31);
      }
      if (lane == 0 && l == 64 && nx2 > 64) coff[64] = carry;
      __syncwarp();
      for (uint32_t b = 0; b < nx2 && nx2 > 64; b += 32) {
        const uint32_t x = b + lane;
        const unsigned long long row = x < nx2 ? xrow[x] : 0ull;
        unsigned long long any = ((unsigned long long)__reduce_or_sync(GMBE_FULL, (uint32_t)(row >> 32)) << 32) |
                                 __reduce_or_sync(GMBE_FULL, (uint32_t)row);
        while (any) {
          const uint32_t j = __ffsll(any) - 1;
          any &= any - 1;
          const bool bit = (row >> j) & 1ull;
          const uint32_t bal = __ballot_sync(GMBE_FULL, bit);
          const uint32_t base = __shfl_sync(GMBE_FULL, j < 32 ? cur0 : cur1, j & 31);
          if (bit) cx[base + __popc(bal & lanemask_lt())] = x;
          if (lane == (j & 31)) {
            if (j < 32) cur0 += __popc(bal);
            else cur1 += __popc(bal);
          }
        }
      }
      __syncwarp();
    }
    PH_STOP(A, 9);
    if (nC > 0) {
      // root node record: candidates in rank order (Alg 2 L6 "smallest first")
      __syncwarp();
      PH_STOP(A, 3);
      if (!dense && !sorted)  // dense / sort mode: occupied list (and so the candidates) already in rank order
        warp_sort_keys(sortbuf, nC, M.sm_sort, (unsigned long long*)rec, 32 - __clz(max(g.n_v, 2u) - 1));
      PH_STOP(A, 2);
      uint32_t* ent = rec + kHdr + W4;
      for (uint32_t j = lane; j < nC; j += 32) {
        const unsigned long long kv = sortbuf[j];
        const uint32_t s = (uint32_t)kv;
        const unsigned long long x = ldv(vals + s);
        uint32_t* ee = ent + (size_t)j * E;
        if (small) {
          ee[0] = (uint32_t)x;
          if (W == 2) ee[1] = (uint32_t)(x >> 32);
          ee[W + 1] = __popcll(x);
        } else {
          for (uint32_t w = 0; w < W; w++) ee[w] = 0;
          ee[W + 1] = (uint32_t)x;
          vals[s] = kCTag | j;
        }
        ee[W] = (uint32_t)(kv >> 32);
      }
      __syncwarp();
      PH_STOP(A, 10);
      if (!small) {
        // pass 2: candidate rows over L_r, and the Γ columns: table value := x << 32 | C tag + entry
        // table value := (x2 + 1) << 32 (0: not in X2) | C tag + entry
        uint32_t n2 = 0;
        for (uint32_t b = 0; b < nocc; b += 32) {
          const uint32_t x = b + lane;
          const uint32_t s2 = x < nocc ? occl[x] : 0u;
          const unsigned long long v2 = x < nocc ? ldv(vals + s2) : 0ull;
          const bool isc = (v2 & kCTag) != 0;
          const uint32_t k = isc ? ent[(size_t)(uint32_t)(v2 & 0x7fffffffull) * E + W + 1] : (uint32_t)v2;
          const bool is2 = x < nocc && k >= 2;
          const uint32_t bal = __ballot_sync(GMBE_FULL, is2);
          const unsigned long long x2 = is2 ? (unsigned long long)(n2 + __popc(bal & lanemask_lt()) + 1) : 0ull;
          n2 += __popc(bal);
          if (x < nocc) vals[s2] = (x2 << 32) | (isc ? (0x80000000ull | (uint32_t)v2) : 0ull);
        }
        if (want_cols)
          for (uint64_t j = lane; j < (uint64_t)l * ncw; j += 32) cols[j] = 0;
        __syncwarp();
        for_each_wedge(g, Lr, l, [&](uint32_t i, uint32_t v, bool act) {
          if (act && v != r) {
            const uint32_t h = dense ? v : ht_find(keys, shift, mask, v);
            const unsigned long long x = ldv(vals + h);
            const uint32_t xi = (uint32_t)(x >> 32);
            if (want_cols && xi) atomicOr(cols + (size_t)i * ncw + ((xi - 1) >> 5), 1u << ((xi - 1) & 31));
            if (x & 0x80000000ull) atomicOr(ent + (size_t)(x & 0x7fffffffull) * E + (i >> 5), 1u << (i & 31));
          }
        }, after);
        __syncwarp();
        __threadfence();  // rows / columns were built with atomics: drop stale L1 lines
      }
      PH_STOP(A, 11);
      for (uint32_t w = lane; w < W4; w += 32) {
        const uint32_t bits = w < W ? l - w * 32 : 0u;
        rec[kHdr + w] = bits >= 32 ? GMBE_FULL : ((1u << bits) - 1u);
      }
      if (lane == 0) {
        rec[0] = nC;
        rec[1] = 0;
        rec[2] = l;
        rec[3] = 0;
        rec[4] = kNone;
        rec[5] = nR + 1;
        rec[6] = (uint32_t)sr;
        rec[7] = (uint32_t)(sr >> 32);
      }
      __syncwarp();
      Tc.map = Lr;
      Tc.W = W;
      Tc.W4 = W4;
      Tc.E = E;
      Tc.root = r;
      Tc.rlist = M.rbuf;
      Tc.cols = want_cols ? cols : nullptr;
      Tc.gx = want_aux && small ? gx : nullptr;
      Tc.ncw = ncw;
      Tc.auxref = 0;
      PH_STOP(A, 12);
      if (want_aux && heavy(P, l, nC)) {
        // the root will be split: share its Γ index with the subtasks through the task pool
        const uint32_t co = pool_alloc(P, r4((uint32_t)aux_words));
        if (co != kNone) {
          uint32_t* cp = pool_ptr(P, co);
          for (uint64_t j = lane; j < aux_words; j += 32) cp[j] = aux[j];
          __syncwarp();
          if (small) Tc.gx = cp;
          else Tc.cols = cp;
          Tc.auxref = co + 1;
        }
      }
      PH_STOP(A, 3);
      *top = rec;
      *lo = align4(rec + rec_need);
    }
  }
  // leave the table clean for the next root (the task no longer needs it)
  __syncwarp();
  for (uint32_t j0 = lane; j0 < (sorted ? 0u : nocc); j0 += 32 * GMBE_CLS_UNROLL) {  // (sort mode: scratch)
    uint32_t sq[GMBE_CLS_UNROLL];
#pragma unroll
    for (int q = 0; q < GMBE_CLS_UNROLL; q++) sq[q] = j0 + 32 * q < nocc ? occl[j0 + 32 * q] : kNone;
#pragma unroll
    for (int q = 0; q < GMBE_CLS_UNROLL; q++)
      if (sq[q] != kNone) {
        if (!dense) keys[sq[q]] = GMBE_EMPTY;
        vals[sq[q]] = 0;
      }
  }
  __syncwarp();
  return *top != nullptr;
}

__device__ __forceinline__ unsigned long long globaltimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ uint32_t smid() {
  uint32_t v;
  asm("mov.u32 %0, %%smid;" : "=r"(v));
  return v;
}
// profiling timeline: one record per root / task (kind 0 / 1)
// info = nodes generated by the record << 32 | min(|L_top|, 65535) << 16 | min(|C_top|, 65535)
__device__ void timeline_rec(const Params& P, uint32_t kind, uint32_t root, unsigned long long t0,
                             unsigned long long info) {
  if (lane_id() != 0) return;
  const unsigned long long t1 = globaltimer();
  const unsigned long long i = atomicAdd(P.timeline, 1ull);
  if (1 + 4 * (i + 1) > P.timeline_cap) return;
  unsigned long long* r = P.timeline + 1 + 4 * i;
  r[0] = ((unsigned long long)smid() << 56) | ((unsigned long long)kind << 48) | root;
  r[1] = t0;
  r[2] = t1;
  r[3] = info;
}
__device__ __forceinline__ unsigned long long tl_info(unsigned long long nodes, uint32_t l, uint32_t c) {
  return (nodes << 32) | ((unsigned long long)min(l, 65535u) << 16) | min(c, 65535u);
}

#ifndef GMBE_MIN_BLOCKS
#define GMBE_MIN_BLOCKS 3  // 80 registers: 24 resident warps per SM (measured best on gh_work)
#endif
#ifndef GMBE_WPB
#define GMBE_WPB 8  // warps per block
#endif
constexpr uint32_t kWpb = GMBE_WPB;
// The warp's memory: its arena slice (clean hash table, rank bitmap, occupied list, dynamic region)
// and its shared-memory slices -- recomputed where needed instead of held across the persistent loop
// (long-lived pointers were the loop's main register spills).
__device__ __forceinline__ WarpMem warp_mem(const Params& P, uint32_t gw, unsigned long long* sm_sort,
                                           uint32_t* skeys, unsigned long long* svals, uint32_t* socc) {
  WarpMem M;
  uint32_t* base = P.arena + (uint64_t)gw * P.arena_words;
  M.keys = base;
  M.vals = (unsigned long long*)(base + P.tmax);
  M.bits = base + 3ull * P.tmax;
  M.occ = M.bits + P.bmax;
  M.dyn = align4(M.occ + P.omax);
  M.dyn_end = base + P.arena_words;
  M.rbuf = P.rbuf ? P.rbuf + (uint64_t)gw * P.rbuf_words : nullptr;
  M.sm_sort = sm_sort;
  M.skeys = skeys;
  M.svals = svals;
  M.socc = socc;
  return M;
}

__global__ void __launch_bounds__(32 * GMBE_WPB, GMBE_MIN_BLOCKS) k_enum(const Params P) {
  __shared__ unsigned long long s_sort[kWpb][kSmemSort];
  __shared__ unsigned long long s_tvals[kWpb][kSmemTable ? kSmemTable : 1];
  __shared__ uint32_t s_tkeys[kWpb][kSmemTable ? kSmemTable : 1];
  __shared__ uint32_t s_tocc[kWpb][kSmemTable ? kSmemTable / 2 : 1];
  __shared__ ThrSmem s_thr[kWpb];
  const uint32_t lane = lane_id();
#define GMBE_WARP_MEM()                                                                                      \
  warp_mem(P, (blockIdx.x * blockDim.x + threadIdx.x) >> 5, s_sort[threadIdx.x >> 5], s_tkeys[threadIdx.x >> 5], \
           s_tvals[threadIdx.x >> 5], s_tocc[threadIdx.x >> 5])
  for (uint32_t j = lane; j < kSmemTable; j += 32) {
    s_tkeys[threadIdx.x >> 5][j] = GMBE_EMPTY;
    s_tvals[threadIdx.x >> 5][j] = 0;
  }
  __syncwarp();
  Acc A;
  A.v = 0;
#ifdef GMBE_PROFILE
  for (int k = 0; k < 16; k++) A.ph[k] = 0;
  A.t0 = 0;
#endif
  bool roots_done = false, is_hungry = false;
  uint32_t idle = 0;
  uint32_t ck_pos = 0, ck_end = 0;  // this warp's claimed run of issue positions [ck_pos, ck_end)
  while (true) {
    // work item: a queued split subtask first (Alg 4 L3-4), else the next root (Alg 4 L6, heaviest =
    // highest rank first); both end in the single dispatch site below
    uint32_t task = kNone;
    if (lane == 0) task = queue_pop(P);  // split subtasks first (Alg 4 L3), also inside a root chunk
    task = __shfl_sync(GMBE_FULL, task, 0);
    if (task == kNone && roots_done) {
      // 3. idle: all roots issued -- wait for a task or for termination (nothing queued or running)
      unsigned long long pend = 0;
      if (lane == 0) pend = ld_volatile(&P.ctrl->pending.v);
      pend = __shfl_sync(GMBE_FULL, pend, 0);
      if (pend == 0) break;
      if (!is_hungry && P.donate) {  // ask the working warps to donate (see donate_reg)
        if (lane == 0) atomicAdd(&P.ctrl->hungry.v, 1ull);
        is_hungry = true;
      }
      __nanosleep(idle < 4 ? 500 : (idle < 16 ? 2000 : 8000));  // exponential-ish backoff
      idle++;
      continue;
    }
    WarpMem M = GMBE_WARP_MEM();
    TaskCtx Tc;
    uint32_t* top = nullptr;
    uint32_t* lo = M.dyn;
    uint32_t lmap = 0, kind = 2, item = 0, tl_l = 0, tl_c = 0;
    const long long c0 = P.per_root_cycles ? clock64() : 0;
    const unsigned long long g0 = P.timeline ? globaltimer() : 0, n0 = P.timeline ? A.get(kAcNodes) : 0ull;
    bool release = true;  // this item ends a unit of `pending` (a task, or a chunk's last root)
    if (task != kNone) {
      if (is_hungry) {
        if (lane == 0) atomicAdd(&P.ctrl->hungry.v, ~0ull);
        is_hungry = false;
      }
      PH_START(A);
      __threadfence();  // acquire: the task was written on another SM
      uint32_t* s = pool_ptr(P, task);
      Tc.W = s[0];
      lmap = s[1];
      Tc.root = s[2];
      const uint32_t rlen = s[3];
      Tc.W4 = r4(Tc.W);
      Tc.E = r4(Tc.W + 2);
      Tc.map = s + kHdr;
      Tc.rlist = M.rbuf;
      Tc.auxref = s[5];
      Tc.ncw = s[6];
      Tc.cols = s[7] == 1 ? pool_ptr(P, Tc.auxref - 1) : nullptr;
      Tc.gx = s[7] == 2 ? pool_ptr(P, Tc.auxref - 1) : nullptr;
      if (M.rbuf)
        for (uint32_t j = lane; j < rlen; j += 32) M.rbuf[j] = s[kHdr + r4(lmap) + j];
      __syncwarp();
      PH_STOP(A, 15);
      top = s + s[4];
      kind = 1;
      item = Tc.root;
      tl_l = top[2];
      tl_c = top[0];
    } else {
      if (ck_pos == ck_end) {
        // claim a run of consecutive issue positions with ONE atomic: single roots in the heavy head
        // of the issue list, P.chunk roots once this warp has seen positions past P.chunk_from (the
        // estimate may be stale; any run length gives disjoint ranges)
        const uint32_t K = ck_end >= P.chunk_from ? P.chunk : 1u;
        unsigned long long t = 0;
        if (lane == 0) {
          atomicAdd(&P.ctrl->pending.v, 1ull);
          // N1: a cursor shared by every GPU takes a system-scope atomic over NVLink
          t = P.shared_cursor ? atomicAdd_system(P.shared_cursor, (unsigned long long)K)
                              : atomicAdd(&P.ctrl->root_cursor.v, (unsigned long long)K);
        }
        t = __shfl_sync(GMBE_FULL, t, 0);
        if (t < P.n_roots) {
          ck_pos = (uint32_t)t;
          ck_end = (uint32_t)min(t + K, (unsigned long long)P.n_roots);
        } else {
          if (lane == 0) atomicAdd(&P.ctrl->pending.v, ~0ull);
          roots_done = true;
          continue;
        }
      }
      const uint32_t rk = P.issue[ck_pos];
      const uint32_t rlb = P.g.off_v[rk], rl = P.g.off_v[rk + 1] - rlb;
      ck_pos++;
      release = ck_pos == ck_end;
      kind = 0;
      item = rk;
      if (run_root(P, rk, rlb, rl, M, A, Tc, &top, &lo)) lmap = top[2];
      if (P.debug & 1024) top = nullptr;  // experiments: root construction only (no subtrees)
      tl_l = rl;
    }
    if (top) dispatch_task(P, Tc, top, lo, M.dyn_end, lmap, A, M.sm_sort, &s_thr[threadIdx.x >> 5]);
    if (P.timeline) timeline_rec(P, kind, item, g0, tl_info(A.get(kAcNodes) - n0, tl_l, tl_c));
    if (P.per_root_cycles && lane == 0)
      atomicAdd(P.per_root_cycles + item, (unsigned long long)(clock64() - c0));
    __syncwarp();
    if (lane == 0 && release) atomicAdd(&P.ctrl->pending.v, ~0ull);
    idle = 0;
  }
#undef GMBE_WARP_MEM
  if (lane < kAcN) atomicAdd(&P.ctrl->count + lane, A.v);  // Ctrl's counters, in kAc* order
#ifdef GMBE_PROFILE
  if (lane == 0 && P.profile)
    for (int k = 0; k < 16; k++) atomicAdd(&P.ctrl->phase[k], A.ph[k]);
#endif
}

#include "gmbe_block.cuh"  // GMBE-BLOCK (block-centric ablation variant)

// ---------------------------------------------------------------- host side
struct Workspace {
  int device = -1;
  void* arena = nullptr;
  size_t arena_bytes = 0;
  uint64_t layout[5] = {0, 0, 0, 0, 0};  // tmax, omax, arena_words, nwarps, bmax of the clean tables
  bool clean = false;
  uint64_t tmax = 0, omax = 0, bmax = 0, dyn = 0, nwarps = 0, pool_auto = 0;  // cached sizing
  bool dyn_capped = false;
  bool dyn_failed = false;  // an arena allocation of the free-memory-derived size failed (halved)
  bool regrow = false;      // the last call ran out of a capped arena: re-check free memory once
  int sms = 0, bps_max = 0, bps_max_blk = 0;
  void* pool = nullptr;
  size_t pool_bytes = 0;
  void* rings = nullptr;
  size_t ring_bytes = 0;
  void* rbuf = nullptr;
  size_t rbuf_bytes = 0;
  void* ctrl = nullptr;
  size_t ctrl_bytes = 0;
  void* per_root = nullptr;
  size_t per_root_bytes = 0;
  void* per_root_cyc = nullptr;
  size_t per_root_cyc_bytes = 0;
  void* shard = nullptr;  // this call's root issue list (part_count > 1) + selection scratch
  size_t shard_bytes = 0;
  uint32_t* sring_h = nullptr;  // streaming output ring (mapped pinned host memory) + its tail word
  uint32_t* sring_d = nullptr;
  uint64_t sring_words = 0;
  bool sring_dirty = false;
};

// roots of one shard (rank % part_count == part_index), kept in the graph's issue order
struct ShardOf {
  uint32_t pc, pi;
  __host__ __device__ __forceinline__ bool operator()(const uint32_t& r) const { return r % pc == pi; }
};

// N4 cost-model parts: position p = b·pc + j of the issue list (heaviest wedge count first) goes to
// part j in even blocks b and to part pc-1-j in odd ones (snake deal = parallel greedy LPT)
__global__ void k_snake_part(const uint32_t* __restrict__ issue, uint32_t n, uint32_t pc, uint32_t pi,
                             uint32_t* __restrict__ out) {
  const uint32_t nb = (n + pc - 1) / pc;
  for (uint32_t b = blockIdx.x * blockDim.x + threadIdx.x; b < nb; b += gridDim.x * blockDim.x) {
    const uint64_t p = (uint64_t)b * pc + ((b & 1) ? pc - 1 - pi : pi);
    if (p < n) out[b] = issue[p];
  }
}

static uint32_t snake_count(uint32_t n, uint32_t pc, uint32_t pi) {
  const uint32_t full = n / pc, rem = n % pc;  // blocks 0..full-1 are complete
  if (!rem) return full;
  const uint32_t j = (full & 1) ? pc - 1 - pi : pi;  // the partial block b = full
  return full + (j < rem ? 1 : 0);
}

cudaError_t ensure(void** p, size_t* have, size_t need) {
  if (*have >= need && *p) return cudaSuccess;
  if (*p) cudaFree(*p);
  *p = nullptr;
  *have = 0;
  const cudaError_t e = cudaMalloc(p, need ? need : 16);
  if (e == cudaSuccess) *have = need;
  return e;
}

// Workspace pool: a call takes an idle workspace of its device (or a new one) and returns it, so
// repeated calls reuse device memory (and its clean tables) and concurrent calls never share one.
std::mutex g_ws_mu;
std::vector<Workspace*> g_ws_idle;
Workspace* ws_acquire(int device) {
  std::lock_guard<std::mutex> lk(g_ws_mu);
  for (size_t i = 0; i < g_ws_idle.size(); i++)
    if (g_ws_idle[i]->device == device) {
      Workspace* w = g_ws_idle[i];
      g_ws_idle.erase(g_ws_idle.begin() + i);
      return w;
    }
  Workspace* w = new Workspace();
  w->device = device;
  return w;
}
void ws_return(Workspace* w) {
  std::lock_guard<std::mutex> lk(g_ws_mu);
  g_ws_idle.push_back(w);
}

}  // namespace

extern "C" uint64_t gmbe_node_buf_bound_bytes(uint64_t dv, uint64_t d2v) { return (3 * dv + 2 * d2v) * 4; }
extern "C" uint64_t gmbe_naive_alloc_bytes(uint64_t dv, uint64_t d2v) { return dv * (dv + d2v) * 4; }

extern "C" void gmbe_release_workspace(const gmbe_graph* G) {
  if (!G) return;
  std::lock_guard<std::mutex> lk(g_ws_mu);
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(G->device);
  for (size_t i = 0; i < g_ws_idle.size();) {
    Workspace* w = g_ws_idle[i];
    if (w->device != G->device) {
      i++;
      continue;
    }
    for (void* p : {w->arena, w->pool, w->rings, w->rbuf, w->ctrl, w->per_root, w->per_root_cyc, w->shard})
      if (p) cudaFree(p);
    if (w->sring_h) cudaFreeHost(w->sring_h);
    delete w;
    g_ws_idle.erase(g_ws_idle.begin() + i);
  }
  cudaSetDevice(prev);
}

static int enumerate_impl(const gmbe_graph* G, const gmbe_opts* opts, gmbe_sink_fn sink, void* user,
                          uint64_t ring_words, gmbe_result* out);

extern "C" int gmbe_enumerate(const gmbe_graph* G, const gmbe_opts* opts, gmbe_result* out) {
  return enumerate_impl(G, opts, nullptr, nullptr, 0, out);
}

extern "C" int gmbe_enumerate_stream(const gmbe_graph* G, const gmbe_opts* opts, gmbe_sink_fn sink, void* user,
                                     uint64_t ring_words, gmbe_result* out) {
  if (!sink) return gmbe_set_error(GMBE_EINVAL, "gmbe_enumerate_stream: NULL sink");
  return enumerate_impl(G, opts, sink, user, ring_words, out);
}

static int enumerate_once(const gmbe_graph* G, const gmbe_opts& o, gmbe_sink_fn sink, void* user,
                          uint64_t ring_words, gmbe_result* out, bool* arena_overflow);

// Degrade path for a per-warp workspace overflow (a root record or a DFS level that does not fit the
// warp's dynamic region): the call is re-run from scratch with larger per-warp regions -- a caller-given
// arena_words is replaced by the automatic size (the full bound, capped by free memory), an automatic
// size is spread over fewer resident warps (24 -> 16 -> 8 per SM, the free-memory cap being shared by
// fewer warps).  The kernel writes nothing the
// caller sees until it completes (counters, bounded records), so the re-run is exact; a streaming call
// (records already delivered) is not re-run.
static int enumerate_impl(const gmbe_graph* G, const gmbe_opts* opts, gmbe_sink_fn sink, void* user,
                          uint64_t ring_words, gmbe_result* out) {
  if (!G || !out) return gmbe_set_error(GMBE_EINVAL, "gmbe_enumerate: NULL argument");
  gmbe_opts o{};
  if (opts && opts->struct_size) {
    if (opts->struct_size > sizeof(gmbe_opts)) return gmbe_set_error(GMBE_EINVAL, "gmbe_enumerate: bad struct_size");
    std::memcpy(&o, opts, opts->struct_size);
  }
  for (uint32_t attempt = 0;; attempt++) {
    bool ovf = false;
    const int rc = enumerate_once(G, o, sink, user, ring_words, out, &ovf);
    if (rc == GMBE_OK) out->retries = attempt;
    if (rc == GMBE_OK || !ovf || sink || attempt >= 6) return rc;
    if (o.arena_words) {
      o.arena_words = 0;  // the automatic size: the full bound, capped by free memory
    } else {
      const uint32_t wps = o.warps_per_sm ? std::min<uint32_t>(o.warps_per_sm, 24u) : 24u;
      if (wps <= kWpb) return rc;
      o.warps_per_sm = wps > 16 ? 16 : kWpb;
    }
  }
}

static int enumerate_once(const gmbe_graph* G, const gmbe_opts& o, gmbe_sink_fn sink, void* user,
                          uint64_t ring_words, gmbe_result* out, bool* arena_overflow) {
  const uint32_t parts = o.part_count ? o.part_count : 1;
  if (o.part_index >= parts) return gmbe_set_error(GMBE_EINVAL, "gmbe_enumerate: part_index >= part_count");
  if (o.part_mode > GMBE_PART_COST) return gmbe_set_error(GMBE_EINVAL, "gmbe_enumerate: bad part_mode");
  if (o.scheduler > GMBE_SCHED_BLOCK) return gmbe_set_error(GMBE_EINVAL, "gmbe_enumerate: bad scheduler");
  if (o.root_cursor && parts > 1)
    return gmbe_set_error(GMBE_EINVAL, "gmbe_enumerate: root_cursor needs part_count <= 1");
  if ((o.out_offsets == nullptr) != (o.out_ids == nullptr))
    return gmbe_set_error(GMBE_EINVAL, "gmbe_enumerate: out_offsets and out_ids must be given together");
  if (sink && o.out_ids)
    return gmbe_set_error(GMBE_EINVAL, "gmbe_enumerate_stream: no bounded output buffers with a sink");
  GMBE_CUDA_TRY(cudaSetDevice(G->device));
  cudaStream_t s = o.cuda_stream ? (cudaStream_t)o.cuda_stream : G->stream;
  const DevGraph& g = G->g;
  std::memset(out, 0, sizeof(*out));
  Workspace* Wp = ws_acquire(G->device);
  struct Ret {
    Workspace* w;
    ~Ret() { ws_return(w); }
  } ret{Wp};
  Workspace& W = *Wp;

  if (W.sms == 0) {  // per-device constants, queried once per workspace
    GMBE_CUDA_TRY(cudaDeviceGetAttribute(&W.sms, cudaDevAttrMultiProcessorCount, G->device));
    GMBE_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&W.bps_max, k_enum, 32 * kWpb, 0));
    GMBE_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&W.bps_max_blk, k_enum_block, kBlkThreads, 0));
  }
  const bool block_mode = o.scheduler == GMBE_SCHED_BLOCK;
  uint32_t wps = o.warps_per_sm ? o.warps_per_sm : 64;
  if (wps < kWpb) wps = kWpb;
  if (wps > 64) wps = 64;
  uint32_t bps = wps / kWpb;
  if ((int)bps > (block_mode ? W.bps_max_blk : W.bps_max)) bps = block_mode ? W.bps_max_blk : W.bps_max;
  if (bps < 1) bps = 1;
  const uint32_t blocks = (uint32_t)W.sms * bps;
  const uint64_t nwarps = (uint64_t)blocks * kWpb;

  // per-warp arena: clean hash table sized for the largest root's wedges, its occupied list, and
  // the dynamic region (root record, node stack, Γ index), bounded by free memory.  A cached layout
  // that already satisfies this graph is reused as is (its tables are clean; no re-initialisation).
  const uint64_t wb = (uint64_t)g.wedge_bound + 64;
  uint64_t tmax = 64;
  while (tmax < 2 * wb) tmax <<= 1;
  const uint64_t bmax = ((uint64_t)(g.n_v + 31) / 32 + 3) & ~3ull;  // rank bitmap of dense-mode roots
  uint64_t omax = (wb + 3) & ~3ull;
  const uint64_t cols_bound = std::min<uint64_t>((uint64_t)g.delta_v * (wb / 32 + 1), 1u << 21);
  const uint64_t dyn_want = o.arena_words ? o.arena_words
                                          : (uint64_t)g.rec_bound * 4 + 4 * wb + 2 * cols_bound + (1u << 18);
  uint64_t arena_words;
  bool reuse = W.arena && W.nwarps == nwarps && W.tmax >= tmax && W.omax >= omax && W.bmax >= bmax &&
               (W.dyn >= dyn_want || (!o.arena_words && W.dyn_capped));
  if (reuse && W.dyn < dyn_want && W.regrow && !W.dyn_failed) {
    // a layout capped by free memory at an earlier call: re-size if there is more room now
    size_t fr = 0, tot = 0;
    GMBE_CUDA_TRY(cudaMemGetInfo(&fr, &tot));
    fr += W.arena_bytes;
    const uint64_t fixed = 3 * W.tmax + W.bmax + W.omax + 8;
    const uint64_t cap_total = (uint64_t)(fr * 0.5) / 4 / nwarps;
    const uint64_t cap_now = cap_total > fixed ? cap_total - fixed : 0;
    if (cap_now > W.dyn + W.dyn / 2) reuse = false;  // (hysteresis: re-size only for a real gain)
  }
  W.regrow = false;
  uint64_t bmax_use = bmax;
  if (reuse) {
    tmax = W.tmax;
    omax = W.omax;
    bmax_use = W.bmax;
    arena_words = W.layout[2];
  } else {
    const uint64_t fixed = 3 * tmax + bmax + omax + 8;
    uint64_t dyn = dyn_want;
    bool capped = false;
    if (!o.arena_words) {
      size_t fr = 0, tot = 0;
      GMBE_CUDA_TRY(cudaMemGetInfo(&fr, &tot));
      fr += W.arena_bytes;  // this workspace's arena is about to be replaced
      const uint64_t cap_total = (uint64_t)(fr * 0.5) / 4 / nwarps;
      const uint64_t cap = cap_total > fixed + (1u << 16) ? cap_total - fixed : (1u << 16);
      if (dyn > cap) {
        dyn = cap;
        capped = true;
      }
    }
    arena_words = (fixed + dyn + 3) & ~3ull;
    W.tmax = tmax;
    W.omax = omax;
    W.bmax = bmax;
    W.dyn = dyn;
    W.dyn_capped = capped;
    W.nwarps = nwarps;
  }
  uint64_t pool_words = o.pool_words;
  if (!pool_words) {  // task pool: subtasks + shared Γ indexes, never reused within a call
    if (!W.pool_auto) {
      size_t fr = 0, tot = 0;
      GMBE_CUDA_TRY(cudaMemGetInfo(&fr, &tot));
      W.pool_auto = std::min<uint64_t>(1ull << 30, (uint64_t)(fr * 0.2) / 4);
    }
    pool_words = W.pool_auto;
  }
  pool_words = (pool_words + 3) & ~3ull;
  uint32_t cap = 1;
  const uint64_t want_cap = o.queue_cap ? o.queue_cap : (1u << 20);
  while (cap < want_cap && cap < (1u << 30)) cap <<= 1;
  if (cap < 16384) cap = 16384;  // > the producers' admission margin
  const bool want_out = o.out_ids != nullptr || sink != nullptr;
  const uint32_t rbuf_words = want_out ? (uint32_t)(wb + 64) : 0;

  {
    cudaError_t ae = ensure(&W.arena, &W.arena_bytes, nwarps * arena_words * 4);
    // another process on this GPU may have taken memory since cudaMemGetInfo: halve the
    // (free-memory-capped) dynamic region and retry, down to its floor
    while (ae == cudaErrorMemoryAllocation && !o.arena_words && W.dyn > (1u << 16)) {
      (void)cudaGetLastError();
      W.dyn = std::max<uint64_t>(W.dyn / 2, 1u << 16);
      W.dyn_capped = true;
      W.dyn_failed = true;  // do not try to grow again on later calls (gmbe_release_workspace resets)
      arena_words = (3 * tmax + bmax_use + omax + 8 + W.dyn + 3) & ~3ull;
      ae = ensure(&W.arena, &W.arena_bytes, nwarps * arena_words * 4);
    }
    GMBE_CUDA_TRY(ae);
  }
  {
    const uint64_t sig[5] = {tmax, omax, arena_words, nwarps, bmax_use};
    if (!W.clean || std::memcmp(sig, W.layout, sizeof(sig)) != 0) {
      // keys := EMPTY, vals := 0 -- once; every root leaves its slots clean again
      GMBE_CUDA_TRY(cudaMemset2DAsync(W.arena, arena_words * 4, 0xff, tmax * 4, nwarps, s));
      GMBE_CUDA_TRY(cudaMemset2DAsync((uint32_t*)W.arena + tmax, arena_words * 4, 0, (2 * tmax + bmax_use) * 4,
                                      nwarps, s));
      std::memcpy(W.layout, sig, sizeof(sig));
      W.clean = true;
    }
  }
  GMBE_CUDA_TRY(ensure(&W.pool, &W.pool_bytes, pool_words * 4));
  GMBE_CUDA_TRY(ensure(&W.rings, &W.ring_bytes, (size_t)cap * 4));
  if (want_out) GMBE_CUDA_TRY(ensure(&W.rbuf, &W.rbuf_bytes, nwarps * rbuf_words * 4));
  GMBE_CUDA_TRY(ensure(&W.ctrl, &W.ctrl_bytes, sizeof(Ctrl)));
  if (o.per_root_count) GMBE_CUDA_TRY(ensure(&W.per_root, &W.per_root_bytes, (size_t)(g.n_v + 1) * 8));
  if (o.per_root_cycles) GMBE_CUDA_TRY(ensure(&W.per_root_cyc, &W.per_root_cyc_bytes, (size_t)(g.n_v + 1) * 8));

  Params P{};
  P.g = g;
  P.part_index = o.part_index;
  P.part_count = parts;
  P.n_roots = g.n_v > o.part_index ? (g.n_v - o.part_index + parts - 1) / parts : 0;
  P.issue = g.issue;
  if (parts > 1 && o.part_mode == GMBE_PART_COST) {
    P.n_roots = snake_count(g.n_v, parts, o.part_index);
    if (P.n_roots) {
      GMBE_CUDA_TRY(ensure(&W.shard, &W.shard_bytes, (size_t)P.n_roots * 4));
      k_snake_part<<<(P.n_roots + 255) / 256, 256, 0, s>>>(g.issue, g.n_v, parts, o.part_index, (uint32_t*)W.shard);
      gmbe_note_launch();
      P.issue = (const uint32_t*)W.shard;
    }
  } else if (parts > 1 && P.n_roots) {
    size_t tb = 0;
    GMBE_CUDA_TRY(cub::DeviceSelect::If(nullptr, tb, g.issue, (uint32_t*)nullptr, (int*)nullptr, (int)g.n_v,
                                        ShardOf{parts, o.part_index}, s));
    const size_t list_b = ((size_t)g.n_v * 4 + 255) & ~(size_t)255;
    GMBE_CUDA_TRY(ensure(&W.shard, &W.shard_bytes, list_b + 256 + tb));
    char* sb = (char*)W.shard;
    GMBE_CUDA_TRY(cub::DeviceSelect::If(sb + list_b + 256, tb, g.issue, (uint32_t*)sb, (int*)(sb + list_b),
                                        (int)g.n_v, ShardOf{parts, o.part_index}, s));
    P.issue = (const uint32_t*)sb;
  }
  P.prune = o.no_prune ? 0 : 1;
  P.split = o.no_split || o.scheduler != GMBE_SCHED_TASK ? 0 : 1;  // WARP / BLOCK: Alg 3 tasks, no split
  P.bound_height = o.bound_height ? o.bound_height : 10;   // paper: 20; retuned for B200
  P.bound_size = o.bound_size ? o.bound_size : 500;     // paper: 1500; scripts/sweep.py
  P.hu_side = g.swapped ? 1 : 0;
  P.arena = (uint32_t*)W.arena;
  P.arena_words = arena_words;
#ifndef GMBE_COL_BUDGET_PCT
#define GMBE_COL_BUDGET_PCT 50  // a root's Γ index may take this % of the warp's dynamic region
#endif
  P.col_budget = W.dyn * GMBE_COL_BUDGET_PCT / 100;
  P.tmax = (uint32_t)tmax;
  P.omax = (uint32_t)omax;
  P.bmax = (uint32_t)bmax_use;
  P.rbuf = want_out ? (uint32_t*)W.rbuf : nullptr;
  P.rbuf_words = rbuf_words;
  P.pool = (uint32_t*)W.pool;
  P.pool_words = pool_words;
  P.tq = (uint32_t*)W.rings;
  P.qmask = cap - 1;
  P.qcap = cap;
  P.ctrl = (Ctrl*)W.ctrl;
  P.out_offsets = (unsigned long long*)o.out_offsets;
  P.out_offsets_cap = want_out ? o.out_offsets_cap : 0;
  P.out_ids = o.out_ids;
  P.out_ids_cap = o.out_ids ? o.out_ids_cap : 0;
  if (sink) {
    // ring of 2^k words >= max(ring_words, 4 * the largest record), mapped pinned host memory
    uint64_t need = std::max<uint64_t>(ring_words ? ring_words : (1ull << 24),
                                       4ull * (3ull + g.delta_u + g.delta_v) + 4096);
    uint64_t words = 1;
    while (words < need) words <<= 1;
    if (W.sring_words != words || W.sring_dirty) {
      if (W.sring_h) cudaFreeHost(W.sring_h);
      W.sring_h = nullptr;
      W.sring_words = 0;
      GMBE_CUDA_TRY(cudaHostAlloc((void**)&W.sring_h, (words + 32) * 4, cudaHostAllocMapped));
      std::memset(W.sring_h, 0, (words + 32) * 4);
      GMBE_CUDA_TRY(cudaHostGetDevicePointer((void**)&W.sring_d, W.sring_h, 0));
      W.sring_words = words;
      W.sring_dirty = false;
    }
    // consumer words after the ring: tail, abort (rec_open's back-pressure wait)
    for (int k = 0; k < 2; k++) *(volatile unsigned long long*)(W.sring_h + words + 16 + 2 * k) = 0;
    P.sring = W.sring_d;
    P.smask = words - 1;
    P.stail = (const unsigned long long*)(W.sring_d + words + 16);
  }
  P.per_root = o.per_root_count ? (unsigned long long*)W.per_root : nullptr;
  P.per_root_cycles = o.per_root_cycles ? (unsigned long long*)W.per_root_cyc : nullptr;
  P.profile = o.phase_cycles ? 1 : 0;
  P.debug = o.reserved0;
  P.donate = (o.reserved0 & 4) || o.scheduler != GMBE_SCHED_TASK ? 0 : 1;
  if (o.scheduler == GMBE_SCHED_WARP) P.debug |= 16;  // one warp per node: no thread-level tier
  P.thr_min_est = o.thr_min ? o.thr_min : GMBE_THR_MIN_EST;
  // root claims: after the heavy head of the issue list (the first 1/8 of the positions, one root
  // per atomic), a warp claims root_chunk consecutive positions per atomic (default 1, <= 32)
  P.chunk = o.root_chunk ? std::min<uint32_t>(o.root_chunk, 32u) : GMBE_ROOT_CHUNK;
  P.chunk_from = P.n_roots / 8;
  // Sort-mode roots trade per-root latency (two radix passes and a grouping sweep instead of one table
  // pass) for L2-resident traffic: they pay when the root builds of every resident warp contend for
  // DRAM (a full graph on one GPU: gh_work 14.8 -> 14.45 ms), not when a shard leaves the GPU
  // latency-bound (1/8 cost parts of gh_work: mean part 2.91 -> 3.31 ms).  On only while the call
  // has many roots per resident warp (and not under the N1 shared cursor, whose issue list is the
  // whole graph's while this GPU takes only its share of it).
  const bool saturated = !o.root_cursor && (uint64_t)P.n_roots >= 8ull * nwarps;
  P.sort_min = saturated ? GMBE_SORT_MIN : kNone;
  // Split threshold (B2): a saturated call splits a little less (bound_size 550: gh_work 14.1 -> 13.9 ms
  // at N=1), a shard more (550 made 1/8 cost parts of gh_work 2.85 -> 2.98 ms mean): same rule as above
  if (!o.bound_size) P.bound_size = saturated ? 550 : 500;
  P.split_wide = o.split_wide ? o.split_wide : GMBE_SPLIT_WIDE;
  P.timeline = (unsigned long long*)o.timeline;
  P.timeline_cap = o.timeline_cap;
  P.shared_cursor = (unsigned long long*)o.root_cursor;
  if (P.timeline) GMBE_CUDA_TRY(cudaMemsetAsync(P.timeline, 0, 8, s));

  Ctrl hc{};
  GMBE_CUDA_TRY(cudaMemcpyAsync(W.ctrl, &hc, sizeof(Ctrl), cudaMemcpyHostToDevice, s));
  GMBE_CUDA_TRY(cudaMemsetAsync(W.rings, 0, (size_t)cap * 4, s));
  if (P.per_root) GMBE_CUDA_TRY(cudaMemsetAsync(W.per_root, 0, (size_t)(g.n_v + 1) * 8, s));
  if (P.per_root_cycles) GMBE_CUDA_TRY(cudaMemsetAsync(W.per_root_cyc, 0, (size_t)(g.n_v + 1) * 8, s));
  GMBE_CUDA_TRY(cudaGetLastError());
  cudaEvent_t e0, e1;
  GMBE_CUDA_TRY(cudaEventCreate(&e0));
  GMBE_CUDA_TRY(cudaEventCreate(&e1));
  GMBE_CUDA_TRY(cudaEventRecord(e0, s));
  if (P.n_roots > 0) {
    if (block_mode) k_enum_block<<<blocks, kBlkThreads, 0, s>>>(P);
    else k_enum<<<blocks, 32 * kWpb, 0, s>>>(P);
    gmbe_note_launch();
  }
  const cudaError_t le = cudaGetLastError();
  GMBE_CUDA_TRY(cudaEventRecord(e1, s));
  GMBE_CUDA_TRY(le);
  uint64_t streamed = 0;
  int sink_rc = 0;
  if (sink) {
    // consumer (this thread, while the kernel runs): deliver records in ring order, zero their
    // words, then advance the tail the producers wait on
    volatile uint32_t* R = W.sring_h;
    volatile unsigned long long* tail = (volatile unsigned long long*)(W.sring_h + W.sring_words + 16);
    volatile unsigned long long* abort_word = tail + 1;  // raised if this consumer stops draining
    const uint64_t mask = W.sring_words - 1;
    std::vector<uint32_t> batch;
    uint64_t c = 0, nb = 0, final_pos = ~0ull;
    bool done = false, failed = false;
    auto flush = [&]() {
      if (!batch.empty()) {
        if (!sink_rc) sink_rc = sink(batch.data(), batch.size(), nb, user);
        batch.clear();
        nb = 0;
      }
    };
    while (true) {
      const uint32_t h = R[c & mask];
      if (h) {
        std::atomic_thread_fence(std::memory_order_acquire);  // the words were published before h
        uint32_t* base = W.sring_h;
        const uint64_t first = (c + 1) & mask, n = h - 1, n1 = std::min<uint64_t>(n, W.sring_words - first);
        const size_t old = batch.size();
        batch.resize(old + n);
        std::memcpy(batch.data() + old, base + first, n1 * 4);
        std::memset(base + first, 0, n1 * 4);
        if (n1 < n) {
          std::memcpy(batch.data() + old + n1, base, (n - n1) * 4);
          std::memset(base, 0, (n - n1) * 4);
        }
        R[c & mask] = 0;
        c += h;
        nb++;
        streamed++;
        std::atomic_thread_fence(std::memory_order_seq_cst);
        *tail = c;
        if (batch.size() >= (1u << 20)) flush();
        continue;
      }
      flush();
      if (done) {
        if (c >= final_pos || failed) break;
        continue;  // the last records' words are still arriving over the bus
      }
      const cudaError_t q = cudaEventQuery(e1);
      if (q == cudaSuccess) {
        Ctrl hc2{};
        GMBE_CUDA_TRY(cudaMemcpy(&hc2, W.ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost));
        final_pos = hc2.out_ids;
        failed = hc2.error != 0;
        done = true;
      } else if (q != cudaErrorNotReady) {
        *abort_word = 1;  // producers waiting on a full ring stop at once
        GMBE_CUDA_TRY(q);
      }
    }
    if (failed || c != final_pos) W.sring_dirty = true;
  }
  GMBE_CUDA_TRY(cudaMemcpyAsync(&hc, W.ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost, s));
  GMBE_CUDA_TRY(cudaStreamSynchronize(s));
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  if ((o.per_root_count || o.per_root_cycles) && g.n_v) {
    std::vector<unsigned long long> pr(g.n_v);
    std::vector<uint32_t> r2i(g.n_v);
    GMBE_CUDA_TRY(cudaMemcpy(r2i.data(), g.rank2id, g.n_v * 4, cudaMemcpyDeviceToHost));
    if (o.per_root_count) {
      GMBE_CUDA_TRY(cudaMemcpy(pr.data(), W.per_root, g.n_v * 8, cudaMemcpyDeviceToHost));
      for (uint32_t rr = 0; rr < g.n_v; rr++) o.per_root_count[r2i[rr]] = pr[rr];
    }
    if (o.per_root_cycles) {
      GMBE_CUDA_TRY(cudaMemcpy(pr.data(), W.per_root_cyc, g.n_v * 8, cudaMemcpyDeviceToHost));
      for (uint32_t rr = 0; rr < g.n_v; rr++) o.per_root_cycles[r2i[rr]] = pr[rr];
    }
  }
  out->count = hc.count;
  out->checksum = hc.checksum;
  out->n_written = sink ? streamed : (hc.out_rec < P.out_offsets_cap ? hc.out_rec : P.out_offsets_cap);
  out->truncated = hc.truncated;
  out->roots_run = hc.roots_run;
  out->nodes = hc.nodes;
  out->nonmax = hc.nonmax;
  out->algo_bytes_cand = hc.abytes;
  out->splits = hc.splits;
  out->tasks = hc.tasks;
  out->donations = hc.donations;
  out->kernel_ms = ms;
  if (o.phase_cycles)
    for (int k = 0; k < 16; k++) o.phase_cycles[k] = hc.phase[k];
  if (hc.error & kErrStream) {
    W.clean = false;
    return gmbe_set_error(GMBE_EINTERNAL, "gmbe_enumerate_stream: the consumer stopped draining the ring");
  }
  if (hc.error) {
    W.clean = false;
    W.regrow = W.dyn_capped;  // a capped arena was too small: the next call re-checks free memory
    *arena_overflow = true;
    return gmbe_set_error(GMBE_EINTERNAL,
                          "gmbe_enumerate: per-warp workspace exceeded; raise opts.arena_words");
  }
  if (sink_rc) return gmbe_set_error(GMBE_EINVAL, "gmbe_enumerate_stream: the sink returned non-zero");
  return GMBE_OK;
}

// ---- shared root cursors -------------------------------------------------------
static_assert(sizeof(cudaIpcMemHandle_t) <= GMBE_IPC_HANDLE_BYTES, "IPC handle size");

extern "C" int gmbe_shared_cursor_create(int32_t device, uint64_t** dptr, void* ipc_handle) {
  if (!dptr) return gmbe_set_error(GMBE_EINVAL, "gmbe_shared_cursor_create: NULL dptr");
  *dptr = nullptr;
  GMBE_CUDA_TRY(cudaSetDevice(device));
  void* p = nullptr;
  GMBE_CUDA_TRY(cudaMalloc(&p, GMBE_CURSOR_SLOTS * 128));
  cudaError_t e = cudaMemset(p, 0, GMBE_CURSOR_SLOTS * 128);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e == cudaSuccess && ipc_handle) {
    cudaIpcMemHandle_t h;
    e = cudaIpcGetMemHandle(&h, p);
    if (e == cudaSuccess) {
      std::memset(ipc_handle, 0, GMBE_IPC_HANDLE_BYTES);
      std::memcpy(ipc_handle, &h, sizeof(h));
    }
  }
  if (e != cudaSuccess) {
    cudaFree(p);
    return gmbe_set_error(GMBE_ECUDA, std::string("gmbe_shared_cursor_create: ") + cudaGetErrorString(e));
  }
  *dptr = (uint64_t*)p;
  return GMBE_OK;
}

extern "C" int gmbe_shared_cursor_open(const void* ipc_handle, int32_t device, uint64_t** dptr) {
  if (!dptr || !ipc_handle) return gmbe_set_error(GMBE_EINVAL, "gmbe_shared_cursor_open: NULL argument");
  *dptr = nullptr;
  GMBE_CUDA_TRY(cudaSetDevice(device));
  cudaIpcMemHandle_t h;
  std::memcpy(&h, ipc_handle, sizeof(h));
  void* p = nullptr;
  GMBE_CUDA_TRY(cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess));
  *dptr = (uint64_t*)p;
  return GMBE_OK;
}

extern "C" int gmbe_shared_cursor_reset(uint64_t* dptr, uint32_t slot, void* cuda_stream) {
  if (!dptr || slot >= GMBE_CURSOR_SLOTS) return gmbe_set_error(GMBE_EINVAL, "gmbe_shared_cursor_reset: bad argument");
  // synchronous: the zero must have landed before any rank can start the call that uses the slot,
  // whatever stream that call runs on
  GMBE_CUDA_TRY(cudaMemsetAsync(dptr + 16 * slot, 0, 8, (cudaStream_t)cuda_stream));
  GMBE_CUDA_TRY(cudaStreamSynchronize((cudaStream_t)cuda_stream));
  return GMBE_OK;
}

extern "C" void gmbe_shared_cursor_close(uint64_t* dptr, int32_t owner) {
  if (!dptr) return;
  if (owner) cudaFree(dptr);
  else cudaIpcCloseMemHandle(dptr);
}
