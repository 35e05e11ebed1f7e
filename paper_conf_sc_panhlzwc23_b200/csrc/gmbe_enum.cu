// gmbe_enum.cu -- the persistent sm_100a enumeration kernel (DESIGN.md steps a3-a8).
//
// One warp = one "procedure".  Each warp loops (Alg 4):
//   1. dequeue a split subtask from the global task queue, else
//   2. take the next root v_s from an atomic cursor (heavy roots first) and build its root node
//      (Alg 3 / Alg 4 L6-13): wedge scan into a per-warp hash table, classification of
//      N2(v_s) into R (absorbed), C (later-ordered candidates) and Q (earlier-ordered, excluded),
//      root skip unless v_s is the earliest vertex of R (Alg 3 L7), emission of (L_r, R_r);
//   3. either split the task's top node into subtasks (Alg 4 L17-26, heavy-node estimate
//      min(|L|,|C|)·|C| > bound_size and min(|L|,|C|) > bound_height) or walk its
//      subtree depth-first (Alg 2) on a per-warp reusable node stack (Sec 4.1).
//   4. exit when all roots are issued and no task is queued or running.
//
// Node representation: all sets of one task are bitmaps over the task's
// local universe (the root's L_r, compacted to the vertices any candidate touches).  A node
// record holds its L mask and one entry per live candidate / excluded vertex:
//     entry = [row[0..W) = N(x) ∩ L_node as bits, id (rank), k = |N(x) ∩ L_node| | pruned<<31]
// so child generation (Alg 2 L8-13) is AND + POPC over rows, Thm 4.1 compares k' with k, and the
// maximality check (Alg 2 L14) is "some excluded row covers L'".
#include <cstring>
#include <string>
#include <vector>

#include "gmbe_internal.cuh"

namespace {

constexpr uint32_t kHdr = 8;  // node record header words
constexpr uint32_t kNone = 0xffffffffu;
constexpr uint32_t kPruned = 0x80000000u;
constexpr uint32_t kRTag = 0xfffffffeu;   // table value of an R vertex (wedge mode)
constexpr uint32_t kClaim = 0xfffffffdu;  // slotmap placeholder while a slot is claimed
constexpr uint32_t kSmemSort = 256;       // per-warp shared-memory sort capacity (keys)

struct Ctrl {
  unsigned long long root_cursor, q_head, q_tail, f_head, f_tail, pending;
  unsigned long long count, checksum, roots_run, nodes, nonmax, algo_bytes, algo_qfull, splits, tasks;
  unsigned long long out_rec, out_ids;
  unsigned int truncated, error;
};

enum : unsigned int { kErrArena = 1, kErrSlab = 2 };

struct Params {
  DevGraph g;
  uint32_t n_roots;  // roots of this shard
  uint32_t part_index, part_count;
  uint32_t prune, split, bound_height, bound_size, counters;
  uint32_t hu_side;   // checksum side of the library's U vertices (0 = caller U)
  uint32_t wedge_l;    // roots with |L_r| > wedge_l use wedge-mode child generation
  uint32_t* arena;    // per warp: keys[tmax] | slotmap[emax] | vals[tmax] (u64) | occ[omax] | dynamic
  uint64_t arena_words;
  uint32_t tmax, emax, omax;
  uint32_t* rbuf;     // per-warp R-list stack (only with output)
  uint32_t rbuf_words;
  uint32_t* slabs;
  uint64_t slab_words;
  uint32_t n_slabs;
  uint32_t* tq;       // task ring (slab ids)
  uint32_t* fq;       // free-slab ring
  uint32_t ring_mask;
  Ctrl* ctrl;
  unsigned long long* out_offsets;
  uint64_t out_offsets_cap;
  uint32_t* out_ids;
  uint64_t out_ids_cap;
  unsigned long long* per_root;
  unsigned long long* per_root_cycles;
};

struct Acc {
  unsigned long long count, checksum, roots_run, nodes, nonmax, abytes, aqfull, splits, tasks;
};

// per-task constants (warp-uniform)
struct TaskCtx {
  const uint32_t* map;  // local universe bit j -> library U id
  uint32_t W, W4, E;    // words per row, padded Lmask words, entry stride
  uint32_t root;        // rank of the root vertex
  uint32_t* rlist;      // R-list stack (output only)
};

__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ uint32_t lanemask_lt() { return (1u << lane_id()) - 1u; }
__device__ __forceinline__ uint32_t r4(uint32_t x) { return (x + 3u) & ~3u; }

__device__ __forceinline__ uint32_t warp_sum(uint32_t x) {
  return __reduce_add_sync(GMBE_FULL, x);
}
__device__ __forceinline__ unsigned long long warp_sum64(unsigned long long x) {
  for (int o = 16; o; o >>= 1) x += __shfl_xor_sync(GMBE_FULL, x, o);
  return x;
}
template <int LPE>
__device__ __forceinline__ uint32_t group_sum(uint32_t x) {
#pragma unroll
  for (int o = LPE / 2; o; o >>= 1) x += __shfl_xor_sync(GMBE_FULL, x, o);
  return x;
}

__device__ __forceinline__ uint32_t next_pow2(uint32_t x) {
  return x <= 1 ? 1u : 1u << (32 - __clz(x - 1));
}

// ---------------------------------------------------------------- per-warp hash table (a3)
__device__ __forceinline__ uint32_t ht_hash(uint32_t v, uint32_t shift) {
  return (v * 2654435761u) >> shift;
}
__device__ __forceinline__ uint32_t ht_insert(uint32_t* keys, uint32_t shift, uint32_t mask, uint32_t v) {
  uint32_t h = ht_hash(v, shift);
  while (true) {
    uint32_t k = __ldcg(keys + h);
    if (k == v) return h;
    if (k == GMBE_EMPTY) {
      uint32_t old = atomicCAS(keys + h, GMBE_EMPTY, v);
      if (old == GMBE_EMPTY || old == v) return h;
    }
    h = (h + 1) & mask;
  }
}
__device__ __forceinline__ uint32_t ht_find(const uint32_t* keys, uint32_t shift, uint32_t mask, uint32_t v) {
  uint32_t h = ht_hash(v, shift);
  while (true) {
    uint32_t k = __ldcg(keys + h);
    if (k == v) return h;
    if (k == GMBE_EMPTY) return kNone;
    h = (h + 1) & mask;
  }
}

// Visit every wedge (i, v): u_i = L[i], v ∈ N(u_i), load-balanced across the warp.
// f(i, v, active) is called by all 32 lanes each step.
template <class F>
__device__ __forceinline__ void for_each_wedge(const DevGraph& g, const uint32_t* L, uint32_t l, F f) {
  const uint32_t lane = lane_id();
  for (uint32_t b = 0; b < l; b += 32) {
    uint32_t i = b + lane, beg = 0, deg = 0;
    if (i < l) {
      uint32_t u = L[i];
      beg = g.off_u[u];
      deg = g.off_u[u + 1] - beg;
    }
    uint32_t inc = deg;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t t = __shfl_up_sync(GMBE_FULL, inc, o);
      if (lane >= (uint32_t)o) inc += t;
    }
    const uint32_t total = __shfl_sync(GMBE_FULL, inc, 31);
    const uint32_t excl = inc - deg;
    for (uint32_t base = 0; base < total; base += 32) {
      const uint32_t p = base + lane;
      uint32_t lo = 0;
#pragma unroll
      for (int st = 16; st; st >>= 1) {
        uint32_t cand = lo + st;
        uint32_t e = __shfl_sync(GMBE_FULL, excl, cand & 31);
        if (cand < 32 && e <= p) lo = cand;
      }
      uint32_t ob = __shfl_sync(GMBE_FULL, beg, lo);
      uint32_t oe = __shfl_sync(GMBE_FULL, excl, lo);
      bool act = p < total;
      uint32_t v = act ? g.adj_u[ob + p - oe] : 0;
      f(b + lo, v, act);
    }
  }
}

// warp bitonic sort of n 64-bit keys in (global) scratch a[0..next_pow2(n))
__device__ void warp_sort64(unsigned long long* a, uint32_t n) {
  const uint32_t lane = lane_id();
  const uint32_t N = next_pow2(n);
  for (uint32_t i = n + lane; i < N; i += 32) a[i] = ~0ull;
  __syncwarp();
  for (uint32_t k = 2; k <= N; k <<= 1) {
    for (uint32_t j = k >> 1; j > 0; j >>= 1) {
      for (uint32_t t = lane; t < N / 2; t += 32) {
        uint32_t i = ((t & ~(j - 1)) << 1) | (t & (j - 1));
        uint32_t p = i + j;
        unsigned long long x = a[i], y = a[p];
        bool up = (i & k) == 0;
        if ((x > y) == up) {
          a[i] = y;
          a[p] = x;
        }
      }
      __syncwarp();
    }
  }
}

// ---------------------------------------------------------------- MPMC rings (a7)
__device__ __forceinline__ unsigned long long ld_volatile(const unsigned long long* p) {
  return *(volatile const unsigned long long*)p;
}
// called by one lane
__device__ void ring_push(uint32_t* ring, uint32_t mask, unsigned long long* tail, uint32_t x) {
  unsigned long long t = atomicAdd(tail, 1ull);
  uint32_t* slot = ring + (t & mask);
  while (atomicCAS(slot, GMBE_EMPTY, x) != GMBE_EMPTY) __nanosleep(64);
}
// called by one lane; returns kNone if empty
__device__ uint32_t ring_pop(uint32_t* ring, uint32_t mask, unsigned long long* head,
                             unsigned long long* tail) {
  while (true) {
    unsigned long long h = ld_volatile(head);
    unsigned long long t = ld_volatile(tail);
    if (h >= t) return kNone;
    if (atomicCAS(head, h, h + 1) == h) {
      uint32_t* slot = ring + (h & mask);
      uint32_t x;
      while ((x = atomicExch(slot, GMBE_EMPTY)) == GMBE_EMPTY) __nanosleep(32);
      return x;
    }
  }
}

// ---------------------------------------------------------------- emission (a8)
__device__ __forceinline__ unsigned long long hash_u(const Params& P, uint32_t u) {
  return gmbe_hid(u, P.hu_side);
}
// combine sums of the library's L (U side) and R (V side) in the caller's roles
__device__ __forceinline__ unsigned long long pair_hash(const Params& P, unsigned long long sl,
                                                        unsigned long long sr) {
  return P.hu_side ? gmbe_pair_hash(sr, sl) : gmbe_pair_hash(sl, sr);
}

// write one output record: L given by bitmap words lmask (W words over map) or, if lmask == null,
// by the explicit list lids[0..nl); R by ranks rl[0..nr).
__device__ void write_record(const Params& P, const uint32_t* lmask, uint32_t W, const uint32_t* map,
                             const uint32_t* lids, uint32_t nl, const uint32_t* rl, uint32_t nr) {
  const uint32_t lane = lane_id();
  unsigned long long rec = 0, off = 0;
  const unsigned long long need = 2ull + nl + nr;
  if (lane == 0) {
    rec = atomicAdd(&P.ctrl->out_rec, 1ull);
    off = atomicAdd(&P.ctrl->out_ids, need);
  }
  rec = __shfl_sync(GMBE_FULL, rec, 0);
  off = __shfl_sync(GMBE_FULL, off, 0);
  if (rec >= P.out_offsets_cap || off + need > P.out_ids_cap) {
    if (lane == 0) {
      atomicOr(&P.ctrl->truncated, 1u);
      if (rec < P.out_offsets_cap) P.out_offsets[rec] = ~0ull;
    }
    return;
  }
  uint32_t* o = P.out_ids + off;
  // caller U ids first: library L unless swapped
  const bool sw = P.hu_side != 0;
  uint32_t* ou = o + 2;
  uint32_t* lpos = sw ? o + 2 + nr : o + 2;   // where library-L ids go
  uint32_t* rpos = sw ? o + 2 : o + 2 + nl;   // where library-R ids go
  if (lane == 0) {
    o[0] = sw ? nr : nl;
    o[1] = sw ? nl : nr;
  }
  (void)ou;
  for (uint32_t j = lane; j < nr; j += 32) rpos[j] = P.g.rank2id[rl[j]];
  if (lmask) {
    uint32_t c = 0;
    for (uint32_t w = 0; w < W; w++) {
      uint32_t word = lmask[w];
      bool b = (word >> lane) & 1u;
      uint32_t bal = __ballot_sync(GMBE_FULL, b);
      if (b) lpos[c + __popc(bal & lanemask_lt())] = map[w * 32 + lane];
      c += __popc(bal);
    }
  } else {
    for (uint32_t j = lane; j < nl; j += 32) lpos[j] = lids[j];
  }
  __syncwarp();
  if (lane == 0) P.out_offsets[rec] = off;
}

// ---------------------------------------------------------------- child generation (a4, a5)
// Generate the child of node `par` via its candidate i into `ch`.
// Returns 0: non-maximal; 1: maximal leaf (C' empty); 2: maximal with C' != ∅ (ch is a valid
// node record whose header is filled except the parent link).
template <int LPE>
__device__ int gen_child(const Params& P, const TaskCtx& T, uint32_t* par, uint32_t i, uint32_t* ch,
                         Acc& A) {
  constexpr uint32_t G = 32 / LPE;
  const uint32_t lane = lane_id(), sub = lane & (LPE - 1), grp = lane / LPE;
  const uint32_t W = T.W, E = T.E;
  const uint32_t nC = par[0], nQ = par[1];
  const uint32_t* pent = par + kHdr + T.W4;
  uint32_t* cent = ch + kHdr + T.W4;
  const uint32_t* vrow = pent + (size_t)i * E;
  const uint32_t vid = vrow[W];
  // L' = L_p ∩ N(v')   (Alg 2 L8)
  uint32_t lpart = 0, xw = 0;
  for (uint32_t w = lane; w < W; w += 32) {
    uint32_t x = par[kHdr + w] & vrow[w];
    ch[kHdr + w] = x;
    if (w == lane) xw = x;
    lpart += __popc(x);
  }
  const uint32_t lc = warp_sum(lpart);
  uint32_t lp0 = __shfl_sync(GMBE_FULL, xw, sub);
  if (sub >= W) lp0 = 0;
  __syncwarp();
  const uint32_t* lpm = ch + kHdr;  // L' words (for W > LPE)

  // ---- later candidates: k', Thm 4.1 marks, R' absorption, C' (Alg 2 L9-13)
  uint32_t nCc = 0;
  uint32_t r_abs = 0;                 // absorbed count (leader lanes)
  unsigned long long sr_abs = 0;      // absorbed hash sum (leader lanes)
  unsigned long long later_k = 0;     // Σ k_p over later candidates (counters)
  const uint32_t rl_base = par[5] + 1;  // R-list position of the first absorbed vertex
  for (uint32_t base = i + 1; base < nC; base += G) {
    const uint32_t j = base + grp;
    const bool in = j < nC;
    const uint32_t* ej = pent + (size_t)j * E;
    uint32_t kraw = in ? ej[W + 1] : kPruned;
    const bool act = !(kraw & kPruned);
    const uint32_t kp = kraw & ~kPruned;
    uint32_t cnt = 0, x0 = 0;
    if (act) {
      for (uint32_t w = sub; w < W; w += LPE) {
        uint32_t x = ej[w] & (w == sub ? lp0 : lpm[w]);
        if (w == sub) x0 = x;
        cnt += __popc(x);
      }
    }
    cnt = group_sum<LPE>(cnt);
    const bool leader = sub == 0;
    if (act && leader && P.prune && cnt == kp) ((uint32_t*)ej)[W + 1] = kraw | kPruned;
    const bool absorb = act && cnt == lc;
    const bool cand = act && cnt > 0 && cnt < lc;
    const uint32_t id = (absorb || cand) ? ej[W] : 0;
    if (absorb && leader) sr_abs += P.g.hv[id];
    if (T.rlist) {
      uint32_t bal = __ballot_sync(GMBE_FULL, absorb && leader);
      if (absorb && leader) T.rlist[rl_base + r_abs + __popc(bal & lanemask_lt())] = id;
      r_abs += __popc(bal);
    } else {
      r_abs += __popc(__ballot_sync(GMBE_FULL, absorb && leader));
    }
    if (P.counters && act && leader) later_k += kp;
    const uint32_t bal = __ballot_sync(GMBE_FULL, cand && leader);
    uint32_t pos = nCc + __popc(bal & lanemask_lt());
    pos = __shfl_sync(GMBE_FULL, pos, grp * LPE);
    if (cand) {
      uint32_t* ce = cent + (size_t)pos * E;
      for (uint32_t w = sub; w < W; w += LPE) ce[w] = (w == sub) ? x0 : (ej[w] & lpm[w]);
      if (leader) {
        ce[W] = id;
        ce[W + 1] = cnt;
      }
    }
    nCc += __popc(bal);
  }

  // ---- maximality vs Q_p ∪ traversed siblings (Alg 2 L14), building Q' if needed
  bool nonmax = false;
  bool build = nCc > 0;
  uint32_t nQc = 0;
  unsigned long long qk = 0, qkfull = 0;
  for (int part = 0; part < 2; part++) {
    const uint32_t beg = part == 0 ? 0 : nC, end = part == 0 ? i : nC + nQ;
    for (uint32_t base = beg; base < end; base += G) {
      const uint32_t j = base + grp;
      const bool in = j < end;
      const uint32_t* ej = pent + (size_t)j * E;
      const uint32_t kraw = in ? ej[W + 1] : kPruned;
      const bool act = !(kraw & kPruned);
      const uint32_t kp = kraw & ~kPruned;
      const bool leader = sub == 0;
      if (P.counters && act && leader) {
        qkfull += kp;
        if (kp >= lc) qk += kp;
      }
      const bool test = !nonmax && act && (build || kp >= lc);
      uint32_t cnt = 0, x0 = 0;
      if (test) {
        for (uint32_t w = sub; w < W; w += LPE) {
          uint32_t x = ej[w] & (w == sub ? lp0 : lpm[w]);
          if (w == sub) x0 = x;
          cnt += __popc(x);
        }
      }
      cnt = group_sum<LPE>(cnt);
      const bool dom = test && cnt == lc;
      if (build) {
        const bool keep = test && cnt > 0;
        const uint32_t bal = __ballot_sync(GMBE_FULL, keep && leader);
        uint32_t pos = nCc + nQc + __popc(bal & lanemask_lt());
        pos = __shfl_sync(GMBE_FULL, pos, grp * LPE);
        if (keep) {
          uint32_t* ce = cent + (size_t)pos * E;
          for (uint32_t w = sub; w < W; w += LPE) ce[w] = (w == sub) ? x0 : (ej[w] & lpm[w]);
          if (leader) {
            ce[W] = ej[W];
            ce[W + 1] = cnt;
          }
        }
        nQc += __popc(bal);
      }
      if (__any_sync(GMBE_FULL, dom)) {
        nonmax = true;
        build = false;
        if (!P.counters) break;
      }
    }
    if (nonmax && !P.counters) break;
  }

  A.nodes++;
  if (P.counters) {
    unsigned long long lk = warp_sum64(later_k), q1 = warp_sum64(qk), q2 = warp_sum64(qkfull);
    A.abytes += 4ull * (lc + lk + q1);
    A.aqfull += 4ull * (lc + lk + q2);
  }
  if (nonmax) {
    A.nonmax++;
    return 0;
  }
  // ---- Output(L', R') (Alg 2 L15)
  const unsigned long long par_sr = ((unsigned long long)par[7] << 32) | par[6];
  const unsigned long long sr = par_sr + P.g.hv[vid] + warp_sum64(sr_abs);
  const uint32_t rlen = par[5] + 1 + r_abs;
  unsigned long long sl = 0;
  for (uint32_t w = 0; w < W; w++) {
    uint32_t word = lpm[w];
    if ((word >> lane) & 1u) sl += hash_u(P, T.map[w * 32 + lane]);
  }
  sl = warp_sum64(sl);
  A.count++;
  A.checksum += pair_hash(P, sl, sr);
  if (P.per_root && lane == 0) atomicAdd(P.per_root + T.root, 1ull);
  if (T.rlist) {
    if (lane == 0) T.rlist[par[5]] = vid;
    __syncwarp();
    if (P.out_ids) write_record(P, lpm, W, T.map, nullptr, lc, T.rlist, rlen);
  }
  if (nCc == 0) return 1;
  if (lane == 0) {
    ch[0] = nCc;
    ch[1] = nQc;
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
  return kHdr + T.W4 + (rec[0] + rec[1]) * T.E;
}

// first unpruned candidate index >= rec[3], or nC
__device__ __forceinline__ uint32_t find_next(const TaskCtx& T, const uint32_t* rec) {
  __syncwarp();  // order the previous child's Thm 4.1 marks before reading them
  const uint32_t nC = rec[0];
  const uint32_t* ent = rec + kHdr + T.W4;
  for (uint32_t b = rec[3]; b < nC; b += 32) {
    uint32_t j = b + lane_id();
    uint32_t k = j < nC ? ent[(size_t)j * T.E + T.W + 1] : kPruned;
    uint32_t bal = __ballot_sync(GMBE_FULL, !(k & kPruned));
    if (bal) return b + __ffs(bal) - 1;
  }
  return nC;
}

// ---------------------------------------------------------------- slab tasks (a7)
__device__ uint32_t slab_alloc(const Params& P) {
  uint32_t s = kNone;
  if (lane_id() == 0) s = ring_pop(P.fq, P.ring_mask, &P.ctrl->f_head, &P.ctrl->f_tail);
  return __shfl_sync(GMBE_FULL, s, 0);
}
__device__ void slab_free(const Params& P, uint32_t s) {
  if (lane_id() == 0) ring_push(P.fq, P.ring_mask, &P.ctrl->f_tail, s);
}
// slab layout: [0]=W [1]=map length [2]=root rank [3]=R length [4]=node offset [5..7] pad |
//              map | R list | node
__device__ __forceinline__ uint32_t slab_node_off(uint32_t lmap, uint32_t rlen) {
  return kHdr + r4(lmap) + r4(rlen);
}

// Walk the subtree of `top` (Alg 2) -- or, when split, hand its children to the task queue.
template <int LPE>
__device__ void run_task(const Params& P, const TaskCtx& T, uint32_t* top, uint32_t* stack_lo,
                         uint32_t* stack_hi, uint32_t lmap, Acc& A) {
  const uint32_t lane = lane_id();
  uint32_t* cur = top;
  uint32_t* sp = stack_lo;  // first free word
  // Alg 4 L17: heavy-node estimate on the task's top node
  const uint32_t nC0 = top[0], l0 = top[2];
  const unsigned long long h0 = min(nC0, l0);
  const bool split_mode = P.split && h0 > P.bound_height && h0 * nC0 > P.bound_size;
  if (split_mode) A.splits++;
  while (true) {
    const uint32_t i = find_next(T, cur);
    if (i >= cur[0]) {
      if (cur == top) break;
      sp = cur;
      const uint32_t po = cur[4];
      cur = po == kNone ? top : stack_lo + po;
      continue;
    }
    if (lane == 0) cur[3] = i + 1;
    __syncwarp();
    const uint32_t max_entries = cur[0] + cur[1] - 1;
    const uint64_t need = kHdr + T.W4 + (uint64_t)max_entries * T.E;
    uint32_t slab = kNone;
    uint32_t* ch;
    uint32_t node_off = 0;
    if (split_mode && cur == top) {
      const uint32_t rlen_max = T.rlist ? cur[5] + 1 + cur[0] : 0;
      node_off = slab_node_off(lmap, rlen_max);
      if (node_off + need <= P.slab_words) slab = slab_alloc(P);
      if (slab != kNone) ch = P.slabs + (uint64_t)slab * P.slab_words + node_off;
    }
    if (slab == kNone) {
      if (sp + need > stack_hi) {
        if (lane == 0) atomicOr(&P.ctrl->error, kErrArena);
        return;
      }
      ch = sp;
    }
    const int r = gen_child<LPE>(P, T, cur, i, ch, A);
    if (slab != kNone) {
      if (r == 2) {
        // self-contained subtask: universe map + R list + the child node (Alg 4 L25)
        uint32_t* s = P.slabs + (uint64_t)slab * P.slab_words;
        const uint32_t rlen = T.rlist ? ch[5] : 0;
        for (uint32_t j = lane; j < lmap; j += 32) s[kHdr + j] = T.map[j];
        if (T.rlist)
          for (uint32_t j = lane; j < rlen; j += 32) s[kHdr + r4(lmap) + j] = T.rlist[j];
        if (lane == 0) {
          s[0] = T.W;
          s[1] = lmap;
          s[2] = T.root;
          s[3] = rlen;
          s[4] = node_off;
          ch[4] = kNone;
          ch[3] = 0;
        }
        A.tasks++;
        __threadfence();
        __syncwarp();
        if (lane == 0) {
          atomicAdd(&P.ctrl->pending, 1ull);
          ring_push(P.tq, P.ring_mask, &P.ctrl->q_tail, slab);
        }
      } else {
        slab_free(P, slab);
      }
      continue;
    }
    if (r == 2) {
      if (lane == 0) ch[4] = (cur == top) ? kNone : (uint32_t)(cur - stack_lo);
      __syncwarp();
      cur = ch;
      sp = ch + rec_words(T, ch);
    }
  }
}

template <int LPE>
__device__ void run_task_any(const Params& P, const TaskCtx& T, uint32_t* top, uint32_t* lo, uint32_t* hi,
                             uint32_t lmap, Acc& A) {
  run_task<LPE>(P, T, top, lo, hi, lmap, A);
}
__device__ void dispatch_task(const Params& P, const TaskCtx& T, uint32_t* top, uint32_t* lo, uint32_t* hi,
                              uint32_t lmap, Acc& A) {
  if (T.W <= 1) run_task<1>(P, T, top, lo, hi, lmap, A);
  else if (T.W <= 2) run_task<2>(P, T, top, lo, hi, lmap, A);
  else if (T.W <= 4) run_task<4>(P, T, top, lo, hi, lmap, A);
  else if (T.W <= 8) run_task<8>(P, T, top, lo, hi, lmap, A);
  else if (T.W <= 16) run_task<16>(P, T, top, lo, hi, lmap, A);
  else run_task<32>(P, T, top, lo, hi, lmap, A);
}

// ---------------------------------------------------------------- small warp sorts
// sort n 64-bit keys in a[0..n) ascending; a has room for next_pow2(n) keys.
__device__ void warp_sort_keys(unsigned long long* a, uint32_t n, unsigned long long* smem) {
  const uint32_t lane = lane_id();
  if (n <= 1) return;
  if (n <= 32) {  // register bitonic network over the warp
    unsigned long long x = lane < n ? a[lane] : ~0ull;
#pragma unroll
    for (uint32_t k = 2; k <= 32; k <<= 1) {
#pragma unroll
      for (uint32_t j = k >> 1; j > 0; j >>= 1) {
        unsigned long long y = __shfl_xor_sync(GMBE_FULL, x, j);
        const bool up = (lane & k) == 0;
        const bool lower = (lane & j) == 0;
        x = (lower == up) ? (x < y ? x : y) : (x < y ? y : x);
      }
    }
    __syncwarp();
    if (lane < n) a[lane] = x;
    __syncwarp();
    return;
  }
  if (next_pow2(n) <= kSmemSort) {  // bitonic in this warp's shared-memory slice
    for (uint32_t j = lane; j < n; j += 32) smem[j] = a[j];
    __syncwarp();
    warp_sort64(smem, n);
    for (uint32_t j = lane; j < n; j += 32) a[j] = smem[j];
    __syncwarp();
    return;
  }
  warp_sort64(a, n);
}

// warp-cooperative insert of v (lanes with act) into the per-warp table; new slots are appended
// to occ (so the table can be cleaned in O(occupied)).  Returns the slot.
__device__ __forceinline__ uint32_t ht_insert_warp(uint32_t* keys, uint32_t shift, uint32_t mask, uint32_t v,
                                                   bool act, uint32_t* occ, uint32_t& nocc) {
  uint32_t h = act ? ht_hash(v, shift) : 0, slot = kNone;
  bool pend = act;
  while (__any_sync(GMBE_FULL, pend)) {
    bool ins = false;
    if (pend) {
      const uint32_t k = __ldcg(keys + h);
      if (k == v) {
        slot = h;
        pend = false;
      } else if (k == GMBE_EMPTY) {
        const uint32_t old = atomicCAS(keys + h, GMBE_EMPTY, v);
        if (old == GMBE_EMPTY || old == v) {
          slot = h;
          pend = false;
          ins = old == GMBE_EMPTY;
        } else {
          h = (h + 1) & mask;
        }
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

// Per-warp memory: a persistently clean hash table (keys EMPTY, vals 0), its occupied-slot list,
// the entry->child-slot map (NONE), and the dynamic region (records, scratch, node stack).
struct WarpMem {
  uint32_t* keys;
  uint32_t* slotmap;
  unsigned long long* vals;
  uint32_t* occ;
  uint32_t* dyn;
  uint32_t* dyn_end;
  uint32_t* rbuf;
  unsigned long long* sm_sort;  // shared-memory sort slice
};

__device__ __forceinline__ uint32_t* align4(uint32_t* p) {
  return (uint32_t*)(((uintptr_t)p + 15) & ~(uintptr_t)15);
}

__device__ __forceinline__ bool fits(const Params& P, const uint32_t* p, const uint32_t* end) {
  if (p <= end) return true;
  if (lane_id() == 0) atomicOr(&P.ctrl->error, kErrArena);
  return false;
}

// Copy a self-contained task (universe map + R list + node record) into a free slab and enqueue
// it (Alg 4 L25).  Returns false if no slab is free or the task does not fit one.
__device__ bool enqueue_record(const Params& P, const uint32_t* map, uint32_t lmap, uint32_t W, uint32_t root,
                               const uint32_t* rlist, uint32_t rlen, const uint32_t* rec, uint32_t words,
                               Acc& A) {
  const uint32_t lane = lane_id();
  const uint32_t node_off = slab_node_off(lmap, rlist ? rlen : 0);
  if (node_off + words > P.slab_words) return false;
  const uint32_t slab = slab_alloc(P);
  if (slab == kNone) return false;
  uint32_t* s = P.slabs + (uint64_t)slab * P.slab_words;
  for (uint32_t j = lane; j < lmap; j += 32) s[kHdr + j] = map[j];
  if (rlist)
    for (uint32_t j = lane; j < rlen; j += 32) s[kHdr + r4(lmap) + j] = rlist[j];
  for (uint32_t j = lane; j < words; j += 32) s[node_off + j] = rec[j];
  if (lane == 0) {
    s[0] = W;
    s[1] = lmap;
    s[2] = root;
    s[3] = rlist ? rlen : 0;
    s[4] = node_off;
  }
  A.tasks++;
  __threadfence();
  __syncwarp();
  if (lane == 0) {
    atomicAdd(&P.ctrl->pending, 1ull);
    ring_push(P.tq, P.ring_mask, &P.ctrl->q_tail, slab);
  }
  return true;
}

__device__ __forceinline__ bool heavy(const Params& P, uint32_t l, uint32_t nC) {
  const unsigned long long h = min(l, nC);  // tree height estimate
  return P.split && h > P.bound_height && h * nC > P.bound_size;
}

// ---------------------------------------------------------------- root record, bitmap mode
// |L_r| <= wedge_l (<= 64): rows N(x) ∩ L_r (one or two words) come straight from the table.
__device__ void bitmap_root(const Params& P, uint32_t r, uint32_t l, const uint32_t* Lr, uint32_t nC, uint32_t nQ,
                            uint32_t nR, unsigned long long sr, uint32_t nocc, WarpMem& M, Acc& A) {
  const uint32_t lane = lane_id();
  TaskCtx Tc;
  Tc.map = Lr;
  Tc.W = (l + 31) / 32;
  Tc.W4 = r4(Tc.W);
  Tc.E = r4(Tc.W + 2);
  Tc.root = r;
  Tc.rlist = M.rbuf;
  const uint32_t W = Tc.W, E = Tc.E;
  unsigned long long* sortbuf = (unsigned long long*)align4(M.dyn);
  uint32_t* rec = align4((uint32_t*)(sortbuf + next_pow2(nC)));
  const uint64_t rec_need = kHdr + Tc.W4 + (uint64_t)(nC + nQ) * E;
  if (!fits(P, rec + rec_need + 64, M.dyn_end)) return;
  uint32_t* ent = rec + kHdr + Tc.W4;
  uint32_t cc = 0, qc = 0;
  for (uint32_t b = 0; b < nocc; b += 32) {
    const uint32_t j = b + lane;
    const bool occ = j < nocc;
    const uint32_t s = occ ? M.occ[j] : 0;
    const uint32_t v = occ ? __ldcg(M.keys + s) : 0;
    const unsigned long long x = occ ? __ldcg(M.vals + s) : 0;
    const uint32_t c = __popcll(x);
    const bool isR = occ && c == l;
    const bool isC = occ && !isR && v > r;
    const bool isQ = occ && !isR && v < r;
    const uint32_t bC = __ballot_sync(GMBE_FULL, isC);
    if (isC) sortbuf[cc + __popc(bC & lanemask_lt())] = ((unsigned long long)v << 32) | s;
    cc += __popc(bC);
    const uint32_t bQ = __ballot_sync(GMBE_FULL, isQ);
    if (isQ) {
      uint32_t* ee = ent + (size_t)(nC + qc + __popc(bQ & lanemask_lt())) * E;
      ee[0] = (uint32_t)x;
      if (W == 2) ee[1] = (uint32_t)(x >> 32);
      ee[W] = v;
      ee[W + 1] = c;
    }
    qc += __popc(bQ);
  }
  __syncwarp();
  warp_sort_keys(sortbuf, nC, M.sm_sort);  // candidates in rank order (Alg 2 L6)
  for (uint32_t j = lane; j < nC; j += 32) {
    const unsigned long long kv = sortbuf[j];
    const unsigned long long x = __ldcg(M.vals + (uint32_t)kv);
    uint32_t* ee = ent + (size_t)j * E;
    ee[0] = (uint32_t)x;
    if (W == 2) ee[1] = (uint32_t)(x >> 32);
    ee[W] = (uint32_t)(kv >> 32);
    ee[W + 1] = __popcll(x);
  }
  for (uint32_t w = lane; w < W; w += 32) {
    const uint32_t bits = l - w * 32;
    rec[kHdr + w] = bits >= 32 ? GMBE_FULL : ((1u << bits) - 1u);
  }
  if (lane == 0) {
    rec[0] = nC;
    rec[1] = nQ;
    rec[2] = l;
    rec[3] = 0;
    rec[4] = kNone;
    rec[5] = nR + 1;
    rec[6] = (uint32_t)sr;
    rec[7] = (uint32_t)(sr >> 32);
  }
  __syncwarp();
  dispatch_task(P, Tc, rec, align4(rec + rec_need), M.dyn_end, l, A);
}

// ---------------------------------------------------------------- root children, wedge mode
// |L_r| > wedge_l: bitmap rows over L_r would cost (|C|+|Q|)·|L_r|/32 words per child.  Instead each
// child L' = L_r ∩ N(c_i) is generated from the wedges of L' (cost Σ_{u∈L'} |N(u)|), with the
// root's table giving every 2-hop vertex's class, and is REBASED onto its own universe L' --
// a self-contained node that is run in place or queued as a subtask.
__device__ void wedge_root(const Params& P, uint32_t r, uint32_t l, const uint32_t* Lr, uint32_t nC, uint32_t nQ,
                           uint32_t nR, unsigned long long sr, uint32_t nocc, uint32_t shift, uint32_t mask,
                           WarpMem& M, Acc& A) {
  const uint32_t lane = lane_id();
  const DevGraph& g = P.g;
  const uint32_t nE = nC + nQ;
  uint32_t* ids = M.dyn;
  uint32_t* ks = ids + r4(nE);  // bit 31 = pruned (C entries)
  unsigned long long* sortbuf = (unsigned long long*)align4(ks + r4(nE));
  uint32_t* Lc = align4((uint32_t*)(sortbuf + next_pow2(max(nC, 1u))));
  uint32_t* after_lc = align4(Lc + l);
  if (!fits(P, after_lc + 64, M.dyn_end)) return;
  // scan 2: entries (C sorted by rank, then Q); table value := entry index (R := kRTag)
  {
    uint32_t cc = 0, qc = 0;
    for (uint32_t b = 0; b < nocc; b += 32) {
      const uint32_t j = b + lane;
      const bool occ = j < nocc;
      const uint32_t s = occ ? M.occ[j] : 0;
      const uint32_t v = occ ? __ldcg(M.keys + s) : 0;
      const uint32_t c = occ ? (uint32_t)__ldcg(M.vals + s) : 0;
      const bool isR = occ && c == l;
      const bool isC = occ && !isR && v > r;
      const bool isQ = occ && !isR && v < r;
      if (isR) M.vals[s] = kRTag;
      const uint32_t bC = __ballot_sync(GMBE_FULL, isC);
      if (isC) sortbuf[cc + __popc(bC & lanemask_lt())] = ((unsigned long long)v << 32) | s;
      cc += __popc(bC);
      const uint32_t bQ = __ballot_sync(GMBE_FULL, isQ);
      if (isQ) {
        const uint32_t e = nC + qc + __popc(bQ & lanemask_lt());
        ids[e] = v;
        ks[e] = c;
        M.vals[s] = e;
      }
      qc += __popc(bQ);
    }
  }
  __syncwarp();
  warp_sort_keys(sortbuf, nC, M.sm_sort);
  for (uint32_t j = lane; j < nC; j += 32) {
    const unsigned long long kv = sortbuf[j];
    const uint32_t s = (uint32_t)kv;
    ids[j] = (uint32_t)(kv >> 32);
    ks[j] = (uint32_t)__ldcg(M.vals + s);
    M.vals[s] = j;
  }
  __syncwarp();
  const bool split_mode = heavy(P, l, nC);
  if (split_mode) A.splits++;
  const uint32_t rl0 = nR + 1;  // R-list length at the root
  for (uint32_t i = 0; i < nC; i++) {
    __syncwarp();
    if (ks[i] & kPruned) continue;
    const uint32_t c = ids[i];
    // L' = L_r ∩ N(c)   (Alg 2 L8), both lists ascending; search the shorter in the longer
    const uint32_t cb = g.off_v[c], cd = g.off_v[c + 1] - cb;
    const uint32_t* Nc = g.adj_v + cb;
    const uint32_t* As = l <= cd ? Lr : Nc;
    const uint32_t* Bs = l <= cd ? Nc : Lr;
    const uint32_t na = min(l, cd), nb = max(l, cd);
    uint32_t lc = 0;
    for (uint32_t b = 0; b < na; b += 32) {
      const uint32_t j = b + lane;
      bool found = false;
      uint32_t x = 0;
      if (j < na) {
        x = As[j];
        uint32_t lo = 0, hi = nb;
        while (lo < hi) {
          const uint32_t mid = (lo + hi) >> 1;
          if (Bs[mid] < x) lo = mid + 1;
          else hi = mid;
        }
        found = lo < nb && Bs[lo] == x;
      }
      const uint32_t bal = __ballot_sync(GMBE_FULL, found);
      if (found) Lc[lc + __popc(bal & lanemask_lt())] = x;
      lc += __popc(bal);
    }
    __syncwarp();
    uint32_t wq = 0;
    for (uint32_t j = lane; j < lc; j += 32) {
      const uint32_t u = Lc[j];
      wq += g.off_u[u + 1] - g.off_u[u];
    }
    const uint32_t wl = warp_sum(wq);
    const uint32_t Wc = (lc + 31) / 32, Ec = r4(Wc + 2);
    const uint32_t nTmax = min(nE, wl);
    uint32_t* tid = after_lc;
    uint32_t* tcnt = tid + r4(nTmax);
    uint32_t* qlist = tcnt + r4(nTmax);
    uint32_t* trow = qlist + r4(nTmax);
    unsigned long long* csort = (unsigned long long*)align4(trow + (uint64_t)nTmax * Wc);
    uint32_t* crec = align4((uint32_t*)(csort + next_pow2(max(nTmax, 1u))));
    const uint64_t crec_need = kHdr + r4(Wc) + (uint64_t)nTmax * Ec;
    if (!fits(P, crec + crec_need + 64, M.dyn_end)) return;
    A.nodes++;
    if (P.counters) {  // algorithmic bytes (before this step's Thm 4.1 marks)
      unsigned long long lk = 0, qk = 0, qf = 0;
      for (uint32_t e = lane; e < nE; e += 32) {
        const uint32_t k = ks[e], kk = k & ~kPruned;
        const bool pr = (k & kPruned) != 0;
        if (e < nC) {
          if (e > i && !pr) lk += kk;
          else if (e < i && !pr) {
            qf += kk;
            if (kk >= lc) qk += kk;
          }
        } else {
          qf += kk;
          if (kk >= lc) qk += kk;
        }
      }
      lk = warp_sum64(lk);
      qk = warp_sum64(qk);
      qf = warp_sum64(qf);
      A.abytes += 4ull * (lc + lk + qk);
      A.aqfull += 4ull * (lc + lk + qf);
    }
    // wedge pass over L': k'(x) = |N(x) ∩ L'| and rows over L' for every touched entry x
    uint32_t nT = 0;
    for_each_wedge(g, Lc, lc, [&](uint32_t j, uint32_t v, bool act) {
      uint32_t e = kNone;
      if (act && v != r && v != c) {
        const uint32_t h = ht_find(M.keys, shift, mask, v);
        const uint32_t x = (uint32_t)__ldcg(M.vals + h);
        if (x != kRTag && !(x < nC && (ks[x] & kPruned))) e = x;
      }
      const bool claim = e != kNone && atomicCAS(M.slotmap + e, kNone, kClaim) == kNone;
      const uint32_t b = __ballot_sync(GMBE_FULL, claim);
      if (claim) {
        const uint32_t idx = nT + __popc(b & lanemask_lt());
        atomicExch(M.slotmap + e, idx);
        tid[idx] = e;
        atomicExch(tcnt + idx, 0u);
        for (uint32_t w = 0; w < Wc; w++) atomicExch(trow + (size_t)idx * Wc + w, 0u);
      }
      nT += __popc(b);
      __syncwarp();
      if (e != kNone) {
        const uint32_t s = __ldcg(M.slotmap + e);
        atomicAdd(tcnt + s, 1u);
        atomicOr(trow + (size_t)s * Wc + (j >> 5), 1u << (j & 31));
      }
    });
    __syncwarp();
    // classify touched vertices (untouched ones have k' = 0: dropped, never pruned)
    uint32_t nCc = 0, nQc = 0, rabs = 0;
    unsigned long long srabs = 0;
    bool dom = false;
    for (uint32_t b = 0; b < nT; b += 32) {
      const uint32_t s = b + lane;
      const bool act = s < nT;
      const uint32_t e = act ? tid[s] : 0;
      const uint32_t kc = act ? __ldcg(tcnt + s) : 0;
      const bool later = act && e < nC && e > i;
      const bool qlike = act && !later;
      const uint32_t kp = later ? (ks[e] & ~kPruned) : 0;
      if (later && P.prune && kc == kp) ks[e] = kp | kPruned;  // Thm 4.1
      const bool absorb = later && kc == lc;
      const bool cand = later && kc < lc;
      dom |= qlike && kc == lc;
      const uint32_t ba = __ballot_sync(GMBE_FULL, absorb);
      if (absorb) {
        const uint32_t id = ids[e];
        srabs += g.hv[id];
        if (M.rbuf) M.rbuf[rl0 + 1 + rabs + __popc(ba & lanemask_lt())] = id;
      }
      rabs += __popc(ba);
      const uint32_t bc = __ballot_sync(GMBE_FULL, cand);
      if (cand) csort[nCc + __popc(bc & lanemask_lt())] = ((unsigned long long)e << 32) | s;
      nCc += __popc(bc);
      const uint32_t bq = __ballot_sync(GMBE_FULL, qlike);
      if (qlike) qlist[nQc + __popc(bq & lanemask_lt())] = s;
      nQc += __popc(bq);
    }
    const bool nonmax = __any_sync(GMBE_FULL, dom);
    if (nonmax) {
      A.nonmax++;
    } else {
      // Output(L', R')
      const unsigned long long srn = sr + g.hv[c] + warp_sum64(srabs);
      const uint32_t rlen = rl0 + 1 + rabs;
      unsigned long long sl = 0;
      for (uint32_t j = lane; j < lc; j += 32) sl += hash_u(P, Lc[j]);
      sl = warp_sum64(sl);
      A.count++;
      A.checksum += pair_hash(P, sl, srn);
      if (P.per_root && lane == 0) atomicAdd(P.per_root + r, 1ull);
      if (M.rbuf) {
        if (lane == 0) M.rbuf[rl0] = c;
        __syncwarp();
        if (P.out_ids) write_record(P, nullptr, 0, nullptr, Lc, lc, M.rbuf, rlen);
      }
      if (nCc > 0) {
        // the rebased child node over universe L'
        __syncwarp();
        warp_sort_keys(csort, nCc, M.sm_sort);
        uint32_t* cent = crec + kHdr + r4(Wc);
        for (uint32_t j = lane; j < nCc + nQc; j += 32) {
          uint32_t e, s;
          if (j < nCc) {
            const unsigned long long kv = csort[j];
            e = (uint32_t)(kv >> 32);
            s = (uint32_t)kv;
          } else {
            s = qlist[j - nCc];
            e = tid[s];
          }
          uint32_t* ee = cent + (size_t)j * Ec;
          for (uint32_t w = 0; w < Wc; w++) ee[w] = __ldcg(trow + (size_t)s * Wc + w);
          ee[Wc] = ids[e];
          ee[Wc + 1] = __ldcg(tcnt + s);
        }
        for (uint32_t w = lane; w < Wc; w += 32) {
          const uint32_t bits = lc - w * 32;
          crec[kHdr + w] = bits >= 32 ? GMBE_FULL : ((1u << bits) - 1u);
        }
        if (lane == 0) {
          crec[0] = nCc;
          crec[1] = nQc;
          crec[2] = lc;
          crec[3] = 0;
          crec[4] = kNone;
          crec[5] = rlen;
          crec[6] = (uint32_t)srn;
          crec[7] = (uint32_t)(srn >> 32);
        }
        __syncwarp();
        const uint32_t words = kHdr + r4(Wc) + (nCc + nQc) * Ec;
        if (!(split_mode && enqueue_record(P, Lc, lc, Wc, r, M.rbuf, rlen, crec, words, A))) {
          TaskCtx Tc;
          Tc.map = Lc;
          Tc.W = Wc;
          Tc.W4 = r4(Wc);
          Tc.E = Ec;
          Tc.root = r;
          Tc.rlist = M.rbuf;
          dispatch_task(P, Tc, crec, align4(crec + words), M.dyn_end, lc, A);
        }
      }
    }
    __syncwarp();
    for (uint32_t s = lane; s < nT; s += 32) M.slotmap[tid[s]] = kNone;
    __syncwarp();
  }
}

// ---------------------------------------------------------------- root task (a3)
// Root v_s (rank r): L_r = N(v_s); wedge scan of N2(v_s) with local sizes k(v) = |N(v) ∩ L_r|.
__device__ void run_root(const Params& P, uint32_t r, WarpMem& M, Acc& A) {
  const uint32_t lane = lane_id();
  const DevGraph& g = P.g;
  const uint32_t lb = g.off_v[r], l = g.off_v[r + 1] - lb;
  if (l == 0) return;  // isolated vertex: in no biclique (A17)
  const uint32_t* Lr = g.adj_v + lb;
  uint32_t wp = 0;
  for (uint32_t j = lane; j < l; j += 32) {
    const uint32_t u = Lr[j];
    wp += g.off_u[u + 1] - g.off_u[u];
  }
  const uint32_t wedges = warp_sum(wp);
  if (P.counters) {
    A.abytes += 4ull * (l + wedges);
    A.aqfull += 4ull * (l + wedges);
  }
  const uint32_t T = next_pow2(max(64u, 2u * wedges));
  if (T > P.tmax) {
    if (lane == 0) atomicOr(&P.ctrl->error, kErrArena);
    return;
  }
  const uint32_t shift = 32 - (31 - __clz(T)), mask = T - 1;
  uint32_t* keys = M.keys;
  unsigned long long* vals = M.vals;
  const bool bm = l <= P.wedge_l;  // bitmap mode: rows of <= 64 bits straight from the table
  // pass 1 (Alg 3 L2-3)
  uint32_t nocc = 0;
  for_each_wedge(g, Lr, l, [&](uint32_t i, uint32_t v, bool act) {
    const bool a = act && v != r;
    const uint32_t h = ht_insert_warp(keys, shift, mask, v, a, M.occ, nocc);
    if (a) {
      if (bm) atomicOr(vals + h, 1ull << i);
      else atomicAdd(vals + h, 1ull);
    }
  });
  __syncwarp();
  // scan 1: k == |L| -> R (skip the root unless v_s is the earliest vertex of R, Alg 3 L7),
  // later-ordered -> C, earlier-ordered -> Q
  uint32_t nC = 0, nQ = 0, nR = 0;
  bool skip = false;
  unsigned long long sr = 0;
  for (uint32_t b = 0; b < nocc; b += 32) {
    const uint32_t j = b + lane;
    const bool occ = j < nocc;
    const uint32_t s = occ ? M.occ[j] : 0;
    const uint32_t v = occ ? __ldcg(keys + s) : 0;
    uint32_t c = 0;
    if (occ) {
      const unsigned long long x = __ldcg(vals + s);
      c = bm ? __popcll(x) : (uint32_t)x;
    }
    const bool isR = occ && c == l;
    skip |= isR && v < r;
    const bool isC = occ && !isR && v > r;
    const bool isQ = occ && !isR && v < r;
    if (isR) sr += g.hv[v];
    const uint32_t bR = __ballot_sync(GMBE_FULL, isR);
    if (M.rbuf && isR) M.rbuf[1 + nR + __popc(bR & lanemask_lt())] = v;
    nR += __popc(bR);
    nC += __popc(__ballot_sync(GMBE_FULL, isC));
    nQ += __popc(__ballot_sync(GMBE_FULL, isQ));
  }
  skip = __any_sync(GMBE_FULL, skip);
  if (!skip) {
    A.roots_run++;
    sr = warp_sum64(sr) + g.hv[r];
    unsigned long long sl = 0;
    for (uint32_t j = lane; j < l; j += 32) sl += hash_u(P, Lr[j]);
    sl = warp_sum64(sl);
    A.count++;  // emit (L_r, R_r) (A5)
    A.checksum += pair_hash(P, sl, sr);
    if (P.per_root && lane == 0) atomicAdd(P.per_root + r, 1ull);
    if (M.rbuf) {
      if (lane == 0) M.rbuf[0] = r;
      __syncwarp();
      if (P.out_ids) write_record(P, nullptr, 0, nullptr, Lr, l, M.rbuf, nR + 1);
    }
    if (nC > 0) {
      if (bm) bitmap_root(P, r, l, Lr, nC, nQ, nR, sr, nocc, M, A);
      else wedge_root(P, r, l, Lr, nC, nQ, nR, sr, nocc, shift, mask, M, A);
    }
  }
  // leave the table clean for the next root
  __syncwarp();
  for (uint32_t j = lane; j < nocc; j += 32) {
    const uint32_t s = M.occ[j];
    keys[s] = GMBE_EMPTY;
    vals[s] = 0;
  }
  __syncwarp();
}


__global__ void __launch_bounds__(256) k_enum(const Params P) {
  __shared__ unsigned long long s_sort[8][kSmemSort];
  const uint32_t lane = lane_id();
  const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  uint32_t* base = P.arena + (uint64_t)gw * P.arena_words;
  WarpMem M;
  M.keys = base;
  M.slotmap = base + P.tmax;
  M.vals = (unsigned long long*)(base + P.tmax + P.emax);
  M.occ = base + P.tmax + P.emax + 2ull * P.tmax;
  M.dyn = align4(M.occ + P.omax);
  M.dyn_end = base + P.arena_words;
  M.rbuf = P.rbuf ? P.rbuf + (uint64_t)gw * P.rbuf_words : nullptr;
  M.sm_sort = s_sort[threadIdx.x >> 5];
  Acc A = {};
  bool roots_done = false;
  uint32_t idle = 0;
  while (true) {
    // 1. split subtasks first (Alg 4 L3-4)
    uint32_t task = kNone;
    if (lane == 0) task = ring_pop(P.tq, P.ring_mask, &P.ctrl->q_head, &P.ctrl->q_tail);
    task = __shfl_sync(GMBE_FULL, task, 0);
    if (task != kNone) {
      __threadfence();  // acquire: the slab was written on another SM
      uint32_t* s = P.slabs + (uint64_t)task * P.slab_words;
      TaskCtx Tc;
      Tc.W = s[0];
      const uint32_t lmap = s[1];
      Tc.root = s[2];
      const uint32_t rlen = s[3];
      Tc.W4 = r4(Tc.W);
      Tc.E = r4(Tc.W + 2);
      Tc.map = s + kHdr;
      Tc.rlist = M.rbuf;
      if (M.rbuf)
        for (uint32_t j = lane; j < rlen; j += 32) M.rbuf[j] = s[kHdr + r4(lmap) + j];
      __syncwarp();
      const long long c0 = clock64();
      dispatch_task(P, Tc, s + s[4], M.dyn, M.dyn_end, lmap, A);
      if (P.per_root_cycles && lane == 0)
        atomicAdd(P.per_root_cycles + Tc.root, (unsigned long long)(clock64() - c0));
      __syncwarp();
      slab_free(P, task);
      if (lane == 0) atomicAdd(&P.ctrl->pending, ~0ull);
      idle = 0;
      continue;
    }
    // 2. next root (Alg 4 L6), heaviest (highest rank) first
    if (!roots_done) {
      unsigned long long t = 0;
      if (lane == 0) {
        atomicAdd(&P.ctrl->pending, 1ull);
        t = atomicAdd(&P.ctrl->root_cursor, 1ull);
      }
      t = __shfl_sync(GMBE_FULL, t, 0);
      if (t < P.n_roots) {
        const uint32_t j = P.n_roots - 1 - (uint32_t)t;
        const long long c0 = clock64();
        run_root(P, P.part_index + j * P.part_count, M, A);
        if (P.per_root_cycles && lane == 0)
          atomicAdd(P.per_root_cycles + P.part_index + j * P.part_count, (unsigned long long)(clock64() - c0));
        __syncwarp();
        if (lane == 0) atomicAdd(&P.ctrl->pending, ~0ull);
        idle = 0;
        continue;
      }
      if (lane == 0) atomicAdd(&P.ctrl->pending, ~0ull);
      roots_done = true;
    }
    // 3. termination: all roots issued and nothing queued or running
    unsigned long long pend = 0;
    if (lane == 0) pend = ld_volatile(&P.ctrl->pending);
    pend = __shfl_sync(GMBE_FULL, pend, 0);
    if (pend == 0) break;
    __nanosleep(idle < 8 ? 256 : 2048);
    idle++;
  }
  if (lane == 0) {
    Ctrl* c = P.ctrl;
    atomicAdd(&c->count, A.count);
    atomicAdd(&c->checksum, A.checksum);
    atomicAdd(&c->roots_run, A.roots_run);
    atomicAdd(&c->nodes, A.nodes);
    atomicAdd(&c->nonmax, A.nonmax);
    atomicAdd(&c->algo_bytes, A.abytes);
    atomicAdd(&c->algo_qfull, A.aqfull);
    atomicAdd(&c->splits, A.splits);
    atomicAdd(&c->tasks, A.tasks);
  }
}

__global__ void k_init_rings(uint32_t* tq, uint32_t* fq, uint32_t cap, uint32_t n_slabs) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < cap; i += gridDim.x * blockDim.x) {
    tq[i] = GMBE_EMPTY;
    fq[i] = i < n_slabs ? i : GMBE_EMPTY;
  }
}

// ---------------------------------------------------------------- host side
struct Workspace {
  int device = -1;
  void* arena = nullptr;
  size_t arena_bytes = 0;
  uint64_t layout[5] = {0, 0, 0, 0, 0};  // tmax, emax, omax, arena_words, nwarps of the clean tables
  bool clean = false;
  void* slabs = nullptr;
  size_t slab_bytes = 0;
  void* rings = nullptr;
  size_t ring_bytes = 0;
  void* rbuf = nullptr;
  size_t rbuf_bytes = 0;
  void* ctrl = nullptr;
  void* per_root = nullptr;
  size_t per_root_bytes = 0;
  void* per_root_cyc = nullptr;
  size_t per_root_cyc_bytes = 0;
};

cudaError_t ensure(void** p, size_t* have, size_t need) {
  if (*have >= need && *p) return cudaSuccess;
  if (*p) cudaFree(*p);
  *p = nullptr;
  *have = 0;
  cudaError_t e = cudaMalloc(p, need ? need : 16);
  if (e == cudaSuccess) *have = need;
  return e;
}

}  // namespace


extern "C" uint64_t gmbe_node_buf_bound_bytes(uint64_t dv, uint64_t d2v) { return (3 * dv + 2 * d2v) * 4; }
extern "C" uint64_t gmbe_naive_alloc_bytes(uint64_t dv, uint64_t d2v) { return dv * (dv + d2v) * 4; }

static Workspace* ws_acquire(int device);
static void ws_return(Workspace* w);

extern "C" int gmbe_enumerate(const gmbe_graph* G, const gmbe_opts* opts, gmbe_result* out) {
  if (!G || !out) return gmbe_set_error(GMBE_EINVAL, "gmbe_enumerate: NULL argument");
  gmbe_opts o{};
  if (opts && opts->struct_size) o = *opts;
  const uint32_t parts = o.part_count ? o.part_count : 1;
  if (o.part_index >= parts) return gmbe_set_error(GMBE_EINVAL, "gmbe_enumerate: part_index >= part_count");
  if ((o.out_offsets == nullptr) != (o.out_ids == nullptr))
    return gmbe_set_error(GMBE_EINVAL, "gmbe_enumerate: out_offsets and out_ids must be given together");
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

  int sms = 0;
  GMBE_CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, G->device));
  uint32_t wps = o.warps_per_sm ? o.warps_per_sm : 32;
  if (wps < 8) wps = 8;
  if (wps > 64) wps = 64;
  int bps_max = 0;
  GMBE_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps_max, k_enum, 256, 0));
  uint32_t bps = wps / 8;
  if ((int)bps > bps_max) bps = bps_max;
  if (bps < 1) bps = 1;
  const uint32_t blocks = (uint32_t)sms * bps;
  const uint64_t nwarps = (uint64_t)blocks * 8;

  // per-warp arena: clean hash table sized for the largest root's wedges, entry map, occupied list,
  // and the dynamic region (root record, rebased children, node stack), bounded by free memory
  const uint64_t wb = (uint64_t)g.wedge_bound + 64;
  uint64_t tmax = 64;
  while (tmax < 2 * wb) tmax <<= 1;
  const uint64_t emax = (wb + 3) & ~3ull, omax = emax;
  const uint64_t fixed = tmax + emax + 2 * tmax + omax + 8;
  uint64_t dyn = o.arena_words;
  if (!dyn) {
    const uint64_t want = 24 * wb + (1u << 18);
    size_t fr = 0, tot = 0;
    GMBE_CUDA_TRY(cudaMemGetInfo(&fr, &tot));
    const uint64_t cap_total = (uint64_t)(fr * 0.5) / 4 / nwarps;
    const uint64_t cap = cap_total > fixed + (1u << 16) ? cap_total - fixed : (1u << 16);
    dyn = want < cap ? want : cap;
  }
  const uint64_t arena_words = (fixed + dyn + 3) & ~3ull;
  uint64_t slab_words = o.slab_words ? o.slab_words : (1u << 16);
  slab_words = (slab_words + 3) & ~3ull;
  uint64_t n_slabs = o.n_slabs ? o.n_slabs : 8192;
  if (n_slabs > (1u << 24)) n_slabs = 1u << 24;
  uint32_t cap = 1;
  while (cap < n_slabs + 64) cap <<= 1;
  const bool want_out = o.out_ids != nullptr;
  const uint32_t rbuf_words = want_out ? (uint32_t)(wb + 64) : 0;

  GMBE_CUDA_TRY(ensure(&W.arena, &W.arena_bytes, nwarps * arena_words * 4));
  {
    const uint64_t sig[5] = {tmax, emax, omax, arena_words, nwarps};
    if (!W.clean || std::memcmp(sig, W.layout, sizeof(sig)) != 0) {
      // keys + slotmap := 0xff.. (EMPTY / NONE), vals := 0 -- once; every root leaves them clean
      GMBE_CUDA_TRY(cudaMemset2DAsync(W.arena, arena_words * 4, 0xff, (tmax + emax) * 4, nwarps, s));
      GMBE_CUDA_TRY(cudaMemset2DAsync((uint32_t*)W.arena + tmax + emax, arena_words * 4, 0, 2 * tmax * 4,
                                      nwarps, s));
      std::memcpy(W.layout, sig, sizeof(sig));
      W.clean = true;
    }
  }
  GMBE_CUDA_TRY(ensure(&W.slabs, &W.slab_bytes, n_slabs * slab_words * 4));
  GMBE_CUDA_TRY(ensure(&W.rings, &W.ring_bytes, (size_t)cap * 2 * 4));
  if (want_out) GMBE_CUDA_TRY(ensure(&W.rbuf, &W.rbuf_bytes, nwarps * rbuf_words * 4));
  size_t ctrl_have = W.ctrl ? sizeof(Ctrl) : 0;
  GMBE_CUDA_TRY(ensure(&W.ctrl, &ctrl_have, sizeof(Ctrl)));
  if (o.per_root_count) GMBE_CUDA_TRY(ensure(&W.per_root, &W.per_root_bytes, (size_t)(g.n_v + 1) * 8));
  if (o.per_root_cycles)
    GMBE_CUDA_TRY(ensure(&W.per_root_cyc, &W.per_root_cyc_bytes, (size_t)(g.n_v + 1) * 8));

  Params P{};
  P.g = g;
  P.part_index = o.part_index;
  P.part_count = parts;
  P.n_roots = g.n_v > o.part_index ? (g.n_v - o.part_index + parts - 1) / parts : 0;
  P.prune = o.no_prune ? 0 : 1;
  P.split = o.no_split ? 0 : 1;
  P.bound_height = o.bound_height ? o.bound_height : 20;
  P.bound_size = o.bound_size ? o.bound_size : 1500;
  P.counters = o.counters ? 1 : 0;
  P.hu_side = g.swapped ? 1 : 0;
  P.wedge_l = o.wedge_l ? (o.wedge_l > 64 ? 64 : o.wedge_l) : 64;
  P.arena = (uint32_t*)W.arena;
  P.arena_words = arena_words;
  P.tmax = (uint32_t)tmax;
  P.emax = (uint32_t)emax;
  P.omax = (uint32_t)omax;
  P.rbuf = want_out ? (uint32_t*)W.rbuf : nullptr;
  P.rbuf_words = rbuf_words;
  P.slabs = (uint32_t*)W.slabs;
  P.slab_words = slab_words;
  P.n_slabs = (uint32_t)n_slabs;
  P.tq = (uint32_t*)W.rings;
  P.fq = (uint32_t*)W.rings + cap;
  P.ring_mask = cap - 1;
  P.ctrl = (Ctrl*)W.ctrl;
  P.out_offsets = (unsigned long long*)o.out_offsets;
  P.out_offsets_cap = want_out ? o.out_offsets_cap : 0;
  P.out_ids = o.out_ids;
  P.out_ids_cap = want_out ? o.out_ids_cap : 0;
  P.per_root = o.per_root_count ? (unsigned long long*)W.per_root : nullptr;
  P.per_root_cycles = o.per_root_cycles ? (unsigned long long*)W.per_root_cyc : nullptr;

  Ctrl hc{};
  hc.f_tail = n_slabs;
  GMBE_CUDA_TRY(cudaMemcpyAsync(W.ctrl, &hc, sizeof(Ctrl), cudaMemcpyHostToDevice, s));
  k_init_rings<<<(cap + 255) / 256 < 1024 ? (cap + 255) / 256 : 1024, 256, 0, s>>>(P.tq, P.fq, cap,
                                                                                    (uint32_t)n_slabs);
  gmbe_note_launch();
  if (P.per_root) GMBE_CUDA_TRY(cudaMemsetAsync(W.per_root, 0, (size_t)(g.n_v + 1) * 8, s));
  if (P.per_root_cycles) GMBE_CUDA_TRY(cudaMemsetAsync(W.per_root_cyc, 0, (size_t)(g.n_v + 1) * 8, s));
  GMBE_CUDA_TRY(cudaGetLastError());
  cudaEvent_t e0, e1;
  GMBE_CUDA_TRY(cudaEventCreate(&e0));
  GMBE_CUDA_TRY(cudaEventCreate(&e1));
  GMBE_CUDA_TRY(cudaEventRecord(e0, s));
  if (P.n_roots > 0) k_enum<<<blocks, 256, 0, s>>>(P), gmbe_note_launch();
  cudaError_t le = cudaGetLastError();
  GMBE_CUDA_TRY(cudaEventRecord(e1, s));
  GMBE_CUDA_TRY(le);
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
  out->n_written = hc.out_rec < P.out_offsets_cap ? hc.out_rec : P.out_offsets_cap;
  out->truncated = hc.truncated;
  out->roots_run = hc.roots_run;
  out->nodes = hc.nodes;
  out->nonmax = hc.nonmax;
  out->algo_bytes = hc.algo_bytes;
  out->algo_bytes_qfull = hc.algo_qfull;
  out->splits = hc.splits;
  out->tasks = hc.tasks;
  out->kernel_ms = ms;
  if (hc.error) W.clean = false;
  if (hc.error)
    return gmbe_set_error(GMBE_EINTERNAL, std::string("gmbe_enumerate: device workspace exceeded (") +
                                              ((hc.error & kErrArena) ? "arena" : "slab") +
                                              "); raise opts.arena_words");
  return GMBE_OK;
}

#include <mutex>
// Workspace pool: a call takes an idle workspace of its device (or a new one) and returns it, so
// repeated calls reuse device memory and concurrent calls never share one.
static std::mutex g_ws_mu;
static std::vector<Workspace*> g_ws_idle;
static Workspace* ws_acquire(int device) {
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
static void ws_return(Workspace* w) {
  std::lock_guard<std::mutex> lk(g_ws_mu);
  g_ws_idle.push_back(w);
}
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
    for (void* p : {w->arena, w->slabs, w->rings, w->rbuf, w->ctrl, w->per_root, w->per_root_cyc})
      if (p) cudaFree(p);
    delete w;
    g_ws_idle.erase(g_ws_idle.begin() + i);
  }
  cudaSetDevice(prev);
}
