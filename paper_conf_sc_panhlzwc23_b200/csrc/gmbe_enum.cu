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
  uint32_t* arena;
  uint64_t arena_words;
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

// ---------------------------------------------------------------- root task (a3)
__device__ void run_root(const Params& P, uint32_t r, uint32_t* arena, uint32_t* rbuf, Acc& A) {
  const uint32_t lane = lane_id();
  const DevGraph& g = P.g;
  const uint32_t lb = g.off_v[r], l = g.off_v[r + 1] - lb;
  if (l == 0) return;  // isolated vertex: in no biclique (A17)
  const uint32_t* Lr = g.adj_v + lb;
  // wedge count (and the root's algorithmic bytes)
  uint32_t wp = 0;
  for (uint32_t j = lane; j < l; j += 32) {
    uint32_t u = Lr[j];
    wp += g.off_u[u + 1] - g.off_u[u];
  }
  const uint32_t wedges = warp_sum(wp);
  if (P.counters) {
    A.abytes += 4ull * (l + wedges);
    A.aqfull += 4ull * (l + wedges);
  }
  uint32_t T = next_pow2(max(64u, 2u * wedges));
  const uint32_t logT = 31 - __clz(T);
  const uint32_t shift = 32 - logT, mask = T - 1;
  uint32_t* keys = arena;
  uint32_t* vals = arena + T;
  if (2ull * T + 64 > P.arena_words) {
    if (lane == 0) atomicOr(&P.ctrl->error, kErrArena);
    return;
  }
  for (uint32_t j = lane; j < T; j += 32) {
    keys[j] = GMBE_EMPTY;
    vals[j] = 0;
  }
  __syncwarp();
  __threadfence_block();
  const bool small = l <= 32;  // rows fit one word: build them directly in pass 1
  // pass 1: N2(v_s) with local neighbourhood sizes k(v_c) = |N(v_c) ∩ L_r| (Alg 3 L2-3)
  for_each_wedge(g, Lr, l, [&](uint32_t i, uint32_t v, bool act) {
    if (act && v != r) {
      uint32_t h = ht_insert(keys, shift, mask, v);
      if (small) atomicOr(vals + h, 1u << i);
      else atomicAdd(vals + h, 1u);
    }
  });
  __syncwarp();
  __threadfence();
  // scan 1: classify.  k == |L| -> R (skip root unless v_s is the earliest in R, Alg 3 L7),
  // later-ordered -> C, earlier-ordered -> Q.
  uint32_t nC = 0, nQ = 0, nR = 0;
  bool skip = false;
  unsigned long long sr = 0;
  for (uint32_t b = 0; b < T; b += 32) {
    const uint32_t s = b + lane;
    const uint32_t v = __ldcg(keys + s);
    const bool occ = v != GMBE_EMPTY;
    uint32_t c = 0;
    if (occ) {
      uint32_t x = __ldcg(vals + s);
      c = small ? __popc(x) : x;
    }
    const bool isR = occ && c == l;
    skip |= isR && v < r;
    const bool isC = occ && !isR && v > r;
    const bool isQ = occ && !isR && v < r;
    if (isR) sr += g.hv[v];
    const uint32_t bR = __ballot_sync(GMBE_FULL, isR);
    if (rbuf && isR) rbuf[1 + nR + __popc(bR & lanemask_lt())] = v;
    nR += __popc(bR);
    nC += __popc(__ballot_sync(GMBE_FULL, isC));
    nQ += __popc(__ballot_sync(GMBE_FULL, isQ));
  }
  if (__any_sync(GMBE_FULL, skip)) {
    __syncwarp();
    return;
  }
  A.roots_run++;
  sr = warp_sum64(sr) + g.hv[r];
  // emit (L_r, R_r)  (A5)
  {
    unsigned long long sl = 0;
    for (uint32_t j = lane; j < l; j += 32) sl += hash_u(P, Lr[j]);
    sl = warp_sum64(sl);
    A.count++;
    A.checksum += pair_hash(P, sl, sr);
    if (P.per_root && lane == 0) atomicAdd(P.per_root + r, 1ull);
    if (rbuf) {
      if (lane == 0) rbuf[0] = r;
      __syncwarp();
      if (P.out_ids) write_record(P, nullptr, 0, nullptr, Lr, l, rbuf, nR + 1);
    }
  }
  if (nC == 0) return;

  // ---- build the root node record.  Scratch after the table: sort buffer | useful bits |
  // useful-word prefix | compacted map | root record | DFS stack.
  uint32_t* scratch = vals + T;
  unsigned long long* sortbuf = (unsigned long long*)(((uintptr_t)scratch + 15) & ~(uintptr_t)15);
  uint32_t* after_sort = (uint32_t*)(sortbuf + next_pow2(nC));
  const uint32_t nuw = (l + 31) / 32;
  uint32_t* useful = after_sort;        // l bits (large roots)
  uint32_t* upre = useful + r4(nuw);    // exclusive prefix popcount of useful words
  uint32_t* mapbuf = upre + r4(nuw);    // compacted universe
  uint32_t* rec = (uint32_t*)(((uintptr_t)(small ? after_sort : mapbuf + r4(l)) + 15) & ~(uintptr_t)15);
  {
    const uint64_t wmax = (l + 31) / 32;
    const uint64_t need = (uint64_t)(rec - arena) + kHdr + r4(wmax) + (uint64_t)(nC + nQ) * r4(wmax + 2) + 64;
    if (need > P.arena_words) {
      if (lane == 0) atomicOr(&P.ctrl->error, kErrArena);
      return;
    }
  }
  uint32_t lu = l;                 // universe size
  const uint32_t* map = Lr;        // universe map
  if (!small) {
    // pass 2: keep only L_r vertices adjacent to some candidate (every child L' lies inside)
    for (uint32_t j = lane; j < nuw; j += 32) useful[j] = 0;
    __syncwarp();
    for_each_wedge(g, Lr, l, [&](uint32_t i, uint32_t v, bool act) {
      if (act && v > r) {
        uint32_t h = ht_find(keys, shift, mask, v);
        if (h != kNone && __ldcg(vals + h) < l) atomicOr(useful + (i >> 5), 1u << (i & 31));
      }
    });
    __syncwarp();
    __threadfence();
    uint32_t c = 0;
    for (uint32_t b = 0; b < l; b += 32) {
      const uint32_t i = b + lane;
      const uint32_t uw = __ldcg(useful + (b >> 5));
      if (lane == 0) upre[b >> 5] = c;
      const bool u = i < l && ((uw >> lane) & 1u);
      const uint32_t bal = __ballot_sync(GMBE_FULL, u);
      if (u) mapbuf[c + __popc(bal & lanemask_lt())] = Lr[i];
      c += __popc(bal);
    }
    lu = c;
    map = mapbuf;
    __syncwarp();
  }
  TaskCtx Tc;
  Tc.map = map;
  Tc.W = (lu + 31) / 32;
  Tc.W4 = r4(Tc.W);
  Tc.E = r4(Tc.W + 2);
  Tc.root = r;
  Tc.rlist = rbuf;
  const uint64_t rec_need = kHdr + Tc.W4 + (uint64_t)(nC + nQ) * Tc.E;
  uint32_t* ent = rec + kHdr + Tc.W4;
  const uint32_t W = Tc.W, E = Tc.E;
  // zero rows of the large-root entries (filled by pass 3)
  if (!small)
    for (uint64_t j = lane; j < (uint64_t)(nC + nQ) * E; j += 32) ent[j] = 0;
  __syncwarp();
  // scan 2: C -> sort buffer, Q -> entries nC.. (table order)
  {
    uint32_t cc = 0, qc = 0;
    for (uint32_t b = 0; b < T; b += 32) {
      const uint32_t s = b + lane;
      const uint32_t v = __ldcg(keys + s);
      const bool occ = v != GMBE_EMPTY;
      uint32_t x = occ ? __ldcg(vals + s) : 0;
      const uint32_t c = small ? __popc(x) : x;
      const bool isR = occ && c == l;
      const bool isC = occ && !isR && v > r;
      const bool isQ = occ && !isR && v < r;
      const uint32_t bC = __ballot_sync(GMBE_FULL, isC);
      if (isC) sortbuf[cc + __popc(bC & lanemask_lt())] = ((unsigned long long)v << 32) | s;
      cc += __popc(bC);
      const uint32_t bQ = __ballot_sync(GMBE_FULL, isQ);
      if (isQ) {
        const uint32_t e = nC + qc + __popc(bQ & lanemask_lt());
        uint32_t* ee = ent + (size_t)e * E;
        if (small) ee[0] = x;
        ee[W] = v;
        ee[W + 1] = c;
        if (!small) vals[s] = e;
      }
      qc += __popc(bQ);
      if (!small && isR) vals[s] = kNone;
    }
  }
  __syncwarp();
  warp_sort64(sortbuf, nC);  // candidates in rank order (Alg 2 L6: smallest first)
  for (uint32_t j = lane; j < nC; j += 32) {
    const unsigned long long kv = sortbuf[j];
    const uint32_t v = (uint32_t)(kv >> 32), s = (uint32_t)kv;
    const uint32_t x = __ldcg(vals + s);
    uint32_t* ee = ent + (size_t)j * E;
    if (small) {
      ee[0] = x;
      ee[W + 1] = __popc(x);
    } else {
      ee[W + 1] = x;
      vals[s] = j;
    }
    ee[W] = v;
  }
  __syncwarp();
  __threadfence();
  if (!small) {
    // pass 3: rows over the compacted universe
    for_each_wedge(g, Lr, l, [&](uint32_t i, uint32_t v, bool act) {
      const uint32_t uw = act ? __ldcg(useful + (i >> 5)) : 0;
      if (act && v != r && ((uw >> (i & 31)) & 1u)) {
        const uint32_t jl = upre[i >> 5] + __popc(uw & ((1u << (i & 31)) - 1u));
        const uint32_t h = ht_find(keys, shift, mask, v);
        const uint32_t e = h == kNone ? kNone : __ldcg(vals + h);
        if (e != kNone) atomicOr(ent + (size_t)e * E + (jl >> 5), 1u << (jl & 31));
      }
    });
    __syncwarp();
    __threadfence();
  }
  // header + L mask (all universe bits)
  for (uint32_t w = lane; w < W; w += 32) {
    const uint32_t bits = lu - w * 32;
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
  uint32_t* lo = rec + rec_need;
  lo = (uint32_t*)(((uintptr_t)lo + 15) & ~(uintptr_t)15);
  dispatch_task(P, Tc, rec, lo, arena + P.arena_words, lu, A);
}

__global__ void __launch_bounds__(256) k_enum(const Params P) {
  const uint32_t lane = lane_id();
  const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  uint32_t* arena = P.arena + (uint64_t)gw * P.arena_words;
  uint32_t* rbuf = P.rbuf ? P.rbuf + (uint64_t)gw * P.rbuf_words : nullptr;
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
      Tc.rlist = rbuf;
      if (rbuf)
        for (uint32_t j = lane; j < rlen; j += 32) rbuf[j] = s[kHdr + r4(lmap) + j];
      __syncwarp();
      uint32_t* top = s + s[4];
      dispatch_task(P, Tc, top, arena, arena + P.arena_words, lmap, A);
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
        run_root(P, P.part_index + j * P.part_count, arena, rbuf, A);
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
  void* slabs = nullptr;
  size_t slab_bytes = 0;
  void* rings = nullptr;
  size_t ring_bytes = 0;
  void* rbuf = nullptr;
  size_t rbuf_bytes = 0;
  void* ctrl = nullptr;
  void* per_root = nullptr;
  size_t per_root_bytes = 0;
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

  // arena sizing: hash table + root record + stack for the worst root (bounded by memory)
  const uint64_t wb = g.wedge_bound + 64;
  const uint64_t Tmax = 1ull << (64 - __builtin_clzll(2 * wb));
  const uint64_t Wmax = (g.delta_v + 31) / 32;
  const uint64_t Emax = (Wmax + 2 + 3) & ~3ull;
  uint64_t arena_words = o.arena_words;
  if (!arena_words) {
    uint64_t want = 2 * Tmax + 2 * Tmax /*sort*/ + 4 * wb + wb * Emax * 3 + (1u << 16);
    size_t fr = 0, tot = 0;
    GMBE_CUDA_TRY(cudaMemGetInfo(&fr, &tot));
    uint64_t cap = (uint64_t)(fr * 0.45) / 4 / nwarps;
    arena_words = want < cap ? want : cap;
    if (arena_words < (1u << 16)) arena_words = 1u << 16;
  }
  arena_words = (arena_words + 3) & ~3ull;
  uint64_t slab_words = o.slab_words ? o.slab_words : (1u << 16);
  slab_words = (slab_words + 3) & ~3ull;
  uint64_t n_slabs = o.n_slabs ? o.n_slabs : 8192;
  if (n_slabs > (1u << 24)) n_slabs = 1u << 24;
  uint32_t cap = 1;
  while (cap < n_slabs + 64) cap <<= 1;
  const bool want_out = o.out_ids != nullptr;
  const uint32_t rbuf_words = want_out ? (uint32_t)(wb + 64) : 0;

  GMBE_CUDA_TRY(ensure(&W.arena, &W.arena_bytes, nwarps * arena_words * 4));
  GMBE_CUDA_TRY(ensure(&W.slabs, &W.slab_bytes, n_slabs * slab_words * 4));
  GMBE_CUDA_TRY(ensure(&W.rings, &W.ring_bytes, (size_t)cap * 2 * 4));
  if (want_out) GMBE_CUDA_TRY(ensure(&W.rbuf, &W.rbuf_bytes, nwarps * rbuf_words * 4));
  size_t ctrl_have = W.ctrl ? sizeof(Ctrl) : 0;
  GMBE_CUDA_TRY(ensure(&W.ctrl, &ctrl_have, sizeof(Ctrl)));
  if (o.per_root_count) GMBE_CUDA_TRY(ensure(&W.per_root, &W.per_root_bytes, (size_t)(g.n_v + 1) * 8));

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
  P.arena = (uint32_t*)W.arena;
  P.arena_words = arena_words;
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

  Ctrl hc{};
  hc.f_tail = n_slabs;
  GMBE_CUDA_TRY(cudaMemcpyAsync(W.ctrl, &hc, sizeof(Ctrl), cudaMemcpyHostToDevice, s));
  k_init_rings<<<(cap + 255) / 256 < 1024 ? (cap + 255) / 256 : 1024, 256, 0, s>>>(P.tq, P.fq, cap,
                                                                                    (uint32_t)n_slabs);
  gmbe_note_launch();
  if (P.per_root) GMBE_CUDA_TRY(cudaMemsetAsync(W.per_root, 0, (size_t)(g.n_v + 1) * 8, s));
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
  if (o.per_root_count && g.n_v) {
    std::vector<unsigned long long> pr(g.n_v);
    std::vector<uint32_t> r2i(g.n_v);
    GMBE_CUDA_TRY(cudaMemcpy(pr.data(), W.per_root, g.n_v * 8, cudaMemcpyDeviceToHost));
    GMBE_CUDA_TRY(cudaMemcpy(r2i.data(), g.rank2id, g.n_v * 4, cudaMemcpyDeviceToHost));
    for (uint32_t rr = 0; rr < g.n_v; rr++) o.per_root_count[r2i[rr]] = pr[rr];
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
    for (void* p : {w->arena, w->slabs, w->rings, w->rbuf, w->ctrl, w->per_root})
      if (p) cudaFree(p);
    delete w;
    g_ws_idle.erase(g_ws_idle.begin() + i);
  }
  cudaSetDevice(prev);
}
