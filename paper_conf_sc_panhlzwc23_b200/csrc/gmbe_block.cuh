// gmbe_block.cuh -- GMBE-BLOCK, the block-centric scheme (Sec 4.3; the variant
// of Sec 6.3, Fig 8 / Fig 9).  Included inside gmbe_enum.cu's anonymous namespace.
//
// One thread block = one Alg 3 task (a first-level root v_s), with no splitting and no task queue:
// blocks draw roots from the same atomic cursor as k_enum (heaviest first) and walk the root's whole
// subtree depth-first.  Inside the block every node is generated cooperatively: the later candidates
// of the parent are dealt over the block's threads (one thread per candidate entry), the compaction
// of C' is a block-wide scan, and the maximality test (Alg 2 L14, |Γ(L')| == |R'|, reading B1) is a
// block-parallel scan of the root's Γ index (or of N(u*) by binary searches when the root has none).
// The root node itself is built by the block's first warp with the same code as k_enum (run_root).
// Thm 4.1 marks a pruned candidate in place (k := kPruned) instead of compacting the parent, so the
// later siblings skip it; the tree and every counter are the canonical ones (reading A9).
//
// This is an ablation variant (the paper's GMBE-BLOCK); it trades k_enum's load balance for more
// threads per task, which is exactly what Fig 9 measures.
constexpr uint32_t kBlkThreads = 32 * kWpb;
constexpr uint32_t kPruned = 0xffffffffu;

struct BlkSmem {
  // the root builder's (warp 0) slices, as in k_enum
  unsigned long long sort[kSmemSort];
  unsigned long long tvals[kSmemTable ? kSmemTable : 1];
  uint32_t tkeys[kSmemTable ? kSmemTable : 1];
  uint32_t tocc[kSmemTable ? kSmemTable / 2 : 1];
  // block reductions / scans
  uint32_t wc[3][kWpb];
  uint32_t w32[kWpb];
  unsigned long long w64[kWpb];
  unsigned long long wkey[kWpb];
  // the current task, published by warp 0
  TaskCtx T;
  uint32_t* top;
  uint32_t* lo;
  uint32_t bc[4];
};

__device__ __forceinline__ uint32_t blk_sum32(uint32_t x, BlkSmem& S) {
  x = __reduce_add_sync(GMBE_FULL, x);
  if (lane_id() == 0) S.w32[threadIdx.x >> 5] = x;
  __syncthreads();
  uint32_t t = 0;
#pragma unroll
  for (uint32_t k = 0; k < kWpb; k++) t += S.w32[k];
  __syncthreads();
  return t;
}
__device__ __forceinline__ unsigned long long blk_sum64(unsigned long long x, BlkSmem& S) {
  x = warp_sum64(x);
  if (lane_id() == 0) S.w64[threadIdx.x >> 5] = x;
  __syncthreads();
  unsigned long long t = 0;
#pragma unroll
  for (uint32_t k = 0; k < kWpb; k++) t += S.w64[k];
  __syncthreads();
  return t;
}
__device__ __forceinline__ unsigned long long blk_min64(unsigned long long x, BlkSmem& S) {
  for (int o = 16; o; o >>= 1) x = min(x, (unsigned long long)__shfl_xor_sync(GMBE_FULL, x, o));
  if (lane_id() == 0) S.wkey[threadIdx.x >> 5] = x;
  __syncthreads();
  unsigned long long t = ~0ull;
#pragma unroll
  for (uint32_t k = 0; k < kWpb; k++) t = min(t, S.wkey[k]);
  __syncthreads();
  return t;
}
// block-wide exclusive positions of three flags (thread order) and their totals
__device__ __forceinline__ void blk_scan3(bool a, bool b, bool c, uint32_t pos[3], uint32_t tot[3], BlkSmem& S) {
  const uint32_t lane = lane_id(), wid = threadIdx.x >> 5;
  const uint32_t ba = __ballot_sync(GMBE_FULL, a), bb = __ballot_sync(GMBE_FULL, b), bcm = __ballot_sync(GMBE_FULL, c);
  if (lane == 0) {
    S.wc[0][wid] = __popc(ba);
    S.wc[1][wid] = __popc(bb);
    S.wc[2][wid] = __popc(bcm);
  }
  __syncthreads();
  const uint32_t lt = lanemask_lt();
  pos[0] = __popc(ba & lt);
  pos[1] = __popc(bb & lt);
  pos[2] = __popc(bcm & lt);
  tot[0] = tot[1] = tot[2] = 0;
#pragma unroll
  for (uint32_t k = 0; k < kWpb; k++) {
#pragma unroll
    for (int f = 0; f < 3; f++) {
      if (k < wid) pos[f] += S.wc[f][k];
      tot[f] += S.wc[f][k];
    }
  }
  __syncthreads();
}

// Alg 2 L14 by the whole block: |Γ(L')| == |R'| with L' = the lc bits of lpm (W words over map).
__device__ bool blk_gamma_is_r(const Params& P, const TaskCtx& T, const uint32_t* lpm, uint32_t lc, uint32_t rlen,
                               BlkSmem& S) {
  const uint32_t tid = threadIdx.x, W = T.W;
  const DevGraph& g = P.g;
  if (lc == 1) {  // Γ({u}) = N(u)
    uint32_t u = kNone;
    for (uint32_t w = tid; w < W; w += kBlkThreads)
      if (lpm[w]) u = T.map[w * 32 + __ffs(lpm[w]) - 1];
    const unsigned long long k = blk_min64(u, S);
    const uint32_t uu = (uint32_t)k;
    return g.off_u[uu + 1] - g.off_u[uu] == rlen;
  }
  if (T.gx) {  // universe <= 64 bits: |Γ(L')| = 1 (v_s) + #X2 rows covering L'
    const unsigned long long lm = ((unsigned long long)(W > 1 ? lpm[1] : 0u) << 32) | lpm[0];
    const uint32_t nx = T.gx[0];
    const unsigned long long* xrow = (const unsigned long long*)(T.gx + 4);
    uint32_t c = 0;
    for (uint32_t x = tid; x < nx; x += kBlkThreads) c += (xrow[x] & lm) == lm;
    return 1 + blk_sum32(c, S) == rlen;
  }
  if (T.cols) {  // |Γ(L')| = 1 + popc(AND_{j∈L'} col_j) over X2
    uint32_t c = 0;
    for (uint32_t xw = tid; xw < T.ncw; xw += kBlkThreads) {
      uint32_t acc = GMBE_FULL;
      for (uint32_t w = 0; w < W && acc; w++)
        for (uint32_t word = lpm[w]; word && acc; word &= word - 1)
          acc &= __ldg(T.cols + (size_t)(w * 32 + __ffs(word) - 1) * T.ncw + xw);
      c += __popc(acc);
    }
    return 1 + blk_sum32(c, S) == rlen;
  }
  // no Γ index: count Γ(L') over N(u*) for the lowest-degree u* ∈ L', one v per thread, membership
  // of v in every N(u), u ∈ L', by binary search
  unsigned long long key = ~0ull;
  for (uint32_t w = tid; w < W; w += kBlkThreads)
    for (uint32_t word = lpm[w]; word; word &= word - 1) {
      const uint32_t u = T.map[w * 32 + __ffs(word) - 1];
      key = min(key, ((unsigned long long)(g.off_u[u + 1] - g.off_u[u]) << 32) | u);
    }
  key = blk_min64(key, S);
  const uint32_t d0 = (uint32_t)(key >> 32), u0 = (uint32_t)key;
  if (d0 <= rlen) return d0 == rlen;  // |Γ(L')| <= deg(u*)
  const uint32_t* n0 = g.adj_u + g.off_u[u0];
  uint32_t c = 0;
  for (uint32_t b = tid; b < d0; b += kBlkThreads) {
    const uint32_t v = __ldg(n0 + b);
    bool all = true;
    for (uint32_t w = 0; w < W && all; w++)
      for (uint32_t word = lpm[w]; word && all; word &= word - 1) {
        const uint32_t u = T.map[w * 32 + __ffs(word) - 1];
        if (u != u0) all = bsearch_rank(g.adj_u + g.off_u[u], g.off_u[u + 1] - g.off_u[u], v);
      }
    c += all;
  }
  return blk_sum32(c, S) == rlen;
}

// Generate the child of `par` via its candidate i into `ch` with the whole block (Alg 2 L6-16).
// Returns 0 non-maximal, 1 maximal leaf, 2 maximal with C' != ∅ (ch holds its record).
__device__ int blk_gen_child(const Params& P, const TaskCtx& T, uint32_t* par, uint32_t i, uint32_t* ch, Acc& A,
                             BlkSmem& S) {
  const uint32_t tid = threadIdx.x, W = T.W, E = T.E;
  const uint32_t nC = par[0];
  uint32_t* pent = par + kHdr + T.W4;
  uint32_t* cent = ch + kHdr + T.W4;
  const uint32_t* vrow = pent + (size_t)i * E;
  const uint32_t vid = vrow[W];
  // L' = L_p ∩ N(v')   (Alg 2 L8)
  uint32_t lpart = 0;
  for (uint32_t w = tid; w < W; w += kBlkThreads) {
    const uint32_t x = par[kHdr + w] & vrow[w];
    ch[kHdr + w] = x;
    lpart += __popc(x);
  }
  const uint32_t lc = blk_sum32(lpart, S);  // (its barrier also publishes L')
  const uint32_t* lpm = ch + kHdr;
  // later candidates (Alg 2 L9-13): one thread per entry; Thm 4.1 marks pruned entries in place
  uint32_t nCc = 0, r_abs = 0;
  unsigned long long sr_abs = 0, later_k = 0;
  const uint32_t rl_base = par[5] + 1;
  for (uint32_t base = i + 1; base < nC; base += kBlkThreads) {
    const uint32_t j = base + tid;
    uint32_t* ej = pent + (size_t)j * E;
    bool in = j < nC;
    uint32_t cnt = 0, id = 0, kp = 0;
    if (in) {
      kp = ej[W + 1];
      in = kp != kPruned;  // removed from C_p by an earlier sibling's Thm 4.1 test
    }
    if (in) {
      for (uint32_t w = 0; w < W; w++) cnt += __popc(ej[w] & lpm[w]);
      id = ej[W];
      later_k += kp;
    }
    const bool absorb = in && cnt == lc;
    const bool cand = in && cnt > 0 && cnt < lc;
    if (absorb) sr_abs += P.g.hv[id];
    uint32_t pos[3], tot[3];
    blk_scan3(absorb, cand, false, pos, tot, S);
    if (T.rlist && absorb) T.rlist[rl_base + r_abs + pos[0]] = id;
    if (cand) {
      uint32_t* ce = cent + (size_t)(nCc + pos[1]) * E;
      for (uint32_t w = 0; w < W; w++) ce[w] = ej[w] & lpm[w];
      ce[W] = id;
      ce[W + 1] = cnt;
    }
    if (in && P.prune && cnt == kp) ej[W + 1] = kPruned;  // Thm 4.1: later siblings skip it
    r_abs += tot[0];
    nCc += tot[1];
  }
  later_k = blk_sum64(later_k, S);
  const unsigned long long sra = blk_sum64(sr_abs, S);
  const uint32_t rlen = par[5] + 1 + r_abs;
  if (tid < 32) {  // (warp 0 holds the block's counters, one per lane)
    A.add(kAcNodes, 1);
    A.add(kAcAbytes, 4ull * (lc + later_k));
  }
  if (!blk_gamma_is_r(P, T, lpm, lc, rlen, S)) {
    if (tid < 32) A.add(kAcNonmax, 1);
    return 0;
  }
  // Output(L', R') (Alg 2 L15)
  unsigned long long sl = 0;
  for (uint32_t w = tid; w < W; w += kBlkThreads)
    for (uint32_t word = lpm[w]; word; word &= word - 1) sl += hash_u(P, T.map[w * 32 + __ffs(word) - 1]);
  sl = blk_sum64(sl, S);
  const unsigned long long par_sr = ((unsigned long long)par[7] << 32) | par[6];
  const unsigned long long sr = par_sr + P.g.hv[vid] + sra;
  if (tid < 32) {
    A.add(kAcCount, 1);
    A.add(kAcChecksum, pair_hash(P, sl, sr));
  }
  if (tid == 0) {
    if (P.per_root) atomicAdd(P.per_root + T.root, 1ull);
    if (T.rlist) T.rlist[par[5]] = vid;
  }
  if (T.rlist) {
    __syncthreads();
    if ((P.out_ids || P.sring) && tid < 32) write_record(P, lpm, W, T.map, nullptr, lc, T.rlist, rlen);
  }
  if (nCc == 0) return 1;
  if (tid == 0) {
    ch[0] = nCc;
    ch[1] = 0;
    ch[2] = lc;
    ch[3] = 0;
    ch[5] = rlen;
    ch[6] = (uint32_t)sr;
    ch[7] = (uint32_t)(sr >> 32);
  }
  __syncthreads();
  return 2;
}

// depth-first walk of a root's subtree by the whole block (no splitting)
__device__ void blk_run_task(const Params& P, const TaskCtx& T, uint32_t* top, uint32_t* stack_lo,
                             uint32_t* stack_hi, Acc& A, BlkSmem& S) {
  const uint32_t tid = threadIdx.x;
  uint32_t* cur = top;
  uint32_t* sp = stack_lo;
  const uint32_t E = T.E;
  while (true) {
    __syncthreads();
    // next unpruned candidate of cur (Alg 2 L6)
    uint32_t i = cur[3];
    const uint32_t nC = cur[0];
    const uint32_t* pent = cur + kHdr + T.W4;
    while (i < nC && pent[(size_t)i * E + T.W + 1] == kPruned) i++;
    if (i >= nC) {  // pop (Alg 2 L4)
      if (cur == top) break;
      sp = cur;
      const uint32_t po = cur[4];
      cur = po == kNone ? top : stack_lo + po;
      continue;
    }
    __syncthreads();
    if (tid == 0) cur[3] = i + 1;
    const uint64_t need = kHdr + T.W4 + (uint64_t)(nC - i - 1) * E + 16;
    if (sp + need > stack_hi) {
      if (tid == 0) atomicOr(&P.ctrl->error, kErrArena);
      return;
    }
    uint32_t* ch = sp;
    const int r = blk_gen_child(P, T, cur, i, ch, A, S);
    if (r == 2) {  // push (Alg 2 L16)
      if (tid == 0) {
        ch[4] = (cur == top) ? kNone : (uint32_t)(cur - stack_lo);
        ch[3] = 0;
      }
      cur = ch;
      sp = align4(ch + kHdr + T.W4 + (size_t)ch[0] * E);  // (ch[0] published by blk_gen_child's barrier)
    }
  }
}

__global__ void __launch_bounds__(kBlkThreads, 1) k_enum_block(const Params P) {
  __shared__ BlkSmem S;
  const uint32_t tid = threadIdx.x, lane = lane_id();
  const uint32_t gw = blockIdx.x * kWpb;  // the arena of the block's first warp
  uint32_t* base = P.arena + (uint64_t)gw * P.arena_words;
  WarpMem M;
  M.keys = base;
  M.vals = (unsigned long long*)(base + P.tmax);
  M.bits = base + 3ull * P.tmax;
  M.occ = M.bits + P.bmax;
  M.dyn = align4(M.occ + P.omax);
  M.dyn_end = base + P.arena_words;
  M.rbuf = P.rbuf ? P.rbuf + (uint64_t)gw * P.rbuf_words : nullptr;
  M.sm_sort = S.sort;
  M.skeys = S.tkeys;
  M.svals = S.tvals;
  M.socc = S.tocc;
  for (uint32_t j = tid; j < kSmemTable; j += kBlkThreads) {
    M.skeys[j] = GMBE_EMPTY;
    M.svals[j] = 0;
  }
  __syncthreads();
  Acc A;  // the block's counters: held (and updated) by warp 0, one per lane, flushed at exit
  A.v = 0;
#ifdef GMBE_PROFILE
  for (int k = 0; k < 16; k++) A.ph[k] = 0;
  A.t0 = 0;
#endif
  while (true) {
    if (tid == 0) {
      const unsigned long long t =
          P.shared_cursor ? atomicAdd_system(P.shared_cursor, 1ull) : atomicAdd(&P.ctrl->root_cursor.v, 1ull);
      S.bc[0] = t < P.n_roots ? P.issue[t] : kNone;
    }
    __syncthreads();
    const uint32_t rk = S.bc[0];
    __syncthreads();
    if (rk == kNone) break;
    const unsigned long long g0 = P.timeline ? globaltimer() : 0, n0 = tid < 32 ? A.get(kAcNodes) : 0;
    const long long c0 = P.per_root_cycles ? clock64() : 0;
    if (tid < 32) {  // Alg 3: the root node, built by warp 0 with k_enum's code
      TaskCtx Tc;
      uint32_t* top = nullptr;
      uint32_t* lo = M.dyn;
      const uint32_t lb = P.g.off_v[rk];
      const bool has = run_root(P, rk, lb, P.g.off_v[rk + 1] - lb, M, A, Tc, &top, &lo);
      if (lane == 0) {
        S.T = Tc;
        S.top = has ? top : nullptr;
        S.lo = lo;
      }
      __syncwarp();
    }
    __syncthreads();
    if (S.top) {
      const TaskCtx T = S.T;
      blk_run_task(P, T, S.top, S.lo, M.dyn_end, A, S);
    }
    __syncthreads();
    const unsigned long long nn = tid < 32 ? A.get(kAcNodes) - n0 : 0;
    if (tid == 0) {
      if (P.timeline)
        timeline_rec(P, 0, rk, g0, tl_info(nn, P.g.off_v[rk + 1] - P.g.off_v[rk], 0));
      if (P.per_root_cycles) atomicAdd(P.per_root_cycles + rk, (unsigned long long)(clock64() - c0));
    }
  }
  if (tid < kAcN) atomicAdd(&P.ctrl->count + tid, A.v);  // warp 0: one counter per lane
}
