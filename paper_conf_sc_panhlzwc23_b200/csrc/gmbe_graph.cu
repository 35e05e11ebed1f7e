// gmbe_graph.cu -- device graph build (DESIGN.md steps a1-a2; Sec 5 "Pre-processing",
// P:1014-1025, and multi-edge removal).
//
//   a1  edge ingest -> validate ids -> orient (V := smaller side) -> pack (u<<bv|v)
//       -> radix sort -> first-copy flags + their scan (dedupe without a host round trip)
//   a2  degrees -> global vertex order (ascending degree, ties by id)
//       -> CSR of V by rank (u ascending) and CSR of U (ranks ascending) by two stable partial-key
//       sorts -> Δ(U), Δ(V), wedge bound (>= Δ2(V)) -> per-rank checksum hash table; one host
//       synchronisation at the very end.
// Sorting / scanning / selection use CUB (library primitives); everything else is our kernels.
#include <cub/cub.cuh>

#include <cstring>
#include <vector>

#include "gmbe_internal.cuh"

namespace {

// a1: validate, orient and pack one edge per key: (u << bv) | v, bv = bits of the library's V ids
__global__ void k_pack_edges(const uint32_t* __restrict__ e, uint64_t m, uint32_t n_u, uint32_t n_v,
                             uint32_t swapped, uint32_t bv, unsigned long long* __restrict__ keys,
                             uint32_t* __restrict__ bad) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m;
       i += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t u = e[2 * i], v = e[2 * i + 1];
    if (u >= n_u || v >= n_v) {
      *bad = 1;
      u = 0;
      v = 0;
    }
    if (swapped) {
      uint32_t t = u;
      u = v;
      v = t;
    }
    keys[i] = ((unsigned long long)u << bv) | v;
  }
}

// a1 dedupe on the (u, v)-sorted keys: flag[i] = first copy of its edge; degrees of
// the unique edges (a2)
__global__ void k_unique_degrees(const unsigned long long* __restrict__ keys, uint64_t m, uint32_t bv,
                                 uint32_t* __restrict__ flag, uint32_t* __restrict__ deg_u,
                                 uint32_t* __restrict__ deg_v) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const unsigned long long k = keys[i];
    const bool first = i == 0 || keys[i - 1] != k;
    flag[i] = first;
    if (first) {
      atomicAdd(&deg_u[k >> bv], 1u);
      atomicAdd(&deg_v[(uint32_t)(k & ((1ull << bv) - 1))], 1u);
    }
  }
}

// sort keys of the global vertex order: (deg << bv) | v -- ascending degree, ties by id (A8)
__global__ void k_order_keys(const uint32_t* __restrict__ deg_v, uint32_t n_v, uint32_t identity, uint32_t bv,
                             unsigned long long* __restrict__ out) {
  for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n_v; v += gridDim.x * blockDim.x)
    out[v] = identity ? (unsigned long long)v : (((unsigned long long)deg_v[v] << bv) | v);
}

__global__ void k_rank_maps(const unsigned long long* __restrict__ sorted, uint32_t n_v, uint32_t bv,
                            uint32_t side_v, uint32_t* __restrict__ rank2id,
                            uint32_t* __restrict__ id2rank, const uint32_t* __restrict__ deg_v,
                            uint32_t* __restrict__ deg_by_rank, unsigned long long* __restrict__ hv) {
  for (uint32_t r = blockIdx.x * blockDim.x + threadIdx.x; r < n_v; r += gridDim.x * blockDim.x) {
    const uint32_t id = (uint32_t)(sorted[r] & ((1ull << bv) - 1));
    rank2id[r] = id;
    id2rank[id] = r;
    deg_by_rank[r] = deg_v[id];
    hv[r] = gmbe_hid(id, side_v);
  }
}

// unique edges in (u, v) order -> (rank(v), u) pairs at their deduplicated position (the exclusive
// scan of the flags); positions [m, m0) get the sentinel key n_v, which every later sort keeps last
__global__ void k_rank_pairs(const unsigned long long* __restrict__ keys, const uint32_t* __restrict__ flag,
                             const uint32_t* __restrict__ pos, uint64_t m0, uint32_t bv,
                             const uint32_t* __restrict__ id2rank, uint32_t n_u, uint32_t n_v,
                             uint32_t* __restrict__ pk, uint32_t* __restrict__ pv, uint32_t* __restrict__ m_out) {
  const uint32_t m = m0 ? pos[m0 - 1] + flag[m0 - 1] : 0u;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m0;
       i += (uint64_t)gridDim.x * blockDim.x) {
    if (flag[i]) {
      const unsigned long long k = keys[i];
      pk[pos[i]] = id2rank[(uint32_t)(k & ((1ull << bv) - 1))];
      pv[pos[i]] = (uint32_t)(k >> bv);
    }
    if (i >= m) {
      pk[i] = n_v;
      pv[i] = n_u;
    }
    if (i == 0) *m_out = m;
  }
}

// one warp per V rank: wedge count Σ_{u∈N(v)} |N(u)| and the maxima.
__global__ void k_issue(const unsigned long long* __restrict__ keys, uint32_t n, uint32_t* __restrict__ issue) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    issue[i] = ~(uint32_t)keys[i];
}

// one warp per V rank: wedge count Σ_{u∈N(v)} |N(u)| (the issue key) and the maxima.  The maxima are
// reduced per block first (one atomic per block and quantity: a per-rank atomic on four addresses
// serialises millions of atomics on light-root graphs).
__global__ void k_bounds(const uint32_t* __restrict__ off_v, const uint32_t* __restrict__ adj_v,
                         const uint32_t* __restrict__ off_u, uint32_t n_v, uint32_t n_u,
                         uint32_t* __restrict__ maxes /* [0]=Δ(V) [1]=Δ(U) [2]=wedge bound */,
                         unsigned long long* __restrict__ rec_bound, unsigned long long* __restrict__ cost_key) {
  __shared__ unsigned long long red[4][32];
  const uint32_t lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
  uint32_t mdv = 0, mdu = 0, mw = 0;
  unsigned long long mrec = 0;
  for (uint32_t r = warp; r < n_v; r += nw) {
    const uint32_t b = off_v[r], e = off_v[r + 1];
    unsigned long long s = 0;
    for (uint32_t i = b + lane; i < e; i += 32) {
      const uint32_t u = adj_v[i];
      s += off_u[u + 1] - off_u[u];
    }
    for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(GMBE_FULL, s, o);
    // issue key: wedges descending, then rank descending (ascending sort of the complements)
    const uint32_t w = (uint32_t)(s > 0xffffffffull ? 0xffffffffull : s);
    if (lane == 0) cost_key[r] = ((unsigned long long)(~w) << 32) | (~r);
    mdv = max(mdv, e - b);
    mw = max(mw, w);
    // root record: <= s candidates, each row of ceil(deg/32) words + id + k, padded to 4
    const unsigned long long stride = (((e - b) + 31) / 32 + 2 + 3) & ~3ull;
    mrec = max(mrec, s * stride);
  }
  for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < n_u; u += gridDim.x * blockDim.x)
    mdu = max(mdu, off_u[u + 1] - off_u[u]);
  for (int o = 16; o; o >>= 1) {
    mdv = max(mdv, __shfl_xor_sync(GMBE_FULL, mdv, o));
    mdu = max(mdu, __shfl_xor_sync(GMBE_FULL, mdu, o));
    mw = max(mw, __shfl_xor_sync(GMBE_FULL, mw, o));
    mrec = max(mrec, (unsigned long long)__shfl_xor_sync(GMBE_FULL, mrec, o));
  }
  if (lane == 0) {
    red[0][wib] = mdv;
    red[1][wib] = mdu;
    red[2][wib] = mw;
    red[3][wib] = mrec;
  }
  __syncthreads();
  if (threadIdx.x < 4) {
    unsigned long long m = 0;
    for (uint32_t k = 0; k < blockDim.x / 32; k++) m = max(m, red[threadIdx.x][k]);
    if (threadIdx.x == 3) atomicMax(rec_bound, m);
    else atomicMax(&maxes[threadIdx.x == 0 ? 0 : (threadIdx.x == 1 ? 1 : 2)], (uint32_t)m);
  }
}

// stream-ordered allocations from the device's default pool (cheap to repeat per step)
struct Tmp {
  cudaStream_t s;
  std::vector<void*> p;
  explicit Tmp(cudaStream_t st) : s(st) {}
  ~Tmp() { free_all(); }
  void free_all() {
    for (void* x : p)
      if (x) cudaFreeAsync(x, s);
    p.clear();
  }
  template <class T>
  cudaError_t alloc(T** out, size_t n) {
    void* q = nullptr;
    cudaError_t e = cudaMallocAsync(&q, n ? n * sizeof(T) : 16, s);
    if (e == cudaSuccess) p.push_back(q);
    *out = (T*)q;
    return e;
  }
  void release(void* q) {  // hand ownership to the caller
    for (auto& x : p)
      if (x == q) x = nullptr;
  }
};

int grid_for(uint64_t n) {
  uint64_t b = (n + 255) / 256;
  if (b < 1) b = 1;
  if (b > 148 * 32) b = 148 * 32;
  return (int)b;
}

cudaError_t radix_sort(Tmp& t, unsigned long long* in, unsigned long long* out, uint64_t n, int end_bit,
                       cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  size_t bytes = 0;
  cudaError_t e = cub::DeviceRadixSort::SortKeys(nullptr, bytes, in, out, (int)n, 0, end_bit, s);
  if (e != cudaSuccess) return e;
  void* tmp;
  e = t.alloc((char**)&tmp, bytes);
  if (e != cudaSuccess) return e;
  return cub::DeviceRadixSort::SortKeys(tmp, bytes, in, out, (int)n, 0, end_bit, s);
}

// stable LSD sort of (key, value) pairs on the low end_bit bits of the keys
cudaError_t radix_sort_pairs(Tmp& t, const uint32_t* kin, uint32_t* kout, const uint32_t* vin, uint32_t* vout,
                             uint64_t n, int end_bit, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  size_t bytes = 0;
  cudaError_t e = cub::DeviceRadixSort::SortPairs(nullptr, bytes, kin, kout, vin, vout, (int)n, 0, end_bit, s);
  if (e != cudaSuccess) return e;
  void* tmp;
  e = t.alloc((char**)&tmp, bytes);
  if (e != cudaSuccess) return e;
  return cub::DeviceRadixSort::SortPairs(tmp, bytes, kin, kout, vin, vout, (int)n, 0, end_bit, s);
}

cudaError_t excl_scan(Tmp& t, const uint32_t* in, uint32_t* out, uint64_t n, cudaStream_t s) {
  size_t bytes = 0;
  cudaError_t e = cub::DeviceScan::ExclusiveSum(nullptr, bytes, in, out, (int)n, s);
  if (e != cudaSuccess) return e;
  void* tmp;
  e = t.alloc((char**)&tmp, bytes);
  if (e != cudaSuccess) return e;
  return cub::DeviceScan::ExclusiveSum(tmp, bytes, in, out, (int)n, s);
}

int bits_for(uint64_t x) {
  int b = 1;
  while (b < 64 && (1ull << b) <= x) b++;
  return b;
}

}  // namespace

extern "C" int gmbe_load_bipartite(uint32_t n_u, uint32_t n_v, const uint32_t* edges_uv,
                                   uint64_t n_edges, const gmbe_load_opts* opts, gmbe_graph** out) {
  if (!out) return gmbe_set_error(GMBE_EINVAL, "gmbe_load_bipartite: out is NULL");
  *out = nullptr;
  if (n_edges && !edges_uv) return gmbe_set_error(GMBE_EINVAL, "gmbe_load_bipartite: edges is NULL");
  // CUB's sorts / selects take int item counts: keep every count below 2^31
  if (n_edges >= (1ull << 31) || n_u >= (1u << 31) || n_v >= (1u << 31))
    return gmbe_set_error(GMBE_EUNSUPPORTED, "gmbe_load_bipartite: n_edges >= 2^31 or |U|,|V| >= 2^31");
  gmbe_load_opts o{};
  o.device = -1;
  if (opts) {
    if (opts->struct_size && opts->struct_size < sizeof(uint32_t) * 2)
      return gmbe_set_error(GMBE_EINVAL, "gmbe_load_bipartite: bad struct_size");
    o = *opts;
  }
  if (o.order > 1) return gmbe_set_error(GMBE_EINVAL, "gmbe_load_bipartite: bad order");
  int dev = o.device;
  if (dev < 0) GMBE_CUDA_TRY(cudaGetDevice(&dev));
  GMBE_CUDA_TRY(cudaSetDevice(dev));
  cudaStream_t s = (cudaStream_t)o.cuda_stream;
  bool own = false;
  if (!s) {
    GMBE_CUDA_TRY(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    own = true;
  }
  {
    // keep freed pool memory cached across calls instead of returning it at every sync
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
      uint64_t thr = ~0ull;
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
  }
  gmbe_graph* G = new gmbe_graph();
  G->device = dev;
  G->stream = s;
  G->own_stream = own;
  G->caller_n_u = n_u;
  G->caller_n_v = n_v;
  G->order = o.order;
  G->nbufs = 0;
  Tmp t(s);
  auto fail = [&](int rc) {
    t.free_all();
    for (int i = 0; i < G->nbufs; i++) cudaFreeAsync(G->bufs[i], s);
    cudaStreamSynchronize(s);
    if (own) cudaStreamDestroy(s);
    delete G;
    return rc;
  };
#define TRY(expr)                                                                           \
  do {                                                                                      \
    cudaError_t _e = (expr);                                                                \
    if (_e != cudaSuccess)                                                                  \
      return fail(gmbe_set_error(_e == cudaErrorMemoryAllocation ? GMBE_ENOMEM : GMBE_ECUDA, \
                                 std::string(#expr) + ": " + cudaGetErrorString(_e)));     \
  } while (0)

  const uint32_t swapped = n_u < n_v ? 1u : 0u;
  const uint32_t NU = swapped ? n_v : n_u, NV = swapped ? n_u : n_v;
  const uint64_t m0 = n_edges;
  const int bu = bits_for(NU), bv = bits_for(NV);  // NU / NV themselves fit (the sentinels below)
  // Host-visible results of the build, read back by the call's ONE host synchronisation at the end:
  // [0] bad id, [1] unique edges m, [2..4] Δ(V), Δ(U), wedge bound, [6..7] root-record bound (u64)
  uint32_t* d_res;
  TRY(t.alloc(&d_res, 8));
  TRY(cudaMemsetAsync(d_res, 0, 8 * sizeof(uint32_t), s));
  uint32_t* maxes = d_res + 2;
  unsigned long long* d_recb = (unsigned long long*)(d_res + 6);
  // a1: ingest -> (u << bv | v) keys -> sort -> dedupe flags (no host round trip: duplicates stay
  // in place, flagged, and are squeezed out by the scatter below)
  const uint32_t* d_e = edges_uv;
  if (m0 && !o.edges_on_device) {
    uint32_t* tmp;
    TRY(t.alloc(&tmp, 2 * m0));
    TRY(cudaMemcpyAsync(tmp, edges_uv, 2 * m0 * sizeof(uint32_t), cudaMemcpyHostToDevice, s));
    d_e = tmp;
  }
  unsigned long long *keys, *keys2;
  TRY(t.alloc(&keys, m0));
  TRY(t.alloc(&keys2, m0));
  if (m0) k_pack_edges<<<grid_for(m0), 256, 0, s>>>(d_e, m0, n_u, n_v, swapped, bv, keys, d_res), gmbe_note_launch();
  TRY(cudaGetLastError());
  TRY(radix_sort(t, keys, keys2, m0, bu + bv, s));
  // a2: degrees of the unique edges and the global order
  uint32_t *deg_u, *deg_v, *deg_by_rank, *id2rank, *flag, *pos;
  TRY(t.alloc(&deg_u, NU + 1));
  TRY(t.alloc(&deg_v, NV + 1));
  TRY(t.alloc(&deg_by_rank, NV + 1));
  TRY(t.alloc(&id2rank, NV + 1));
  TRY(t.alloc(&flag, m0));
  TRY(t.alloc(&pos, m0));
  TRY(cudaMemsetAsync(deg_u, 0, (NU + 1) * sizeof(uint32_t), s));
  TRY(cudaMemsetAsync(deg_v, 0, (NV + 1) * sizeof(uint32_t), s));
  TRY(cudaMemsetAsync(deg_by_rank, 0, (NV + 1) * sizeof(uint32_t), s));
  if (m0) k_unique_degrees<<<grid_for(m0), 256, 0, s>>>(keys2, m0, bv, flag, deg_u, deg_v), gmbe_note_launch();
  if (m0) TRY(excl_scan(t, flag, pos, m0, s));
  unsigned long long *okeys, *okeys2;
  TRY(t.alloc(&okeys, NV));
  TRY(t.alloc(&okeys2, NV));
  if (NV) k_order_keys<<<grid_for(NV), 256, 0, s>>>(deg_v, NV, o.order == GMBE_ORDER_IDENTITY, bv, okeys), gmbe_note_launch();
  TRY(radix_sort(t, okeys, okeys2, NV, bv + bits_for(m0 + 1), s));
  // persistent buffers (adjacency arrays sized m0 >= m; the tail past m holds the sentinels)
  uint32_t *off_v, *adj_v, *off_u, *adj_u, *rank2id;
  unsigned long long* hv;
  TRY(t.alloc(&off_v, NV + 1));
  TRY(t.alloc(&adj_v, m0));
  TRY(t.alloc(&off_u, NU + 1));
  TRY(t.alloc(&adj_u, m0));
  TRY(t.alloc(&rank2id, NV));
  TRY(t.alloc(&hv, NV));
  // library V side == caller V (hash side 1) unless swapped (then caller U, side 0)
  if (NV)
    k_rank_maps<<<grid_for(NV), 256, 0, s>>>(okeys2, NV, bv, swapped ? 0u : 1u, rank2id, id2rank, deg_v,
                                             deg_by_rank, hv), gmbe_note_launch();
  TRY(excl_scan(t, deg_by_rank, off_v, (uint64_t)NV + 1, s));
  TRY(excl_scan(t, deg_u, off_u, (uint64_t)NU + 1, s));
  if (m0) {
    // CSR_V (rank-major, u ascending) and CSR_U (u-major, ranks ascending) by two STABLE sorts on
    // partial keys: the unique edges arrive u-major with v ascending; sorting them by rank alone
    // keeps u ascending inside each rank; sorting that by u alone keeps ranks ascending inside each u
    uint32_t *pk, *pv, *sk;
    TRY(t.alloc(&pk, m0));
    TRY(t.alloc(&pv, m0));
    TRY(t.alloc(&sk, m0));
    k_rank_pairs<<<grid_for(m0), 256, 0, s>>>(keys2, flag, pos, m0, bv, id2rank, NU, NV, pk, pv, d_res + 1),
        gmbe_note_launch();
    TRY(radix_sort_pairs(t, pk, sk, pv, adj_v, m0, bv, s));   // (rank, u): adj_v = the u's
    TRY(radix_sort_pairs(t, adj_v, pv, sk, adj_u, m0, bu, s));  // (u, rank): adj_u = the ranks
  }
  uint32_t* issue;
  TRY(t.alloc(&issue, NV + 1));
  unsigned long long *ck, *ck2;
  TRY(t.alloc(&ck, NV + 1));
  TRY(t.alloc(&ck2, NV + 1));
  if (NV || NU) k_bounds<<<grid_for((uint64_t)NV * 32 + NU), 256, 0, s>>>(off_v, adj_v, off_u, NV, NU, maxes, d_recb, ck), gmbe_note_launch();
  TRY(cudaGetLastError());
  // root issue order: most wedges first (the schedule only; the tree is fixed by the rank order)
  TRY(radix_sort(t, ck, ck2, NV, 64, s));
  if (NV) k_issue<<<grid_for(NV), 256, 0, s>>>(ck2, NV, issue), gmbe_note_launch();
  TRY(cudaGetLastError());
  uint32_t hres[8];
  TRY(cudaMemcpyAsync(hres, d_res, sizeof(hres), cudaMemcpyDeviceToHost, s));
  TRY(cudaStreamSynchronize(s));  // the build's only host synchronisation
  if (hres[0]) return fail(gmbe_set_error(GMBE_EINVAL, "gmbe_load_bipartite: edge id out of range"));
  const uint64_t m = hres[1];
  const uint32_t* hm = hres + 2;
  unsigned long long h_recb = 0;
  std::memcpy(&h_recb, hres + 6, 8);

  void* keep[] = {off_v, adj_v, off_u, adj_u, rank2id, hv, issue};
  for (void* q : keep) {
    t.release(q);
    G->bufs[G->nbufs++] = q;
  }
  DevGraph& g = G->g;
  g.n_u = NU;
  g.n_v = NV;
  g.m = m;
  g.swapped = swapped;
  g.off_v = off_v;
  g.adj_v = adj_v;
  g.off_u = off_u;
  g.adj_u = adj_u;
  g.rank2id = rank2id;
  g.hv = hv;
  g.issue = issue;
  g.delta_v = hm[0];
  g.delta_u = hm[1];
  g.wedge_bound = hm[2];
  g.rec_bound = h_recb;
  *out = G;
  return GMBE_OK;
#undef TRY
}

extern "C" int gmbe_graph_info_get(const gmbe_graph* G, gmbe_graph_info* out) {
  if (!G || !out) return gmbe_set_error(GMBE_EINVAL, "gmbe_graph_info_get: NULL argument");
  out->n_u = G->caller_n_u;
  out->n_v = G->caller_n_v;
  out->n_edges_unique = G->g.m;
  out->delta_u = G->g.delta_u;
  out->delta_v = G->g.delta_v;
  // Σ_{u∈N(v)} (|N(u)| - 1) = wedges - |N(v)|; bounded by the max wedge count
  out->wedge_bound_v = G->g.wedge_bound;
  out->swapped = G->g.swapped;
  out->order = G->order;
  out->device = (uint32_t)G->device;
  return GMBE_OK;
}

extern "C" void gmbe_free_graph(gmbe_graph* G) {
  if (!G) return;
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(G->device);
  cudaStreamSynchronize(G->stream);
  for (int i = 0; i < G->nbufs; i++) cudaFreeAsync(G->bufs[i], G->stream);
  cudaStreamSynchronize(G->stream);
  if (G->own_stream) cudaStreamDestroy(G->stream);
  cudaSetDevice(prev);
  delete G;
}
