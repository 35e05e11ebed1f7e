// gmbe_internal.cuh -- shared definitions of the sm_100a MBE library (not part of the C ABI).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>

#include "../../include/gmbe.h"

#define GMBE_FULL 0xffffffffu
#define GMBE_EMPTY 0xffffffffu

// Device-resident graph in the library's orientation (V = the smaller side).
// V vertices are identified by their RANK in the global vertex order (ascending degree, ties by
// id); U vertices keep their id on the library's U side.
struct DevGraph {
  uint32_t n_u, n_v;        // library orientation
  uint64_t m;               // unique edges
  uint32_t swapped;         // library U == caller V
  const uint32_t* off_v;    // [n_v+1]  CSR of V by rank
  const uint32_t* adj_v;    // [m]      u ids, ascending
  const uint32_t* off_u;    // [n_u+1]  CSR of U
  const uint32_t* adj_u;    // [m]      v ranks, ascending
  const uint32_t* rank2id;  // [n_v]    rank -> id on the library's V side (== caller id of that side)
  const unsigned long long* hv;  // [n_v] checksum hash of each V vertex by rank (caller roles)
  const uint32_t* issue;    // [n_v]    ranks by wedges descending: the root issue order (schedule only)
  uint32_t delta_u, delta_v, wedge_bound;  // wedge_bound = max_v Σ_{u∈N(v)} |N(u)|
  uint64_t rec_bound;  // max_v wedges(v) * entry stride(|N(v)|): bound on a root node record (words)
};

struct gmbe_graph {
  int device;
  cudaStream_t stream;
  bool own_stream;
  uint32_t caller_n_u, caller_n_v;
  uint32_t order;
  DevGraph g;
  // owned device buffers
  void* bufs[8];
  int nbufs;
};

// count of this library's own kernel launches (gmbe_api.cu)
void gmbe_note_launch();

// thread-local error plumbing (gmbe_api.cu)
int gmbe_set_error(int code, const std::string& msg);
#define GMBE_CUDA_TRY(expr)                                                              \
  do {                                                                                   \
    cudaError_t _e = (expr);                                                             \
    if (_e != cudaSuccess)                                                               \
      return gmbe_set_error(_e == cudaErrorMemoryAllocation ? GMBE_ENOMEM : GMBE_ECUDA,  \
                            std::string(#expr) + ": " + cudaGetErrorString(_e));         \
  } while (0)

// Checksum spec, device side.  Written independently of oracle/.
__host__ __device__ __forceinline__ unsigned long long gmbe_mix64(unsigned long long x) {
  x ^= x >> 30;
  x *= 0xBF58476D1CE4E5B9ULL;
  x ^= x >> 27;
  x *= 0x94D049BB133111EBULL;
  x ^= x >> 31;
  return x;
}
// hash of a caller id on side `side` (0 = caller U, 1 = caller V)
__host__ __device__ __forceinline__ unsigned long long gmbe_hid(uint32_t id, uint32_t side) {
  return gmbe_mix64(2ull * id + side + 0x9E3779B97F4A7C15ULL);
}
__host__ __device__ __forceinline__ unsigned long long gmbe_pair_hash(unsigned long long s_caller_u,
                                                                      unsigned long long s_caller_v) {
  return gmbe_mix64(s_caller_u + 0xD6E8FEB86659FD93ULL * gmbe_mix64(s_caller_v));
}
