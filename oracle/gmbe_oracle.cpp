// gmbe_oracle.cpp -- plain, single-threaded CPU oracle for maximal biclique enumeration (MBE).
//
// *** TEST INFRASTRUCTURE ONLY. ***  Only tests/, __graft_entry__.smoke() and bench.py's
// cpu_baseline / --impl reference legs may load this library.  It shares NO code, header,
// table or constant generator with the CUDA path (paper_conf_sc_panhlzwc23_b200/csrc), and it
// never reads anything the CUDA path produced.
//
// What it computes (PAPER.md = /root/reference/PAPER.md, cited as P:<line>):
//   * The set of maximal bicliques of G(U,V,E): pairs (L,R), L in U, R in V, both non-empty,
//     every u in L adjacent to every v in R, not contained in a larger biclique.
//     Empty-side pairs are excluded (Fig 1 counts 6 for G0; reading A1).
//   * count and checksum = sum over bicliques of h(L,R) mod 2^64, h as frozen in DESIGN.md
//     ("Checksum"), over the CALLER's original ids and roles.
//   * Work counters of the canonical tree (degree order + Thm 4.1, no split): nodes, nonmax,
//     algo_bytes, algo_bytes_qfull, and algo_bytes_cand = the wedge + candidate terms alone
//     (DESIGN.md "Algorithmic bytes").
//
// How: the textbook set-enumeration tree of Alg 1 with an explicit excluded set Q
// (P:377-380), first level = Alg 3 root tasks with the root check "v_s is the
// earliest vertex of R_s" (Alg 3 L7), and optional pro-active pruning by local neighbourhood
// size (Thm 4.1).  Readings of the garbled / silent spots are DESIGN.md A1-A18.
// Sets are sorted std::vector<uint32_t>; no blocking, no fusion, no bit tricks.
//
// Parity pins (tests/test_oracle.py): literal brute force over all subsets of V (|V|<=16),
// restricted brute force on ER(40,40,.15) (211 bicliques), the paper's G0 (6 bicliques, Fig 1/2,
// Ex 2.1, Fig 5 tree), closed forms (crown 2^n-2, K_ab 1, matching n, star 1, empty 0),
// Galois closure of every emitted pair, and invariance under relabelling / transposition /
// order / prune.
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <pthread.h>
#include <time.h>
#include <vector>

namespace {

// ---- checksum spec (written independently of the CUDA side) ----
uint64_t splitmix_finalize(uint64_t x) {
  x ^= x >> 30;
  x *= 0xBF58476D1CE4E5B9ULL;
  x ^= x >> 27;
  x *= 0x94D049BB133111EBULL;
  x ^= x >> 31;
  return x;
}
uint64_t hash_caller_u(uint64_t u) { return splitmix_finalize(2 * u + 0x9E3779B97F4A7C15ULL); }
uint64_t hash_caller_v(uint64_t v) { return splitmix_finalize(2 * v + 1 + 0x9E3779B97F4A7C15ULL); }
uint64_t biclique_hash(uint64_t sum_l, uint64_t sum_r) {
  return splitmix_finalize(sum_l + 0xD6E8FEB86659FD93ULL * splitmix_finalize(sum_r));
}

typedef std::vector<uint32_t> Set;  // always sorted ascending

// |A ∩ B| for sorted A, B.
uint64_t intersection_size(const Set& a, const Set& b) {
  const Set& small = a.size() <= b.size() ? a : b;
  const Set& large = a.size() <= b.size() ? b : a;
  uint64_t n = 0;
  for (uint32_t x : small)
    if (std::binary_search(large.begin(), large.end(), x)) n++;
  return n;
}

// A ∩ B for sorted A, B.
Set intersection(const Set& a, const Set& b) {
  Set out;
  std::set_intersection(a.begin(), a.end(), b.begin(), b.end(), std::back_inserter(out));
  return out;
}

struct Options {
  int order;  // 0 = ascending degree, 1 = identity
  int prune;  // Thm 4.1
  uint32_t shard_i, shard_n;
  int check_closure;
  uint64_t* rec_offsets;
  uint64_t rec_cap;
  uint32_t* rec_ids;
  uint64_t ids_cap;
  uint64_t* per_root_count;
  const uint8_t* root_mask;  // optional: run only the roots v (internal V id) with root_mask[v] != 0
  uint64_t* per_root_ns;     // optional: wall-clock ns spent on each root (internal V id)
};

struct Result {
  uint64_t count, checksum, roots_run, nodes, nonmax, algo_bytes, algo_bytes_qfull;
  uint64_t n_written, ids_written, truncated, closure_failures, algo_bytes_cand;
};

struct Oracle {
  // Internal orientation: V is the side with fewer vertices; on a tie keep the
  // caller's orientation (reading A11).
  bool swapped;
  uint32_t nU, nV;
  std::vector<Set> NV;  // N(v), v in internal V: internal U ids ascending
  std::vector<Set> NU;  // N(u), u in internal U: internal V ids ascending
  std::vector<uint32_t> rank;  // position of v in the global vertex order
  Options opt;
  Result res;
  uint32_t current_root;

  // hashes of internal ids, in the caller's roles
  uint64_t hash_internal_u(uint32_t u) const { return swapped ? hash_caller_v(u) : hash_caller_u(u); }
  uint64_t hash_internal_v(uint32_t v) const { return swapped ? hash_caller_u(v) : hash_caller_v(v); }

  bool rank_less(uint32_t a, uint32_t b) const { return rank[a] < rank[b]; }

  // Gamma(R) = ∩_{v in R} N(v) and Gamma(L) = ∩_{u in L} N(u)
  Set gamma_of_r(const Set& r) const {
    Set g = NV[r[0]];
    for (size_t i = 1; i < r.size(); i++) g = intersection(g, NV[r[i]]);
    return g;
  }
  Set gamma_of_l(const Set& l) const {
    Set g = NU[l[0]];
    for (size_t i = 1; i < l.size(); i++) g = intersection(g, NU[l[i]]);
    return g;
  }

  // Output(L, R) (Alg 1 L10, Alg 2 L15).  R arrives in rank order; sort it by id here.
  void emit(const Set& l, const std::vector<uint32_t>& r_in) {
    Set r = r_in;
    std::sort(r.begin(), r.end());
    if (opt.check_closure) {
      if (gamma_of_r(r) != l || gamma_of_l(l) != r) res.closure_failures++;
    }
    uint64_t sl = 0, sr = 0;
    for (uint32_t u : l) sl += hash_internal_u(u);
    for (uint32_t v : r) sr += hash_internal_v(v);
    // caller roles: the caller's L is the internal R when the sides were swapped
    uint64_t h = swapped ? biclique_hash(sr, sl) : biclique_hash(sl, sr);
    res.count++;
    res.checksum += h;
    if (opt.per_root_count) opt.per_root_count[current_root]++;
    if (opt.rec_offsets || opt.rec_ids) {
      const Set& cl = swapped ? r : l;  // caller U side
      const Set& cr = swapped ? l : r;  // caller V side
      uint64_t need = 2 + cl.size() + cr.size();
      if (res.n_written < opt.rec_cap && res.ids_written + need <= opt.ids_cap) {
        opt.rec_offsets[res.n_written++] = res.ids_written;
        uint32_t* p = opt.rec_ids + res.ids_written;
        p[0] = (uint32_t)cl.size();
        p[1] = (uint32_t)cr.size();
        std::copy(cl.begin(), cl.end(), p + 2);
        std::copy(cr.begin(), cr.end(), p + 2 + cl.size());
        res.ids_written += need;
      } else {
        res.truncated = 1;
      }
    }
  }

  // Alg 1 / Alg 2 node expansion with explicit Q; SURVEY 8(c) O2.
  //   l, r: the node's biclique; c: candidates in rank order; q: excluded set;
  //   kl[j] = |N(c[j]) ∩ l| (the parent's local neighbourhood sizes, Sec 4.2);
  //   kq[j] = |N(q[j]) ∩ l| (same quantity for the excluded vertices, carried along the same way).
  void search(const Set& l, const std::vector<uint32_t>& r, const std::vector<uint32_t>& c,
              const std::vector<uint32_t>& q, const std::vector<uint64_t>& kl,
              const std::vector<uint64_t>& kq) {
    std::vector<char> pruned(c.size(), 0);
    for (size_t i = 0; i < c.size(); i++) {
      if (pruned[i]) continue;
      uint32_t vp = c[i];
      // Alg 2 L8: L' = L_p ∩ N(v')
      Set lp = intersection(l, NV[vp]);
      res.nodes++;
      // "later" = untraversed candidates after v', taken before this step's marking (A6)
      std::vector<size_t> later;
      for (size_t j = i + 1; j < c.size(); j++)
        if (!pruned[j]) later.push_back(j);
      // Alg 2 L9-13: local neighbourhood sizes w.r.t. L'
      std::vector<uint64_t> kp(c.size(), 0);
      for (size_t j : later) kp[j] = intersection_size(NV[c[j]], lp);
      // Thm 4.1: |N_L(c)| unchanged from parent p to this child => prune c from C_p
      // for the later siblings.  Applied whether or not this child is maximal (A6).
      if (opt.prune)
        for (size_t j : later)
          if (kp[j] == kl[j]) pruned[j] = 1;
      // Q' = (Q ∪ traversed earlier siblings) restricted to vertices touching L' (A7)
      std::vector<uint32_t> qset = q;
      std::vector<uint64_t> kqset = kq;  // kqset[j] = |N(qset[j]) ∩ l|
      for (size_t j = 0; j < i; j++)
        if (!pruned[j]) qset.push_back(c[j]), kqset.push_back(kl[j]);
      // algorithmic bytes of this node: 4*(|L'| + sum_later k_p + sum_{Q, k_p>=|L'|} k_p)
      uint64_t words = lp.size();
      for (size_t j : later) words += kl[j];
      uint64_t qwords = 0, qwords_full = 0;
      for (uint64_t kx : kqset) {
        qwords_full += kx;
        if (kx >= lp.size()) qwords += kx;
      }
      res.algo_bytes += 4 * (words + qwords);
      res.algo_bytes_qfull += 4 * (words + qwords_full);
      res.algo_bytes_cand += 4 * words;
      // Maximality check (Alg 2 L14 "R' == Gamma(L')"): non-maximal iff some excluded vertex is
      // adjacent to all of L'.  The subtree of a non-maximal node is skipped (A3).
      std::vector<uint32_t> qnext;
      std::vector<uint64_t> kqnext;
      bool maximal = true;
      for (uint32_t x : qset) {
        uint64_t kx = intersection_size(NV[x], lp);
        if (kx == lp.size()) maximal = false;
        if (kx > 0) qnext.push_back(x), kqnext.push_back(kx);
      }
      if (!maximal) {
        res.nonmax++;
        continue;
      }
      // Alg 2 L10-13: absorb full-neighbourhood candidates into R', partial ones into C'
      std::vector<uint32_t> rnext = r;
      rnext.push_back(vp);
      std::vector<uint32_t> cnext;
      std::vector<uint64_t> knext;
      for (size_t j : later) {
        if (kp[j] == lp.size()) {
          rnext.push_back(c[j]);
        } else if (kp[j] > 0) {
          cnext.push_back(c[j]);
          knext.push_back(kp[j]);
        }
      }
      emit(lp, rnext);
      if (!cnext.empty()) search(lp, rnext, cnext, qnext, knext, kqnext);
    }
  }

  // First level of the tree = Alg 3 tasks (Alg 4 L6-13): one per v_s in V.
  void run_root(uint32_t vs) {
    const Set& l = NV[vs];
    if (l.empty()) return;  // isolated vertices are in no biclique (A17)
    current_root = vs;
    // wedge bytes of the root (counted for every non-isolated root, skipped or not)
    uint64_t wedge_words = l.size();
    for (uint32_t u : l) wedge_words += NU[u].size();
    res.algo_bytes += 4 * wedge_words;
    res.algo_bytes_qfull += 4 * wedge_words;
    res.algo_bytes_cand += 4 * wedge_words;
    // N2(v_s) = ∪_{u in N(v_s)} N(u) - {v_s}
    Set n2;
    for (uint32_t u : l) n2.insert(n2.end(), NU[u].begin(), NU[u].end());
    std::sort(n2.begin(), n2.end());
    n2.erase(std::unique(n2.begin(), n2.end()), n2.end());
    std::vector<uint32_t> r{vs}, c, q;
    std::vector<uint64_t> kq;
    for (uint32_t vc : n2) {
      if (vc == vs) continue;
      uint64_t k = intersection_size(NV[vc], l);
      if (k == l.size()) {
        // Alg 3 L3-4 / L7: v_c joins R_s; v_s must be the earliest vertex of R_s, else skip (A2)
        if (rank_less(vc, vs)) return;
        r.push_back(vc);
      } else if (rank_less(vs, vc)) {
        c.push_back(vc);  // Alg 3 L5-6: later-ordered partial neighbour -> candidate
      } else {
        q.push_back(vc);  // earlier-ordered partial neighbour -> excluded set
        kq.push_back(k);
      }
    }
    res.roots_run++;
    std::sort(c.begin(), c.end(), [this](uint32_t a, uint32_t b) { return rank_less(a, b); });
    std::vector<uint64_t> k;
    for (uint32_t vc : c) k.push_back(intersection_size(NV[vc], l));
    emit(l, r);  // the root's own biclique (A5)
    if (!c.empty()) search(l, r, c, q, k, kq);
  }

  void run() {
    std::vector<uint32_t> by_rank(nV);
    for (uint32_t v = 0; v < nV; v++) by_rank[rank[v]] = v;
    for (uint32_t rk = 0; rk < nV; rk++) {
      const uint32_t v = by_rank[rk];
      if (rk % opt.shard_n != opt.shard_i) continue;
      if (opt.root_mask && !opt.root_mask[v]) continue;
      if (opt.per_root_ns) {
        timespec t0, t1;
        clock_gettime(CLOCK_MONOTONIC, &t0);
        run_root(v);
        clock_gettime(CLOCK_MONOTONIC, &t1);
        opt.per_root_ns[v] += (uint64_t)((t1.tv_sec - t0.tv_sec) * 1000000000LL + (t1.tv_nsec - t0.tv_nsec));
      } else {
        run_root(v);
      }
    }
  }
};

struct ThreadArgs {
  Oracle* o;
};
void* thread_main(void* p) {
  ((ThreadArgs*)p)->o->run();
  return nullptr;
}

}  // namespace

extern "C" {

typedef struct {
  uint64_t count, checksum, roots_run, nodes, nonmax, algo_bytes, algo_bytes_qfull;
  uint64_t n_written, ids_written, truncated, closure_failures, algo_bytes_cand;
} oracle_result;

// Returns 0 on success, -1 on invalid arguments.
// edges: n_edges (u,v) pairs interleaved, caller ids.  Duplicates collapse.
// order: 0 ascending degree (ties: ascending id, reading A8), 1 identity.
// per_root_count (optional): indexed by the internal-V id of the root (caller's V id unless the
//   sides were swapped, in which case the caller's U id).
// root_mask (optional, same indexing): enumerate only the roots with root_mask[v] != 0 (a root
//   sample for timing; like shards, masks partition the output).  per_root_ns (optional, same
//   indexing): wall-clock nanoseconds spent on each root's tree (timing only).
int oracle_mbe(uint32_t n_u, uint32_t n_v, const uint32_t* edges, uint64_t n_edges, int order,
               int prune, uint32_t shard_i, uint32_t shard_n, int check_closure,
               uint64_t* rec_offsets, uint64_t rec_cap, uint32_t* rec_ids, uint64_t ids_cap,
               uint64_t* per_root_count, const uint8_t* root_mask, uint64_t* per_root_ns,
               oracle_result* out) {
  if (!out || shard_n == 0 || shard_i >= shard_n || (n_edges && !edges)) return -1;
  for (uint64_t e = 0; e < n_edges; e++)
    if (edges[2 * e] >= n_u || edges[2 * e + 1] >= n_v) return -1;
  Oracle o;
  o.swapped = n_u < n_v;
  o.nU = o.swapped ? n_v : n_u;
  o.nV = o.swapped ? n_u : n_v;
  o.NV.assign(o.nV, Set());
  o.NU.assign(o.nU, Set());
  for (uint64_t e = 0; e < n_edges; e++) {
    uint32_t u = edges[2 * e], v = edges[2 * e + 1];
    if (o.swapped) std::swap(u, v);
    o.NV[v].push_back(u);
    o.NU[u].push_back(v);
  }
  for (Set& s : o.NV) {
    std::sort(s.begin(), s.end());
    s.erase(std::unique(s.begin(), s.end()), s.end());
  }
  for (Set& s : o.NU) {
    std::sort(s.begin(), s.end());
    s.erase(std::unique(s.begin(), s.end()), s.end());
  }
  // vertex order: ascending |N(v)|, ties by id (A8) -- or identity
  std::vector<uint32_t> by_rank(o.nV);
  for (uint32_t v = 0; v < o.nV; v++) by_rank[v] = v;
  if (order == 0)
    std::stable_sort(by_rank.begin(), by_rank.end(),
                     [&o](uint32_t a, uint32_t b) { return o.NV[a].size() < o.NV[b].size(); });
  o.rank.assign(o.nV, 0);
  for (uint32_t r = 0; r < o.nV; r++) o.rank[by_rank[r]] = r;
  o.opt = Options{order, prune, shard_i, shard_n, check_closure, rec_offsets, rec_cap,
                  rec_ids, ids_cap, per_root_count, root_mask, per_root_ns};
  if (!rec_offsets || !rec_ids) o.opt.rec_offsets = nullptr, o.opt.rec_ids = nullptr;
  std::memset(&o.res, 0, sizeof(o.res));
  // recursion depth <= min(|L|,|C|) <= Delta(V): run on a thread with a large stack
  pthread_attr_t attr;
  pthread_attr_init(&attr);
  pthread_attr_setstacksize(&attr, (size_t)1 << 30);
  pthread_t th;
  ThreadArgs args{&o};
  if (pthread_create(&th, &attr, thread_main, &args) != 0) {
    o.run();
  } else {
    pthread_join(th, nullptr);
  }
  pthread_attr_destroy(&attr);
  std::memcpy(out, &o.res, sizeof(oracle_result));
  return 0;
}

}  // extern "C"
