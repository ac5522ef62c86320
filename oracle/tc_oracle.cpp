// tc_oracle.cpp — CPU ORACLE for exact triangle counting.  TEST INFRASTRUCTURE.
//
// Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / reference
// leg may load this library.  It shares no code, header, table or helper with
// the CUDA path (paper_conf_ipps_li0ptz24_b200/csrc); the only common input is
// the seeded edge list from tcgen/.
//
// What it computes: T(G) = |{ {x,y,z} : xy, yz, xz in E }|
// for the simple undirected graph G obtained from the raw pair list by
// ignoring direction, dropping self-loops and merging duplicates (PAPER.md
// "removing vertices that are not connected to any edges, eliminating
// self-loop edges, and resolving duplicate edges ... do not alter the number
// of triangles").  ITC is exact, so the oracle is that definition
// evaluated by the plain node-iterator / Forward algorithm the paper cites as
// Polak's CPU ancestor (refs [13, 18]):
//
//   1. canonicalise every pair to (min, max), drop a == b, sort + unique
//   2. deg[x] = undirected degree after cleaning
//   3. orient x -> y iff (deg x, x) < (deg y, y)   [no relabelling]
//   4. each out-list N+(x) sorted ascending by id
//   5. T = sum_x sum_{y in N+(x)} |N+(x) ∩ N+(y)| via std::set_intersection
//      over FULL rows (no suffix trick, no hints, no hashing)
//
// Step 3 is the only reading the paper leaves open (C-1/C-3 in DESIGN.md):
// each triangle {x,y,z} with x<y<z in the chosen total order is counted once,
// at edge x->y with witness z.  The `order` argument exists so tests can pin
// that T does not depend on the order (id order, hashed order).
//
// Parity pins (tests/test_oracle_pins.py): closed forms (K_n = C(n,3),
// bipartite / trees / grids = 0, wheel, friendship, K_{a,b,c} = abc, Turán),
// the karate club = 45 (tests/golden), trace(A^3)/6 and sum(A∘(L·U))/2
// by brute force on random tiny graphs, and invariance under the P:287 cleaning.
#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdint>
#include <cstring>
#include <thread>
#include <vector>

namespace {

struct CountingIterator {  // output iterator that only counts assignments
  uint64_t* c;
  CountingIterator& operator*() { return *this; }
  CountingIterator& operator=(int32_t) { return *this; }
  CountingIterator& operator++() { ++*c; return *this; }
  CountingIterator operator++(int) { ++*c; return *this; }
};

inline uint64_t splitmix(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

double ms_since(std::chrono::steady_clock::time_point t0) {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
}

}  // namespace

extern "C" {

typedef struct {
  uint64_t triangles;           // T (over the counted rows; all rows unless sampling)
  int64_t m;                    // unique undirected edges after cleaning
  int64_t n_active;             // vertices with degree > 0
  int64_t max_out_degree;       // max |N+(x)|
  uint64_t merge_steps_total;   // sum over oriented edges x->y of |N+(x)| + |N+(y)|
  uint64_t merge_steps_counted; // the same over the rows actually counted
  double build_ms;              // steps 1-4
  double count_ms;              // step 5
  int32_t threads;              // worker threads used in step 5
  int32_t sampled;              // 1 when sample_stride > 1
} tco_result;

struct tco_graph {
  int64_t n = 0, m = 0, n_active = 0, max_out = 0;
  std::vector<int64_t> off;  // row offsets of the oriented lists
  std::vector<int32_t> adj;  // N+(x), ascending by id
  double build_ms = 0;
};

// Steps 1-4.  Returns NULL on invalid argument (an id < 0 or >= n, null
// pointer).  n < 0 means "max id + 1".  order: 0 = (degree, id), 1 = id,
// 2 = (hash(id), id).
tco_graph* tco_build(const int32_t* src, const int32_t* dst, int64_t num_pairs, int64_t n,
                     int order) {
  if (num_pairs < 0 || (num_pairs > 0 && (!src || !dst))) return nullptr;
  auto t0 = std::chrono::steady_clock::now();
  if (n < 0) {
    int64_t mx = -1;
    for (int64_t i = 0; i < num_pairs; ++i) mx = std::max<int64_t>(mx, std::max(src[i], dst[i]));
    n = mx + 1;
  }
  // 1. canonicalise, drop self-loops, sort + unique
  std::vector<uint64_t> keys;
  keys.reserve(num_pairs);
  for (int64_t i = 0; i < num_pairs; ++i) {
    int64_t a = src[i], b = dst[i];
    if (a < 0 || b < 0 || a >= n || b >= n) return nullptr;
    if (a == b) continue;
    uint64_t lo = (uint64_t)std::min(a, b), hi = (uint64_t)std::max(a, b);
    keys.push_back((lo << 32) | hi);
  }
  std::sort(keys.begin(), keys.end());
  keys.erase(std::unique(keys.begin(), keys.end()), keys.end());
  const int64_t m = (int64_t)keys.size();
  // 2. undirected degree
  std::vector<int64_t> deg(n, 0);
  for (uint64_t k : keys) {
    ++deg[k >> 32];
    ++deg[k & 0xffffffffu];
  }
  // 3. orientation
  auto before = [&](int64_t x, int64_t y) -> bool {
    if (order == 1) return x < y;
    if (order == 2) {
      uint64_t hx = splitmix((uint64_t)x), hy = splitmix((uint64_t)y);
      return hx != hy ? hx < hy : x < y;
    }
    return deg[x] != deg[y] ? deg[x] < deg[y] : x < y;
  };
  tco_graph* g = new tco_graph();
  std::vector<int64_t>& off = g->off;
  off.assign(n + 1, 0);
  for (uint64_t k : keys) {
    int64_t a = (int64_t)(k >> 32), b = (int64_t)(k & 0xffffffffu);
    ++off[(before(a, b) ? a : b) + 1];
  }
  for (int64_t x = 0; x < n; ++x) off[x + 1] += off[x];
  std::vector<int32_t>& adj = g->adj;
  adj.resize(m);
  {
    std::vector<int64_t> fill(off.begin(), off.end() - 1);
    for (uint64_t k : keys) {
      int64_t a = (int64_t)(k >> 32), b = (int64_t)(k & 0xffffffffu);
      if (before(a, b)) adj[fill[a]++] = (int32_t)b; else adj[fill[b]++] = (int32_t)a;
    }
  }
  // 4. rows ascending by id
  int64_t max_out = 0, n_active = 0;
  for (int64_t x = 0; x < n; ++x) {
    std::sort(adj.begin() + off[x], adj.begin() + off[x + 1]);
    max_out = std::max(max_out, off[x + 1] - off[x]);
    n_active += deg[x] > 0;
  }
  g->n = n;
  g->m = m;
  g->n_active = n_active;
  g->max_out = max_out;
  g->build_ms = ms_since(t0);
  return g;
}

void tco_free(tco_graph* g) { delete g; }

// Step 5 over the rows x with x % sample_stride == sample_offset (all rows
// when sample_stride <= 1).  threads <= 0 means hardware_concurrency().
int tco_count_rows(const tco_graph* g, int threads, int64_t sample_stride, int64_t sample_offset,
                   tco_result* out) {
  if (!g || !out) return 1;
  std::memset(out, 0, sizeof(*out));
  const int64_t n = g->n;
  const int64_t* off = g->off.data();
  const int32_t* adj = g->adj.data();
  // 5. T = sum over oriented edges of |N+(x) ∩ N+(y)|, rows in dynamic chunks
  auto t1 = std::chrono::steady_clock::now();
  int nt = threads > 0 ? threads : (int)std::thread::hardware_concurrency();
  if (nt < 1) nt = 1;
  const int64_t chunk = 1024;
  std::atomic<int64_t> next{0};
  std::vector<uint64_t> part_t(nt, 0), part_steps(nt, 0), part_all(nt, 0);
  auto worker = [&](int w) {
    uint64_t t = 0, steps = 0, all = 0;
    for (;;) {
      int64_t b = next.fetch_add(chunk);
      if (b >= n) break;
      int64_t e = std::min(n, b + chunk);
      for (int64_t x = b; x < e; ++x) {
        const int32_t* xb = adj + off[x];
        const int32_t* xe = adj + off[x + 1];
        bool counted = sample_stride <= 1 || x % sample_stride == sample_offset;
        for (const int32_t* p = xb; p != xe; ++p) {
          const int32_t* yb = adj + off[*p];
          const int32_t* ye = adj + off[*p + 1];
          uint64_t s = (uint64_t)(xe - xb) + (uint64_t)(ye - yb);
          all += s;
          if (!counted) continue;
          steps += s;
          uint64_t c = 0;
          std::set_intersection(xb, xe, yb, ye, CountingIterator{&c});
          t += c;
        }
      }
    }
    part_t[w] = t;
    part_steps[w] = steps;
    part_all[w] = all;
  };
  std::vector<std::thread> pool;
  for (int w = 0; w < nt; ++w) pool.emplace_back(worker, w);
  for (auto& th : pool) th.join();
  for (int w = 0; w < nt; ++w) {
    out->triangles += part_t[w];
    out->merge_steps_counted += part_steps[w];
    out->merge_steps_total += part_all[w];
  }
  out->count_ms = ms_since(t1);
  out->build_ms = g->build_ms;
  out->m = g->m;
  out->n_active = g->n_active;
  out->max_out_degree = g->max_out;
  out->threads = nt;
  out->sampled = sample_stride > 1;
  return 0;
}

// ---------------------------------------------------------------------------
// Per-edge support: for every edge {a,b} of the
// cleaned simple graph, sup(a,b) = the number of triangles that contain it =
// |N(a) ∩ N(b)| over the FULL undirected neighbourhoods (a triangle {a,b,w}
// is exactly a common neighbour w; Fig. 1(b) computes the same wSet for
// one edge).  This is the definition written out: no orientation, no suffix,
// no hashing.  The k-truss / clustering-coefficient applications P:39 names
// consume these values.  Pins: tests/test_oracle_pins.py (closed forms such as
// K_n -> n-2, wheel spokes 2 / rim 1, friendship 1; (A·A)∘A by brute force;
// sum = 3T).
struct tco_support_graph {
  int64_t n = 0, m = 0;
  std::vector<uint64_t> keys;  // canonical (min << 32 | max), ascending = edge order
  std::vector<int64_t> off;    // undirected CSR offsets
  std::vector<int32_t> adj;    // N(x), ascending
};

// Steps 1-2 of tco_build plus the undirected adjacency.  NULL on invalid input.
tco_support_graph* tco_support_build(const int32_t* src, const int32_t* dst, int64_t num_pairs,
                                     int64_t n) {
  if (num_pairs < 0 || (num_pairs > 0 && (!src || !dst))) return nullptr;
  if (n < 0) {
    int64_t mx = -1;
    for (int64_t i = 0; i < num_pairs; ++i) mx = std::max<int64_t>(mx, std::max(src[i], dst[i]));
    n = mx + 1;
  }
  tco_support_graph* g = new tco_support_graph();
  std::vector<uint64_t>& keys = g->keys;
  keys.reserve(num_pairs);
  for (int64_t i = 0; i < num_pairs; ++i) {
    int64_t a = src[i], b = dst[i];
    if (a < 0 || b < 0 || a >= n || b >= n) {
      delete g;
      return nullptr;
    }
    if (a == b) continue;  // self-loops do not take part in triangles
    uint64_t lo = (uint64_t)std::min(a, b), hi = (uint64_t)std::max(a, b);
    keys.push_back((lo << 32) | hi);
  }
  std::sort(keys.begin(), keys.end());
  keys.erase(std::unique(keys.begin(), keys.end()), keys.end());  // merge duplicates
  g->n = n;
  g->m = (int64_t)keys.size();
  g->off.assign(n + 1, 0);
  for (uint64_t k : keys) {
    ++g->off[(k >> 32) + 1];
    ++g->off[(k & 0xffffffffu) + 1];
  }
  for (int64_t x = 0; x < n; ++x) g->off[x + 1] += g->off[x];
  g->adj.resize(2 * g->m);
  std::vector<int64_t> fill(g->off.begin(), g->off.end() - 1);
  for (uint64_t k : keys) {  // keys ascending -> each N(x) is filled in ascending order
    int64_t a = (int64_t)(k >> 32), b = (int64_t)(k & 0xffffffffu);
    g->adj[fill[a]++] = (int32_t)b;
  }
  for (uint64_t k : keys) {
    int64_t a = (int64_t)(k >> 32), b = (int64_t)(k & 0xffffffffu);
    g->adj[fill[b]++] = (int32_t)a;
  }
  for (int64_t x = 0; x < n; ++x) std::sort(g->adj.begin() + g->off[x], g->adj.begin() + g->off[x + 1]);
  return g;
}

int64_t tco_support_m(const tco_support_graph* g) { return g ? g->m : -1; }

void tco_support_free(tco_support_graph* g) { delete g; }

// |N(a) ∩ N(b)| for one pair (the support if {a,b} is an edge).
static uint64_t common_neighbours(const tco_support_graph* g, int64_t a, int64_t b) {
  uint64_t c = 0;
  std::set_intersection(g->adj.begin() + g->off[a], g->adj.begin() + g->off[a + 1],
                        g->adj.begin() + g->off[b], g->adj.begin() + g->off[b + 1],
                        CountingIterator{&c});
  return c;
}

// All edges: out_a/out_b/out_sup (length m) in ascending (a, b), a < b.
int tco_support_all(const tco_support_graph* g, int threads, int32_t* out_a, int32_t* out_b,
                    uint32_t* out_sup) {
  if (!g || (g->m > 0 && (!out_a || !out_b || !out_sup))) return 1;
  int nt = threads > 0 ? threads : (int)std::thread::hardware_concurrency();
  if (nt < 1) nt = 1;
  std::atomic<int64_t> next{0};
  const int64_t chunk = 4096;
  auto worker = [&]() {
    for (;;) {
      int64_t b0 = next.fetch_add(chunk);
      if (b0 >= g->m) break;
      for (int64_t i = b0; i < std::min(g->m, b0 + chunk); ++i) {
        const int64_t a = (int64_t)(g->keys[i] >> 32), b = (int64_t)(g->keys[i] & 0xffffffffu);
        out_a[i] = (int32_t)a;
        out_b[i] = (int32_t)b;
        out_sup[i] = (uint32_t)common_neighbours(g, a, b);
      }
    }
  };
  std::vector<std::thread> pool;
  for (int w = 0; w < nt; ++w) pool.emplace_back(worker);
  for (auto& th : pool) th.join();
  return 0;
}

// Sampled pairs (any a, b): out[i] = |N(a_i) ∩ N(b_i)| if {a_i, b_i} is an
// edge, else -1.  Lets a test check sampled outputs at full size.
int tco_support_pairs(const tco_support_graph* g, const int32_t* a, const int32_t* b, int64_t k,
                      int64_t* out) {
  if (!g || (k > 0 && (!a || !b || !out))) return 1;
  for (int64_t i = 0; i < k; ++i) {
    int64_t x = std::min(a[i], b[i]), y = std::max(a[i], b[i]);
    if (x < 0 || y >= g->n || x == y) {
      out[i] = -1;
      continue;
    }
    const uint64_t key = ((uint64_t)x << 32) | (uint64_t)y;
    if (!std::binary_search(g->keys.begin(), g->keys.end(), key)) {
      out[i] = -1;
      continue;
    }
    out[i] = (int64_t)common_neighbours(g, x, y);
  }
  return 0;
}

// Steps 1-5 in one call.  Returns 0 on success, 1 on invalid argument.
// sample_stride > 1 counts only rows x with x % sample_stride == 0.
int tco_count(const int32_t* src, const int32_t* dst, int64_t num_pairs, int64_t n, int order,
              int threads, int64_t sample_stride, tco_result* out) {
  if (!out) return 1;
  std::memset(out, 0, sizeof(*out));
  tco_graph* g = tco_build(src, dst, num_pairs, n, order);
  if (!g) return 1;
  int rc = tco_count_rows(g, threads, sample_stride, 0, out);
  tco_free(g);
  return rc;
}

}  // extern "C"
