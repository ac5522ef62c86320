// tcgen.cpp — seeded synthetic edge-list generators (see include/tcgen.h).
//
// Input generators only: shared by the CUDA path's tests/bench and by the CPU
// oracle's tests, and holding none of the counting arithmetic.  Workload
// shapes: SURVEY.md §8(d) (configs C1..C5), Table II.
#include "tcgen.h"

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstring>
#include <thread>
#include <vector>

namespace {

int g_threads = 0;

int num_threads() {
  int t = g_threads > 0 ? g_threads : (int)std::thread::hardware_concurrency();
  return t > 0 ? t : 1;
}

// splitmix64 finaliser (Steele, Lea, Flood 2014) — the counter-based RNG.
inline uint64_t mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// One random 64-bit word per (seed, stream, counter).
inline uint64_t rng(uint64_t seed, uint64_t stream, uint64_t counter) {
  return mix64(mix64(seed * 0xD1B54A32D192ED03ull + stream) ^ counter);
}

// Run f(begin, end) over [0, n) in equal contiguous slices, one per thread.
template <class F>
void parallel_for(int64_t n, F f) {
  int t = num_threads();
  if (n < (int64_t)1 << 16 || t == 1) {
    f((int64_t)0, n);
    return;
  }
  std::vector<std::thread> pool;
  for (int i = 0; i < t; ++i) {
    int64_t b = n * i / t, e = n * (i + 1) / t;
    pool.emplace_back([=] { f(b, e); });
  }
  for (auto& th : pool) th.join();
}

// Seeded bijection of [0, 2^bits): a product of invertible steps on bits-bit
// integers (odd multiply mod 2^bits, xor-shift right, add constant).
struct LabelPerm {
  uint64_t mask, m1, m2, a1;
  int s;
  LabelPerm(uint64_t seed, int bits) {
    mask = (bits >= 64) ? ~0ull : ((1ull << bits) - 1);
    m1 = (mix64(seed ^ 0x1111) | 1ull);
    m2 = (mix64(seed ^ 0x2222) | 1ull);
    a1 = mix64(seed ^ 0x3333);
    s = bits / 2 > 0 ? bits / 2 : 1;
  }
  uint64_t operator()(uint64_t x) const {
    x = (x * m1) & mask;
    x ^= x >> s;
    x = (x + a1) & mask;
    x = (x * m2) & mask;
    x ^= x >> s;
    return x;
  }
};

}  // namespace

extern "C" {

void tcgen_set_threads(int threads) { g_threads = threads; }

int64_t tcgen_rmat(uint64_t seed, int scale, int64_t edge_factor, uint32_t thr_a,
                   uint32_t thr_ab, uint32_t thr_abc, int permute, int32_t* src,
                   int32_t* dst) {
  if (scale < 1 || scale > 31 || edge_factor < 1 || !src || !dst) return -1;
  if (!(thr_a <= thr_ab && thr_ab <= thr_abc)) return -1;
  const int64_t m = edge_factor << scale;
  LabelPerm perm(seed ^ 0xA5A5A5A5ull, scale);
  parallel_for(m, [&](int64_t b, int64_t e) {
    for (int64_t i = b; i < e; ++i) {
      uint64_t s = 0, d = 0;
      uint64_t word = 0;
      for (int l = 0; l < scale; ++l) {
        if ((l & 1) == 0) word = rng(seed, 1, ((uint64_t)i << 5) | (uint64_t)(l >> 1));
        uint32_t r = (l & 1) ? (uint32_t)(word >> 32) : (uint32_t)word;
        // quadrant: 0 = (0,0), 1 = (0,1), 2 = (1,0), 3 = (1,1)
        uint64_t sb = (r >= thr_ab) ? 1 : 0;
        uint64_t db = (r >= thr_a && r < thr_ab) || (r >= thr_abc) ? 1 : 0;
        s = (s << 1) | sb;
        d = (d << 1) | db;
      }
      if (permute) {
        s = perm(s);
        d = perm(d);
      }
      src[i] = (int32_t)s;
      dst[i] = (int32_t)d;
    }
  });
  return m;
}

int64_t tcgen_chung_lu(uint64_t seed, int64_t n, int64_t num_pairs, double gamma,
                       double w_max, int32_t* src, int32_t* dst) {
  if (n < 1 || n > 0x7fffffffLL || num_pairs < 0 || gamma <= 1.0 || w_max <= 0 || !src ||
      !dst)
    return -1;
  const double ex = -1.0 / (gamma - 1.0);
  // Solve c so that sum_i min(w_max, c (i+1)^ex) = 2 * num_pairs (bisection;
  // the sum is monotone in c).  Deterministic: sequential double arithmetic.
  std::vector<double> pw(n);
  for (int64_t i = 0; i < n; ++i) pw[i] = std::pow((double)(i + 1), ex);
  auto total = [&](double c) {
    double t = 0;
    for (int64_t i = 0; i < n; ++i) t += std::min(w_max, c * pw[i]);
    return t;
  };
  const double target = 2.0 * (double)num_pairs;
  double lo = 0, hi = 1;
  while (total(hi) < target && hi < 1e300) hi *= 2;
  for (int it = 0; it < 64; ++it) {
    double mid = 0.5 * (lo + hi);
    if (total(mid) < target) lo = mid; else hi = mid;
  }
  const double c = hi;
  // 64-bit fixed-point CDF: cdf[i] = floor(2^64 * sum_{j<=i} w_j / W), cdf[n-1] = 2^64-1.
  std::vector<double> cum(n);
  double acc = 0;
  for (int64_t i = 0; i < n; ++i) {
    acc += std::min(w_max, c * pw[i]);
    cum[i] = acc;
  }
  std::vector<uint64_t> cdf(n);
  for (int64_t i = 0; i < n; ++i) {
    long double f = (long double)cum[i] / (long double)acc;
    long double v = f * 18446744073709551616.0L;
    cdf[i] = (v >= 18446744073709551615.0L) ? ~0ull : (uint64_t)v;
  }
  cdf[n - 1] = ~0ull;
  parallel_for(num_pairs, [&](int64_t b, int64_t e) {
    for (int64_t i = b; i < e; ++i) {
      for (int side = 0; side < 2; ++side) {
        uint64_t r = rng(seed, 2, ((uint64_t)i << 1) | (uint64_t)side);
        // first index with cdf > r (r < 2^64-1 = cdf[n-1] unless r is all ones)
        int64_t k = std::upper_bound(cdf.begin(), cdf.end(), r) - cdf.begin();
        if (k >= n) k = n - 1;
        (side ? dst : src)[i] = (int32_t)k;
      }
    }
  });
  return num_pairs;
}

int64_t tcgen_lattice_capacity(int64_t side) {
  if (side < 1) return -1;
  return 2 * side * (side - 1) + (side - 1) * (side - 1);
}

int64_t tcgen_lattice(uint64_t seed, int64_t side, uint32_t thr_keep, uint32_t thr_diag,
                      int32_t* src, int32_t* dst) {
  if (side < 1 || side * side > 0x7fffffffLL || !src || !dst) return -1;
  // Candidate j in [0, cap): [0, H) horizontal, [H, 2H) vertical, [2H, cap) diagonal,
  // H = side*(side-1).  Kept when rng(seed, 3, j) (low 32 bits) < threshold.
  const int64_t H = side * (side - 1);
  const int64_t cap = tcgen_lattice_capacity(side);
  auto candidate = [&](int64_t j, int64_t* a, int64_t* b) -> bool {
    uint32_t r = (uint32_t)rng(seed, 3, (uint64_t)j);
    if (j < H) {
      int64_t row = j / (side - 1), col = j % (side - 1);
      *a = row * side + col;
      *b = *a + 1;
      return r < thr_keep;
    } else if (j < 2 * H) {
      int64_t k = j - H, row = k / side, col = k % side;
      *a = row * side + col;
      *b = *a + side;
      return r < thr_keep;
    } else {
      int64_t k = j - 2 * H, row = k / (side - 1), col = k % (side - 1);
      *a = row * side + col;
      *b = *a + side + 1;
      return r < thr_diag;
    }
  };
  int t = num_threads();
  if (cap < (int64_t)1 << 16) t = 1;
  std::vector<int64_t> counts(t + 1, 0);
  auto slice = [&](int i, int64_t* b, int64_t* e) {
    *b = cap * i / t;
    *e = cap * (i + 1) / t;
  };
  {
    std::vector<std::thread> pool;
    for (int i = 0; i < t; ++i)
      pool.emplace_back([&, i] {
        int64_t b, e, a_, b_, c = 0;
        slice(i, &b, &e);
        for (int64_t j = b; j < e; ++j) c += candidate(j, &a_, &b_);
        counts[i + 1] = c;
      });
    for (auto& th : pool) th.join();
  }
  for (int i = 0; i < t; ++i) counts[i + 1] += counts[i];
  {
    std::vector<std::thread> pool;
    for (int i = 0; i < t; ++i)
      pool.emplace_back([&, i] {
        int64_t b, e, a_, b_, o = counts[i];
        slice(i, &b, &e);
        for (int64_t j = b; j < e; ++j)
          if (candidate(j, &a_, &b_)) {
            src[o] = (int32_t)a_;
            dst[o] = (int32_t)b_;
            ++o;
          }
      });
    for (auto& th : pool) th.join();
  }
  return counts[t];
}

uint64_t tcgen_checksum(const int32_t* src, const int32_t* dst, int64_t num_pairs) {
  uint64_t h = 0xCBF29CE484222325ull;
  for (int64_t i = 0; i < num_pairs; ++i) {
    h = (h ^ (uint32_t)src[i]) * 0x100000001B3ull;
    h = (h ^ (uint32_t)dst[i]) * 0x100000001B3ull;
  }
  return h;
}

}  // extern "C"
