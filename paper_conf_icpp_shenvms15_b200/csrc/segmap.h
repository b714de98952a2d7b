// Interval map over [0, n): disjoint segments, each carrying a value.
// Used by the planner for the ownership directory (D7), last-writer tracking
// (DP-Perf / DP-Dep dependency chains) and cross-stream hazard tracking.
#pragma once

#include <cstdint>
#include <iterator>
#include <map>

namespace mm {

template <class T>
class SegMap {
 public:
  struct Seg { int64_t hi; T v; };

  void reset(int64_t n, const T& v) {
    m_.clear();
    n_ = n;
    if (n > 0) m_.emplace(0, Seg{n, v});
  }
  int64_t size() const { return n_; }

  // Calls f(lo, hi, T&) for each segment piece inside [lo, hi), splitting the
  // boundary segments so that f may modify the value of exactly that piece.
  template <class F>
  void modify(int64_t lo, int64_t hi, F f) {
    if (lo >= hi) return;
    split(lo);
    split(hi);
    for (auto it = m_.find(lo); it != m_.end() && it->first < hi; ++it)
      f(it->first, it->second.hi, it->second.v);
    merge_around(lo, hi);
  }

  // Read-only walk over [lo, hi) (values clipped to the window).
  template <class F>
  void visit(int64_t lo, int64_t hi, F f) const {
    if (lo >= hi || m_.empty()) return;
    auto it = m_.upper_bound(lo);
    if (it != m_.begin()) --it;
    for (; it != m_.end() && it->first < hi; ++it) {
      int64_t a = it->first > lo ? it->first : lo;
      int64_t b = it->second.hi < hi ? it->second.hi : hi;
      if (a < b) f(a, b, it->second.v);
    }
  }

  void assign(int64_t lo, int64_t hi, const T& v) {
    if (lo >= hi) return;
    split(lo);
    split(hi);
    auto it = m_.find(lo);
    while (it != m_.end() && it->first < hi) it = m_.erase(it);
    m_.emplace(lo, Seg{hi, v});
    merge_around(lo, hi);
  }

  size_t segments() const { return m_.size(); }

 private:
  void split(int64_t x) {
    if (x <= 0 || x >= n_) return;
    auto it = m_.upper_bound(x);
    if (it == m_.begin()) return;
    --it;
    if (it->first == x || it->second.hi <= x) return;
    Seg right{it->second.hi, it->second.v};
    it->second.hi = x;
    m_.emplace(x, right);
  }
  void merge_around(int64_t lo, int64_t hi) {
    auto it = m_.upper_bound(lo);
    if (it != m_.begin()) --it;
    if (it != m_.begin()) --it;
    while (it != m_.end() && it->first <= hi) {
      auto nx = std::next(it);
      if (nx != m_.end() && it->second.hi == nx->first && it->second.v == nx->second.v) {
        it->second.hi = nx->second.hi;
        m_.erase(nx);
      } else {
        it = nx;
      }
    }
  }
  std::map<int64_t, Seg> m_;
  int64_t n_ = 0;
};

}  // namespace mm
