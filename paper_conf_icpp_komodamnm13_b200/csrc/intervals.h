// Sorted, disjoint, coalesced sets of half-open int64 intervals [lo, hi).
// Host-only data structure behind the per-region validity table (which elements of which
// replica hold the current value) — the runtime state the paper's data loader consults to
// "avoid additional data movement" (L125 §IV.C). Sizes stay O(P) per region in practice.
#pragma once
#include <algorithm>
#include <cstdint>
#include <vector>

namespace accmg {

struct Ival {
    int64_t lo, hi;
};

class IntervalSet {
public:
    IntervalSet() = default;
    IntervalSet(int64_t lo, int64_t hi) { add(lo, hi); }

    bool empty() const { return v_.empty(); }
    const std::vector<Ival>& items() const { return v_; }
    void clear() { v_.clear(); }

    int64_t total() const {
        int64_t t = 0;
        for (auto& x : v_) t += x.hi - x.lo;
        return t;
    }

    void add(int64_t lo, int64_t hi) {
        if (lo >= hi) return;
        std::vector<Ival> out;
        out.reserve(v_.size() + 1);
        size_t i = 0;
        while (i < v_.size() && v_[i].hi < lo) out.push_back(v_[i++]);
        int64_t nlo = lo, nhi = hi;
        while (i < v_.size() && v_[i].lo <= hi) {
            nlo = std::min(nlo, v_[i].lo);
            nhi = std::max(nhi, v_[i].hi);
            ++i;
        }
        out.push_back({nlo, nhi});
        while (i < v_.size()) out.push_back(v_[i++]);
        v_.swap(out);
    }
    void add(const IntervalSet& o) {
        for (auto& x : o.v_) add(x.lo, x.hi);
    }

    void subtract(int64_t lo, int64_t hi) {
        if (lo >= hi) return;
        std::vector<Ival> out;
        out.reserve(v_.size() + 1);
        for (auto& x : v_) {
            if (x.hi <= lo || x.lo >= hi) { out.push_back(x); continue; }
            if (x.lo < lo) out.push_back({x.lo, lo});
            if (x.hi > hi) out.push_back({hi, x.hi});
        }
        v_.swap(out);
    }
    void subtract(const IntervalSet& o) {
        for (auto& x : o.v_) subtract(x.lo, x.hi);
    }

    IntervalSet intersect(const IntervalSet& o) const {
        IntervalSet r;
        size_t i = 0, j = 0;
        while (i < v_.size() && j < o.v_.size()) {
            int64_t lo = std::max(v_[i].lo, o.v_[j].lo);
            int64_t hi = std::min(v_[i].hi, o.v_[j].hi);
            if (lo < hi) r.v_.push_back({lo, hi});
            if (v_[i].hi < o.v_[j].hi) ++i; else ++j;
        }
        return r;
    }

    bool overlaps(const IntervalSet& o) const { return !intersect(o).empty(); }

    bool contains(const IntervalSet& o) const {
        IntervalSet t = o;
        t.subtract(*this);
        return t.empty();
    }

private:
    std::vector<Ival> v_;
};

}  // namespace accmg
