// host_core.h -- pure-integer host side of the hot path (no CUDA).
//
//   region analyzer: declared affine taps x partition box ->
//     canonical byte ranges.  Replaces the paper's polyhedral access maps
//     (§4.1) and generated enumerators (§6.1-6.2).
//   validity tracker (a3/a7): sorted disjoint segments -> mask of holders.
//     Generalises the paper's B-tree of segments -> owner (§8.1).
#pragma once

#include <cstdint>
#include <string>
#include <vector>

#include "pk_api.h"

namespace pk {

struct Range {
    uint64_t b, e;  // [b, e) bytes
};
using RangeList = std::vector<Range>;

struct Status {
    int code = PK_OK;
    std::string msg;
    bool ok() const { return code == PK_OK; }
    static Status Ok() { return {}; }
    static Status Err(int c, std::string m) { return Status{c, std::move(m)}; }
};

// int64 checked arithmetic (reading Q12; the paper ignores overflow).
bool mul_ok(int64_t a, int64_t b, int64_t* out);
bool add_ok(int64_t a, int64_t b, int64_t* out);

struct EvalEnv {
    const int64_t* scalars;
    int nscalars;
    int32_t block[3];
};

Status eval_expr(const pk_expr& e, const EvalEnv& env, int64_t* out);

struct Iv {
    int64_t lo, hi;  // [lo, hi)
};

// Index set of one array dimension of one tap over a partition (see pk_dim_map
// in pk_api.h).  box6 = (zmin,zmax,ymin,ymax,xmin,xmax).
Status dim_index_set(const pk_dim_map& dm, const int64_t box6[6], int64_t shape_k,
                     const EvalEnv& env, std::vector<Iv>* out);

// Canonical byte ranges of one tap (product of its dim index sets, row-major
// linearisation; rows whose trailing dims are full collapse into one range).
Status tap_ranges(const pk_affine_access& tap, const int64_t box6[6], int ndim,
                  const int64_t* shape, int64_t elem_bytes, const EvalEnv& env,
                  RangeList* out);

// Sort + merge overlapping/adjacent ranges in place (canonical form).
void canonicalize(RangeList* r);
// Union of canonical lists.
RangeList union_ranges(const RangeList& a, const RangeList& b);
uint64_t total_bytes(const RangeList& r);

// ---------------------------------------------------------------- tracker
struct Seg {
    uint64_t b, e;
    uint64_t mask;
};

class Tracker {
public:
    void init(uint64_t size, uint64_t mask);
    uint64_t size() const { return size_; }
    const std::vector<Seg>& segments() const { return segs_; }
    void set_segments(const std::vector<Seg>& s) { segs_ = s; }  // restore a memoised state
    uint64_t fingerprint() const {                                 // FNV-1a over the segments
        uint64_t h = 1469598103934665603ull;
        for (const Seg& s : segs_)
            for (uint64_t v : {s.b, s.e, s.mask}) { h ^= v; h *= 1099511628211ull; }
        return h;
    }
    // Visit the pieces of [b,e) with their masks, in order.
    template <class F>
    void query(uint64_t b, uint64_t e, F&& f) const;
    // mask := f(mask) on every byte of the canonical list `r`; re-coalesces.
    template <class F>
    void apply(const RangeList& r, F&& f);
    void assign(const RangeList& r, uint64_t mask) {
        apply(r, [mask](uint64_t) { return mask; });
    }
    void add_bit(const RangeList& r, int p) {
        const uint64_t bit = 1ull << p;
        apply(r, [bit](uint64_t m) { return m | bit; });
    }

private:
    size_t first_overlapping(uint64_t b) const;
    uint64_t size_ = 0;
    std::vector<Seg> segs_;
};

inline size_t Tracker::first_overlapping(uint64_t b) const {
    size_t lo = 0, hi = segs_.size();
    while (lo < hi) {  // first seg with e > b
        size_t mid = (lo + hi) / 2;
        if (segs_[mid].e <= b) lo = mid + 1; else hi = mid;
    }
    return lo;
}

template <class F>
void Tracker::query(uint64_t b, uint64_t e, F&& f) const {
    for (size_t i = first_overlapping(b); i < segs_.size() && segs_[i].b < e; ++i) {
        uint64_t lo = segs_[i].b > b ? segs_[i].b : b;
        uint64_t hi = segs_[i].e < e ? segs_[i].e : e;
        if (lo < hi) f(lo, hi, segs_[i].mask);
    }
}

template <class F>
void Tracker::apply(const RangeList& r, F&& f) {
    if (r.empty()) return;
    std::vector<Seg> out;
    out.reserve(segs_.size() + 2 * r.size() + 2);
    auto push = [&out](uint64_t b, uint64_t e, uint64_t m) {
        if (b >= e) return;
        if (!out.empty() && out.back().e == b && out.back().mask == m) out.back().e = e;
        else out.push_back(Seg{b, e, m});
    };
    size_t ri = 0;
    for (const Seg& s : segs_) {
        uint64_t cur = s.b;
        while (ri < r.size() && r[ri].e <= cur) ++ri;
        size_t rj = ri;
        while (cur < s.e) {
            if (rj >= r.size() || r[rj].b >= s.e) { push(cur, s.e, s.mask); cur = s.e; break; }
            uint64_t rb = r[rj].b > cur ? r[rj].b : cur;
            if (rb > cur) { push(cur, rb, s.mask); cur = rb; }
            uint64_t re = r[rj].e < s.e ? r[rj].e : s.e;
            push(cur, re, f(s.mask));
            cur = re;
            if (r[rj].e <= s.e) ++rj;
        }
    }
    segs_.swap(out);
}

}  // namespace pk
