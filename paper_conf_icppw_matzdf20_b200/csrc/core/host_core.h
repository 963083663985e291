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
#include <memory>
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
RangeList intersect_ranges(const RangeList& a, const RangeList& b);  // a, b canonical
uint64_t total_bytes(const RangeList& r);

// ---------------------------------------------------------------- tracker
struct Seg {
    uint64_t b, e;
    uint64_t mask;
    bool operator==(const Seg& o) const { return b == o.b && e == o.e && mask == o.mask; }
};

// Segment vectors are immutable and shared: a memoised state (graph replay) is
// restored by pointer, and every mutation builds a fresh vector (copy-on-write).
using SegVec = std::vector<Seg>;
using SegState = std::shared_ptr<const SegVec>;

class Tracker {
public:
    void init(uint64_t size, uint64_t mask);
    uint64_t size() const { return size_; }
    const SegVec& segments() const { return *segs_; }
    SegState state() const { return segs_; }
    void set_state(SegState s, uint64_t fp) {  // restore a memoised state in O(1)
        segs_ = std::move(s);
        fp_ = fp;
        fp_valid_ = true;
    }
    uint64_t fingerprint() const {  // FNV-1a over the segments, cached until the next mutation
        if (!fp_valid_) {
            uint64_t h = 1469598103934665603ull;
            for (const Seg& s : *segs_)
                for (uint64_t v : {s.b, s.e, s.mask}) { h ^= v; h *= 1099511628211ull; }
            fp_ = h;
            fp_valid_ = true;
        }
        return fp_;
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
    SegState segs_ = std::make_shared<const SegVec>();
    mutable uint64_t fp_ = 0;
    mutable bool fp_valid_ = false;
};

inline size_t Tracker::first_overlapping(uint64_t b) const {
    const SegVec& sg = *segs_;
    size_t lo = 0, hi = sg.size();
    while (lo < hi) {  // first seg with e > b
        size_t mid = (lo + hi) / 2;
        if (sg[mid].e <= b) lo = mid + 1; else hi = mid;
    }
    return lo;
}

template <class F>
void Tracker::query(uint64_t b, uint64_t e, F&& f) const {
    const SegVec& sg = *segs_;
    for (size_t i = first_overlapping(b); i < sg.size() && sg[i].b < e; ++i) {
        uint64_t lo = sg[i].b > b ? sg[i].b : b;
        uint64_t hi = sg[i].e < e ? sg[i].e : e;
        if (lo < hi) f(lo, hi, sg[i].mask);
    }
}

template <class F>
void Tracker::apply(const RangeList& r, F&& f) {
    if (r.empty()) return;
    SegVec out;
    out.reserve(segs_->size() + 2 * r.size() + 2);
    auto push = [&out](uint64_t b, uint64_t e, uint64_t m) {
        if (b >= e) return;
        if (!out.empty() && out.back().e == b && out.back().mask == m) out.back().e = e;
        else out.push_back(Seg{b, e, m});
    };
    size_t ri = 0;
    for (const Seg& s : *segs_) {
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
    segs_ = std::make_shared<const SegVec>(std::move(out));
    fp_valid_ = false;
}

}  // namespace pk
