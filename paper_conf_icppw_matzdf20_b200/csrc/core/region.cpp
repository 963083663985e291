// region.cpp -- region analyzer.
//
// The paper models each externally visible array access as a map from the
// 6-D block coordinates (blockOff, blockId; threadId projected out under
// 0 <= threadId < blockDim) to array points (§4.1), constrains its
// domain to a partition box (§6) and enumerates the image row by row
// as first/last ranges (§6.1), once per convex piece so that a union
// is not over-approximated.  Here the maps are declared, separable
// block boxes (pk_dim_map), so each tap's image is a product of 1-D interval
// sets computed in closed form, and the union over taps is exact.
#include <algorithm>
#include <cstdio>

#include "host_core.h"

namespace pk {

bool mul_ok(int64_t a, int64_t b, int64_t* out) { return !__builtin_mul_overflow(a, b, out); }
bool add_ok(int64_t a, int64_t b, int64_t* out) { return !__builtin_add_overflow(a, b, out); }

Status eval_expr(const pk_expr& e, const EvalEnv& env, int64_t* out) {
    int64_t v = e.c0, t;
    for (int s = 0; s < PK_MAX_SCALARS; ++s) {
        if (e.c_scalar[s] == 0) continue;
        if (s >= env.nscalars)
            return Status::Err(PK_ERR_INVALID, "descriptor uses scalar " + std::to_string(s) +
                                                   " but only " + std::to_string(env.nscalars) +
                                                   " scalars were passed");
        if (!mul_ok(e.c_scalar[s], env.scalars[s], &t) || !add_ok(v, t, &v))
            return Status::Err(PK_ERR_OVERFLOW, "int64 overflow evaluating a descriptor expression");
    }
    for (int w = 0; w < 3; ++w) {
        if (e.c_blockdim[w] == 0) continue;
        if (!mul_ok(e.c_blockdim[w], env.block[w], &t) || !add_ok(v, t, &v))
            return Status::Err(PK_ERR_OVERFLOW, "int64 overflow evaluating a descriptor expression");
    }
    *out = v;
    return Status::Ok();
}

static void merge_ivs(std::vector<Iv>* v) {
    auto& a = *v;
    std::sort(a.begin(), a.end(), [](const Iv& x, const Iv& y) { return x.lo < y.lo; });
    size_t n = 0;
    for (size_t i = 0; i < a.size(); ++i) {
        if (a[i].lo >= a[i].hi) continue;
        if (n && a[i].lo <= a[n - 1].hi) a[n - 1].hi = std::max(a[n - 1].hi, a[i].hi);
        else a[n++] = a[i];
    }
    a.resize(n);
}

Status dim_index_set(const pk_dim_map& dm, const int64_t box6[6], int64_t shape_k,
                     const EvalEnv& env, std::vector<Iv>* out) {
    out->clear();
    int64_t scale = 0, extent = 0, glo = 0, ghi = 0, off = 0;
    Status st;
    if (!(st = eval_expr(dm.extent, env, &extent)).ok()) return st;
    if (!(st = eval_expr(dm.offset, env, &off)).ok()) return st;
    const bool guard = dm.flags & PK_DIM_GUARD;
    if (guard) {
        if (!(st = eval_expr(dm.guard_lo, env, &glo)).ok()) return st;
        if (!(st = eval_expr(dm.guard_hi, env, &ghi)).ok()) return st;
    }
    if (extent <= 0) return Status::Ok();
    std::vector<Iv> pos;
    if (dm.grid_dim < 0) {
        pos.push_back({0, extent});
    } else {
        if (dm.grid_dim > 2) return Status::Err(PK_ERR_INVALID, "grid_dim must be -1, 0, 1 or 2");
        if (!(st = eval_expr(dm.scale, env, &scale)).ok()) return st;
        if (scale < 0) return Status::Err(PK_ERR_INVALID, "negative descriptor scale");
        // box6 order (zmin,zmax,ymin,ymax,xmin,xmax); grid_dim 0=x 1=y 2=z
        const int64_t m = box6[2 * (2 - dm.grid_dim)], M = box6[2 * (2 - dm.grid_dim) + 1];
        if (m >= M) return Status::Ok();
        int64_t a, b, c;
        if (extent >= scale) {
            // blocks overlap or touch: one interval [m*scale, (M-1)*scale + extent)
            if (!mul_ok(m, scale, &a) || !mul_ok(M - 1, scale, &b) || !add_ok(b, extent, &c))
                return Status::Err(PK_ERR_OVERFLOW, "int64 overflow in block range");
            pos.push_back({a, c});
        } else {
            // gaps between blocks: one interval per block (exact)
            if ((M - m) > (int64_t)1 << 26)
                return Status::Err(PK_ERR_INVALID, "strided descriptor over too many blocks");
            pos.reserve(M - m);
            for (int64_t blk = m; blk < M; ++blk) {
                if (!mul_ok(blk, scale, &a) || !add_ok(a, extent, &c))
                    return Status::Err(PK_ERR_OVERFLOW, "int64 overflow in block range");
                pos.push_back({a, c});
            }
        }
    }
    for (Iv& iv : pos) {
        if (guard) {
            iv.lo = std::max(iv.lo, glo);
            iv.hi = std::min(iv.hi, ghi);
        }
        if (iv.lo >= iv.hi) continue;
        int64_t lo, hi;
        if (!add_ok(iv.lo, off, &lo) || !add_ok(iv.hi, off, &hi))
            return Status::Err(PK_ERR_OVERFLOW, "int64 overflow applying offset");
        if (dm.flags & PK_DIM_CLAMP) {
            // monotone map: image of [lo,hi) is [clamp(lo), clamp(hi-1)+1)
            if (shape_k <= 0) continue;
            int64_t a = std::min(std::max(lo, (int64_t)0), shape_k - 1);
            int64_t b = std::min(std::max(hi - 1, (int64_t)0), shape_k - 1) + 1;
            out->push_back({a, b});
        } else {
            if (lo < 0 || hi > shape_k) {
                char buf[160];
                snprintf(buf, sizeof buf, "access [%lld, %lld) outside [0, %lld) of an unclamped dimension",
                         (long long)lo, (long long)hi, (long long)shape_k);
                return Status::Err(PK_ERR_OUT_OF_BOUNDS, buf);
            }
            out->push_back({lo, hi});
        }
    }
    merge_ivs(out);
    return Status::Ok();
}

Status tap_ranges(const pk_affine_access& tap, const int64_t box6[6], int ndim,
                  const int64_t* shape, int64_t elem_bytes, const EvalEnv& env,
                  RangeList* out) {
    out->clear();
    if (tap.ndim != ndim)
        return Status::Err(PK_ERR_INVALID, "descriptor ndim " + std::to_string(tap.ndim) +
                                               " != buffer ndim " + std::to_string(ndim));
    // a partition without thread blocks touches nothing (even grid_dim == -1 maps)
    if (box6[0] >= box6[1] || box6[2] >= box6[3] || box6[4] >= box6[5]) return Status::Ok();
    int used[3] = {0, 0, 0};
    for (int k = 0; k < ndim; ++k) {
        int g = tap.dim[k].grid_dim;
        if (g >= 0 && g <= 2 && used[g]++)
            return Status::Err(PK_ERR_INVALID,
                               "a grid dimension drives two array dimensions of one tap (not separable)");
    }
    // The image is a product: if any dimension's set is empty no thread accesses
    // anything, so an unclamped out-of-bounds dimension is only an error when
    // every other dimension is non-empty.
    std::vector<Iv> sets[PK_MAX_DIMS];
    Status oob;
    bool any_empty = false;
    for (int k = 0; k < ndim; ++k) {
        Status st = dim_index_set(tap.dim[k], box6, shape[k], env, &sets[k]);
        if (st.code == PK_ERR_OUT_OF_BOUNDS) {
            if (oob.ok()) oob = st;
            continue;
        }
        if (!st.ok()) return st;
        if (sets[k].empty()) any_empty = true;
    }
    if (any_empty) return Status::Ok();  // empty image
    if (!oob.ok()) return oob;
    // strides in bytes; full_from[k]: dims k..ndim-1 are fully covered
    int64_t stride[PK_MAX_DIMS];
    bool full_from[PK_MAX_DIMS + 1];
    stride[ndim - 1] = elem_bytes;
    for (int k = ndim - 2; k >= 0; --k)
        if (!mul_ok(stride[k + 1], shape[k + 1], &stride[k]))
            return Status::Err(PK_ERR_OVERFLOW, "buffer too large");
    full_from[ndim] = true;
    for (int k = ndim - 1; k >= 0; --k)
        full_from[k] = full_from[k + 1] && sets[k].size() == 1 && sets[k][0].lo == 0 &&
                       sets[k][0].hi == shape[k];
    // row-wise enumeration: fix all dims but the trailing non-full ones
    auto emit = [&](auto&& self, int k, int64_t base) -> void {
        for (const Iv& iv : sets[k]) {
            if (k == ndim - 1 || full_from[k + 1]) {
                uint64_t b = (uint64_t)(base + iv.lo * stride[k]);
                uint64_t e = (uint64_t)(base + iv.hi * stride[k]);
                if (!out->empty() && out->back().e == b) out->back().e = e;
                else out->push_back(Range{b, e});
            } else {
                for (int64_t i = iv.lo; i < iv.hi; ++i) self(self, k + 1, base + i * stride[k]);
            }
        }
    };
    emit(emit, 0, 0);
    return Status::Ok();
}

void canonicalize(RangeList* r) {
    auto& a = *r;
    std::sort(a.begin(), a.end(), [](const Range& x, const Range& y) { return x.b < y.b; });
    size_t n = 0;
    for (size_t i = 0; i < a.size(); ++i) {
        if (a[i].b >= a[i].e) continue;
        if (n && a[i].b <= a[n - 1].e) a[n - 1].e = std::max(a[n - 1].e, a[i].e);
        else a[n++] = a[i];
    }
    a.resize(n);
}

RangeList union_ranges(const RangeList& a, const RangeList& b) {
    RangeList r;
    r.reserve(a.size() + b.size());
    r.insert(r.end(), a.begin(), a.end());
    r.insert(r.end(), b.begin(), b.end());
    canonicalize(&r);
    return r;
}

RangeList intersect_ranges(const RangeList& a, const RangeList& b) {
    // both canonical (sorted, disjoint): linear merge
    RangeList r;
    size_t i = 0, j = 0;
    while (i < a.size() && j < b.size()) {
        const uint64_t lo = std::max(a[i].b, b[j].b), hi = std::min(a[i].e, b[j].e);
        if (lo < hi) r.push_back(Range{lo, hi});
        if (a[i].e < b[j].e) ++i;
        else ++j;
    }
    return r;
}

uint64_t total_bytes(const RangeList& r) {
    uint64_t t = 0;
    for (const Range& x : r) t += x.e - x.b;
    return t;
}

void Tracker::init(uint64_t size, uint64_t mask) {
    size_ = size;
    SegVec v;
    if (size) v.push_back(Seg{0, size, mask});
    segs_ = std::make_shared<const SegVec>(std::move(v));
    fp_valid_ = false;
}

}  // namespace pk
