// locmon.h — Segment Location Monitor (Alg 2, §4.4), internal.
//
// Tracks, per datum, where each segment lives: `lastOutput` (the segments the
// last task wrote, one entry per location, plus whether the outputs are
// partials that need aggregation) and `upToDate` (every location holding an
// unmodified instance of a segment, so later tasks skip the copy).  Boxes are
// N-dimensional half-open rectangles (N <= 3).  Pure host code: the runtime
// (api.cpp) turns the returned copy list into peer copies / NCCL send-recv.
#pragma once
#include <stdint.h>

#include <map>
#include <vector>

#include "mapsm.h"

namespace mapsm {

struct Box {
    int64_t lo[MAPSM_MAX_DIMS], hi[MAPSM_MAX_DIMS];
};

bool box_empty(const Box& a, int nd);
bool box_intersect(const Box& a, const Box& b, int nd, Box* out);
// a \ b as at most 2*nd disjoint boxes appended to out
void box_subtract(const Box& a, const Box& b, int nd, std::vector<Box>& out);

struct LocEntry {
    int loc;
    Box box;
};

struct CopyOp {
    int src, dst;
    Box box;
};

class LocationMonitor {
public:
    explicit LocationMonitor(int ndims) : nd_(ndims) {}
    int ndims() const { return nd_; }
    // A task wrote `segs` of `datum` (a new version): lastOutput := segs,
    // upToDate := segs unless they are partials awaiting aggregation.
    void output(int datum, const std::vector<LocEntry>& segs, bool needs_aggregation);
    // Alg 2: copies that bring `required` of `datum` up to date on `target`.
    // Returns MAPSM_ESTATE for an unknown datum, MAPSM_EINVAL if part of
    // `required` has no source (outside every lastOutput segment).
    mapsm_status query(int datum, const Box& required, int target, std::vector<CopyOp>& ops,
                       bool* needs_aggregation) const;
    // Copies completed: record the copied segments as up to date (Alg 2's
    // closing step).  Ignored for partials awaiting aggregation.
    void copied(int datum, const std::vector<CopyOp>& ops);
    bool known(int datum) const { return data_.count(datum) != 0; }
    void forget(int datum) { data_.erase(datum); }

private:
    struct Datum {
        std::vector<LocEntry> last_output;
        std::vector<LocEntry> up_to_date;
        bool needs_aggregation = false;
    };
    int nd_;
    std::map<int, Datum> data_;
};

}  // namespace mapsm
