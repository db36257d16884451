// lower.h — validation and lowering of parsed segments to device descriptors.
#pragma once
#include <string>

#include "ctx.h"

namespace gpl {

// Build segment -> BuildDesc + the hash-table shape it produces.
// `trivial` = no filter and no probe (every row inserted; header known on host).
gpl_status lower_build(gpl_ctx* ctx, const Segment& s, BuildDesc* d, HashTable* shape, bool* trivial,
                       std::string* err);

// Probe segment -> PipeDesc (everything but the schedule/smem layout) + facts.
// split: probes executed before the survivor queue (-1 = auto heuristic).
// With `ins` (the DIRECT table shape lower_build chose), a build segment is
// lowered to the same pipeline with an insert sink (SINK_INSERT).
gpl_status lower_probe(gpl_ctx* ctx, const Segment& s, int split, PipeDesc* d, LowerInfo* li, std::string* err,
                       const HashTable* ins = nullptr);

// Host computation of the header of a trivial build (all rows inserted).
HTHeader trivial_header(int64_t count, long long kmin, long long kmax, int64_t cap_slots, int load_pct);

int64_t next_pow2(int64_t x);

}  // namespace gpl
