// Device-side canonical ordering of stored cliques (canon.cu).
#pragma once

#include "common.cuh"

namespace mce {
// rows: int32[nrows * width] on the device, sorted in place row by row; `out`
// receives the rows in lexicographic order.  Scratch from `pool` (caller
// resets it).  Returns false (nothing done) for rows wider than 8192.
bool canonicalize_device(int32_t *rows, int64_t nrows, int width, int64_t n_vertices, int32_t *out, Pool &pool,
                         cudaStream_t s);
}  // namespace mce
