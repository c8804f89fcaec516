// plr_blelloch_i32.cu -- the Scan comparator (plr_blelloch.cuh): int32 data, Z/2^32 ring.
#include "plr_blelloch.cuh"
#include "plr_launch.h"

namespace plr {
cudaError_t blelloch_i32(const uint32_t* x, uint32_t* y, long long n, const uint32_t* c, int k, const uint32_t* alpha, int p,
                           void* tmp, size_t& tmp_bytes, cudaStream_t s) {
    switch (k) {
        case 1: return blelloch::scan<uint32_t, 1>(x, y, n, c, alpha, p, tmp, tmp_bytes, s);
        case 2: return blelloch::scan<uint32_t, 2>(x, y, n, c, alpha, p, tmp, tmp_bytes, s);
        case 3: return blelloch::scan<uint32_t, 3>(x, y, n, c, alpha, p, tmp, tmp_bytes, s);
        case 4: return blelloch::scan<uint32_t, 4>(x, y, n, c, alpha, p, tmp, tmp_bytes, s);
    }
    return cudaErrorInvalidValue;
}
}  // namespace plr
