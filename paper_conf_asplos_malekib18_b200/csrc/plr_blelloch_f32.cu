// plr_blelloch_f32.cu -- the Scan comparator (plr_blelloch.cuh): fp32 data, fp32 arithmetic.
#include "plr_blelloch.cuh"
#include "plr_launch.h"

namespace plr {
cudaError_t blelloch_f32(const float* x, float* y, long long n, const float* c, int k, const float* alpha, int p,
                           void* tmp, size_t& tmp_bytes, cudaStream_t s) {
    switch (k) {
        case 1: return blelloch::scan<float, 1>(x, y, n, c, alpha, p, tmp, tmp_bytes, s);
        case 2: return blelloch::scan<float, 2>(x, y, n, c, alpha, p, tmp, tmp_bytes, s);
        case 3: return blelloch::scan<float, 3>(x, y, n, c, alpha, p, tmp, tmp_bytes, s);
        case 4: return blelloch::scan<float, 4>(x, y, n, c, alpha, p, tmp, tmp_bytes, s);
    }
    return cudaErrorInvalidValue;
}
}  // namespace plr
