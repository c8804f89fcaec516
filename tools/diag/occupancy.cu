// Occupancy / attribute probe of the DECAY kernels (diagnostic, not product code):
// prints registers, static smem and CTAs per SM at the dynamic smem each launch uses.
#include <cstdio>
#include "plr_kernels_dect.cuh"
using namespace plr;
template <class F>
void probe(const char* name, F kern, int threads, size_t smem) {
    cudaFuncAttributes a{};
    cudaFuncGetAttributes(&a, kern);
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int occ = -1;
    cudaError_t e2 = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, threads, smem);
    printf("%-40s regs %d static %zu dyn %zu threads %d -> %d CTAs/SM (%s / %s)\n", name, a.numRegs, a.sharedSizeBytes,
           smem, threads, occ, cudaGetErrorString(e), cudaGetErrorString(e2));
}
int main() {
    using LDT = dev::LayoutDT<float, double, 3, 31, 4, 2, 2, 2>;
    using LD = dev::Layout<float, double, 3, 31, 4, 4, 1>;
    probe("dect<f,d,3,3> own smem", &dev::plr_scan_dect_kernel<float, double, 3, 3, 31, 4, 2, 2, 1, 3>, 192, LDT::bytes);
    probe("dect<f,d,3,3> DEC smem", &dev::plr_scan_dect_kernel<float, double, 3, 3, 31, 4, 2, 2, 1, 3>, 192, LD::bytes);
    probe("dec<f,d,3,3>", &dev::plr_scan_kernel<float, double, 3, 3, 31, 4, 4, 1, 1, true, true, 3, true>, 192, LD::bytes);
    for (size_t s = 40 << 10; s <= 80 << 10; s += 8 << 10)
        probe("dect<f,d,3,3> sweep", &dev::plr_scan_dect_kernel<float, double, 3, 3, 31, 4, 2, 2, 1, 3>, 192, s);
    return 0;
}
