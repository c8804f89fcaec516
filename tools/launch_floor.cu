// launch_floor.cu -- per-launch device floor of the building blocks of the
// scan kernels (small-n investigation): an empty kernel, the same
// with ~200 KB dynamic shared memory, with a 512-column TMEM alloc/dealloc,
// with mbarrier init + one 30 KB bulk load, and a 6.4 KB __grid_constant__
// parameter block.  Each variant: 1 CTA and 148 CTAs, 200 launches captured in
// one CUDA graph, replayed 10x, CUDA events around the replays.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o launch_floor tools/launch_floor.cu
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e_)); return 1; } } while (0)

struct Big { uint32_t w[1600]; };   // 6.4 KB of kernel parameters

__global__ void k_empty(int* out) { if (threadIdx.x == 0 && out[0] == 12345) out[1] = 1; }

__global__ void k_smem(int* out) {
    extern __shared__ uint32_t sm[];
    if (threadIdx.x == 0) { sm[0] = blockIdx.x; if (sm[0] == 12345u && out[0] == 1) out[1] = 1; }
}

__global__ void k_params(const __grid_constant__ Big b, int* out) {
    if (threadIdx.x == 0 && b.w[blockIdx.x % 1600] == 12345u) out[1] = 1;
}

__global__ void k_tmem(int* out) {
    __shared__ uint32_t base;
    const int warp = threadIdx.x >> 5;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                     ::"r"((uint32_t)__cvta_generic_to_shared(&base)), "r"(512) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t t = base;
    __syncthreads();
    if (warp == 0)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(t), "r"(512) : "memory");
    if (threadIdx.x == 0 && out[0] == 12345) out[1] = (int)t;
}

__global__ void k_bulk(const uint32_t* x, int* out) {
    extern __shared__ __align__(128) uint32_t sm[];
    __shared__ __align__(8) uint64_t bar;
    const uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar);
    const uint32_t bytes = 7936 * 4;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(bytes) : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     ::"r"((uint32_t)__cvta_generic_to_shared(sm)), "l"(x + (size_t)blockIdx.x * 7936), "r"(bytes), "r"(b)
                     : "memory");
        uint32_t ok = 0;
        while (!ok)
            asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], 0;\n\t"
                         "selp.u32 %0, 1, 0, p;\n\t}" : "=r"(ok) : "r"(b) : "memory");
        if (sm[5] == 12345u && out[0] == 1) out[1] = 1;
    }
}

template <typename F>
static float per_launch_us(F launch, cudaStream_t s) {
    cudaGraph_t g;
    cudaGraphExec_t ge;
    cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal);
    for (int i = 0; i < 200; i++) launch();
    cudaStreamEndCapture(s, &g);
    cudaGraphInstantiate(&ge, g, 0);
    cudaGraphLaunch(ge, s);
    cudaStreamSynchronize(s);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0, s);
    for (int r = 0; r < 10; r++) cudaGraphLaunch(ge, s);
    cudaEventRecord(e1, s);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    cudaGraphExecDestroy(ge);
    cudaGraphDestroy(g);
    return ms * 1000.f / 2000.f;
}

int main() {
    cudaStream_t s;
    CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    int* out;
    uint32_t* x;
    CK(cudaMalloc(&out, 64));
    CK(cudaMemset(out, 0, 64));
    CK(cudaMalloc(&x, (size_t)148 * 7936 * 4));
    CK(cudaMemset(x, 0, (size_t)148 * 7936 * 4));
    const int big = 200 * 1024;
    CK(cudaFuncSetAttribute(k_smem, cudaFuncAttributeMaxDynamicSharedMemorySize, big));
    CK(cudaFuncSetAttribute(k_bulk, cudaFuncAttributeMaxDynamicSharedMemorySize, big));
    Big bp = {};
    for (int grid : {1, 148}) {
        printf("{\"grid\": %d, \"empty_us\": %.2f, \"smem200k_us\": %.2f, \"params6k_us\": %.2f, "
               "\"tmem512_us\": %.2f, \"bulk30k_smem200k_us\": %.2f}\n", grid,
               per_launch_us([&] { k_empty<<<grid, 384, 0, s>>>(out); }, s),
               per_launch_us([&] { k_smem<<<grid, 384, big, s>>>(out); }, s),
               per_launch_us([&] { k_params<<<grid, 384, 0, s>>>(bp, out); }, s),
               per_launch_us([&] { k_tmem<<<grid, 384, 0, s>>>(out); }, s),
               per_launch_us([&] { k_bulk<<<grid, 384, big, s>>>(x, out); }, s));
    }
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
    return 0;
}
