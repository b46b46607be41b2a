// Which TMEM (lane, column) does each thread receive from tcgen05.ld.16x256b?
// Every thread of warp 0 stores (lane << 16 | col) into its own TMEM lane with
// 32x32b stores; then the warp reads 16 lanes x 256 bit (x2 = 16 columns) at
// lane bases 0 and 16 and prints the decoded (lane, col) of each register.
#include <cstdio>
#include <cstdint>

__global__ void k(uint32_t* out)
{
    __shared__ uint32_t s_base;
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" ::"r"(
            (uint32_t)__cvta_generic_to_shared(&s_base)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t base = s_base;
    const uint32_t t = threadIdx.x;
    if (t < 32) {
        for (int c = 0; c < 16; ++c) {
            uint32_t v = (t << 16) | c;
            asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(base + c), "r"(v));
        }
        asm volatile("tcgen05.wait::st.sync.aligned;");
        for (int h = 0; h < 2; ++h) {
            uint32_t r[8];
            asm volatile("tcgen05.ld.sync.aligned.16x256b.x2.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];\n\t"
                         "tcgen05.wait::ld.sync.aligned;"
                         : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
                           "=r"(r[7])
                         : "r"(base + ((16u * h) << 16)));
            for (int i = 0; i < 8; ++i) out[(h * 32 + t) * 8 + i] = r[i];
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (t < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" ::"r"(base));
}

int main()
{
    uint32_t* d;
    cudaMalloc(&d, 2 * 32 * 8 * 4);
    k<<<1, 128>>>(d);
    uint32_t h[2 * 32 * 8];
    cudaError_t e = cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
    for (int hh = 0; hh < 2; ++hh)
        for (int t = 0; t < 32; ++t) {
            printf("h%d t%2d:", hh, t);
            for (int i = 0; i < 8; ++i) printf(" (%u,%u)", h[(hh * 32 + t) * 8 + i] >> 16, h[(hh * 32 + t) * 8 + i] & 0xFFFF);
            printf("\n");
        }
    return 0;
}
