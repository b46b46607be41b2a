// curand_bench.cu -- cuRAND host-API throughput on the same B200, as context
// for the bitsliced keystream (BASELINE.json: "next to cuRAND on the same
// B200").  Generates `bytes` of uint32 output per call into HBM.
//   build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o curand_bench curand_bench.cu -lcurand
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#include <curand.h>
#include <curand_kernel.h>

#define CK(x) do { auto r_ = (x); if (r_ != 0) { printf("error %d at %s:%d\n", int(r_), __FILE__, __LINE__); exit(1); } } while (0)

// device-API XORWOW "consume" kernel: every thread draws `per` uint32 and folds
// them into a checksum (register-consume comparison to the CHECKSUM layout).
__global__ void xorwow_consume(unsigned long long seed, int per, unsigned long long* out)
{
    curandStateXORWOW_t s;
    const unsigned id = blockIdx.x * blockDim.x + threadIdx.x;
    curand_init(seed, id, 0, &s);
    unsigned acc = 0;
    for (int i = 0; i < per; ++i) acc ^= curand(&s);
    if (acc == 0x9e3779b9u) atomicAdd(out, 1ull);
}

__global__ void philox_consume(unsigned long long seed, int per, unsigned long long* out)
{
    curandStatePhilox4_32_10_t s;
    const unsigned id = blockIdx.x * blockDim.x + threadIdx.x;
    curand_init(seed, id, 0, &s);
    unsigned acc = 0;
    for (int i = 0; i < per; i += 4) {
        uint4 v = curand4(&s);
        acc ^= v.x ^ v.y ^ v.z ^ v.w;
    }
    if (acc == 0x9e3779b9u) atomicAdd(out, 1ull);
}

int main(int argc, char** argv)
{
    const size_t bytes = (argc > 1 ? atoll(argv[1]) : (4ull << 30));
    const size_t n = bytes / 4;
    unsigned* buf;
    CK(cudaMalloc(&buf, bytes));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    struct { const char* name; curandRngType_t t; } gens[] = {
        {"XORWOW", CURAND_RNG_PSEUDO_XORWOW},
        {"PHILOX4_32_10", CURAND_RNG_PSEUDO_PHILOX4_32_10},
        {"MTGP32", CURAND_RNG_PSEUDO_MTGP32},
        {"MRG32K3A", CURAND_RNG_PSEUDO_MRG32K3A},
    };
    for (auto& g : gens) {
        curandGenerator_t gen;
        CK(curandCreateGenerator(&gen, g.t));
        CK(curandSetPseudoRandomGeneratorSeed(gen, 0x5EED2020ull));
        CK(curandGenerate(gen, buf, n));  // warm-up (state setup)
        cudaDeviceSynchronize();
        float best = 1e30f;
        for (int r = 0; r < 3; ++r) {
            cudaEventRecord(e0);
            CK(curandGenerate(gen, buf, n));
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (ms < best) best = ms;
        }
        printf("{\"curand\": \"%s\", \"api\": \"host curandGenerate uint32\", \"bytes\": %zu, \"ms\": %.3f, "
               "\"tbps\": %.4f, \"hbm_write_gbs\": %.1f}\n",
               g.name, bytes, best, bytes * 8.0 / (best * 1e-3) / 1e12, bytes / (best * 1e-3) / 1e9);
        curandDestroyGenerator(gen);
    }
    unsigned long long* d;
    CK(cudaMalloc(&d, 8));
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int threads = sms * 2048, per = 4096;
    for (int v = 0; v < 2; ++v) {
        float best = 1e30f;
        for (int r = 0; r < 3; ++r) {
            cudaEventRecord(e0);
            if (v == 0) xorwow_consume<<<threads / 256, 256>>>(1, per, d);
            else philox_consume<<<threads / 256, 256>>>(1, per, d);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (ms < best) best = ms;
        }
        const double bits = double(threads) * per * 32;
        printf("{\"curand\": \"%s\", \"api\": \"device API consume (curand_init + draws, XOR-folded)\", "
               "\"bits\": %.0f, \"ms\": %.3f, \"tbps\": %.4f}\n", v ? "PHILOX4_32_10" : "XORWOW", bits, best,
               bits / (best * 1e-3) / 1e12);
    }
    return 0;
}
