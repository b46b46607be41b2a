cd tools/microbench && ./alu_peak 200000 && ./curand_bench 4294967296
