// pg_prf.cuh — counter-based input generator of the CUDA path (X8):
// SplitMix64; RAND32(seed, tag, idx) = low32(sm(sm(seed) ^ (tag << 48) ^ idx)).
#pragma once
__device__ __forceinline__ unsigned long long pg_sm64(unsigned long long x) {
    x += 0x9E3779B97F4A7C15ull;
    unsigned long long z = x;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
__device__ __forceinline__ unsigned int pg_rand32(unsigned long long seed, unsigned long long tag,
                                                  unsigned long long idx) {
    return (unsigned int)pg_sm64(pg_sm64(seed) ^ (tag << 48) ^ idx);
}
// the same with sm(seed) ^ (tag << 48) computed once per (seed, array)
__device__ __forceinline__ unsigned int pg_rand32_k(unsigned long long key, unsigned long long idx) {
    return (unsigned int)pg_sm64(key ^ idx);
}
