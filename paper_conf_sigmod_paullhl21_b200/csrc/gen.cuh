// gen.cuh — counter-based synthetic input generator (DESIGN.md
// §3).  Bit-identical to paper_conf_sigmod_paullhl21_b200/datagen.py: every
// floating-point step of the Zipf sampler uses explicitly rounded
// operations (__dmul_rn/__dadd_rn/__dsub_rn, no FMA contraction), so CUDA and
// numpy produce the same ranks.  Not part of the join; runs before the timed
// region.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

namespace mgj_gen {

constexpr uint64_t SEED_R = 0x5EED0052ull, SEED_S = 0x5EED0053ull;
constexpr uint64_t SEED_Z = 0x5EED005Aull, SEED_X = 0x5EED0058ull;

__device__ __forceinline__ uint64_t perm_k(uint64_t x, int k, uint64_t s) {
    const uint64_t M = (1ull << k) - 1;
    const int h = (k + 1) / 2;
    x = (x ^ s) & M;
    x = (x * 0x9E3779B1ull) & M;
    x ^= x >> h;
    x = (x * 0x85EBCA6Bull) & M;
    x ^= x >> h;
    x = (x * 0xC2B2AE35ull) & M;
    x ^= x >> h;
    return x;
}

__device__ __forceinline__ uint64_t perm_n(uint64_t x, uint64_t n, int k, uint64_t s) {
    uint64_t y = perm_k(x, k, s);
    while (y >= n) y = perm_k(y, k, s);
    return y;
}

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

__device__ inline double exp2_frac(double f) {
    // 1/i!, i = 0..17 (same bit patterns as datagen.EXP_COEF_HEX)
    const double coef[18] = {0x1.0000000000000p+0, 0x1.0000000000000p+0, 0x1.0000000000000p-1,
                             0x1.5555555555555p-3, 0x1.5555555555555p-5, 0x1.1111111111111p-7,
                             0x1.6c16c16c16c17p-10, 0x1.a01a01a01a01ap-13, 0x1.a01a01a01a01ap-16,
                             0x1.71de3a556c734p-19, 0x1.27e4fb7789f5cp-22, 0x1.ae64567f544e4p-26,
                             0x1.1eed8eff8d898p-29, 0x1.6124613a86d09p-33, 0x1.93974a8c07c9dp-37,
                             0x1.ae7f3e733b81fp-41, 0x1.ae7f3e733b81fp-45, 0x1.952c77030ad4ap-49};
    const double x = __dmul_rn(f, 0x1.62e42fefa39efp-1);
    double p = coef[17];
#pragma unroll
    for (int i = 16; i >= 0; --i) p = __dadd_rn(__dmul_rn(p, x), coef[i]);
    return p;
}

__device__ inline uint64_t zipf_rank(uint64_t j, uint64_t n, int k, int zmode) {
    const double u = __dmul_rn((double)(mix64(j ^ SEED_Z) >> 11), 0x1p-53);
    double r;
    if (zmode == 0) {
        r = floor(__dmul_rn(u, (double)n));
    } else if (zmode == 1) {  // z = 0.5
        const double a = __dsqrt_rn((double)n);
        double t = __dmul_rn(__dsub_rn(a, 1.0), u);
        t = __dadd_rn(t, 1.0);
        r = floor(__dmul_rn(t, t)) - 1.0;
    } else {  // z = 1
        const double y = __dmul_rn((double)k, u);
        const double e = floor(y);
        const double f = __dsub_rn(y, e);
        r = floor(ldexp(exp2_frac(f), (int)e)) - 1.0;
    }
    if (r < 0.0) r = 0.0;
    if (r > (double)(n - 1)) r = (double)(n - 1);
    return (uint64_t)r;
}

// kind 0 unique, 1 zipf, 2 wide; rel 0 = R, 1 = S.
__global__ void k_gen(int kind, int rel, uint64_t n_r, uint64_t n_s, int zmode, uint64_t row0, uint64_t count,
                      void *keys, void *pays) {
    const uint64_t n = rel == 0 ? n_r : n_s;
    int k = 1;
    while ((1ull << k) < n) ++k;
    const uint64_t seed = rel == 0 ? SEED_R : SEED_S;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count;
         i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t row = row0 + i;
        if (kind == 0) {
            static_cast<uint32_t *>(keys)[i] = (uint32_t)perm_n(row, n, k, seed);
            static_cast<uint32_t *>(pays)[i] = (uint32_t)row;
        } else if (kind == 2) {
            static_cast<uint64_t *>(keys)[i] = mix64(perm_n(row, n, k, seed));
            static_cast<uint64_t *>(pays)[i] = row + (rel == 0 ? (1ull << 40) : (1ull << 41));
        } else {
            int kr = 1;
            while ((1ull << kr) < n_r) ++kr;
            if (rel == 0) {
                static_cast<uint32_t *>(keys)[i] = (uint32_t)perm_k(row, kr, SEED_R);
            } else {
                const uint64_t r = zipf_rank(row, n_r, kr, zmode);
                const uint64_t key = (row & 1) ? n_r + perm_k(r, kr, SEED_X) : perm_k(r, kr, SEED_R);
                static_cast<uint32_t *>(keys)[i] = (uint32_t)key;
            }
            static_cast<uint32_t *>(pays)[i] = (uint32_t)row;
        }
    }
}

}  // namespace mgj_gen
