/*
 * gen/rmat.c — seeded synthetic graph generator (input recipe only).
 *
 * This module holds NONE of the Core Graph method's arithmetic: it only
 * draws the directed, weighted R-MAT edge lists that both the CPU oracle
 * (oracle/) and the CUDA path consume.  The CUDA path carries an
 * independent device implementation of the same counter-based definition
 * (paper_conf_eurosys_0002a0a024_b200/csrc/gen.cu); a GPU test checks the two produce
 * identical edge lists.
 *
 * Definition:
 *   splitmix64(x)             the standard 64-bit finaliser (Steele et al.)
 *   S  = max(1, ceil(log2 n))                         R-MAT scale
 *   kL = splitmix64(seed ^ 0x243F6A8885A308D3)        level key
 *   for edge e, level l in [0,S):
 *       x  = top 32 bits of splitmix64(kL ^ ((e << 6) | l))
 *       quadrant: x < tA -> (0,0); x < tAB -> (0,1); x < tABC -> (1,0); else (1,1)
 *       (row bit, col bit) set bit l of (u, v)
 *   tA/tAB/tABC = floor(a*2^32), floor((a+b)*2^32), floor((a+b+c)*2^32)
 *   fold to [0,n):  u = (u * n) >> S   (multiply-shift; identity when n = 2^S)
 *   permute (optional): Feistel bijection on [0, 2^(2h)), h = ceil(S/2),
 *       4 rounds, round key kR_r = splitmix64(seed ^ (0x13198A2E03707344 + r)),
 *       F(R) = splitmix64(R ^ kR_r) & (2^h - 1), (L,R) <- (R, L ^ F(R));
 *       cycle-walk (re-apply) until the value is < n.
 *   weight: w = 1 + splitmix64(kW ^ e) % w_max,
 *       kW = splitmix64(seed ^ 0xA4093822299F31D0)
 *
 * The paper's inputs are R-MAT / power-law graphs with integer weights in
 * [1, log(n)+1] (§3) and R-MAT parameters
 * RMAT1 (.57,.19,.19,.05) etc. (Table 13a).
 */
#include <stdint.h>
#include <stddef.h>

static inline uint64_t splitmix64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

uint64_t gen_splitmix64(uint64_t x) { return splitmix64(x); }

uint32_t gen_scale(uint64_t n) {
    uint32_t s = 1;
    while ((1ull << s) < n) ++s;
    return s;
}

static uint64_t feistel(uint64_t x, uint32_t h, const uint64_t k[4]) {
    const uint64_t mask = (1ull << h) - 1ull;
    uint64_t L = x >> h, R = x & mask;
    for (int r = 0; r < 4; ++r) {
        uint64_t nl = R;
        uint64_t nr = L ^ (splitmix64(R ^ k[r]) & mask);
        L = nl;
        R = nr;
    }
    return (L << h) | R;
}

uint64_t gen_permute(uint64_t x, uint64_t n, uint64_t seed) {
    uint32_t S = gen_scale(n);
    uint32_t h = (S + 1) / 2;
    uint64_t k[4];
    for (int r = 0; r < 4; ++r) k[r] = splitmix64(seed ^ (0x13198A2E03707344ull + (uint64_t)r));
    uint64_t y = feistel(x, h, k);
    while (y >= n) y = feistel(y, h, k);
    return y;
}

/*
 * Generate edges [e0, e0+count) of the R-MAT stream.
 * Thresholds are passed as integers so every implementation draws the
 * same quadrants.  src/dst/w are caller-owned arrays of `count` entries.
 */
void gen_rmat(uint64_t n, uint32_t tA, uint32_t tAB, uint32_t tABC, uint32_t w_max,
              uint64_t seed, int permute, uint64_t e0, uint64_t count,
              uint32_t* src, uint32_t* dst, uint32_t* w) {
    const uint32_t S = gen_scale(n);
    const uint32_t h = (S + 1) / 2;
    const uint64_t kL = splitmix64(seed ^ 0x243F6A8885A308D3ull);
    const uint64_t kW = splitmix64(seed ^ 0xA4093822299F31D0ull);
    uint64_t k[4];
    for (int r = 0; r < 4; ++r) k[r] = splitmix64(seed ^ (0x13198A2E03707344ull + (uint64_t)r));
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)count; ++i) {
        uint64_t e = e0 + (uint64_t)i;
        uint64_t u = 0, v = 0;
        for (uint32_t l = 0; l < S; ++l) {
            uint32_t x = (uint32_t)(splitmix64(kL ^ ((e << 6) | l)) >> 32);
            uint64_t rb, cb;
            if (x < tA)        { rb = 0; cb = 0; }
            else if (x < tAB)  { rb = 0; cb = 1; }
            else if (x < tABC) { rb = 1; cb = 0; }
            else               { rb = 1; cb = 1; }
            u |= rb << l;
            v |= cb << l;
        }
        u = (u * n) >> S;
        v = (v * n) >> S;
        if (permute) {
            uint64_t y = feistel(u, h, k);
            while (y >= n) y = feistel(y, h, k);
            u = y;
            y = feistel(v, h, k);
            while (y >= n) y = feistel(y, h, k);
            v = y;
        }
        src[i] = (uint32_t)u;
        dst[i] = (uint32_t)v;
        w[i] = 1u + (uint32_t)(splitmix64(kW ^ e) % (uint64_t)w_max);
    }
}
