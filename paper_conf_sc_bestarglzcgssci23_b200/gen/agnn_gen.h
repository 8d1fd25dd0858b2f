/*
 * agnn_gen.h — seeded synthetic-input generators shared by the oracle side
 * (host, via libagnngen.so) and the GPU path (device kernels in gen_device.cu).
 *
 * This header holds NO arithmetic of the A-GNN method: only a counter-based
 * RNG, graph edge-sample generators and feature/weight fillers. Both sides
 * evaluate the same integer functions, so host and device draws are
 * bit-identical.
 *
 * Recipes (DESIGN.md §3 "input recipe"):
 *   Kronecker : Graph500 initiator (A,B,C,D) = (0.57,0.19,0.19,0.05), one
 *               quadrant draw per level ("based on the
 *               Graph500 Kronecker generator"), then a seeded bijective label
 *               scramble.
 *   R-MAT     : the same draws, no scramble (degree skew concentrated in low
 *               vertex ids).
 *   ER        : G(n, M) uniform ordered pairs (PAPER.md:366 §7.3, :414 "Rand").
 *   Features  : H ~ U[-1,1) on the 2^-23 grid (exact in fp32 and fp64);
 *               W, a ~ Glorot-uniform +-sqrt(6/(k+k')), the bound passed in as
 *               a float computed by the caller; R (dL/dH_out) ~ U[-1,1).
 */
#ifndef AGNN_GEN_H
#define AGNN_GEN_H
#include <stdint.h>

#if defined(__CUDACC__)
#define AGEN_HD __host__ __device__ __forceinline__
#else
#define AGEN_HD static inline
#endif

/* RNG stream ids (graph=0, H=1, W^l=2+l, a^l=100+l, R=200) */
#define AGEN_STREAM_GRAPH    0ull
#define AGEN_STREAM_H        1ull
#define AGEN_STREAM_W(l)     (2ull + (uint64_t)(l))
#define AGEN_STREAM_A(l)     (100ull + (uint64_t)(l))
#define AGEN_STREAM_R        200ull
#define AGEN_STREAM_SCRAMBLE 300ull

enum { AGEN_ER = 0, AGEN_KRON = 1, AGEN_RMAT = 2 };

/* splitmix64 finaliser */
AGEN_HD uint64_t agen_mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

/* counter-based draw: a pure function of (seed, stream, index) */
AGEN_HD uint64_t agen_u64(uint64_t seed, uint64_t stream, uint64_t idx) {
  uint64_t key = agen_mix64(seed ^ agen_mix64(stream * 0xD1B54A32D192ED03ull + 0x632BE59BD9B4E019ull));
  return agen_mix64(key + idx * 0x9E3779B97F4A7C15ull);
}

/* U[-1,1) on the 2^-23 grid: exactly representable in fp32 */
AGEN_HD float agen_unif_pm1(uint64_t seed, uint64_t stream, uint64_t idx) {
  int32_t q = (int32_t)(agen_u64(seed, stream, idx) >> 40) - (int32_t)(1 << 23);
  return (float)q * (1.0f / 8388608.0f);
}

/* Graph500 initiator thresholds on 32-bit uniforms: floor(p * 2^32) */
#define AGEN_TA   2448131358u  /* 0.57                */
#define AGEN_TAB  3264175144u  /* 0.57 + 0.19 = 0.76  */
#define AGEN_TABC 4080218931u  /* 0.95                */

/* seeded bijection of [0, 2^scale) (odd multiply / xor-shift / xor key) */
AGEN_HD uint32_t agen_scramble(uint64_t seed, int scale, uint32_t v) {
  const uint64_t mask = (scale >= 64) ? ~0ull : ((1ull << scale) - 1ull);
  const uint64_t k1 = agen_u64(seed, AGEN_STREAM_SCRAMBLE, 0) | 1ull;
  const uint64_t k2 = agen_u64(seed, AGEN_STREAM_SCRAMBLE, 1) | 1ull;
  const uint64_t k3 = agen_u64(seed, AGEN_STREAM_SCRAMBLE, 2);
  const int h = scale / 2 > 0 ? scale / 2 : 1;
  uint64_t x = v;
  x = (x * k1) & mask;
  x ^= x >> h;
  x = (x * k2) & mask;
  x ^= x >> h;
  x ^= k3 & mask;
  return (uint32_t)x;
}

/* One Kronecker / R-MAT sample e: `scale` quadrant draws, two per u64. */
AGEN_HD void agen_kron_pair(uint64_t seed, int scale, uint64_t e, int scramble,
                            uint32_t* src, uint32_t* dst) {
  uint32_t s = 0, d = 0;
  for (int l = 0; l < scale; l += 2) {
    const uint64_t u = agen_u64(seed, AGEN_STREAM_GRAPH, e * 32ull + (uint64_t)(l >> 1));
    for (int b = 0; b < 2 && l + b < scale; ++b) {
      const uint32_t r = (uint32_t)(b ? (u >> 32) : u);
      const uint32_t q = r < AGEN_TA ? 0u : r < AGEN_TAB ? 1u : r < AGEN_TABC ? 2u : 3u;
      s |= (q >> 1) << (l + b);
      d |= (q & 1u) << (l + b);
    }
  }
  if (scramble) {
    s = agen_scramble(seed, scale, s);
    d = agen_scramble(seed, scale, d);
  }
  *src = s;
  *dst = d;
}

/* One G(n,M) sample e: two uniform vertex ids by multiply-shift. */
AGEN_HD void agen_er_pair(uint64_t seed, uint64_t n, uint64_t e, uint32_t* src, uint32_t* dst) {
  const uint64_t u = agen_u64(seed, AGEN_STREAM_GRAPH, e);
  *src = (uint32_t)(((u & 0xFFFFFFFFull) * n) >> 32);
  *dst = (uint32_t)(((u >> 32) * n) >> 32);
}

AGEN_HD void agen_pair(int kind, uint64_t seed, int scale, uint64_t n, uint64_t e,
                       uint32_t* src, uint32_t* dst) {
  if (kind == AGEN_ER) agen_er_pair(seed, n, e, src, dst);
  else agen_kron_pair(seed, scale, e, kind == AGEN_KRON, src, dst);
}

#endif /* AGNN_GEN_H */
