/* cstgen/cst_gen.h — the seeded, counter-based input generator.
 *
 * This module is the ONLY code shared between the oracle (oracle/) and the CUDA
 * path (libcst's device filler).  It holds none of the stencil arithmetic: it maps
 * (seed, array id, global padded index) to a double in [-1, 1).
 *
 *   h = splitmix64(splitmix64(seed ^ (array_id * 0x9E3779B97F4A7C15)) ^ g)
 *   v = 2 * ((h >> 11) * 2^-53) - 1                       (exact in FP64)
 *
 *   g = ((z + H) * (NY + 2H) + (y + H)) * (NX + 2H) + (x + H)
 *
 * where (x, y, z) is a GLOBAL coordinate in [-H, N + H) per axis and H is the grid
 * halo width.  g uses the logical padded extents, never a pitch, so any rank (or the
 * oracle) can regenerate any point — including the true neighbour values in a slab's
 * halo — without the global array.  A Python/numpy twin lives in cstgen/gen.py.
 *
 * Usable from C, C++ and CUDA (host and device).
 */
#ifndef CST_GEN_H
#define CST_GEN_H

#include <stdint.h>

#if defined(__CUDACC__) || defined(__CUDACC_RTC__)
#define CSTGEN_FN __host__ __device__ static inline
#else
#define CSTGEN_FN static inline
#endif

#define CSTGEN_GOLDEN 0x9E3779B97F4A7C15ULL

/* Standard splitmix64 finaliser (Steele, Lea, Flood 2014), all arithmetic mod 2^64. */
CSTGEN_FN uint64_t cstgen_splitmix64(uint64_t x) {
  uint64_t z = x + CSTGEN_GOLDEN;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

/* Per-array stream key; hoist out of loops. */
CSTGEN_FN uint64_t cstgen_key(uint64_t seed, uint64_t array_id) {
  return cstgen_splitmix64(seed ^ (array_id * CSTGEN_GOLDEN));
}

/* Value for stream key `key` at counter g, in [-1, 1). */
CSTGEN_FN double cstgen_value(uint64_t key, uint64_t g) {
  uint64_t h = cstgen_splitmix64(key ^ g);
  return 2.0 * ((double)(h >> 11) * 0x1.0p-53) - 1.0;
}

/* Global padded counter for (x, y, z) in [-H, N+H). */
CSTGEN_FN uint64_t cstgen_index(int64_t nx, int64_t ny, int64_t halo,
                                int64_t x, int64_t y, int64_t z) {
  return (uint64_t)(((z + halo) * (ny + 2 * halo) + (y + halo)) * (nx + 2 * halo) + (x + halo));
}

CSTGEN_FN double cstgen_at(uint64_t seed, uint64_t array_id, int64_t nx, int64_t ny,
                           int64_t halo, int64_t x, int64_t y, int64_t z) {
  return cstgen_value(cstgen_key(seed, array_id), cstgen_index(nx, ny, halo, x, y, z));
}

#endif /* CST_GEN_H */
