/*
 * synth/table_gen.c -- seeded synthetic INPUT generator (not part of the method).
 *
 * The embedding table of the synthetic workloads is "self-describing": 32-bit word w
 * of row k is
 *
 *     word(k, w) = lo32( splitmix64( seed ^ (k * W + w) ) ),   W = row_bytes / 4
 *
 * so any row can be re-derived from its key alone ("what pins
 * each part").  Random 32-bit words include NaN / denormal bit patterns on purpose, so a
 * float-typed copy anywhere on the path shows up as a bit mismatch.
 *
 * This file is shared by the oracle side (tests) and the product side (bench inputs) as
 * the one seeded input generator; it holds none of the method's arithmetic (no locate,
 * no bucketing, no gather).  Built by __graft_entry__.build() into synth/libsynth.so.
 */
#include <stdint.h>
#include <stddef.h>

static inline uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

/* Fill rows [row_begin, row_end) of a row-major table whose row 'row_begin' starts at
 * dst.  words_per_row = row_bytes / 4.  Parallel over rows (OpenMP); each page is first
 * touched by the thread that fills it. */
void synth_fill_table(uint32_t *dst, uint64_t row_begin, uint64_t row_end,
                      uint32_t words_per_row, uint64_t seed) {
  const int64_t nrows = (int64_t)(row_end - row_begin);
#pragma omp parallel for schedule(static)
  for (int64_t r = 0; r < nrows; ++r) {
    const uint64_t k = row_begin + (uint64_t)r;
    uint32_t *row = dst + (uint64_t)r * words_per_row;
    const uint64_t base = k * (uint64_t)words_per_row;
    for (uint32_t w = 0; w < words_per_row; ++w)
      row[w] = (uint32_t)splitmix64(seed ^ (base + w));
  }
}

/* Re-derive the rows of an arbitrary key list (out-of-range keys -> zero row), used by
 * tests to pin gathers without a second copy of a large table. */
void synth_rows_for_keys(uint32_t *dst, const int64_t *keys, uint64_t n, uint64_t num_rows,
                         uint32_t words_per_row, uint64_t seed) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < (int64_t)n; ++i) {
    uint32_t *row = dst + (uint64_t)i * words_per_row;
    const int64_t k = keys[i];
    if (k < 0 || (uint64_t)k >= num_rows) {
      for (uint32_t w = 0; w < words_per_row; ++w) row[w] = 0u;
      continue;
    }
    const uint64_t base = (uint64_t)k * (uint64_t)words_per_row;
    for (uint32_t w = 0; w < words_per_row; ++w)
      row[w] = (uint32_t)splitmix64(seed ^ (base + w));
  }
}
