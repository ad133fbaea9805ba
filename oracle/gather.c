/*
 * oracle/gather.c -- CPU ORACLE for ugache_extract.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * may load this.  It shares no code with paper_conf_sosp_songz0c23_b200/csrc.
 *
 * What it computes is the plain definition of embedding extraction:
 *   "The embedding layer extracts corresponding entries for each key from the embedding
 *    table into a continuous output region."            -- PAPER.md P:266-269 (section 2)
 *   extract(): for each key i of the batch, locate its entry and write output[i]
 *                                                        -- P:597-615 (section 3.2 listing)
 *   output is in the original key order                  -- P:626-627
 * Every replica of a read-only entry is identical, so the result does not
 * depend on where the entry is cached: out[i] = table[keys[i]].  Out-of-range keys
 * (reading R2) produce a zero row and are counted.
 */
#include <stdint.h>
#include <string.h>

static int64_t gather_impl(const uint8_t *table, uint64_t num_rows, uint32_t row_bytes,
                           const void *keys, int key_is_u32, uint64_t n, uint8_t *out) {
  int64_t bad = 0;
#pragma omp parallel for schedule(static) reduction(+ : bad)
  for (int64_t i = 0; i < (int64_t)n; ++i) {
    int64_t k = key_is_u32 ? (int64_t)((const uint32_t *)keys)[i] : ((const int64_t *)keys)[i];
    uint8_t *dst = out + (uint64_t)i * row_bytes;
    if (k < 0 || (uint64_t)k >= num_rows) {
      memset(dst, 0, row_bytes);
      bad += 1;
    } else {
      memcpy(dst, table + (uint64_t)k * row_bytes, row_bytes);
    }
  }
  return bad;
}

/* out[i*R .. (i+1)*R) = table[keys[i]*R ..) ; returns the number of out-of-range keys. */
int64_t oracle_gather_i64(const uint8_t *table, uint64_t num_rows, uint32_t row_bytes,
                          const int64_t *keys, uint64_t n, uint8_t *out) {
  return gather_impl(table, num_rows, row_bytes, keys, 0, n, out);
}

int64_t oracle_gather_u32(const uint8_t *table, uint64_t num_rows, uint32_t row_bytes,
                          const uint32_t *keys, uint64_t n, uint8_t *out) {
  return gather_impl(table, num_rows, row_bytes, keys, 1, n, out);
}
