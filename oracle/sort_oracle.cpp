/*
 * ORACLE — TEST INFRASTRUCTURE ONLY. Not part of libblugby; the product path never loads it.
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg may
 * load or call this library (it is linked into oracle/liboracle.so).
 *
 * The paper's sort offload (§3), as plain definitions:
 *   - partial key: "a partial binary sortable representation of the column": the 4 bytes
 *     [4w, 4w + 4) of a row's binary-sortable key, read most significant byte first, so that
 *     unsigned comparison of partial keys is lexicographic comparison of those bytes;
 *   - the GPU sort of the partial key buffer ("sorted the partial key buffer based upon the
 *     4-byte partial key"): (key, payload) pairs in non-decreasing key order; equal keys keep their
 *     buffer order (the radix sort the paper cites, [18], is stable) — std::stable_sort;
 *   - duplicate ranges ("If there exists more than one tuple for which the first 4 bytes are
 *     identical ... We call such a group of tuples a duplicate range"): maximal runs of >= 2 equal
 *     keys in the sorted buffer;
 *   - the completed sort ("The sort is complete when there are no more jobs on the
 *     queue"): the permutation that orders rows by their whole W-byte key, lexicographically on
 *     unsigned bytes, rows with identical keys in row order — std::stable_sort with memcmp. (The
 *     job queue reaches exactly this: every step is a stable sort of a duplicate range by its next
 *     4 bytes, starting from row order.)
 * No radix digits, no passes, no segments: library sorts and memcmp only. Shares no code with
 * paper_conf_sigmod_merajispcksygnk16_b200/csrc. Pins: tests/test_oracle_pins.py.
 */
#include <stdint.h>
#include <string.h>

#include <algorithm>
#include <vector>

extern "C" {

/* keys_out[i] = bytes rows[i*W + 4*word .. + 4] as a big-endian u32 (bytes past W read as 0). */
void oracle_partial_keys(const uint8_t* rows, uint64_t n, uint32_t W, uint32_t word, uint32_t* keys_out) {
  for (uint64_t i = 0; i < n; ++i) {
    uint32_t k = 0;
    for (uint32_t b = 0; b < 4; ++b) {
      const uint32_t pos = 4 * word + b;
      const uint32_t byte = pos < W ? rows[i * W + pos] : 0u;
      k = (k << 8) | byte;
    }
    keys_out[i] = k;
  }
}

/* Stable sort of the (key, payload) buffer by key. */
void oracle_sort_pairs(const uint32_t* keys, const uint32_t* payload, uint64_t n, uint32_t* keys_out,
                       uint32_t* payload_out) {
  std::vector<uint64_t> idx(n);
  for (uint64_t i = 0; i < n; ++i) idx[i] = i;
  std::stable_sort(idx.begin(), idx.end(), [&](uint64_t a, uint64_t b) { return keys[a] < keys[b]; });
  for (uint64_t i = 0; i < n; ++i) {
    keys_out[i] = keys[idx[i]];
    payload_out[i] = payload[idx[i]];
  }
}

/* Maximal runs of >= 2 equal keys in a sorted buffer; returns how many (starts/lens may be NULL to
 * count only; otherwise they hold room for n / 2 entries). */
uint64_t oracle_dup_ranges(const uint32_t* sorted_keys, uint64_t n, uint64_t* starts, uint64_t* lens) {
  uint64_t r = 0, i = 0;
  while (i < n) {
    uint64_t j = i + 1;
    while (j < n && sorted_keys[j] == sorted_keys[i]) ++j;
    if (j - i >= 2) {
      if (starts) starts[r] = i;
      if (lens) lens[r] = j - i;
      ++r;
    }
    i = j;
  }
  return r;
}

/* The completed sort: perm_out[p] = the row at position p of the stable lexicographic order. */
void oracle_sort_rows(const uint8_t* rows, uint64_t n, uint32_t W, uint32_t* perm_out) {
  std::vector<uint32_t> idx(n);
  for (uint64_t i = 0; i < n; ++i) idx[i] = (uint32_t)i;
  std::stable_sort(idx.begin(), idx.end(),
                   [&](uint32_t a, uint32_t b) { return memcmp(rows + (uint64_t)a * W, rows + (uint64_t)b * W, W) < 0; });
  for (uint64_t i = 0; i < n; ++i) perm_out[i] = idx[i];
}

}  // extern "C"
