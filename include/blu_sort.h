/*
 * blu_sort.h — libblugby's sort offload (the paper's other GPU operator, §3, P:76-88;
 * SURVEY.md §8(f) NEXT-4). Same library and conventions as blu_gby.h: status codes, stream-ordered
 * device work, nothing throws across the ABI, blu_gby_last_error() for detail.
 *
 * The paper's design: rows live unmoved in the Sort Data Store; the sort works on a "partial key
 * buffer" whose entries are a 4-byte "partial binary sortable representation" of the sort key plus
 * a 4-byte payload pointing back at the row. The GPU sorts the buffer on the 4-byte key with
 * a radix sort ([18]) and identifies "duplicate ranges" (runs of equal partial keys);
 * each duplicate range becomes a new job sorted on the next 4 bytes, until no job is left.
 *
 * B200 design: one stable LSD radix sort (8-bit digits, warp-match ranking, one
 * persistent CTA range per SM pair) serves both the first level (u32 partial keys) and every later
 * level, where ALL duplicate ranges of a level form one batched job: the key is (range id << 32 |
 * next partial key), so one sort orders every range internally at once instead of one job per range.
 *
 * Limits: n < 2^32 rows (4-byte payloads); W (key bytes per row) a multiple of 4, 4..1024.
 */
#ifndef BLU_SORT_H
#define BLU_SORT_H

#include <stdint.h>

#include "blu_gby.h"

#ifdef __cplusplus
extern "C" {
#endif

/* keys_out[i] = bytes [4*word, 4*word + 4) of row i read most significant first (a binary-
 * sortable u32). rows: DEVICE, n x W bytes row-major (the SDS); keys_out: DEVICE, n u32. */
blu_status_t blu_sort_partial_keys(const uint8_t* rows, uint64_t n, uint32_t W, uint32_t word, uint32_t* keys_out,
                                   void* stream);

/* stable sort of the partial key buffer (keys_in[i], payload_in[i]) by key, into keys_out /
 * payload_out (all DEVICE, n u32 each; outputs must not alias inputs). Equal keys keep their input
 * order. Errors: BLU_E_INVALID (NULL pointers with n > 0, aliasing, n >= 2^32), BLU_E_OOM, BLU_E_CUDA. */
blu_status_t blu_sort_pairs(const uint32_t* keys_in, const uint32_t* payload_in, uint64_t n, uint32_t* keys_out,
                            uint32_t* payload_out, void* stream);

/* duplicate ranges of a sorted DEVICE buffer: maximal runs of >= 2 equal keys, in order.
 * starts / lens: DEVICE, room for `cap` entries each (n / 2 always suffices); *n_ranges (HOST) gets
 * the number found (only min(cap, found) are written). Synchronises `stream`. */
blu_status_t blu_sort_dup_ranges(const uint32_t* sorted_keys, uint64_t n, uint64_t* starts, uint64_t* lens, uint64_t cap,
                                 uint64_t* n_ranges, void* stream);

typedef struct {
    uint32_t levels;        /* partial-key levels sorted (1 = the first 4 bytes decided everything) */
    uint64_t ranges[256];   /* ranges[l] = duplicate ranges left after level l                        */
    uint64_t active[256];   /* active[l] = rows inside those ranges (the next level's job size)      */
    float ms[256];          /* device time of level l (sort + range detection), CUDA events          */
    /* the dominant kernel, the radix downsweep (read + scatter of keys and payloads), timed per
       launch with CUDA events on `stream`: summed time, launches, algorithmic bytes moved          */
    float downsweep_ms;
    uint32_t downsweep_launches;
    uint64_t downsweep_bytes;
} blu_sort_stats_t;

/* P:76-86, the whole job queue: perm_out[p] (DEVICE, n u32) = the row at position p of the stable
 * lexicographic order of rows (DEVICE, n x W bytes): rows with identical keys stay in row order.
 * Level l sorts the rows still inside duplicate ranges by (range, partial key l). stats (HOST) may
 * be NULL. Synchronises `stream` once per level (the host reads the size of the next job). */
blu_status_t blu_sort_rows(const uint8_t* rows, uint64_t n, uint32_t W, uint32_t* perm_out, void* stream,
                           blu_sort_stats_t* stats);

#ifdef __cplusplus
}
#endif

#endif /* BLU_SORT_H */
