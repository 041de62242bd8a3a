/*
 * ORACLE — TEST INFRASTRUCTURE ONLY. Not part of libblugby; the product path never loads it.
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg may
 * load or call this library (it is linked into oracle/liboracle.so).
 *
 * The group-count estimate the paper feeds to the GPU runtime ("We use CPU threads
 * to load data and then use a simple hash function and KMV[2] algorithm to estimate the number of
 * groups"; "the estimated number of groups"), written out plainly:
 *
 *   1. the grouping value of row i is its key tuple, concatenated ("CCAT") as the mixed-radix
 *      number  sum_j code_j[i] * prod_{l<j} dict_l  (dictionary keys), or the code itself (a single
 *      sparse key) — reading A3;
 *   2. the "simple hash function" (reading K-1): h = fmix64(value XOR salt), the Murmur3
 *      64-bit finalizer (the paper names Murmur for hashing), salt = "kmv_salt" as ASCII;
 *      the all-ones hash is dropped (reading K-2: it is the empty mark, never a sample);
 *   3. KMV ("K-minimum values", the paper's [2]): keep the k smallest DISTINCT hash values; with
 *      U_(k) the k-th smallest, est = (k - 1) * 2^64 / U_(k); if fewer than k distinct hashes exist
 *      the estimate is their exact count.
 * A std::set holds the distinct hashes; nothing is blocked, sampled or merged. Shares no code with
 * paper_conf_sigmod_merajispcksygnk16_b200/csrc. Pins: tests/test_oracle_pins.py (exact count
 * below k vs a Python set, the estimator's relative-error bound over many key sets, invariance
 * under row order and duplication, fmix64 bijectivity).
 */
#include <stdint.h>

#include <iterator>
#include <set>

extern "C" {

static uint64_t oracle_fmix64(uint64_t h) {  // MurmurHash3 fmix64 (Appleby), step by step
    h ^= h >> 33;
    h *= 0xff51afd7ed558ccdull;
    h ^= h >> 33;
    h *= 0xc4ceb9fe1a85ec53ull;
    h ^= h >> 33;
    return h;
}

uint64_t oracle_fmix64_export(uint64_t h) { return oracle_fmix64(h); }

/* key_cols: n_keys host arrays; key_is64[j]: 1 = int64 codes, 0 = int32; dict[j] = dictionary size
 * (0 = sparse, only with n_keys == 1). Returns the estimate; *exact = 1 when fewer than k distinct
 * hashes were seen (the estimate is then the exact count of distinct hashes). */
double oracle_kmv(const void* const* key_cols, const int32_t* key_is64, const uint64_t* dict, int32_t n_keys,
                  uint64_t n, uint32_t k, int32_t* exact) {
    const uint64_t salt = 0x6b6d765f73616c74ull;  // "kmv_salt"
    std::set<uint64_t> distinct;
    for (uint64_t i = 0; i < n; ++i) {
        uint64_t value = 0, radix = 1;
        for (int32_t j = 0; j < n_keys; ++j) {
            const int64_t code = key_is64[j] ? ((const int64_t*)key_cols[j])[i] : (int64_t)((const int32_t*)key_cols[j])[i];
            value += (uint64_t)code * radix;
            radix *= dict[j] ? dict[j] : 1;
        }
        const uint64_t h = oracle_fmix64(value ^ salt);
        if (h != ~0ull) distinct.insert(h);
    }
    if (distinct.size() < k) {
        if (exact) *exact = 1;
        return (double)distinct.size();
    }
    if (exact) *exact = 0;
    const uint64_t kth = *std::next(distinct.begin(), (long)k - 1);
    return (double)(k - 1) * 18446744073709551616.0 / (double)kth;
}

}  // extern "C"
