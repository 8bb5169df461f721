/*
 * jitc_oracle.c -- plain, slow, obviously-correct CPU oracle for the JIT
 * checkpointing data path (TEST INFRASTRUCTURE ONLY).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  The product path
 * (libjitc.so + its Python binding) never links, loads or calls it, and this
 * file shares no code, header, table or constant generator with the CUDA path.
 *
 * What the paper fixes and what is our reading:
 *   - The state to capture is "model parameters and optimizer state"
 *     (§1.1, §4.2.1).
 *   - Buffers are compared across replicas / executions by checksums
 *     (§4.1); the paper names no function.  Reading R2: JF64, a
 *     per-chunk wrap-around sum of fmix64(word ^ key(g)), fmix64 being the
 *     MurmurHash3 64-bit finalizer.
 *   - The checkpoint image is a byte concatenation in registration order,
 *     256-byte aligned, zero padded (reading R4).
 *
 * Pins (tests/test_oracle_*.py): fmix64 against the SMHasher verification
 * value of MurmurHash3_x64_128 (0x6384BA69) and the textbook inverse;
 * splitmix64 against Vigna's published seed-1234567 sequence; JF64 by
 * brute-force single-bit-flip detection, chunk-merge linearity and word-order
 * sensitivity; pack/unpack by round trip.  Every loop below is the plain
 * definition: no blocking, no vectorisation, no reordering.
 */
#include <stdint.h>
#include <stddef.h>
#include <string.h>

#define ORC_PHI 0x9E3779B97F4A7C15ULL

/* MurmurHash3 fmix64 finalizer (Appleby, SMHasher).  Reading R2 / O3. */
uint64_t orc_fmix64(uint64_t x) {
    x ^= x >> 33;
    x *= 0xff51afd7ed558ccdULL;
    x ^= x >> 33;
    x *= 0xc4ceb9fe1a85ec53ULL;
    x ^= x >> 33;
    return x;
}

/* splitmix64 output function for state z (Steele, Lea, Flood; Vigna's C
 * reference): the counter-based generator behind the synthetic state (O9). */
uint64_t orc_splitmix64(uint64_t z) {
    z += ORC_PHI;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

/* Little-endian u64 word at byte offset 8*g of buf. */
static uint64_t load_le64(const uint8_t* p) {
    uint64_t w = 0;
    for (int b = 7; b >= 0; --b) w = (w << 8) | (uint64_t)p[b];
    return w;
}

/* JF64 term for image word index g holding value w (O3):
 *   term(g) = fmix64(w ^ ((g + 1) * PHI))  (mod 2^64). */
uint64_t orc_jf64_term(uint64_t w, uint64_t g) {
    return orc_fmix64(w ^ ((g + 1) * ORC_PHI));
}

/* JF64 chunk digests of an image fragment (O3).
 * image     : the bytes of image words [g0, g0 + n_words)
 * g0        : global word index of image[0] (image byte offset / 8)
 * n_words   : number of 8-byte words in the fragment
 * chunk_words: C / 8
 * d         : digest array indexed by GLOBAL chunk id; d[g / chunk_words] += term
 * The caller zeroes d.  Word-by-word, in order. */
void orc_jf64_accumulate(const uint8_t* image, uint64_t g0, uint64_t n_words,
                         uint64_t chunk_words, uint64_t* d) {
    for (uint64_t i = 0; i < n_words; ++i) {
        uint64_t g = g0 + i;
        uint64_t w = load_le64(image + 8 * i);
        d[g / chunk_words] += orc_jf64_term(w, g);
    }
}

/* root = fmix64(layout_hash ^ n_c); then root = fmix64(root ^ d[c]) in chunk
 * order (O3). */
uint64_t orc_root(uint64_t layout_hash, const uint64_t* d, uint64_t n_c) {
    uint64_t r = orc_fmix64(layout_hash ^ n_c);
    for (uint64_t c = 0; c < n_c; ++c) r = orc_fmix64(r ^ d[c]);
    return r;
}

/* fold_fmix64(xs): h = 0; for x in xs: h = fmix64(h ^ x)   (O1). */
uint64_t orc_fold_fmix64(const uint64_t* xs, uint64_t n) {
    uint64_t h = 0;
    for (uint64_t i = 0; i < n; ++i) h = orc_fmix64(h ^ xs[i]);
    return h;
}

/* O2 pack: image[off[i] : off[i] + nbytes[i]] = tensor i; everything else 0. */
void orc_pack(const uint8_t* const* src, const uint64_t* nbytes, const uint64_t* off,
              uint64_t n, uint8_t* image, uint64_t L) {
    memset(image, 0, L);
    for (uint64_t i = 0; i < n; ++i) memcpy(image + off[i], src[i], nbytes[i]);
}

/* O8 unpack: tensor i = image[off[i] : off[i] + nbytes[i]]. */
void orc_unpack(const uint8_t* image, uint8_t* const* dst, const uint64_t* nbytes,
                const uint64_t* off, uint64_t n) {
    for (uint64_t i = 0; i < n; ++i) memcpy(dst[i], image + off[i], nbytes[i]);
}

/* ---------------------------------------------------------------------------
 * O9 synthetic-state generator (integer only; one draw per element j).
 *   x    = splitmix64(seed ^ fmix64((group << 48) ^ (tensor_id << 32)) ^ j)
 *   sign = x >> 63            (0 when force_pos)
 *   exp  = lo + ((x >> 32) & 0xFFFF) % (hi - lo + 1)
 *   mant = x & 0x7FFFFF
 * fp32 bits = sign<<31 | exp<<23 | mant.  bf16 = RNE(fp32) by the integer rule
 *   (u + 0x7FFF + ((u >> 16) & 1)) >> 16.
 * Elements [j0, j0 + count) are produced, so any slice of a tensor can be
 * generated on its own (used for sampled full-size parity).
 * ------------------------------------------------------------------------- */
static uint32_t gen_fp32_bits(uint64_t seed, uint32_t group, uint32_t tensor_id, uint64_t j,
                              uint32_t lo, uint32_t hi, int force_pos) {
    uint64_t key = orc_fmix64(((uint64_t)group << 48) ^ ((uint64_t)tensor_id << 32));
    uint64_t x = orc_splitmix64(seed ^ key ^ j);
    uint32_t sign = force_pos ? 0u : (uint32_t)(x >> 63);
    uint32_t e = lo + (uint32_t)(((x >> 32) & 0xFFFFULL) % (uint64_t)(hi - lo + 1));
    uint32_t mant = (uint32_t)(x & 0x7FFFFFULL);
    return (sign << 31) | (e << 23) | mant;
}

static uint16_t rne_bf16(uint32_t u) {
    return (uint16_t)((u + 0x7FFFu + ((u >> 16) & 1u)) >> 16);
}

void orc_gen_fp32(uint32_t* out, uint64_t j0, uint64_t count, uint64_t seed, uint32_t group,
                  uint32_t tensor_id, uint32_t lo, uint32_t hi, int force_pos) {
    for (uint64_t i = 0; i < count; ++i)
        out[i] = gen_fp32_bits(seed, group, tensor_id, j0 + i, lo, hi, force_pos);
}

void orc_gen_bf16(uint16_t* out, uint64_t j0, uint64_t count, uint64_t seed, uint32_t group,
                  uint32_t tensor_id, uint32_t lo, uint32_t hi, int force_pos) {
    for (uint64_t i = 0; i < count; ++i)
        out[i] = rne_bf16(gen_fp32_bits(seed, group, tensor_id, j0 + i, lo, hi, force_pos));
}

/* O10 synthetic optimizer update U_v on an fp32 tensor (master / m / v):
 * word32[j] ^= fmix64(((tensor_id << 40) ^ j) ^ (v * PHI)) & 0xFFFF
 * (low 16 mantissa bits only, so magnitudes stay realistic). */
void orc_update_fp32(uint32_t* x, uint64_t j0, uint64_t count, uint32_t tensor_id, uint64_t v) {
    for (uint64_t i = 0; i < count; ++i) {
        uint64_t j = j0 + i;
        uint64_t h = orc_fmix64((((uint64_t)tensor_id << 40) ^ j) ^ (v * ORC_PHI));
        x[i] ^= (uint32_t)(h & 0xFFFFULL);
    }
}

/* bf16 params re-derived from their fp32 master after an update: p = RNE(m). */
void orc_rne_bf16(const uint32_t* master, uint16_t* out, uint64_t count) {
    for (uint64_t i = 0; i < count; ++i) out[i] = rne_bf16(master[i]);
}
