/*
 * micco_inputs/synth.h — the seeded, counter-based hadron-node generator.
 *
 * This is INPUT GENERATION ONLY: it holds none of the method's arithmetic
 * (no contraction, no reduction).  It is the one piece of code that both the
 * CPU oracle (oracle/) and the CUDA library (paper_conf_ipps_wangr0e22_b200/)
 * include, so that both sides see bit-identical node tensors without either
 * one producing inputs for the other (task rule ③; SURVEY.md §8(d) "Common
 * generator").  micco_inputs/gen.py is a numpy restatement of the same
 * function; tests/test_inputs.py checks the two agree bit for bit.
 *
 * Element e (complex, flat index over [Lt][N]...[N], t slowest) of the node
 * with key `key` under stream `seed`:
 *     base = splitmix64(seed ^ (key * 0xD1B54A32D192ED03))
 *     x_p  = splitmix64(base + 2*e + p)         p = 0 (re), 1 (im)
 *     mode MICCO_SYNTH_UNIFORM: v_p = (2 * ((x_p >> 11) * 2^-53) - 1) * scale
 *                               (uniform on [-scale, scale))
 *     mode MICCO_SYNTH_INT3:    v_p = (double)((int)(x_p % 3) - 1)  in {-1,0,1}
 *                               (exact-integer mode for bit-exact parity,
 *                                SURVEY.md §8(c) "Bit-exact GPU parity")
 * Output is interleaved (re, im) doubles, the layout of the C-ABI
 * (include/micco.h, micco_add_hadron_node).
 */
#ifndef MICCO_INPUTS_SYNTH_H
#define MICCO_INPUTS_SYNTH_H

#include <stdint.h>

#define MICCO_SYNTH_UNIFORM 0
#define MICCO_SYNTH_INT3 1

static inline uint64_t micco_synth_splitmix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

static inline double micco_synth_value(uint64_t x, int mode, double scale) {
  if (mode == MICCO_SYNTH_INT3) return (double)((int)(x % 3ULL) - 1);
  double u = (double)(x >> 11) * 0x1.0p-53;
  return (2.0 * u - 1.0) * scale;
}

/* Fill complex elements [first, first + count) of node `key` into dst
 * (2*count doubles, interleaved re/im). */
static inline void micco_synth_fill(double *dst, uint64_t seed, uint64_t key, int64_t first,
                                    int64_t count, int mode, double scale) {
  uint64_t base = micco_synth_splitmix64(seed ^ (key * 0xD1B54A32D192ED03ULL));
  for (int64_t e = 0; e < count; ++e) {
    uint64_t ctr = base + 2ULL * (uint64_t)(first + e);
    dst[2 * e] = micco_synth_value(micco_synth_splitmix64(ctr), mode, scale);
    dst[2 * e + 1] = micco_synth_value(micco_synth_splitmix64(ctr + 1ULL), mode, scale);
  }
}

#endif
