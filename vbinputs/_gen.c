/* Fast host implementation of the vbinputs counter-hash generator (same draws as the numpy
 * reference in vbinputs/__init__.py; tests pin the two together bit for bit).  Holds no
 * GEMM arithmetic.  Writes the EXACT fp64 value of each (optionally rounded) input. */
#include <stdint.h>
#include <string.h>

static inline uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

static inline double round_bf16(float f) {
  uint32_t b;
  memcpy(&b, &f, 4);
  b = (b + 0x7FFFu + ((b >> 16) & 1u)) & 0xFFFF0000u;
  float r;
  memcpy(&r, &b, 4);
  return (double)r;
}

/* dtype: 0 = f32, 1 = bf16, 2 = f16.  out: rows*cols doubles, row-major, unpadded. */
void vbgen_fill_f64(uint64_t mkey, int64_t rows, int64_t cols, int dtype, double *out) {
  const int64_t n = rows * cols;
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    const uint64_t h = splitmix64(mkey + (uint64_t)i);
    const float v = (float)(uint32_t)(h >> 40) * 0x1p-23f - 1.0f;
    if (dtype == 0) out[i] = (double)v;
    else if (dtype == 1) out[i] = round_bf16(v);
    else out[i] = (double)(_Float16)v;
  }
}
