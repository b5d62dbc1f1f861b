/*
 * synth.h -- C ABI of libsynth: device-side twins of the seeded input generators in
 * synth/__init__.py (counter-based splitmix64 hash).  They
 * produce the synthetic tables and sparse inputs of the paper's experiments
 * ("inputs are generated synthetically"; L260/L329 pooling factors)
 * at full size directly in HBM.  They hold NONE of the method's arithmetic and are
 * never timed.  Bit-exactness with the numpy generator is tested in
 * tests/test_synth_gpu.py.  All calls are asynchronous on `stream` (cudaStream_t as
 * void*) and return 0 on success, a cudaError_t value otherwise.
 */
#ifndef SYNTH_H_
#define SYNTH_H_
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

/* W[rows][dim]; wdtype 0 = f32, 1 = bf16; mode 0 = float, 1 = int, 2 = identity. */
int synth_gen_table(void* w, int64_t rows, int32_t dim, int32_t wdtype, int32_t mode, uint64_t seed, int64_t t,
                    void* stream);
/* out[b] = L(t, b) ~ U{pmin..pmax}, b in [0, batch). */
int synth_gen_lengths(int64_t* out, int64_t batch, uint64_t seed, int64_t t, int64_t pmin, int64_t pmax, void* stream);
/* out[j] = x_t[pos0 + j], j in [0, count); dist 0 = uniform, 1 = zipf (cdf: device float64[num_rows]);
 * row = (a*k0 + c) mod num_rows for zipf. */
int synth_gen_indices(int64_t* out, int64_t count, int64_t pos0, uint64_t seed, int64_t t, int64_t num_rows,
                      int32_t dist, const double* cdf, int64_t a, int64_t c, void* stream);

#ifdef __cplusplus
}
#endif
#endif
