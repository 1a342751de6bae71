// Instantiations of the fused update kernel (svicd_impl.cuh) for the 8-neighbourhood and
// fp32 system-matrix records.
#define SVICD_NNB 8
#define SVICD_U8 false
#define SVICD_SUFFIX n8_f32
#include "svicd_impl.cuh"
