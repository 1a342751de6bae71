// Instantiations of the fused update kernel (svicd_impl.cuh) for the 26-neighbourhood and
// fp32 system-matrix records.
#define SVICD_NNB 26
#define SVICD_U8 false
#define SVICD_SUFFIX n26_f32
#include "svicd_impl.cuh"
