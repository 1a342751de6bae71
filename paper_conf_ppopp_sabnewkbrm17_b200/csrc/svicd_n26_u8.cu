// Instantiations of the fused update kernel (svicd_impl.cuh) for the 26-neighbourhood and
// uint8 system-matrix records.
#define SVICD_NNB 26
#define SVICD_U8 true
#define SVICD_SUFFIX n26_u8
#include "svicd_impl.cuh"
