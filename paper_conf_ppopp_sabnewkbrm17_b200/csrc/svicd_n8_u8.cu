// Instantiations of the fused update kernel (svicd_impl.cuh) for the 8-neighbourhood and
// uint8 system-matrix records.
#define SVICD_NNB 8
#define SVICD_U8 true
#define SVICD_SUFFIX n8_u8
#include "svicd_impl.cuh"
