// Host-side entry points of the fused update kernel (svicd_impl.cuh): shared-memory layout size,
// scratch size, and the dispatch to the translation unit holding the (neighbourhood, A type)
// instantiations (svicd_n{8,26}_{u8,f32}.cu).
#include "svicd_impl.cuh"

namespace mbir {

#define SVICD_DECL(sfx)                                                   \
    int svicd_resident_##sfx(const IcdParams& p, int vpt, int cl);        \
    cudaError_t svicd_launch_##sfx(const IcdParams& p, int vpt, int cl, int grid, cudaStream_t st);
SVICD_DECL(n8_u8)
SVICD_DECL(n8_f32)
SVICD_DECL(n26_u8)
SVICD_DECL(n26_f32)

int svicd_smem_bytes(const IcdParams& p, int vpt, int nnb, bool quantize, int cl)
{
    return svicd_layout(p.rows, p.side, p.S2, nnb, p.A.VA, quantize, ring_depth(quantize), p.nvw, vpt, p.V, cl).total;
}

int svicd_resident_ctas(const IcdParams& p, int vpt, int nnb, bool quantize, int cl)
{
    if (nnb == 26) return quantize ? svicd_resident_n26_u8(p, vpt, cl) : svicd_resident_n26_f32(p, vpt, cl);
    return quantize ? svicd_resident_n8_u8(p, vpt, cl) : svicd_resident_n8_f32(p, vpt, cl);
}

int svicd_scratch_floats(int vpt, int nwin) { return svb_cols(vpt) * 32 * nwin; }

cudaError_t launch_svicd(const IcdParams& p, int vpt, int nnb, bool quantize, int cl, int grid, cudaStream_t st)
{
    if (nnb == 26) return quantize ? svicd_launch_n26_u8(p, vpt, cl, grid, st) : svicd_launch_n26_f32(p, vpt, cl, grid, st);
    return quantize ? svicd_launch_n8_u8(p, vpt, cl, grid, st) : svicd_launch_n8_f32(p, vpt, cl, grid, st);
}

}  // namespace mbir
