// Fused kernel instantiation for occupancy k=6 (__launch_bounds__(256, 6)); one
// translation unit per k so the K=8 variants compile in parallel.
#include "fused_impl.cuh"
RECFLEX_INSTANTIATE_FUSED(6)
