// Fused kernel instantiation for occupancy k=2 (__launch_bounds__(256, 2)); one
// translation unit per k so the K=8 variants compile in parallel.
#include "fused_impl.cuh"
RECFLEX_INSTANTIATE_FUSED(2)
