// Explicit instantiation of the scan kernel and launchers for element type uint64_t, orders 1..8.
#include "sam_launch.cuh"
SAM_INSTANTIATE(uint64_t)
