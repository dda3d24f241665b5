// Explicit instantiation of the scan kernel and launchers for element type float, orders 1..8.
#include "sam_launch.cuh"
SAM_INSTANTIATE(float)
