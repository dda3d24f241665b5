// Explicit instantiation of the scan kernel and launchers for element type double, orders 1..8.
#include "sam_launch.cuh"
SAM_INSTANTIATE(double)
