// Explicit instantiation of the scan kernels for d = 6 (see scan.cuh).
#include "scan.cuh"
KDE_INSTANTIATE_SCAN(6)
