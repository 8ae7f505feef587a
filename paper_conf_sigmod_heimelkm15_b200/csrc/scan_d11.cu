// Explicit instantiation of the scan kernels for d = 11 (see scan.cuh).
#include "scan.cuh"
KDE_INSTANTIATE_SCAN(11)
