// k_d3.cu -- kernels for degree d = 3 (see k_impl.cuh)
#define BZK_D 3
#include "k_impl.cuh"
