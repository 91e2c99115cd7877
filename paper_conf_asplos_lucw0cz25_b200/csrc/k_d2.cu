// k_d2.cu -- kernels for degree d = 2 (see k_impl.cuh)
#define BZK_D 2
#include "k_impl.cuh"
