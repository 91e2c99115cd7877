// k_d1.cu -- kernels for degree d = 1 (see k_impl.cuh)
#define BZK_D 1
#include "k_impl.cuh"
