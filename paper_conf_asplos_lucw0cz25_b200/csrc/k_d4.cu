// k_d4.cu -- kernels for degree d = 4 (see k_impl.cuh)
#define BZK_D 4
#include "k_impl.cuh"
