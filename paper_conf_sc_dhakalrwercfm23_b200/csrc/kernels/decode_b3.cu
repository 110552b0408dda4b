// decode_kernel<B> instantiation for B = 3
#include "decode_impl.cuh"

MX_DECODE_INSTANTIATE(3)
