// decode_kernel<B> instantiation for B = 4
#include "decode_impl.cuh"

MX_DECODE_INSTANTIATE(4)
