// Decode megakernel translation unit; the implementation lives in decode_impl.cuh.
#include "decode_impl.cuh"
