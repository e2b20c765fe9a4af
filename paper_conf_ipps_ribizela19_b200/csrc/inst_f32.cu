// inst_f32.cu -- the driver and kernels instantiated for float.
#define SS_INST_T float
#include "driver.cuh"
