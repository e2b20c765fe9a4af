// inst_i32.cu -- the driver and kernels instantiated for int.
#define SS_INST_T int
#include "driver.cuh"
